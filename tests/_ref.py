"""Test-side helpers: a third, pure-Python implementation of the stimulus hash and
MISR (readings R2, R5), pinned by tests/golden/*.txt, plus golden readers."""
import os

import numpy as np

M64 = (1 << 64) - 1
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def mix64(z):
    z = (z + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def stim_word(seed, p, c, w):
    return mix64(mix64(mix64(seed ^ p) ^ c) ^ w)


def misr_step(sig, v):
    fb = 0x42F0E1EBA9EA3693 if (sig >> 63) & 1 else 0
    return ((sig << 1) & M64) ^ fb ^ v


def pi_bits(seed, n_pi, cycle, lanes):
    """PI values [n_pi][len(lanes)] (0/1) of the counter-based stimulus, reading R2."""
    lanes = np.asarray(lanes, dtype=np.uint64)
    words = sorted(set((lanes >> np.uint64(6)).tolist()))
    out = np.zeros((n_pi, lanes.shape[0]), dtype=np.uint8)
    for p in range(n_pi):
        wv = {w: stim_word(seed, p, cycle, w) for w in words}
        out[p] = [(wv[int(s) >> 6] >> (int(s) & 63)) & 1 for s in lanes.tolist()]
    return out


def golden_lines(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]


def bits_to_int(bits):
    """bits [..., n] (LSB first) -> python ints via object arithmetic."""
    bits = np.asarray(bits, dtype=np.uint64)
    acc = np.zeros(bits.shape[:-1], dtype=object)
    for i in range(bits.shape[-1]):
        acc = acc + (bits[..., i].astype(object) << i)
    return acc


def mix64_np(z):
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def stim_words_np(seed, p, c, words):
    """Vectorised H(seed, p, c, w) over an array of global word indices (reading R2)."""
    a = mix64_np(np.uint64(seed) ^ np.uint64(p))
    b = mix64_np(a ^ np.uint64(c))
    return mix64_np(b ^ np.asarray(words, dtype=np.uint64))


def pi_lanes_np(seed, n_pi, cycle, n_lanes, lane_offset=0):
    """PI bits [n_pi][n_lanes] for consecutive lanes starting at lane_offset (multiple of 64)."""
    words = np.arange(lane_offset // 64, lane_offset // 64 + n_lanes // 64, dtype=np.uint64)
    out = np.empty((n_pi, n_lanes), dtype=np.uint8)
    for p in range(n_pi):
        w = stim_words_np(seed, p, cycle, words)
        out[p] = np.unpackbits(w.view(np.uint8), bitorder="little")
    return out
