"""An iterative AES-128 encryption core as a LUT netlist (a real circuit of the kind in the
paper's Table I: "AES"), built from FIPS-197.  Input construction only: the
S-box, MixColumns and key schedule are TABULATED into truth tables the way a netlist author
writes LUTs (Fig. 3); nothing here simulates the circuit.

Ports (bit j of byte i is bit 8*i + j; byte i is state row i % 4, column i // 4):
  PIs   0..127 plaintext, 128..255 key, 256 start
  regs  0..127 state S, 128..255 round key K, 256..259 round counter
  POs   0..127 the state register S
Behaviour: a cycle with start = 1 loads S = plaintext xor key, K = key, counter = 1; each
following cycle performs round `counter` (SubBytes, ShiftRows, MixColumns except in round
10, AddRoundKey with the next round key, which is also latched into K).  After the load
cycle and 10 round cycles the state register holds the ciphertext, so the POs of the 12th
cycle (outputs are sampled before the latch, R4) show it.

The S-box bits are 8-input LUTs (the paper's L = 8 regime); MixColumns output bits are
XOR trees of <= 4-input LUTs.
"""
from __future__ import annotations

from .netlists import Builder, Netlist, tt_of


def _xtime(a: int) -> int:
    a <<= 1
    return (a ^ 0x11B) if a & 0x100 else a


def _gmul(a: int, b: int) -> int:
    r = 0
    while b:
        if b & 1:
            r ^= a
        a = _xtime(a)
        b >>= 1
    return r


def sbox_table() -> list[int]:
    """FIPS-197 §5.1.1: multiplicative inverse in GF(2^8) (0 -> 0) then the affine map."""
    inv = [0] * 256
    for x in range(1, 256):
        for y in range(1, 256):
            if _gmul(x, y) == 1:
                inv[x] = y
                break
    out = []
    for x in range(256):
        b = inv[x]
        s = b
        for i in range(1, 5):
            s ^= ((b << i) | (b >> (8 - i))) & 0xFF
        out.append(s ^ 0x63)
    return out


RCON = [0x00, 0x01, 0x02, 0x04, 0x08, 0x10, 0x20, 0x40, 0x80, 0x1B, 0x36, 0, 0, 0, 0, 0]


def _xor_tree(b: Builder, bits: list):
    """XOR of the given nets with <= 4-input XOR LUTs (a balanced tree)."""
    bits = list(bits)
    if len(bits) == 1:
        return bits[0]
    while len(bits) > 1:
        nxt = []
        for i in range(0, len(bits), 4):
            grp = bits[i:i + 4]
            if len(grp) == 1:
                nxt.append(grp[0])
            else:
                nxt.append(b.gate(tt_of(len(grp), lambda *x: sum(x) & 1), *grp))
        bits = nxt
    return bits[0]


def _mix_masks() -> list[list[tuple[int, int]]]:
    """For output bit (row r, bit j) of a MixColumns column: the (row, bit) inputs XORed."""
    coef = [[2, 3, 1, 1], [1, 2, 3, 1], [1, 1, 2, 3], [3, 1, 1, 2]]
    masks = []
    for r in range(4):
        for j in range(8):
            terms = []
            for c in range(4):
                for i in range(8):                 # contribution of input bit (c, i)
                    if (_gmul(1 << i, coef[r][c]) >> j) & 1:
                        terms.append((c, i))
            masks.append(terms)
    return masks


def aes128_core() -> Netlist:
    b = Builder()
    PT = [b.pi() for _ in range(128)]
    KEY = [b.pi() for _ in range(128)]
    START = b.pi()
    S = [b.reg(0) for _ in range(128)]
    K = [b.reg(0) for _ in range(128)]
    CTR = [b.reg(0) for _ in range(4)]
    SB = sbox_table()

    def sbox_bits(byte_bits):
        return [b.gate(sum(((SB[m] >> j) & 1) << m for m in range(256)), *byte_bits) for j in range(8)]

    # SubBytes + ShiftRows
    sb = [sbox_bits(S[8 * i:8 * i + 8]) for i in range(16)]
    sr = [None] * 16
    for r in range(4):
        for c in range(4):
            sr[r + 4 * c] = sb[r + 4 * ((c + r) % 4)]
    # MixColumns
    masks = _mix_masks()
    mc = [None] * 16
    for c in range(4):
        col = [sr[r + 4 * c] for r in range(4)]
        for r in range(4):
            mc[r + 4 * c] = [_xor_tree(b, [col[cc][i] for cc, i in masks[8 * r + j]]) for j in range(8)]
    # round constant and last-round flag from the counter (4-input LUTs)
    rc = [b.gate(tt_of(4, lambda *x, j=j: (RCON[sum(v << i for i, v in enumerate(x))] >> j) & 1), *CTR)
          for j in range(8)]
    last = b.gate(tt_of(4, lambda *x: int(sum(v << i for i, v in enumerate(x)) == 10)), *CTR)
    # key schedule: temp = SubWord(RotWord(w3)) ^ Rcon; w0' = w0 ^ temp; wi' = wi ^ w(i-1)'
    w3 = [K[96 + 8 * i:96 + 8 * i + 8] for i in range(4)]
    rot = [w3[1], w3[2], w3[3], w3[0]]
    sub = [sbox_bits(x) for x in rot]
    nk = [None] * 128
    for i in range(4):
        for j in range(8):
            t = 8 * i + j
            if i == 0:
                nk[t] = b.gate(tt_of(3, lambda x, y, z: x ^ y ^ z), K[t], sub[i][j], rc[j])
            else:
                nk[t] = b.gate(tt_of(2, lambda x, y: x ^ y), K[t], sub[i][j])
    for w in range(1, 4):
        for t in range(32):
            nk[32 * w + t] = b.gate(tt_of(2, lambda x, y: x ^ y), K[32 * w + t], nk[32 * (w - 1) + t])
    # next state and key
    for i in range(16):
        for j in range(8):
            t = 8 * i + j
            ark = b.gate(tt_of(4, lambda l, m, s, k: (s if l else m) ^ k), last, mc[i][j], sr[i][j], nk[t])
            b.set_d(S[t], b.gate(tt_of(4, lambda st, p, k, a: (p ^ k) if st else a), START, PT[t], KEY[t], ark))
    for t in range(128):
        b.set_d(K[t], b.gate(tt_of(3, lambda st, k, n: k if st else n), START, KEY[t], nk[t]))
    for j in range(4):
        nxt = b.gate(tt_of(5, lambda st, *c, j=j: (int(j == 0) if st else
                                                   ((sum(v << i for i, v in enumerate(c)) + 1) >> j) & 1)),
                     START, *CTR)
        b.set_d(CTR[j], nxt)
    for t in range(128):
        b.out(S[t])
    return b.build("aes128", meta={"cycles_to_ciphertext": 12})


def aes_stimulus(keys, pts, cycles: int = 12):
    """Host stimulus [cycles][257][lanes / 64] (uint64): cycle 0 loads each lane's plaintext and
    key with start = 1; later cycles drive start = 0 (and zeros on the data inputs).
    keys, pts: uint8 arrays [lanes][16], lanes a multiple of 64."""
    import numpy as np
    keys = np.asarray(keys, dtype=np.uint8)
    pts = np.asarray(pts, dtype=np.uint8)
    lanes = keys.shape[0]
    assert lanes % 64 == 0 and pts.shape == keys.shape == (lanes, 16)
    bits = np.zeros((257, lanes), dtype=np.uint8)
    bits[0:128] = np.unpackbits(pts, axis=1, bitorder="little").T      # bit 8*i + j
    bits[128:256] = np.unpackbits(keys, axis=1, bitorder="little").T
    bits[256] = 1
    stim = np.zeros((cycles, 257, lanes // 64), dtype=np.uint64)
    stim[0] = np.packbits(bits, axis=1, bitorder="little").view(np.uint64)
    return stim


def ciphertexts(po_bits):
    """PO bits [lanes][128] (outputs of cycle 11) -> uint8 [lanes][16]."""
    import numpy as np
    return np.packbits(np.asarray(po_bits, dtype=np.uint8), axis=1, bitorder="little")
