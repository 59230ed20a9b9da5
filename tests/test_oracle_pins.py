"""Pins of the CPU oracle against values it does not produce itself (CPU only).

Every test cites what fixes the expected value: a published number (tests/golden),
a closed form of the mathematics, or brute force with a different algorithm.
"""
import itertools

import numpy as np
import pytest

import oracle
from oracle import mobius
import workloads
from workloads import netlists as W
from tests import _ref


# ---------------------------------------------------------------- hashing / MISR

def test_mix64_matches_published_splitmix64():
    gamma = 0x9E3779B97F4A7C15
    for i, hexv in _ref.golden_lines("splitmix64_seed0.txt"):
        z = (int(i) * gamma) & _ref.M64
        assert oracle.mix64(z) == int(hexv, 16)
        assert _ref.mix64(z) == int(hexv, 16)


def test_misr_is_crc64_ecma182():
    (_, msg), (_, check) = _ref.golden_lines("crc64_ecma182.txt")
    sig = 0
    for byte in msg.encode():
        for b in range(7, -1, -1):
            sig = oracle.misr_step(sig, (byte >> b) & 1)
    for _ in range(64):
        sig = oracle.misr_step(sig, 0)
    assert sig == int(check, 16)


def test_stim_hash_three_ways():
    rng = np.random.default_rng(0)
    for _ in range(200):
        s, p, c, w = (int(x) for x in rng.integers(0, 2**63, size=4))
        assert oracle.stim_word(s, p, c, w) == _ref.stim_word(s, p, c, w)
        v = int(rng.integers(0, 2**63))
        assert oracle.misr_step(s, v) == _ref.misr_step(s, v)


# ---------------------------------------------------------------- Möbius / polynomial

def test_mobius_textbook_closed_forms():
    for name, k, tth, *w in _ref.golden_lines("mobius_closed_forms.txt"):
        k, tt = int(k), int(tth, 16)
        assert oracle.mobius_def(tt, k) == [int(x) for x in w], name
        assert mobius.coeffs_alg1(tt, k) == [int(x) for x in w], name


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
def test_mobius_parity_and_or_closed_forms(k):
    # parity_k = (1 - prod(1 - 2x_i))/2  ->  w_S = (-1)^{|S|+1} 2^{|S|-1}  (S != {})
    # AND_k = prod x_i -> w = delta_{S=[k]};  OR_k = 1 - prod(1-x_i) -> (-1)^{|S|+1}
    n = 1 << k
    par = sum(1 << m for m in range(n) if bin(m).count("1") % 2)
    andk = 1 << (n - 1)
    ork = ((1 << n) - 1) ^ 1
    exp_par = [0] + [(-1) ** (bin(S).count("1") + 1) * 2 ** (bin(S).count("1") - 1)
                     for S in range(1, n)]
    exp_and = [0] * (n - 1) + [1]
    exp_or = [0] + [(-1) ** (bin(S).count("1") + 1) for S in range(1, n)]
    assert oracle.mobius_def(par, k) == exp_par
    assert oracle.mobius_def(andk, k) == exp_and
    assert oracle.mobius_def(ork, k) == exp_or


def _all_tts_coeffs(k):
    n = 1 << k
    return np.array([oracle.mobius_def(tt, k) for tt in range(1 << n)], dtype=np.int64)


def test_polynomial_reproduces_every_4input_truth_table():
    """Eq. 1 holds for all 2^16 functions of 4 inputs: f(x) = sum_{S ⊆ x} w_S."""
    k, n = 4, 16
    w = _all_tts_coeffs(k)                               # [65536, 16]
    tts = np.arange(1 << n, dtype=np.int64)
    for x in range(n):
        subset = np.array([(S & ~x) == 0 for S in range(n)])   # h_S(x) = prod_{s in S} x_s
        val = w[:, subset].sum(axis=1)
        assert np.array_equal(val, (tts >> x) & 1)
    # |w_S| <= 2^{|S|-1}  (attained by parity)
    bound = np.array([0 if S == 0 else 2 ** (bin(S).count("1") - 1) for S in range(n)])
    bound[0] = 1
    assert (np.abs(w) <= bound).all()
    # w_S mod 2 is the Zhegalkin (ANF, GF(2)) coefficient: GF(2) butterfly
    anf = ((tts[:, None] >> np.arange(n)[None, :]) & 1).copy()
    for i in range(k):
        for m in range(n):
            if m >> i & 1:
                anf[:, m] ^= anf[:, m ^ (1 << i)]
    assert np.array_equal(w & 1, anf)


def test_perceptron_network_equals_truth_table_k3_all_and_k4_sample():
    """Eq. 2-3: the Theta-neuron network of Fig. 2 computes f exactly."""
    for tt in range(256):
        w = oracle.mobius_def(tt, 3)
        for x in range(8):
            assert oracle.poly_eval(w, 3, x) == (tt >> x) & 1
    rng = np.random.default_rng(1)
    for tt in rng.integers(0, 1 << 16, size=300):
        w = oracle.mobius_def(int(tt), 4)
        for x in range(16):
            assert oracle.poly_eval(w, 4, x) == (int(tt) >> x) & 1


def test_algorithm1_literal_equals_definition():
    for k in (0, 1, 2, 3):
        for tt in range(1 << (1 << k)):
            assert mobius.coeffs_alg1(tt, k) == oracle.mobius_def(tt, k)
    rng = np.random.default_rng(2)
    for tt in rng.integers(0, 1 << 16, size=500):
        assert mobius.coeffs_alg1(int(tt), 4) == oracle.mobius_def(int(tt), 4)
    for tt in rng.integers(0, 2**62, size=20):
        assert mobius.coeffs_alg1(int(tt), 6) == oracle.mobius_def(int(tt), 6)


@pytest.mark.parametrize("k", [7, 8])
def test_wide_gates_algorithm1_definition_and_eq1(k):
    """k = 7, 8 (the paper's L = 7 regime, Table I): Algorithm 1 read literally equals the
    inclusion-exclusion definition, Eq. 1 reproduces the table at all 2^k points, the
    coefficients obey |w_S| <= 2^{|S|-1} (so int16 holds them) and the Theta network of
    Eq. 2-3 outputs exactly f."""
    rng = np.random.default_rng(k)
    n = 1 << k
    for trial in range(4):
        words = rng.integers(0, np.iinfo(np.uint64).max, size=n // 64, dtype=np.uint64, endpoint=True)
        tt = sum(int(w) << (64 * i) for i, w in enumerate(words))
        w = oracle.mobius_def_wide(words, k)
        assert mobius.coeffs_alg1(tt, k) == w
        for x in range(n):
            assert sum(w[S] for S in range(n) if (S & ~x) == 0) == (tt >> x) & 1
        assert all(abs(w[S]) <= max(1, 2 ** (bin(S).count("1") - 1)) for S in range(n))
        for x in rng.integers(0, n, size=40):
            assert oracle.poly_eval(w, k, int(x)) == (tt >> int(x)) & 1
    # parity_8 attains the bound: w_S = (-1)^{|S|+1} 2^{|S|-1}
    par = sum(((bin(m).count("1") & 1) << m) for m in range(n))
    wp = oracle.mobius_def_wide([(par >> (64 * i)) & (2**64 - 1) for i in range(n // 64)], k)
    assert all(wp[S] == (0 if S == 0 else (-1) ** (bin(S).count("1") + 1) * 2 ** (bin(S).count("1") - 1))
               for S in range(n))


def test_algorithm1_operation_count():
    """"our algorithm requires at most 2^L L operations".  The subtractions Algorithm 1
    performs are COUNTED while it runs (oracle/mobius.py instruments its merge); the count is
    L 2^(L-1) — each of the L recursion depths merges 2^(L-1) coefficient pairs in total — and
    independent of the table."""
    rng = np.random.default_rng(3)
    for L in range(0, 11):
        for tt in (0, (1 << (1 << L)) - 1, int(rng.integers(0, 2**63)) & ((1 << (1 << L)) - 1)):
            n = mobius.alg1_op_count(L, tt)
            assert n == (L * 2 ** (L - 1) if L else 0), (L, n)
            assert n <= (2 ** L) * L


def test_threshold_function_claims():
    """AND, OR, NOT, MAJ are threshold functions, XOR is not (brute force)."""
    def is_threshold(tt, k, rng_w=range(-3, 4)):
        for ws in itertools.product(rng_w, repeat=k):
            for b in range(-4, 5):
                if all(((sum(ws[i] * ((x >> i) & 1) for i in range(k)) - b) > 0) ==
                       bool((tt >> x) & 1) for x in range(1 << k)):
                    return True
        return False
    assert is_threshold(W.AND2, 2) and is_threshold(W.OR2, 2)
    assert is_threshold(W.NOT, 1) and is_threshold(W.MAJ3, 3)
    assert not is_threshold(W.XOR2, 2)


# ---------------------------------------------------------------- combinational closed forms

def _exhaustive_adder_stim(nbits):
    lanes = 1 << (2 * nbits)
    words = lanes // 64
    s = np.arange(lanes, dtype=np.uint64)
    stim = np.zeros((1, 2 * nbits, words), dtype=np.uint64)
    for p in range(2 * nbits):
        bits = (s >> np.uint64(p)) & np.uint64(1)
        stim[0, p] = (bits.reshape(words, 64) << np.arange(64, dtype=np.uint64)).sum(
            axis=1, dtype=np.uint64)
    return stim, s


def test_adder_exhaustive_equals_a_plus_b():
    nl = workloads.adder(8)
    stim, s = _exhaustive_adder_stim(8)
    r = oracle.simulate(nl, s, 1, host_stim=stim, want=("last",))
    got = (r["last"].astype(np.int64) << np.arange(9)).sum(axis=1)
    a, b = s & 0xFF, s >> np.uint64(8)
    assert np.array_equal(got, (a + b).astype(np.int64))


def test_adder_hash_stimulus_equals_a_plus_b():
    nl = workloads.adder(8)
    lanes = np.arange(1024, dtype=np.uint64)
    r = oracle.simulate(nl, lanes, 1, seed=1, want=("last",))
    pi = _ref.pi_bits(1, 16, 0, lanes).astype(np.int64)
    a = (pi[:8] << np.arange(8)[:, None]).sum(0)
    b = (pi[8:] << np.arange(8)[:, None]).sum(0)
    got = (r["last"].astype(np.int64) << np.arange(9)).sum(axis=1)
    assert np.array_equal(got, a + b)


def test_multiplier_equals_a_times_b():
    nl = workloads.array_multiplier(32)
    lanes = np.concatenate([np.arange(0, 2048), np.arange((1 << 20) - 2048, 1 << 20)]).astype(np.uint64)
    r = oracle.simulate(nl, lanes, 1, seed=2, want=("last",))
    pi = _ref.pi_bits(2, 64, 0, lanes)
    a = _ref.bits_to_int(pi[:32].T)
    b = _ref.bits_to_int(pi[32:].T)
    got = _ref.bits_to_int(r["last"])
    assert (got == a * b).all()


# ---------------------------------------------------------------- sequential closed forms

def _lfsr16_sequence(n):
    s = [1] + [0] * 15                       # s1..s16
    seq = []
    for _ in range(n):
        seq.append(list(s))
        fb = s[15] ^ s[14] ^ s[12] ^ s[3]    # taps 16, 15, 13, 4
        s = [fb] + s[:15]
    return np.array(seq, dtype=np.uint8)


def test_software_lfsr_is_maximal():
    # x^16 + x^15 + x^13 + x^4 + 1 is primitive: the state recurs after exactly 2^16 - 1
    seq = _lfsr16_sequence(65536)
    packed = _ref.bits_to_int(seq)
    assert packed[65535] == packed[0]
    assert len(set(packed[:65535].tolist())) == 65535


def test_probes_lfsr_and_counters():
    nl = workloads.probes_circuit()
    cycles = 65600
    lanes = np.array([0, 63, 64, 1000], dtype=np.uint64)
    r = oracle.simulate(nl, lanes, cycles, seed=7, want=("trace", "regs"))
    tr = r["trace"]                                        # [lane][cycle][30]
    lf = _lfsr16_sequence(cycles)
    for li in range(len(lanes)):
        assert np.array_equal(tr[li, :, 0:16], lf)
        cnt8 = _ref.bits_to_int(tr[li, :300, 16:24])
        assert (cnt8 == np.arange(300) % 256).all()
    # 6-bit counter enabled by PI 0: Q(c) = #{c' < c : en(c') = 1} mod 64
    c_chk = 200
    r2 = oracle.simulate(nl, lanes, c_chk, seed=7, want=("trace",))
    en = np.stack([_ref.pi_bits(7, 1, c, lanes)[0] for c in range(c_chk)], axis=1)  # [lane][c]
    exp = np.concatenate([np.zeros((len(lanes), 1), int), np.cumsum(en, axis=1)[:, :-1]], axis=1) % 64
    got = np.stack([_ref.bits_to_int(r2["trace"][li, :, 24:30]) for li in range(len(lanes))])
    assert (got == exp).all()


def test_register_edge_cases_closed_forms():
    nl = workloads.register_edge_cases()
    lanes = np.arange(128, dtype=np.uint64)
    C = 12
    r = oracle.simulate(nl, lanes, C, seed=11, want=("trace", "regs"))
    tr = r["trace"].astype(int)                            # [lane][c][10]
    p0 = np.stack([_ref.pi_bits(11, 2, c, lanes) for c in range(C)], axis=2)  # [2][lane][c]

    def delayed(d):
        out = np.zeros((len(lanes), C), int)
        out[:, d:] = p0[0][:, :C - d]
        return out
    assert np.array_equal(tr[:, :, 0], delayed(1))          # a  <- PI0
    assert np.array_equal(tr[:, :, 1], delayed(2))          # b1 <- a
    assert np.array_equal(tr[:, :, 2], delayed(3))
    assert np.array_equal(tr[:, :, 3], delayed(4))
    assert (tr[:, :, 4] == 1).all()                         # hold
    assert np.array_equal(tr[:, :, 5], np.tile(1 - np.arange(C) % 2, (len(lanes), 1)))
    assert np.array_equal(tr[:, :, 6], np.tile(np.arange(C) % 2, (len(lanes), 1)))
    assert (tr[:, :, 7] == 0).all() and (tr[:, :, 8] == 1).all()
    assert np.array_equal(tr[:, :, 9], p0[0] & p0[1])
    # final registers = Q(C): a = PI0(C-1), x = 1 iff C even
    assert np.array_equal(r["regs"][:, 0], p0[0][:, C - 1])
    assert (r["regs"][:, 5] == (1 - C % 2)).all()


# ---------------------------------------------------------------- brute force, different algorithm

def _full_tt(nl, g):
    """The whole truth table of gate g as one Python int (k <= 8: up to 4 words)."""
    t = int(nl.gate_tt[g])
    if nl.gate_tt_hi is not None:
        for j in range(3):
            t |= int(nl.gate_tt_hi[g, j]) << (64 * (j + 1))
    return t


def _recursive_eval(nl, pis, q):
    """Value of every net by memoised recursion on the definition (no topological sort)."""
    base = nl.n_pi + nl.n_reg
    memo = {}

    def val(n):
        if n < nl.n_pi:
            return pis[n]
        if n < base:
            return q[n - nl.n_pi]
        if n in memo:
            return memo[n]
        g = n - base
        idx = 0
        for j, x in enumerate(nl.inputs_of(g).tolist()):
            idx |= val(x) << j
        memo[n] = (_full_tt(nl, g) >> idx) & 1
        return memo[n]
    return val


@pytest.mark.parametrize("seed", range(12))
def test_tiny_netlists_bruteforce(seed):
    nl = workloads.random_tiny(seed, n_pi=4, n_reg=3, n_gates=25, n_po=6,
                               max_k=(4, 6, 8)[seed % 3])
    cycles = 5
    lanes = np.arange(64, dtype=np.uint64)
    stim = workloads.random_host_stimulus(100 + seed, cycles, nl.n_pi, 1)
    # cycle 0 enumerates all 2^4 PI vectors over lanes 0..15 (brute force of the inputs)
    for p in range(nl.n_pi):
        word = 0
        for s in range(16):
            word |= ((s >> p) & 1) << s
        stim[0, p, 0] = (int(stim[0, p, 0]) & ~0xFFFF) | word
    for mode in ("tt", "poly"):
        r = oracle.simulate(nl, lanes, cycles, host_stim=stim, mode=mode)
        assert r["violations"] == 0
        for li in range(64):
            q = [int(x) for x in nl.reg_init]
            sig = 0
            for c in range(cycles):
                pis = [(int(stim[c, p, 0]) >> li) & 1 for p in range(nl.n_pi)]
                val = _recursive_eval(nl, pis, q)
                outs = [val(int(o)) for o in nl.po]
                assert list(r["trace"][li, c]) == outs
                v = 0
                for o, b in enumerate(outs):
                    v ^= b << (o % 64)
                sig = _ref.misr_step(sig, v)
                q = [val(int(d)) for d in nl.reg_d]
            assert list(r["regs"][li]) == q
            assert int(r["sig"][li]) == sig


def test_gate_order_does_not_matter():
    nl = workloads.synthetic(3000, 120, 16, 40, 12, seed=9, name="s")
    pn = nl.permuted(5)
    lanes = np.array([0, 1, 63, 64, 200, 4095], dtype=np.uint64)
    a = oracle.simulate(nl, lanes, 20, seed=3)
    b = oracle.simulate(pn, lanes, 20, seed=3)
    for key in ("trace", "regs", "sig"):
        assert np.array_equal(a[key], b[key])


def test_poly_mode_equals_tt_mode_on_synthetic():
    nl = workloads.synthetic(5000, 200, 32, 48, 16, seed=10, name="s")
    lanes = np.arange(0, 640, 5, dtype=np.uint64)
    a = oracle.simulate(nl, lanes, 8, seed=4, mode="tt")
    b = oracle.simulate(nl, lanes, 8, seed=4, mode="poly")
    assert b["violations"] == 0
    for key in ("trace", "regs", "sig"):
        assert np.array_equal(a[key], b[key])


def test_combinational_loop_rejected():
    b = W.Builder()
    p = b.pi()
    b.gates.append(([("gate", 1), p], W.AND2))
    b.gates.append(([("gate", 0), p], W.OR2))
    b.out(("gate", 0))
    nl = b.build("loop")
    assert oracle.topo_order(nl) is None
    with pytest.raises(ValueError):
        oracle.simulate(nl, np.array([0], dtype=np.uint64), 1)


def test_asap_depth_of_structural_circuits():
    # ripple-carry adder: the carry chain is the critical path — sum bit i of a
    # ripple adder built from (XOR, XOR, AND, AND, OR) cells is at depth 2i+1 ... 2i+2
    lv = oracle.asap_levels(workloads.adder(8))
    assert lv.max() == 15
    # n x n array multiplier of ripple-carry rows: depth 6n - 8 (n >= 3), so 184 at n = 32
    # (SURVEY §8(a) row a2); checked against an independent memoised-DFS longest path
    def dfs_depth(nl):
        base = nl.n_pi + nl.n_reg
        memo = {}
        for g0 in range(nl.n_gates):                     # iterative DFS, any order
            stack = [g0]
            while stack:
                g = stack[-1]
                if g in memo:
                    stack.pop()
                    continue
                ins = [int(n) - base for n in nl.gate_in[nl.gate_in_off[g]:nl.gate_in_off[g + 1]] if n >= base]
                todo = [h for h in ins if h not in memo]
                if todo:
                    stack.extend(todo)
                    continue
                memo[g] = 0 if nl.gate_k[g] == 0 else 1 + max((memo[h] for h in ins), default=0)
                stack.pop()
        return memo
    for n in (3, 4, 5, 8, 13, 16, 32):
        nl = workloads.array_multiplier(n)
        lv = oracle.asap_levels(nl)
        assert lv.max() == 6 * n - 8, (n, lv.max())
        if n <= 16:
            d = dfs_depth(nl)
            assert all(int(lv[g]) == d[g] for g in range(nl.n_gates))
    assert oracle.asap_levels(workloads.array_multiplier(32)).max() == 184
