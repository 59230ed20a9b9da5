"""Seeded netlist generators — the ONLY module shared by the oracle side and the CUDA side.

This module builds *inputs*: gate netlists with truth tables, registers and I/O.
It holds none of the method's arithmetic — no gate evaluation, no levelization,
no polynomial compilation, no stimulus hashing.  Truth tables of library cells
are written out as constants / by tabulating a Python lambda over the 2^k
points (that is how a netlist *author* writes a LUT, Fig. 3).

Netlist array format (the bulk format of ``gs_netlist_load_arrays``, see
include/gsim.h):

* net ids ``[0, n_pi)``                 primary inputs (PI p is net p)
* net ids ``[n_pi, n_pi + n_reg)``      register outputs Q (the FF "pseudo-inputs",
                                        PAPER.md P:237-241)
* net ids ``[n_pi + n_reg, ...)``       gate outputs, gate g is net n_pi + n_reg + g
* ``gate_k[g]``                         fan-in k of gate g (0 <= k <= 8; L of P:167)
* ``gate_in[gate_in_off[g]:gate_in_off[g+1]]`` input nets x_0..x_{k-1}
* ``gate_tt[g]``                        truth table, LSB-first: bit m = f(x) with
                                        x_i = bit i of m (reading R1);
                                        bits 0..63
* ``gate_tt_hi[g]`` (optional)          bits 64..255 of the table as 3 more uint64
                                        words, for gates with k = 7, 8 (None if none)
* ``reg_init[r]``, ``reg_d[r]``         initial Q and the net feeding D (the FF
                                        "pseudo-output")
* ``po[o]``                             primary-output nets
"""
from __future__ import annotations

from dataclasses import dataclass, field
import numpy as np

U32 = np.uint32


# ----------------------------------------------------------------------------
# truth-table authoring helpers (input construction only)
# ----------------------------------------------------------------------------

def tt_of(k: int, f) -> int:
    """Tabulate a k-input Python predicate into an LSB-first truth table."""
    tt = 0
    for m in range(1 << k):
        xs = tuple((m >> i) & 1 for i in range(k))
        if f(*xs):
            tt |= 1 << m
    return tt


BUF = tt_of(1, lambda a: a)
NOT = tt_of(1, lambda a: 1 - a)
AND2 = tt_of(2, lambda a, b: a & b)
OR2 = tt_of(2, lambda a, b: a | b)
XOR2 = tt_of(2, lambda a, b: a ^ b)
NAND2 = tt_of(2, lambda a, b: 1 - (a & b))
NOR2 = tt_of(2, lambda a, b: 1 - (a | b))
XNOR2 = tt_of(2, lambda a, b: 1 - (a ^ b))
AOI21 = tt_of(3, lambda a, b, c: 1 - ((a & b) | c))
OAI21 = tt_of(3, lambda a, b, c: 1 - ((a | b) & c))
MUX21 = tt_of(3, lambda a, b, s: b if s else a)
MAJ3 = tt_of(3, lambda a, b, c: 1 if a + b + c >= 2 else 0)
AND3 = tt_of(3, lambda a, b, c: a & b & c)
XOR3 = tt_of(3, lambda a, b, c: a ^ b ^ c)
AND4 = tt_of(4, lambda a, b, c, d: a & b & c & d)
XOR4 = tt_of(4, lambda a, b, c, d: a ^ b ^ c ^ d)
AOI22 = tt_of(4, lambda a, b, c, d: 1 - ((a & b) | (c & d)))
OAI22 = tt_of(4, lambda a, b, c, d: 1 - ((a | b) & (c | d)))
OR4 = tt_of(4, lambda a, b, c, d: a | b | c | d)
NOR4 = tt_of(4, lambda a, b, c, d: 1 - (a | b | c | d))

LIBRARY = {
    2: [AND2, OR2, NAND2, NOR2, XOR2, XNOR2],
    3: [AOI21, OAI21, MUX21, MAJ3, AND3, XOR3],
    4: [AND4, XOR4, AOI22, OAI22, OR4, NOR4],
}


# ----------------------------------------------------------------------------
# netlist container
# ----------------------------------------------------------------------------

@dataclass
class Netlist:
    n_pi: int
    reg_init: np.ndarray          # uint8 [n_reg]
    reg_d: np.ndarray             # uint32 [n_reg]
    gate_k: np.ndarray            # uint8 [n_gates]
    gate_in_off: np.ndarray       # uint32 [n_gates + 1]
    gate_in: np.ndarray           # uint32 [E]
    gate_tt: np.ndarray           # uint64 [n_gates]
    po: np.ndarray                # uint32 [n_po]
    name: str = ""
    meta: dict = field(default_factory=dict)
    gate_tt_hi: np.ndarray | None = None   # uint64 [n_gates][3] (k = 7, 8) or None

    @property
    def n_reg(self) -> int:
        return int(self.reg_init.shape[0])

    @property
    def n_gates(self) -> int:
        return int(self.gate_k.shape[0])

    @property
    def n_po(self) -> int:
        return int(self.po.shape[0])

    @property
    def n_nets(self) -> int:
        return self.n_pi + self.n_reg + self.n_gates

    def gate_net(self, g: int) -> int:
        return self.n_pi + self.n_reg + g

    def q_net(self, r: int) -> int:
        return self.n_pi + r

    def inputs_of(self, g: int) -> np.ndarray:
        return self.gate_in[self.gate_in_off[g]:self.gate_in_off[g + 1]]

    def permuted(self, seed: int) -> "Netlist":
        """Same circuit with gate ids shuffled (tests that nobody relies on id order)."""
        rng = np.random.default_rng(seed)
        G = self.n_gates
        perm = rng.permutation(G)              # new gate j = old gate perm[j]
        inv = np.empty(G, dtype=np.int64)
        inv[perm] = np.arange(G)
        base = self.n_pi + self.n_reg

        def remap(nets):
            nets = nets.astype(np.int64)
            out = nets.copy()
            m = nets >= base
            out[m] = base + inv[nets[m] - base]
            return out.astype(U32)

        k = self.gate_k[perm]
        off = np.zeros(G + 1, dtype=np.int64)
        off[1:] = np.cumsum(k.astype(np.int64))
        ins = np.empty(int(off[-1]), dtype=U32)
        for j in range(G):
            ins[off[j]:off[j + 1]] = self.inputs_of(int(perm[j]))
        return Netlist(self.n_pi, self.reg_init.copy(), remap(self.reg_d), k.copy(),
                       off.astype(U32), remap(ins), self.gate_tt[perm].copy(), remap(self.po),
                       name=self.name + "+perm", meta=dict(self.meta),
                       gate_tt_hi=None if self.gate_tt_hi is None else self.gate_tt_hi[perm].copy())


class Builder:
    """Incremental structural netlist builder (small circuits; probes)."""

    def __init__(self):
        self.n_pi = 0
        self.reg_init: list[int] = []
        self.reg_d: list = []
        self.gates: list[tuple[list, int]] = []
        self.pos: list = []

    # references are tagged tuples, resolved to net ids by build()
    def pi(self):
        self.n_pi += 1
        return ("pi", self.n_pi - 1)

    def reg(self, init: int = 0):
        self.reg_init.append(int(init))
        self.reg_d.append(None)
        return ("reg", len(self.reg_init) - 1)

    def set_d(self, q, d):
        assert q[0] == "reg"
        self.reg_d[q[1]] = d

    def gate(self, tt: int, *ins):
        self.gates.append((list(ins), int(tt)))
        return ("gate", len(self.gates) - 1)

    def out(self, net):
        self.pos.append(net)
        return len(self.pos) - 1

    def build(self, name: str = "", meta: dict | None = None) -> Netlist:
        n_pi, n_reg = self.n_pi, len(self.reg_init)

        def nid(ref):
            kind, i = ref
            return {"pi": i, "reg": n_pi + i, "gate": n_pi + n_reg + i}[kind]

        ks = np.array([len(ins) for ins, _ in self.gates], dtype=np.uint8)
        off = np.zeros(len(self.gates) + 1, dtype=np.int64)
        off[1:] = np.cumsum(ks.astype(np.int64))
        ins = np.array([nid(r) for g, _ in self.gates for r in g], dtype=U32)
        assert all(d is not None for d in self.reg_d), "register without D"
        M64 = (1 << 64) - 1
        wide = any(len(g) > 6 for g, _ in self.gates)
        hi = (np.array([[(tt >> (64 * j)) & M64 for j in (1, 2, 3)] for _, tt in self.gates], dtype=np.uint64)
              if wide else None)
        return Netlist(
            n_pi=n_pi,
            reg_init=np.array(self.reg_init, dtype=np.uint8),
            reg_d=np.array([nid(d) for d in self.reg_d], dtype=U32),
            gate_k=ks, gate_in_off=off.astype(U32), gate_in=ins,
            gate_tt=np.array([tt & M64 for _, tt in self.gates], dtype=np.uint64),
            po=np.array([nid(p) for p in self.pos], dtype=U32),
            name=name, meta=meta or {}, gate_tt_hi=hi)


# ----------------------------------------------------------------------------
# structural circuits (C1, C2) and sequential probes
# ----------------------------------------------------------------------------

def _full_add(b: Builder, x, y, c):
    """Sum/carry of the present operands among (x, y, c); None = absent (0)."""
    ops = [v for v in (x, y, c) if v is not None]
    if len(ops) == 0:
        return None, None
    if len(ops) == 1:
        return ops[0], None
    if len(ops) == 2:
        return b.gate(XOR2, *ops), b.gate(AND2, *ops)
    t = b.gate(XOR2, x, y)
    s = b.gate(XOR2, t, c)
    g = b.gate(AND2, x, y)
    p = b.gate(AND2, t, c)
    return s, b.gate(OR2, g, p)


def adder(nbits: int = 8) -> Netlist:
    """C1: n-bit ripple-carry adder, a = PI 0..n-1, b = PI n..2n-1 (bit i = PI i).

    POs: sum bits 0..n-1 then carry-out (n+1 outputs), i.e. out = a + b.
    8 bits: half adder + 7 full adders of 2-input XOR/AND/OR = 37 gates.
    """
    b = Builder()
    A = [b.pi() for _ in range(nbits)]
    B = [b.pi() for _ in range(nbits)]
    c = None
    for i in range(nbits):
        s, c = _full_add(b, A[i], B[i], c)
        b.out(s)
    b.out(c)
    return b.build(f"add{nbits}", {"a_pis": list(range(nbits)),
                                   "b_pis": list(range(nbits, 2 * nbits))})


def array_multiplier(nbits: int = 32) -> Netlist:
    """C2: n x n unsigned array multiplier (AND partial products + row ripple adders).

    a = PI 0..n-1, b = PI n..2n-1, 2n POs = a*b (bit o = PO o).  32 bits: 5,888 gates.
    """
    b = Builder()
    A = [b.pi() for _ in range(nbits)]
    B = [b.pi() for _ in range(nbits)]
    pp = [[b.gate(AND2, A[j], B[i]) for j in range(nbits)] for i in range(nbits)]
    acc: dict[int, object] = {j: pp[0][j] for j in range(nbits)}
    for i in range(1, nbits):
        c = None
        for j in range(nbits):
            pos = i + j
            s, c = _full_add(b, acc.get(pos), pp[i][j], c)
            acc[pos] = s
        if c is not None:
            acc[i + nbits] = c
    for pos in range(2 * nbits):
        b.out(acc[pos])
    return b.build(f"mul{nbits}", {"a_pis": list(range(nbits)),
                                   "b_pis": list(range(nbits, 2 * nbits))})


LFSR16_TAPS = (16, 15, 13, 4)   # x^16 + x^15 + x^13 + x^4 + 1


def add_lfsr16(b: Builder):
    """Fibonacci LFSR: s1 <- s16^s15^s13^s4 (one XOR4 LUT), s_i <- s_{i-1} (shift chain).

    Returns the Q refs [s1..s16]; s1 starts at 1, the rest at 0.
    """
    s = [b.reg(1 if i == 0 else 0) for i in range(16)]
    fb = b.gate(XOR4, *[s[t - 1] for t in LFSR16_TAPS])
    b.set_d(s[0], fb)
    for i in range(1, 16):
        b.set_d(s[i], s[i - 1])
    return s


def add_counter(b: Builder, nbits: int, enable=None):
    """Binary up-counter; counts cycles (enable None) or cycles with enable = 1."""
    q = [b.reg(0) for _ in range(nbits)]
    carry = enable
    for i in range(nbits):
        if carry is None:
            b.set_d(q[i], b.gate(NOT, q[i]))
            carry = q[i]
        else:
            b.set_d(q[i], b.gate(XOR2, q[i], carry))
            if i + 1 < nbits:
                carry = b.gate(AND2, q[i], carry)
    return q


def probes_circuit() -> Netlist:
    """Stand-alone probe circuit: LFSR16, 8-bit counter, 6-bit counter enabled by PI 0."""
    b = Builder()
    en = b.pi()
    lf = add_lfsr16(b)
    c8 = add_counter(b, 8)
    c6 = add_counter(b, 6, enable=en)
    for q in lf + c8 + c6:
        b.out(q)
    return b.build("probes", {"probe_po": {"lfsr16": (0, 16), "cnt8": (16, 24), "cnt6": (24, 30)},
                              "cnt6_enable_pi": 0})


def register_edge_cases() -> Netlist:
    """Registers fed by a PI, by other registers (shift chain, swap) and by themselves.

    PI 0 -> a; a -> b1 -> b2 -> b3 (delay line); h holds (D = own Q, init 1);
    x <-> y swap (init 1, 0); plus constant-0/1 LUTs (k = 0) and an AND of PI 0, 1.
    POs: a, b1, b2, b3, h, x, y, const0, const1, and2(PI0, PI1).
    """
    b = Builder()
    p0, p1 = b.pi(), b.pi()
    a = b.reg(0)
    b.set_d(a, p0)
    b1, b2, b3 = b.reg(0), b.reg(0), b.reg(0)
    b.set_d(b1, a)
    b.set_d(b2, b1)
    b.set_d(b3, b2)
    h = b.reg(1)
    b.set_d(h, h)
    x, y = b.reg(1), b.reg(0)
    b.set_d(x, y)
    b.set_d(y, x)
    c0 = b.gate(0)
    c1 = b.gate(1)
    g = b.gate(AND2, p0, p1)
    for n in (a, b1, b2, b3, h, x, y, c0, c1, g):
        b.out(n)
    return b.build("regedge")


# ----------------------------------------------------------------------------
# seeded synthetic sequential netlists (C3, C4, C5) — recipe in SURVEY.md §8(d)
# ----------------------------------------------------------------------------

def _m0_masks(k: int) -> list[int]:
    return [sum(1 << m for m in range(1 << k) if not (m >> i) & 1) for i in range(k)]


def _random_full_support_tts(rng, k: int, n: int) -> np.ndarray:
    """n uniform random k-input truth tables that depend on every input."""
    out = np.empty(n, dtype=np.uint64)
    todo = np.arange(n)
    width = 1 << k
    masks = _m0_masks(k)
    while todo.size:
        t = rng.integers(0, 1 << width, size=todo.size, dtype=np.uint64) if width < 64 else \
            rng.integers(0, np.iinfo(np.uint64).max, size=todo.size, dtype=np.uint64, endpoint=True)
        ok = np.ones(todo.size, dtype=bool)
        for i in range(k):
            sh = np.uint64(1 << i)
            ok &= ((t >> sh) ^ t) & np.uint64(masks[i]) != 0
        out[todo[ok]] = t[ok]
        todo = todo[~ok]
    return out


def _level_widths(rng, n_gates: int, depth: int) -> np.ndarray:
    lv = np.arange(1, depth + 1)
    w = (np.exp(-lv / (0.35 * depth)) + 0.02) * rng.lognormal(0.0, 0.5, size=depth)
    forced = (lv % 8) == 0
    out = np.zeros(depth, dtype=np.int64)
    out[forced] = rng.integers(1, 33, size=int(forced.sum()))
    rest = n_gates - int(out.sum())
    ww = np.where(forced, 0.0, w)
    ww = ww / ww.sum() * rest
    base = np.floor(ww).astype(np.int64)
    base[forced] = 0
    rem = rest - int(base.sum())
    frac_order = np.argsort(-(ww - base), kind="stable")
    frac_order = frac_order[~forced[frac_order]]
    base[frac_order[:rem]] += 1
    out[~forced] = base[~forced]
    out = np.maximum(out, 1)
    # keep the exact total (maximum(…,1) may have added a few)
    excess = int(out.sum()) - n_gates
    i = int(np.argmax(out))
    out[i] -= excess
    return out


def synthetic(n_gates: int, n_reg: int, n_pi: int, n_po: int, depth: int, seed: int,
              name: str = "synthetic", with_probes: bool = True) -> Netlist:
    """Seeded synthetic sequential netlist, shaped like SURVEY.md §8(d) C3–C5.

    * level widths w_l ∝ exp(-l/(0.35 D)) + 0.02 with log-normal(σ=0.5) noise,
      every 8th level forced to <= 32 gates (front-loaded, unbalanced: P:62);
    * k ∈ {2,3,4} with p = {0.3, 0.4, 0.3}; input 0 from level l-1 (so ASAP = l),
      other inputs from l-1 (0.6), l-2..l-8 (0.3), any earlier net incl. PI/Q (0.1);
    * TTs: 50 % library cells, 50 % uniform random full-support TTs;
    * register D from the last quarter of levels w.p. 0.7, else any net;
    * probes (LFSR16, 8-bit counter, 6-bit counter enabled by PI 0) embedded as
      POs 0..29 when ``with_probes``.
    """
    rng = np.random.default_rng(seed)
    # ---- probes first (small structural circuits) -------------------------
    b = Builder()
    for _ in range(n_pi):
        b.pi()
    probe_po = {}
    if with_probes:
        lf = add_lfsr16(b)
        c8 = add_counter(b, 8)
        c6 = add_counter(b, 6, enable=("pi", 0))
        probe_q = lf + c8 + c6
        probe_po = {"lfsr16": (0, 16), "cnt8": (16, 24), "cnt6": (24, 30)}
    else:
        probe_q = []
    n_probe_regs = len(b.reg_init)
    n_probe_gates = len(b.gates)
    assert n_reg >= n_probe_regs and n_gates > n_probe_gates and n_po >= len(probe_q)
    n_reg_total = n_reg
    base = n_pi + n_reg_total                    # first gate net id
    G_rest = n_gates - n_probe_gates

    # probe gates -> arrays (their nets reference PIs / probe regs / probe gates)
    def nid(ref):
        kind, i = ref
        return {"pi": i, "reg": n_pi + i, "gate": base + i}[kind]

    k_parts = [np.array([len(ins) for ins, _ in b.gates], dtype=np.uint8)]
    in_parts = [np.array([nid(r) for ins, _ in b.gates for r in ins], dtype=np.int64)]
    tt_parts = [np.array([tt for _, tt in b.gates], dtype=np.uint64)]

    widths = _level_widths(rng, G_rest, depth)
    lvl_start = np.zeros(depth + 2, dtype=np.int64)   # net id of first gate of level l (1-based)
    lvl_start[1] = base + n_probe_gates
    for l in range(1, depth + 1):
        lvl_start[l + 1] = lvl_start[l] + widths[l - 1]
    # level 0 ("sources") = PIs and register Qs: nets [0, base)

    def level_range(l):
        if l <= 0:
            return 0, base
        return int(lvl_start[l]), int(lvl_start[l + 1])

    ks = np.array([2, 3, 4], dtype=np.uint8)
    for l in range(1, depth + 1):
        n = int(widths[l - 1])
        k = rng.choice(ks, size=n, p=[0.3, 0.4, 0.3])
        lo0, hi0 = level_range(l - 1)
        cols = []
        cols.append(rng.integers(lo0, hi0, size=n))
        for j in range(1, 4):
            cat = rng.choice(3, size=n, p=[0.6, 0.3, 0.1])
            c = rng.integers(lo0, hi0, size=n)
            # l-2 .. l-8 : a uniformly chosen earlier level among those that exist
            far_l = l - rng.integers(2, 9, size=n)
            far_l = np.maximum(far_l, 0)
            fl_lo = np.where(far_l <= 0, 0, lvl_start[np.maximum(far_l, 1)])
            fl_hi = np.where(far_l <= 0, base, lvl_start[np.maximum(far_l, 1) + 1])
            far = fl_lo + (rng.random(n) * (fl_hi - fl_lo)).astype(np.int64)
            anyn = rng.integers(0, lvl_start[l], size=n)
            c = np.where(cat == 1, far, c)
            c = np.where(cat == 2, anyn, c)
            cols.append(c)
        ins = np.stack(cols, axis=1)                  # [n, 4]
        # resample duplicate inputs a few times (duplicates remain legal, P:165 / Q9);
        # column 0 is never touched so ASAP(g) = l holds by construction
        for _ in range(4):
            dup_any = False
            for a in range(1, 4):
                dup = np.zeros(n, dtype=bool)
                for c2 in range(a):
                    dup |= ins[:, a] == ins[:, c2]
                dup &= a < k
                if dup.any():
                    dup_any = True
                    ins[dup, a] = rng.integers(0, lvl_start[l], size=int(dup.sum()))
            if not dup_any:
                break
        tt = np.empty(n, dtype=np.uint64)
        lib = rng.random(n) < 0.5
        for kk in (2, 3, 4):
            sel = k == kk
            nl = int((sel & lib).sum())
            libs = np.array(LIBRARY[kk], dtype=np.uint64)
            tt[sel & lib] = libs[rng.integers(0, len(libs), size=nl)]
            nr = int((sel & ~lib).sum())
            tt[sel & ~lib] = _random_full_support_tts(rng, kk, nr)
        mask = np.arange(4)[None, :] < k[:, None]
        k_parts.append(k.astype(np.uint8))
        in_parts.append(ins[mask])          # row-major: gate by gate, first k columns
        tt_parts.append(tt)

    gate_k = np.concatenate(k_parts)
    gate_in = np.concatenate(in_parts).astype(U32)
    gate_tt = np.concatenate(tt_parts)
    off = np.zeros(n_gates + 1, dtype=np.int64)
    off[1:] = np.cumsum(gate_k.astype(np.int64))

    # ---- registers ------------------------------------------------------------
    reg_init = np.zeros(n_reg_total, dtype=np.uint8)
    reg_d = np.zeros(n_reg_total, dtype=np.int64)
    reg_init[:n_probe_regs] = b.reg_init
    reg_d[:n_probe_regs] = [nid(d) for d in b.reg_d]
    nr = n_reg_total - n_probe_regs
    reg_init[n_probe_regs:] = rng.integers(0, 2, size=nr)
    last_q_lo = int(lvl_start[depth - depth // 4 + 1]) if depth >= 4 else int(lvl_start[1])
    hi_all = int(lvl_start[depth + 1])
    late = rng.random(nr) < 0.7
    reg_d[n_probe_regs:] = np.where(late, rng.integers(last_q_lo, hi_all, size=nr),
                                    rng.integers(0, hi_all, size=nr))

    # ---- primary outputs -------------------------------------------------------
    po = np.zeros(n_po, dtype=np.int64)
    po[:len(probe_q)] = [nid(q) for q in probe_q]
    rest = n_po - len(probe_q)
    late = rng.random(rest) < 0.7
    po[len(probe_q):] = np.where(late, rng.integers(last_q_lo, hi_all, size=rest),
                                 rng.integers(base, hi_all, size=rest))
    return Netlist(n_pi, reg_init, reg_d.astype(U32), gate_k, off.astype(U32), gate_in,
                   gate_tt, po.astype(U32), name=name,
                   meta={"probe_po": probe_po, "cnt6_enable_pi": 0, "depth": depth,
                         "level_widths": widths.tolist(), "seed": seed})


def random_tiny(seed: int, n_pi: int = 4, n_reg: int = 3, n_gates: int = 30,
                n_po: int = 6, max_k: int = 4) -> Netlist:
    """Tiny random sequential netlist (brute-force tests): gates only read earlier nets.
    max_k up to 8: tables of k = 7, 8 gates spill into ``gate_tt_hi``."""
    rng = np.random.default_rng(seed)
    base = n_pi + n_reg
    ks = rng.integers(0, max_k + 1, size=n_gates).astype(np.uint8)
    ins, tts = [], []
    hi = np.zeros((n_gates, 3), dtype=np.uint64)
    for g in range(n_gates):
        k = int(ks[g])
        avail = base + g
        if avail == 0:
            k = 0
            ks[g] = 0
        ins.extend(int(x) for x in rng.integers(0, avail, size=k))
        if k < 6:
            tts.append(int(rng.integers(0, 1 << (1 << k), dtype=np.uint64)))
        else:
            words = rng.integers(0, np.iinfo(np.uint64).max, size=4, dtype=np.uint64, endpoint=True)
            nw = (1 << k) // 64
            tts.append(int(words[0]))
            hi[g, :nw - 1] = words[1:nw]
    off = np.zeros(n_gates + 1, dtype=np.int64)
    off[1:] = np.cumsum(ks.astype(np.int64))
    return Netlist(n_pi, rng.integers(0, 2, size=n_reg).astype(np.uint8),
                   rng.integers(0, base + n_gates, size=n_reg).astype(U32), ks,
                   off.astype(U32), np.array(ins, dtype=U32), np.array(tts, dtype=np.uint64),
                   rng.integers(0, base + n_gates, size=n_po).astype(U32), name=f"tiny{seed}",
                   gate_tt_hi=hi if max_k > 6 else None)
