"""Cone collapsing into <= L-input LUTs (gs_compile_opts.lut_k, PAPER.md
P:151): the collapsed LUT netlist is read back through gs_program_gate_lut and
simulated by the ORACLE next to the original netlist — same outputs, registers and
signatures on every lane and cycle — so the compiler transformation is checked on CPU
against a simulator that shares no code with it.  Closed forms (a+b) are checked too.
"""
import numpy as np
import pytest

import oracle
import workloads
import paper_conf_ipps_gavierrprs23_b200 as gs
from tests._build import ensure_built

ensure_built()


def collapsed_netlist(nl, L, balance=True):
    prog = gs.Netlist.from_arrays(nl).compile(balance=balance, lut_k=L)
    ks, ins, tts = [], [], []
    for g in range(nl.n_gates):
        i, t = prog.gate_lut(g)
        ks.append(len(i))
        ins.extend(i)
        tts.append(t)
    off = np.zeros(nl.n_gates + 1, dtype=np.int64)
    off[1:] = np.cumsum(ks)
    lo = np.array([t & (2**64 - 1) for t in tts], dtype=np.uint64)
    hi = np.array([[(t >> (64 * j)) & (2**64 - 1) for j in (1, 2, 3)] for t in tts], dtype=np.uint64)
    c = workloads.Netlist(nl.n_pi, nl.reg_init, nl.reg_d, np.array(ks, dtype=np.uint8),
                          off.astype(np.uint32), np.array(ins, dtype=np.uint32), lo, nl.po,
                          name=nl.name + f"_L{L}", meta=nl.meta,
                          gate_tt_hi=hi if max(ks, default=0) > 6 else None)
    return prog, c


CASES = [("adder", lambda: workloads.adder(8)), ("mult8", lambda: workloads.array_multiplier(8)),
         ("wide8", lambda: workloads.random_tiny(7, n_pi=6, n_reg=4, n_gates=80, n_po=10, max_k=8)),
         ("tiny3", lambda: workloads.random_tiny(3, n_pi=5, n_reg=4, n_gates=120, n_po=10)),
         ("tiny9", lambda: workloads.random_tiny(9, n_pi=6, n_reg=6, n_gates=200, n_po=12, max_k=3)),
         ("regs", workloads.register_edge_cases), ("probes", workloads.probes_circuit),
         ("synth", lambda: workloads.synthetic(3000, 120, 16, 40, 12, seed=9, name="s"))]


@pytest.mark.parametrize("L", [2, 3, 4, 6, 8])
@pytest.mark.parametrize("name,make", CASES)
def test_collapsed_netlist_simulates_identically(name, make, L):
    nl = make()
    prog, c = collapsed_netlist(nl, L)
    base = prog.info
    # every LUT the compiler produced has at most L inputs unless it was already wider
    wide = c.gate_k > L
    assert (c.gate_k[wide] == nl.gate_k[wide]).all()
    lanes = np.arange(0, 4096, 7)
    cycles = 6
    a = oracle.simulate(nl, lanes, cycles, seed=17)
    b = oracle.simulate(c, lanes, cycles, seed=17)
    for key in ("trace", "regs", "sig"):
        assert np.array_equal(a[key], b[key]), key
    # absorbed gates are unreferenced
    dead = set(int(g) for g in np.nonzero((c.gate_k == 0) & (nl.gate_k > 0))[0])
    gate_nets = {nl.n_pi + nl.n_reg + g for g in dead}
    assert not gate_nets & set(c.gate_in.tolist())
    assert not gate_nets & set(int(x) for x in nl.po) and not gate_nets & set(int(x) for x in nl.reg_d)
    assert base["n_eval_gates"] == int((c.gate_k > 0).sum())


@pytest.mark.parametrize("L", [3, 4, 5, 6])
def test_collapse_reduces_depth_and_keeps_adder_closed_form(L):
    nl = workloads.adder(8)
    flat = gs.Netlist.from_arrays(nl).compile()
    prog, c = collapsed_netlist(nl, L)
    assert prog.info["n_levels"] < flat.info["n_levels"]
    assert prog.info["n_eval_gates"] < flat.info["n_eval_gates"]
    # exhaustive a + b through the oracle on the collapsed LUT netlist
    a = np.arange(1 << 16) & 0xFF
    b = np.arange(1 << 16) >> 8
    bits = np.concatenate([(a[None, :] >> np.arange(8)[:, None]) & 1,
                           (b[None, :] >> np.arange(8)[:, None]) & 1]).astype(np.uint8)
    words = np.packbits(bits, axis=1, bitorder="little").view(np.uint64)[None]
    o = oracle.simulate(c, np.arange(1 << 16), 1, host_stim=words, want=("last",))
    out = o["last"].astype(np.int64)
    assert np.array_equal((out << np.arange(9)[None, :]).sum(1), a + b)


def test_collapse_depth_never_increases_and_multiplier_halves():
    nl = workloads.array_multiplier(32)
    flat = gs.Netlist.from_arrays(nl).compile(balance=False).info["n_levels"]
    for L in range(2, 7):
        lv = gs.Netlist.from_arrays(nl).compile(balance=False, lut_k=L).info["n_levels"]
        assert lv <= flat
    assert gs.Netlist.from_arrays(nl).compile(lut_k=6).info["n_levels"] <= flat // 2


def test_lut_k_argument_checks():
    nl = gs.Netlist.from_arrays(workloads.adder(4))
    for bad in (1, 9):
        with pytest.raises(gs.GsError) as e:
            nl.compile(lut_k=bad)
        assert e.value.code == gs.GS_ERR_ARG
    with pytest.raises(gs.GsError):
        nl.compile(max_k=3, lut_k=4)
