"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle, bit-exact.

Every comparison is element by element on the same seeded inputs; the oracle never
sees anything the GPU produced.  Closed forms (a+b, a*b, LFSR, counters) are checked
on ALL lanes where the oracle would be too slow.
"""
import os

import numpy as np
import pytest

import oracle
import workloads
from workloads import netlists as W
import paper_conf_ipps_gavierrprs23_b200 as gs
from tests import _ref
from tests._build import ensure_built

pytestmark = pytest.mark.gpu
ensure_built()


def compile_nl(nl, balance=True):
    return gs.Netlist.from_arrays(nl).compile(balance=balance)


def gpu_trace_bits(tr, words_sel):
    """GPU trace [cycles][po][ntw] -> bits [lanes_of_traced_words][cycles][po]."""
    bits = gs.unpack_lanes(tr)                         # [c][po][ntw*64]
    return np.transpose(bits, (2, 0, 1))


def run_gpu(nl, lanes, cycles, kernel="lut", seed=None, host_stim=None, trace_words=(),
            lane_offset=0, balance=True, use_graphs=True, prog=None, **simkw):
    prog = prog or compile_nl(nl, balance)
    sim = gs.Sim(prog, lanes, lane_offset=lane_offset, kernel=kernel, trace_words=trace_words,
                 trace_cycles=cycles if len(trace_words) else 0, use_graphs=use_graphs, **simkw)
    if host_stim is not None:
        sim.bind_host(host_stim)
    else:
        sim.bind_generated(seed)
    sim.step(cycles)
    sim.sync()
    out = dict(outputs=sim.read_outputs(), regs=sim.read_registers(),
               sigs=sim.read_lane_signatures(), signature=sim.signature())
    if len(trace_words):
        out["trace"] = sim.read_trace()
    sim.close()
    return out


def lane_bits(words_2d, lanes_idx):
    """[rows][W] words -> [len(lanes_idx)][rows] bits for the given local lanes."""
    b = gs.unpack_lanes(words_2d)
    return b[:, lanes_idx].T


KERNELS = ["lut", "poly", "ab"]
BENCH_BALANCE = {"balanced": 1, "asap": 0, "alap": 2}      # bench.py --levels -> gs_compile_opts.balance


# ------------------------------------------------------------------ C1: adder
@pytest.mark.parametrize("kernel", KERNELS)
def test_c1_adder_generated_equals_a_plus_b_and_oracle(kernel):
    cfg = workloads.CONFIGS["C1"]
    nl = cfg.netlist()
    r = run_gpu(nl, cfg.lanes, 1, kernel, seed=cfg.stim_seed, trace_words=range(cfg.lanes // 64))
    lanes = np.arange(cfg.lanes)
    got = lane_bits(r["outputs"], lanes)                                # [lanes][9]
    pi = _ref.pi_lanes_np(cfg.stim_seed, 16, 0, cfg.lanes).astype(np.int64)
    a = (pi[:8] << np.arange(8)[:, None]).sum(0)
    b = (pi[8:] << np.arange(8)[:, None]).sum(0)
    assert np.array_equal((got.astype(np.int64) << np.arange(9)).sum(1), a + b)
    o = oracle.simulate(nl, lanes, 1, seed=cfg.stim_seed)
    assert np.array_equal(got, o["last"])
    assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"])
    assert np.array_equal(r["sigs"], o["sig"])
    assert r["signature"]["lane_sig_sum"] == oracle.lane_sig_sum(o["sig"], lanes)
    assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0
    assert r["signature"]["out_popcount"] == int(o["trace"].sum())


def test_c1_adder_exhaustive_host_stimulus():
    nl = workloads.adder(8)
    lanes = 1 << 16
    s = np.arange(lanes, dtype=np.uint64)
    stim = np.zeros((1, 16, lanes // 64), dtype=np.uint64)
    for p in range(16):
        bits = ((s >> np.uint64(p)) & np.uint64(1)).astype(np.uint8)
        stim[0, p] = np.packbits(bits, bitorder="little").view(np.uint64)
    for kernel in KERNELS:
        r = run_gpu(nl, lanes, 1, kernel, host_stim=stim)
        got = lane_bits(r["outputs"], np.arange(lanes)).astype(np.int64)
        assert np.array_equal((got << np.arange(9)).sum(1), ((s & np.uint64(0xFF)) + (s >> np.uint64(8))).astype(np.int64))
        assert r["signature"]["ab_mismatch"] == 0


# ------------------------------------------------------------------ tiny brute force
@pytest.mark.parametrize("seed", range(10))
@pytest.mark.parametrize("kernel", KERNELS)
def test_tiny_random_netlists_all_lanes_all_cycles(seed, kernel):
    nl = workloads.random_tiny(seed, n_pi=5, n_reg=4, n_gates=40, n_po=7, max_k=4 if seed % 3 else 6)
    lanes, cycles = 256, 7
    stim = workloads.random_host_stimulus(1000 + seed, cycles, nl.n_pi, lanes // 64)
    r = run_gpu(nl, lanes, cycles, kernel, host_stim=stim, trace_words=range(lanes // 64),
                use_graphs=bool(seed % 2))
    o = oracle.simulate(nl, np.arange(lanes), cycles, host_stim=stim)
    assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"])
    assert np.array_equal(lane_bits(r["regs"], np.arange(lanes)), o["regs"])
    assert np.array_equal(lane_bits(r["outputs"], np.arange(lanes)), o["last"])
    assert np.array_equal(r["sigs"], o["sig"])
    assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0


@pytest.mark.parametrize("kernel", KERNELS)
def test_register_edge_cases_and_probes(kernel):
    for nl in (workloads.register_edge_cases(), workloads.probes_circuit()):
        lanes, cycles = 192, 300            # 3 words: exercises the 8-byte vector path
        r = run_gpu(nl, lanes, cycles, kernel, seed=77, trace_words=range(3))
        o = oracle.simulate(nl, np.arange(lanes), cycles, seed=77)
        assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"])
        assert np.array_equal(lane_bits(r["regs"], np.arange(lanes)), o["regs"])
        assert np.array_equal(r["sigs"], o["sig"])


# ------------------------------------------------------------------ C2: multiplier
def test_c2_multiplier_all_lanes_equal_a_times_b():
    cfg = workloads.CONFIGS["C2"]
    nl = cfg.netlist()
    r = run_gpu(nl, cfg.lanes, 1, "lut", seed=cfg.stim_seed)
    bits = gs.unpack_lanes(r["outputs"]).astype(np.uint64)             # [64][lanes]
    prod = np.zeros(cfg.lanes, dtype=np.uint64)
    for o in range(64):
        prod |= bits[o] << np.uint64(o)
    pi = _ref.pi_lanes_np(cfg.stim_seed, 64, 0, cfg.lanes).astype(np.uint64)
    a = np.zeros(cfg.lanes, dtype=np.uint64)
    b = np.zeros(cfg.lanes, dtype=np.uint64)
    for i in range(32):
        a |= pi[i] << np.uint64(i)
        b |= pi[32 + i] << np.uint64(i)
    with np.errstate(over="ignore"):
        assert np.array_equal(prod, a * b)
    # >= 4,096 lanes against the oracle: both ends and a seeded spread
    sample = np.unique(np.concatenate([np.arange(0, 1024), np.arange(cfg.lanes - 1024, cfg.lanes),
                                       np.random.default_rng(0).integers(0, cfg.lanes, 2560)]))
    assert len(sample) >= 4096
    o = oracle.simulate(nl, sample, 1, seed=cfg.stim_seed, want=("last",))
    assert np.array_equal(lane_bits(r["outputs"], sample), o["last"])


def test_c2_kernels_agree():
    cfg = workloads.CONFIGS["C2"]
    r = run_gpu(cfg.netlist(), 1 << 16, 1, "ab", seed=cfg.stim_seed)
    assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0


# ------------------------------------------------------------------ sequential synthetic
def probe_closed_forms(nl, outputs_bits, last_cycle, seed, n_lanes, lane_offset=0):
    """LFSR16 / 8-bit counter / enabled 6-bit counter at the last cycle, all lanes."""
    pp = nl.meta["probe_po"]
    lf = outputs_bits[:, pp["lfsr16"][0]:pp["lfsr16"][1]]
    s = [1] + [0] * 15
    for _ in range(last_cycle):
        s = [s[15] ^ s[14] ^ s[12] ^ s[3]] + s[:15]
    assert (lf == np.array(s, dtype=np.uint8)[None, :]).all()
    c8 = (outputs_bits[:, 16:24].astype(np.int64) << np.arange(8)).sum(1)
    assert (c8 == last_cycle % 256).all()
    en = np.zeros(n_lanes, dtype=np.int64)
    for c in range(last_cycle):
        en += _ref.pi_lanes_np(seed, 1, c, n_lanes, lane_offset)[0]
    c6 = (outputs_bits[:, 24:30].astype(np.int64) << np.arange(6)).sum(1)
    assert (c6 == en % 64).all()


def sampled_lane_check(nl, r, sample_local, lane_offset, cycles, seed, trace_words):
    o = oracle.simulate(nl, sample_local + lane_offset, cycles, seed=seed)
    tb = gpu_trace_bits(r["trace"], None)                  # [ntw*64][c][po]
    pos = {w: i for i, w in enumerate(trace_words)}
    rows = np.array([pos[s // 64] * 64 + s % 64 for s in sample_local])
    assert np.array_equal(tb[rows], o["trace"])
    assert np.array_equal(lane_bits(r["regs"], sample_local), o["regs"])
    assert np.array_equal(r["sigs"][sample_local], o["sig"])


def trace_lane_bits(tr, trace_words, lanes_local):
    """GPU trace [cycles][po][ntw] uint64 -> bits [len(lanes_local)][cycles][po] of the given
    local lanes (each lane's word must be traced)."""
    pos = {int(w): i for i, w in enumerate(trace_words)}
    cols = np.array([pos[int(s) // 64] for s in lanes_local])
    sh = np.array([int(s) % 64 for s in lanes_local], dtype=np.uint64)
    x = tr[:, :, cols]                                          # [c][po][n]
    bits = ((x >> sh[None, None, :]) & np.uint64(1)).astype(np.uint8)
    return np.transpose(bits, (2, 0, 1))


def full_config_check(nl, r, trace_words, sample_local, lane_offset, cycles, seed):
    """Every output of every cycle (trace), every register bit after the last cycle and the
    per-lane MISR of the sampled lanes against the oracle run on the same global lanes."""
    o = oracle.simulate(nl, np.asarray(sample_local) + lane_offset, cycles, seed=seed)
    got = trace_lane_bits(r["trace"], trace_words, sample_local)
    assert got.shape == o["trace"].shape
    bad = np.argwhere(got != o["trace"])
    assert len(bad) == 0, f"{len(bad)} output bits differ, first (lane, cycle, po) {bad[:3].tolist()}"
    assert np.array_equal(lane_bits(r["regs"], sample_local), o["regs"])
    assert np.array_equal(r["sigs"][sample_local], o["sig"])
    return o


@pytest.mark.slow
def test_c3_full_config_all_lanes_prefix_and_probes():
    """C3 (BASELINE configs[2]) at full size: ALL 16,384 lanes, every output of every cycle,
    registers and per-lane MISR vs the oracle over a 50-cycle prefix (SURVEY §8(c) "all lanes
    on C1-C3"); the 1,000-cycle run is checked on 256 lanes below."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    W_ = cfg.lanes // 64
    cycles = 50
    r = run_gpu(nl, cfg.lanes, cycles, "lut", seed=cfg.stim_seed, trace_words=range(W_))
    o = oracle.simulate(nl, np.arange(cfg.lanes), cycles, seed=cfg.stim_seed)
    assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"])
    assert np.array_equal(lane_bits(r["regs"], np.arange(cfg.lanes)), o["regs"])
    assert np.array_equal(r["sigs"], o["sig"])
    assert r["signature"]["lane_sig_sum"] == oracle.lane_sig_sum(o["sig"], np.arange(cfg.lanes))


@pytest.mark.slow
def test_c3_full_config_256_lanes_every_cycle_and_probes():
    """C3 for all 1,000 cycles in the bench's launch configuration: 256 lanes (64 words, the
    lane-group boundaries included) every cycle vs the oracle, probes on every lane."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    sample = workloads.sample_lanes(cfg.lanes, 1, 256, seed=3)
    tw = sorted(set((sample // 64).tolist()))
    r = run_gpu(nl, cfg.lanes, cfg.cycles, "lut", seed=cfg.stim_seed, trace_words=tw)
    full_config_check(nl, r, tw, sample, 0, cfg.cycles, cfg.stim_seed)
    probe_closed_forms(nl, gs.unpack_lanes(r["outputs"]).T, cfg.cycles - 1, cfg.stim_seed, cfg.lanes)
    assert r["signature"]["cycles"] == cfg.cycles


def test_c3_kernel_ab_cross_check_and_poly_parity():
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    a = run_gpu(nl, 4096, 40, "ab", seed=cfg.stim_seed, prog=prog)
    assert a["signature"]["ab_mismatch"] == 0 and a["signature"]["invariant_violations"] == 0
    b = run_gpu(nl, 4096, 40, "poly", seed=cfg.stim_seed, prog=prog)
    c = run_gpu(nl, 4096, 40, "lut", seed=cfg.stim_seed, prog=prog)
    assert np.array_equal(b["sigs"], c["sigs"]) and np.array_equal(b["regs"], c["regs"])
    assert b["signature"]["invariant_violations"] == 0


def test_sharding_and_balance_invariance():
    """lane_sig_sum of P shards (global lane offsets) == 1 shard; levels do not matter."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    full = run_gpu(nl, 8192, 60, "lut", seed=9, prog=prog)
    tot = 0
    for sh in range(4):
        part = run_gpu(nl, 2048, 60, "lut", seed=9, lane_offset=sh * 2048, prog=prog)
        assert np.array_equal(part["sigs"], full["sigs"][sh * 2048:(sh + 1) * 2048])
        tot = (tot + part["signature"]["lane_sig_sum"]) % (1 << 64)
    assert tot == full["signature"]["lane_sig_sum"]
    unbal = run_gpu(nl, 8192, 60, "lut", seed=9, balance=False)
    assert np.array_equal(unbal["sigs"], full["sigs"])


@pytest.mark.parametrize("kernel", ["lut", "tile", "ab"])
def test_sub_batches_by_lane_offset(kernel):
    """One sim re-targeted over 4 lane ranges (gs_sim_set_lane_offset, re-captured graphs)
    == one 4x wider sim: every lane signature and register, and the summed lane_sig_sum;
    the oracle on sampled lanes of every sub-batch."""
    nl = workloads.synthetic(6000, 300, 32, 48, 20, seed=21, name="sub")
    prog = compile_nl(nl)
    cycles, sub = 30, 4096
    full = run_gpu(nl, 4 * sub, cycles, kernel, seed=5, prog=prog)
    sim = gs.Sim(prog, sub, kernel=kernel)
    sim.bind_generated(5)
    tot = 0
    for j in (2, 0, 3, 1):                     # out of order, and back to a used offset
        sim.set_lane_offset(j * sub)
        sim.step(cycles - 7)
        sim.step(7)
        sim.sync()
        sigs, regs = sim.read_lane_signatures(), sim.read_registers()
        assert sim.cycle == cycles
        assert np.array_equal(sigs, full["sigs"][j * sub:(j + 1) * sub])
        assert np.array_equal(regs, full["regs"][:, j * sub // 64:(j + 1) * sub // 64])
        tot = (tot + sim.signature()["lane_sig_sum"]) % (1 << 64)
        pick = np.array([0, 63, 64, sub - 1])
        o = oracle.simulate(nl, pick + j * sub, cycles, seed=5)
        assert np.array_equal(sigs[pick], o["sig"])
    sim.close()
    assert tot == full["signature"]["lane_sig_sum"]
    with pytest.raises(gs.GsError):
        s2 = gs.Sim(prog, sub, kernel=kernel)
        try:
            s2.set_lane_offset(32)
        finally:
            s2.close()


def test_step_granularity_graphs_and_resume():
    nl = workloads.synthetic(20000, 800, 32, 48, 24, seed=12, name="s")
    prog = compile_nl(nl)
    ref = run_gpu(nl, 2048, 50, "lut", seed=3, prog=prog)
    sim = gs.Sim(prog, 2048, use_graphs=False)
    sim.bind_generated(3)
    for _ in range(20):
        sim.step(1)
    regs = sim.read_registers()
    sim.step(30)
    assert np.array_equal(sim.read_registers(), ref["regs"])
    assert np.array_equal(sim.read_lane_signatures(), ref["sigs"])
    sim.close()
    # resume: a fresh sim whose own history diverged (zeroed registers), restored from
    # the checkpoint (registers at cycle 20) -> identical registers and outputs after
    sim2 = gs.Sim(prog, 2048)
    sim2.bind_generated(3)
    sim2.write_registers(np.zeros_like(regs))
    sim2.step(20)
    sim2.write_registers(regs)
    sim2.step(30)
    assert np.array_equal(sim2.read_registers(), ref["regs"])
    assert np.array_equal(sim2.read_outputs(), ref["outputs"])
    sim2.reset()
    sim2.step(50)
    assert np.array_equal(sim2.read_lane_signatures(), ref["sigs"])
    sim2.close()


def test_negative_flipped_truth_table_bit_is_detected():
    """Tests the tests: one flipped truth-table bit in an observed gate must be caught."""
    nl = workloads.synthetic(5000, 200, 32, 48, 16, seed=10, name="s")
    base = nl.n_pi + nl.n_reg
    g = int(nl.po[40]) - base                       # a gate that drives a primary output
    assert g >= 0 and nl.gate_k[g] >= 2
    bad = workloads.Netlist(nl.n_pi, nl.reg_init, nl.reg_d, nl.gate_k, nl.gate_in_off, nl.gate_in,
                            nl.gate_tt.copy(), nl.po, name="bad", meta=nl.meta)
    bad.gate_tt[g] ^= np.uint64(1)                  # f(0,..,0) flipped
    lanes = np.arange(1024)
    r = run_gpu(bad, 1024, 20, "lut", seed=5, trace_words=range(16))
    o = oracle.simulate(nl, lanes, 20, seed=5)
    assert not np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"])
    assert not np.array_equal(r["sigs"], o["sig"])
    # and the flipped design agrees with the oracle run on the same flipped design
    ob = oracle.simulate(bad, lanes, 20, seed=5)
    assert np.array_equal(r["sigs"], ob["sig"])


def test_loaded_program_simulates_identically(tmp_path):
    """A program saved to a file and loaded back runs bit-identically (kernels A and T)."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    f = str(tmp_path / "c3.gsp")
    prog.save(f)
    loaded = gs.Program.load(f)
    for kernel in ("lut", "auto"):
        a = run_gpu(nl, 4096, 15, kernel, seed=3, prog=prog)
        b = run_gpu(nl, 4096, 15, kernel, seed=3, prog=loaded)
        for key in ("outputs", "regs", "sigs"):
            assert np.array_equal(a[key], b[key]), (kernel, key)


def test_errors_on_device():
    prog = compile_nl(workloads.adder(8))
    sim = gs.Sim(prog, 128)
    with pytest.raises(gs.GsError) as e:
        sim.step(1)
    assert e.value.code == gs.GS_ERR_STATE
    sim.bind_host(np.zeros((2, 16, 2), dtype=np.uint64))
    sim.step(2)
    with pytest.raises(gs.GsError) as e:
        sim.step(1)
    assert e.value.code == gs.GS_ERR_STATE
    with pytest.raises(gs.GsError) as e:
        gs._call("gs_sim_read_outputs", sim.h, np.zeros(4, np.uint64).ctypes.data_as(gs.C.c_void_p), 4)
    assert e.value.code == gs.GS_ERR_BUFFER_TOO_SMALL
    sim.close()


@pytest.mark.parametrize("lanes", [8192, 65536])
@pytest.mark.parametrize("flags", [gs.GS_SIM_NO_PDL, gs.GS_SIM_NO_GRID_STRIDE])
def test_launch_options_do_not_change_results(flags, lanes):
    """PDL off, no grid stride: bit-identical (8,192 lanes: one 16-byte vector per thread;
    65,536: four, as on C4)."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    a = run_gpu(nl, lanes, 20, "lut", seed=4, prog=prog)
    b = run_gpu(nl, lanes, 20, "lut", seed=4, prog=prog, flags=flags)
    for key in ("outputs", "regs", "sigs"):
        assert np.array_equal(a[key], b[key]), key


@pytest.mark.parametrize("flags", [2, 4, 64, 128, 256, 1 << 20])
def test_retired_and_unknown_flags_are_rejected(flags):
    """Flag bits retired in 0.2.0 (L2 hints, bulk gathers, global kernel-T slots) and unknown
    bits are argument errors, not silently ignored."""
    prog = compile_nl(workloads.adder(8))
    with pytest.raises(gs.GsError) as e:
        gs.Sim(prog, 1024, flags=flags)
    assert e.value.code == gs.GS_ERR_ARG


# ------------------------------------------------------------------ random valid level assignments
@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("kernel", ["lut", "tile", "poly", "ab"])
def test_random_level_assignments_do_not_change_results(seed, kernel):
    """Any valid level assignment gives the same simulation (R11): seeded random
    levels in [1 + max input level, ALAP] (uneven, sometimes empty levels), every lane and
    register vs the oracle."""
    nl = workloads.synthetic(3000, 120, 20, 32, 16, seed=30 + seed, name="lv")
    prog = gs.Netlist.from_arrays(nl).compile(level_seed=seed)
    lanes, cycles = 8192, 6
    r = run_gpu(nl, lanes, cycles, kernel, seed=seed, prog=prog)
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=seed, want=("last", "regs", "sig"))
    assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"])
    assert np.array_equal(gs.unpack_lanes(r["regs"]).T, o["regs"])
    assert np.array_equal(r["sigs"], o["sig"])
    assert r["signature"]["ab_mismatch"] == 0


# ------------------------------------------------------------------ degenerate netlists
def _degenerate_netlists():
    B = W.Builder
    out = {}
    b = B()                                  # no gates at all: PIs and registers straight to POs
    p0, p1 = b.pi(), b.pi()
    r = b.reg(1)
    b.set_d(r, p1)
    b.out(p0), b.out(r), b.out(p0)           # an output listed twice
    out["no_gates"] = b.build("no_gates")
    b = B()                                  # no PIs: a free-running 3-bit counter
    q = [b.reg(0) for _ in range(3)]
    t0 = b.gate(0b01, q[0])                                  # NOT
    c1 = b.gate(0b0110, q[0], q[1])                          # XOR
    a01 = b.gate(0b1000, q[0], q[1])
    c2 = b.gate(0b0110, a01, q[2])
    for r_, d in zip(q, (t0, c1, c2)):
        b.set_d(r_, d)
    for r_ in q:
        b.out(r_)
    out["no_pis"] = b.build("no_pis")
    b = B()                                  # only constant (k = 0) gates and a 1-input buffer
    p0 = b.pi()
    c0, c1 = b.gate(0), b.gate(1)
    buf = b.gate(0b10, p0)
    b.out(c0), b.out(c1), b.out(buf)
    out["consts"] = b.build("consts")
    b = B()                                  # registers only, no outputs observed except one
    r1, r2 = b.reg(1), b.reg(0)
    b.set_d(r1, r2), b.set_d(r2, r1)
    b.out(r1)
    out["swap_only"] = b.build("swap_only")
    return out


@pytest.mark.parametrize("name", ["no_gates", "no_pis", "consts", "swap_only"])
@pytest.mark.parametrize("kernel", ["auto", "lut", "poly", "ab", "tile"])
def test_degenerate_netlists_every_kernel(name, kernel):
    """Degenerate circuits (no gates, no primary inputs, only constant LUTs, registers only)
    on every kernel, every lane and register vs the oracle; step(0) is a no-op."""
    nl = _degenerate_netlists()[name]
    prog = compile_nl(nl)
    lanes, cycles = 256, 5
    sim = gs.Sim(prog, lanes, kernel=kernel)
    sim.bind_generated(17)
    sim.step(0)
    assert sim.cycle == 0
    sim.step(cycles)
    sim.sync()
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=17, want=("last", "regs", "sig"))
    assert np.array_equal(gs.unpack_lanes(sim.read_outputs()).T, o["last"])
    if nl.n_reg:
        assert np.array_equal(gs.unpack_lanes(sim.read_registers()).T, o["regs"])
    assert np.array_equal(sim.read_lane_signatures(), o["sig"])
    assert sim.signature()["cycles"] == cycles
    sim.close()


# ------------------------------------------------------------------ kernel A, concurrent lane groups
@pytest.mark.parametrize("groups,lanes,graphs", [(2, 8192, True), (4, 16384, True), (3, 12288, True),
                                                 (2, 8192, False), (8, 32768, True), (6, 24576, False)])
def test_lane_groups_every_lane_vs_oracle(groups, lanes, graphs):
    """Lane groups (each group's level chain a concurrent graph branch / stream): a sequential
    netlist with fused latches and Q-bank inputs, every lane, every cycle's trace of sampled
    words, registers and signatures vs the oracle; identical to the single-chain run."""
    nl = workloads.synthetic(3000, 120, 20, 32, 16, seed=22, name="groups")
    prog = compile_nl(nl)
    cycles = 9
    W_ = lanes // 64
    tw = [0, W_ // groups - 1, W_ // groups, W_ - 1]           # group boundaries
    r = run_gpu(nl, lanes, cycles, "lut", seed=3, prog=prog, lane_groups=groups, use_graphs=graphs,
                trace_words=tw, lane_offset=64 * 77)
    o = oracle.simulate(nl, np.arange(lanes) + 64 * 77, cycles, seed=3)
    assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"])
    assert np.array_equal(gs.unpack_lanes(r["regs"]).T, o["regs"])
    assert np.array_equal(r["sigs"], o["sig"])
    tb = gpu_trace_bits(r["trace"], None)
    sel = np.concatenate([np.arange(64) + 64 * w for w in tw])
    assert np.array_equal(tb, o["trace"][sel])
    b = run_gpu(nl, lanes, cycles, "lut", seed=3, prog=prog, lane_groups=1, lane_offset=64 * 77)
    for key in ("outputs", "regs", "sigs"):
        assert np.array_equal(r[key], b[key]), key


def test_lane_groups_reject_bad_shapes():
    nl = workloads.synthetic(2000, 60, 8, 32, 8, seed=2, name="g")
    prog = compile_nl(nl)
    for kw in (dict(lanes=8192, lane_groups=3), dict(lanes=4096, lane_groups=2),
               dict(lanes=8192, lane_groups=2, kernel="poly")):
        kernel = kw.pop("kernel", "lut")
        with pytest.raises(gs.GsError) as e:
            gs.Sim(prog, kernel=kernel, **kw)
        assert e.value.code == gs.GS_ERR_ARG


# ------------------------------------------------------------------ kernel C (cluster slabs)
@pytest.mark.parametrize("cs,slab,lanes", [(1, 128, 4096), (2, 256, 8192), (4, 512, 16384), (2, 128, 2048),
                                            (8, 256, 8192), (2, 1024, 16384)])
def test_cluster_kernel_every_lane_vs_oracle(cs, slab, lanes):
    """Kernel C (a thread-block cluster owns a lane slab and walks every level of every cycle
    of the step, cluster barrier between levels): a sequential netlist with fused latches, Q
    inputs, 5-6-input LUTs and leftover latches; every lane's outputs, registers, signature
    and the trace of boundary words vs the oracle; steps split over several launches; a lane
    offset; identical to kernel A."""
    nls = [workloads.synthetic(3000, 120, 20, 32, 16, seed=23, name="cl"),
           workloads.random_tiny(5, n_pi=6, n_reg=5, n_gates=300, n_po=12, max_k=6),
           workloads.register_edge_cases()]
    for nl in nls:
        prog = compile_nl(nl)
        W_ = lanes // 64
        tw = [0, slab // 64 - 1, slab // 64, W_ - 1]
        sim = gs.Sim(prog, lanes, kernel="cluster", cluster_size=cs, slab_lanes=slab, trace_words=tw,
                     trace_cycles=11, lane_offset=64 * 31)
        sim.bind_generated(8)
        for n in (1, 3, 7):
            sim.step(n)
        sim.sync()
        o = oracle.simulate(nl, np.arange(lanes) + 64 * 31, 11, seed=8)
        assert np.array_equal(gs.unpack_lanes(sim.read_outputs()).T, o["last"])
        assert np.array_equal(gs.unpack_lanes(sim.read_registers()).T, o["regs"])
        assert np.array_equal(sim.read_lane_signatures(), o["sig"])
        sel = np.concatenate([np.arange(64) + 64 * w for w in tw])
        assert np.array_equal(gpu_trace_bits(sim.read_trace(), None), o["trace"][sel])
        sig = sim.signature()
        assert sig["cycles"] == 11 and sig["out_popcount"] == int(o["trace"].sum())
        sim.close()


def test_cluster_kernel_c3_equals_lut_and_streamed_io():
    """Kernel C on C3 (100k gates, 4k registers) at 16,384 lanes == kernel A on every lane;
    and gs_sim_run_streamed (host stimuli in, every output out) through kernel C == kernel A."""
    cfg = workloads.CONFIGS["C3"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    c = run_gpu(nl, cfg.lanes, 30, "cluster", seed=3, prog=prog)
    a = run_gpu(nl, cfg.lanes, 30, "lut", seed=3, prog=prog)
    for key in ("outputs", "regs", "sigs"):
        assert np.array_equal(c[key], a[key]), key
    assert c["signature"]["lane_sig_sum"] == a["signature"]["lane_sig_sum"]
    assert c["signature"]["out_popcount"] == a["signature"]["out_popcount"]
    W_ = 4096 // 64
    stim = workloads.random_host_stimulus(9, 12, nl.n_pi, W_)
    outs = []
    for kernel in ("cluster", "lut"):
        sim = gs.Sim(prog, 4096, kernel=kernel)
        out = np.zeros((12, nl.n_po, W_), dtype=np.uint64)
        sim.run_streamed(stim, out, chunk=5)
        sim.sync()
        outs.append((out, sim.read_lane_signatures()))
        sim.close()
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


def test_cluster_kernel_rejects_bad_shapes():
    prog = compile_nl(workloads.adder(8))
    for kw in (dict(slab_lanes=192), dict(slab_lanes=384), dict(slab_lanes=2048), dict(cluster_size=3)):
        with pytest.raises(gs.GsError) as e:
            gs.Sim(prog, 1024, kernel="cluster", **kw)
        assert e.value.code == gs.GS_ERR_ARG


# ------------------------------------------------------------------ cone collapsing (lut_k)
@pytest.mark.parametrize("L", [3, 6])
@pytest.mark.parametrize("kernel", ["lut", "poly", "ab", "tile"])
def test_collapsed_program_equals_oracle_of_original_netlist(kernel, L):
    """Programs compiled with lut_k = L (wider LUTs, fewer levels) vs the oracle run on the
    ORIGINAL netlist: every lane, every cycle."""
    nls = [workloads.adder(8), workloads.random_tiny(4, n_pi=6, n_reg=5, n_gates=300, n_po=12),
           workloads.synthetic(3000, 120, 16, 40, 12, seed=9, name="s")]
    for nl in nls:
        prog = gs.Netlist.from_arrays(nl).compile(lut_k=L)
        r = run_gpu(nl, 4096, 7, kernel, seed=23, prog=prog, trace_words=[0, 40, 63])
        o = oracle.simulate(nl, np.arange(4096), 7, seed=23)
        assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"])
        assert np.array_equal(gs.unpack_lanes(r["regs"]).T, o["regs"])
        assert np.array_equal(r["sigs"], o["sig"])
        rows = np.concatenate([np.arange(0, 64), np.arange(40 * 64, 41 * 64), np.arange(63 * 64, 64 * 64)])
        assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"][rows])
        assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0


def test_collapsed_multiplier_all_lanes_equal_a_times_b():
    cfg = workloads.CONFIGS["C2"]
    nl = cfg.netlist()
    prog = gs.Netlist.from_arrays(nl).compile(lut_k=6)
    assert prog.info["n_levels"] <= 92
    r = run_gpu(nl, cfg.lanes, 1, "auto", seed=cfg.stim_seed, prog=prog)
    bits = gs.unpack_lanes(r["outputs"]).astype(np.uint64)
    prod = (bits << np.arange(64, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    pis = _ref.pi_lanes_np(cfg.stim_seed, 64, 0, cfg.lanes).astype(np.uint64)
    x = (pis[:32] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    y = (pis[32:] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    assert np.array_equal(prod, x * y)


# ------------------------------------------------------------------ 7-8-input LUTs (kernel B)
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_wide_luts_every_kernel_all_lanes_vs_oracle(seed):
    """Gates with k = 7, 8 (256-bit tables): kernel B with up to 256 sparse terms per gate,
    kernels A / T by Shannon expansion over the 64-bit sub-tables."""
    nl = workloads.random_tiny(seed, n_pi=8, n_reg=6, n_gates=250, n_po=14, max_k=8)
    assert (nl.gate_k > 6).any()
    prog = compile_nl(nl)
    for kernel in ("poly", "auto", "lut", "ab", "tile"):
        r = run_gpu(nl, 4096, 9, kernel, seed=31, prog=prog, trace_words=[0, 17, 63])
        o = oracle.simulate(nl, np.arange(4096), 9, seed=31)
        assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"])
        assert np.array_equal(gs.unpack_lanes(r["regs"]).T, o["regs"])
        assert np.array_equal(r["sigs"], o["sig"])
        rows = np.concatenate([np.arange(0, 64), np.arange(17 * 64, 18 * 64), np.arange(63 * 64, 64 * 64)])
        assert np.array_equal(gpu_trace_bits(r["trace"], None), o["trace"][rows])
        assert r["signature"]["invariant_violations"] == 0 and r["signature"]["ab_mismatch"] == 0


@pytest.mark.parametrize("L", [7, 8])
def test_collapsed_to_8_input_luts_closed_forms(L):
    """The paper's L = 7 regime: the adder and the multiplier collapsed into <= L-input
    LUTs and run on kernel B still give a+b (exhaustively) and a*b (1M lanes)."""
    nl = workloads.adder(8)
    prog = gs.Netlist.from_arrays(nl).compile(lut_k=L)
    a = np.arange(1 << 16) & 0xFF
    b = np.arange(1 << 16) >> 8
    bits = np.concatenate([(a[None, :] >> np.arange(8)[:, None]) & 1,
                           (b[None, :] >> np.arange(8)[:, None]) & 1]).astype(np.uint8)
    words = np.packbits(bits, axis=1, bitorder="little").view(np.uint64)[None]
    e = run_gpu(nl, 1 << 16, 1, "auto", host_stim=words, prog=prog)
    out = gs.unpack_lanes(e["outputs"]).astype(np.int64)
    assert np.array_equal((out << np.arange(9)[:, None]).sum(0), a + b)
    cfg = workloads.CONFIGS["C2"]
    prog = gs.Netlist.from_arrays(cfg.netlist()).compile(lut_k=L)
    r = run_gpu(cfg.netlist(), cfg.lanes, 1, "auto", seed=cfg.stim_seed, prog=prog)
    assert r["signature"]["invariant_violations"] == 0
    bits = gs.unpack_lanes(r["outputs"]).astype(np.uint64)
    prod = (bits << np.arange(64, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    pis = _ref.pi_lanes_np(cfg.stim_seed, 64, 0, cfg.lanes).astype(np.uint64)
    x = (pis[:32] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    y = (pis[32:] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    assert np.array_equal(prod, x * y)


# ------------------------------------------------------------------ streamed host I/O (f3)
@pytest.mark.parametrize("kernel,chunk,lanes", [("lut", 4, 2048), ("lut", 0, 2048), ("tile", 7, 2048),
                                               ("poly", 5, 2048), ("lut", 6, 16384)])   # 16,384: 4 lane groups
def test_run_streamed_every_output_every_cycle_vs_oracle(kernel, chunk, lanes):
    """gs_sim_run_streamed: host stimuli in, EVERY output of EVERY cycle out (paper P:271),
    chunks pipelined on a copy stream; compared with the oracle on every lane and cycle."""
    import torch
    nl = workloads.random_tiny(8, n_pi=7, n_reg=6, n_gates=400, n_po=20, max_k=4)
    prog = compile_nl(nl)
    cycles = 30
    W_ = lanes // 64
    stim = workloads.random_host_stimulus(5, cycles, nl.n_pi, W_)
    pin_in = torch.from_numpy(stim.view(np.int64)).pin_memory()
    pin_out = torch.zeros((cycles, nl.n_po, W_), dtype=torch.int64).pin_memory()
    sim = gs.Sim(prog, lanes, kernel=kernel)
    sim.run_streamed(pin_in.numpy().view(np.uint64), pin_out.numpy().view(np.uint64), chunk=chunk)
    sim.sync()
    out = pin_out.numpy().view(np.uint64)
    o = oracle.simulate(nl, np.arange(lanes), cycles, host_stim=stim)
    bits = gs.unpack_lanes(out)                               # [c][po][lanes]
    assert np.array_equal(np.transpose(bits, (2, 0, 1)), o["trace"])
    assert np.array_equal(sim.read_lane_signatures(), o["sig"])
    assert np.array_equal(gs.unpack_lanes(sim.read_registers()).T, o["regs"])
    # a second streamed run continues from the registers (cycle 30..59)
    stim2 = workloads.random_host_stimulus(6, cycles, nl.n_pi, W_)
    sim.run_streamed(np.ascontiguousarray(stim2), None, chunk=chunk)
    sim.sync()
    both = np.concatenate([stim, stim2])
    o2 = oracle.simulate(nl, np.arange(lanes), 2 * cycles, host_stim=both, want=("regs", "sig"))
    assert np.array_equal(sim.read_lane_signatures(), o2["sig"])
    sim.close()


# ------------------------------------------------------------------ kernel T (tile-resident)
@pytest.mark.parametrize("tw", [0, 4, 8, 16, 32])
def test_tile_adder_all_lanes_and_exhaustive(tw):
    cfg = workloads.CONFIGS["C1"]
    nl = cfg.netlist()
    r = run_gpu(nl, cfg.lanes, 1, "tile", seed=cfg.stim_seed, tile_words=tw)
    o = oracle.simulate(nl, np.arange(cfg.lanes), 1, seed=cfg.stim_seed)
    assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"])
    assert np.array_equal(r["sigs"], o["sig"])
    # exhaustive 2^16 inputs through host-bound stimuli
    a = np.arange(1 << 16) & 0xFF
    b = np.arange(1 << 16) >> 8
    bits = np.concatenate([(a[None, :] >> np.arange(8)[:, None]) & 1,
                           (b[None, :] >> np.arange(8)[:, None]) & 1]).astype(np.uint8)
    words = np.packbits(bits, axis=1, bitorder="little").view(np.uint64)[None]
    e = run_gpu(nl, 1 << 16, 1, "tile", host_stim=words, tile_words=tw)
    out = gs.unpack_lanes(e["outputs"]).astype(np.int64)
    assert np.array_equal((out << np.arange(9)[:, None]).sum(0), a + b)


@pytest.mark.parametrize("balance", [False, True])
def test_tile_tiny_wide_gates_registers_all_lanes_step_split(balance):
    """k up to 6, register edge cases; cycles split over several gs_sim_step calls."""
    nls = [workloads.random_tiny(s, n_pi=6, n_reg=5, n_gates=300, n_po=12, max_k=6) for s in (5, 6)]
    nls += [workloads.register_edge_cases(), workloads.probes_circuit()]
    for nl in nls:
        prog = compile_nl(nl, balance)
        sim = gs.Sim(prog, 2048, kernel="tile", trace_words=[0, 7, 31], trace_cycles=11)
        sim.bind_generated(13)
        for n in (1, 3, 7):
            sim.step(n)
        o = oracle.simulate(nl, np.arange(2048), 11, seed=13)
        assert np.array_equal(gs.unpack_lanes(sim.read_outputs()).T, o["last"])
        assert np.array_equal(gs.unpack_lanes(sim.read_registers()).T, o["regs"])
        assert np.array_equal(sim.read_lane_signatures(), o["sig"])
        tb = gpu_trace_bits(sim.read_trace(), None)
        rows = np.concatenate([np.arange(0, 64), np.arange(7 * 64, 8 * 64), np.arange(31 * 64, 32 * 64)])
        assert np.array_equal(tb, o["trace"][rows])
        sig = sim.signature()
        assert sig["cycles"] == 11
        assert sig["out_popcount"] == int(o["trace"].sum())
        sim.close()


def test_tile_c2_multiplier_all_lanes_equals_lut():
    cfg = workloads.CONFIGS["C2"]
    nl = cfg.netlist()
    prog = compile_nl(nl)
    t = run_gpu(nl, cfg.lanes, 2, "tile", seed=cfg.stim_seed, prog=prog)
    a = run_gpu(nl, cfg.lanes, 2, "lut", seed=cfg.stim_seed, prog=prog)
    assert np.array_equal(t["outputs"], a["outputs"]) and np.array_equal(t["sigs"], a["sigs"])
    bits = gs.unpack_lanes(t["outputs"]).astype(np.uint64)        # [64][lanes], last cycle = 1
    prod = (bits << np.arange(64, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    from tests._ref import pi_lanes_np
    pis = pi_lanes_np(cfg.stim_seed, 64, 1, cfg.lanes, 0).astype(np.uint64)
    x = (pis[:32] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    y = (pis[32:] << np.arange(32, dtype=np.uint64)[:, None]).sum(0, dtype=np.uint64)
    assert np.array_equal(prod, x * y)


@pytest.mark.parametrize("tw,ng", [(0, 0), (4, 1), (4, 2), (8, 1)])
def test_tile_sequential_synthetic_all_lanes_probes_resume(tw, ng):
    """8k-gate sequential synthetic netlist (C3 recipe, smaller): every lane vs the oracle."""
    nl = workloads.synthetic(8000, 300, 32, 48, 24, seed=21, name="t8k")
    prog = compile_nl(nl)
    lanes, cycles = 4096, 40
    t = run_gpu(nl, lanes, cycles, "tile", seed=5, prog=prog, trace_words=[0, 33, 63], tile_words=tw,
                tile_groups=ng)
    a = run_gpu(nl, lanes, cycles, "lut", seed=5, prog=prog)
    for key in ("outputs", "regs", "sigs"):
        assert np.array_equal(t[key], a[key]), key
    assert t["signature"]["out_popcount"] == a["signature"]["out_popcount"]
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=5, want=("last", "regs", "sig"))
    assert np.array_equal(t["sigs"], o["sig"])
    assert np.array_equal(gs.unpack_lanes(t["regs"]).T, o["regs"])
    probe_closed_forms(nl, gs.unpack_lanes(t["outputs"]).T, cycles - 1, 5, lanes)
    # resume through register write-back
    sim = gs.Sim(prog, lanes, kernel="tile", tile_words=tw, tile_groups=ng)
    sim.bind_generated(5)
    sim.step(13)
    regs = sim.read_registers()
    sim.write_registers(np.zeros_like(regs))
    sim.write_registers(regs)
    sim.step(cycles - 13)
    assert np.array_equal(sim.read_registers(), a["regs"])
    assert np.array_equal(sim.read_lane_signatures(), a["sigs"])
    sim.close()


@pytest.mark.parametrize("flags", [16, 32])
def test_tile_descriptor_sources_global_and_tma_stream(flags):
    """Kernel T with descriptors read from global memory (16) or streamed one level at a time
    by TMA bulk copies into a shared-memory double buffer (32): every lane vs the oracle,
    steps split over several launches (the TMA stream restarts at each tile and step)."""
    nl = workloads.synthetic(8000, 300, 32, 48, 24, seed=21, name="t8k")
    prog = compile_nl(nl)
    lanes = 4096
    sim = gs.Sim(prog, lanes, kernel="tile", flags=flags, trace_words=[0, 31, 63], trace_cycles=20)
    sim.bind_generated(5)
    for n in (1, 6, 13):
        sim.step(n)
    o = oracle.simulate(nl, np.arange(lanes), 20, seed=5)
    assert np.array_equal(sim.read_lane_signatures(), o["sig"])
    assert np.array_equal(gs.unpack_lanes(sim.read_registers()).T, o["regs"])
    assert np.array_equal(gs.unpack_lanes(sim.read_outputs()).T, o["last"])
    rows = np.concatenate([np.arange(0, 64), np.arange(31 * 64, 32 * 64), np.arange(63 * 64, 64 * 64)])
    assert np.array_equal(gpu_trace_bits(sim.read_trace(), None), o["trace"][rows])
    sim.close()


def test_auto_kernel_selection():
    """AUTO = kernel T (one launch per step) when the circuit fits shared memory, else A."""
    for name, lanes, tile, L in (("C1", 1024, True, 0), ("C2", 1 << 14, True, 0), ("C3", 4096, False, 0),
                                 ("C2", 1 << 14, False, 6)):
        prog = gs.Netlist.from_arrays(workloads.CONFIGS[name].netlist()).compile(lut_k=L)
        sim = gs.Sim(prog, lanes, kernel="auto")
        assert (sim.launches_per_cycle() == 1) == tile, name
        li = sim.launch                                   # gs_sim_get_launch: the resolved plan
        assert li["kernel"] == (gs.GS_KERNEL_TILE if tile else gs.GS_KERNEL_LUT), (name, li)
        if tile:
            assert li["tile_words"] in (4, 8, 16, 32, 64) and li["grid"] >= 1 and li["live_slots"] > 0
            assert li["tile_groups"] in (1, 2, 4) and li["tile_desc"] & 3 in (0, 1, 2)
            assert bool(li["tile_desc"] & 4) == (name in ("C1", "C2") and L == 0)   # narrow: k <= 2, no regs
        else:
            assert li["lane_groups"] == sim.config["lane_groups"] >= 1
        sim.bind_generated(1)
        sim.step(2)
        ref = run_gpu(workloads.CONFIGS[name].netlist(), lanes, 2, "lut", seed=1, prog=prog)
        assert np.array_equal(sim.read_lane_signatures(), ref["sigs"])
        sim.close()


def test_tile_rejects_oversized_or_misaligned():
    prog = compile_nl(workloads.adder(8))
    with pytest.raises(gs.GsError) as e:
        gs.Sim(prog, 1024 + 64, kernel="tile", tile_words=8)
    assert e.value.code == gs.GS_ERR_ARG
    for name in ("C3", "C4"):                     # live state larger than shared memory
        big = compile_nl(workloads.CONFIGS[name].netlist())
        with pytest.raises(gs.GsError) as e:
            gs.Sim(big, 4096, kernel="tile")
        assert e.value.code == gs.GS_ERR_ARG


# ------------------------------------------------------------------ full-size configs
@pytest.mark.slow
def test_c4_full_config_256_lanes_every_cycle_and_probes():
    """C4 (BASELINE configs[3]) at full size in the launch configuration `bench.py --config C4`
    times (65,536 lanes, kernel A, auto = 4 concurrent lane groups, CUDA graphs): 256 lanes
    spread over the batch (lanes 0/63/64/last, both sides of every lane-group boundary) x all
    1,000 cycles vs the oracle — every output bit of every cycle, every register bit, the
    per-lane MISR — and the probes' closed forms on every lane."""
    import bench
    cfg = workloads.CONFIGS["C4"]
    nl = cfg.netlist()
    prog = gs.Netlist.from_arrays(nl).compile(balance=BENCH_BALANCE[bench.AUTO_LEVELS.get("C4", "balanced")])
    sample = workloads.sample_lanes(cfg.lanes, 1, 256, seed=4)
    assert {0, 63, 64, cfg.lanes - 1} <= set(sample.tolist())
    tw = sorted(set((sample // 64).tolist()))
    sim = gs.Sim(prog, cfg.lanes, kernel="lut", trace_words=tw, trace_cycles=cfg.cycles)
    assert sim.config["lane_groups"] == 4
    sim.bind_generated(cfg.stim_seed)
    sim.step(cfg.cycles)
    sim.sync()
    r = dict(outputs=sim.read_outputs(), regs=sim.read_registers(), sigs=sim.read_lane_signatures(),
             trace=sim.read_trace())
    sim.close()
    full_config_check(nl, r, tw, sample, 0, cfg.cycles, cfg.stim_seed)
    probe_closed_forms(nl, gs.unpack_lanes(r["outputs"]).T, cfg.cycles - 1, cfg.stim_seed, cfg.lanes)


@pytest.mark.slow
def test_c5_every_shard_32_lanes_every_cycle_bench_config():
    """C5 (BASELINE configs[4]) at full size over its whole 262,144-lane batch in the launch
    configuration bench.py times (10M gates, sub-batches of bench.DEFAULT_SUB_LANES lanes in
    one workspace re-targeted by gs_sim_set_lane_offset, each from reset, auto lane groups):
    32 lanes of every one of the 8 shards (256 in all, shard- and group-boundary lanes
    included) x all 100 cycles vs the oracle, and the probes on every lane of every shard."""
    import bench
    cfg = workloads.CONFIGS["C5"]
    nl = cfg.netlist()
    prog = gs.Netlist.from_arrays(nl).compile(balance=BENCH_BALANCE[bench.AUTO_LEVELS.get("C5", "balanced")])
    sub = bench.DEFAULT_SUB_LANES
    sample = workloads.sample_lanes(cfg.lanes, cfg.shards, 256 // cfg.shards, seed=5, lanes_per_word=2)
    tw_all = sorted(set((sample % sub // 64).tolist()))        # local words of any sub-batch
    sim = gs.Sim(prog, sub, kernel="lut", trace_words=tw_all, trace_cycles=cfg.cycles)
    sim.bind_generated(cfg.stim_seed)
    o = oracle.simulate(nl, sample, cfg.cycles, seed=cfg.stim_seed)
    tot = 0
    checked = 0
    for j in range(cfg.lanes // sub):
        off = j * sub
        sim.set_lane_offset(off)
        sim.step(cfg.cycles)
        sim.sync()
        m = (sample >= off) & (sample < off + sub)
        loc = sample[m] - off
        got = trace_lane_bits(sim.read_trace(), tw_all, loc)
        assert np.array_equal(got, o["trace"][m]), j
        assert np.array_equal(lane_bits(sim.read_registers(), loc), o["regs"][m]), j
        sigs = sim.read_lane_signatures()
        assert np.array_equal(sigs[loc], o["sig"][m]), j
        probe_closed_forms(nl, gs.unpack_lanes(sim.read_outputs()).T, cfg.cycles - 1, cfg.stim_seed, sub, off)
        tot = (tot + sim.signature()["lane_sig_sum"]) % (1 << 64)
        checked += int(m.sum())
    sim.close()
    assert checked == len(sample) == 256
    assert tot != 0


@pytest.mark.parametrize("gates,groups,depth", [(40000, 1, 8), (40000, 4, 4), (60000, 4, 3), (130000, 4, 6)])
def test_grid_stride_branch_every_lane_vs_oracle(gates, groups, depth):
    """Kernel A's grid-stride launches (a level 1-4 waves of resident CTAs deep runs on
    exactly the resident CTAs, which stride over the level) at 65,536 lanes, with 4 and 16
    vectors per warp unit (U = 4, 2, 1 by level width: ~2.9k gates / 1 group, ~3.6k, 6k, 10k
    gates / 4 groups): every lane vs the oracle, and the branch provably taken
    (gs_profile.grid_stride_launches > 0)."""
    nl = workloads.synthetic(gates, gates // 25, 32, 48, depth, seed=60 + groups, name="gstride")
    prog = compile_nl(nl)
    lanes, cycles = 65536, 2
    sim = gs.Sim(prog, lanes, kernel="lut", lane_groups=groups)
    assert sim.config["lane_groups"] == groups
    sim.bind_generated(6)
    sim.step(cycles - 1)
    pr = sim.profile_step(1)
    assert pr["grid_stride_launches"] > 0, pr
    sim.sync()
    out, regs, sigs = sim.read_outputs(), sim.read_registers(), sim.read_lane_signatures()
    sim.close()
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=6, want=("last", "regs", "sig"))
    assert np.array_equal(gs.unpack_lanes(out).T, o["last"])
    assert np.array_equal(gs.unpack_lanes(regs).T, o["regs"])
    assert np.array_equal(sigs, o["sig"])


@pytest.mark.parametrize("lanes,groups,lut_k", [(4096, 1, 0), (8192, 1, 0), (8192, 2, 0), (4096, 1, 6)])
def test_multi_gate_warp_units_every_lane_vs_oracle(lanes, groups, lut_k):
    """Kernel A on short rows (4,096 lanes per lane group: 4 gates x 1 vector per thread;
    8,192 in one group: 2 gates x 2 vectors): wide levels (~50k gates) with k-group edges
    inside a warp unit, levels whose width is not a multiple of the unit, fused latches, and
    (lut_k = 6, cone-collapsed) k = 5, 6 gates on the one-gate-at-a-time branch: every lane
    vs the oracle of the original netlist, and the branch provably taken."""
    nl = workloads.synthetic(200000, 8000, 32, 48, 4, seed=70 + lanes // 4096 + groups, name="gp")
    prog = gs.Netlist.from_arrays(nl).compile(lut_k=lut_k)
    if lut_k:
        assert sum(prog.info["k_hist"][5:]) > 0
    cycles = 3
    sim = gs.Sim(prog, lanes, kernel="lut", lane_groups=groups)
    assert sim.config["lane_groups"] == groups
    sim.bind_generated(7)
    sim.step(cycles - 1)
    pr = sim.profile_step(1)
    assert pr["multi_gate_launches"] > 0, pr
    sim.sync()
    out, regs, sigs = sim.read_outputs(), sim.read_registers(), sim.read_lane_signatures()
    sim.close()
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=7, want=("last", "regs", "sig"))
    assert np.array_equal(gs.unpack_lanes(out).T, o["last"])
    assert np.array_equal(gs.unpack_lanes(regs).T, o["regs"])
    assert np.array_equal(sigs, o["sig"])


@pytest.mark.parametrize("slab,min_gates,balance,groups",
                         [(4096, 10000, False, 1), (8192, 1, True, 1), (4096, 1, False, 1), (4096, 10000, False, 2)])
def test_slab_schedule_every_lane_vs_oracle(slab, min_gates, balance, groups):
    """Kernel A's segmented slab schedule: runs of levels >= min_gates wide go slab after slab
    (4,096-lane slabs take the multi-gate units), the other levels over all lanes of the lane
    group (16,384 lanes, 1 or 2 concurrent groups); every lane vs the oracle, and the same
    lane_sig_sum as the plain schedule."""
    nl = workloads.synthetic(200000, 8000, 32, 48, 4, seed=80 + slab // 4096, name="slab")
    prog = compile_nl(nl, balance)
    lanes, cycles = 16384, 3
    sim = gs.Sim(prog, lanes, kernel="lut", slab_lanes=slab, slab_min_gates=min_gates, lane_groups=groups)
    assert sim.launch["slab_lanes"] == slab and sim.config["lane_groups"] == groups
    widths = prog.level_widths()
    wide = int((widths >= min_gates).sum())
    assert 0 < wide
    per_cycle = sim.launches_per_cycle()
    assert per_cycle == 2 + groups * ((len(widths) - wide) + wide * (lanes // groups // slab))
    sim.bind_generated(8)
    sim.step(cycles - 1)
    pr = sim.profile_step(1)
    assert pr["level_launches"] == per_cycle - 2
    sim.sync()
    out, regs, sigs = sim.read_outputs(), sim.read_registers(), sim.read_lane_signatures()
    sig = sim.signature()
    sim.close()
    o = oracle.simulate(nl, np.arange(lanes), cycles, seed=8, want=("last", "regs", "sig"))
    assert np.array_equal(gs.unpack_lanes(out).T, o["last"])
    assert np.array_equal(gs.unpack_lanes(regs).T, o["regs"])
    assert np.array_equal(sigs, o["sig"])
    assert sig["lane_sig_sum"] == run_gpu(nl, lanes, cycles, seed=8, prog=prog)["signature"]["lane_sig_sum"]


def test_slab_schedule_bad_shapes_rejected():
    nl = workloads.synthetic(3000, 100, 16, 48, 4, seed=81, name="slabbad")
    prog = compile_nl(nl)
    for kw in (dict(slab_lanes=2048), dict(slab_lanes=12288), dict(slab_lanes=8192, lane_groups=4)):
        with pytest.raises(gs.GsError):
            gs.Sim(prog, 16384, kernel="lut", **kw)


# ------------------------------------------------------------------ seeded fuzzing
def _fuzz_netlist(rng, case):
    """Random sequential netlist: sizes, fan-in mix (k = 0..6, repeated inputs allowed),
    registers fed by gates / PIs / Qs, outputs on any net."""
    n_pi = int(rng.integers(1, 20))
    n_reg = int(rng.integers(0, 30))
    n_gates = int(rng.integers(5, 1500))
    n_po = int(rng.integers(1, 80))
    max_k = int(rng.integers(1, 9))
    return workloads.random_tiny(int(rng.integers(0, 2**31)), n_pi=n_pi, n_reg=n_reg, n_gates=n_gates,
                                 n_po=n_po, max_k=max_k)


@pytest.mark.parametrize("case", range(int(os.environ.get("GS_FUZZ_CASES", "32"))))
def test_fuzz_every_kernel_all_lanes_vs_oracle(case):
    """Seeded random netlists through every kernel / schedule / compile option, every lane and
    cycle against the oracle (outputs of the last cycle, registers, per-lane signatures)."""
    rng = np.random.default_rng(1000 + case)
    nl = _fuzz_netlist(rng, case)
    lanes = int(rng.choice([64, 192, 128, 256, 1024, 4096, 8192]))
    offset = 64 * int(rng.integers(0, 1000))              # global lane of local lane 0
    cycles = int(rng.integers(1, 12))
    seed = int(rng.integers(0, 2**40))
    balance = bool(rng.integers(0, 2))
    lut_k = int(rng.choice([0, 0, 3, 4, 6, 8]))
    prog = gs.Netlist.from_arrays(nl).compile(balance=balance, lut_k=lut_k)
    o = oracle.simulate(nl, np.arange(lanes) + offset, cycles, seed=seed, want=("last", "regs", "sig"))
    kernels = ["lut", "poly", "ab", "auto"] + (["tile", "cluster"] if lanes % 128 == 0 else [])
    runs = [(k, {}) if k != "cluster" else (k, dict(slab_lanes=128, cluster_size=[1, 2, 4][case % 3]))
            for k in kernels]
    # opt-in launch options: one pick per case for kernel A, one descriptor source for T
    opt = [dict(flags=gs.GS_SIM_NO_PDL), dict(flags=gs.GS_SIM_NO_GRID_STRIDE), dict(lane_groups=1),
           dict(lane_groups=2)][case % 4]
    if "lane_groups" in opt and (lanes // 128) % max(opt["lane_groups"], 1) or lanes < 8192:
        opt = dict(flags=gs.GS_SIM_NO_PDL)
    runs.append(("lut", opt))
    if lanes % 128 == 0:
        runs.append(("tile", dict(flags=[gs.GS_SIM_TILE_DESC_GLOBAL, gs.GS_SIM_TILE_DESC_TMA][case % 2])))
    for kernel, kw in runs:
        try:
            r = run_gpu(nl, lanes, cycles, kernel, seed=seed, prog=prog, lane_offset=offset, **kw)
        except gs.GsError as e:           # a forced descriptor source the plan cannot hold
            if kernel == "tile" and kw and e.code == gs.GS_ERR_ARG:
                continue
            raise
        tag = f"{kernel} {kw}"
        assert np.array_equal(gs.unpack_lanes(r["outputs"]).T, o["last"]), tag
        assert np.array_equal(gs.unpack_lanes(r["regs"]).T, o["regs"]), tag
        assert np.array_equal(r["sigs"], o["sig"]), tag
        assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0


# ------------------------------------------------------------------ AES-128 core (FIPS-197)
@pytest.mark.parametrize("kernel", ["auto", "lut", "tile", "poly", "ab"])
def test_aes128_core_every_lane(kernel):
    """A real circuit of the paper's Table I family: the iterative AES-128 core (8-input S-box
    LUTs, 260 registers).  Ciphertexts on every lane equal the oracle's, the first 256 equal an
    independent textbook AES, lane 0 is FIPS-197 Appendix C.1."""
    from workloads import aes
    from tests import _aes_ref
    nl = aes.aes128_core()
    prog = compile_nl(nl)
    lanes = 4096
    rng = np.random.default_rng(11)
    keys = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    pts = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    keys[0] = np.frombuffer(bytes.fromhex("000102030405060708090a0b0c0d0e0f"), dtype=np.uint8)
    pts[0] = np.frombuffer(bytes.fromhex("00112233445566778899aabbccddeeff"), dtype=np.uint8)
    stim = aes.aes_stimulus(keys, pts)
    r = run_gpu(nl, lanes, 12, kernel, host_stim=stim, prog=prog)
    ct = aes.ciphertexts(gs.unpack_lanes(r["outputs"]).T)
    assert bytes(ct[0]).hex() == "69c4e0d86a7b0430d8cdb78070b4c55a"
    o = oracle.simulate(nl, np.arange(lanes), 12, host_stim=stim, want=("last", "sig"))
    assert np.array_equal(ct, aes.ciphertexts(o["last"]))
    assert np.array_equal(r["sigs"], o["sig"])
    for s in range(256):
        assert bytes(ct[s]) == _aes_ref.encrypt(bytes(keys[s]), bytes(pts[s]))
    assert r["signature"]["ab_mismatch"] == 0 and r["signature"]["invariant_violations"] == 0


@pytest.mark.parametrize("kernel", ["lut", "tile"])
def test_stimulus_hash_cuda_equals_python_every_word(kernel):
    """The device counter hash (reading R2) against the independent Python implementation
    (tests/_ref.py), word by word: primary outputs wired straight to the primary inputs,
    every word of every cycle recorded by the trace; lane offset != 0."""
    b = W.Builder()
    pis = [b.pi() for _ in range(20)]
    for p in pis:
        b.out(p)
    b.out(b.gate(W.NOT, pis[0]))
    nl = b.build("pi_to_po")
    lanes, cycles, offset, seed = 2048, 5, 64 * 777, 0xC0FFEE
    W_ = lanes // 64
    r = run_gpu(nl, lanes, cycles, kernel, seed=seed, trace_words=list(range(W_)), lane_offset=offset)
    tr = r["trace"]                                        # [cycle][po][word]
    words = np.arange(offset // 64, offset // 64 + W_, dtype=np.uint64)
    for c in range(cycles):
        for p in range(20):
            assert np.array_equal(tr[c, p], _ref.stim_words_np(seed, p, c, words)), (c, p)
        assert np.array_equal(tr[c, 20], ~_ref.stim_words_np(seed, 0, c, words))
