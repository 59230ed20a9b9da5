#!/usr/bin/env python
"""AES-128 encryptions per second with the iterative AES core netlist (workloads/aes.py):
every lane encrypts its own block (load cycle + 10 round cycles = 11 cycles per block),
stimuli streamed from pinned host memory and every output of every cycle streamed back
(gs_sim_run_streamed), per kernel and per L (cone collapsing).  Lane 0 checks FIPS-197 C.1."""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from workloads import aes
    import paper_conf_ipps_gavierrprs23_b200 as gs
    nl = aes.aes128_core()
    lanes = 1 << 20
    rng = np.random.default_rng(3)
    keys = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    pts = rng.integers(0, 256, size=(lanes, 16), dtype=np.uint8)
    keys[0] = np.frombuffer(bytes.fromhex("000102030405060708090a0b0c0d0e0f"), dtype=np.uint8)
    pts[0] = np.frombuffer(bytes.fromhex("00112233445566778899aabbccddeeff"), dtype=np.uint8)
    stim = aes.aes_stimulus(keys, pts, cycles=11)
    pin = torch.from_numpy(stim.view(np.int64)).pin_memory().numpy().view(np.uint64)
    out = torch.zeros((11, 128, lanes // 64), dtype=torch.int64).pin_memory().numpy().view(np.uint64)
    for L in (0, 6, 8):
        prog = gs.Netlist.from_arrays(nl).compile(lut_k=L)
        for kernel in ("lut", "tile", "auto"):
            try:
                sim = gs.Sim(prog, lanes, kernel=kernel)
            except gs.GsError as e:
                print(json.dumps({"L": L, "kernel": kernel, "error": str(e)}), flush=True)
                continue
            sim.run_streamed(pin, out)
            sim.sync()
            assert bytes(aes.ciphertexts(gs.unpack_lanes(sim.read_registers()[:128]).T)[0]).hex() == \
                "69c4e0d86a7b0430d8cdb78070b4c55a"
            reps = 5
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sim.stream)
            for _ in range(reps):
                sim.reset()
                sim.run_streamed(pin, out)
            e1.record(sim.stream)
            torch.cuda.synchronize()
            s = e0.elapsed_time(e1) / 1e3 / reps
            # device-resident: the stimuli already in HBM (gs_sim_bind_stimulus_device)
            dev = torch.from_numpy(stim.view(np.int64)).to(sim.device)
            d0, d1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            d0.record(sim.stream)
            for _ in range(reps):
                sim.reset()
                sim.bind_device(dev, 11)
                sim.step(11)
            d1.record(sim.stream)
            torch.cuda.synchronize()
            sd = d0.elapsed_time(d1) / 1e3 / reps
            print(json.dumps({"L": L, "kernel": kernel, "luts": prog.info["n_eval_gates"],
                              "levels": prog.info["n_levels"], "lanes": lanes,
                              "ms_per_11_cycles_incl_host_io": s * 1e3,
                              "aes_blocks_per_s": lanes / s,
                              "ms_per_11_cycles_device_resident": sd * 1e3,
                              "aes_blocks_per_s_device_resident": lanes / sd,
                              "lut_sgc_per_s": prog.info["n_eval_gates"] * lanes * 11 / s}), flush=True)
            sim.close()


if __name__ == "__main__":
    main()
