#!/usr/bin/env python
"""Table I-style compile statistics for this repo's circuits: gates
(+ flip-flops), layers (levels), "connections" (nonzero polynomial coefficients, i.e. the
hidden->output weights of the merged network), hidden neurons (sum 2^k),
sparsity of the merged-layer weight matrix, compile time and the saved program size
("Memory (MB)").  CPU only.  usage: python scripts/table1.py > profiles/r01_table1_stats.md"""
import os
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import workloads
    from workloads import aes
    import paper_conf_ipps_gavierrprs23_b200 as gs
    rows = [("C1 adder8", workloads.adder(8)), ("C2 mult32", workloads.array_multiplier(32)),
            ("AES-128 core", aes.aes128_core()), ("C3 synth 100k", workloads.CONFIGS["C3"].netlist()),
            ("C4 synth 1M", workloads.CONFIGS["C4"].netlist())]
    print("| circuit | L | gates | FFs | LUTs | layers | connections | hidden neurons | sparsity | compile s | program MB |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    for name, nl in rows:
        for L in (0, 4, 8):
            t = time.perf_counter()
            p = gs.Netlist.from_arrays(nl).compile(lut_k=L)
            dt = time.perf_counter() - t
            i = p.info
            with tempfile.TemporaryDirectory() as d:
                f = os.path.join(d, "p.gsp")
                p.save(f)
                mb = os.path.getsize(f) / 1e6
            # merged layer l: hidden neurons of level l x signals feeding it; the weight matrix
            # of the merged network is (sum hidden) x (sum signals) with `connections` nonzeros
            signals = i["n_pi"] + i["n_reg"] + i["n_eval_gates"]
            sparsity = 1.0 - i["nnz_coeffs"] / max(1, i["hidden_neurons"] * signals / max(1, i["n_levels"]))
            print(f"| {name} | {L or 'as built'} | {int((nl.gate_k > 0).sum())} | {nl.n_reg} | {i['n_eval_gates']} | "
                  f"{i['n_levels']} | {i['nnz_coeffs']} | {i['hidden_neurons']} | {sparsity:.5f} | {dt:.2f} | {mb:.1f} |")


if __name__ == "__main__":
    main()
