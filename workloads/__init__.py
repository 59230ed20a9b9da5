"""Seeded synthetic inputs shared by the oracle side and the CUDA side (no method arithmetic).

See DESIGN.md §"Input recipe".  The five configurations are BASELINE.json `configs`.
"""
from __future__ import annotations

from dataclasses import dataclass
import functools

import numpy as np

from .netlists import (Netlist, Builder, adder, array_multiplier, synthetic, probes_circuit,
                       register_edge_cases, random_tiny, LIBRARY, tt_of)


@dataclass(frozen=True)
class Config:
    name: str          # C1..C5
    label: str         # BASELINE.json configs[i]
    lanes: int         # stimuli (lanes) of the whole job
    cycles: int        # clock cycles
    stim_seed: int
    shards: int = 1    # GPUs the lanes are split over in the paper-scale run

    def netlist(self) -> Netlist:
        return build_netlist(self.name)


CONFIGS = {
    "C1": Config("C1", "8-bit ripple-carry adder, 1024 random stimuli, 1 cycle", 1024, 1, 1),
    "C2": Config("C2", "32x32 array multiplier, 1M stimuli", 1 << 20, 1, 2),
    "C3": Config("C3", "synthetic sequential ~100k gates + 4k regs, 16k stimuli x 1k cycles",
                 16384, 1000, 3),
    "C4": Config("C4", "RISC-V-core-scale synthetic ~1M gates + 50k regs, 64k stimuli x 1k cycles",
                 65536, 1000, 4),
    "C5": Config("C5", "NVDLA-scale synthetic ~10M gates + 500k regs, 256k stimuli x 100 cycles",
                 262144, 100, 5, shards=8),
}


@functools.lru_cache(maxsize=4)
def build_netlist(name: str) -> Netlist:
    if name == "C1":
        return adder(8)
    if name == "C2":
        return array_multiplier(32)
    if name == "C3":
        return synthetic(100_000, 4_000, 64, 64, 40, seed=3, name="C3")
    if name == "C4":
        return synthetic(1_000_000, 50_000, 256, 256, 64, seed=4, name="C4")
    if name == "C5":
        return synthetic(10_000_000, 500_000, 1024, 1024, 100, seed=5, name="C5")
    raise KeyError(name)


def random_host_stimulus(seed: int, cycles: int, n_pi: int, words: int) -> np.ndarray:
    """Paper-style host stimulus [cycle][pi][word] of uniform random uint64 words."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, np.iinfo(np.uint64).max, size=(cycles, n_pi, words),
                        dtype=np.uint64, endpoint=True)


__all__ = ["Netlist", "Builder", "Config", "CONFIGS", "build_netlist", "adder",
           "array_multiplier", "synthetic", "probes_circuit", "register_edge_cases",
           "random_tiny", "random_host_stimulus", "LIBRARY", "tt_of"]
