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


def sample_lanes(lanes_total: int, shards: int = 1, per_shard: int = 256, seed: int = 0,
                 groups: int = 4, lanes_per_word: int = 4) -> np.ndarray:
    """Deterministic lane sample for the oracle comparison at full size (SURVEY §8(c) "Whole
    engine"): ``per_shard`` lanes in every one of ``shards`` equal shards, grouped
    ``lanes_per_word`` to a 64-lane word (so a trace of few words covers them), always
    including (in this priority while room is left) each shard's first, last and second
    word, the words on both sides of every boundary between ``groups`` equal lane groups of
    the shard, and bits 0 and 63 of every chosen word.  Selection only: no method
    arithmetic."""
    rng = np.random.default_rng(seed)
    per = lanes_total // shards
    W = per // 64
    nw = max(1, per_shard // lanes_per_word)
    out = []
    for sh in range(shards):
        must = [0, W - 1, 1]                        # lanes 0, 63, 64 and the last lane
        for g in range(1, groups):
            if W % groups == 0:
                must += [g * W // groups - 1, g * W // groups]
        must = list(dict.fromkeys(w for w in must if 0 <= w < W))[:nw]
        rest = np.setdiff1d(np.arange(W), must)
        pick = list(must) + sorted(rng.choice(rest, size=min(nw - len(must), len(rest)), replace=False).tolist())
        for w in sorted(pick):
            bits = {0, 63} if lanes_per_word >= 2 else {0}
            while len(bits) < min(lanes_per_word, 64):
                bits.add(int(rng.integers(0, 64)))
            out += [sh * per + 64 * w + b for b in sorted(bits)]
    return np.array(out, dtype=np.int64)


def random_host_stimulus(seed: int, cycles: int, n_pi: int, words: int) -> np.ndarray:
    """Paper-style host stimulus [cycle][pi][word] of uniform random uint64 words."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, np.iinfo(np.uint64).max, size=(cycles, n_pi, words),
                        dtype=np.uint64, endpoint=True)


__all__ = ["Netlist", "Builder", "Config", "CONFIGS", "build_netlist", "adder", "sample_lanes",
           "array_multiplier", "synthetic", "probes_circuit", "register_edge_cases",
           "random_tiny", "random_host_stimulus", "LIBRARY", "tt_of"]
