"""Multi-GPU plumbing: stimulus sharding and the one collective of the path.

Stimuli are independent (the paper's "stimulus parallelism"), so
the batch is split into contiguous global lane ranges, one per rank, each rank
holding the full netlist.  The stimulus hash is keyed on the global word, so the
union of the shards is bit-identical to the 1-GPU run.  The only data exchanged is
the per-shard signature vector, reduced with one all-reduce(SUM) (mod 2^64) over
NCCL/NVLink on GPUs or gloo on CPU; timings are reduced with MAX.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

SIG_KEYS = ("lane_sig_sum", "out_popcount", "ab_mismatch", "invariant_violations", "cycles")


def shard(lanes_total: int, world: int, rank: int) -> tuple[int, int]:
    """(lane_offset, lanes) of `rank`: contiguous, 64-lane aligned, as even as possible."""
    words = lanes_total // 64
    assert words * 64 == lanes_total
    lo = (words * rank) // world
    hi = (words * (rank + 1)) // world
    return lo * 64, (hi - lo) * 64


def _device():
    return torch.device("cuda", torch.cuda.current_device()) if dist.get_backend() == "nccl" \
        else torch.device("cpu")


def _to_i64(v: int) -> int:
    v &= (1 << 64) - 1
    return v - (1 << 64) if v >= (1 << 63) else v


def reduce_signature(sig: dict) -> dict:
    """All-reduce(SUM) of the signature vector; int64 two's-complement wraps mod 2^64."""
    t = torch.tensor([_to_i64(int(sig[k])) for k in SIG_KEYS], dtype=torch.int64, device=_device())
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    out = {k: int(x) & ((1 << 64) - 1) for k, x in zip(SIG_KEYS, t.tolist())}
    out["cycles"] //= dist.get_world_size()
    return out


def max_over_ranks(x: float) -> float:
    t = torch.tensor([float(x)], dtype=torch.float64, device=_device())
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def check_same_program(program_hash: int) -> None:
    """Every rank compiled the same program (deterministic generator + compiler)."""
    h = _to_i64(program_hash)
    t = torch.tensor([h, -h], dtype=torch.int64, device=_device())
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if int(t[0]) != h or int(t[1]) != -h:
        raise RuntimeError("ranks compiled different programs")
