"""Multi-process host logic of the sharded path (dist.py) on CPU: gloo, world size 2.

The GPU path shards stimuli across ranks with no data-path collective; the only exchange
is the all-reduce of the per-shard signature vector (mod 2^64) and the MAX of the
timings.  These tests run that plumbing with the gloo backend.
"""
import os
import socket

import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_gavierrprs23_b200 import dist as gdist


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = {}
        # signature terms that wrap mod 2^64 when summed
        big = (1 << 64) - 5 if rank == 0 else 7
        sig = {"lane_sig_sum": big, "out_popcount": 10 + rank, "ab_mismatch": 0,
               "invariant_violations": rank, "cycles": 100}
        res["sig"] = gdist.reduce_signature(sig)
        res["max"] = gdist.max_over_ranks(1.5 + rank)
        gdist.check_same_program(0xDEADBEEFCAFEF00D)
        try:
            gdist.check_same_program(1234 + rank)
            res["mismatch_detected"] = False
        except RuntimeError:
            res["mismatch_detected"] = True
        res["shard"] = gdist.shard(64 * 10, world, rank)
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks_reduce_max_and_program_check():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(world):
        s = out[r]["sig"]
        assert s["lane_sig_sum"] == 2                    # (2^64 - 5 + 7) mod 2^64
        assert s["out_popcount"] == 21
        assert s["invariant_violations"] == 1
        assert s["cycles"] == 100                        # averaged, not summed
        assert out[r]["max"] == 2.5
        assert out[r]["mismatch_detected"]
    # shards are contiguous, 64-lane aligned, cover the batch exactly once
    (o0, n0), (o1, n1) = out[0]["shard"], out[1]["shard"]
    assert o0 == 0 and o1 == n0 and n0 + n1 == 640 and n0 % 64 == 0 and n1 % 64 == 0


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_shard_partition(world):
    lanes = 64 * 37
    covered = []
    for r in range(world):
        off, n = gdist.shard(lanes, world, r)
        assert off % 64 == 0 and n % 64 == 0
        covered.extend(range(off, off + n))
    assert covered == list(range(lanes))
