"""Multi-process (world_size 2, gloo, CPU) coverage of the N>1 bench path.

The data path has no collective: in the sweep every rank transposes the same shapes in its
own memory, in config 5b ranks own disjoint contiguous shards of independent matrices; the
only collectives are the timing/throughput reductions (SUM, MAX).  These
tests run the bench's own sharding and reduction helpers in two real processes.
"""
import os
import socket

import pytest
import torch.multiprocessing as mp

from conftest import ROOT


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out):
    import sys
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    import bench

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sums, maxs = bench.reduce_over_ranks([rank + 1.0, 10.0 * rank], [rank * 3.0 + 1], world, "cpu")
        shapes = bench.rank_shapes(rank, 4)
        lo, hi = bench.shard_batch(4096, rank, world)
        # the sweep metric: same calls on every rank, per call the max time over ranks
        call_bytes = [2e9, 4e9, 1e9]
        call_ms = [1.0, 2.0, 4.0] if rank == 0 else [2.0, 1.0, 4.0]
        per_call, t_max, agg = bench.aggregate_calls(call_bytes, call_ms, world, "cpu")
        out[rank] = (sums, maxs, shapes, (lo, hi), per_call, t_max, agg)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_rank_sharding_and_reductions(world):
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    r0, r1 = out[0], out[1]
    # reductions: SUM and MAX of the per-rank values, identical on every rank
    assert r0[0] == r1[0] == [3.0, 10.0]
    assert r0[1] == r1[1] == [4.0]
    # the same shapes on every rank (N = 1 and N > 1 time the same per-GPU workload)
    assert len(r0[2]) == len(r1[2]) == 4 and r0[2] == r1[2]
    # per call: max over ranks of the time, job throughput = world x bytes / that time
    assert r0[5] == r1[5] == [2.0, 2.0, 4.0]
    assert r0[4] == r1[4] == [2 * 2e9 / 2e-3 / 1e9, 2 * 4e9 / 2e-3 / 1e9, 2 * 1e9 / 4e-3 / 1e9]
    # aggregate: both ranks' bytes over the max of the summed times (7 ms on both)
    assert abs(r0[6] - 2 * 7e9 / 7e-3 / 1e9) < 1e-6 and r0[6] == r1[6]
    # config 5b: contiguous shards covering [0, 4096) exactly once
    assert r0[3] == (0, 2048) and r1[3] == (2048, 4096)


def test_shard_batch_partitions_exactly():
    import bench
    for batch in (1, 7, 4096, 4097):
        for world in (1, 2, 3, 4, 8):
            seen = []
            for r in range(world):
                lo, hi = bench.shard_batch(batch, r, world)
                seen.extend(range(lo, hi))
            assert seen == list(range(batch))
