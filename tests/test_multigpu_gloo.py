"""Host-side logic of the N>1 path on CPU with gloo (world size 2): the sharding of pointer arrays
across ranks (contiguous blocks of whole arrays, replicated table, no collective on the
data path) and the max-over-ranks timing reduction bench.py uses.  Each rank runs the CPU oracle on
its shard; rank 0 checks that the shards partition the batch and that the per-rank results equal a
single-process run over the whole batch."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from oracle import Oracle
    cfg = dict(bench.CONFIGS["T"])
    wl = bench.Workload(cfg, rank, world)
    o = Oracle()
    for b, s in zip(wl.bases.tolist(), wl.sizes.tolist()):
        assert o.declareAlloc(b, s, readonly=True) == 0
    slots = wl.host_sample(wl.n)                      # this rank's whole shard
    ref = slots.copy()
    assert o.mapSlots(ref) == 0
    rc = torch.tensor([u["refCount"] for u in o.dump()], dtype=torch.int64)
    rcs = [torch.zeros_like(rc) for _ in range(world)]
    dist.all_gather(rcs, rc)
    o.advanceEpoch()
    assert o.unmapSlots(ref, release=True) == 0
    assert (ref == slots).all()
    # shard bookkeeping + results to rank 0
    info = torch.tensor([wl.first_array, wl.arrays_per_rank, wl.start, wl.n], dtype=torch.int64)
    gathered = [torch.zeros_like(info) for _ in range(world)]
    dist.all_gather(gathered, info)
    # max-over-ranks timing, as bench.py does
    t = torch.tensor([float(10 + rank)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        out.put(([g.tolist() for g in gathered], float(t.item()), sum(x for x in rcs).tolist()))
    o.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_sharding_and_reduction(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    shards, tmax, rc_sum = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    import bench
    cfg = bench.CONFIGS["T"]
    # contiguous, disjoint, complete cover of the arrays
    firsts = sorted((s[0], s[1], s[2], s[3]) for s in shards)
    assert firsts[0][0] == 0
    for (f0, n0, st0, c0), (f1, n1, st1, c1) in zip(firsts, firsts[1:]):
        assert f0 + n0 == f1 and st0 + c0 == st1
    assert sum(s[1] for s in shards) == cfg["arrays"]
    assert tmax == 10.0 + world - 1
    # every slot was mapped by exactly one rank: the per-rank refcounts add up to a single-process run
    from oracle import Oracle
    wl = bench.Workload(dict(cfg), 0, 1)
    o = Oracle()
    for b, s in zip(wl.bases.tolist(), wl.sizes.tolist()):
        assert o.declareAlloc(b, s, readonly=True) == 0
    slots = wl.host_sample(wl.n)
    ref = slots.copy()
    assert o.mapSlots(ref) == 0
    assert [u["refCount"] for u in o.dump()] == rc_sum
    assert sum(rc_sum) == wl.n - int((slots == 0).sum())
    o.close()
