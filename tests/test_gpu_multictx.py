"""The N>1 path on one device (SURVEY §4 tier 6, §8(e)): 2 and 4 CGCM contexts -- one per simulated
rank, each with its own replica of the table, arena, streams and epoch -- driven concurrently from
their own host threads, each translating its shard of an E-shaped batch (contiguous blocks of whole
pointer arrays, bench.py's Workload split) with the timed step of bench.py (mapArrayDevice,
advanceEpoch, unmapArrayDevice + release).  Every rank's forward output is compared with the CPU
oracle run on the same shard in canonical form (AU index in base order, offset inside the AU: the
device addresses themselves are implementation-defined, A22), its refcounts with the oracle's, and
the reverse pass must restore the shard.  There is no collective: ranks share nothing but the GPU.
"""
import threading

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu

CFG = dict(U=1 << 14, arrays=8, slots=1 << 16, seed=5, name="E-shaped, reduced")


def canonical(slots, bases, devptrs, sizes):
    """(unit index, offset) of every non-null device pointer, from a table dump (devptr per unit)."""
    order = np.argsort(devptrs)
    d = devptrs[order]
    k = np.searchsorted(d, slots, side="right") - 1
    assert (k >= 0).all()
    u = order[k]
    off = slots - devptrs[u]
    assert (off <= sizes[u]).all()
    return u, off


def run_rank(ctx, wl, out, barrier, r):
    import torch
    ctx.make_current()
    torch.cuda.set_device(0)
    q = torch.from_numpy(wl.host_sample(wl.n).view(np.int64).copy()).cuda()
    orig = q.clone()
    barrier.wait()                                     # the ranks' calls overlap on the device
    s1 = ctx.mapArrayDevice(q.data_ptr(), wl.n)
    torch.cuda.synchronize()
    fwd = q.cpu().numpy().view(np.uint64).copy()
    tab = ctx.dump_np()
    ctx.advanceEpoch()
    s2 = ctx.unmapArrayDevice(q.data_ptr(), wl.n, release=True)
    torch.cuda.synchronize()
    out[r] = dict(status=(s1, s2), fwd=fwd, tab=tab, back=bool(torch.equal(q, orig)),
                  rc_after=ctx.dump_np()["refCount"].copy(), storage=ctx.storage())


@pytest.mark.parametrize("world", [2, 4])
def test_contexts_per_rank_on_one_device(world):
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    import bench
    from oracle import Oracle
    wls = [bench.Workload(dict(CFG), r, world) for r in range(world)]
    ctxs = []
    try:
        for wl in wls:
            c = cg.Context(0, arena_bytes=int(wl.sizes.sum()) + (256 << 20))
            assert c.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
            ctxs.append(c)
        out = [None] * world
        barrier = threading.Barrier(world)
        ts = [threading.Thread(target=run_rank, args=(ctxs[r], wls[r], out, barrier, r)) for r in range(world)]
        for t in ts:
            t.start()
        for t in ts:
            t.join()
        # shards: contiguous, disjoint, complete
        assert [wl.first_array for wl in wls] == [r * CFG["arrays"] // world for r in range(world)]
        assert sum(wl.n for wl in wls) == CFG["arrays"] * CFG["slots"]
        rc_total = np.zeros(CFG["U"], dtype=np.int64)
        for r, wl in enumerate(wls):
            res = out[r]
            assert res is not None and res["status"] == (0, 0), f"rank {r}: {res and res['status']}"
            assert res["back"], f"rank {r}: reverse pass did not restore the shard"
            assert (res["rc_after"] == 0).all() and res["storage"]["extents"] == 0
            # the oracle on the same shard (sim mode: its own device addresses) -> canonical form
            o = Oracle()
            try:
                for b, s in zip(wl.bases.tolist(), wl.sizes.tolist()):
                    assert o.declareAlloc(b, s, readonly=True) == 0
                slots = wl.host_sample(wl.n)
                ref = slots.copy()
                assert o.mapSlots(ref) == 0
                od = o.dump()
                odev = np.array([u["devptr"] for u in od], dtype=np.uint64)
                orc = np.array([u["refCount"] for u in od], dtype=np.int64)
            finally:
                o.close()
            tab = res["tab"]
            assert (tab["base"] == wl.bases).all()
            assert (tab["refCount"] == orc).all(), f"rank {r}: refcounts differ from the oracle"
            nz = slots != 0
            assert (res["fwd"][~nz] == 0).all()
            gu, go = canonical(res["fwd"][nz], tab["base"], np.where(tab["devptr"] > 0, tab["devptr"], 0).astype(np.uint64),
                               wl.sizes)
            ou, oo = canonical(ref[nz], wl.bases, odev, wl.sizes)
            assert (gu == ou).all() and (go == oo).all(), f"rank {r}: canonical translations differ"
            rc_total += tab["refCount"]
        # the shards together are the single-process batch: refcounts add up to one run over all arrays
        whole = bench.Workload(dict(CFG), 0, 1)
        qa = whole.host_sample(whole.n)
        idx = np.searchsorted(whole.bases, qa[qa != 0], side="right") - 1
        W.release_reservation(whole.R, whole.span)
        assert (rc_total == np.bincount(idx, minlength=CFG["U"])).all()
    finally:
        for c in ctxs:
            c.make_current()
            c.close()
        for wl in wls:
            W.release_reservation(wl.R, wl.span)
