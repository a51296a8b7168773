"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(cgcm_mapArrayDevice / cgcm_unmapArrayDevice over device-resident arrays, one call per batch):

* config C: 2^20 AUs, 2^26 interior pointers (all of them checked by properties, 2^16 sampled slots
  checked one by one against the CPU oracle in replay mode);
* config E: the full 2^22-AU table and all 256 arrays (2^28 pointers) in ONE call -- exactly the
  launch bench.py times (one cgcm_mapArrayDevice / cgcm_unmapArrayDevice over 2^28 slots).

Properties checked on every slot: refcount[u] == number of slots pointing into u (A8), the reverse
translation restores every slot (round trip), read-only units are never copied back.
"""
import numpy as np
import pytest

import workloads as W

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def run_full(U, arrays, slots_per_array, seed, sample=1 << 16):
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle

    offs, sizes, span = W.table_layout(U, seed)
    R = W.reserve_readonly(span)
    bases = offs + np.uint64(R)
    n = arrays * slots_per_array
    ctx = cg.Context(0, arena_bytes=int(sizes.sum()) + span // 8 + n * 24 + (4 << 30))
    try:
        assert ctx.declareBatch(bases, sizes, readonly=True) == 0
        ot = torch.from_numpy(offs.view(np.int64)).cuda()
        st = torch.from_numpy(sizes.view(np.int64)).cuda()
        q, u = W.queries_t(ot, st, n, seed)
        d = q + R
        orig = d.clone()
        assert ctx.mapArrayDevice(d.data_ptr(), n) == 0
        # A8: refcount == number of slots pointing into the unit (every unit, every slot)
        dump = ctx.dump_np()
        rc = dump["refCount"]
        cnt = torch.bincount(u, minlength=U).cpu().numpy()
        assert (rc == cnt).all()
        dev = dump["devptr"]
        # forward translation of every slot: devptr(u) + (p - base(u))  (vectorised on the GPU)
        devt = torch.from_numpy(dev.view(np.int64)).cuda()
        bt = torch.from_numpy(bases.view(np.int64)).cuda()
        assert torch.equal(d, devt[u] + (orig - bt[u]))
        del devt, bt
        # 2^16 sampled slots one by one through the oracle (replay mode: the GPU's device addresses)
        rng = np.random.default_rng(seed)
        idx = np.sort(rng.choice(n, size=min(sample, n), replace=False))
        ps = orig.cpu().numpy().view(np.uint64)[idx]
        gs = d.cpu().numpy().view(np.uint64)[idx]
        o = Oracle()
        for b, s in zip(bases.tolist(), sizes.tolist()):
            assert o.declareAlloc(b, s, readonly=True) == 0
        units = np.unique(u.cpu().numpy()[idx])
        for k in units.tolist():
            o.replay(int(bases[k]), int(dev[k]))
        stt, out = o.mapBatch(ps)
        assert stt == 0 and (out == gs).all()
        o.close()
        # a3 + a4 + release: round trip, nothing copied back (read-only), all references dropped
        ctx.advanceEpoch()
        assert ctx.unmapArrayDevice(d.data_ptr(), n, release=True) == 0
        assert torch.equal(d, orig)
        s = ctx.stats()
        assert s["d2h_units"] == 0 and s["rev_translations"] == n and s["fwd_translations"] == n
        assert (ctx.dump_np()["refCount"] == 0).all()
        si = ctx.storage()
        assert si["extents"] == 0 and si["shadows_live"] == 0      # every copy freed, shadow consumed
    finally:
        ctx.close()
        W.release_reservation(R, span)


def test_config_C_full_size():
    run_full(1 << 20, 64, 1 << 20, 3)


def test_config_E_full_table():
    run_full(1 << 22, 256, 1 << 20, 5)


def test_config_D_full_size():
    """Config D at full size: 2^24 node AUs of 32 B (allocated in a seeded permutation order) and a child
    table of 2^25 slots; mapArray + map(root), 24 bottom-up S3 levels, unmapArray + unmap, releases.
    Checked: every subtree sum bit-exact against a vectorised recomputation with the same association,
    copy counts N+1 each way, N forward / N-1 reverse translations, the child table restored."""
    import math
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from tests.harness import host_read

    N = 1 << 24
    vals = W.tree_values(N)
    order = W.tree_alloc_order(N)
    pos = np.empty(N, dtype=np.int64)
    pos[order] = np.arange(N)
    nodes_t = torch.zeros(N * 32, dtype=torch.uint8, pin_memory=True)
    nodes = nodes_t.data_ptr()
    arena = nodes_t.numpy().view(np.float64).reshape(N, 4)
    arena[:, 1] = vals[order]
    arena.view(np.int64)[:, 0] = order
    addr = np.uint64(nodes) + np.uint64(32) * pos.astype(np.uint64)
    child = W.tree_children(N)
    table_t = torch.zeros(2 * N, dtype=torch.int64, pin_memory=True)
    table = np.where(child >= 0, addr[np.maximum(child, 0)], 0).astype(np.uint64)
    table_t.numpy().view(np.uint64)[:] = table
    CB = table_t.data_ptr()
    ctx = cg.Context(0, arena_bytes=4 << 30)
    try:
        bases = np.uint64(nodes) + np.uint64(32) * np.arange(N, dtype=np.uint64)
        assert ctx.declareBatch(bases, np.full(N, 32, dtype=np.uint64)) == 0
        assert ctx.declareAlloc(CB, 16 * N) == 0
        st, cdev = ctx.mapArray(CB)
        assert st == 0
        st, rdev = ctx.map(int(addr[0]))
        assert st == 0
        for dlev in range(int(math.log2(N)), -1, -1):
            lo, hi = (1 << dlev) - 1, min((1 << (dlev + 1)) - 1, N)
            assert ctx.sample_treesum_level(cdev, rdev, N, lo, hi) == 0
            ctx.synchronize()
            ctx.advanceEpoch()
        assert ctx.unmapArray(CB) == 0
        assert ctx.unmap(int(addr[0])) == 0
        assert ctx.releaseArray(CB) == 0
        assert ctx.release(int(addr[0])) == 0
        s = ctx.stats()
        assert (s["h2d_units"], s["h2d_bytes"]) == (N + 1, 48 * N)
        assert (s["d2h_units"], s["d2h_bytes"]) == (N + 1, 48 * N)
        assert s["fwd_translations"] == N and s["rev_translations"] == N - 1
        assert (table_t.numpy().view(np.uint64) == table).all()
        # subtree sums, level by level with the kernel's association: (val + left) + right
        exp = np.zeros(N)
        for dlev in range(int(math.log2(N)), -1, -1):
            lo, hi = (1 << dlev) - 1, min((1 << (dlev + 1)) - 1, N)
            i = np.arange(lo, hi)
            sm = vals[i].copy()
            l, r = 2 * i + 1, 2 * i + 2
            ml, mr = l < N, r < N
            sm[ml] = sm[ml] + exp[l[ml]]
            sm[mr] = sm[mr] + exp[r[mr]]
            exp[i] = sm
        got = arena[pos, 2]
        assert got.tobytes() == exp.tobytes()
        assert abs(got[0] - math.fsum(vals)) <= 1e-12 * abs(math.fsum(vals))
        assert all(u["refCount"] == 0 for u in ctx.dump()[:1000])
    finally:
        ctx.close()
