"""GPU parity tests: the CUDA path (libcgcm.so through the C ABI) against the CPU oracle, element by
element, on seeded inputs.  Needs a B200 (run via gpurun); marked `gpu`.
"""
import numpy as np
import pytest

import workloads as W
from tests.harness import Pair, HostBuf, host_read, host_write

pytestmark = pytest.mark.gpu

ALPHA = 0.999


@pytest.fixture(scope="module")
def cgcm_mod():
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    return cg


@pytest.fixture(params=[0, 8, 16, 40], ids=["auto", "shadow", "levels", "shadow-v2"])
def pair(cgcm_mod, request):
    from oracle import Oracle
    ctx = cgcm_mod.Context(0, arena_bytes=1 << 30, flags=request.param)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    p.check_balance()   # raises if storage leaked after a test that released everything
    ctx.close()
    o.close()


def test_native_library_is_loaded(cgcm_mod):
    import os
    maps = open("/proc/self/maps").read()
    cgcm_mod.lib()
    maps = open("/proc/self/maps").read()
    assert os.path.realpath(cgcm_mod.LIB_PATH) in maps


def test_scalar_map_unmap_release(pair):
    P = pair
    buf = HostBuf(1 << 16)
    bases = [buf.addr + 0x1000 * k + 8 * k for k in range(8)]
    for k, b in enumerate(bases):
        assert P.declare(b, 64 + 40 * k, np.full(64 + 40 * k, k + 1, dtype=np.uint8)) == 0
    P.check("declared")
    for k, b in enumerate(bases):
        for off in (0, 1, (64 + 40 * k) // 2, 64 + 40 * k):
            P.run("map", b + off)
    P.check("mapped")
    P.check_device_units()
    # GPU function writes (raw device write), launch, unmap copies once per epoch
    for u in P.g.dump():
        P.g.dev_write(u["devptr"], np.full(u["size"], 0xAB, dtype=np.uint8))
        P.o.dev_write(u["devptr"], np.full(u["size"], 0xAB, dtype=np.uint8))
    P.run("unmap", bases[0])           # no launch since map: no copy (A5 R1)
    P.advance()
    for b in bases:
        P.run("unmap", b)
        P.run("unmap", b + 3)          # same epoch: no second copy
    P.check("unmapped")
    for b in bases:
        for _ in range(4):
            P.run("release", b)
    P.check("released")
    P.run("release", bases[0])         # underflow -> NOT_MAPPED
    P.run("map", 0)                    # NULL
    P.check("end")


def test_mapArray_roundtrip_permutation(pair):
    P = pair
    buf = HostBuf(1 << 20)
    rows = [buf.addr + 0x800 * k for k in range(16)]
    for k, r in enumerate(rows):
        P.declare(r, 256, np.full(32, k + 0.5))
    pp = buf.addr + 0x80000
    targets = [r + 8 * (k % 5) for k, r in enumerate(rows)] + [0, rows[3]]
    P.declare(pp, 8 * len(targets), np.asarray(targets, dtype=np.uint64))
    st, d = P.run("mapArray", pp)
    assert st == 0
    P.check("mapArray")
    P.check_device_units()
    dev = P.g.dev_read(d, 8 * len(targets)).view(np.uint64).copy()
    perm = np.array([5, 2, 9, 0, 1, 3, 4, 6, 7, 8, 10, 11, 12, 13, 14, 15, 16, 17])
    P.g.dev_write(d, dev[perm])
    P.o.dev_write(d, dev[perm])
    P.advance()
    P.run("unmapArray", pp)
    P.check("unmapArray permuted")
    got = np.frombuffer(host_read(pp, 8 * len(targets)), dtype=np.uint64)
    assert (got == np.asarray(targets, dtype=np.uint64)[perm]).all()
    P.g.dev_write(d, dev)
    P.o.dev_write(d, dev)
    P.advance()
    P.run("unmapArray", pp)
    P.run("releaseArray", pp)
    P.check("released")
    assert all(u["refCount"] == 0 for u in P.g.dump())


def setup_A(P, nrows, ncols, seed=1):
    """double **rows: nrows row AUs + the row-pointer AU from the pinned header-free heap."""
    vals = W.config_A_values(nrows, ncols, seed)
    rows = [P.malloc(8 * ncols, vals[r]) for r in range(nrows)]
    pp = P.malloc(8 * nrows, np.asarray(rows, dtype=np.uint64))
    return rows, pp, vals


@pytest.mark.parametrize("promoted", [False, True])
def test_config_A_naive_vs_promoted(pair, promoted):
    P = pair
    nrows = ncols = 256
    iters = 100
    rows, pp, vals = setup_A(P, nrows, ncols)
    P.check("setup")

    def step(d):
        assert P.g.sample_scale(d, nrows, ncols, ALPHA) == 0
        P.g.synchronize()
        P.o.kernel_scale(d, nrows, ncols, ALPHA)
        P.advance()

    if not promoted:
        for it in range(iters):
            st, d = P.run("mapArray", pp)
            step(d)
            P.run("unmapArray", pp)
            P.run("releaseArray", pp)
            if it % 25 == 0:
                P.check(f"iter {it}")
    else:
        st, d0 = P.run("mapArray", pp)
        for it in range(iters):
            st, d = P.run("mapArray", pp)
            assert d == d0
            step(d)
            P.run("releaseArray", pp)
            if it % 25 == 0:
                P.check(f"iter {it}")
        P.run("unmapArray", pp)
        P.run("releaseArray", pp)
    P.check("end")
    s = P.g.stats()
    if promoted:
        assert (s["h2d_units"], s["h2d_bytes"], s["d2h_units"], s["d2h_bytes"]) == (257, 526336, 257, 526336)
    else:
        assert (s["h2d_units"], s["h2d_bytes"]) == (25700, 52633600)
        assert (s["d2h_units"], s["d2h_bytes"]) == (25700, 52633600)
    x = vals.copy()
    for _ in range(iters):
        x = x * np.float64(ALPHA)
    got = np.stack([np.frombuffer(host_read(a, 8 * ncols), dtype=np.float64) for a in rows])
    assert got.tobytes() == x.tobytes()


def test_errors_leave_state_unchanged(pair):
    P = pair
    buf = HostBuf(1 << 16)
    a, b = buf.addr + 0x1000, buf.addr + 0x2000
    P.declare(a, 64, np.arange(8, dtype=np.uint64))
    P.declare(b, 64)
    pp = buf.addr + 0x8000
    P.declare(pp, 24, np.array([a, b + 8, buf.addr + 0x3000], dtype=np.uint64))
    P.run("mapArray", pp)                          # last slot unregistered
    P.run("mapBatch", [a, a + 64, a + 65])         # past the end
    P.run("mapBatch", [a, a + 0x800])              # gap
    P.run("unmap", a)
    P.run("release", a)
    P.check("after errors")
    P.run("map", a)
    P.run("releaseBatch", [a, a + 8])              # second release underflows
    P.check("after release underflow")
    assert P.g.undeclare(a) == P.o.undeclare(a) == -5
    assert P.g.declareAlloc(a + 0x30, 8) == -3
    P.run("release", a)
    host_write(pp, np.array([a, b + 8, 0], dtype=np.uint64))
    P.sync_host_to_oracle(pp, 24)
    P.run("mapArray", pp)
    P.run("release", b)                            # steal the element's reference
    P.run("releaseArray", pp)                      # underflow on b -> rolled back
    P.check("after releaseArray underflow")


def test_self_referential_pool(pair):
    P = pair
    buf = HostBuf(4096)
    pool, n = buf.addr, 8
    P.declare(pool, 8 * n, np.array([pool + 8 * ((k + 1) % n) for k in range(n)], dtype=np.uint64))
    P.run("mapArray", pool)
    P.check("mapped")
    P.check_device_units()
    P.advance()
    P.run("unmapArray", pool)
    P.check("unmapped")
    P.run("releaseArray", pool)
    P.check("released")


def test_globals(pair):
    P = pair
    buf = HostBuf(4096)
    P.declare_global("g_ro", buf.addr, 48, ro=True)
    P.declare_global("g_rw", buf.addr + 256, 48)
    for _ in range(2):
        P.run("map", buf.addr)
        P.run("map", buf.addr + 256)
        P.advance()
        P.run("unmap", buf.addr)
        P.run("unmap", buf.addr + 256)
        P.run("release", buf.addr)
        P.run("release", buf.addr + 256)
        P.check("globals cycle")
    assert P.g.declareGlobal("g_ro", buf.addr + 1024, 8) == -6


def config_C_setup(P, U, seed=3):
    offs, sizes, span = W.table_layout(U, seed)
    R = W.reserve_readonly(span)
    bases = offs + np.uint64(R)
    assert P.g.declareBatch(bases, sizes, readonly=True) == 0
    for b, s in zip(bases, sizes):
        assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
    return offs, sizes, R, span


@pytest.mark.parametrize("U,Q", [(1 << 12, (1 << 16) + 13), (50000, 300001)])
def test_config_C_device_arrays(pair, U, Q):
    """mapArrayDevice / unmapArrayDevice (+release) vs the oracle's mapSlots / unmapSlots."""
    import torch
    P = pair
    offs, sizes, R, span = config_C_setup(P, U)
    q, u = W.queries(offs, sizes, Q, 3)
    slots = (q + np.uint64(R)).astype(np.uint64)
    slots[::97] = 0                                        # NULL slots
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    assert P.g.mapArrayDevice(d.data_ptr(), Q) == 0
    P.feed_replay()
    ref = slots.copy()
    assert P.o.mapSlots(ref) == 0
    got = d.cpu().numpy().view(np.uint64)
    assert (got == ref).all()
    P.check("mapped")
    P.advance()
    assert P.g.unmapArrayDevice(d.data_ptr(), Q, release=True) == 0
    assert P.o.unmapSlots(ref, release=True) == 0
    got = d.cpu().numpy().view(np.uint64)
    assert (got == ref).all() and (got == slots).all()
    P.check("unmapped")
    W.release_reservation(R, span)


def test_config_C_device_array_errors(pair):
    import torch
    P = pair
    offs, sizes, R, span = config_C_setup(P, 1000)
    q, u = W.queries(offs, sizes, 5000, 3)
    slots = (q + np.uint64(R)).astype(np.uint64)
    slots[1234] = np.uint64(R) + offs[10] + sizes[10] + np.uint64(1) if offs[11] - offs[10] > sizes[10] + 1 \
        else np.uint64(R + span + 100)
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    before = P.g.dump()
    assert P.g.mapArrayDevice(d.data_ptr(), len(slots)) == -2
    assert (d.cpu().numpy().view(np.uint64) == slots).all()      # in-place rewrite rolled back
    assert P.g.dump() == before
    W.release_reservation(R, span)


def tree_sums(vals, N):
    out = np.zeros(N)
    for i in range(N - 1, -1, -1):
        s = vals[i]
        if 2 * i + 1 < N:
            s = s + out[2 * i + 1]
        if 2 * i + 2 < N:
            s = s + out[2 * i + 2]
        out[i] = s
    return out


@pytest.mark.parametrize("N", [1, 7, 1000, 1 << 14])
def test_config_D_tree(pair, N):
    P = pair
    import math
    vals = W.tree_values(N)
    order = W.tree_alloc_order(N)
    nodes = P.g.malloc(32 * N)
    P.g.undeclare(nodes)
    pos = np.empty(N, dtype=np.int64)
    pos[order] = np.arange(N)
    addr = np.uint64(nodes) + np.uint64(32) * pos.astype(np.uint64)
    arena = np.zeros((N, 4), dtype=np.float64)
    arena[:, 1] = vals[order]
    arena.view(np.int64)[:, 0] = order
    host_write(nodes, arena)
    bases = [nodes + 32 * k for k in range(N)]
    assert P.g.declareBatch(bases, [32] * N) == 0
    for b in bases:
        P.o.declareAlloc(b, 32)
    P.units.update({b: 32 for b in bases})
    P.o.host_write(nodes, arena)
    child = W.tree_children(N)
    table = np.where(child >= 0, addr[np.maximum(child, 0)], 0).astype(np.uint64)
    CB = P.g.malloc(16 * N)
    P.g.undeclare(CB)
    P.declare(CB, 16 * N, table)
    st, cdev = P.run("mapArray", CB)
    st, rdev = P.run("map", int(addr[0]))
    depth = int(math.floor(math.log2(N))) if N > 1 else 0
    for dlev in range(depth, -1, -1):
        lo, hi = (1 << dlev) - 1, min((1 << (dlev + 1)) - 1, N)
        assert P.g.sample_treesum_level(cdev, rdev, N, lo, hi) == 0
        P.g.synchronize()
        P.o.kernel_treesum_level(cdev, rdev, N, lo, hi)
        P.advance()
    P.run("unmapArray", CB)
    P.run("unmap", int(addr[0]))
    P.run("releaseArray", CB)
    P.run("release", int(addr[0]))
    P.check("tree done")
    exp = tree_sums(vals, N)
    got = np.frombuffer(host_read(nodes, 32 * N), dtype=np.float64).reshape(N, 4)[pos, 2]
    assert got.tobytes() == exp.tobytes()


def test_random_stress(pair):
    """Seeded random interleavings of declare/map/mapArray/advance/unmap/release (SURVEY §4 tier 3)."""
    P = pair
    rng = np.random.default_rng(7)
    buf = HostBuf(1 << 20)
    units = []
    cur = buf.addr
    for k in range(300):
        cur += int(rng.integers(0, 3)) * 16
        size = int(rng.integers(1, 40)) * 8
        units.append((cur, size))
        cur += size
    for b, s in units:
        P.declare(b, s, rng.integers(0, 255, s, dtype=np.uint8))
    arrays = []
    for j in range(6):  # pointer arrays into random units (interior, one-past-end, NULL, aliases)
        n = int(rng.integers(1, 40))
        tg = []
        for _ in range(n):
            b, s = units[int(rng.integers(0, len(units)))]
            r = rng.random()
            tg.append(0 if r < 0.1 else b + int(rng.integers(0, s + 1)))
        cur = (cur + 64) // 32 * 32
        pa = cur
        cur += 8 * n + int(rng.integers(1, 5)) * 8
        P.declare(pa, 8 * n, np.asarray(tg, dtype=np.uint64))
        arrays.append(pa)
    mapped_arrays = []
    own = {}   # scalar references this test took (releases stay balanced, as compiler-inserted calls are)
    for step in range(400):
        r = rng.random()
        if r < 0.25:
            b, s = units[int(rng.integers(0, len(units)))]
            st, _ = P.run("map", b + int(rng.integers(0, s + 1)))
            if st == 0:
                own[b] = own.get(b, 0) + 1
        elif r < 0.35:
            b, s = units[int(rng.integers(0, len(units)))]
            P.run("unmap", b)
        elif r < 0.45:
            held = [b for b, c in own.items() if c > 0]
            if held:
                b = held[int(rng.integers(0, len(held)))]
                P.run("release", b + 1 if dict(units)[b] > 1 else b)
                own[b] -= 1
            else:
                b, s = units[int(rng.integers(0, len(units)))]
                if P.o.dump and all(u["refCount"] == 0 for u in P.o.dump() if u["base"] == b):
                    P.run("release", b)   # never mapped: NOT_MAPPED on both sides
        elif r < 0.6:
            pa = arrays[int(rng.integers(0, len(arrays)))]
            st, _ = P.run("mapArray", pa)
            if st == 0:
                mapped_arrays.append(pa)
        elif r < 0.7 and mapped_arrays:
            pa = mapped_arrays[int(rng.integers(0, len(mapped_arrays)))]
            P.run("unmapArray", pa)
        elif r < 0.8 and mapped_arrays:
            pa = mapped_arrays.pop(int(rng.integers(0, len(mapped_arrays))))
            P.run("releaseArray", pa)
        elif r < 0.9:
            P.advance()
        else:
            ps = [units[int(rng.integers(0, len(units)))][0] for _ in range(int(rng.integers(1, 20)))]
            P.run("mapBatch", ps)
        if step % 20 == 0:
            P.check(f"step {step}")
    P.check("end")


@pytest.mark.parametrize("promoted", [False, True])
def test_config_B_gemm_reduced(pair, promoted):
    """Config B shape at n = 256, 4 row-blocks of 64: 3 jagged matrices, one S2 launch per block.
    Counts, refcounts and A/B bytes exact; C within 1e-12 relative of the oracle's long-double S2."""
    P = pair
    n, blk = 256, 64
    mats, vals = [], []
    for m in range(3):
        v = W.config_B_values(n, 2, m)
        rows = [P.malloc(8 * n, v[r]) for r in range(n)]
        mats.append(P.malloc(8 * n, np.asarray(rows, dtype=np.uint64)))
        vals.append((rows, v))
    A, B, Cm = mats

    def block(b0, devs):
        assert P.g.sample_gemm_rows(devs[0], devs[1], devs[2], n, b0, blk, 1.5, 1.2) == 0
        P.g.synchronize()
        P.o.kernel_gemm_rows(devs[0], devs[1], devs[2], n, b0, blk, 1.5, 1.2)
        P.advance()

    if promoted:
        for pp in mats:
            P.run("mapArray", pp)
    for b0 in range(0, n, blk):
        devs = [P.run("mapArray", pp)[1] for pp in mats]
        block(b0, devs)
        if not promoted:
            P.run("unmapArray", Cm)
        for pp in mats:
            P.run("releaseArray", pp)
    if promoted:
        P.run("unmapArray", Cm)
        for pp in mats:
            P.run("releaseArray", pp)
    gd, od = P.g.dump(), P.o.dump()
    assert gd == od
    gs, os_ = P.g.stats(), P.o.stats()
    for f in ("h2d_units", "h2d_bytes", "d2h_units", "d2h_bytes", "fwd_translations", "rev_translations"):
        assert gs[f] == os_[f], f
    blocks = n // blk
    if promoted:
        assert (gs["h2d_units"], gs["d2h_units"]) == (3 * (n + 1), n + 1)
    else:
        assert (gs["h2d_units"], gs["d2h_units"]) == (blocks * 3 * (n + 1), blocks * (n + 1))
    for (rows, v), pp in zip(vals[:2], mats[:2]):
        got = np.stack([np.frombuffer(host_read(a, 8 * n), dtype=np.float64) for a in rows])
        assert got.tobytes() == v.tobytes()
    rows_c = vals[2][0]
    gc = np.stack([np.frombuffer(host_read(a, 8 * n), dtype=np.float64) for a in rows_c])
    oc = np.stack([P.o.host_read(a, 8 * n).view(np.float64) for a in rows_c])
    assert np.max(np.abs(gc - oc) / np.abs(oc)) < 1e-12


@pytest.mark.parametrize("release", [False, True])
def test_unmapArrayDevice_error_rolls_back(pair, release):
    """A large reverse pass (snapshot rollback) and a small one (journal rollback) hitting an
    unregistered device pointer: UNREGISTERED, device slots, refcounts and epochs unchanged."""
    import torch
    P = pair
    offs, sizes, R, span = config_C_setup(P, 8192)
    for n in (60000, 100):                      # >= U/8: snapshot mode; < U/8: journal mode
        q, u = W.queries(offs, sizes, n, 3)
        slots = (q + np.uint64(R)).astype(np.uint64)
        d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
        assert P.g.mapArrayDevice(d.data_ptr(), n) == 0
        P.g.advanceEpoch()
        bad = d.clone()
        bad[n // 2] = 12345                      # not a device copy
        before = P.g.dump()
        assert P.g.unmapArrayDevice(bad.data_ptr(), n, release=release) == -2
        assert P.g.dump() == before
        bad[n // 2] = d[n // 2]
        assert torch.equal(bad, d)               # the in-place reverse rewrite was undone
        assert P.g.unmapArrayDevice(d.data_ptr(), n, release=True) == 0
        assert (d.cpu().numpy().view(np.uint64) == slots).all()
    W.release_reservation(R, span)


def test_device_array_shadow_fallback_on_modified_slots(pair):
    """The reverse pass reads the forward pass's shadow only for unchanged slots: a GPU function that
    permutes / clears / re-points slots (violating R13-ii on purpose) still gets the exact reverse
    lookup of the oracle."""
    import torch
    P = pair
    offs, sizes, R, span = config_C_setup(P, 4096)
    n = (1 << 17) + 5
    q, u = W.queries(offs, sizes, n, 3)
    slots = (q + np.uint64(R)).astype(np.uint64)
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    assert P.g.mapArrayDevice(d.data_ptr(), n) == 0
    P.feed_replay()
    ref = slots.copy()
    assert P.o.mapSlots(ref) == 0
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    # the "GPU function": permute a third of the slots, NULL a few, point one at a unit's start
    perm = torch.randperm(n // 3, generator=torch.Generator().manual_seed(1)).cuda()
    d[: n // 3] = d[: n // 3][perm]
    d[7] = 0
    d[n - 1] = d[n - 2]
    ref[: n // 3] = ref[: n // 3][perm.cpu().numpy()]
    ref[7] = 0
    ref[n - 1] = ref[n - 2]
    P.advance()
    # refcounts: the NULLed slot and the duplicated one make the release unbalanced for two units;
    # both sides must agree on the outcome (status and state)
    st_g = P.g.unmapArrayDevice(d.data_ptr(), n, release=True)
    st_o = P.o.unmapSlots(ref, release=True)
    assert st_g == st_o
    if st_g != 0:
        return
    got = d.cpu().numpy().view(np.uint64)
    assert (got == ref).all()
    P.check("after modified-slot unmap")
    W.release_reservation(R, span)


def test_heap_churn_calloc_realloc_alloca(pair):
    """NEXT-1: heap wrappers and declareAlloca scopes keep the allocation table current under churn
    (P:L171-179); mapped AUs cannot move or expire; every step mirrored into the oracle."""
    P = pair
    g, o = P.g, P.o
    rng = np.random.default_rng(3)
    live = {}
    for step in range(60):
        r = rng.random()
        if r < 0.3 or not live:
            n = int(rng.integers(1, 300))
            a = g.calloc(n, 1)
            assert a and host_read(a, n) == bytes(n)
            assert o.declareAlloc(a, n) == 0
            o.host_write(a, bytes(n))
            live[a] = n
        elif r < 0.55:
            a = list(live)[int(rng.integers(0, len(live)))]
            n = int(rng.integers(1, 600))
            old = host_read(a, live[a])
            b = g.realloc(a, n)
            assert b
            assert host_read(b, min(n, live[a])) == old[:min(n, live[a])]
            assert o.undeclare(a) == 0
            assert o.declareAlloc(b, n) == 0
            o.host_write(b, np.frombuffer(host_read(b, n), dtype=np.uint8))
            del live[a]
            live[b] = n
        elif r < 0.75:
            a = list(live)[int(rng.integers(0, len(live)))]
            P.units[a] = live[a]
            P.run("map", a)
            b = g.realloc(a, live[a] + 64)             # mapped: cannot move
            assert b == 0
            P.run("release", a)
        else:
            a = list(live)[int(rng.integers(0, len(live)))]
            assert g.free(a) == 0 and o.undeclare(a) == 0
            del live[a]
            P.units.pop(a, None)
        P.units.update(live)
        if step % 10 == 0:
            P.check(f"churn {step}")
    # declareAlloca scopes
    assert g.scopeEnter() == 0
    xs = [g.declareAlloca(64 + 8 * k) for k in range(5)]
    for k, x in enumerate(xs):
        assert x and o.declareAlloc(x, 64 + 8 * k) == 0
        o.host_write(x, np.frombuffer(host_read(x, 64 + 8 * k), dtype=np.uint8))
        P.units[x] = 64 + 8 * k
    P.run("map", xs[2])
    assert g.scopeExit() == -5                         # a mapped stack variable keeps the scope
    P.run("release", xs[2])
    assert g.scopeExit() == 0
    for x in xs:
        assert o.undeclare(x) == 0
        P.units.pop(x)
    P.check("after scopes")


def test_host_arrays_large_overlap_and_shadows(pair):
    """mapArrays / unmapArrays / releaseArrays on outers large enough for the transfer overlap (one
    copy group per extent: spacers keep the outers in separate extents) and for recorded shadows
    (>= 2^16 slots), with a GPU function that re-points some slots in between (the reverse passes
    fall back to full lookups for them).  Every slot, unit and counter against the oracle."""
    P = pair
    offs, sizes, R, span = config_C_setup(P, 4096)
    ns = [(1 << 16) + 3, 1 << 17, (1 << 16) + 100]
    outers = []
    for k, n in enumerate(ns):
        q, _ = W.queries(offs, sizes, n, 30 + k)
        vals = (q + np.uint64(R)).astype(np.uint64)
        vals[:: 97 + k] = 0
        outers.append(P.malloc(8 * n, vals))
        P.malloc(200 << 10)                               # spacer: the next outer is another extent
    st, gptrs = P.run("mapArrays", outers)
    assert st == 0
    P.check("mapArrays")
    P.check_device_units()
    # the "GPU function": swap two halves of outer 1's first 1000 slots, NULL one, duplicate one
    d1 = int(gptrs[1])
    dev = P.g.dev_read(d1, 8 * 2000).view(np.uint64).copy()
    new = dev.copy()
    new[:1000], new[1000:2000] = dev[1000:2000], dev[:1000]
    new[5] = 0
    new[6] = new[7]
    P.g.dev_write(d1, new)
    P.o.dev_write(d1, new)
    P.advance()
    P.run("unmapArrays", outers)
    P.check("unmapArrays")
    st = P.run("releaseArrays", outers)
    P.check("releaseArrays")
    W.release_reservation(R, span)


def test_global_bound_to_device_symbol(pair):
    """NEXT-4: a global whose device copy is a module's __device__ variable (Alg. 1's cuModuleGetGlobal
    branch).  map returns the symbol's address, GPU code that names the
    variable sees the host values, copy-back returns what it wrote, re-maps reuse the symbol (A14),
    and a second symbol range overlapping it is rejected (A7)."""
    P = pair
    sym, nbytes = P.g.sample_global()
    assert nbytes == 512 * 8
    buf = HostBuf(8192)
    vals = W.config_A_values(1, 512, 7)[0]                       # fp64 in [1, 2)
    host_write(buf.addr, vals)
    s1 = P.g.declareGlobalSymbol("g_sym", buf.addr, nbytes, False, sym)
    s2 = P.o.declareGlobal("g_sym", buf.addr, nbytes)
    assert s1 == s2 == 0
    P.units[buf.addr] = nbytes
    P.o.host_write(buf.addr, np.frombuffer(host_read(buf.addr, nbytes), dtype=np.uint8))
    assert P.g.declareGlobalSymbol("g_sym2", buf.addr + 6000, 64, False, sym + 8) == -3   # overlaps g_sym
    assert P.g.declareGlobalSymbol("g_sym", buf.addr + 6000, 64, False, sym + nbytes + 64) == -6
    expect = vals.copy()
    for it in range(3):
        st, d = P.run("map", buf.addr + 8 * it)                 # interior pointer: symbol + offset
        assert d == sym + 8 * it
        assert P.g.sample_scale_global(ALPHA) == 0
        P.g.synchronize()
        expect = expect * ALPHA                                   # one correctly rounded multiply (A21)
        P.o.dev_write(sym, expect.view(np.uint8))
        P.advance()
        P.run("unmap", buf.addr + 8 * it)
        P.run("release", buf.addr + 8 * it)
        P.check(f"symbol global, cycle {it}")
        got = np.frombuffer(host_read(buf.addr, nbytes), dtype=np.float64)
        assert (got == expect).all()
    assert P.undeclare(buf.addr) == 0


@pytest.mark.parametrize("check", [False, True], ids=["region", "region+checker"])
def test_region_promotes_config_A(pair, check):
    """NEXT-2: cgcm_regionBegin/End perform Listing 4's hoisted mapArray / unmapArray+releaseArray
    (A11) around a loop whose body keeps its own mapArray + releaseArray; compared
    with the oracle running the promoted sequence explicitly.  With the modOrRef checker on, the
    loop (which never touches host memory) records no violation."""
    P = pair
    nrows = ncols = 64
    rows, pp, vals = setup_A(P, nrows, ncols)
    assert P.g.regionBegin([pp], [P.g.REGION_MAPARRAY], check=check) == 0
    P.feed_replay()
    assert P.o.mapArray(pp)[0] == 0
    for it in range(10):
        st, d = P.run("mapArray", pp)
        assert P.g.sample_scale(d, nrows, ncols, ALPHA) == 0
        P.g.synchronize()
        P.o.kernel_scale(d, nrows, ncols, ALPHA)
        P.advance()
        P.run("releaseArray", pp)
    s, v = P.g.regionEnd()
    assert (s, v) == (0, 0)
    assert P.o.unmapArray(pp) == 0 and P.o.releaseArray(pp) == 0
    P.check("after region")
    st = P.g.stats()
    assert st["h2d_units"] == nrows + 1 and st["d2h_units"] == nrows + 1   # once each way (promoted)
    got = np.stack([np.frombuffer(host_read(a, 8 * ncols), dtype=np.float64) for a in rows])
    exp = vals.copy()
    for _ in range(10):
        exp = exp * ALPHA
    assert (got == exp).all()


def test_region_checker_counts_cpu_accesses(pair):
    """The dynamic modOrRef checker: a CPU read of a promoted AU inside the region is
    counted and cgcm_regionEnd reports CGCM_E_MODREF; the access itself completes (the page is
    reopened) and the runtime state stays equal to the oracle's."""
    P = pair
    buf = HostBuf(1 << 20, align=4096)
    base = buf.addr + 8192
    P.declare(base, 4096, np.arange(512, dtype=np.float64))
    assert P.g.regionBegin([base], [P.g.REGION_MAP], check=True) == 0
    P.feed_replay()
    assert P.o.map(base)[0] == 0
    P.advance()
    seen = np.frombuffer(host_read(base + 64, 16), dtype=np.float64)   # the CPU references the AU
    assert list(seen) == [8.0, 9.0]
    s, v = P.g.regionEnd()
    assert s == -11                                                       # CGCM_E_MODREF
    assert v >= 1
    assert P.o.unmap(base) == 0 and P.o.release(base) == 0
    P.check("after checked region")
    assert P.g.regionEnd()[0] == -1                                       # no open region


def test_many_small_arrays_cycle_the_upload_ring(pair):
    """Thousands of small outers per call: every call uploads ~100s of KB of pointers, unit ops and
    segment tables through the pinned staging ring, so its halves are retired and reused (event
    fences) many times; every state vs the oracle after each cycle."""
    P = pair
    rows = [P.malloc(64, np.arange(8, dtype=np.float64) + r) for r in range(64)]
    outers = []
    for k in range(3000):
        sl = np.array([rows[(k * 7 + i) % 64] + 8 * (i % 8) for i in range(4)], dtype=np.uint64)
        outers.append(P.malloc(32, sl))
    for cyc in range(5):
        st, d = P.run("mapArrays", outers)
        P.advance()
        P.run("unmapArrays", outers)
        P.run("releaseArrays", outers)
        if cyc % 2 == 0:
            P.check(f"cycle {cyc}")
    P.check("end")
    assert all(u["refCount"] == 0 for u in P.g.dump())


def test_degenerate_batches(pair):
    """Edge cases of the batch forms (SURVEY §8(b) "data-parallel batch forms (same semantics as the
    sequential loop)"): empty batches, all-NULL batches and arrays, outer AUs with 0 / 1 slot and a
    trailing partial word (A10: the ⌊size/8⌋ words are slots, trailing bytes verbatim), adjacent AUs
    where one's one-past-the-end address is the next one's base (A7 greatestLTE picks the later base),
    and one outer named twice in one mapArrays batch (sequential semantics: two references)."""
    P = pair
    buf = HostBuf(1 << 16)
    for name in ("mapBatch", "unmapBatch", "releaseBatch", "mapArrays", "unmapArrays", "releaseArrays"):
        st = P.run(name, [])
        assert (st[0] if isinstance(st, tuple) else st) == 0, name
    P.check("empty batches")
    P.run("mapBatch", [0, 0, 0])
    P.check("all-NULL batch")
    a, b = buf.addr + 0x1000, buf.addr + 0x1040           # a ends exactly at b's base
    P.declare(a, 64, np.arange(8, dtype=np.uint64))
    P.declare(b, 40, np.arange(5, dtype=np.uint64) + 100)
    st, d = P.run("mapBatch", [a + 64, a + 63, b + 40, b])
    assert st == 0
    P.check("adjacent boundary")
    nul = buf.addr + 0x2000
    P.declare(nul, 8 * 64)                                # 64 NULL slots
    one = buf.addr + 0x3000
    P.declare(one, 8, np.array([a + 8], dtype=np.uint64))
    tiny = buf.addr + 0x3100
    P.declare(tiny, 4, np.array([7, 7, 7, 7], dtype=np.uint8))  # no whole slot
    rag = buf.addr + 0x3200
    P.declare(rag, 20, np.concatenate([np.array([b + 16, a], dtype=np.uint64).view(np.uint8),
                                       np.array([1, 2, 3, 4], dtype=np.uint8)]))
    for pp in (nul, one, tiny, rag):
        st, _ = P.run("mapArray", pp)
        assert st == 0
    P.check("degenerate outers mapped")
    P.check_device_units()
    P.advance()
    for pp in (nul, one, tiny, rag):
        P.run("unmapArray", pp)
    P.check("degenerate outers unmapped")
    for pp in (nul, one, tiny, rag):
        P.run("releaseArray", pp)
    P.check("degenerate outers released")
    st, _ = P.run("mapArrays", [rag, one, rag])           # the same outer twice in one batch
    P.check("duplicate outer mapped")
    P.check_device_units()
    P.advance()
    P.run("unmapArrays", [rag, one, rag])
    P.run("releaseArrays", [rag, one, rag])
    P.check("duplicate outer released")
    P.run("mapArray", rag)                                # already array-mapped: A9 re-map, twice over
    P.run("mapArrays", [rag, rag, one])
    P.check("duplicate re-map")
    P.check_device_units()
    P.advance()
    P.run("unmapArrays", [one, rag, rag])
    P.run("releaseArrays", [rag, rag, one])
    P.run("releaseArray", rag)
    P.check("duplicate re-map released")
    P.run("releaseBatch", [a + 64, a + 63, b + 40, b])
    P.check("end")
    assert all(u["refCount"] == 0 for u in P.g.dump())


def _nested_outers(P, order):
    buf = HostBuf(1 << 16)
    r0, r1, z = buf.addr + 0x1000, buf.addr + 0x1100, buf.addr + 0x1200
    P.declare(r0, 32, np.arange(4, dtype=np.float64))
    P.declare(r1, 48, np.arange(6, dtype=np.float64) + 0.5)
    P.declare(z, 64, np.arange(8, dtype=np.uint64) + 9)
    Y = buf.addr + 0x2000
    P.declare(Y, 16, np.array([r0, r1 + 8], dtype=np.uint64))
    X = buf.addr + 0x3000
    P.declare(X, 24, np.array([Y, z + 8, 0], dtype=np.uint64))
    batch = [X, Y] if order == "outer_first" else [Y, X]
    st, _ = P.run("mapArrays", batch)
    assert st == 0
    P.check("nested mapped")
    P.check_device_units()
    P.advance()
    P.run("unmapArrays", batch)
    P.check("nested unmapped")
    P.run("releaseArrays", batch)
    P.check("nested released")
    assert all(u["refCount"] == 0 for u in P.g.dump())


@pytest.mark.parametrize("order", ["outer_first", "inner_first"])
def test_nested_outers_in_one_batch(pair, order):
    """An outer that is also an element of another outer of the same mapArrays batch (a jagged array
    of pointer arrays): the batch has the sequential semantics of SURVEY §8(b), so whichever outer
    comes first decides whether the inner one is activated raw (element, Alg. 1) and later
    re-translated in place (A23), or activated as an array and then only referenced (A9)."""
    _nested_outers(pair, order)


def test_lenient_duplicate_outers(cgcm_mod):
    """Lenient mode (A18): unregistered slots pass through and are counted once per mapArray call --
    a batch naming the outer twice counts them twice, as its sequential loop would."""
    from oracle import Oracle
    LENIENT = 2
    ctx = cgcm_mod.Context(0, arena_bytes=1 << 28, flags=LENIENT)
    o = Oracle(LENIENT)
    P = Pair(ctx, o)
    try:
        buf = HostBuf(1 << 16)
        a = buf.addr + 0x1000
        P.declare(a, 64, np.arange(8, dtype=np.uint64))
        stray = buf.addr + 0x8000                          # never declared
        pp = buf.addr + 0x2000
        P.declare(pp, 32, np.array([a + 8, stray, 0, a], dtype=np.uint64))
        st, _ = P.run("mapArrays", [pp, pp])
        assert st == 0
        P.check("lenient mapped")
        P.check_device_units()
        P.advance()
        P.run("unmapArrays", [pp, pp])
        P.run("releaseArrays", [pp, pp])
        P.check("lenient released")
    finally:
        ctx.close()
        o.close()


def _batch_errors(P):
    buf = HostBuf(1 << 16)
    a, b = buf.addr + 0x1000, buf.addr + 0x1100
    P.declare(a, 64, np.arange(8, dtype=np.uint64))
    P.declare(b, 64, np.arange(8, dtype=np.uint64) + 50)
    pp = buf.addr + 0x2000
    P.declare(pp, 24, np.array([a, b + 16, 0], dtype=np.uint64))
    qq = buf.addr + 0x2100
    P.declare(qq, 16, np.array([a + 8, buf.addr + 0x9000], dtype=np.uint64))   # second slot unregistered
    ro = buf.addr + 0x2200
    P.declare(ro, 16, np.array([b, a + 56], dtype=np.uint64), readonly=True)
    undeclared = buf.addr + 0x7000
    P.run("mapArrays", [pp, undeclared])                 # outer miss: nothing happens
    P.check("outer miss")
    P.run("mapArrays", [pp, qq])                         # element miss in the second outer
    P.check("element miss")
    st, _ = P.run("mapArrays", [pp, ro])
    assert st == 0
    P.check("mapped")
    P.check_device_units()
    P.g.dev_write(P.g.dump()[0]["devptr"], np.full(64, 0xCD, dtype=np.uint8))   # GPU writes a
    P.o.dev_write(P.o.dump()[0]["devptr"], np.full(64, 0xCD, dtype=np.uint8))
    P.advance()
    P.run("unmapArrays", [pp, qq])                       # qq not mapped: no copy-back happens
    P.check("unmap error")
    P.run("releaseArrays", [pp, pp])                     # second release underflows the outer
    P.check("release underflow")
    P.run("unmapArrays", [ro, pp])                       # read-only outer: no copy of ro itself
    P.check("unmapped")
    P.run("releaseArrays", [ro, pp])
    P.check("released")
    assert all(u["refCount"] == 0 for u in P.g.dump())


def test_batch_errors_roll_back(pair):
    """All-or-nothing batches: an outer miss, an element miss in a later outer, an
    unmap of an unmapped outer and a duplicate release that underflows leave refcounts, epochs, the
    table, host and device bytes as they were; a read-only outer (Alg. 2: no copy-back) is not
    copied back by unmapArray while its elements are."""
    _batch_errors(pair)


def test_device_array_ragged_slices(pair):
    """mapArrayDevice / unmapArrayDevice over slices that start on an odd slot (8 B off the kernels'
    16-byte chunk grid), lengths 1, 2, 3, 31 and 1025 + 1 (ragged tails), an empty slice, and two slices
    mapped together then unmapped in the other order (the recorded shadows are per slice)."""
    import torch
    P = pair
    offs, sizes, R, span = config_C_setup(P, 2000)
    q, u = W.queries(offs, sizes, 4096, 5)
    slots = (q + np.uint64(R)).astype(np.uint64)
    slots[::13] = 0
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    base = d.data_ptr()
    assert P.g.mapArrayDevice(base + 8, 0) == 0 and P.g.unmapArrayDevice(base + 8, 0) == 0
    P.check("empty")
    ref = slots.copy()
    for (s0, n) in [(1, 1), (3, 2), (5, 3), (9, 31), (101, 1026)]:
        assert P.g.mapArrayDevice(base + 8 * s0, n) == 0
        P.feed_replay()
        seg = ref[s0:s0 + n].copy()
        assert P.o.mapSlots(seg) == 0
        ref[s0:s0 + n] = seg
        assert (d.cpu().numpy().view(np.uint64) == ref).all(), (s0, n)
        P.check(f"mapped {s0}+{n}")
    P.advance()
    for (s0, n) in [(101, 1026), (5, 3), (1, 1), (9, 31), (3, 2)]:
        assert P.g.unmapArrayDevice(base + 8 * s0, n, release=True) == 0
        seg = ref[s0:s0 + n].copy()
        assert P.o.unmapSlots(seg, release=True) == 0
        ref[s0:s0 + n] = seg
        assert (d.cpu().numpy().view(np.uint64) == ref).all(), (s0, n)
        P.check(f"unmapped {s0}+{n}")
    assert (ref == slots).all()
    W.release_reservation(R, span)


def test_global_pointer_arrays(pair):
    """A global array of pointers (the outer is a global: never freed, keeps its device
    copy) whose slots point at heap rows and at a read-only global, cycled naive-style twice with GPU
    writes between map and unmap; the same devptr is reused by the second cycle."""
    P = pair
    buf = HostBuf(1 << 16)
    rows = [buf.addr + 0x1000 + 0x100 * k for k in range(6)]
    for k, r in enumerate(rows):
        P.declare(r, 64, np.full(8, k + 0.25))
    gro = buf.addr + 0x4000
    P.declare_global("tbl_ro", gro, 40, ro=True)
    host_write(gro, np.arange(5, dtype=np.uint64))
    P.sync_host_to_oracle(gro, 40)
    gpp = buf.addr + 0x5000
    host_write(gpp, np.array(rows + [gro + 8, 0], dtype=np.uint64))
    P.declare_global("row_ptrs", gpp, 8 * 8)
    P.sync_host_to_oracle(gpp, 64)
    devs = []
    for cyc in range(2):
        st, d = P.run("mapArray", gpp)
        assert st == 0
        devs.append(d)
        P.check(f"cycle {cyc} mapped")
        P.check_device_units()
        for u in P.g.dump():
            if u["base"] in rows[::2]:
                P.g.dev_write(u["devptr"], np.full(64, 0x10 + cyc, dtype=np.uint8))
                P.o.dev_write(u["devptr"], np.full(64, 0x10 + cyc, dtype=np.uint8))
        P.advance()
        P.run("unmapArray", gpp)
        P.check(f"cycle {cyc} unmapped")
        assert P.g.undeclare(rows[0]) == P.o.undeclare(rows[0])
        P.run("releaseArray", gpp)
        P.check(f"cycle {cyc} released")
    assert devs[0] == devs[1]
    assert np.frombuffer(host_read(gpp, 64), dtype=np.uint64).tolist() == rows + [gro + 8, 0]


def _check_mod_stale_epochs(P, what):
    """Pair.check with one relaxation, DESIGN A28: after the device's u32 epoch origin moves, a unit
    whose epoch is stale may dump a different stale value; whether it is current may not change."""
    from tests.harness import COMPARED_STATS
    gd, od = P.g.dump(), P.o.dump()
    assert len(gd) == len(od), what
    ge, oe = P.g.epoch, P.o.epoch
    assert ge == oe, what
    for a, b in zip(gd, od):
        assert {k: v for k, v in a.items() if k != "epoch"} == {k: v for k, v in b.items() if k != "epoch"}, \
            f"{what}: gpu={a} oracle={b}"
        assert (a["epoch"] == ge) == (b["epoch"] == oe), f"{what}: currency differs gpu={a} oracle={b}"
        if b["epoch"] == oe or b["epoch"] + 8 > oe:
            assert a["epoch"] == b["epoch"] or a["epoch"] != ge, f"{what}: gpu={a} oracle={b}"
    gs, os_ = P.g.stats(), P.o.stats()
    for f in COMPARED_STATS:
        assert gs[f] == os_[f], f"{what}: stat {f} gpu={gs[f]} oracle={os_[f]}"
    for base, n in P.units.items():
        assert host_read(base, n) == P.o.host_read(base, n).tobytes(), f"{what}: host bytes of {hex(base)}"


def test_epoch_origin_move(pair):
    """DESIGN A28: the device keeps u32 epochs relative to an origin that moves when the relative
    epoch would reach 2^32 - 16.  Drive globalEpoch across that point with
    cgcm_advanceEpochs (= n launches) and check every copy decision of Alg. 2 (copy iff
    epoch != globalEpoch and not read-only, at most once per epoch) against the oracle's u64 epochs:
    units left stale across the move, units made current just before it, read-only units."""
    P = pair
    buf = HostBuf(1 << 16)
    us = [buf.addr + 0x1000 + 0x200 * k for k in range(5)]
    for k, u in enumerate(us):
        P.declare(u, 128, np.full(16, k + 0.5), readonly=(k == 4))
    for u in us:
        P.run("map", u)
    assert P.g.advanceEpochs(0xFFFFFFE0) == -1      # the product ABI's bound on one call (cgcm.h, A28);
    P.check("bound")                                # the oracle's u64 epochs have none: nothing changed
    jump = 0xFFFFFFF0 - 6
    for n in (1 << 31, jump - (1 << 31)):
        assert P.g.advanceEpochs(n) == 0 and P.o.advanceEpochs(n) == 0
    P.check("jumped")                                     # no origin move yet: exact
    P.run("unmap", us[0])                                 # stale since the map: copied
    for step in range(12):                                # the origin moves during these launches
        for u in P.g.dump():
            if u["base"] in (us[1], us[3]):
                P.g.dev_write(u["devptr"], np.full(128, 0x40 + step, dtype=np.uint8))
                P.o.dev_write(u["devptr"], np.full(128, 0x40 + step, dtype=np.uint8))
        P.advance()
        P.run("unmap", us[1])                             # copied every launch
        P.run("unmap", us[1])                             # ... once
        P.run("unmap", us[4])                             # read-only: never copied
        if step == 4:
            P.run("unmap", us[3])                         # current just before the move
        _check_mod_stale_epochs(P, f"step {step}")
    P.run("unmap", us[2])                                 # stale across the move: still copied
    P.run("unmap", us[3])
    _check_mod_stale_epochs(P, "after")
    assert P.g.epoch - jump > 12 - 1
    for u in us:
        P.run("release", u)
    _check_mod_stale_epochs(P, "released")
    s = P.g.stats()
    assert s["d2h_units"] == P.o.stats()["d2h_units"] >= 12 + 3


def test_unit_over_4GiB(cgcm_mod):
    """A26: an AU larger than 2^32 bytes (its size lives in the cold 64-bit column; the hot word holds
    the escape) -- interior pointers beyond 4 GiB, one-past-the-end (A7), the gap after it, through
    mapBatch (k_slots) and mapArrayDevice (k_map_pd), against the oracle.  The AU is read-only zero
    pages (PROT_READ reservation: no RAM), so activation copies 5 GiB H2D and nothing is copied back."""
    import torch
    from oracle import Oracle
    big_size = (5 << 30) + 12345
    span = big_size + (4 << 20)
    R = W.reserve_readonly(span)
    ctx = cgcm_mod.Context(0, arena_bytes=(5 << 30) + (256 << 20), flags=0)
    o = Oracle()
    P = Pair(ctx, o)
    try:
        u0, big = R, R + 0x10000
        u2 = big + big_size + 64
        for base, size in ((u0, 4096), (big, big_size), (u2, 1000)):
            assert P.g.declareAlloc(base, size, True) == 0 and P.o.declareAlloc(base, size, True) == 0
        pts = [big + (4 << 30) + 7, u0 + 8, big, big + big_size, u2 + 5, 0, big + (1 << 32), big + big_size - 1]
        st, _ = P.run("mapBatch", pts)
        assert st == 0
        P.check("mapped")
        P.run("mapBatch", [big + 8, big + big_size + 1])  # the gap after the end: UNREGISTERED
        P.check("gap")
        slots = np.array([big + (3 << 30) + 3, u2, big + big_size, 0, big + (1 << 32) - 8, u0 + 4095,
                          big + 17, big + (5 << 30)], dtype=np.uint64)
        d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
        assert P.g.mapArrayDevice(d.data_ptr(), len(slots)) == 0
        ref = slots.copy()
        assert P.o.mapSlots(ref) == 0
        assert (d.cpu().numpy().view(np.uint64) == ref).all()
        P.check("device slots mapped")
        P.advance()
        assert P.g.unmapArrayDevice(d.data_ptr(), len(slots), release=True) == 0
        assert P.o.unmapSlots(ref, release=True) == 0
        assert (d.cpu().numpy().view(np.uint64) == slots).all()
        P.run("unmapBatch", pts)
        P.run("releaseBatch", pts)
        P.check("released")
        assert all(u["refCount"] == 0 for u in P.g.dump())
    finally:
        ctx.close()
        o.close()
        W.release_reservation(R, span)


def test_compact_word_escapes(pair):
    """The forward kernel's 4-byte unit word escapes to the 8-byte hot word when a unit's size is
    >= 2^18 B or its device extent id >= 2^11 (cgcm_dev.h make_hotc): 2600 units activated by 2600
    separate map calls (one extent each), two units of 300 KB and 3 MiB, then 50,000 device slots
    over all of them mapped / unmapped+released against the oracle (mapSlots / unmapSlots)."""
    import torch
    P = pair
    buf = HostBuf(8 << 20)
    K = 2600
    bases = [buf.addr + 256 * k for k in range(K)] + [buf.addr + (1 << 20), buf.addr + (2 << 20)]
    sizes = [64 + 8 * (k % 7) for k in range(K)] + [300000, 3 << 20]
    for b, s in zip(bases, sizes):
        assert P.g.declareAlloc(b, s) == 0 and P.o.declareAlloc(b, s) == 0
    gst = [P.g.map(b)[0] for b in bases]                  # one activation (one extent) per call
    P.feed_replay()
    ost = [P.o.map(b)[0] for b in bases]
    assert gst == ost == [0] * len(bases)
    P.check("activated one by one")
    rng = np.random.default_rng(11)
    Q = 50000
    u = rng.integers(0, len(bases), Q)
    u[:2000] = rng.integers(K, K + 2, 2000)               # plenty of slots into the big units
    off = (rng.random(Q) * (np.array(sizes, dtype=np.float64)[u] + 1)).astype(np.uint64)
    slots = (np.array(bases, dtype=np.uint64)[u] + off).astype(np.uint64)
    slots[::41] = 0
    rng.shuffle(slots)
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    assert P.g.mapArrayDevice(d.data_ptr(), Q) == 0
    ref = slots.copy()
    assert P.o.mapSlots(ref) == 0
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    P.check("slots mapped")
    P.advance()
    assert P.g.unmapArrayDevice(d.data_ptr(), Q, release=True) == 0
    assert P.o.unmapSlots(ref, release=True) == 0
    assert (d.cpu().numpy().view(np.uint64) == slots).all()
    P.check("slots unmapped")
    P.run("releaseBatch", bases)
    P.check("released")


@pytest.mark.parametrize("seed,nested", [(2024, False), (7, False), (99, True)])
def test_random_array_batches(pair, seed, nested):
    _random_array_batches(pair, seed, nested)


def test_random_array_batches_lenient(cgcm_mod):
    """The same random program in lenient mode (A18) with stray (undeclared) pointers in the outers:
    they pass through both ways and are counted per call."""
    from oracle import Oracle
    ctx = cgcm_mod.Context(0, arena_bytes=1 << 28, flags=2)
    o = Oracle(2)
    try:
        _random_array_batches(Pair(ctx, o), 31, True, stray=True)
    finally:
        ctx.close()
        o.close()


@pytest.mark.parametrize("seed", [51, 52, 53, 54, 55, 56])
def test_random_array_batches_with_churn(pair, seed):
    """The batch-form program with declares / undeclares of extra leaves between calls and the CPU
    rewriting slots of outers that are not mapped (legal: A16 only forbids writes to mapped AUs), so
    outers gain pointers to new units and to units that are later undeclared."""
    _random_array_batches(pair, seed, True, churn=True)


def _random_array_batches(pair, seed, nested, stray=False, churn=False):
    """Seeded random differential run of the batch forms: mapArrays / unmapArrays / releaseArrays over
    multisets of 12 outers (repeats within a batch, SURVEY §8(b) sequential semantics), GPU writes to
    leaf units between launches, occasional unbalanced calls (NOT_MAPPED, all-or-nothing); full state
    compared with the oracle after every call."""
    P = pair
    rng = np.random.default_rng(seed)
    buf = HostBuf(1 << 20)
    leaves = [buf.addr + 0x100 * k for k in range(64)]
    outer_bases = [buf.addr + 0x10000 + 0x1000 * j for j in range(12)]
    for k, a in enumerate(leaves):
        P.declare(a, 48 + 8 * (k % 5), rng.integers(0, 255, 48 + 8 * (k % 5), dtype=np.uint8))
    outers = []
    for j in range(12):
        o = buf.addr + 0x10000 + 0x1000 * j
        n = int(rng.integers(0, 40))
        tg = [0 if rng.random() < 0.1 else leaves[int(rng.integers(0, 64))] + 8 * int(rng.integers(0, 6))
              for _ in range(n)]
        if nested and j < 3 and n:                        # outers 0-2 also point at outers 9-11
            tg[0] = outer_bases[9 + j]
        if stray and n > 1:
            tg[-1] = buf.addr + 0x80000 + 8 * j          # never declared
        P.declare(o, 8 * n + int(rng.integers(0, 8)) if n else 8, np.asarray(tg + [0], dtype=np.uint64)
                  .view(np.uint8)[:8 * n + 8])
        outers.append(o)
    held = {o: 0 for o in outers}
    rng2 = np.random.default_rng(seed + 1000)
    extra = []
    for step in range(150):
        if churn and rng2.random() < 0.25:
            rc = {u["base"]: u["refCount"] for u in P.o.dump()}
            if extra and rng2.random() < 0.4:
                b = extra[int(rng2.integers(0, len(extra)))]
                assert P.undeclare(b) == (0 if rc.get(b, 0) == 0 else -5)
                if rc.get(b, 0) == 0:
                    extra.remove(b)
            else:
                b = buf.addr + 0x40000 + 0x100 * int(rng2.integers(0, 512))
                if b not in extra:                     # (P.declare writes the host bytes first)
                    assert P.declare(b, 40, rng2.integers(0, 255, 40, dtype=np.uint8)) == 0
                    extra.append(b)
            j = int(rng2.integers(0, 12))
            o = outers[j]
            size = P.units[o]
            if rc.get(o, 0) == 0 and size >= 8 and extra:   # the CPU rewrites an unmapped outer's slot
                slot = int(rng2.integers(0, size // 8))
                v = extra[int(rng2.integers(0, len(extra)))] + int(rng2.integers(0, 41))
                host_write(o + 8 * slot, np.array([v], dtype=np.uint64))
                P.sync_host_to_oracle(o, size)
        r = rng.random()
        k = int(rng.integers(1, 6))
        if r < 0.4:
            batch = [outers[int(i)] for i in rng.integers(0, 12, k)]
            st, _ = P.run("mapArrays", batch)
            if st == 0:
                for o in batch:
                    held[o] += 1
        elif r < 0.6:
            live = [o for o in outers if held[o] > 0]
            batch = [live[int(i)] for i in rng.integers(0, len(live), k)] if live and rng.random() < 0.9 \
                else [outers[int(i)] for i in rng.integers(0, 12, k)]
            P.run("unmapArrays", batch)
        elif r < 0.85:
            live = [o for o in outers for _ in range(held[o])]
            if live and rng.random() < 0.9:
                idx = rng.choice(len(live), size=min(k, len(live)), replace=False)
                batch = [live[int(i)] for i in idx]
            else:
                batch = [outers[int(i)] for i in rng.integers(0, 12, k)]
            st = P.run("releaseArrays", batch)
            if st == 0:
                for o in batch:
                    held[o] -= 1
        else:
            for u in P.g.dump():
                if u["refCount"] > 0 and u["base"] in leaves and rng.random() < 0.3:
                    v = rng.integers(0, 255, u["size"], dtype=np.uint8)
                    P.g.dev_write(u["devptr"], v)
                    P.o.dev_write(u["devptr"], v)
            P.advance()
        P.check(f"step {step}")
    P.check_device_units()
    P.drain()


@pytest.mark.parametrize("seed", [5, 17])
def test_random_scalar_batches(pair, seed):
    _random_scalar_batches(pair, seed)


@pytest.mark.parametrize("seed", [61, 62, 63])
def test_random_scalar_batches_with_churn(pair, seed):
    """The scalar batch program with heap AUs declared / undeclared between calls (table rebuilds while
    units are mapped; undeclare of a mapped AU is BUSY)."""
    _random_scalar_batches(pair, seed, churn=True)


def _random_scalar_batches(pair, seed, churn=False):
    """Seeded random differential run of mapBatch / unmapBatch / releaseBatch over interior pointers
    with repeats inside a batch (a batch = its sequential loop: repeated unmaps copy at most once per
    epoch, repeated releases count down), heap AUs and two globals (never freed), GPU writes between
    launches, unbalanced releases (NOT_MAPPED, all-or-nothing); state compared after every call."""
    P = pair
    rng = np.random.default_rng(seed)
    buf = HostBuf(1 << 18)
    units = []
    for k in range(80):
        b, s = buf.addr + 0x200 * k, int(rng.integers(1, 60)) * 8
        P.declare(b, s, rng.integers(0, 255, s, dtype=np.uint8))
        units.append((b, s))
    for k, ro in ((0, False), (1, True)):
        b, s = buf.addr + 0x20000 + 0x400 * k, 96
        P.declare_global(f"g{seed}_{k}", b, s, ro=ro)
        units.append((b, s))
    held = {}
    rng2 = np.random.default_rng(seed + 1000)
    xbuf = HostBuf(1 << 16)
    extra = []
    for step in range(150):
        if churn and rng2.random() < 0.3:
            if extra and rng2.random() < 0.4:
                b, sz = extra[int(rng2.integers(0, len(extra)))]
                rc = {u["base"]: u["refCount"] for u in P.o.dump()}.get(b, 0)
                assert P.undeclare(b) == (0 if rc == 0 else -5)
                if rc == 0:
                    extra.remove((b, sz))
                    units.remove((b, sz))
            else:
                b = xbuf.addr + 0x100 * int(rng2.integers(0, 256))
                if all(b != e[0] for e in extra):
                    sz = 8 * int(rng2.integers(1, 32))
                    assert P.declare(b, sz, rng2.integers(0, 255, sz, dtype=np.uint8)) == 0
                    extra.append((b, sz))
                    units.append((b, sz))
        r = rng.random()
        k = int(rng.integers(1, 12))
        pick = [units[int(i)] for i in rng.integers(0, len(units), k)]
        ps = [b + int(rng.integers(0, s + 1)) for b, s in pick]
        if r < 0.35:
            st, _ = P.run("mapBatch", ps)
            if st == 0:
                for b, _s in pick:
                    held[b] = held.get(b, 0) + 1
        elif r < 0.55:
            live = [b for b, c in held.items() if c > 0]
            if live:
                P.run("unmapBatch", [live[int(i)] + 1 for i in rng.integers(0, len(live), k)])
        elif r < 0.8:
            pool = [b for b, c in held.items() for _ in range(c)]
            if pool and rng.random() < 0.9:
                idx = rng.choice(len(pool), size=min(k, len(pool)), replace=False)
                batch = [pool[int(i)] for i in idx]
            else:
                batch = [b for b, _s in pick]
            st = P.run("releaseBatch", batch)
            if st == 0:
                for b in batch:
                    held[b] -= 1
        else:
            for u in P.g.dump():
                if u["refCount"] > 0 and rng.random() < 0.3:
                    v = rng.integers(0, 255, u["size"], dtype=np.uint8)
                    P.g.dev_write(u["devptr"], v)
                    P.o.dev_write(u["devptr"], v)
            P.advance()
        P.check(f"step {step}")
    P.check_device_units()
    P.drain()


@pytest.mark.parametrize("seed", [3, 8])
def test_random_device_slices(pair, seed):
    _random_device_slices(pair, seed)


def test_random_device_slices_lenient(cgcm_mod):
    """The same random program in lenient mode (A18) with stray (undeclared) pointers in the slices."""
    from oracle import Oracle
    ctx = cgcm_mod.Context(0, arena_bytes=1 << 28, flags=2)
    o = Oracle(2)
    try:
        _random_device_slices(Pair(ctx, o), 13, stray=True)
    finally:
        ctx.close()
        o.close()


@pytest.mark.parametrize("seed", [21, 22, 23, 24])
def test_random_device_slices_with_table_churn(pair, seed):
    """The device-slice program with declares / undeclares between calls (a0: the table and its index
    are rebuilt and unit indices move while slices hold recorded shadows), new units written into slices
    that hold CPU pointers, and slices pointing at undeclared units (UNREGISTERED, all-or-nothing)."""
    _random_device_slices(pair, seed, churn=True)


def _random_device_slices(pair, seed, stray=False, churn=False):
    """Seeded random differential run of the device-array path (the hot kernels k_map_pd / k_unmap_sh
    and their fallbacks): six disjoint slices of one device buffer (odd starts, ragged lengths) are
    mapped, optionally permuted within the slice by a "GPU function" (the shadow fallback), unmapped
    with or without the fused release (then released later through releaseBatch), interleaved with
    scalar maps / releases of the same units and epoch advances; state compared after every call."""
    import torch
    P = pair
    rng = np.random.default_rng(seed)
    offs, sizes, R, span = config_C_setup(P, 3000, seed=seed)
    bounds = [(1, 700), (701, 1), (703, 2050), (2760, 33), (2800, 4096 + 3), (6900, 257)]
    total = 7200
    q, _u = W.queries(offs, sizes, total, seed + 1)
    slots = (q + np.uint64(R)).astype(np.uint64)
    slots[rng.random(total) < 0.05] = 0
    if stray:
        slots[rng.random(total) < 0.03] = np.uint64(R + span + 64)
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    ref = slots.copy()
    base = d.data_ptr()
    state = ["cpu"] * len(bounds)       # cpu: holds CPU pointers, no refs; gpu: mapped; held: CPU ptrs + refs
    own = []
    rng2 = np.random.default_rng(seed + 1000)
    xbuf = HostBuf(1 << 16)
    extra = []                          # heap units declared by the churn
    for step in range(80):
        if churn and rng2.random() < 0.25:
            if extra and rng2.random() < 0.4:
                b = extra[int(rng2.integers(0, len(extra)))]
                rc = {u["base"]: u["refCount"] for u in P.o.dump()}.get(b, 0)
                assert P.undeclare(b) == (0 if rc == 0 else -5)
                if rc == 0:
                    extra.remove(b)
            else:
                b = xbuf.addr + 0x100 * int(rng2.integers(0, 256))
                if b not in extra:                     # (P.declare writes the host bytes first)
                    assert P.declare(b, 64, rng2.integers(0, 255, 64, dtype=np.uint8)) == 0
                    extra.append(b)
            j = int(rng2.integers(0, len(bounds)))
            if state[j] == "cpu" and extra:             # point a CPU-state slot at an extra unit
                k = bounds[j][0] + int(rng2.integers(0, bounds[j][1]))
                v = np.uint64(extra[int(rng2.integers(0, len(extra)))] + int(rng2.integers(0, 65)))
                ref[k] = v
                d[k] = int(v)
        r = rng.random()
        i = int(rng.integers(0, len(bounds)))
        s0, n = bounds[i]
        if r < 0.3 and state[i] == "cpu":
            st = P.g.mapArrayDevice(base + 8 * s0, n)
            P.feed_replay()
            seg = ref[s0:s0 + n].copy()
            assert st == P.o.mapSlots(seg)
            if st == 0:
                ref[s0:s0 + n] = seg
                state[i] = "gpu"
        elif r < 0.55 and state[i] == "gpu":
            if rng.random() < 0.3 and n > 1:           # the "GPU function" permutes the slice
                perm = rng.permutation(n)
                ref[s0:s0 + n] = ref[s0:s0 + n][perm]
                d[s0:s0 + n] = d[s0:s0 + n][torch.from_numpy(perm).cuda()]
            rel = bool(rng.random() < 0.6)
            st = P.g.unmapArrayDevice(base + 8 * s0, n, release=rel)
            seg = ref[s0:s0 + n].copy()
            assert st == P.o.unmapSlots(seg, release=rel)
            if st == 0:
                ref[s0:s0 + n] = seg
                state[i] = "cpu" if rel else "held"
        elif r < 0.65 and state[i] == "held":
            nz = [int(x) for x in ref[s0:s0 + n] if x != 0]
            st = P.run("releaseBatch", nz)
            if st == 0:
                state[i] = "cpu"
        elif r < 0.8:
            j = int(rng.integers(0, len(offs)))
            p = R + int(offs[j]) + int(rng.integers(0, int(sizes[j]) + 1))
            st, _ = P.run("map", p)
            if st == 0:
                own.append(p)
        elif r < 0.9 and own:
            P.run("release", own.pop(int(rng.integers(0, len(own)))))
        else:
            P.advance()
        assert (d.cpu().numpy().view(np.uint64) == ref).all(), f"step {step}"
        P.check(f"step {step}")
    clean = True                        # unmap + release the slices still mapped, then drain the rest
    for i, (s0, n) in enumerate(bounds):
        if state[i] == "gpu":
            st = P.g.unmapArrayDevice(base + 8 * s0, n, release=True)
            seg = ref[s0:s0 + n].copy()
            assert st == P.o.unmapSlots(seg, release=True)
            if st == 0:
                ref[s0:s0 + n] = seg
                state[i] = "cpu"
            clean = clean and st == 0
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    P.check("slices unmapped")
    P.drain(shadows=clean)
    W.release_reservation(R, span)


def test_region_mixed_kinds_and_repeats(pair):
    """cgcm_regionBegin over an array outer named twice and two scalar AUs (one of them also an element
    of the outer): the hoisted calls are the sequential loop in order, regionEnd unmaps + releases each
    pointer in reverse order (Listing 4, A11); the loop body keeps its own map / release.
    Compared with the oracle running that promoted sequence explicitly."""
    P = pair
    buf = HostBuf(1 << 16)
    rows = [buf.addr + 0x200 * k for k in range(8)]
    for k, r in enumerate(rows):
        P.declare(r, 64, np.full(8, k + 1.0))
    pp = buf.addr + 0x4000
    P.declare(pp, 8 * 9, np.asarray(rows + [0], dtype=np.uint64))
    x = buf.addr + 0x5000
    P.declare(x, 128, np.arange(16, dtype=np.float64))
    ptrs = [pp, x, pp, rows[3] + 8]
    kinds = [P.g.REGION_MAPARRAY, P.g.REGION_MAP, P.g.REGION_MAPARRAY, P.g.REGION_MAP]
    assert P.g.regionBegin(ptrs, kinds) == 0
    P.feed_replay()
    for p, k in zip(ptrs, kinds):
        assert (P.o.mapArray(p) if k == P.g.REGION_MAPARRAY else P.o.map(p))[0] == 0
    P.check("region begun")
    for it in range(4):
        P.run("map", x + 8)
        for u in P.g.dump():
            if u["base"] in (rows[it], x):
                v = np.full(u["size"], 0x30 + it, dtype=np.uint8)
                P.g.dev_write(u["devptr"], v)
                P.o.dev_write(u["devptr"], v)
        P.advance()
        P.run("release", x + 8)
        P.check(f"iteration {it}")
    s, v = P.g.regionEnd()
    assert (s, v) == (0, 0)
    for p, k in reversed(list(zip(ptrs, kinds))):
        if k == P.g.REGION_MAPARRAY:
            assert P.o.unmapArray(p) == 0 and P.o.releaseArray(p) == 0
        else:
            assert P.o.unmap(p) == 0 and P.o.release(p) == 0
    P.check("region ended")
    assert all(u["refCount"] == 0 for u in P.g.dump())


@pytest.mark.parametrize("flags,program", [(1, "arrays"), (1, "scalars"), (1, "slices"), (3, "arrays"),
                                           (2, "scalars"), (3, "slices")],
                         ids=["literal-arrays", "literal-scalars", "literal-slices", "literal+lenient-arrays",
                              "lenient-scalars", "literal+lenient-slices"])
def test_random_programs_other_modes(cgcm_mod, flags, program):
    """The random differential programs under CGCM_LITERAL_EPOCH (A5's literal reading: map never sets
    the AU epoch, so the first unmap after a map copies back even without a launch) and lenient mode
    (A18), against the oracle created with the same flags."""
    from oracle import Oracle
    ctx = cgcm_mod.Context(0, arena_bytes=1 << 28, flags=flags)
    o = Oracle(flags)
    try:
        P = Pair(ctx, o)
        if program == "arrays":
            _random_array_batches(P, 41, True, stray=bool(flags & 2))
        elif program == "scalars":
            _random_scalar_batches(P, 43)
        else:
            _random_device_slices(P, 47, stray=bool(flags & 2))
    finally:
        ctx.close()
        o.close()
