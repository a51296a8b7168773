"""Transfer planning on the device (activation packs, copy-back runs; cgcm_dev.h PackDesc / CopyRun): lists
of >= 2^16 units are planned by segmented scans on the GPU and the host issues one DMA per pack / run.
Parity against the oracle on a table built to exercise every planning rule: host gaps of 0 (adjacent
units: one run), small gaps (a pack with gaps: gathered through pinned staging), gaps above 64 KiB (new
pack), 64-MiB window changes (new pack), array-mapped units inside the copy-back list (reverse
translated, A12), read-only units (never copied back), NULL slots.  Everything the pair harness compares
(translations, refcounts, epochs, copy counters, extents, host bytes) after every call."""
import numpy as np
import pytest

from tests.harness import Pair, HostBuf

pytestmark = pytest.mark.gpu

N = 70000


def layout(seed=11):
    rng = np.random.default_rng(seed)
    sizes = (16 * rng.integers(1, 17, N)).astype(np.uint64)            # 16..256 B
    gaps = np.where(rng.random(N) < 0.5, 0, 16 * rng.integers(1, 20, N)).astype(np.uint64)
    gaps[rng.random(N) < 0.001] = 96 << 10                             # > 64 KiB: a new pack
    offs = np.zeros(N, dtype=np.uint64)
    offs[1:] = np.cumsum(sizes[:-1] + gaps[:-1])
    return offs, sizes, int(offs[-1] + sizes[-1])


@pytest.fixture
def P():
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    ctx = cg.Context(0, arena_bytes=1 << 30)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    ctx.close()
    o.close()


def test_planned_activation_and_copy_back(P):
    import torch
    offs, sizes, span = layout()
    W = 64 << 20                              # the planner's pack window: make the span cross one
    buf = HostBuf(span + W + (1 << 20))
    rng = np.random.default_rng(5)
    img = rng.integers(0, 255, span, dtype=np.uint8)
    cross = (buf.addr + span // 2 + W - 1) // W * W      # a window boundary inside [addr + span/2, + W)
    base0 = (cross - span // 2) // 256 * 256
    assert buf.addr <= base0 and base0 + span <= buf.addr + len(buf.arr)
    bases = offs + np.uint64(base0)
    ro = rng.random(N) < 0.05
    from tests.harness import host_write
    host_write(base0, img)
    for ro_val in (False, True):
        sel = np.flatnonzero(ro == ro_val)
        assert P.g.declareBatch(bases[sel], sizes[sel], readonly=ro_val) == 0
    for b, s, r in zip(bases.tolist(), sizes.tolist(), ro.tolist()):
        assert P.o.declareAlloc(b, s, readonly=r) == 0
    P.o.host_write(base0, img)
    for b, s in zip(bases.tolist(), sizes.tolist()):
        P.units[b] = s
    # two small array outers (their own AUs, outside the table span) whose slots point into the table
    obuf = HostBuf(1 << 16)
    outers = [obuf.addr + 0x1000 * k for k in range(2)]
    for k, o in enumerate(outers):
        tgt = np.asarray([int(bases[(k * 977 + 31 * i) % N]) + 8 * (i % 2) for i in range(16)], dtype=np.uint64)
        assert P.declare(o, 8 * 16, tgt) == 0
    # the device array: every unit once (interior pointers), NULLs, and the two outers
    q = bases + (np.arange(N, dtype=np.uint64) % sizes)
    q[::1000] = 0
    q = np.concatenate([q, np.asarray(outers, dtype=np.uint64)])
    d = torch.from_numpy(q.view(np.int64).copy()).cuda()
    for o in outers:
        P.run("mapArray", o)                  # array-mapped before the big map: they hold references
    P.check("outers")
    st = P.g.mapArrayDevice(d.data_ptr(), len(q))
    P.feed_replay()
    ref = q.copy()
    assert st == P.o.mapSlots(ref) == 0
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    P.check("planned activation")
    P.check_device_units()
    # a "GPU function" writes every writable unit
    for u in P.g.dump():
        if u["devptr"] and not (u["flags"] & 2) and u["base"] not in outers:
            v = np.full(u["size"], (u["base"] >> 4) & 0xFF, dtype=np.uint8)
            P.g.dev_write(u["devptr"], v)
            P.o.dev_write(u["devptr"], v)
    P.advance()
    st = P.g.unmapArrayDevice(d.data_ptr(), len(q), release=False)
    seg = ref.copy()
    assert st == P.o.unmapSlots(seg, release=False) == 0
    assert (d.cpu().numpy().view(np.uint64) == seg).all()
    P.check("planned copy-back")
    nz = [int(x) for x in seg if x]
    assert P.run("releaseBatch", nz) == 0
    for o in outers:
        P.run("unmapArray", o)
        P.run("releaseArray", o)
    P.check("released")
    assert P.check_balance("end")
