"""Batched table merge (NEXT-1: the run-time keeps allocInfoMap current as the program allocates):
declarations between calls are appended to the device table as delta units instead of a rebuild, and
every lookup path (page-directory hot kernels, generic slot kernel, reverse lookups, outer-pointer lookups,
glue kernels) consults them where the main table misses (A7's one-past-the-end rule is kept by rebuilding
instead when a declaration starts exactly where a main unit ends).
Compared with the oracle after every call, on a config-C-shaped page-directory table with declarations
placed in its gaps -- including a delta unit starting exactly at a main unit's end and a main unit starting
exactly at a delta unit's end (one-past-the-end pointers resolve to the unit with the greater base; a
declaration touching a main unit's end takes a rebuild instead of the merge)."""
import numpy as np
import pytest

import workloads as W
from tests.harness import Pair, HostBuf

pytestmark = pytest.mark.gpu


@pytest.fixture(params=[0, 8], ids=["auto", "shadow"])
def P(request):
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    ctx = cg.Context(0, arena_bytes=1 << 30, flags=request.param)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    ctx.close()
    o.close()


def test_declares_between_batches_are_merged(P):
    import torch
    U = 4000
    rng = np.random.default_rng(9)
    sizes = (16 * rng.integers(4, 64, U)).astype(np.uint64)
    gaps = (16 * rng.integers(8, 40, U)).astype(np.uint64)               # >= 128 B between main units
    offs = np.zeros(U, dtype=np.uint64)
    offs[1:] = np.cumsum(sizes[:-1] + gaps[:-1])
    span = int(offs[-1] + sizes[-1]) + 4096
    buf = HostBuf(span)
    base0 = buf.addr
    img = rng.integers(0, 255, span, dtype=np.uint8)
    from tests.harness import host_write
    host_write(base0, img)
    bases = offs + np.uint64(base0)
    assert P.g.declareBatch(bases, sizes) == 0
    for b, s in zip(bases.tolist(), sizes.tolist()):
        assert P.o.declareAlloc(b, s) == 0
    P.o.host_write(base0, img)
    for b, s in zip(bases.tolist(), sizes.tolist()):
        P.units[b] = s
    P.check("main table")
    assert P.g.indexInfo()["pd_segments"] >= 1
    merges0 = P.g.stats()["table_merges"]
    d_units = []
    for rnd in range(4):
        # declarations in gaps: touching the previous unit's end, touching the next unit's start, free-standing
        new = []
        for k in rng.choice(U - 1, 12, replace=False):
            end = int(bases[k] + sizes[k])
            nxt = int(bases[k + 1])
            room = nxt - end
            # odd rounds include units touching a main unit's end (those rebuild the table), even rounds
            # only units the delta merge takes
            kind = k % 3 if rnd % 2 else 1 + k % 2
            if kind == 0:
                b, s = end, 16                          # starts exactly at a main unit's end
            elif kind == 1:
                b, s = nxt - 32, 32                     # ends exactly where the next main unit starts
            else:
                b, s = end + 48, 16
            if s + 16 > room or any(abs(b - x) < 64 for x, _ in d_units + new):
                continue
            new.append((b, s))
        for b, s in new:
            assert P.declare(b, s) == 0
        d_units += new
        # a device array over main units, delta units (interior, start, one past the end), misses in gaps
        q = [int(bases[i]) + int(rng.integers(0, int(sizes[i]) + 1)) for i in rng.integers(0, U, 3000)]
        for b, s in d_units:
            q += [b, b + s // 2, b + s]
        q = np.asarray(q, dtype=np.uint64)
        d = torch.from_numpy(q.view(np.int64).copy()).cuda()
        st = P.g.mapArrayDevice(d.data_ptr(), len(q))
        P.feed_replay()
        ref = q.copy()
        assert st == P.o.mapSlots(ref) == 0
        assert (d.cpu().numpy().view(np.uint64) == ref).all(), f"round {rnd}: translations differ"
        P.check(f"round {rnd} mapped")
        pick = [b for b, s in d_units[:3]] + [int(bases[5])]
        for p_ in pick:
            P.run("map", p_ + 1)                         # scalar paths (lookup_points) see them too
        P.advance()
        st = P.g.unmapArrayDevice(d.data_ptr(), len(q), release=True)
        seg = ref.copy()
        assert st == P.o.unmapSlots(seg, release=True) == 0
        assert (d.cpu().numpy().view(np.uint64) == q).all()
        for p_ in pick:
            P.run("unmap", p_ + 1)
            P.run("release", p_ + 1)
        P.check(f"round {rnd} unmapped")
    st = P.g.stats()
    assert st["table_merges"] > merges0 and st["table_rebuilds"] > 1    # both paths taken
    # an undeclare of a delta unit: the next call rebuilds (and still agrees)
    b, s = d_units[0]
    assert P.undeclare(b) == 0
    P.run("map", int(bases[7]))
    P.run("release", int(bases[7]))
    P.check("after undeclare")
    assert P.check_balance("end")
