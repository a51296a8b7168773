"""GPU parity of the page directory (the hot kernels' forward index) on a table built to
hit every case of its lookup: crowded pages (offsets in the overflow array, several sectors),
segments cut at the largest start-to-start distances (more candidate cuts than PD_MAXSEG), units
starting exactly on page boundaries, adjacent units (one past the end = the next base, A7), the tail
of a large unit beyond its segment's pages, pointers in gaps, before the first and after the last
unit.  Every slot is compared with the oracle (greatestLTE + A7 over a std::map) in
lenient mode, where misses pass through and are counted (A18).
"""
import numpy as np
import pytest

import workloads as W
from tests.harness import Pair

pytestmark = pytest.mark.gpu

LENIENT, FORCE_SHADOW, NO_PAGEDIR = 2, 8, 16


def layout(seed=11, nclusters=90):
    """(offsets, sizes, span) of a mixed table, offsets relative to the reservation start."""
    rng_i = [0]

    def r(n):  # seeded integers in [0, n)
        rng_i[0] += 1
        return int(W.randint(seed, 7, np.array([rng_i[0]], dtype=np.uint64), n)[0])

    offs, sizes = [], []
    pos = 4096
    for c in range(nclusters):
        kind = c % 5
        if kind == 0:      # crowded: 300 units of 1..8 B with 0..8 B gaps
            for _ in range(300):
                s = 1 + r(8)
                offs.append(pos); sizes.append(s)
                pos += s + r(9)
        elif kind == 1:    # the configs' distribution: log-uniform 16 B..64 KiB, gaps 0..4080 B
            for _ in range(200):
                s = max(16, int(16 * 4096 ** (r(1 << 20) / float(1 << 20))) // 16 * 16)
                offs.append(pos); sizes.append(s)
                pos += s + 16 * r(256)
        elif kind == 2:    # units on 32 KiB boundaries (page starts for every page size)
            pos = (pos + 32767) // 32768 * 32768
            for _ in range(50):
                s = 32768 if r(4) == 0 else 1 + r(32768)
                offs.append(pos); sizes.append(s)
                pos += 32768
        elif kind == 3:    # adjacent units
            for _ in range(100):
                s = 16 + r(241)
                offs.append(pos); sizes.append(s)
                pos += s
        else:              # one large unit (its tail lies beyond its segment's pages), then small ones
            s = (1 << 20) + r(2 << 20)
            offs.append(pos); sizes.append(s)
            pos += s + r(64)
            for _ in range(20):
                s = 16 + r(1000)
                offs.append(pos); sizes.append(s)
                pos += s + r(100)
        pos += (1 << 20) + r(7 << 20)  # candidate segment cut
    return np.array(offs, dtype=np.uint64), np.array(sizes, dtype=np.uint64), pos + 4096


def queries(offs, sizes, seed=12):
    n = len(offs)
    idx = np.arange(n, dtype=np.uint64)
    interior = offs + W.randint(seed, 1, idx, sizes)
    ends = offs + sizes
    gap_next = np.append(offs[1:], np.uint64(1 << 62)) - ends
    in_gap = ends[gap_next >= 2] + np.uint64(1)                   # misses
    q = np.concatenate([offs, offs + sizes - np.uint64(1), ends, interior, in_gap,
                        np.array([1, 4000, int(ends[-1]) + 1, int(ends[-1]) + 3000], dtype=np.uint64)])
    perm = W.permutation(seed, 2, len(q))
    return q[perm]


@pytest.fixture(scope="module")
def table():
    return layout()


@pytest.mark.parametrize("flags", [0, FORCE_SHADOW, NO_PAGEDIR], ids=["pagedir", "pagedir-shadow", "levels"])
def test_pagedir_lookup_cases(table, flags):
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    offs, sizes, span = table
    R = W.reserve_readonly(span)
    ctx = cg.Context(0, arena_bytes=1 << 30, flags=LENIENT | flags)
    o = Oracle(LENIENT)
    P = Pair(ctx, o)
    try:
        bases = offs + np.uint64(R)
        assert P.g.declareBatch(bases, sizes, readonly=True) == 0
        for b, s in zip(bases, sizes):
            assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
        info = P.g.indexInfo()
        if flags & NO_PAGEDIR:
            assert info["pd_segments"] == 0
        else:
            assert info["pd_segments"] == 64          # 108 candidate cuts, the 63 largest taken
            assert info["pd_overflow_pages"] > 0
        slots = queries(offs, sizes) + np.uint64(R)
        slots[::101] = 0
        n = len(slots)
        d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
        assert P.g.mapArrayDevice(d.data_ptr(), n) == 0
        P.feed_replay()
        ref = slots.copy()
        assert P.o.mapSlots(ref) == 0
        got = d.cpu().numpy().view(np.uint64)
        bad = np.nonzero(got != ref)[0]
        assert len(bad) == 0, [(hex(int(slots[i])), hex(int(got[i])), hex(int(ref[i]))) for i in bad[:8]]
        P.check("mapped")
        P.advance()
        assert P.g.unmapArrayDevice(d.data_ptr(), n, release=True) == 0
        assert P.o.unmapSlots(ref, release=True) == 0
        got = d.cpu().numpy().view(np.uint64)
        assert (got == ref).all() and (got == slots).all()
        P.check("unmapped")
    finally:
        ctx.close()
        o.close()
        W.release_reservation(R, span)


PG = 0x8000                                  # the largest page: 32 KiB (cgcm_dev.h PD_MAXSHIFT = 15)


def layout_max_pages():
    """Segments that exercise the largest pages (P = 15): page offsets reach PD_PAD = 0x7FFF (the padding
    value of the entry's u16 offsets) and a unit's end crosses whole pages.  Segment 0 takes P = 15;
    segment 1 has a unit starting at page offset 0x7FFF, so it must fall back to a smaller page
    (build_pd's rule)."""
    offs, sizes = [], []
    S0 = 1 << 20
    pos = S0
    for k in range(120):                     # ~2 starts per 32 KiB page, never crowded
        s = 10000 + 16 * (k % 7)
        offs.append(pos); sizes.append(s)
        pos += 15000 + 16 * (k % 5)
    pos = (pos + PG - 1) // PG * PG + S0 % PG
    big = pos                                # a unit covering whole pages, then one ending on PG - 1
    offs.append(pos); sizes.append(3 * PG + 0x1234)
    pos += 4 * PG
    offs.append(pos); sizes.append(PG - 1)   # [A, A + PG - 1]: its one-past-end is the next page start
    pos += 2 * PG
    S1 = pos + (8 << 20)                     # segment 1
    pos = S1
    offs.append(pos); sizes.append(100)
    offs.append(S1 + PG - 1); sizes.append(10)   # start at page offset 0x7FFF of a 32 KiB page
    offs.append(S1 + PG + 0x20); sizes.append(4000)
    pos = S1 + 3 * PG
    for k in range(60):
        offs.append(pos); sizes.append(4500)
        pos += 12500
    return (np.array(offs, dtype=np.uint64), np.array(sizes, dtype=np.uint64), pos + (1 << 20), S0, S1, big)


def test_pagedir_max_pages():
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    offs, sizes, span, S0, S1, big = layout_max_pages()
    R = W.reserve_readonly(span)
    ctx = cg.Context(0, arena_bytes=1 << 28, flags=LENIENT)
    o = Oracle(LENIENT)
    P = Pair(ctx, o)
    try:
        bases = offs + np.uint64(R)
        assert P.g.declareBatch(bases, sizes, readonly=True) == 0
        for b, s in zip(bases, sizes):
            assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
        info = P.g.indexInfo()
        assert info["pd_segments"] == 2
        assert info["pd_max_shift"] == 15 and info["pd_min_shift"] <= 14, info
        q = [offs, offs + sizes - np.uint64(1), offs + sizes, offs + sizes + np.uint64(1)]
        for S, npages in ((S0, 72), (S1, 40)):   # every page start, its last byte and neighbours
            A = np.uint64(S) + np.arange(npages, dtype=np.uint64) * np.uint64(PG)
            q += [A, A + np.uint64(PG - 1), A + np.uint64(PG - 2), A + np.uint64(PG // 2), A + np.uint64(PG // 2 - 1)]
        q.append(np.array([big + PG + PG - 1, big + 3 * PG + 0x1234, big + 3 * PG + 0x1235],
                          dtype=np.uint64))
        slots = np.concatenate(q) + np.uint64(R)
        n = len(slots)
        d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
        assert P.g.mapArrayDevice(d.data_ptr(), n) == 0
        P.feed_replay()
        ref = slots.copy()
        assert P.o.mapSlots(ref) == 0
        got = d.cpu().numpy().view(np.uint64)
        bad = np.nonzero(got != ref)[0]
        assert len(bad) == 0, [(hex(int(slots[i]) - R), hex(int(got[i])), hex(int(ref[i]))) for i in bad[:8]]
        P.check("mapped")
        P.advance()
        assert P.g.unmapArrayDevice(d.data_ptr(), n, release=True) == 0
        assert P.o.unmapSlots(ref, release=True) == 0
        got = d.cpu().numpy().view(np.uint64)
        assert (got == ref).all() and (got == slots).all()
        P.check("unmapped")
    finally:
        ctx.close()
        o.close()
        W.release_reservation(R, span)


@pytest.mark.parametrize("flags", [0, FORCE_SHADOW], ids=["pagedir", "pagedir-shadow"])
def test_pagedir_activation_free_cycles(flags):
    """k_map_pd's translations must follow every activation (new extent), free and re-activation of
    the units it lands on.  Rounds of mapArrayDevice / unmapArrayDevice(release) over different unit
    subsets, with a pinned subset held across rounds by a second array; every translation, refcount
    and epoch vs the oracle."""
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    U = 3000
    offs, sizes, span = W.table_layout(U, 21)
    R = W.reserve_readonly(span)
    ctx = cg.Context(0, arena_bytes=1 << 30, flags=flags)
    o = Oracle()
    P = Pair(ctx, o)
    try:
        bases = offs + np.uint64(R)
        assert P.g.declareBatch(bases, sizes, readonly=True) == 0
        for b, s in zip(bases, sizes):
            assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
        assert P.g.indexInfo()["pd_segments"] > 0
        pins = (offs[::7] + np.uint64(R)).astype(np.uint64)       # held across all rounds
        dp = torch.from_numpy(pins.view(np.int64).copy()).cuda()
        assert P.g.mapArrayDevice(dp.data_ptr(), len(pins)) == 0
        P.feed_replay()
        pref = pins.copy()
        assert P.o.mapSlots(pref) == 0
        assert (dp.cpu().numpy().view(np.uint64) == pref).all()
        for r in range(4):
            q, u = W.queries(offs, sizes, 20000 + 101 * r, 30 + r)
            keep = (u % np.uint64(4)) != np.uint64(r)              # a different subset each round
            slots = (q[keep] + np.uint64(R)).astype(np.uint64)
            slots[::53] = 0
            n = len(slots)
            d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
            assert P.g.mapArrayDevice(d.data_ptr(), n) == 0
            P.feed_replay()
            ref = slots.copy()
            assert P.o.mapSlots(ref) == 0
            got = d.cpu().numpy().view(np.uint64)
            bad = np.nonzero(got != ref)[0]
            assert len(bad) == 0, (r, [(hex(int(got[i])), hex(int(ref[i]))) for i in bad[:4]])
            if r % 2:
                P.check(f"round {r} mapped")
            P.advance()
            assert P.g.unmapArrayDevice(d.data_ptr(), n, release=True) == 0
            assert P.o.unmapSlots(ref, release=True) == 0
            assert (d.cpu().numpy().view(np.uint64) == slots).all()
            P.check(f"round {r} released")
        P.advance()
        assert P.g.unmapArrayDevice(dp.data_ptr(), len(pins), release=True) == 0
        assert P.o.unmapSlots(pref, release=True) == 0
        P.check("pins released")
        assert all(x["refCount"] == 0 for x in P.g.dump())
    finally:
        ctx.close()
        o.close()
        W.release_reservation(R, span)
