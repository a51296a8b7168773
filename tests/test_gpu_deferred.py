"""Deferred references: a forward map of a device array with a shadow records the
reference of each slot whose unit is already active in the slot's shadow word instead of adding it to
the unit's refcount; the matching unmapArrayDevice(CGCM_RELEASE) drops it, and every other call first
adds it to the refcount.  None of this may be observable: after every call the full state (refcounts,
epochs, active flags, copies, host bytes, stats) equals the oracle's, which counts every reference
("Mapping a pointer ... increases ... reference count"; Alg. 3 frees at zero).

Each case below is a sequence where a wrong deferral would show: a unit freed while a deferred
reference still holds it, a refcount off by the deferred count, a leaked copy, or a reference lost
when a GPU function rewrote a slot.
"""
import numpy as np
import pytest

import workloads as W
from tests.harness import Pair

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


def setup(P, U=3000, Q=(1 << 16) + 5, seed=3):
    import torch
    offs, sizes, span = W.table_layout(U, seed)
    R = W.reserve_readonly(span)
    bases = offs + np.uint64(R)
    assert P.g.declareBatch(bases, sizes, readonly=True) == 0
    for b, s in zip(bases, sizes):
        assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
    q, _ = W.queries(offs, sizes, Q, seed)
    slots = (q + np.uint64(R)).astype(np.uint64)
    slots[::89] = 0
    d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
    return bases, sizes, R, span, slots, d


def gmap(P, d, s0, n, ref):
    st = P.g.mapArrayDevice(d.data_ptr() + 8 * s0, n)
    P.feed_replay()
    seg = ref[s0:s0 + n].copy()
    assert st == P.o.mapSlots(seg)
    if st == 0:
        ref[s0:s0 + n] = seg
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    return st


def gunmap(P, d, s0, n, ref, release):
    st = P.g.unmapArrayDevice(d.data_ptr() + 8 * s0, n, release=release)
    seg = ref[s0:s0 + n].copy()
    assert st == P.o.unmapSlots(seg, release=release)
    if st == 0:
        ref[s0:s0 + n] = seg
    assert (d.cpu().numpy().view(np.uint64) == ref).all()
    return st


def test_deferred_released_by_matching_unmap(P):
    """Units active through a pin slice; a second slice over the same units defers its references;
    its release-unmap drops them; the pins keep every unit active; then the pins go and all is freed."""
    bases, sizes, R, span, slots, d = setup(P)
    ref = slots.copy()
    n = len(slots)
    pins = n // 2
    assert gmap(P, d, 0, pins, ref) == 0            # activations: ordinary references
    P.check("pins")
    assert gmap(P, d, pins, n - pins, ref) == 0     # units already active: deferred where so
    P.check("deferred map")                         # dumpTable materialises: refcounts exact
    P.advance()
    assert gunmap(P, d, pins, n - pins, ref, True) == 0
    P.check("deferred released")
    P.advance()
    assert gunmap(P, d, 0, pins, ref, True) == 0
    P.check("pins released")
    assert P.check_balance("end")
    W.release_reservation(R, span)


def test_deferred_then_other_calls(P):
    """Between the deferring map and its unmap: a scalar map/release of the same units, a table
    declare, an unmap WITHOUT release, a release through releaseBatch -- each must see exact counts."""
    bases, sizes, R, span, slots, d = setup(P, Q=40000)
    ref = slots.copy()
    n = len(slots)
    assert gmap(P, d, 0, 20000, ref) == 0
    P.check("a")
    # slice B deferred, then a scalar release of a unit B references: must not free it
    assert gmap(P, d, 20000, 20000, ref) == 0
    hp = int(slots[20001] if slots[20001] else slots[20002])
    P.run("map", hp)
    P.run("release", hp)
    P.check("scalar in between")
    # unmap B without release: its deferred references become ordinary ones
    P.advance()
    assert gunmap(P, d, 20000, 20000, ref, False) == 0
    P.check("unmapped, references held")
    nz = [int(x) for x in ref[20000:40000] if x]
    assert P.run("releaseBatch", nz) == 0
    P.check("released by batch")
    # map B again (deferred), declare a new unit (table rebuild), then release-unmap B
    assert gmap(P, d, 20000, 20000, ref) == 0
    extra = W.reserve_readonly(1 << 16)
    assert P.declare(extra, 64, readonly=True) == 0
    P.advance()
    assert gunmap(P, d, 20000, 20000, ref, True) == 0
    P.check("after declare")
    assert gunmap(P, d, 0, 20000, ref, True) == 0
    P.check("end")
    assert P.check_balance("end")
    W.release_reservation(extra, 1 << 16)
    W.release_reservation(R, span)


def test_deferred_slots_rewritten_by_gpu(P):
    """A GPU function permutes a deferred slice, overwrites some slots with other valid pointers, and
    writes NULL into others: the references taken by the map stay with the units the map saw (they
    are materialised), the release goes to the units the slots now point to (oracle semantics)."""
    import torch
    bases, sizes, R, span, slots, d = setup(P, Q=30000)
    ref = slots.copy()
    assert gmap(P, d, 0, 15000, ref) == 0           # pins (activations)
    assert gmap(P, d, 15000, 15000, ref) == 0       # deferred
    rng = np.random.default_rng(7)
    seg = ref[15000:30000].copy()
    perm = rng.permutation(len(seg))
    seg = seg[perm]
    seg[rng.random(len(seg)) < 0.02] = 0                           # NULL written by the GPU
    pick = np.flatnonzero(rng.random(len(seg)) < 0.02)
    seg[pick] = ref[rng.integers(0, 15000, len(pick))]              # pointers into pinned units
    ref[15000:30000] = seg
    d[15000:30000] = torch.from_numpy(seg.view(np.int64).copy()).cuda()
    P.advance()
    st = gunmap(P, d, 15000, 15000, ref, True)
    P.check(f"rewritten slice unmapped ({st})")
    st2 = gunmap(P, d, 0, 15000, ref, True)          # (may fail: the rewritten slice released its units)
    P.check(f"pins unmapped ({st2})")
    P.drain(shadows=st2 == 0)
    W.release_reservation(R, span)


def test_deferring_map_that_fails_rolls_back(P):
    """A deferring map over a slice with one unregistered pointer fails (strict): nothing changes."""
    bases, sizes, R, span, slots, d = setup(P, Q=20000)
    ref = slots.copy()
    assert gmap(P, d, 0, 10000, ref) == 0
    P.check("pins")
    bad = int(R) + int(span) + 4096                                # past the reservation: no AU
    ref2 = ref.copy()
    ref2[17777] = bad
    d[17777] = bad
    st = gmap(P, d, 10000, 10000, ref2)
    assert st == -2                                                # CGCM_E_UNREGISTERED
    P.check("failed map")
    d[17777] = int(slots[17777])
    assert gmap(P, d, 10000, 10000, ref) == 0
    P.advance()
    assert gunmap(P, d, 10000, 10000, ref, True) == 0
    assert gunmap(P, d, 0, 10000, ref, True) == 0
    P.check("end")
    assert P.check_balance("end")
    W.release_reservation(R, span)
