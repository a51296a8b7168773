"""Asynchronous releases (runtime.cpp `release_arrays_async`): a releaseArray that consumes the references an
asynchronous A9 re-map added (a lease) is queued without a host wait; every other release takes the general
path.  None of this may be observable: after every call the full state (refcounts, epochs, flags, copies,
host bytes, statistics) equals the oracle's (Alg. 3: release = refCount - 1, free at 0; A9: a
re-map of an array-mapped outer only adds references).

Each sequence below either keeps a lease valid (the queued path must give the oracle's state) or breaks it
(another release in between, more releases than re-maps, a table change) so that the general path has to
find a unit reaching 0, an underflow or a freed copy.
"""
import numpy as np
import pytest

from tests.harness import Pair
from tests.test_gpu_parity import setup_A

pytestmark = pytest.mark.gpu


@pytest.fixture(params=[0, 8], ids=["auto", "shadow"])
def P(request):
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    ctx = cg.Context(0, arena_bytes=1 << 30, flags=request.param)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    p.check_balance()
    ctx.close()
    o.close()


def test_leased_releases_match_the_oracle(P):
    rows, pp, _ = setup_A(P, 16, 8)
    P.run("mapArray", pp)                 # the array mapping (general path)
    for depth in (1, 2, 3):
        for _ in range(depth):
            P.run("mapArray", pp)         # queued re-maps: one lease each
        P.check(f"after {depth} re-maps")
        for _ in range(depth):
            P.run("releaseArray", pp)     # queued releases consume them
            P.check("leased release")
    P.run("unmapArray", pp)
    P.run("releaseArray", pp)             # no lease left: the general path frees everything
    P.check("end")


def test_lease_broken_by_an_element_release(P):
    rows, pp, _ = setup_A(P, 8, 8)
    P.run("mapArray", pp)
    P.run("map", rows[3])                 # an extra reference on one element
    P.run("mapArray", pp)                 # lease
    P.run("release", rows[3])             # another release: the lease no longer proves anything
    P.run("releaseArray", pp)             # general path
    P.check("after the broken lease")
    P.run("releaseArray", pp)             # last reference: frees the outer and every element
    P.check("end")


def test_more_releases_than_leases(P):
    rows, pp, _ = setup_A(P, 8, 8)
    P.run("mapArray", pp)
    P.run("mapArray", pp)
    P.run("releaseArray", pp)             # leased
    P.run("releaseArray", pp)             # general path, reaches 0
    st = P.run("releaseArray", pp)        # nothing left: NOT_MAPPED on both sides, state unchanged
    assert st != 0
    P.check("end")


def test_lease_survives_epochs_and_kernels_but_not_table_changes(P):
    rows, pp, vals = setup_A(P, 8, 8)
    P.run("mapArray", pp)
    P.run("mapArray", pp)
    P.advance()                           # GPU function launches do not release references
    P.run("releaseArray", pp)             # leased
    P.run("mapArray", pp)                 # lease again ...
    extra = P.malloc(64, np.arange(8, dtype=np.uint64))   # ... then a declaration changes the table
    P.run("releaseArray", pp)
    P.check("after the table change")
    P.run("unmapArray", pp)
    P.run("releaseArray", pp)
    P.check("end")
