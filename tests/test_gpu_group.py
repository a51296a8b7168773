"""Coherence groups on the GPU (NEXT-3, reading A31; include/cgcm.h "coherence groups"): two and three
CGCM contexts on one device (stand-ins for GPUs of one box: own tables, arenas, streams and epochs),
joined in a group, against oracles joined in a group (shared host memory, own devices).  An activation
on one context copies an AU from a peer's dirty device copy instead of the host; everything the pair
harness compares -- refcounts, per-context epochs, copies (h2d / d2h / peer units and bytes), device
bytes and host bytes -- must equal the oracles' after every call."""
import numpy as np
import pytest

from tests.harness import Pair, HostBuf

pytestmark = pytest.mark.gpu


@pytest.fixture
def grp(request):
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    n = getattr(request, "param", 2)
    g = cg.group_create()
    ctxs = [cg.Context(0, arena_bytes=1 << 28) for _ in range(n)]
    os_ = [Oracle() for _ in range(n)]
    for c, o in zip(ctxs, os_):
        assert c.groupJoin(g) == 0
        assert o.groupJoin(os_[0]) == 0
    pairs = [Pair(c, o, switch=True) for c, o in zip(ctxs, os_)]
    yield pairs
    for c in ctxs:
        c.make_current()
        c.groupLeave()
        c.close()
    assert cg.group_destroy(g) == 0
    for o in reversed(os_):
        o.close()


def declare_all(pairs, base, size, data, readonly=False):
    for P in pairs:
        assert P.declare(base, size, data, readonly=readonly) == 0


def dev_fill(P, base, v):
    u = {x["base"]: x for x in P.g.dump()}[base]
    b = np.full(u["size"], v, dtype=np.uint8)
    P.g.dev_write(u["devptr"], b)
    P.o.dev_write(u["devptr"], b)


def test_handoff_through_a_dirty_peer(grp):
    A, B = grp
    buf = HostBuf(1 << 16)
    X, Y = buf.addr + 0x100, buf.addr + 0x2000
    declare_all(grp, X, 256, np.full(256, 1, dtype=np.uint8))
    declare_all(grp, Y, 96, np.full(96, 4, dtype=np.uint8), readonly=True)
    A.run("map", X)
    A.run("map", Y)
    dev_fill(A, X, 2)                        # a GPU function on A writes X
    A.advance()                              # X dirty on A; Y read-only: never dirty
    B.run("map", X + 8)                      # from A's device copy (peer), not the host's 1s
    B.run("map", Y)                          # from the host
    for P in grp:
        P.check("B mapped")
        P.check_device_units()
    assert B.g.stats()["peer_units"] == 1 and B.g.stats()["h2d_units"] == 1
    dev_fill(B, X, 3)
    B.advance()
    B.run("unmap", X)                        # B's epoch gate: copied back (3s)
    A.run("release", X)                      # A drops its copy without unmapping
    for P in grp:
        P.check("handed off")
    B.run("release", X + 8)
    for P in grp:
        P.run("release", Y)
        P.check("end")
        assert P.check_balance("end")


@pytest.mark.parametrize("grp", [3], indirect=True)
def test_clean_peers_and_chains(grp):
    """A clean holder is no source; the first dirty member in join order is; after an unmap the host is
    current again."""
    A, B, Cc = grp
    buf = HostBuf(1 << 20)
    units = [buf.addr + 0x1000 * k for k in range(8)]
    for k, u in enumerate(units):
        declare_all(grp, u, 64 + 32 * k, np.full(64 + 32 * k, k + 1, dtype=np.uint8))
    for u in units:
        A.run("map", u)                     # A holds all, clean
    for u in units[:4]:
        B.run("map", u)                     # clean holder: from the host
    assert B.g.stats()["peer_units"] == 0
    for u in units[4:]:
        dev_fill(A, u, 0x50)
    A.advance()                             # all of A's units dirty now
    for u in units[4:]:
        B.run("map", u)                     # from A
    assert B.g.stats()["peer_units"] == 4
    for u in units[4:6]:
        dev_fill(B, u, 0x60)
    B.advance()
    for u in units[4:]:
        Cc.run("map", u)                    # A is first in join order and dirty: from A (0x50)
    for P in grp:
        P.check("C mapped")
        P.check_device_units()
    for u in units[4:]:
        A.run("unmap", u)                   # A's copy back: host = 0x50
        A.run("release", u)
    for P in grp:
        P.check("A unmapped")
    for u in units[4:]:
        Cc.run("release", u)
        Cc.run("map", u)                    # B is now the only dirty holder: from B
    for P in grp:
        P.check("C re-mapped")
        P.check_device_units()
    for P in grp:
        P.drain()
