"""Pins for the oracle's coherence groups (NEXT-3, reading A31 of DESIGN.md §3): several devices share one
host memory; each keeps its own table, refcounts and epochs (per-GPU epochs); an activation on device d
copies an AU from a peer c's device copy instead of the host when c holds it active and dirty -- c
launched a GPU function since the AU became coherent there, so c's unmap would copy it back (Alg. 2,
P:L216-219) -- and writable.  The paper is single-GPU; the mapping semantics extended are
P:L181-189.

Expected values are hand counts and byte patterns written by the test; the equivalence pin compares the
group's result with a single oracle that moves the data through the host (unmap, then map), which is
what CGCM does without peers."""
import numpy as np

from oracle import Oracle, OK


def group(n=2):
    os_ = [Oracle() for _ in range(n)]
    for o in os_:
        assert o.groupJoin(os_[0]) == OK
    return os_


def close(os_):
    for o in reversed(os_):
        o.close()


def dev_bytes(o, base, n):
    u = {x["base"]: x for x in o.dump()}[base]
    return o.dev_read(u["devptr"], n).tobytes()


def dev_fill(o, base, n, v):
    u = {x["base"]: x for x in o.dump()}[base]
    o.dev_write(u["devptr"], np.full(n, v, dtype=np.uint8))


def test_dirty_peer_copy_hand_counts():
    A, B = group()
    try:
        X, n = 0x10000, 64
        for o in (A, B):
            assert o.declareAlloc(X, n) == OK
        A.host_write(X, np.full(n, 1, dtype=np.uint8))          # shared host: B sees it too
        assert B.host_read(X, n).tobytes() == bytes([1]) * n
        assert A.map(X)[0] == OK
        dev_fill(A, X, n, 2)                                     # a GPU function on A writes X
        A.advanceEpoch()                                         # A launched: X dirty on A
        assert B.map(X)[0] == OK
        assert dev_bytes(B, X, n) == bytes([2]) * n              # from A's device, not the host's 1s
        sb = B.stats()
        assert (sb["peer_units"], sb["peer_bytes"], sb["h2d_units"]) == (1, n, 0)
        dev_fill(B, X, n, 3)
        B.advanceEpoch()
        assert B.unmap(X) == OK                                  # B's epoch gate: copy back
        assert A.host_read(X, n).tobytes() == bytes([3]) * n
        assert B.stats()["d2h_units"] == 1
        assert A.unmap(X) == OK                                  # A's copy is stale on A too: copied back
        assert A.host_read(X, n).tobytes() == bytes([2]) * n     # (concurrent writers: last unmap wins)
        for o in (A, B):
            assert o.release(X) == OK
    finally:
        close([A, B])


def test_clean_or_readonly_or_unmapped_peer_is_not_a_source():
    A, B, Cc = group(3)
    try:
        X, Y, Z, n = 0x10000, 0x20000, 0x30000, 32
        for o in (A, B, Cc):
            assert o.declareAlloc(X, n) == OK
            assert o.declareAlloc(Y, n, readonly=True) == OK
            assert o.declareAlloc(Z, n) == OK
        for b in (X, Y, Z):
            A.host_write(b, np.full(n, 5, dtype=np.uint8))
        for b in (X, Y, Z):
            assert A.map(b)[0] == OK
        assert B.map(X)[0] == OK                                 # A mapped X but launched nothing: clean
        assert dev_bytes(B, X, n) == bytes([5]) * n and B.stats()["peer_units"] == 0
        dev_fill(A, Y, n, 9)
        dev_fill(A, Z, n, 9)
        A.advanceEpoch()
        assert B.map(Y)[0] == OK                                 # read-only: never dirty, host is current
        assert dev_bytes(B, Y, n) == bytes([5]) * n
        assert A.unmap(Z) == OK and A.release(Z) == OK           # copied back, then gone from A
        assert B.map(Z)[0] == OK                                 # from the host, which now holds A's 9s
        assert dev_bytes(B, Z, n) == bytes([9]) * n and B.stats()["peer_units"] == 0
        dev_fill(B, Z, n, 7)
        B.advanceEpoch()
        assert Cc.map(Z)[0] == OK                                # B is the dirty holder now
        assert dev_bytes(Cc, Z, n) == bytes([7]) * n and Cc.stats()["peer_units"] == 1
    finally:
        close([A, B, Cc])


def test_peer_copy_equals_the_host_round_trip():
    """A pipeline of two GPU functions on two devices: the group (peer copy) ends with the same host
    bytes as one oracle that hands the data over through the host, and moves fewer host bytes."""
    rng = np.random.default_rng(3)
    units = [(0x10000 + 0x1000 * k, 64 + 8 * k) for k in range(6)]
    init = {b: rng.integers(0, 255, n, dtype=np.uint8) for b, n in units}

    def gpu_fn(o, b, n, salt):                                   # the "GPU function": y = x * 3 + salt
        x = o.dev_read({u["base"]: u for u in o.dump()}[b]["devptr"], n).astype(np.uint16)
        dev_fill_bytes(o, b, ((x * 3 + salt) % 256).astype(np.uint8))

    def dev_fill_bytes(o, b, v):
        o.dev_write({u["base"]: u for u in o.dump()}[b]["devptr"], v)

    A, B = group()
    try:
        for o in (A, B):
            for b, n in units:
                assert o.declareAlloc(b, n) == OK
        for b, n in units:
            A.host_write(b, init[b])
        for b, n in units:
            assert A.map(b)[0] == OK
            gpu_fn(A, b, n, 1)
        A.advanceEpoch()
        for b, n in units:                                       # B takes over while A still holds them
            assert B.map(b)[0] == OK
            gpu_fn(B, b, n, 2)
            assert A.release(b) == OK                            # A drops its copy without unmapping
        B.advanceEpoch()
        for b, n in units:
            assert B.unmap(b) == OK and B.release(b) == OK
        got = {b: A.host_read(b, n).tobytes() for b, n in units}
        moved = sum(o.stats()["h2d_bytes"] + o.stats()["d2h_bytes"] for o in (A, B))
    finally:
        close([A, B])
    S = Oracle()
    try:
        for b, n in units:
            assert S.declareAlloc(b, n) == OK
            S.host_write(b, init[b])
        for b, n in units:
            assert S.map(b)[0] == OK
            gpu_fn(S, b, n, 1)
        S.advanceEpoch()
        for b, n in units:                                       # hand over through the host
            assert S.unmap(b) == OK and S.release(b) == OK
            assert S.map(b)[0] == OK
            gpu_fn(S, b, n, 2)
        S.advanceEpoch()
        for b, n in units:
            assert S.unmap(b) == OK and S.release(b) == OK
        ref = {b: S.host_read(b, n).tobytes() for b, n in units}
        moved_s = S.stats()["h2d_bytes"] + S.stats()["d2h_bytes"]
    finally:
        S.close()
    assert got == ref
    total = sum(n for _, n in units)
    assert moved == 2 * total and moved_s == 4 * total        # one H2D + one D2H vs two of each
