"""Pins for the oracle's map / unmap / release and array variants (SURVEY §8(c) "What pins each part").

Every expected value here comes from the paper's statements or from mathematics, never from the
oracle itself:
  * closed form of Alg. 1's return value  devptr + (ptr - base)
  * pointer differences preserved inside an AU
  * aliases map into ONE GPU AU
  * copy only on activation (A2)
  * at most one copy-back per AU per epoch; none if up to date
  * read-only never copied back; globals never freed, same address
  * unmapArray o mapArray is the identity on a legal pointer array (R13)
  * a permutation of device slots comes back as the same permutation        (reverse lookup, a3)
"""
import numpy as np
import pytest

from oracle import (Oracle, OK, E_INVALID, E_UNREGISTERED, E_OVERLAP, E_NOT_MAPPED, E_BUSY,
                    E_DUPLICATE, LITERAL_EPOCH, UNIT_ARRAYMAPPED, UNIT_ACTIVE)


def unit(o, base):
    return {u["base"]: u for u in o.dump()}[base]


def snapshot(o, regions):
    return (o.dump(), o.stats(), o.epoch, [o.host_read(b, n).tobytes() for b, n in regions])


def test_map_closed_form_and_invariants(oracle):
    o = oracle
    bases = [0x10000 + 0x1000 * k + 8 * k for k in range(8)]
    sizes = [64 + 40 * k for k in range(8)]
    for b, s in zip(bases, sizes):
        assert o.declareAlloc(b, s) == OK
    outs = {}
    for b, s in zip(bases, sizes):
        for off in (0, 1, s // 2, s):            # interior and one-past-end (A7)
            st, t = o.map(b + off)
            assert st == OK
            outs[(b, off)] = t
    for b, s in zip(bases, sizes):
        u = unit(o, b)
        assert u["refCount"] == 4                  # +1 per map call
        for off in (0, 1, s // 2, s):
            assert outs[(b, off)] == u["devptr"] + off        # Alg. 1 last line
        assert outs[(b, s)] - outs[(b, 1)] == s - 1           # differences preserved
        assert u["devptr"] % 256 == b % 256
    rng = sorted((unit(o, b)["devptr"], unit(o, b)["devptr"] + s) for b, s in zip(bases, sizes))
    for (a0, a1), (b0, b1) in zip(rng, rng[1:]):
        assert a1 < b0                                        # disjoint and never adjacent (A7)
    st = o.stats()
    assert st["h2d_units"] == 8 and st["h2d_bytes"] == sum(sizes)   # one copy per activation (A2)
    assert st["activations"] == 8 and st["fwd_translations"] == 32


def test_map_copies_bytes_and_unmap_epoch_gate(oracle):
    o = oracle
    b, n = 0x40000, 256
    data = np.arange(n, dtype=np.uint8)
    assert o.declareAlloc(b, n) == OK
    o.host_write(b, data)
    st, d = o.map(b)
    assert st == OK and (o.dev_read(d, n) == data).all()
    # no launch since the map: the CPU copy is up to date -> no copy (A5 R1)
    assert o.unmap(b) == OK and o.stats()["d2h_units"] == 0
    # GPU function writes, epoch advances, unmap copies exactly once
    o.dev_write(d, data[::-1].copy())
    o.advanceEpoch()
    assert o.unmap(b) == OK
    assert (o.host_read(b, n) == data[::-1]).all()
    assert o.unmap(b) == OK and o.unmap(b + 5) == OK           # same epoch: no second copy
    assert o.stats()["d2h_units"] == 1 and o.stats()["d2h_bytes"] == n
    o.advanceEpoch()
    assert o.unmap(b) == OK and o.stats()["d2h_units"] == 2
    assert unit(o, b)["epoch"] == o.epoch


def test_literal_epoch_mode_differs_only_without_launch():
    o = Oracle(LITERAL_EPOCH)
    assert o.declareAlloc(0x1000, 64) == OK      # declared at epoch 0 (A20)
    o.advanceEpoch()                              # a launch before the map
    assert o.map(0x1000)[0] == OK                 # literal Alg. 1 leaves epoch at 0
    assert o.unmap(0x1000) == OK
    assert o.stats()["d2h_units"] == 1            # 0 != 1 -> copy
    r1 = Oracle()
    assert r1.declareAlloc(0x1000, 64) == OK
    r1.advanceEpoch()
    assert r1.map(0x1000)[0] == OK
    assert r1.unmap(0x1000) == OK
    assert r1.stats()["d2h_units"] == 0           # R1: epoch set at activation
    o.close(); r1.close()


def test_map_of_active_unit_does_not_copy(oracle):
    o = oracle
    assert o.declareAlloc(0x1000, 100) == OK
    for _ in range(5):
        assert o.map(0x1010)[0] == OK
    assert o.stats()["h2d_units"] == 1 and unit(o, 0x1000)["refCount"] == 5


def test_release_frees_and_readonly_global(oracle):
    o = oracle
    assert o.declareGlobal("g_ro", 0x9000, 48, ro=True) == OK
    assert o.declareGlobal("g_rw", 0xA000, 48, ro=False) == OK
    assert o.declareAlloc(0xB000, 48) == OK
    d = {}
    for b in (0x9000, 0xA000, 0xB000):
        st, d[b] = o.map(b)
        assert st == OK
    o.advanceEpoch()
    for b in (0x9000, 0xA000, 0xB000):
        assert o.unmap(b) == OK
    assert o.stats()["d2h_units"] == 2            # read-only never copied back
    for b in (0x9000, 0xA000, 0xB000):
        assert o.release(b) == OK
    st = o.stats()
    assert st["frees"] == 1                       # globals are not freed
    for b in (0x9000, 0xA000):
        u = unit(o, b)
        assert u["refCount"] == 0 and u["devptr"] == d[b] and not (u["flags"] & UNIT_ACTIVE)
        s, t = o.map(b)
        assert s == OK and t == d[b]              # same named region on re-map (A14)
    assert o.stats()["h2d_units"] == 5            # ... re-copied at refCount 0 (Alg. 1)
    assert o.release(0xB000) == E_NOT_MAPPED      # A13
    assert unit(o, 0xB000)["devptr"] == 0


def test_alias_preservation_mapBatch(oracle):
    o = oracle
    assert o.declareAlloc(0x5000, 1024) == OK
    ps = [0x5000 + 8 * k for k in range(50)] + [0, 0x5000 + 1024]
    st, out = o.mapBatch(ps)
    assert st == OK
    u = unit(o, 0x5000)
    assert u["refCount"] == 51                    # A8: +1 per non-null pointer
    assert int(out[50]) == 0                      # A6
    assert all(int(t) == u["devptr"] + (p - 0x5000) for p, t in zip(ps, out) if p)
    assert o.stats()["h2d_units"] == 1 and o.stats()["null_slots"] == 1


def build_pointer_array(o, pp, targets):
    n = len(targets)
    assert o.declareAlloc(pp, 8 * n) == OK
    o.host_write(pp, np.asarray(targets, dtype=np.uint64))


def test_mapArray_roundtrip_and_permutation(oracle):
    o = oracle
    rows = [0x100000 + 0x800 * k for k in range(16)]
    for k, r in enumerate(rows):
        assert o.declareAlloc(r, 256) == OK
        o.host_write(r, np.full(32, k + 0.5))
    pp = 0x200000
    targets = [r + 8 * (k % 5) for k, r in enumerate(rows)] + [0, rows[3]]   # interior, NULL, alias
    build_pointer_array(o, pp, targets)
    st, d = o.mapArray(pp)
    assert st == OK
    dt = {u["base"]: u for u in o.dump()}
    dev = o.dev_read(d, 8 * len(targets)).view(np.uint64)
    for t, g in zip(targets, dev):
        if t == 0:
            assert g == 0
        else:
            b = max(r for r in rows if r <= t)
            assert int(g) == dt[b]["devptr"] + (t - b)
    assert dt[rows[3]]["refCount"] == 2 and dt[pp]["refCount"] == 1
    assert dt[pp]["flags"] & UNIT_ARRAYMAPPED
    assert o.stats()["h2d_units"] == 17 and o.stats()["fwd_translations"] == 17
    # permute the device slots (breaks R13-ii on purpose) -> host comes back permuted
    perm = np.array([5, 2, 9, 0, 1, 3, 4, 6, 7, 8, 10, 11, 12, 13, 14, 15, 16, 17])
    o.dev_write(d, dev[perm].copy())
    o.advanceEpoch()
    assert o.unmapArray(pp) == OK
    host = o.host_read(pp, 8 * len(targets)).view(np.uint64)
    assert (host == np.asarray(targets, dtype=np.uint64)[perm]).all()
    assert o.stats()["d2h_units"] == 17            # outer + 16 distinct rows, once each
    # restore, next epoch: identity round trip
    o.dev_write(d, dev.copy())
    o.advanceEpoch()
    assert o.unmapArray(pp) == OK
    assert (o.host_read(pp, 8 * len(targets)).view(np.uint64) == np.asarray(targets, np.uint64)).all()
    assert o.releaseArray(pp) == OK
    assert all(u["refCount"] == 0 for u in o.dump())
    assert o.stats()["frees"] == 17


def test_mapArray_trailing_bytes_verbatim(oracle):
    o = oracle
    assert o.declareAlloc(0x3000, 64) == OK
    pp = 0x4000
    assert o.declareAlloc(pp, 8 * 3 + 5) == OK      # 3 slots + 5 trailing bytes (A10)
    o.host_write(pp, np.array([0x3000, 0x3008, 0], dtype=np.uint64))
    o.host_write(pp + 24, bytes([1, 2, 3, 4, 5]))
    st, d = o.mapArray(pp + 8)
    assert st == OK and d == unit(o, pp)["devptr"] + 8
    assert bytes(o.dev_read(unit(o, pp)["devptr"] + 24, 5)) == bytes([1, 2, 3, 4, 5])
    assert unit(o, 0x3000)["refCount"] == 2


def test_self_referential_pool(oracle):
    """A9/A12: a pool AU whose slots point into itself (config D' shape)."""
    o = oracle
    pool = 0x70000
    n = 8
    assert o.declareAlloc(pool, 8 * n) == OK
    o.host_write(pool, np.array([pool + 8 * ((k + 1) % n) for k in range(n)], dtype=np.uint64))
    st, d = o.mapArray(pool)
    assert st == OK
    u = unit(o, pool)
    assert u["refCount"] == 1 + n and o.stats()["h2d_units"] == 1
    dev = o.dev_read(d, 8 * n).view(np.uint64)
    assert all(int(dev[k]) == d + 8 * ((k + 1) % n) for k in range(n))
    o.advanceEpoch()
    assert o.unmapArray(pool) == OK
    assert o.stats()["d2h_units"] == 1              # the self-reference is skipped by its epoch
    host = o.host_read(pool, 8 * n).view(np.uint64)
    assert all(int(host[k]) == pool + 8 * ((k + 1) % n) for k in range(n))
    assert o.releaseArray(pool) == OK and unit(o, pool)["refCount"] == 0


def test_errors_leave_state_unchanged(oracle):
    o = oracle
    assert o.declareAlloc(0x1000, 64) == OK
    assert o.declareAlloc(0x2000, 64) == OK
    o.host_write(0x1000, np.arange(8, dtype=np.uint64))
    pp = 0x8000
    build_pointer_array(o, pp, [0x1000, 0x2008, 0x3000])         # last slot unregistered
    regions = [(0x1000, 64), (0x2000, 64), (pp, 24)]
    before = snapshot(o, regions)
    assert o.mapArray(pp)[0] == E_UNREGISTERED
    assert o.mapBatch([0x1000, 0x1040, 0x1041])[0] == E_UNREGISTERED   # past the end
    assert o.mapBatch([0x1000, 0x1800])[0] == E_UNREGISTERED           # gap
    assert o.unmap(0x1000) == E_NOT_MAPPED and o.release(0x1000) == E_NOT_MAPPED
    assert snapshot(o, regions) == before
    # partial success then failure inside one releaseBatch -> rolled back
    assert o.map(0x1000)[0] == OK
    mid = snapshot(o, regions)
    assert o.releaseBatch([0x1000, 0x1008]) == E_NOT_MAPPED            # second release underflows
    assert snapshot(o, regions) == mid
    assert o.undeclare(0x1000) == E_BUSY
    assert o.undeclare(0x1001) == E_UNREGISTERED
    assert o.declareAlloc(0x1030, 8) == E_OVERLAP
    assert o.declareAlloc(0x0ff8, 9) == E_OVERLAP
    assert o.declareAlloc(0x0ff8, 8) == OK                             # adjacent is fine
    assert o.declareAlloc(0x5000, 0) == E_INVALID
    assert o.declareGlobal("g", 0x6000, 8) == OK
    assert o.declareGlobal("g", 0x7000, 8) == E_DUPLICATE
    # releaseArray whose element decrements would underflow
    assert o.release(0x1000) == OK
    before = snapshot(o, regions)
    o.host_write(pp, np.array([0x1000, 0x2008, 0], dtype=np.uint64))
    assert o.mapArray(pp)[0] == OK
    assert o.release(0x2000) == OK                                     # steal the element's reference
    mid = snapshot(o, regions)
    assert o.releaseArray(pp) == E_NOT_MAPPED
    assert snapshot(o, regions) == mid


def test_unmapSlots_mapSlots_device_arrays(oracle):
    o = oracle
    bases = [0x10000 + 0x100 * k for k in range(10)]
    for b in bases:
        assert o.declareAlloc(b, 0x80) == OK
    q = np.array([b + 0x10 for b in bases] + [0, bases[0], bases[9] + 0x80], dtype=np.uint64)
    slots = q.copy()
    assert o.mapSlots(slots) == OK
    dt = {u["base"]: u for u in o.dump()}
    assert dt[bases[0]]["refCount"] == 2 and dt[bases[9]]["refCount"] == 2
    for p, t in zip(q, slots):
        if p:
            b = max(x for x in bases if x <= p)
            assert int(t) == dt[b]["devptr"] + (int(p) - b)
    o.advanceEpoch()
    assert o.unmapSlots(slots, release=True) == OK
    assert (slots == q).all()                                          # reverse == original
    assert all(u["refCount"] == 0 for u in o.dump())
    st = o.stats()
    assert st["d2h_units"] == 10 and st["rev_translations"] == 12 and st["fwd_translations"] == 12
    bad = np.array([12345], dtype=np.uint64)
    assert o.unmapSlots(bad) == E_UNREGISTERED and bad[0] == 12345


def test_device_copies_never_adjacent_unless_host_adjacent(oracle):
    """A7: a one-past-the-end GPU pointer must reverse to the same unit it came from."""
    o = oracle
    bases = [0x10000 * (k + 1) for k in range(6)]        # 256-aligned, sizes multiple of 256
    for b in bases:
        assert o.declareAlloc(b, 512) == OK
    d = [o.map(b)[1] for b in bases]
    for b, g in zip(bases, d):
        end = g + 512                                      # one past the end on the device
        assert o.devLookup(end) == (b, g)
        s = np.array([end], dtype=np.uint64)
        assert o.unmapSlots(s) == OK and int(s[0]) == b + 512


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_batch_forms_are_their_sequential_loops(seed):
    """the batch forms have "the same semantics as the sequential loop".  Oracle A runs a
    random program through mapArrays / unmapArrays / releaseArrays / mapBatch / unmapBatch / releaseBatch
    on multisets (repeats, nested outers); oracle B runs the same program through the single calls in
    batch order.  After every successful batch their full states agree.  A failing batch must leave A
    unchanged (all-or-nothing) and its sequential loop must fail too (checked on a replayed copy)."""
    rng = np.random.default_rng(seed)
    leaves = [0x100000 + 0x100 * k for k in range(40)]
    outers = [0x200000 + 0x1000 * j for j in range(8)]
    regions, init = [], []
    for k, a in enumerate(leaves):
        n = 32 + 8 * (k % 4)
        init.append((a, np.full(n, k, dtype=np.uint8)))
        regions.append((a, n))
    for j, p in enumerate(outers):
        n = int(rng.integers(1, 12))
        tg = [0 if rng.random() < 0.15 else leaves[int(rng.integers(0, 40))] + 8 * int(rng.integers(0, 4))
              for _ in range(n)]
        if j < 2:
            tg[0] = outers[6 + j]                      # nested: outers 0, 1 point at outers 6, 7
        init.append((p, np.asarray(tg, dtype=np.uint64)))
        regions.append((p, 8 * n))
    singles = {"mapArrays": "mapArray", "unmapArrays": "unmapArray", "releaseArrays": "releaseArray",
               "mapBatch": "map", "unmapBatch": "unmap", "releaseBatch": "release"}

    def fresh():
        o = Oracle()
        for (b, data), (_b, n) in zip(init, regions):
            assert o.declareAlloc(b, n) == OK
            o.host_write(b, data)
        return o

    def run_loop(o, name, batch):
        for p in batch:
            r = getattr(o, singles[name])(p)
            st = r[0] if isinstance(r, tuple) else r
            if st != OK:
                return st
        return OK

    A, B = fresh(), fresh()
    log = []
    held = {"a": [], "s": []}                          # references taken: outers / scalar pointers
    n_ok = n_err = 0
    for step in range(150):
        name = list(singles)[int(rng.integers(0, 6))]
        k = int(rng.integers(1, 6))
        kind = "a" if "Arrays" in name else "s"
        if name.startswith("map") or not held[kind] or rng.random() < 0.1:
            pool = outers if kind == "a" else [b + int(rng.integers(0, n + 1)) for b, n in regions[:40]]
            batch = [pool[int(i)] for i in rng.integers(0, len(pool), k)]
        else:
            batch = [held[kind][int(i)] for i in rng.choice(len(held[kind]), min(k, len(held[kind])), replace=False)]
        before = snapshot(A, regions)
        ra = getattr(A, name)(batch)
        sa = ra[0] if isinstance(ra, tuple) else ra
        if sa != OK:
            n_err += 1
            assert snapshot(A, regions) == before, (step, name)      # all-or-nothing
            C = fresh()
            for nm, bt in log:
                assert (run_loop(C, nm, bt) if nm != "advance" else C.advanceEpoch()) == OK
            assert run_loop(C, name, batch) != OK, (step, name)       # the loop fails as well
            C.close()
            continue
        n_ok += 1
        assert run_loop(B, name, batch) == OK, (step, name)
        log.append((name, batch))
        if name.startswith("map"):
            held[kind] += batch
        elif name.startswith("release"):
            for p in batch:
                if p in held[kind]:                    # (a random release may hit another pointer's unit)
                    held[kind].remove(p)
        if rng.random() < 0.2:
            A.advanceEpoch()
            B.advanceEpoch()
            log.append(("advance", None))
        assert snapshot(A, regions) == snapshot(B, regions), (step, name)
    assert n_ok > 100 and n_err >= 1
    A.close()
    B.close()


# ---- A18 lenient mode, pinned by hand (VERDICT r1 "What's weak" 1) -----------------------------------
# Reading A18 (field-insensitive typing may label a struct holding data words
# as a pointer array): in lenient mode a non-null word that no AU covers passes through unchanged, is
# counted once per word per call (`passthrough`), and takes no reference; unmap/release of an
# uncovered pointer are no-ops returning OK.  Every expected value below is counted by hand from that
# reading; none is read back from the oracle.
def _lenient_setup(o):
    A, B, PP = 0x10000, 0x20000, 0x30000
    STRAY = 0x50000                                   # below DEV0, in no host AU and no device copy
    assert o.declareAlloc(A, 64) == OK
    assert o.declareAlloc(B, 64) == OK
    o.host_write(A, np.arange(64, dtype=np.uint8))
    o.host_write(B, np.arange(64, 128, dtype=np.uint8))
    words = np.array([A + 8, STRAY, 0, B, STRAY], dtype=np.uint64)   # the stray word twice, one NULL
    assert o.declareAlloc(PP, 8 * len(words)) == OK
    o.host_write(PP, words)
    return A, B, PP, STRAY, words


def test_lenient_mode_hand_counts():
    from oracle import LENIENT
    o = Oracle(LENIENT)
    try:
        A, B, PP, STRAY, words = _lenient_setup(o)
        st, d = o.mapArray(PP)
        assert st == OK
        u = {x["base"]: x for x in o.dump()}
        dev = o.dev_read(u[PP]["devptr"], 8 * len(words)).view(np.uint64)
        # device slots: translated, stray raw (twice), NULL, translated
        assert list(dev) == [u[A]["devptr"] + 8, STRAY, 0, u[B]["devptr"], STRAY]
        s = o.stats()
        assert s["passthrough"] == 2                      # per word, not per distinct value or per call
        assert s["null_slots"] == 1
        assert s["fwd_translations"] == 2                 # A+8 and B only
        assert s["h2d_units"] == 3 and s["activations"] == 3
        assert (u[PP]["refCount"], u[A]["refCount"], u[B]["refCount"]) == (1, 1, 1)   # no ref for STRAY
        o.advanceEpoch()
        assert o.unmapArray(PP) == OK
        host = o.host_read(PP, 8 * len(words)).view(np.uint64)
        assert (host == words).all()                      # the stray word comes back unchanged
        s = o.stats()
        assert s["passthrough"] == 4                      # + 2: the outer is reversed once, its 2 stray words each pass
        assert s["rev_translations"] == 2
        assert s["d2h_units"] == 3                        # outer + A + B; nothing for STRAY
        # scalar calls on an uncovered pointer: OK and no effect
        before = (o.dump(), o.stats())
        assert o.unmap(STRAY) == OK and o.release(STRAY) == OK
        assert (o.dump(), o.stats()) == before
        st, t = o.map(STRAY)
        assert st == OK and t == STRAY and o.stats()["passthrough"] == 5
        assert o.releaseArray(PP) == OK
        assert all(x["refCount"] == 0 for x in o.dump())
        assert o.stats()["frees"] == 3
        # device slots: the same stray passes through mapSlots / unmapSlots
        slots = np.array([STRAY, A + 1, 0], dtype=np.uint64)
        assert o.mapSlots(slots) == OK
        assert int(slots[0]) == STRAY and int(slots[2]) == 0
        assert {x["base"]: x for x in o.dump()}[A]["refCount"] == 1
        o.advanceEpoch()
        assert o.unmapSlots(slots, release=True) == OK
        assert list(slots) == [STRAY, A + 1, 0]
        assert all(x["refCount"] == 0 for x in o.dump())
    finally:
        o.close()


def test_strict_mode_rejects_the_same_program():
    o = Oracle()
    try:
        A, B, PP, STRAY, words = _lenient_setup(o)
        before = (o.dump(), o.stats())
        assert o.mapArray(PP)[0] == E_UNREGISTERED        # A18 strict: every non-null slot must hit
        assert (o.dump(), o.stats()) == before            # all-or-nothing
        assert o.map(STRAY)[0] == E_UNREGISTERED
        assert o.unmap(STRAY) == E_UNREGISTERED and o.release(STRAY) == E_UNREGISTERED
        assert o.mapSlots(np.array([STRAY], dtype=np.uint64)) == E_UNREGISTERED
    finally:
        o.close()
