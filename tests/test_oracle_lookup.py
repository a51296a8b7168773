"""Pins for the oracle's greatestLTE lookup (a1) and devLookup (a3) -- brute force on tiny tables.

P:L167-170 (§3.1): "finds the greatest key in the allocation map less than or equal to the pointer";
reading A7: accepted iff p - base <= size (one past the end accepted).  The brute force below is a
linear scan over the unit list -- no tree, no bisect -- checked exhaustively over every address of
[minbase - 16, maxend + 16] for seeded random tiny tables with adjacency and gaps.
"""
import numpy as np
import pytest

import workloads as W
from oracle import Oracle, OK, E_UNREGISTERED


def tiny_table(seed, U):
    sizes = 1 + W.randint(seed, 1, np.arange(U, dtype=np.uint64), 64).astype(np.int64)
    gaps = W.randint(seed, 2, np.arange(U, dtype=np.uint64), 33).astype(np.int64)  # 0..32, 0 = adjacent
    bases, cur = [], 0x10000 + int(W.randint(seed, 3, 0, 64))
    for k in range(U):
        cur += int(gaps[k])
        bases.append(cur)
        cur += int(sizes[k])
    return bases, [int(s) for s in sizes]


def brute_lookup(bases, sizes, p):
    best = None
    for b, s in zip(bases, sizes):          # linear scan: greatest base <= p
        if b <= p and (best is None or b > best[0]):
            best = (b, s)
    if best is None or p - best[0] > best[1]:
        return None
    return best


@pytest.mark.parametrize("seed", range(12))
def test_greatestLTE_bruteforce(seed):
    U = 1 + seed * 3 % 32
    bases, sizes = tiny_table(seed, U)
    o = Oracle()
    order = W.permutation(seed, 9, U)       # declaration order must not matter
    for k in order:
        assert o.declareAlloc(bases[k], sizes[k]) == OK
    lo, hi = bases[0] - 16, bases[-1] + sizes[-1] + 16
    for p in range(lo, hi + 1):
        assert o.lookup(p) == brute_lookup(bases, sizes, p), hex(p)
    o.close()


def test_adjacent_one_past_end_picks_next():
    """A7: if another AU starts exactly at base+size, greatestLTE picks that AU (as printed)."""
    o = Oracle()
    assert o.declareAlloc(0x1000, 16) == OK
    assert o.declareAlloc(0x1010, 8) == OK
    assert o.lookup(0x1010) == (0x1010, 8)
    assert o.lookup(0x1018) == (0x1010, 8)      # one past the end of the second
    assert o.lookup(0x1019) is None
    assert o.lookup(0xfff) is None
    o.close()


@pytest.mark.parametrize("seed", range(6))
def test_devLookup_bruteforce(seed):
    U = 4 + seed * 5
    bases, sizes = tiny_table(seed + 100, U)
    o = Oracle()
    for b, s in zip(bases, sizes):
        assert o.declareAlloc(b, s) == OK
    active = [k for k in range(U) if (k * 7 + seed) % 3 != 0]
    for k in active:
        s, t = o.map(bases[k])
        assert s == OK
    d = {u["base"]: u for u in o.dump()}
    dbases = [d[bases[k]]["devptr"] for k in active]
    dsizes = [sizes[k] for k in active]
    lo, hi = min(dbases) - 16, max(x + y for x, y in zip(dbases, dsizes)) + 16
    for g in range(lo, hi + 1):
        exp = brute_lookup(dbases, dsizes, g)
        got = o.devLookup(g)
        if exp is None:
            assert got is None, hex(g)
        else:
            k = active[dbases.index(exp[0])]
            assert got == (bases[k], exp[0]), hex(g)
    o.close()


def test_lookup_below_first_and_in_gap(oracle):
    assert oracle.declareAlloc(0x2000, 32) == OK
    assert oracle.declareAlloc(0x2040, 32) == OK
    assert oracle.map(0x1fff)[0] == E_UNREGISTERED
    assert oracle.map(0x2021)[0] == E_UNREGISTERED   # gap
    assert oracle.map(0x2060)[0] == OK                # one past the end
    assert oracle.map(0x2061)[0] == E_UNREGISTERED    # past the end
