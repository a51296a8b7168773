"""Pins for the oracle's glue-kernel interpreter (NEXT-4; §5.3 "Glue Kernels": a small CPU
region between two GPU functions is "transform[ed] into a single-threaded GPU function", which
"obviates the need to copy the allocation units between GPU and CPU memories").

Every expected value comes from arithmetic done here in Python (closed forms, IEEE binary64 as Python
floats compute it, a host-side run of the same CPU region on plain numpy memory), never from the
oracle itself.
"""
import struct

import numpy as np

from oracle import Oracle, OK, E_INVALID, E_UNREGISTERED, E_NOT_MAPPED

MOVI, ADD, ADDI, SUB, MUL, FADD, FSUB, FMUL, FDIV, LD, ST, BNZ, HALT = range(1, 14)


def f2u(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def u2f(u):
    return struct.unpack("<d", struct.pack("<Q", int(u)))[0]


def test_integer_loop_closed_form(oracle):
    # r1 = sum_{k=1..100} k with a counted loop: r2 = 100; loop: r1 += r2; r2 -= 1; bnz r2
    prog = [(MOVI, 2, 0, 0, 100), (MOVI, 3, 0, 0, 1), (ADD, 1, 1, 2, 0), (SUB, 2, 2, 3, 0), (BNZ, 0, 2, 0, 2),
            (HALT, 0, 0, 0, 0), (MOVI, 1, 0, 0, 7)]
    st, r = oracle.runGlue(prog, [])
    assert st == OK and int(r[1]) == 5050 and int(r[2]) == 0            # HALT skipped the last MOVI
    st, r = oracle.runGlue([(MOVI, 4, 0, 0, -3), (MUL, 5, 4, 4, 0), (ADDI, 6, 5, 0, -10)], [])
    assert st == OK and int(r[5]) == 9 and int(r[6]) == (9 - 10) % (1 << 64)


def test_float_ops_are_ieee_binary64(oracle):
    a, b = 0.1, 0.2
    prog = [(MOVI, 1, 0, 0, f2u(a)), (MOVI, 2, 0, 0, f2u(b)), (FADD, 3, 1, 2, 0), (FSUB, 4, 1, 2, 0),
            (FMUL, 5, 1, 2, 0), (FDIV, 6, 1, 2, 0)]
    prog = [(o, d, x, y, imm - (1 << 64) if imm >= (1 << 63) else imm) for (o, d, x, y, imm) in prog]
    st, r = oracle.runGlue(prog, [])
    assert st == OK
    assert u2f(r[3]) == a + b and u2f(r[4]) == a - b and u2f(r[5]) == a * b and u2f(r[6]) == a / b
    assert u2f(r[3]) != 0.3                                               # rounding is real, not decimal


def test_errors(oracle):
    o = oracle
    assert o.runGlue([(MOVI, 32, 0, 0, 1)], [])[0] == E_INVALID            # register out of range
    assert o.runGlue([(BNZ, 0, 1, 0, 5)], [])[0] == E_INVALID              # jump target out of range
    assert o.runGlue([(99, 0, 0, 0, 0)], [])[0] == E_INVALID               # unknown op
    loop = [(MOVI, 1, 0, 0, 1), (BNZ, 0, 1, 0, 1)]
    assert o.runGlue(loop, [], max_steps=1000)[0] == E_INVALID             # step limit
    b = 0x10000
    assert o.declareAlloc(b, 64) == OK
    assert o.runGlue([(LD, 1, 0, 0, 0)], [b])[0] == E_NOT_MAPPED           # not mapped
    assert o.runGlue([(LD, 1, 0, 0, 0)], [0x90000])[0] == E_UNREGISTERED   # not an AU
    assert o.map(b)[0] == OK
    assert o.runGlue([(LD, 1, 0, 0, 56)], [b])[0] == OK                    # last word
    assert o.runGlue([(LD, 1, 0, 0, 64)], [b])[0] == E_UNREGISTERED        # one past the end: no 8 bytes
    assert o.runGlue([(LD, 1, 0, 0, 4)], [b])[0] == E_UNREGISTERED         # misaligned
    assert o.runGlue([(LD, 1, 0, 0, -8)], [b])[0] == E_UNREGISTERED        # before the copy


def jagged(o, base, nrows, ncols, vals):
    rows = [base + 0x1000 * r for r in range(nrows)]
    for r, a in enumerate(rows):
        assert o.declareAlloc(a, 8 * ncols) == OK
        o.host_write(a, np.asarray(vals[r], dtype=np.float64))
    pp = base + 0x1000 * nrows
    assert o.declareAlloc(pp, 8 * nrows) == OK
    o.host_write(pp, np.asarray(rows, dtype=np.uint64))
    return rows, pp


# the CPU region of the example: x[0][0] = x[0][0] + 2 * x[1][1];  x[2][5] = x[0][0] / 4
def region_on_host(m):
    m[0, 0] = m[0, 0] + 2.0 * m[1, 1]
    m[2, 5] = m[0, 0] / 4.0


def region_program():
    two, four = f2u(2.0), f2u(4.0)
    return [(LD, 1, 0, 0, 0), (LD, 2, 0, 0, 8), (LD, 3, 0, 0, 16),   # row pointers (GPU pointers)
            (LD, 4, 1, 0, 0), (LD, 5, 2, 0, 8),                      # x[0][0], x[1][1]
            (MOVI, 6, 0, 0, two), (FMUL, 5, 5, 6, 0), (FADD, 4, 4, 5, 0), (ST, 0, 1, 4, 0),
            (MOVI, 6, 0, 0, four), (FDIV, 7, 4, 6, 0), (ST, 0, 3, 7, 40)]


def test_glue_equals_the_host_region_and_copies_nothing(oracle):
    """Promoted loop with the region as a glue kernel == naive loop with the region run on the CPU between
    unmap and map; the glue loop moves no AU inside the loop."""
    nrows, ncols, iters = 4, 8, 3
    vals = np.arange(nrows * ncols, dtype=np.float64).reshape(nrows, ncols) / 8 + 1
    # expected: the naive program on plain host memory (S1 scale by 0.5, then the region), iterated
    m = vals.copy()
    for _ in range(iters):
        m *= 0.5
        region_on_host(m)
    o = oracle
    rows, pp = jagged(o, 0x100000, nrows, ncols, vals)
    st, d = o.mapArray(pp)
    assert st == OK
    s0 = o.stats()
    for _ in range(iters):
        assert o.mapArray(pp)[0] == OK
        o.kernel_scale(d, nrows, ncols, 0.5)
        o.advanceEpoch()
        st, _r = o.runGlue(region_program(), [pp])
        assert st == OK
        o.advanceEpoch()
        assert o.releaseArray(pp) == OK
    s1 = o.stats()
    assert (s1["h2d_units"], s1["d2h_units"]) == (s0["h2d_units"], s0["d2h_units"])   # nothing moved
    assert o.unmapArray(pp) == OK and o.releaseArray(pp) == OK
    got = np.stack([o.host_read(a, 8 * ncols).view(np.float64) for a in rows])
    assert got.tobytes() == m.tobytes()
