"""Glue kernels on the GPU (NEXT-4; §5.3) against the oracle's interpreter: the same
programs through cgcm_launchGlue (one GPU thread over the mapped AUs' device copies) and the oracle's
runGlue (its simulated device, replay mode), with the full state compared after every call -- final
registers, status codes of the error cases, host bytes after the unmaps, copy counters."""
import numpy as np
import pytest

from tests.harness import Pair, HostBuf
from tests.test_oracle_glue import MOVI, ADD, LD, ST, BNZ, SUB, region_program, region_on_host

pytestmark = pytest.mark.gpu


@pytest.fixture
def P():
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    ctx = cg.Context(0, arena_bytes=1 << 28)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    ctx.close()
    o.close()


def glue(P, prog, ptrs, max_steps=1 << 20):
    sg, rg = P.g.launchGlue(prog, ptrs, max_steps)
    so, ro = P.o.runGlue(prog, ptrs, max_steps)
    assert sg == so, (sg, so)
    if sg == 0:
        assert (rg == ro).all(), (rg, ro)
    return sg, rg


def test_glue_region_in_a_promoted_loop(P):
    nrows, ncols, iters = 4, 8, 3
    vals = np.arange(nrows * ncols, dtype=np.float64).reshape(nrows, ncols) / 8 + 1
    buf = HostBuf(1 << 16)
    rows = [buf.addr + 0x1000 * r for r in range(nrows)]
    for r, a in enumerate(rows):
        assert P.declare(a, 8 * ncols, vals[r]) == 0
    pp = buf.addr + 0x1000 * nrows
    assert P.declare(pp, 8 * nrows, np.asarray(rows, dtype=np.uint64)) == 0
    m = vals.copy()
    for _ in range(iters):
        m *= 0.5
        region_on_host(m)
    st, d = P.run("mapArray", pp)
    assert st == 0
    P.check("promoted")
    s0 = P.g.stats()
    for it in range(iters):
        st, d2 = P.run("mapArray", pp)
        assert P.g.sample_scale(d2, nrows, ncols, 0.5) == 0
        P.g.synchronize()
        assert P.o.kernel_scale(d2, nrows, ncols, 0.5) == 0
        P.advance()
        assert glue(P, region_program(), [pp])[0] == 0
        P.advance()
        P.run("releaseArray", pp)
        P.check(f"iteration {it}")
        P.check_device_units()
    s1 = P.g.stats()
    assert (s1["h2d_units"], s1["d2h_units"]) == (s0["h2d_units"], s0["d2h_units"])   # no copies in the loop
    P.run("unmapArray", pp)
    P.run("releaseArray", pp)
    P.check("end")
    got = np.stack([np.frombuffer(bytes(P.o.host_read(a, 8 * ncols)), dtype=np.float64) for a in rows])
    assert got.tobytes() == m.tobytes()


def test_glue_errors_and_loops(P):
    buf = HostBuf(1 << 16)
    a, b = buf.addr + 0x100, buf.addr + 0x2000
    assert P.declare(a, 64, np.arange(8, dtype=np.uint64)) == 0
    assert P.declare(b, 24, np.arange(3, dtype=np.uint64) + 100) == 0
    # sum of a's 8 words through a counted loop over a pointer register
    prog = [(MOVI, 2, 0, 0, 8), (MOVI, 3, 0, 0, 1), (LD, 4, 0, 0, 0), (ADD, 1, 1, 4, 0), (MOVI, 5, 0, 0, 8),
            (ADD, 0, 0, 5, 0), (SUB, 2, 2, 3, 0), (BNZ, 0, 2, 0, 2)]
    assert glue(P, prog, [a])[0] == -4                       # not mapped yet (CGCM_E_NOT_MAPPED)
    P.run("map", a)
    st, r = glue(P, prog, [a])
    assert st == 0 and int(r[1]) == 28
    assert glue(P, [(LD, 1, 0, 0, 64)], [a])[0] == -2        # one past the end: outside the copy
    assert glue(P, [(LD, 1, 0, 0, 4)], [a])[0] == -2         # misaligned
    assert glue(P, [(LD, 1, 0, 0, 0)], [b])[0] == -4         # b not mapped
    P.run("map", b)
    st, r = glue(P, [(LD, 1, 1, 0, 16), (ST, 0, 0, 1, 56)], [a, b])   # a[7] = b[2]
    assert st == 0
    assert glue(P, [(MOVI, 1, 0, 0, 1), (BNZ, 0, 1, 0, 1)], [], max_steps=500)[0] == -1   # step limit
    assert glue(P, [(MOVI, 40, 0, 0, 1)], [])[0] == -1
    P.advance()
    P.run("unmap", a)
    P.run("unmap", b)
    P.check("after glue stores")                             # a[7] == 102 on both sides
    assert int(np.frombuffer(bytes(P.o.host_read(a, 64)), dtype=np.uint64)[7]) == 102
    P.run("release", a)
    P.run("release", b)
    P.check("end")
