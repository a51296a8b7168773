"""The pipelined device-array passes (k_fwd_fast / k_fwd_fix, k_rev_fast / k_rev_fix in csrc/kernels.cu) when
one launch mixes warp groups of 64 ordinary slots (the short path) with groups the general per-chunk code
has to redo: a NULL (A6), a pointer into an AU that is not active yet (Alg. 1's activation), a
slot a GPU function rewrote before the unmap (shadow check fails, the reverse lookup decides), ragged ends
and a slice that starts at an odd slot (the shadow's 8-byte alignment).  Every call is compared with the
oracle (mapSlots / unmapSlots) slot by slot, and the full state after it (Pair.check).
"""
import numpy as np
import pytest

import workloads as W
from tests.harness import Pair
from tests.test_gpu_deferred import gmap, gunmap

pytestmark = pytest.mark.gpu


@pytest.fixture(params=[8, 40], ids=["shadow-v3", "shadow-v2"])
def P(request):
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    from oracle import Oracle
    ctx = cg.Context(0, arena_bytes=1 << 30, flags=request.param)
    o = Oracle()
    p = Pair(ctx, o)
    yield p
    ctx.close()
    o.close()


@pytest.mark.parametrize("s0", [0, 1])
def test_short_and_general_groups_in_one_launch(P, s0):
    import torch
    U, Q = 4096, 3 * (1 << 16) + 77
    offs, sizes, span = W.table_layout(U, 11)
    R = W.reserve_readonly(span)
    bases = offs + np.uint64(R)
    assert P.g.declareBatch(bases, sizes, readonly=True) == 0
    for b, s in zip(bases, sizes):
        assert P.o.declareAlloc(int(b), int(s), readonly=True) == 0
    # keep the first 4000 units active: one interior pointer each, mapped and left mapped
    keep = (bases[:4000] + sizes[:4000] // np.uint64(2)).astype(np.uint64)
    dk = torch.from_numpy(keep.view(np.int64).copy()).cuda()
    kref = keep.copy()
    assert gmap(P, dk, 0, len(keep), kref) == 0
    P.check("kept active")
    # the array under test: interior pointers into the active units, with rare slots sprinkled so that
    # about one warp group in five needs the general code
    rng = np.random.default_rng(5)
    u = rng.integers(0, 4000, Q)
    q = (bases[u] + (rng.random(Q) * sizes[u]).astype(np.uint64)).astype(np.uint64)
    rare = rng.choice(Q, Q // 320, replace=False)
    q[rare[0::3]] = 0                                                   # NULL
    q[rare[1::3]] = bases[4000 + rare[1::3] % 96]                       # inactive units: activation
    q[Q - 5:] = q[:5]                                                   # ragged tail
    buf = np.zeros(Q + 1, dtype=np.uint64)
    buf[s0:s0 + Q] = q
    d = torch.from_numpy(buf.view(np.int64).copy()).cuda()
    ref = buf.copy()
    assert gmap(P, d, s0, Q, ref) == 0
    P.check("mapped")
    P.advance()
    # a GPU function rewrites a few slots inside the same units (still valid device pointers)
    dd = d.cpu().numpy().view(np.uint64).copy()
    ordinary = np.ones(Q, dtype=bool)
    ordinary[rare] = False
    ordinary[Q - 5:] = False
    hits = [i for i in rng.choice(np.flatnonzero(ordinary), 50, replace=False)]
    for i in hits:  # the same unit, half way back towards its base
        dd[s0 + i] = dd[s0 + i] - np.uint64((q[i] - bases[u[i]]) // np.uint64(2))
    d.copy_(torch.from_numpy(dd.view(np.int64)))
    ref[s0:s0 + Q] = dd[s0:s0 + Q]
    assert gunmap(P, d, s0, Q, ref, release=True) == 0
    P.check("unmapped")
    assert gunmap(P, dk, 0, len(keep), kref, release=True) == 0
    P.check("end")
    W.release_reservation(R, span)
