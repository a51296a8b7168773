"""Debug helper: mapArrayDevice + unmapArrayDevice round trip at a mid size (several pipeline
iterations per thread), checked against the inputs.  python tools/dbg_mid.py [U] [Q]"""
import sys
import numpy as np
import torch
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import workloads as W
import paper_conf_pldi_jablinpjjba11_b200 as cg

U = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 16
Q = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 23
offs, sizes, span = W.table_layout(U, 3)
R = W.reserve_readonly(span)
ctx = cg.Context(0, arena_bytes=int(sizes.sum()) + Q * 24 + (1 << 30))
assert ctx.declareBatch(offs + np.uint64(R), sizes, readonly=True) == 0
print(ctx.indexInfo())
q, u = W.queries(offs, sizes, Q, 3)
slots = (q + np.uint64(R)).astype(np.uint64)
d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
for it in range(3):
    s1 = ctx.mapArrayDevice(d.data_ptr(), Q)
    ctx.advanceEpoch()
    s2 = ctx.unmapArrayDevice(d.data_ptr(), Q, release=True)
    ok = (d.cpu().numpy().view(np.uint64) == slots).all()
    print("iter", it, s1, s2, ok, cg.strerror(s1), ctx.L.cgcm_lastCudaError().decode())
