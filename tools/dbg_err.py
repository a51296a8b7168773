import numpy as np, torch, sys
sys.path.insert(0, '/root/repo')
import workloads as W
import paper_conf_pldi_jablinpjjba11_b200 as cg
ctx = cg.Context(0, arena_bytes=1 << 30)
offs, sizes, span = W.table_layout(1000, 3)
R = W.reserve_readonly(span)
assert ctx.declareBatch(offs + np.uint64(R), sizes, readonly=True) == 0
q, u = W.queries(offs, sizes, 5000, 3)
slots = (q + np.uint64(R)).astype(np.uint64)
slots[1234] = np.uint64(R + span + 100)
d = torch.from_numpy(slots.view(np.int64).copy()).cuda()
s = ctx.mapArrayDevice(d.data_ptr(), len(slots))
print("status", s, ctx.L.cgcm_lastCudaError().decode())
