"""Per-call latency anatomy of config A's promoted loop (in-loop mapArray + releaseArray of an active,
array-mapped 256-slot outer): host wall time per call, for the ncu launch list of the same run."""
import os, sys, time
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import paper_conf_pldi_jablinpjjba11_b200 as cg  # noqa: E402
ctx = cg.Context(0, arena_bytes=1 << 28)
rows = [ctx.malloc(2048) for _ in range(256)]
pp = ctx.malloc(2048)
np.ctypeslib.as_array((np.ctypeslib.ctypes.c_uint64 * 256).from_address(pp))[:] = rows
st, d0 = ctx.mapArray(pp)
tm, tr = [], []
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 200):
    t0 = time.perf_counter(); s, d = ctx.mapArray(pp); t1 = time.perf_counter()
    ctx.advanceEpoch()
    t2 = time.perf_counter(); ctx.releaseArray(pp); t3 = time.perf_counter()
    tm.append(t1 - t0); tr.append(t3 - t2)
ctx.unmapArray(pp); ctx.releaseArray(pp)
print({"mapArray_us_median": round(1e6 * float(np.median(tm)), 1), "releaseArray_us_median": round(1e6 * float(np.median(tr)), 1),
       "kernel_launches": ctx.stats()["kernel_launches"]})
ctx.close()
