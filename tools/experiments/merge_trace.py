"""Where does a step go when one AU is declared before it (NEXT-1 delta merge)?  Config C, CGCM_PROFILE
kernel times per launch and CGCM_TRACE host phases, with and without a declaration between steps."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import bench  # noqa: E402
import paper_conf_pldi_jablinpjjba11_b200 as cg  # noqa: E402
import workloads as W  # noqa: E402

wl = bench.Workload(dict(bench.CONFIGS["C"]), 0, 1)
ctx = cg.Context(0, arena_bytes=int(wl.sizes.sum()) + (6 << 30), flags=cg.PROFILE)
assert ctx.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
pins = torch.from_numpy(wl.bases.view(np.int64).copy()).cuda()
assert ctx.mapArrayDevice(pins.data_ptr(), wl.U) == 0
q, _ = wl.device_queries(torch.device("cuda", 0))
R = W.reserve_readonly(1 << 20)


def step():
    assert ctx.mapArrayDevice(q.data_ptr(), wl.n) == 0
    ctx.advanceEpoch()
    assert ctx.unmapArrayDevice(q.data_ptr(), wl.n, release=True) == 0


for _ in range(3):
    step()
torch.cuda.synchronize()
nd = [0]
for declare in (False, True, False, True):
    ctx.resetStats()
    t0 = time.perf_counter()
    for k in range(5):
        if declare:
            assert ctx.declareAlloc(R + 4096 * nd[0], 1024, True) == 0
            nd[0] += 1
        step()
    torch.cuda.synchronize()
    st = ctx.stats()
    print(f"declare={declare} wall/step {1e3 * (time.perf_counter() - t0) / 5:.3f} ms  fwd {st['fwd_kernel_ms'] / max(1, st['fwd_kernel_calls']):.3f} "
          f"rev {st['rev_kernel_ms'] / max(1, st['rev_kernel_calls']):.3f} launches {st['kernel_launches']} merges {st['table_merges']} "
          f"rebuilds {st['table_rebuilds']}", flush=True)
