"""CGCM_TRACE=1 python tools/trace_A_promoted.py: host-side phases of the promoted config-A loop
(queued re-map / leased release), 50 iterations after a warm-up."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import bench_configs as bc  # noqa: E402

bc.config_A("promoted", iters=3)
r = bc.config_A("promoted", iters=50)
print(r)
import paper_conf_pldi_jablinpjjba11_b200 as cg  # noqa: E402
ctx = cg.Context(0, arena_bytes=1 << 28)
t0 = time.perf_counter()
for _ in range(20000):
    ctx.L.cgcm_epoch()
print("ctypes call us", (time.perf_counter() - t0) / 20000 * 1e6, file=sys.stderr)
