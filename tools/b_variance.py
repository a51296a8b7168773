"""python tools/b_variance.py [CGCM_TRACE=1] (GPU box, repo root): config B's promoted loop five times in one
process -- the run-to-run spread that exposed a pinned-buffer allocation inside the first map
(profiles/r02bw_trace.log, r02bx_trace.log)."""
import os
import sys

sys.path.insert(0, os.getcwd())
sys.path.insert(0, os.path.join(os.getcwd(), "tools"))
import bench_configs as bc  # noqa: E402

bc.config_B(True, n=256)
for i in range(5):
    r = bc.config_B(True)
    print("promoted", i, r["seconds"], r["kernel_launches"], flush=True)
