"""CGCM_TRACE=1 python tools/trace_A.py (GPU box, repo root): host-side phases of config A's naive loop
(20 iterations after a warm-up); profiles/r02ta_*, r02tn_* were taken with it."""
import json
import os
import sys

sys.path.insert(0, os.getcwd())
sys.path.insert(0, os.path.join(os.getcwd(), "tools"))
import bench_configs as bc  # noqa: E402

bc.config_A("promoted", iters=3)
print(json.dumps(bc.config_A("naive", iters=20)))
