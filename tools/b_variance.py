import os, sys, time, json
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tools"))
import bench_configs as bc
bc.config_B(True, n=256)
for i in range(5):
    r = bc.config_B(True)
    print("promoted", i, r["seconds"], r["kernel_launches"], flush=True)
