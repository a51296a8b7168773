import sys, os, json
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tools"))
import bench_configs as bc
bc.config_A("promoted", iters=3)
r = bc.config_A("naive", iters=20)
print(json.dumps(r))
