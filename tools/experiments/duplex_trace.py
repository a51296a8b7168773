"""Timeline of the duplex e2e (bench.run_e2e_duplex's schedule): per thread, start/end of every call."""
import ctypes, os, sys, threading, time
import numpy as np
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_pldi_jablinpjjba11_b200 as cg  # noqa: E402

wl = bench.Workload(bench.CONFIGS["E"], 0, 1)
dev = torch.device("cuda", 0)
mk = lambda f=0: cg.Context(0, arena_bytes=int(wl.sizes.sum()) + wl.span // 8 + 128 * wl.slots * 8 * 4 + (6 << 30), flags=f)
ctxs = [mk(int(os.environ.get("CTX0_FLAGS", "0"))), mk()]
host = np.ascontiguousarray(wl.device_queries(dev).cpu().numpy().view(np.uint64))
A, S = wl.arrays_per_rank, wl.slots
outs = [[], []]
for k, c in enumerate(ctxs):
    c.make_current()
    assert c.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
    pins = torch.from_numpy(wl.bases.view(np.int64).copy()).to(dev)
    assert c.mapArrayDevice(pins.data_ptr(), wl.U) == 0
    for a in range(k * A // 2, (k + 1) * A // 2):
        p = c.malloc(8 * S)
        ctypes.memmove(p, host[a * S:(a + 1) * S].ctypes.data, 8 * S)
        outs[k].append(p)
T0 = [0.0]
log = []
lag = threading.Event()
def step(k):
    c, o = ctxs[k], outs[k]
    for name, fn in (("map", lambda: c.mapArrays(o)), ("adv", c.advanceEpoch), ("unmap", lambda: c.unmapArrays(o)),
                     ("rel", lambda: c.releaseArrays(o))):
        t = time.perf_counter()
        fn()
        log.append((k, name, round(1e3 * (t - T0[0]), 1), round(1e3 * (time.perf_counter() - T0[0]), 1)))
        if k == 0 and name == "map":
            lag.set()
def worker(k):
    ctxs[k].make_current()
    if k == 1:
        lag.wait()
    for _ in range(3):
        step(k)
for k in (0, 1):
    ctxs[k].make_current(); step(k)
torch.cuda.synchronize(); log.clear(); lag.clear()
T0[0] = time.perf_counter()
ts = [threading.Thread(target=worker, args=(k,)) for k in (0, 1)]
[t.start() for t in ts]; [t.join() for t in ts]
print("total ms", round(1e3 * (time.perf_counter() - T0[0]), 1))
for x in sorted(log, key=lambda r: r[2]):
    print(x)
for c in ctxs:
    c.make_current(); c.close()
