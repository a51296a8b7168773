"""Time the three calls of bench.py's e2e step separately (host wall clock around each call, which
returns synchronously) plus the hot-kernel event times the runtime records (CGCM_PROFILE).
python tools/e2e_breakdown.py [--config E|C] [--steps 3]"""
import argparse
import ctypes
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="E")
    ap.add_argument("--steps", type=int, default=3)
    a = ap.parse_args()
    wl = bench.Workload(bench.CONFIGS[a.config], 0, 1)
    dev = torch.device("cuda", 0)
    ctx = cg.Context(0, arena_bytes=int(wl.sizes.sum()) + wl.span // 8 + wl.n * 32 + (6 << 30), flags=cg.PROFILE)
    assert ctx.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
    pins = torch.from_numpy(wl.bases.view(np.int64).copy()).to(dev)
    assert ctx.mapArrayDevice(pins.data_ptr(), wl.U) == 0
    host = np.ascontiguousarray(wl.device_queries(dev).cpu().numpy().view(np.uint64))
    S = wl.slots
    outers = []
    for k in range(wl.arrays_per_rank):
        p = ctx.malloc(8 * S)
        ctypes.memmove(p, host[k * S:(k + 1) * S].ctypes.data, 8 * S)
        outers.append(p)
    print("link", bench.host_link(dev))
    for it in range(a.steps + 1):
        st0 = ctx.stats()
        t0 = time.perf_counter()
        s1, _ = ctx.mapArrays(outers)
        t1 = time.perf_counter()
        ctx.advanceEpoch()
        s2 = ctx.unmapArrays(outers)
        t2 = time.perf_counter()
        s3 = ctx.releaseArrays(outers)
        torch.cuda.synchronize()
        t3 = time.perf_counter()
        st1 = ctx.stats()
        d = {k: st1[k] - st0[k] for k in ("fwd_kernel_ms", "rev_kernel_ms", "h2d_bytes", "d2h_bytes",
                                          "h2d_memcpy_calls", "d2h_memcpy_calls", "kernel_launches")}
        print(f"step {it}: status {s1} {s2} {s3}  mapArrays {1e3 * (t1 - t0):.2f} ms  unmapArrays "
              f"{1e3 * (t2 - t1):.2f} ms  releaseArrays {1e3 * (t3 - t2):.2f} ms  total {1e3 * (t3 - t0):.2f} ms  {d}")


if __name__ == "__main__":
    main()
