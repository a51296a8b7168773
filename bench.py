#!/usr/bin/env python
"""Benchmark of the CGCM hot path on B200 (the driver's contract; DESIGN.md §8 explains every key).

Workload (default, BASELINE.json configs[4] "E"): an allocation table of 2^22 units (sizes
log-uniform 16 B-64 KiB, gaps 0-4080 B, in a PROT_READ reservation, declared read-only and kept
active by one setup map each) and 2^28 interior CPU pointers in 256 pointer arrays of 2^20 slots;
rank r of N translates arrays [r*256/N, (r+1)*256/N) against its own replica of the table.
`--config C` runs configs[2] (2^20 units, 2^26 pointers) instead.

One step = one pass of the whole hot path over the rank's batch, through the C ABI:
  cgcm_mapArrayDevice   a1 lookup + a2 forward rewrite in place + per-slot refcount (Alg. 1)
  cgcm_advanceEpoch     one GPU function launch happened
  cgcm_unmapArrayDevice a1 reverse lookup + a3 reverse rewrite in place + a4 epoch gate of every AU
                        touched (Alg. 2; read-only units: no copy) + release of every slot (Alg. 3)
`value` = pointer translations per second (2 per slot per step: forward and reverse), inputs resident
in HBM; `e2e` = the same metric through cgcm_mapArrays/unmapArrays/releaseArrays on the pointer arrays
in pinned host memory (host<->device copies of the arrays inside the timed region).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

CONFIGS = {
    "E": dict(U=1 << 22, arrays=256, slots=1 << 20, seed=5, name="E: 2^28 interior pointers in 256 arrays, "
              "replicated 2^22-unit table"),
    "C": dict(U=1 << 20, arrays=64, slots=1 << 20, seed=3, name="C: 2^26 interior pointers, 2^20-unit table"),
    "T": dict(U=1 << 12, arrays=8, slots=1 << 12, seed=3, name="T: tiny debug configuration"),
    # kernel experiments only (not bench lines): E's batch against smaller tables (table working set vs L2)
    "E20": dict(U=1 << 20, arrays=256, slots=1 << 20, seed=5, name="experiment: E's batch, 2^20-unit table"),
    "E21": dict(U=1 << 21, arrays=256, slots=1 << 20, seed=5, name="experiment: E's batch, 2^21-unit table"),
}
METRIC = "translated pointers/sec and map+unmap GB/s per B200 (and 8-GPU), % of HBM roofline"
BYTES_PER_TRANSLATION = 16  # 8 B read + 8 B write of the pointer slot


def env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0}, "fallback"


def start_clock_sampler(uuid: str | None):
    cmd = ["nvidia-smi", "--query-gpu=uuid,clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
           "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
           "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
           "--format=csv,noheader,nounits", "-lms", "20"]
    if uuid:
        cmd[1:1] = ["-i", uuid]
    try:
        return subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
    except Exception:
        return None


def stop_clock_sampler(p):
    if p is None:
        return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
    p.terminate()
    try:
        out, _ = p.communicate(timeout=5)
    except Exception:
        p.kill()
        out = ""
    sm, mx, reasons = [], [], set()
    names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
    for line in out.strip().splitlines():
        f = [x.strip() for x in line.split(",")]
        if len(f) < 8:
            continue
        try:
            sm.append(float(f[1]))
            mx.append(float(f[2]))
        except ValueError:
            continue
        for n, v in zip(names, f[4:8]):
            if v.lower().startswith("active"):
                reasons.add(n)
    return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
            "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------------------------
# the workload
# ---------------------------------------------------------------------------------------------
class Workload:
    def __init__(self, cfg, rank, world):
        self.cfg = cfg
        self.U = cfg["U"]
        self.seed = cfg["seed"]
        self.offs, self.sizes, self.span = W.table_layout(self.U, self.seed)
        self.R = W.reserve_readonly(self.span)
        self.bases = self.offs + np.uint64(self.R)
        A = cfg["arrays"]
        assert A % world == 0, "arrays must divide evenly across ranks"
        self.arrays_per_rank = A // world
        self.slots = cfg["slots"]
        self.first_array = rank * self.arrays_per_rank
        self.n = self.arrays_per_rank * self.slots
        self.start = self.first_array * self.slots  # query index of this rank's first slot

    def device_queries(self, device):
        import torch
        ot = torch.from_numpy(self.offs.view(np.int64)).to(device)
        st = torch.from_numpy(self.sizes.view(np.int64)).to(device)
        q, u = W.queries_t(ot, st, self.n, self.seed, start=self.start)
        q += self.R
        return q, u

    def host_sample(self, n):
        q, _ = W.queries(self.offs, self.sizes, n, self.seed, start=self.start)
        return (q + np.uint64(self.R)).astype(np.uint64)


def run_cgcm(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import paper_conf_pldi_jablinpjjba11_b200 as cg

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    cfg = CONFIGS[args.config]
    t0 = time.time()
    wl = Workload(cfg, rank, world)
    total_bytes = int(wl.sizes.sum())
    arena = total_bytes + wl.span // 8 + wl.n * 8 * 4 + (6 << 30)
    ctx = cg.Context(local_rank, arena_bytes=arena, flags=cg.PROFILE)
    assert ctx.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
    # one reference per unit held for the whole run (map promotion of the table's maps)
    pins = torch.from_numpy(wl.bases.view(np.int64).copy()).to(dev)
    s = ctx.mapArrayDevice(pins.data_ptr(), wl.U)
    assert s == 0, cg.strerror(s)
    setup_act_s = time.time() - t0
    q, q_unit = wl.device_queries(dev)
    q_ref = q.clone()
    torch.cuda.synchronize()
    setup_s = time.time() - t0

    def step():
        s1 = ctx.mapArrayDevice(q.data_ptr(), wl.n)
        ctx.advanceEpoch()
        s2 = ctx.unmapArrayDevice(q.data_ptr(), wl.n, release=True)
        if s1 or s2:
            raise RuntimeError(f"step failed: {cg.strerror(s1)} / {cg.strerror(s2)}")

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    assert torch.equal(q, q_ref), "round trip changed the pointer arrays"

    uuid = None
    try:
        uuid = str(torch.cuda.get_device_properties(dev).uuid)
        if uuid and not uuid.startswith("GPU-"):
            uuid = "GPU-" + uuid
    except Exception:
        uuid = None
    sampler = start_clock_sampler(uuid)
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ctx.resetStats()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(ctx.main)
    for _ in range(args.steps):
        step()
    ev1.record(ctx.main)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = stop_clock_sampler(sampler)
    ms = ev0.elapsed_time(ev1)
    st = ctx.stats()
    index_format = int(ctx.indexInfo().get("pd_format", 0))
    assert torch.equal(q, q_ref), "round trip changed the pointer arrays"
    if world > 1:
        ms = max_over_ranks(ms, dev)
    ms_per_step = ms / args.steps
    parity = full_size_check(ctx, wl, q, q_ref, q_unit, pins_held=1)
    del q_unit
    merge = declares_between_batches(ctx, step, reps=min(16, args.steps))
    translations = 2 * wl.n * world * args.steps
    value = translations / (ms / 1e3)

    # roofline of the dominant kernel (per-launch event times on the launch stream)
    peaks, peak_kind = measured_peaks()
    fwd_ms = st["fwd_kernel_ms"] / max(1, st["fwd_kernel_calls"])
    rev_ms = st["rev_kernel_ms"] / max(1, st["rev_kernel_calls"])
    fwd_slots = st["fwd_kernel_slots"] / max(1, st["fwd_kernel_calls"])
    rev_slots = st["rev_kernel_slots"] / max(1, st["rev_kernel_calls"])
    dom = "rev" if rev_ms >= fwd_ms else "fwd"
    kms, kslots = (rev_ms, rev_slots) if dom == "rev" else (fwd_ms, fwd_slots)
    achieved = BYTES_PER_TRANSLATION * kslots / (kms / 1e3) / 1e9
    traffic = None
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof):
        try:
            with open(prof) as f:
                traffic = json.load(f).get(args.config, {}).get(dom)
        except Exception:
            traffic = None
    roofline = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": traffic,
                # the hot kernels cgcm_mapArrayDevice / cgcm_unmapArrayDevice launch on one segment
                "kernel": "k_rev_fast<DEC> (rev)" if dom == "rev" else "k_fwd_fast (fwd)",
                "peak_source": peak_kind,
                "fwd_ms_per_launch": round(fwd_ms, 4), "rev_ms_per_launch": round(rev_ms, 4),
                "fwd_gbs": round(BYTES_PER_TRANSLATION * fwd_slots / (fwd_ms / 1e3) / 1e9, 1) if fwd_ms else None,
                "rev_gbs": round(BYTES_PER_TRANSLATION * rev_slots / (rev_ms / 1e3) / 1e9, 1) if rev_ms else None}
    roofline["l2_random_ops"] = l2_op_roof(fwd_ms, fwd_slots, rev_ms, rev_slots, index_format)
    gpu_launches = int(st["kernel_launches"])

    # the e2e legs run on fresh contexts without CGCM_PROFILE (its per-launch event syncs would serialise
    # the host threads of the duplex leg); the hot-path context is released first
    ctx.close()
    e2e = None
    if not args.no_e2e:
        ctxa = table_context(wl, dev, local_rank, wl.n)
        try:
            e2e = run_e2e(args, ctxa, wl, q_ref, dev, world, rank)
            if not args.no_duplex:
                try:
                    dup = run_e2e_duplex(args, ctxa, wl, q_ref, dev, world, rank, e2e["host_link"], local_rank)
                except Exception as ex:  # e.g. not enough device memory for a second replica
                    dup = None
                    e2e["duplex_error"] = str(ex)[:200]
                if dup is not None:
                    dup["single_context"] = e2e
                    e2e = dup
        finally:
            ctxa.make_current()
            ctxa.close()

    result = {
        "metric": METRIC, "value": round(value, 1), "unit": "pointer translations/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic (seeded splitmix64; PROT_READ zero-page table, interior pointers)",
        "config": {"workload": cfg["name"], "units": wl.U, "pointers_per_step": wl.n * world,
                   "pointers_per_rank": wl.n, "arrays": cfg["arrays"], "parallelism": f"replicated table, "
                   f"{cfg['arrays'] // world} arrays per rank", "l2": "inputs (2 GiB/GPU of pointer slots at E) "
                   "exceed L2 between iterations; table stays L2-resident by design",
                   "translations_per_step": 2 * wl.n * world},
        "roofline": roofline, "gpu_launches": gpu_launches, "clocks": clocks, "e2e": e2e, "parity": parity,
        "merge": merge,
        "setup_s": round(setup_s, 1), "setup_activation_s": round(setup_act_s, 1),
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        result["cpu_baseline"] = cpu_baseline(wl, args.cpu_sample, steps=3)
    return result


def declares_between_batches(ctx, step, reps):
    """NEXT-1: the cost of keeping the table current while map batches run -- one new AU declared
    between every two steps of the timed workload (merged into the device table as a delta unit, no
    rebuild), vs the same steps without declarations; CUDA events around each run."""
    import torch
    span = 1 << 20
    R = W.reserve_readonly(span)
    try:
        def run(declare):
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            ev0.record(ctx.main)
            for k in range(reps):
                if declare:
                    assert ctx.declareAlloc(R + 4096 * run.n, 1024, True) == 0
                    run.n += 1
                step()
            ev1.record(ctx.main)
            torch.cuda.synchronize()
            return ev0.elapsed_time(ev1), time.perf_counter() - t0
        run.n = 0
        assert ctx.declareAlloc(R + 4096 * 255, 1024, True) == 0  # first merge: lazy module loading, not timed
        step()
        s0 = ctx.stats()
        base_ms, base_wall = run(False)
        with_ms, with_wall = run(True)
        s1 = ctx.stats()
        return {"declares": reps, "ms_per_step_without": round(base_ms / reps, 4),
                "ms_per_step_with_one_declare": round(with_ms / reps, 4),
                "us_per_declare_between_batches": round(1e3 * (with_ms - base_ms) / reps, 1),  # device time
                "us_per_declare_wall": round(1e6 * (with_wall - base_wall) / reps, 1),
                "declares_per_s_with_batches": round(reps / max(1e-9, with_wall), 1),
                "table_merges": s1["table_merges"] - s0["table_merges"],
                "table_rebuilds": s1["table_rebuilds"] - s0["table_rebuilds"]}
    finally:
        pass


def full_size_check(ctx, wl, q, q_ref, q_unit, pins_held):
    """Parity of the timed call at the benchmarked size, outside the timed region: one more
    cgcm_mapArrayDevice over all of the rank's slots in the timed launch configuration, then every slot
    is compared with Alg. 1's closed form devptr(u) + (p - base(u)) (u = the unit the seeded
    generator drew the query from, the table's devptr and base from cgcm_dumpTable), every unit's
    refcount with the setup reference + the number of slots pointing into it (A8), and after
    cgcm_unmapArrayDevice(release) every slot with its original CPU pointer and every refcount with the
    setup reference alone (a3 round trip + Alg. 3).  Vectorised with torch on the GPU (the oracle's
    one-by-one sampled check at this size is tests/test_gpu_fullsize.py)."""
    import torch
    dev = q.device
    t0 = time.time()
    assert ctx.mapArrayDevice(q.data_ptr(), wl.n) == 0
    tab = ctx.dump_np()
    devt = torch.from_numpy(tab["devptr"].view(np.int64)).to(dev)
    bt = torch.from_numpy(tab["base"].view(np.int64)).to(dev)
    fwd_ok = bool(torch.equal(q, devt[q_unit] + (q_ref - bt[q_unit])))
    del devt, bt
    cnt = torch.bincount(q_unit, minlength=wl.U).cpu().numpy()
    rc_ok = bool((tab["refCount"] == cnt + pins_held).all())
    ctx.advanceEpoch()
    assert ctx.unmapArrayDevice(q.data_ptr(), wl.n, release=True) == 0
    rev_ok = bool(torch.equal(q, q_ref))
    rc_back = bool((ctx.dump_np()["refCount"] == pins_held).all())
    ok = fwd_ok and rc_ok and rev_ok and rc_back
    if not ok:
        raise RuntimeError(f"full-size parity failed: fwd {fwd_ok} rc {rc_ok} rev {rev_ok} rc_back {rc_back}")
    return {"checked_slots": wl.n, "forward_closed_form": fwd_ok, "refcounts": rc_ok, "roundtrip": rev_ok,
            "released": rc_back, "seconds": round(time.time() - t0, 1),
            "how": "every slot vs devptr(u)+(p-base(u)); refcount == 1 + #slots in u; reverse == original"}


def l2_op_roof(fwd_ms, fwd_slots, rev_ms, rev_slots, pd_format):
    """The roof that binds: each hot kernel's time is bounded below by its random L2
    operations per slot divided by the measured rate of random 32-byte gathers into an L2-resident array on
    this GPU (tools/l2_gather.cu, committed log).  With deferred references (the timed calls) neither pass
    issues a refcount reduction: k_fwd_fast gathers the page entry and, with v2 entries (E), the unit's
    compact word (v3 entries, C: the entry alone); k_rev_fast gathers the unit's state word."""
    g, r = 238.9, 188.4  # G/s, profiles/r01j_l2_gather.log (gather32 at 48 MiB, red_s32)
    try:
        with open(os.path.join(ROOT, "profiles", "r01j_l2_gather.log")) as f:
            for ln in f:
                d = json.loads(ln)
                if d.get("test") == "gather32" and d.get("buffer_MiB") == 48:
                    g = d["G_per_s"]
                if d.get("test") == "red_s32":
                    r = d["G_per_s"]
    except Exception:
        pass
    fg = 1 if pd_format == 3 else 2
    fwd_floor = fwd_slots * fg / g / 1e6  # ms
    rev_floor = rev_slots * 1 / g / 1e6
    return {"gather_gps": g, "source": "profiles/r01j_l2_gather.log",
            "fwd_ops_per_slot": "page entry" + (" + unit word" if fg == 2 else "") + f" (v{pd_format} entries)",
            "rev_ops_per_slot": "state word",
            "fwd_floor_ms": round(fwd_floor, 4), "rev_floor_ms": round(rev_floor, 4),
            "fwd_frac": round(fwd_floor / fwd_ms, 4) if fwd_ms else None,
            "rev_frac": round(rev_floor / rev_ms, 4) if rev_ms else None}


def host_link(dev, nbytes=256 << 20, reps=10):
    """Pinned host<->device copy bandwidth of this GPU's link (256 MiB, best of 10, CUDA
    events): H2D, D2H, and both directions at once on two streams (bidir = total bytes / span)."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    h2 = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d2 = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    s = torch.cuda.Stream(device=dev)
    s2 = torch.cuda.Stream(device=dev)
    best = None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e2 = torch.cuda.Event()
        torch.cuda.synchronize(dev)
        e0.record(s)
        s2.wait_event(e0)
        with torch.cuda.stream(s):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        e2.record(s2)
        s.wait_event(e2)
        e1.record(s)
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
    out = {"bidir_gbs": round(2 * nbytes / (best / 1e3) / 1e9, 1)}
    for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
        best = None
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(s):
                e0.record(s)
                fn()
                e1.record(s)
            e1.synchronize()
            ms = e0.elapsed_time(e1)
            best = ms if best is None else min(best, ms)
        out[name + "_gbs"] = round(nbytes / (best / 1e3) / 1e9, 1)
    return out


def run_e2e(args, ctx, wl, q_ref, dev, world, rank):
    """Same metric through the host-array public API: cgcm_mapArrays / unmapArrays / releaseArrays on
    the rank's pointer arrays in pinned host memory (raw arrays H2D, translated in place, reverse
    translated and copied back every step)."""
    import ctypes
    import torch
    A, S = wl.arrays_per_rank, wl.slots
    host = np.ascontiguousarray(q_ref.cpu().numpy().view(np.uint64))
    outers = []
    for a in range(A):
        p = ctx.malloc(8 * S)
        if not p:
            return {"value": None, "error": "cgcm_malloc failed"}
        ctypes.memmove(p, host[a * S:(a + 1) * S].ctypes.data, 8 * S)
        outers.append(p)

    def step():
        s1, _ = ctx.mapArrays(outers)
        ctx.advanceEpoch()
        s2 = ctx.unmapArrays(outers)
        s3 = ctx.releaseArrays(outers)
        if s1 or s2 or s3:
            raise RuntimeError(f"e2e step failed {s1} {s2} {s3}: {ctx.L.cgcm_lastCudaError().decode()}")

    step()
    torch.cuda.synchronize()
    steps = max(1, min(args.steps, args.e2e_steps))
    st0 = ctx.stats()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(ctx.main)
    for _ in range(steps):
        step()
    ev1.record(ctx.main)
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1)
    st1 = ctx.stats()
    ok = all(np.array_equal(np.ctypeslib.as_array((ctypes.c_uint64 * S).from_address(p)), host[a * S:(a + 1) * S])
             for a, p in enumerate(outers))
    for p in outers:
        ctx.free(p)
    if world > 1:
        import torch.distributed as dist
        ms = max_over_ranks(ms, dev)
    link = host_link(dev)
    h2d = (st1["h2d_bytes"] - st0["h2d_bytes"]) // steps
    d2h = (st1["d2h_bytes"] - st0["d2h_bytes"]) // steps
    floor_ms = 1e3 * (h2d / (link["h2d_gbs"] * 1e9) + d2h / (link["d2h_gbs"] * 1e9))
    return {"value": round(2 * wl.n * world * steps / (ms / 1e3), 1), "unit": "pointer translations/s",
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "host_link": link, "host_link_floor_ms_per_step": round(floor_ms, 3),
            "frac_of_host_link": round(floor_ms / (ms / steps), 4),
            "ms_per_step": round(ms / steps, 3), "steps": steps,
            "api": "cgcm_mapArrays+advanceEpoch+cgcm_unmapArrays+cgcm_releaseArrays (pinned host arrays)",
            "host_arrays_roundtrip_ok": bool(ok)}


def table_context(wl, dev, local_rank, nslots):
    """A context holding the workload's table, every unit kept active by one setup reference (as the
    hot-path context), with arena room for nslots pointer slots of arrays and their scratch."""
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    c = cg.Context(local_rank, arena_bytes=int(wl.sizes.sum()) + wl.span // 8 + nslots * 8 * 4 + (6 << 30))
    assert c.declareBatch(wl.bases, wl.sizes, readonly=True) == 0
    pins = torch.from_numpy(wl.bases.view(np.int64).copy()).to(dev)
    s = c.mapArrayDevice(pins.data_ptr(), wl.U)
    assert s == 0, cg.strerror(s)
    torch.cuda.synchronize()
    return c


def run_e2e_duplex(args, ctx, wl, q_ref, dev, world, rank, link, local_rank):
    """The e2e step with both directions of the (full-duplex) host link busy: the rank's arrays are
    split into k parts (--e2e-parts, default 2; 3 measured slower), each driven through its own context (its own replica of
    the table, arena and streams) by its own host thread, part i starting once part i-1's first upload is
    done -- while one part copies its translated arrays back (unmapArrays), another uploads its raw arrays
    (mapArrays), and the per-call overheads of one part hide behind the others' copies.  Same public calls,
    same bytes every step; CUDA events on the first context's main stream span all threads."""
    import ctypes
    import threading
    import torch
    A, S = wl.arrays_per_rank, wl.slots
    K = max(2, min(args.e2e_parts, A))
    if A < 2:
        return None
    host = np.ascontiguousarray(q_ref.cpu().numpy().view(np.uint64))
    bounds = [A * k // K for k in range(K + 1)]
    ctxs = [ctx] + [table_context(wl, dev, local_rank, (bounds[k + 1] - bounds[k]) * S) for k in range(1, K)]
    try:
        parts = [(ctxs[k], list(range(bounds[k], bounds[k + 1]))) for k in range(K)]
        outers = [[] for _ in range(K)]
        for k, (c, rng) in enumerate(parts):
            c.make_current()
            for a in rng:
                p = c.malloc(8 * S)
                assert p, "cgcm_malloc failed"
                ctypes.memmove(p, host[a * S:(a + 1) * S].ctypes.data, 8 * S)
                outers[k].append(p)
        errs = []

        trace = [] if os.environ.get("CGCM_BENCH_TRACE") else None
        started = [threading.Event() for _ in range(K)]

        def step(k):
            c, o = parts[k][0], outers[k]
            t0 = time.perf_counter()
            s1, _ = c.mapArrays(o)
            if k + 1 < K and not started[k + 1].is_set():
                started[k + 1].set()  # the next part starts once this part's first upload is done
            c.advanceEpoch()
            t1 = time.perf_counter()
            s2 = c.unmapArrays(o)
            t2 = time.perf_counter()
            s3 = c.releaseArrays(o)
            if trace is not None:
                trace.append((k, round(1e3 * t0, 1), round(1e3 * t1, 1), round(1e3 * t2, 1), round(1e3 * time.perf_counter(), 1)))
            if s1 or s2 or s3:
                errs.append((k, s1, s2, s3, c.L.cgcm_lastCudaError().decode()))

        def worker(k, steps):
            parts[k][0].make_current()
            started[k].wait()
            for _ in range(steps):
                step(k)

        for e in started:
            e.set()
        for k in range(K):  # warm-up, one part at a time
            parts[k][0].make_current()
            step(k)
        torch.cuda.synchronize()
        steps = max(1, min(args.steps, args.e2e_steps))
        st0 = [c.stats() for c, _ in parts]
        for e in started[1:]:
            e.clear()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(ctx.main)
        ts = [threading.Thread(target=worker, args=(k, steps)) for k in range(K)]
        for t in ts:
            t.start()
        for t in ts:
            t.join()
        for c in ctxs[1:]:
            e = torch.cuda.Event()
            e.record(c.main)
            ctx.main.wait_event(e)
        ev1.record(ctx.main)
        torch.cuda.synchronize()
        if errs:
            raise RuntimeError(f"e2e duplex step failed: {errs[0]}")
        if trace:
            z = min(x[1] for x in trace)
            for x in sorted(trace, key=lambda r: r[1]):
                print("duplex", x[0], [round(v - z, 1) for v in x[1:]], file=sys.stderr)
        ms = ev0.elapsed_time(ev1)
        st1 = [c.stats() for c, _ in parts]
        ok = all(np.array_equal(np.ctypeslib.as_array((ctypes.c_uint64 * S).from_address(p)), host[a * S:(a + 1) * S])
                 for k in range(K) for a, p in zip(parts[k][1], outers[k]))
        for k in range(K):
            parts[k][0].make_current()
            for p in outers[k]:
                parts[k][0].free(p)
    finally:
        for c in ctxs[1:]:
            c.close()
        ctx.make_current()
    if world > 1:
        import torch.distributed as dist
        ms = max_over_ranks(ms, dev)
    h2d = sum(b["h2d_bytes"] - a["h2d_bytes"] for a, b in zip(st0, st1)) // steps
    d2h = sum(b["d2h_bytes"] - a["d2h_bytes"] for a, b in zip(st0, st1)) // steps
    floor_ms = 1e3 * (h2d + d2h) / (link["bidir_gbs"] * 1e9)  # both directions busy at once
    return {"value": round(2 * wl.n * world * steps / (ms / 1e3), 1), "unit": "pointer translations/s",
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "host_link": link, "host_link_floor_ms_per_step": round(floor_ms, 3),
            "frac_of_host_link": round(floor_ms / (ms / steps), 4),
            "ms_per_step": round(ms / steps, 3), "steps": steps,
            "api": "cgcm_mapArrays+advanceEpoch+cgcm_unmapArrays+cgcm_releaseArrays (pinned host arrays), "
                   f"{K} parts through {K} contexts, each one upload phase behind the previous (full-duplex link)",
            "host_arrays_roundtrip_ok": bool(ok)}


# ---------------------------------------------------------------------------------------------
# CPU oracle timing (the cpu_baseline leg and the --impl reference arm)
# ---------------------------------------------------------------------------------------------
def oracle_setup(wl):
    from oracle import Oracle
    o = Oracle()
    for b, s in zip(wl.bases.tolist(), wl.sizes.tolist()):
        assert o.declareAlloc(b, s, readonly=True) == 0
    pins = wl.bases.astype(np.uint64).copy()
    assert o.mapSlots(pins) == 0     # the same setup references the GPU run holds
    return o


def oracle_step(o, slots):
    s = slots.copy()
    t0 = time.perf_counter()
    assert o.mapSlots(s) == 0
    o.advanceEpoch()
    assert o.unmapSlots(s, release=True) == 0
    return time.perf_counter() - t0, s


def host_info():
    """The GPU box's host CPU (record nproc and the CPU model)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "affinity": len(os.sched_getaffinity(0)), "cpu_model": model}


def cpu_baseline(wl, sample, steps=1, o=None):
    """The CPU oracle timed on one core (pinned with sched_setaffinity, the taskset -c of SURVEY §8(d)),
    best of `steps` (one step when a step exceeds 10 s), on the first `sample` slots of the workload;
    plus the timing-only all-cores std::upper_bound baseline (tools/cpu_baseline.cpp) on 1/16 of it."""
    allowed = os.sched_getaffinity(0)
    core = min(allowed)
    o = o or oracle_setup(wl)
    slots = wl.host_sample(sample)
    best = None
    os.sched_setaffinity(0, {core})
    try:
        for k in range(steps):
            dt, s = oracle_step(o, slots)
            assert (s == slots).all()
            best = dt if best is None else min(best, dt)
            if dt > 10:
                break
    finally:
        os.sched_setaffinity(0, allowed)
    o.close()
    res = {"value": round(2 * sample / best, 1), "unit": "pointer translations/s", "cores": 1, "kind": "oracle",
           "sample": f"first {sample} slots of rank 0's arrays (same table, same setup references): "
                     f"mapSlots + advanceEpoch + unmapSlots(release), single-threaded C++ std::map oracle pinned "
                     f"to core {core}, best of up to {steps}",
           "seconds": round(best, 3), "host": host_info()}
    try:
        res["all_cores"] = cpu_all_cores(wl, min(wl.n, 1 << 24))
    except Exception as ex:  # timing-only extra: never fails the bench
        res["all_cores"] = {"error": str(ex)[:200]}
    return res


def cpu_all_cores(wl, n, reps=3):
    """tools/cpu_baseline.cpp: the step as a straightforward OpenMP program over all host cores (sorted
    table + std::upper_bound, atomic refcounts, epoch gate), timing only, best of reps."""
    import ctypes
    lib = build_cpu_baseline()
    L = ctypes.CDLL(lib)
    L.cpu_baseline_step.restype = ctypes.c_double
    L.cpu_baseline_step.argtypes = [ctypes.c_void_p] * 3 + [ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64,
                                                            ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
    L.cpu_baseline_threads.restype = ctypes.c_int
    threads = len(os.sched_getaffinity(0))
    base = np.ascontiguousarray(wl.bases, dtype=np.uint64)
    size = np.ascontiguousarray(wl.sizes, dtype=np.uint64)
    dev = (base - np.uint64(1 << 40)).astype(np.uint64)          # a mirrored device layout
    slots = wl.host_sample(n)
    ref = slots.copy()
    tr = ctypes.c_uint64(0)
    sec = L.cpu_baseline_step(base.ctypes.data, size.ctypes.data, dev.ctypes.data, len(base), slots.ctypes.data,
                              n, threads, reps, ctypes.byref(tr))
    if sec <= 0 or not (slots == ref).all():
        raise RuntimeError("cpu baseline step failed")
    return {"value": round(tr.value / sec, 1), "unit": "pointer translations/s", "cores": threads,
            "kind": "all-cores std::upper_bound (tools/cpu_baseline.cpp, timing only)",
            "sample": f"first {n} slots of rank 0's arrays (1/{max(1, wl.n // n)} of the rank's batch), best of {reps}",
            "seconds": round(sec, 3)}


def build_cpu_baseline():
    src = os.path.join(ROOT, "tools", "cpu_baseline.cpp")
    lib = os.path.join(ROOT, "tools", "libcpu_baseline.so")
    if not os.path.exists(lib) or os.path.getmtime(lib) < os.path.getmtime(src):
        subprocess.check_call(["g++", "-O3", "-std=c++17", "-fopenmp", "-shared", "-fPIC", "-o", lib, src])
    return lib


def run_reference(args, rank, world):
    if rank != 0:
        return None
    cfg = CONFIGS[args.config]
    wl = Workload(cfg, 0, 1)
    o = oracle_setup(wl)
    slots = wl.host_sample(args.ref_sample)
    for _ in range(args.warmup):
        oracle_step(o, slots)
    total = 0.0
    for _ in range(args.steps):
        dt, s = oracle_step(o, slots)
        total += dt
    o.close()
    value = 2 * args.ref_sample * args.steps / total
    cpu = {"value": round(value, 1), "unit": "pointer translations/s", "cores": 1, "kind": "oracle",
           "sample": f"{args.ref_sample} slots per step of rank 0's arrays against the full table"}
    return {"impl": "reference", "metric": METRIC, "value": round(value, 1), "unit": "pointer translations/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(total / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u64", "data": "synthetic", "config": {"workload": cfg["name"],
            "units": wl.U, "pointers_per_step": args.ref_sample, "parallelism": "single core"},
            "cpu_baseline": cpu, "e2e": {"value": round(value, 1), "unit": "pointer translations/s",
                                         "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def max_over_ranks(x, dev):
    """The max of x over all ranks (NCCL: on the device; gloo, --allow-shared-gpu: on the host)."""
    import torch
    import torch.distributed as dist
    on_dev = dist.get_backend() == "nccl"
    t = torch.tensor([x], dtype=torch.float64, device=dev if on_dev else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def run_config_line(args):
    """bench.py --config A|B|D: the secondary configs as one contract-shaped JSON line each,
    with the CPU oracle timed beside them (tools/bench_configs.py holds both sides)."""
    import importlib.util
    import torch
    spec = importlib.util.spec_from_file_location("bench_configs", os.path.join(ROOT, "tools", "bench_configs.py"))
    bc = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(bc)
    torch.cuda.set_device(0)
    link = host_link(torch.device("cuda", 0))
    sampler = start_clock_sampler(None)
    common = {"n_gpus": 1, "warmup": args.warmup, "scaling": "strong", "vs_baseline": None, "dtype": "u64+f64",
              "data": "synthetic (seeded splitmix64 values; pinned cgcm_malloc heap)"}
    if args.config == "A":
        for _ in range(args.warmup):
            bc.config_A("promoted", iters=3)  # lazy module loading, clocks
        modes = {m: bc.config_A(m) for m in ("naive", "promoted", "region", "region_check")}
        clocks = stop_clock_sampler(sampler)
        pro, nai = modes["promoted"], modes["naive"]
        orc = {m: bc.oracle_A(m) for m in ("naive", "promoted")}
        it = pro["iterations"]
        res = {"metric": "config A (jagged 256x256 fp64, 100 iterations of mapArray/S1/unmapArray/releaseArray): "
                         "us per iteration, map-promoted loop", "value": pro["us_per_iteration"],
               "unit": "us/iteration", "higher_is_better": False, "steps": it,
               "ms_per_step": round(pro["us_per_iteration"] / 1e3, 4), **common,
               "config": {"workload": "A: 256 row AUs of 2 KiB + the row-pointer AU (BASELINE configs[0])",
                          "mode": "promoted (Listing 4)"},
               "modes": modes, "speedup_promoted_vs_naive": round(nai["us_per_iteration"] / pro["us_per_iteration"], 2),
               "e2e": {"value": pro["us_per_iteration"], "unit": "us/iteration",
                       "h2d_bytes_per_step": pro["h2d_bytes"] // it, "d2h_bytes_per_step": pro["d2h_bytes"] // it,
                       "naive_us_per_iteration": nai["us_per_iteration"],
                       "naive_h2d_bytes_per_step": nai["h2d_bytes"] // it, "naive_d2h_bytes_per_step": nai["d2h_bytes"] // it},
               "roofline": {"bound": "latency", "achieved": None, "peak": None, "unit": "us/call", "frac": None,
                            "traffic": None, "note": "512 KiB per naive iteration: call latency, not bandwidth, binds"},
               "gpu_launches": pro["kernel_launches"], "clocks": clocks, "host_link": link,
               "cpu_baseline": {"value": orc["promoted"]["us_per_iteration"], "unit": "us/iteration", "cores": 1,
                                "kind": "oracle", "sample": "the whole config (100 iterations), simulated memories",
                                "naive_us_per_iteration": orc["naive"]["us_per_iteration"], "host": host_info()}}
    elif args.config == "B":
        bc.config_B(True, n=256)  # warm-up
        modes = {"promoted": bc.config_B(True), "naive": bc.config_B(False)}
        clocks = stop_clock_sampler(sampler)
        pro, nai = modes["promoted"], modes["naive"]
        orc = {"promoted": bc.oracle_B(True), "naive": bc.oracle_B(False)}
        res = {"metric": "config B (PolyBench-shaped gemm on jagged 4096^2 fp64, 64 row-blocks): seconds for the "
                         "whole loop, map-promoted", "value": pro["seconds"], "unit": "s", "higher_is_better": False,
               "steps": 64, "ms_per_step": round(1e3 * pro["seconds"] / 64, 3), **common,
               "config": {"workload": "B: 3 x 4096 row AUs of 32 KiB + 3 row-pointer AUs (BASELINE configs[1])",
                          "mode": "promoted"},
               "modes": modes, "speedup_promoted_vs_naive": round(nai["seconds"] / pro["seconds"], 2),
               "e2e": {"value": pro["seconds"], "unit": "s", "h2d_bytes_per_step": pro["h2d_bytes"] // 64,
                       "d2h_bytes_per_step": pro["d2h_bytes"] // 64, "naive_seconds": nai["seconds"]},
               "roofline": {"bound": "host_link", "achieved": round((nai["h2d_bytes"] + nai["d2h_bytes"]) / nai["seconds"] / 1e9, 2),
                            "peak": link["h2d_gbs"], "unit": "GB/s",
                            "frac": round((nai["h2d_bytes"] + nai["d2h_bytes"]) / nai["seconds"] / 1e9 / link["h2d_gbs"], 4),
                            "traffic": None, "note": "naive loop: copy bytes over its wall time vs one-way link"},
               "gpu_launches": pro["kernel_launches"], "clocks": clocks, "host_link": link,
               "cpu_baseline": {"value": orc["promoted"]["seconds"], "unit": "s", "cores": 1, "kind": "oracle",
                                "sample": orc["promoted"]["sample"], "naive_seconds": orc["naive"]["seconds"],
                                "host": host_info()}}
    elif args.config == "D":
        bc.config_D(N=1 << 16)  # warm-up
        d = bc.config_D()
        clocks = stop_clock_sampler(sampler)
        orc = bc.oracle_D(1 << 20)
        b = 48 * d["nodes"]
        gbs = 2 * b / (d["map_seconds"] + d["unmap_seconds"]) / 1e9
        res = {"metric": "config D (2^24-node pointer tree): map+unmap GB/s over the host link",
               "value": round(gbs, 2), "unit": "GB/s", "higher_is_better": True, "steps": 1,
               "ms_per_step": round(1e3 * (d["map_seconds"] + d["unmap_seconds"]), 2), **common,
               "config": {"workload": "D: 2^24 node AUs of 32 B + child table of 2^25 slots (BASELINE configs[3])"},
               "detail": d,
               "e2e": {"value": round(gbs, 2), "unit": "GB/s", "h2d_bytes_per_step": d["h2d_bytes"],
                       "d2h_bytes_per_step": d["d2h_bytes"]},
               "roofline": {"bound": "host_link", "achieved": round(gbs, 2), "peak": link["h2d_gbs"], "unit": "GB/s",
                            "frac": round(gbs / link["h2d_gbs"], 4), "traffic": None},
               "gpu_launches": d["kernel_launches"], "clocks": clocks, "host_link": link,
               "cpu_baseline": {"value": round(2 * 48 * orc["nodes"] / (orc["map_seconds"] + orc["unmap_seconds"]) / 1e9, 4),
                                "unit": "GB/s", "cores": 1, "kind": "oracle",
                                "sample": f"{orc['nodes']} nodes (1/16 of 2^24), simulated memories", "detail": orc,
                                "host": host_info()}}
    else:
        raise SystemExit(f"unknown config {args.config}")
    print(json.dumps(res), flush=True)


def relaunch_under_torchrun(args):
    """`python bench.py --gpus N` without a launcher: re-execute under torch.distributed.run with one
    rank per GPU (rendezvous on 127.0.0.1), so that --gpus is never silently ignored."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    r = subprocess.run(cmd)
    sys.exit(r.returncode)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)  # ~200 ms timed at E: several clock samples
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="cgcm", choices=["cgcm", "reference"])
    ap.add_argument("--config", default="E", choices=sorted(CONFIGS) + ["A", "B", "D"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-duplex", action="store_true", help="e2e through one context only")
    ap.add_argument("--e2e-steps", type=int, default=6)
    ap.add_argument("--e2e-parts", type=int, default=2, help="contexts (threads) of the duplex e2e leg (3: slower, profiles/r02e3_*)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=1 << 21)
    ap.add_argument("--ref-sample", type=int, default=1 << 19)
    ap.add_argument("--allow-shared-gpu", action="store_true",
                    help="testing only: let several ranks share one GPU (numbers are meaningless)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch_under_torchrun(args)  # does not return
    rank, world, local_rank = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}: launch one rank per GPU")
    if args.impl != "reference":
        import torch
        if torch.cuda.device_count() < world and not args.allow_shared_gpu:
            sys.exit(f"bench.py: {world} ranks need {world} GPUs, this node has {torch.cuda.device_count()}")
        if args.allow_shared_gpu:
            local_rank = local_rank % max(1, torch.cuda.device_count())
    if args.config in ("A", "B", "D"):
        if args.impl == "reference":
            print(json.dumps({"impl": "reference", "unavailable": "configs A/B/D: the oracle runs beside the GPU "
                              "in the same line (cpu_baseline)"}))
            return
        run_config_line(args)
        return
    if args.impl == "reference":
        res = run_reference(args, rank, world)
        if res is not None:
            print(json.dumps(res), flush=True)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if args.allow_shared_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    res = run_cgcm(args, rank, world, local_rank)
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
