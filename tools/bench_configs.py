#!/usr/bin/env python
"""Secondary measurements for the configs that are not the bench line: config A (jagged
256x256, naive-cyclic vs map-promoted, 100 iterations: us per iteration and per call), config B (jagged gemm
4096^2, 64 row-blocks, naive vs promoted: seconds, host-link GB/s of the copies), config D (2^24-node tree:
map+unmap GB/s over the host link, translations/s).  Prints one JSON line per measurement."""
import json
import math
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_pldi_jablinpjjba11_b200 as cg  # noqa: E402
import workloads as W  # noqa: E402


def timed(fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    return time.perf_counter() - t0


def config_A(mode, iters=100):
    """mode: naive | promoted (hand-hoisted, Listing 4) | region (cgcm_regionBegin/End, NEXT-2) |
    region_check (+ the mprotect modOrRef checker)"""
    promoted = mode != "naive"
    ctx = cg.Context(0, arena_bytes=1 << 30)
    nrows = ncols = 256
    vals = W.config_A_values(nrows, ncols, 1)
    rows = []
    for r in range(nrows):
        a = ctx.malloc(8 * ncols)
        np.ctypeslib.as_array((np.ctypeslib.ctypes.c_double * ncols).from_address(a))[:] = vals[r]
        rows.append(a)
    pp = ctx.malloc(8 * nrows)
    np.ctypeslib.as_array((np.ctypeslib.ctypes.c_uint64 * nrows).from_address(pp))[:] = rows
    calls = {"mapArray": 0.0, "kernel": 0.0, "unmapArray": 0.0, "releaseArray": 0.0}

    def tcall(name, fn):
        t0 = time.perf_counter()
        r = fn()
        calls[name] += time.perf_counter() - t0
        return r

    viol = [None]

    def run():
        if mode == "promoted":
            st, d0 = ctx.mapArray(pp)
        elif mode.startswith("region"):
            assert ctx.regionBegin([pp], [ctx.REGION_MAPARRAY], check=mode == "region_check") == 0
        for _ in range(iters):
            st, d = tcall("mapArray", lambda: ctx.mapArray(pp))
            tcall("kernel", lambda: (ctx.sample_scale(d, nrows, ncols, 0.999), ctx.synchronize()))
            ctx.advanceEpoch()
            if not promoted:
                tcall("unmapArray", lambda: ctx.unmapArray(pp))
            tcall("releaseArray", lambda: ctx.releaseArray(pp))
        if mode == "promoted":
            ctx.unmapArray(pp)
            ctx.releaseArray(pp)
        elif mode.startswith("region"):
            s_, viol[0] = ctx.regionEnd()
            assert s_ == 0, s_

    t = timed(run)
    s = ctx.stats()
    ctx.close()
    return {"config": "A", "mode": mode, "iterations": iters, "region_violations": viol[0],
            "us_per_iteration": round(1e6 * t / iters, 1),
            "us_per_call": {k: round(1e6 * v / iters, 1) for k, v in calls.items()},
            "h2d_units": s["h2d_units"], "h2d_bytes": s["h2d_bytes"], "d2h_units": s["d2h_units"],
            "d2h_bytes": s["d2h_bytes"], "h2d_memcpy_calls": s["h2d_memcpy_calls"],
            "d2h_memcpy_calls": s["d2h_memcpy_calls"], "kernel_launches": s["kernel_launches"]}


def config_B(promoted, n=4096, blk=64):
    ctx = cg.Context(0, arena_bytes=2 << 30)
    mats = []
    for m in range(3):
        v = W.config_B_values(n, 2, m)
        rows = []
        for r in range(n):
            a = ctx.malloc(8 * n)
            np.ctypeslib.as_array((np.ctypeslib.ctypes.c_double * n).from_address(a))[:] = v[r]
            rows.append(a)
        pp = ctx.malloc(8 * n)
        np.ctypeslib.as_array((np.ctypeslib.ctypes.c_uint64 * n).from_address(pp))[:] = rows
        mats.append(pp)
    A, B, C = mats

    def run():
        if promoted:
            for pp in mats:
                ctx.mapArray(pp)
        for b0 in range(0, n, blk):
            d = [ctx.mapArray(pp)[1] for pp in mats]
            ctx.sample_gemm_rows(d[0], d[1], d[2], n, b0, blk, 1.5, 1.2)
            ctx.synchronize()
            ctx.advanceEpoch()
            if not promoted:
                ctx.unmapArray(C)
            for pp in mats:
                ctx.releaseArray(pp)
        if promoted:
            ctx.unmapArray(C)
            for pp in mats:
                ctx.releaseArray(pp)

    t = timed(run)
    s = ctx.stats()
    ctx.close()
    moved = s["h2d_bytes"] + s["d2h_bytes"]
    return {"config": "B", "mode": "promoted" if promoted else "naive", "seconds": round(t, 3),
            "h2d_units": s["h2d_units"], "h2d_bytes": s["h2d_bytes"], "d2h_units": s["d2h_units"],
            "d2h_bytes": s["d2h_bytes"], "copy_GBs_over_wall": round(moved / t / 1e9, 2),
            "h2d_memcpy_calls": s["h2d_memcpy_calls"], "d2h_memcpy_calls": s["d2h_memcpy_calls"],
            "gemm_flops": 2 * n ** 3, "kernel_launches": s["kernel_launches"]}


def config_D(N=1 << 24):
    vals = W.tree_values(N)
    order = W.tree_alloc_order(N)
    pos = np.empty(N, dtype=np.int64)
    pos[order] = np.arange(N)
    nodes_t = torch.zeros(N * 32, dtype=torch.uint8, pin_memory=True)
    arena = nodes_t.numpy().view(np.float64).reshape(N, 4)
    arena[:, 1] = vals[order]
    addr = np.uint64(nodes_t.data_ptr()) + np.uint64(32) * pos.astype(np.uint64)
    child = W.tree_children(N)
    table_t = torch.zeros(2 * N, dtype=torch.int64, pin_memory=True)
    table_t.numpy().view(np.uint64)[:] = np.where(child >= 0, addr[np.maximum(child, 0)], 0)
    ctx = cg.Context(0, arena_bytes=4 << 30)
    bases = np.uint64(nodes_t.data_ptr()) + np.uint64(32) * np.arange(N, dtype=np.uint64)
    td = timed(lambda: (ctx.declareBatch(bases, np.full(N, 32, dtype=np.uint64)),
                        ctx.declareAlloc(table_t.data_ptr(), 16 * N)))
    CB, root = table_t.data_ptr(), int(addr[0])
    tb = timed(lambda: (ctx.map(root), ctx.release(root)))  # first call: device table + index build
    tm = timed(lambda: (ctx.mapArray(CB), ctx.map(root)))
    cdev = ctx.mapArray(CB)[1]
    ctx.releaseArray(CB)
    rdev = ctx.map(root)[1]
    ctx.release(root)
    for dlev in range(int(math.log2(N)), -1, -1):
        lo, hi = (1 << dlev) - 1, min((1 << (dlev + 1)) - 1, N)
        ctx.sample_treesum_level(cdev, rdev, N, lo, hi)
        ctx.synchronize()
        ctx.advanceEpoch()
    tu = timed(lambda: (ctx.unmapArray(CB), ctx.unmap(root)))
    ctx.releaseArray(CB)
    ctx.release(root)
    s = ctx.stats()
    ctx.close()
    b = 48 * N
    return {"config": "D", "nodes": N, "declare_seconds": round(td, 4), "table_build_seconds": round(tb, 4),
            "map_seconds": round(tm, 4), "unmap_seconds": round(tu, 4),
            "map_GBs": round(b / tm / 1e9, 2), "unmap_GBs": round(b / tu / 1e9, 2),
            "map_translations_per_s": round(N / tm, 1), "unmap_translations_per_s": round((N - 1) / tu, 1),
            "h2d_bytes": s["h2d_bytes"], "d2h_bytes": s["d2h_bytes"], "kernel_launches": s["kernel_launches"],
            "h2d_memcpy_calls": s["h2d_memcpy_calls"], "d2h_memcpy_calls": s["d2h_memcpy_calls"]}


# ---------------------------------------------------------------------------------------------
# The CPU oracle on the same configs (bench.py --config A|B|D cpu_baseline: "the oracle as it stands",
# one core).  Host and device memory are the oracle's simulated memories; the addresses are synthetic.
# ---------------------------------------------------------------------------------------------
def _oracle():
    sys.path.insert(0, ROOT)
    from oracle import Oracle
    return Oracle()


def _oracle_jagged(o, nrows, ncols, vals, base):
    """nrows row AUs of 8*ncols bytes, host-adjacent (as cgcm_malloc lays them out), + the row-pointer AU."""
    rows = [base + 8 * ncols * r for r in range(nrows)]
    for r, a in enumerate(rows):
        assert o.declareAlloc(a, 8 * ncols) == 0
        o.host_write(a, np.ascontiguousarray(vals[r], dtype=np.float64))
    pp = base + 8 * ncols * nrows
    assert o.declareAlloc(pp, 8 * nrows) == 0
    o.host_write(pp, np.asarray(rows, dtype=np.uint64))
    return rows, pp


def oracle_A(mode, iters=100):
    o = _oracle()
    nrows = ncols = 256
    _rows, pp = _oracle_jagged(o, nrows, ncols, W.config_A_values(nrows, ncols, 1), 0x10000000)
    t0 = time.perf_counter()
    if mode == "promoted":
        assert o.mapArray(pp)[0] == 0
    for _ in range(iters):
        st, d = o.mapArray(pp)
        assert st == 0
        o.kernel_scale(d, nrows, ncols, 0.999)
        o.advanceEpoch()
        if mode == "naive":
            assert o.unmapArray(pp) == 0
        assert o.releaseArray(pp) == 0
    if mode == "promoted":
        assert o.unmapArray(pp) == 0 and o.releaseArray(pp) == 0
    t = time.perf_counter() - t0
    s = o.stats()
    o.close()
    return {"mode": mode, "us_per_iteration": round(1e6 * t / iters, 1), "iterations": iters,
            "h2d_units": s["h2d_units"], "d2h_units": s["d2h_units"]}


def oracle_B(promoted, n=4096, blk=64, gemm_rows=1):
    """One row-block of the loop (the maps / unmaps / releases of a block, the gemm of `gemm_rows` of its
    rows) timed on the oracle and scaled to the whole loop: blocks x (calls + blk/gemm_rows x gemm)."""
    o = _oracle()
    mats = []
    for m in range(3):
        _r, pp = _oracle_jagged(o, n, n, W.config_B_values(n, 2, m), 0x100000000 * (m + 1))
        mats.append(pp)
    C = mats[2]
    t_pro = 0.0
    if promoted:
        t0 = time.perf_counter()
        for pp in mats:
            assert o.mapArray(pp)[0] == 0
        t_pro = time.perf_counter() - t0
    t0 = time.perf_counter()
    d = [o.mapArray(pp)[1] for pp in mats]
    t_map = time.perf_counter() - t0
    t0 = time.perf_counter()
    o.kernel_gemm_rows(d[0], d[1], d[2], n, 0, gemm_rows, 1.5, 1.2)
    t_gemm = time.perf_counter() - t0
    o.advanceEpoch()
    t0 = time.perf_counter()
    if not promoted:
        assert o.unmapArray(C) == 0
    for pp in mats:
        assert o.releaseArray(pp) == 0
    t_unmap = time.perf_counter() - t0
    t_epi = 0.0
    if promoted:
        t0 = time.perf_counter()
        assert o.unmapArray(C) == 0
        for pp in mats:
            assert o.releaseArray(pp) == 0
        t_epi = time.perf_counter() - t0
    o.close()
    blocks = n // blk
    total = t_pro + t_epi + blocks * (t_map + t_unmap + t_gemm * blk / gemm_rows)
    return {"mode": "promoted" if promoted else "naive", "seconds": round(total, 1),
            "sample": f"block 0 timed (its maps/unmaps/releases + the gemm of {gemm_rows} of its {blk} rows), "
                      f"scaled x{blocks} blocks x{blk // gemm_rows} rows",
            "per_block_calls_s": round(t_map + t_unmap, 3), "gemm_row_s": round(t_gemm / gemm_rows, 3)}


def oracle_D(N=1 << 20):
    """Config D's map + levels + unmap on the oracle at N nodes (a 1/16 subset of 2^24 when N = 2^20)."""
    o = _oracle()
    vals = W.tree_values(N)
    order = W.tree_alloc_order(N)
    pos = np.empty(N, dtype=np.int64)
    pos[order] = np.arange(N)
    nodes = 0x10000000
    addr = np.uint64(nodes) + np.uint64(32) * pos.astype(np.uint64)
    for k in range(N):
        assert o.declareAlloc(nodes + 32 * k, 32) == 0
    img = np.zeros((N, 4))
    img[:, 1] = vals[order]
    img.view(np.int64)[:, 0] = order
    o.host_write(nodes, img)
    child = W.tree_children(N)
    CB = 0x800000000
    assert o.declareAlloc(CB, 16 * N) == 0
    o.host_write(CB, np.where(child >= 0, addr[np.maximum(child, 0)], 0).astype(np.uint64))
    t0 = time.perf_counter()
    st, cdev = o.mapArray(CB)
    st2, rdev = o.map(int(addr[0]))
    tm = time.perf_counter() - t0
    assert st == 0 and st2 == 0
    t0 = time.perf_counter()
    for dlev in range(int(math.log2(N)), -1, -1):
        lo, hi = (1 << dlev) - 1, min((1 << (dlev + 1)) - 1, N)
        o.kernel_treesum_level(cdev, rdev, N, lo, hi)
        o.advanceEpoch()
    tk = time.perf_counter() - t0
    t0 = time.perf_counter()
    assert o.unmapArray(CB) == 0 and o.unmap(int(addr[0])) == 0
    tu = time.perf_counter() - t0
    o.close()
    b = 48 * N
    return {"nodes": N, "map_seconds": round(tm, 3), "levels_seconds": round(tk, 3), "unmap_seconds": round(tu, 3),
            "map_GBs": round(b / tm / 1e9, 4), "unmap_GBs": round(b / tu / 1e9, 4)}


if __name__ == "__main__":
    which = sys.argv[1:] or ["A", "B", "D"]
    for w in which:
        if w == "A":
            config_A("promoted", iters=3)  # warm-up: lazy module loading, clocks (not reported)
            for m in ("naive", "promoted", "region", "region_check"):
                print(json.dumps(config_A(m)), flush=True)
        elif w == "B":
            config_B(True, n=256)  # warm-up: lazy module loading of the sample gemm, clocks (not reported)
            for p in (True, False):
                print(json.dumps(config_B(p)), flush=True)
        elif w == "D":
            print(json.dumps(config_D()), flush=True)
