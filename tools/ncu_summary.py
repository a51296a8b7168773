#!/usr/bin/env python
"""Summarise ncu evidence into profiles/ (committed): per-kernel metrics of a --set full capture and
the kernel-time shares of a launch list (gpu__time_duration.sum, --clock-control none).

usage: tools/ncu_summary.py --round r01 --config E --report gpurun_out/r01/prof_E.ncu-rep \
           --launches gpurun_out/r01/launches_bench_default.csv
Writes profiles/<round>_<config>_summary.md and merges DRAM bytes per launch into profiles/ncu_traffic.json
(bench.py reports them as roofline.traffic).
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput %"),
    ("lts__t_requests_srcunit_tex.sum", "L2 requests from L1"),
    ("lts__t_requests_srcunit_ltcfabric.sum", "L2 requests over the die-to-die fabric"),
    ("lts__t_tag_requests.avg.pct_of_peak_sustained_elapsed", "L2 tag lookups % of peak"),
    ("lts__t_sectors_srcunit_tex.sum", "L2 sectors from L1"),
    ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed", "L1 data-pipe wavefronts % of peak"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("sm__inst_executed.sum.pct_of_peak_sustained_elapsed", "issue % of peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def kind_of(name):
    """'rev' for the reverse passes -- k_rev_* (round 2), k_unmap_sh, k_slots<1, ...> (DIR_REV = 1) -- else 'fwd'."""
    return "rev" if ("k_rev" in name or "k_unmap" in name or
                     ("k_slots" in name and ("<1," in name or "(int)1," in name))) else "fwd"


def raw_rows(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def to_bytes(v, unit):
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)
    return float(v) * mult


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", required=True)
    ap.add_argument("--config", required=True)
    ap.add_argument("--report", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--slots", type=int, required=True, help="slots per hot-kernel launch")
    args = ap.parse_args()
    hdr, units, rows = raw_rows(args.report)
    lines = [f"# ncu summary {args.round} config {args.config}", "",
             f"source: `{os.path.basename(args.report)}` (ncu --set full --clock-control none, cold replays)", ""]
    traffic = {}
    for row in rows:
        name = row[hdr.index("Kernel Name")]
        kind = kind_of(name)
        lines.append(f"## {name}")
        lines.append("")
        lines.append("| metric | value |")
        lines.append("|---|---|")
        vals = {}
        for key, label in METRICS:
            if key in hdr:
                i = hdr.index(key)
                vals[key] = (row[i], units[i])
                lines.append(f"| {label} (`{key}`) | {row[i]} {units[i]} |")
        dr = to_bytes(*vals["dram__bytes_read.sum"]) + to_bytes(*vals["dram__bytes_write.sum"])
        req = float(vals["lts__t_requests_srcunit_tex.sum"][0])
        fab = float(vals.get("lts__t_requests_srcunit_ltcfabric.sum", ("0", ""))[0])
        inst = float(vals["smsp__inst_executed.sum"][0])
        lines.append(f"| DRAM bytes per launch (read+write) | {dr:.4g} B ({dr / args.slots:.2f} B/slot; "
                     f"algorithmic 16 B/slot) |")
        lines.append(f"| L2 requests per slot | {req / args.slots:.2f} (+ {fab / args.slots:.2f} fabric) |")
        lines.append(f"| thread instructions per slot | {inst * 32 / args.slots:.1f} |")
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued"):
                try:
                    stalls.append((float(row[i]), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                except ValueError:
                    pass
        tot = sum(v for v, _ in stalls) or 1
        top = ", ".join(f"{n} {100 * v / tot:.0f}%" for v, n in sorted(stalls, reverse=True)[:6])
        lines.append(f"| warp stall samples | {top} |")
        lines.append("")
        traffic[kind] = dr
    if args.launches:
        times = collections.Counter()
        counts = collections.Counter()
        with open(args.launches) as f:
            txt = [ln for ln in f if not ln.startswith("==")]
        rd = csv.reader(io.StringIO("".join(txt)))
        h = next(rd)
        ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
        ui = h.index("Metric Unit")
        for r in rd:
            if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
                continue
            v = float(r[vi].replace(",", ""))
            v *= {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0,
                  "second": 1e3, "s": 1e3}.get(r[ui], 1.0)
            key = r[ki].split("(")[0]
            times[key] += v
            counts[key] += 1
        total = sum(times.values())
        lines += [f"## launch list `{os.path.basename(args.launches)}` (whole command, serialised)", "",
                  "| kernel | launches | total ms | share |", "|---|---|---|---|"]
        for k, v in times.most_common(15):
            lines.append(f"| `{k[:90]}` | {counts[k]} | {v:.3f} | {100 * v / total:.1f}% |")
        lines.append("")
        # this library's kernels only (the bench's input generation runs torch kernels outside the timed region)
        own = {k: v for k, v in times.items() if "cgcm::" in k}
        tot_own = sum(own.values()) or 1.0
        lines += ["### this library's kernels only (cgcm::*)", "",
                  "| kernel | launches | total ms | share of cgcm time |", "|---|---|---|---|"]
        for k, v in sorted(own.items(), key=lambda x: -x[1]):
            lines.append(f"| `{k[:90]}` | {counts[k]} | {v:.3f} | {100 * v / tot_own:.1f}% |")
        lines.append("")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    out = os.path.join(ROOT, "profiles", f"{args.round}_{args.config}_summary.md")
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    tj = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    data = {}
    if os.path.exists(tj):
        with open(tj) as f:
            data = json.load(f)
    data[args.config] = {k: round(v) for k, v in traffic.items()}
    data[args.config]["source"] = os.path.basename(out)
    with open(tj, "w") as f:
        json.dump(data, f, indent=1)
    print("wrote", out)


if __name__ == "__main__":
    main()
