#!/usr/bin/env python
"""Kernel A/B on the GPU box: run bench.py (no e2e, no CPU baseline) once per variant build and print
the forward / reverse kernel times side by side.

  python -m paper_conf_pldi_jablinpjjba11_b200.build --variant build/ab/NAME -DFOO ...   (here, on CPU)
  python tools/ab.py --configs E,C build/ab/base build/ab/NAME ...                       (via gpurun)

Variants run interleaved (base, v1, ..., base, v1, ...) --rounds times so clock drift hits all alike.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(spec, config, steps):
    # spec = LIBDIR[@VAR=VAL,VAR=VAL]: a variant build plus environment overrides
    libdir, _, extra = spec.partition("@")
    env = dict(os.environ, CGCM_LIBDIR=os.path.abspath(libdir))
    env.update(kv.split("=", 1) for kv in extra.split(",") if kv)
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", config, "--steps", str(steps), "--warmup", "3",
           "--no-e2e", "--no-cpu-baseline"]
    r = subprocess.run(cmd, capture_output=True, text=True, env=env, cwd=ROOT)
    line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    if not line:
        return {"error": (r.stderr or r.stdout)[-400:]}
    d = json.loads(line[-1])
    rf = d["roofline"]
    return {"value_G": round(d["value"] / 1e9, 2), "fwd_ms": rf["fwd_ms_per_launch"], "rev_ms": rf["rev_ms_per_launch"],
            "sm_mhz": d["clocks"]["sm_mhz"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="E", help="comma-separated")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--rounds", type=int, default=2)
    ap.add_argument("libdirs", nargs="+")
    a = ap.parse_args()
    for c in a.configs.split(","):
        for rnd in range(a.rounds):
            for ld in a.libdirs:
                print(json.dumps({"config": c, "round": rnd, "variant": os.path.basename(ld.split("@")[0].rstrip("/")) + ld.partition("@")[1] + ld.partition("@")[2],
                                  **run(ld, c, a.steps)}), flush=True)


if __name__ == "__main__":
    main()
