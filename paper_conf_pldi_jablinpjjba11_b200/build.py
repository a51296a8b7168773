"""Build the in-tree CUDA shared libraries for sm_100a (nvcc cross-compiles; no GPU needed).

  libcgcm.so          the product: kernels.cu + runtime.cpp behind include/cgcm.h
  libcgcm_samples.so  test-only sample GPU functions (S1 scale, S2 jagged gemm, S3 tree sums)

Rebuilds only when a source is newer than the library.
"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INC = os.path.join(ROOT, "include")
NVCC = os.environ.get("NVCC", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", INC, "-I", CSRC]

LIB = os.path.join(PKG, "libcgcm.so")
SAMPLES = os.path.join(PKG, "libcgcm_samples.so")


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        raise RuntimeError(f"build failed: {cmd[-1]}")
    return r.stdout + r.stderr


def build_variant(out_dir: str, defines: list[str]) -> str:
    """Build libcgcm.so with extra -D defines into out_dir (kernel A/B experiments; the binding loads
    it when CGCM_LIBDIR=out_dir).  Returns the library path."""
    os.makedirs(out_dir, exist_ok=True)
    objs = []
    jobs = []
    for name, src in (("kernels", os.path.join(CSRC, "kernels.cu")), ("runtime", os.path.join(CSRC, "runtime.cpp"))):
        obj = os.path.join(out_dir, name + ".o")
        lang = ["-x", "cu"] if src.endswith(".cu") else ["-x", "c++"]
        jobs.append([NVCC] + ARCH + COMMON + [f"-D{d}" for d in defines] + lang + ["-c", src, "-o", obj])
        objs.append(obj)
    with ThreadPoolExecutor(max_workers=2) as ex:
        list(ex.map(_run, jobs))
    lib = os.path.join(out_dir, "libcgcm.so")
    _run([NVCC] + ARCH + ["-shared", "-o", lib] + objs + ["-lcudart"])
    return lib


def build(verbose: bool = False) -> None:
    hdrs = [os.path.join(INC, "cgcm.h"), os.path.join(CSRC, "cgcm_dev.h")]
    units = {
        "kernels": os.path.join(CSRC, "kernels.cu"),
        "runtime": os.path.join(CSRC, "runtime.cpp"),
    }
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    jobs = []
    for name, src in units.items():
        obj = os.path.join(objdir, name + ".o")
        if _stale(obj, [src] + hdrs):
            lang = ["-x", "cu"] if src.endswith(".cu") else ["-x", "c++"]
            extra = ["-Xptxas", "-v"] if (verbose and src.endswith(".cu")) else []
            jobs.append([NVCC] + ARCH + COMMON + extra + lang + ["-c", src, "-o", obj])
    samples_src = os.path.join(CSRC, "samples.cu")
    samples_obj = os.path.join(objdir, "samples.o")
    if os.path.exists(samples_src) and _stale(samples_obj, [samples_src]):
        jobs.append([NVCC] + ARCH + COMMON + ["-x", "cu", "-c", samples_src, "-o", samples_obj])
    with ThreadPoolExecutor(max_workers=3) as ex:
        outs = list(ex.map(_run, jobs))
    if verbose:
        for o in outs:
            sys.stdout.write(o)
    objs = [os.path.join(objdir, n + ".o") for n in units]
    if _stale(LIB, objs):
        _run([NVCC] + ARCH + ["-shared", "-o", LIB] + objs + ["-lcudart"])
    if os.path.exists(samples_src) and _stale(SAMPLES, [samples_obj]):
        _run([NVCC] + ARCH + ["-shared", "-o", SAMPLES, samples_obj, "-lcudart"])


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "--variant":  # --variant OUT_DIR [DEFINE ...]
        print("built", build_variant(sys.argv[2], sys.argv[3:]))
    else:
        build(verbose="-v" in sys.argv)
        print("built", LIB)
