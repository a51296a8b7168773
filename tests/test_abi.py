"""CPU-side checks of the boundary: the C-ABI library builds for sm_100a, loads, and exports every
symbol include/cgcm.h declares; the oracle and the product share no code; the product never
imports the oracle; errors without a GPU are loud (no CPU fallback)."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_pldi_jablinpjjba11_b200")


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "cgcm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cgcm_\w+)\s*\(", src)))


@pytest.fixture(scope="module")
def built():
    import __graft_entry__
    __graft_entry__.build()
    return os.path.join(PKG, "libcgcm.so")


def test_library_exports_every_declared_symbol(built):
    out = subprocess.run(["nm", "-D", "--defined-only", built], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (cgcm_\w+)", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    assert len(declared_symbols()) >= 30


def test_library_loads_and_binds_every_symbol(built):
    import ctypes
    L = ctypes.CDLL(built)
    for s in declared_symbols():
        assert hasattr(L, s), s
    L.cgcm_strerror.restype = ctypes.c_char_p
    assert L.cgcm_strerror(-2) == b"pointer not inside a declared allocation unit"


def test_calls_without_context_fail_loudly(built):
    import ctypes
    L = ctypes.CDLL(built)
    out = ctypes.c_uint64(0)
    assert L.cgcm_map(ctypes.c_void_p(0x1000), ctypes.byref(out)) == -10   # CGCM_E_NOCTX
    assert L.cgcm_advanceEpoch() == -10


def test_sm100a_cubin(built):
    out = subprocess.run(["cuobjdump", "--list-elf", built], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_codes_match_oracle_contract():
    import oracle
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    for name in ["OK", "E_INVALID", "E_UNREGISTERED", "E_OVERLAP", "E_NOT_MAPPED", "E_BUSY", "E_DUPLICATE",
                 "E_NOMEM"]:
        assert getattr(cg, name) == getattr(oracle, name), name
    hdr = open(os.path.join(ROOT, "include", "cgcm.h")).read()
    for name, val in [("CGCM_E_UNREGISTERED", -2), ("CGCM_E_NOT_MAPPED", -4), ("CGCM_E_BUSY", -5)]:
        assert re.search(rf"{name} = {val}\b", hdr)


def test_oracle_and_product_are_independent():
    """No shared code: the product sources never mention the oracle and vice versa."""
    prod = []
    for d, _, fs in os.walk(PKG):
        for f in fs:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                prod.append(os.path.join(d, f))
    for f in prod:
        txt = open(f).read()
        for bad in ("import oracle", "from oracle", "liboracle", "cgcm_oracle", "ref_create"):
            assert bad not in txt, (f, bad)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".cpp", ".h")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "cgcm_dev.h" not in txt and "include/cgcm.h" not in txt.replace("include/cgcm.h)", "")
            assert "import paper_conf" not in txt


def test_python_binding_requires_cuda():
    import torch
    import paper_conf_pldi_jablinpjjba11_b200 as cg
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(cg.CgcmError):
        cg.Context(0, arena_bytes=1 << 20)


def test_sass_has_no_odd_uniform_descriptor_pairs(built):
    """ptxas 12.9 once encoded a cp.async cache-policy descriptor as desc[UR1] (an odd uniform-register
    pair), an illegal instruction at run time (k_map_pd3's prologue).  Guard the build against it."""
    import shutil
    so = os.path.join(PKG, "libcgcm.so")
    if not shutil.which("cuobjdump") or not os.path.exists(so):
        pytest.skip("cuobjdump or libcgcm.so missing")
    sass = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
    bad = [ln.strip() for ln in sass.splitlines() if re.search(r"desc\[UR([0-9]+)\]", ln)
           and int(re.search(r"desc\[UR([0-9]+)\]", ln).group(1)) % 2]
    assert not bad, bad[:4]
