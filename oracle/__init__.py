"""ctypes wrapper of the CPU ORACLE (oracle/cgcm_oracle.cpp).  TEST INFRASTRUCTURE ONLY.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` / ``--impl reference``
legs may import this module.  The product package never imports it
(tests/test_abi.py::test_oracle_and_product_are_independent checks that), and this module imports nothing from the product.

Paper: Jablin et al., "Automatic CPU-GPU Communication Management and Optimization", PLDI 2011.
The oracle follows Algorithms 1-3, Table 2 and P:L203-207.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")

OK = 0
E_INVALID, E_UNREGISTERED, E_OVERLAP, E_NOT_MAPPED, E_BUSY, E_DUPLICATE, E_NOMEM = (
    -1, -2, -3, -4, -5, -6, -7)
LITERAL_EPOCH, LENIENT = 1, 2
UNIT_GLOBAL, UNIT_READONLY, UNIT_ARRAYMAPPED, UNIT_ACTIVE = 1, 2, 4, 8


class RefUnit(C.Structure):
    _fields_ = [("base", C.c_uint64), ("size", C.c_uint64), ("devptr", C.c_uint64),
                ("refCount", C.c_int64), ("epoch", C.c_uint64), ("flags", C.c_uint32),
                ("pad", C.c_uint32)]


STAT_FIELDS = ["h2d_units", "h2d_bytes", "d2h_units", "d2h_bytes", "activations", "frees",
               "fwd_translations", "rev_translations", "null_slots", "passthrough", "peer_units", "peer_bytes"]


class RefStats(C.Structure):
    _fields_ = [(f, C.c_uint64) for f in STAT_FIELDS]


def build(force: bool = False) -> str:
    """Compile liboracle.so with plain g++ (no CUDA)."""
    src = os.path.join(HERE, "cgcm_oracle.cpp")
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(HERE, "cgcm_oracle.h"))):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-shared", "-fPIC", "-Wall", "-o", LIB, src])
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        u64, vp, st, pu64 = C.c_uint64, C.c_void_p, C.c_size_t, C.POINTER(C.c_uint64)
        sig = {
            "ref_create": (vp, [C.c_uint]), "ref_destroy": (None, [vp]), "ref_groupJoin": (C.c_int, [vp, vp]),
            "ref_declareAlloc": (C.c_int, [vp, u64, u64]),
            "ref_declareAllocFlags": (C.c_int, [vp, u64, u64, C.c_uint]),
            "ref_declareGlobal": (C.c_int, [vp, C.c_char_p, u64, u64, C.c_int]),
            "ref_undeclare": (C.c_int, [vp, u64]),
            "ref_hostWrite": (C.c_int, [vp, u64, vp, u64]), "ref_hostRead": (C.c_int, [vp, u64, vp, u64]),
            "ref_devWrite": (C.c_int, [vp, u64, vp, u64]), "ref_devRead": (C.c_int, [vp, u64, vp, u64]),
            "ref_map": (C.c_int, [vp, u64, pu64]), "ref_unmap": (C.c_int, [vp, u64]),
            "ref_release": (C.c_int, [vp, u64]),
            "ref_mapArray": (C.c_int, [vp, u64, pu64]), "ref_unmapArray": (C.c_int, [vp, u64]),
            "ref_releaseArray": (C.c_int, [vp, u64]),
            "ref_advanceEpoch": (C.c_int, [vp]), "ref_advanceEpochs": (C.c_int, [vp, u64]), "ref_epoch": (u64, [vp]),
            "ref_mapBatch": (C.c_int, [vp, vp, st, vp]), "ref_unmapBatch": (C.c_int, [vp, vp, st]),
            "ref_releaseBatch": (C.c_int, [vp, vp, st]),
            "ref_mapArrays": (C.c_int, [vp, vp, st, vp]), "ref_unmapArrays": (C.c_int, [vp, vp, st]),
            "ref_releaseArrays": (C.c_int, [vp, vp, st]),
            "ref_mapSlots": (C.c_int, [vp, vp, st]), "ref_unmapSlots": (C.c_int, [vp, vp, st, C.c_int]),
            "ref_stats": (C.c_int, [vp, C.POINTER(RefStats)]),
            "ref_dumpTable": (C.c_int, [vp, vp, st, C.POINTER(C.c_size_t)]),
            "ref_replayDevptr": (C.c_int, [vp, u64, u64]),
            "ref_lookup": (C.c_int, [vp, u64, pu64, pu64]),
            "ref_devLookup": (C.c_int, [vp, u64, pu64, pu64]),
            "ref_runGlue": (C.c_int, [vp, vp, st, vp, st, u64, vp]),
            "ref_kernel_scale": (C.c_int, [vp, u64, u64, u64, C.c_double]),
            "ref_kernel_treesum_level": (C.c_int, [vp, u64, u64, u64, u64, u64]),
            "ref_kernel_gemm_rows": (C.c_int, [vp, u64, u64, u64, u64, u64, u64, C.c_double, C.c_double]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype, f.argtypes = res, args
        _lib = L
    return _lib


def _u64arr(xs) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(xs, dtype=np.uint64))


GLUE_OP = np.dtype([("op", "<u4"), ("dst", "<u4"), ("a", "<u4"), ("b", "<u4"), ("imm", "<i8")])


def glue_program(rows) -> np.ndarray:
    return np.array([tuple(int(v) for v in r) for r in rows], dtype=GLUE_OP)


class Oracle:
    """One oracle context (allocInfoMap + globalEpoch + simulated host/device memory)."""

    def __init__(self, flags: int = 0):
        self.L = lib()
        self.h = self.L.ref_create(flags)

    def close(self):
        if self.h:
            self.L.ref_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # registration
    def groupJoin(self, leader):
        """NEXT-3: join the coherence group of `leader` (shared host memory, own device/table/epochs)."""
        return self.L.ref_groupJoin(self.h, leader.h)

    def declareAlloc(self, base, size, readonly=False):
        if readonly:
            return self.L.ref_declareAllocFlags(self.h, base, size, UNIT_READONLY)
        return self.L.ref_declareAlloc(self.h, base, size)

    def declareGlobal(self, name, base, size, ro=False):
        return self.L.ref_declareGlobal(self.h, name.encode() if name is not None else None, base, size, int(ro))

    def undeclare(self, base):
        return self.L.ref_undeclare(self.h, base)

    # simulated memories
    def host_write(self, addr, data):
        b = np.ascontiguousarray(np.frombuffer(bytes(data), dtype=np.uint8)) if not isinstance(data, np.ndarray) \
            else np.ascontiguousarray(data).view(np.uint8).reshape(-1)
        return self.L.ref_hostWrite(self.h, addr, b.ctypes.data, b.nbytes)

    def host_read(self, addr, n) -> np.ndarray:
        out = np.zeros(n, dtype=np.uint8)
        self.L.ref_hostRead(self.h, addr, out.ctypes.data, n)
        return out

    def dev_write(self, addr, data):
        b = np.ascontiguousarray(data).view(np.uint8).reshape(-1)
        return self.L.ref_devWrite(self.h, addr, b.ctypes.data, b.nbytes)

    def dev_read(self, addr, n) -> np.ndarray:
        out = np.zeros(n, dtype=np.uint8)
        self.L.ref_devRead(self.h, addr, out.ctypes.data, n)
        return out

    # Table 2 operations
    def map(self, p):
        out = C.c_uint64(0)
        s = self.L.ref_map(self.h, p, C.byref(out))
        return s, out.value

    def unmap(self, p):
        return self.L.ref_unmap(self.h, p)

    def release(self, p):
        return self.L.ref_release(self.h, p)

    def mapArray(self, pp):
        out = C.c_uint64(0)
        s = self.L.ref_mapArray(self.h, pp, C.byref(out))
        return s, out.value

    def unmapArray(self, pp):
        return self.L.ref_unmapArray(self.h, pp)

    def releaseArray(self, pp):
        return self.L.ref_releaseArray(self.h, pp)

    def advanceEpoch(self):
        return self.L.ref_advanceEpoch(self.h)

    def advanceEpochs(self, n):
        return self.L.ref_advanceEpochs(self.h, n)

    @property
    def epoch(self):
        return self.L.ref_epoch(self.h)

    def mapBatch(self, ps):
        a = _u64arr(ps)
        out = np.zeros(len(a), dtype=np.uint64)
        s = self.L.ref_mapBatch(self.h, a.ctypes.data, len(a), out.ctypes.data)
        return s, out

    def unmapBatch(self, ps):
        a = _u64arr(ps)
        return self.L.ref_unmapBatch(self.h, a.ctypes.data, len(a))

    def releaseBatch(self, ps):
        a = _u64arr(ps)
        return self.L.ref_releaseBatch(self.h, a.ctypes.data, len(a))

    def mapArrays(self, pps):
        a = _u64arr(pps)
        out = np.zeros(len(a), dtype=np.uint64)
        s = self.L.ref_mapArrays(self.h, a.ctypes.data, len(a), out.ctypes.data)
        return s, out

    def unmapArrays(self, pps):
        a = _u64arr(pps)
        return self.L.ref_unmapArrays(self.h, a.ctypes.data, len(a))

    def releaseArrays(self, pps):
        a = _u64arr(pps)
        return self.L.ref_releaseArrays(self.h, a.ctypes.data, len(a))

    def mapSlots(self, slots: np.ndarray):
        assert slots.dtype == np.uint64 and slots.flags.c_contiguous
        return self.L.ref_mapSlots(self.h, slots.ctypes.data, len(slots))

    def unmapSlots(self, slots: np.ndarray, release=False):
        assert slots.dtype == np.uint64 and slots.flags.c_contiguous
        return self.L.ref_unmapSlots(self.h, slots.ctypes.data, len(slots), int(release))

    # introspection
    def stats(self) -> dict:
        s = RefStats()
        self.L.ref_stats(self.h, C.byref(s))
        return {f: getattr(s, f) for f in STAT_FIELDS}

    def dump(self) -> list:
        n = C.c_size_t(0)
        self.L.ref_dumpTable(self.h, None, 0, C.byref(n))
        arr = (RefUnit * max(1, n.value))()
        self.L.ref_dumpTable(self.h, C.cast(arr, C.c_void_p), n.value, C.byref(n))
        return [dict(base=u.base, size=u.size, devptr=u.devptr, refCount=u.refCount, epoch=u.epoch,
                     flags=u.flags) for u in arr[:n.value]]

    def replay(self, base, devptr):
        return self.L.ref_replayDevptr(self.h, base, devptr)

    def lookup(self, p):
        b, s = C.c_uint64(0), C.c_uint64(0)
        r = self.L.ref_lookup(self.h, p, C.byref(b), C.byref(s))
        return (b.value, s.value) if r == 0 else None

    def devLookup(self, g):
        b, d = C.c_uint64(0), C.c_uint64(0)
        r = self.L.ref_devLookup(self.h, g, C.byref(b), C.byref(d))
        return (b.value, d.value) if r == 0 else None

    # sample GPU functions on the simulated device
    def kernel_scale(self, rows_dev, nrows, ncols, alpha):
        return self.L.ref_kernel_scale(self.h, rows_dev, nrows, ncols, alpha)

    def kernel_treesum_level(self, child_dev, root_dev, nnodes, lo, hi):
        return self.L.ref_kernel_treesum_level(self.h, child_dev, root_dev, nnodes, lo, hi)

    def runGlue(self, prog, ptrs, max_steps=1 << 20):
        """The glue-kernel program (rows of (op, dst, a, b, imm)) on the simulated device; (status, regs)."""
        arr = glue_program(prog)
        p = _u64arr(ptrs)
        regs = np.zeros(32, dtype=np.uint64)
        s = self.L.ref_runGlue(self.h, arr.ctypes.data, len(arr), p.ctypes.data, len(p), max_steps,
                               regs.ctypes.data)
        return s, regs

    def kernel_gemm_rows(self, A, B, Cm, n, row0, nrows, alpha, beta):
        return self.L.ref_kernel_gemm_rows(self.h, A, B, Cm, n, row0, nrows, alpha, beta)
