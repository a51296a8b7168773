"""Python binding of the B200-native CGCM run-time library (libcgcm.so, include/cgcm.h).

Argument marshalling only: every lookup, translation, refcount and epoch decision runs in the CUDA
kernels behind the C ABI.  PyTorch provides the device arena and the streams (plumbing).  There is
no CPU fallback: importing works anywhere, but every call needs the in-tree libcgcm.so and a CUDA
device, and raises if either is missing.

Functions mirror the C names (``cgcm_map`` -> ``map``) and return the C status codes so that they
can be compared one to one with the oracle's.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# CGCM_LIBDIR: load a variant build of the same library (kernel A/B experiments, build.py --variant)
LIB_PATH = os.path.join(os.environ.get("CGCM_LIBDIR") or HERE, "libcgcm.so")
SAMPLES_PATH = os.path.join(HERE, "libcgcm_samples.so")

OK = 0
E_INVALID, E_UNREGISTERED, E_OVERLAP, E_NOT_MAPPED, E_BUSY, E_DUPLICATE, E_NOMEM, E_CUDA, E_MIXED, E_NOCTX, E_MODREF = (
    -1, -2, -3, -4, -5, -6, -7, -8, -9, -10, -11)
LITERAL_EPOCH, LENIENT, PROFILE, FORCE_SHADOW, NO_PAGEDIR, PD_V2 = 1, 2, 4, 8, 16, 32
UNIT_GLOBAL, UNIT_READONLY, UNIT_ARRAYMAPPED, UNIT_ACTIVE = 1, 2, 4, 8
RELEASE = 1


class Unit(C.Structure):
    _fields_ = [("base", C.c_uint64), ("size", C.c_uint64), ("devptr", C.c_uint64), ("refCount", C.c_int64),
                ("epoch", C.c_uint64), ("flags", C.c_uint32), ("pad", C.c_uint32)]


STAT_FIELDS = ["h2d_units", "h2d_bytes", "d2h_units", "d2h_bytes", "activations", "frees", "fwd_translations",
               "rev_translations", "null_slots", "passthrough", "h2d_memcpy_calls", "d2h_memcpy_calls",
               "kernel_launches", "table_rebuilds", "rev_rebuilds"]


class Stats(C.Structure):
    _fields_ = [(f, C.c_uint64) for f in STAT_FIELDS] + [
        ("fwd_kernel_ms", C.c_double), ("rev_kernel_ms", C.c_double), ("fwd_kernel_calls", C.c_uint64),
        ("rev_kernel_calls", C.c_uint64), ("fwd_kernel_slots", C.c_uint64), ("rev_kernel_slots", C.c_uint64),
        ("peer_units", C.c_uint64), ("peer_bytes", C.c_uint64), ("peer_memcpy_calls", C.c_uint64),
        ("table_merges", C.c_uint64)]


class IndexInfo(C.Structure):
    _fields_ = [("units", C.c_uint64), ("levels", C.c_uint32), ("pd_segments", C.c_uint32),
                ("pd_pages", C.c_uint64), ("pd_overflow_pages", C.c_uint64), ("pd_bytes", C.c_uint64),
                ("pd_min_shift", C.c_uint32), ("pd_max_shift", C.c_uint32), ("pd_format", C.c_uint32),
                ("pad", C.c_uint32)]


class Extent(C.Structure):
    _fields_ = [("addr", C.c_uint64), ("bytes", C.c_uint64), ("live", C.c_int64), ("external", C.c_uint32),
                ("pad", C.c_uint32)]


class StorageInfo(C.Structure):
    _fields_ = [(f, C.c_uint64) for f in (
        "extents", "extent_bytes", "external_extents", "shadows_live", "shadow_live_bytes", "shadows_cached",
        "shadow_cached_bytes", "arena_used", "arena_capacity")]


class CgcmError(RuntimeError):
    pass


_lib = None
_samples = None


def lib():
    """Load libcgcm.so (fails loudly if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise CgcmError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        u64, vp, sz, i = C.c_uint64, C.c_void_p, C.c_size_t, C.c_int
        sig = {
            "cgcm_init": (i, [i, vp, sz, vp, vp, C.c_uint]), "cgcm_finalize": (i, []),
            "cgcm_getContext": (vp, []), "cgcm_setContext": (i, [vp]),
            "cgcm_strerror": (C.c_char_p, [i]), "cgcm_lastCudaError": (C.c_char_p, []),
            "cgcm_declareAlloc": (i, [vp, sz]), "cgcm_declareAllocFlags": (i, [vp, sz, C.c_uint]),
            "cgcm_declareBatch": (i, [vp, vp, sz, C.c_uint]), "cgcm_undeclare": (i, [vp]),
            "cgcm_declareGlobal": (i, [C.c_char_p, vp, sz, i]),
            "cgcm_declareGlobalSymbol": (i, [C.c_char_p, vp, sz, i, vp]),
            "cgcm_regionBegin": (i, [vp, vp, sz, C.c_uint]),
            "cgcm_regionEnd": (i, [C.POINTER(C.c_size_t)]),
            "cgcm_malloc": (vp, [sz]), "cgcm_free": (i, [vp]),
            "cgcm_calloc": (vp, [sz, sz]), "cgcm_realloc": (vp, [vp, sz]),
            "cgcm_declareAlloca": (vp, [sz]), "cgcm_scopeEnter": (i, []), "cgcm_scopeExit": (i, []),
            "cgcm_map": (i, [vp, vp]), "cgcm_unmap": (i, [vp]), "cgcm_release": (i, [vp]),
            "cgcm_mapArray": (i, [vp, vp]), "cgcm_unmapArray": (i, [vp]), "cgcm_releaseArray": (i, [vp]),
            "cgcm_advanceEpoch": (i, []), "cgcm_advanceEpochs": (i, [u64]), "cgcm_epoch": (u64, []),
            "cgcm_mapBatch": (i, [vp, sz, vp]), "cgcm_unmapBatch": (i, [vp, sz]),
            "cgcm_releaseBatch": (i, [vp, sz]),
            "cgcm_mapArrays": (i, [vp, sz, vp]), "cgcm_unmapArrays": (i, [vp, sz]),
            "cgcm_releaseArrays": (i, [vp, sz]),
            "cgcm_mapArrayDevice": (i, [vp, sz]), "cgcm_unmapArrayDevice": (i, [vp, sz, C.c_uint]),
            "cgcm_stats": (i, [C.POINTER(Stats)]), "cgcm_resetStats": (i, []),
            "cgcm_dumpTable": (i, [vp, sz, C.POINTER(C.c_size_t)]),
            "cgcm_arenaUsage": (i, [C.POINTER(C.c_size_t), C.POINTER(C.c_size_t)]),
            "cgcm_indexInfo": (i, [C.POINTER(IndexInfo)]),
            "cgcm_dumpExtents": (i, [C.c_void_p, C.c_size_t, C.POINTER(C.c_size_t)]),
            "cgcm_storageInfo": (i, [C.POINTER(StorageInfo)]),
            "cgcm_launchGlue": (i, [C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t, C.c_uint64, C.c_void_p]),
            "cgcm_groupCreate": (i, [C.POINTER(C.c_void_p)]), "cgcm_groupJoin": (i, [C.c_void_p]),
            "cgcm_groupLeave": (i, []), "cgcm_groupDestroy": (i, [C.c_void_p]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype, f.argtypes = res, args
        _lib = L
    return _lib


def samples():
    """Test-only sample GPU functions (S1/S2/S3)."""
    global _samples
    if _samples is None:
        if not os.path.exists(SAMPLES_PATH):
            raise CgcmError(f"{SAMPLES_PATH} is missing: run __graft_entry__.build()")
        S = C.CDLL(SAMPLES_PATH)
        u64, vp = C.c_uint64, C.c_void_p
        S.cgcm_sample_scale.restype = C.c_int
        S.cgcm_sample_scale.argtypes = [u64, u64, u64, C.c_double, vp]
        S.cgcm_sample_treesum_level.restype = C.c_int
        S.cgcm_sample_treesum_level.argtypes = [u64, u64, u64, u64, u64, vp]
        S.cgcm_sample_global_addr.restype = C.c_int
        S.cgcm_sample_global_addr.argtypes = [C.POINTER(C.c_void_p), C.POINTER(C.c_size_t)]
        S.cgcm_sample_scale_global.restype = C.c_int
        S.cgcm_sample_scale_global.argtypes = [C.c_double, vp]
        S.cgcm_sample_gemm_rows.restype = C.c_int
        S.cgcm_sample_gemm_rows.argtypes = [u64, u64, u64, C.c_int, C.c_int, C.c_int, C.c_double, C.c_double, vp]
        S.cgcm_test_d2h.restype = C.c_int
        S.cgcm_test_d2h.argtypes = [vp, u64, u64]
        S.cgcm_test_h2d.restype = C.c_int
        S.cgcm_test_h2d.argtypes = [u64, vp, u64]
        _samples = S
    return _samples


def _u64(xs) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(xs, dtype=np.uint64))


def group_create():
    """A new coherence group (NEXT-3); contexts join it with Context.groupJoin."""
    g = C.c_void_p()
    s = lib().cgcm_groupCreate(C.byref(g))
    if s != OK:
        raise CgcmError(f"groupCreate: {strerror(s)}")
    return g.value


def group_destroy(g) -> int:
    return lib().cgcm_groupDestroy(g)


class Context:
    """One CGCM context on one CUDA device.  PyTorch allocates the device arena and the streams."""

    def __init__(self, device: int = 0, arena_bytes: int | None = None, flags: int = 0):
        import torch  # plumbing only: device memory + streams
        if not torch.cuda.is_available():
            raise CgcmError("CUDA device required: libcgcm has no CPU fallback")
        self.L = lib()
        self.device = device
        dev = torch.device("cuda", device)
        if arena_bytes is None:
            free, _total = torch.cuda.mem_get_info(dev)
            arena_bytes = int(min(free * 0.5, 16 << 30))
        self.arena = torch.empty(arena_bytes, dtype=torch.uint8, device=dev)
        self.main = torch.cuda.Stream(device=dev)
        self.copy = torch.cuda.Stream(device=dev)
        s = self.L.cgcm_init(device, self.arena.data_ptr(), arena_bytes, self.main.cuda_stream,
                             self.copy.cuda_stream, flags)
        if s != OK:
            raise CgcmError(f"cgcm_init failed: {strerror(s)} {self.L.cgcm_lastCudaError().decode()}")
        self.handle = self.L.cgcm_getContext()

    # context switching (one context per device / thread)
    def make_current(self):
        return self.L.cgcm_setContext(self.handle)

    def close(self):
        if self.handle:
            self.make_current()
            self.L.cgcm_finalize()
            self.handle = None
            self.arena = None

    @property
    def stream_handle(self) -> int:
        return self.main.cuda_stream

    # ---- registration ----
    def declareAlloc(self, base: int, size: int, readonly: bool = False) -> int:
        if readonly:
            return self.L.cgcm_declareAllocFlags(base, size, UNIT_READONLY)
        return self.L.cgcm_declareAlloc(base, size)

    def declareBatch(self, bases, sizes, readonly: bool = False) -> int:
        b, s = _u64(bases), _u64(sizes)
        return self.L.cgcm_declareBatch(b.ctypes.data, s.ctypes.data, len(b), UNIT_READONLY if readonly else 0)

    def declareGlobal(self, name, base, size, ro=False) -> int:
        return self.L.cgcm_declareGlobal(name.encode() if name is not None else None, base, size, int(ro))

    def declareGlobalSymbol(self, name, base, size, ro, dev_symbol) -> int:
        return self.L.cgcm_declareGlobalSymbol(name.encode() if name is not None else None, base, size, int(ro),
                                               dev_symbol)

    # ---- map-promotion regions (NEXT-2) ----
    REGION_MAP, REGION_MAPARRAY, REGION_CHECK = 0, 1, 1

    def regionBegin(self, ptrs, kinds, check=False) -> int:
        n = len(ptrs)
        pa = (C.c_uint64 * max(n, 1))(*ptrs)
        ka = (C.c_uint * max(n, 1))(*kinds)
        return self.L.cgcm_regionBegin(C.addressof(pa), C.addressof(ka), n, 1 if check else 0)

    def regionEnd(self):
        v = C.c_size_t()
        s = self.L.cgcm_regionEnd(C.byref(v))
        return s, v.value

    def undeclare(self, base: int) -> int:
        return self.L.cgcm_undeclare(base)

    def malloc(self, n: int) -> int:
        return self.L.cgcm_malloc(n) or 0

    def free(self, p: int) -> int:
        return self.L.cgcm_free(p)

    def calloc(self, nmemb: int, size: int) -> int:
        return self.L.cgcm_calloc(nmemb, size) or 0

    def realloc(self, p: int, n: int) -> int:
        return self.L.cgcm_realloc(p, n) or 0

    def declareAlloca(self, n: int) -> int:
        return self.L.cgcm_declareAlloca(n) or 0

    def scopeEnter(self) -> int:
        return self.L.cgcm_scopeEnter()

    def scopeExit(self) -> int:
        return self.L.cgcm_scopeExit()

    # ---- Table 2 ----
    def map(self, p: int):
        out = C.c_uint64(0)
        s = self.L.cgcm_map(p, C.byref(out))
        return s, out.value

    def unmap(self, p: int) -> int:
        return self.L.cgcm_unmap(p)

    def release(self, p: int) -> int:
        return self.L.cgcm_release(p)

    def mapArray(self, pp: int):
        out = C.c_uint64(0)
        s = self.L.cgcm_mapArray(pp, C.byref(out))
        return s, out.value

    def unmapArray(self, pp: int) -> int:
        return self.L.cgcm_unmapArray(pp)

    def releaseArray(self, pp: int) -> int:
        return self.L.cgcm_releaseArray(pp)

    def advanceEpoch(self) -> int:
        return self.L.cgcm_advanceEpoch()

    def advanceEpochs(self, n: int) -> int:
        return self.L.cgcm_advanceEpochs(n)

    @property
    def epoch(self) -> int:
        return self.L.cgcm_epoch()

    # ---- batch forms ----
    def mapBatch(self, ps):
        a = _u64(ps)
        out = np.zeros(len(a), dtype=np.uint64)
        s = self.L.cgcm_mapBatch(a.ctypes.data, len(a), out.ctypes.data)
        return s, out

    def unmapBatch(self, ps) -> int:
        a = _u64(ps)
        return self.L.cgcm_unmapBatch(a.ctypes.data, len(a))

    def releaseBatch(self, ps) -> int:
        a = _u64(ps)
        return self.L.cgcm_releaseBatch(a.ctypes.data, len(a))

    def mapArrays(self, pps):
        a = _u64(pps)
        out = np.zeros(len(a), dtype=np.uint64)
        s = self.L.cgcm_mapArrays(a.ctypes.data, len(a), out.ctypes.data)
        return s, out

    def unmapArrays(self, pps) -> int:
        a = _u64(pps)
        return self.L.cgcm_unmapArrays(a.ctypes.data, len(a))

    def releaseArrays(self, pps) -> int:
        a = _u64(pps)
        return self.L.cgcm_releaseArrays(a.ctypes.data, len(a))

    def mapArrayDevice(self, dptr: int, n: int) -> int:
        return self.L.cgcm_mapArrayDevice(dptr, n)

    def unmapArrayDevice(self, dptr: int, n: int, release: bool = False) -> int:
        return self.L.cgcm_unmapArrayDevice(dptr, n, RELEASE if release else 0)

    # ---- introspection ----
    def stats(self) -> dict:
        st = Stats()
        self.L.cgcm_stats(C.byref(st))
        d = {f: getattr(st, f) for f in STAT_FIELDS}
        for f in ("fwd_kernel_ms", "rev_kernel_ms", "fwd_kernel_calls", "rev_kernel_calls", "fwd_kernel_slots",
                  "rev_kernel_slots", "peer_units", "peer_bytes", "peer_memcpy_calls", "table_merges"):
            d[f] = getattr(st, f)
        return d

    def resetStats(self) -> int:
        return self.L.cgcm_resetStats()

    def dump(self) -> list:
        n = C.c_size_t(0)
        self.L.cgcm_dumpTable(None, 0, C.byref(n))
        arr = (Unit * max(1, n.value))()
        s = self.L.cgcm_dumpTable(C.cast(arr, C.c_void_p), n.value, C.byref(n))
        if s != OK:
            raise CgcmError(f"dumpTable: {strerror(s)}")
        return [dict(base=u.base, size=u.size, devptr=u.devptr, refCount=u.refCount, epoch=u.epoch, flags=u.flags)
                for u in arr[:n.value]]

    def arenaUsage(self):
        u, c = C.c_size_t(0), C.c_size_t(0)
        self.L.cgcm_arenaUsage(C.byref(u), C.byref(c))
        return u.value, c.value

    def indexInfo(self) -> dict:
        ii = IndexInfo()
        s = self.L.cgcm_indexInfo(C.byref(ii))
        if s != OK:
            raise CgcmError(f"indexInfo: {strerror(s)}")
        return {f: getattr(ii, f) for f, _ in IndexInfo._fields_}

    # ---- coherence groups (NEXT-3) ----
    def groupJoin(self, group) -> int:
        self.make_current()
        return self.L.cgcm_groupJoin(group)

    def groupLeave(self) -> int:
        self.make_current()
        return self.L.cgcm_groupLeave()

    # ---- glue kernels (NEXT-4) ----
    GLUE = dict(MOVI=1, ADD=2, ADDI=3, SUB=4, MUL=5, FADD=6, FSUB=7, FMUL=8, FDIV=9, LD=10, ST=11, BNZ=12, HALT=13)

    def launchGlue(self, prog, ptrs, max_steps=1 << 20):
        """Run a glue program (rows of (op, dst, a, b, imm), ops by number or name) as one GPU thread over
        the mapped AUs of ptrs (registers 0..len(ptrs)-1).  Returns (status, final registers)."""
        import numpy as np
        dt = np.dtype([("op", "<u4"), ("dst", "<u4"), ("a", "<u4"), ("b", "<u4"), ("imm", "<i8")])
        rows = [((self.GLUE[r[0]] if isinstance(r[0], str) else int(r[0])),) + tuple(int(v) for v in r[1:]) for r in prog]
        arr = np.array(rows, dtype=dt)
        p = np.asarray([int(x) for x in ptrs], dtype=np.uint64)
        regs = np.zeros(32, dtype=np.uint64)
        s = self.L.cgcm_launchGlue(arr.ctypes.data if len(arr) else None, len(arr),
                                   p.ctypes.data if len(p) else None, len(p), max_steps, regs.ctypes.data)
        return s, regs

    def dump_np(self):
        """The unit table as a numpy structured array (fields of cgcm_unit_t) -- for large tables."""
        import numpy as np
        n = C.c_size_t(0)
        self.L.cgcm_dumpTable(None, 0, C.byref(n))
        arr = (Unit * max(1, n.value))()
        s = self.L.cgcm_dumpTable(C.cast(arr, C.c_void_p), n.value, C.byref(n))
        if s != OK:
            raise CgcmError(f"dumpTable: {strerror(s)}")
        dt = np.dtype([("base", "<u8"), ("size", "<u8"), ("devptr", "<u8"), ("refCount", "<i8"),
                       ("epoch", "<u8"), ("flags", "<u4"), ("pad", "<u4")])
        return np.frombuffer(arr, dtype=dt, count=n.value).copy()

    def extents(self) -> list:
        n = C.c_size_t(0)
        self.L.cgcm_dumpExtents(None, 0, C.byref(n))
        arr = (Extent * max(1, n.value))()
        s = self.L.cgcm_dumpExtents(C.cast(arr, C.c_void_p), n.value, C.byref(n))
        if s != OK:
            raise CgcmError(f"dumpExtents: {strerror(s)}")
        return [{f: getattr(arr[k], f) for f, _ in Extent._fields_ if f != "pad"} for k in range(n.value)]

    def storage(self) -> dict:
        si = StorageInfo()
        s = self.L.cgcm_storageInfo(C.byref(si))
        if s != OK:
            raise CgcmError(f"storageInfo: {strerror(s)}")
        return {f: getattr(si, f) for f, _ in StorageInfo._fields_}

    # ---- test-only sample GPU functions on the main stream ----
    def sample_scale(self, rows_dev, nrows, ncols, alpha):
        return samples().cgcm_sample_scale(rows_dev, nrows, ncols, alpha, self.main.cuda_stream)

    def sample_global(self):
        """(device address, bytes) of the test-only __device__ array of libcgcm_samples.so"""
        a, n = C.c_void_p(), C.c_size_t()
        if samples().cgcm_sample_global_addr(C.byref(a), C.byref(n)) != 0:
            raise CgcmError("cudaGetSymbolAddress failed")
        return a.value, n.value

    def sample_scale_global(self, alpha):
        return samples().cgcm_sample_scale_global(alpha, self.main.cuda_stream)

    def sample_treesum_level(self, child_dev, root_dev, nnodes, lo, hi):
        return samples().cgcm_sample_treesum_level(child_dev, root_dev, nnodes, lo, hi, self.main.cuda_stream)

    def sample_gemm_rows(self, A, B, Cm, n, row0, nrows, alpha, beta):
        return samples().cgcm_sample_gemm_rows(A, B, Cm, n, row0, nrows, alpha, beta, self.main.cuda_stream)

    def dev_read(self, addr: int, n: int) -> np.ndarray:
        self.main.synchronize()
        out = np.zeros(n, dtype=np.uint8)
        if n and samples().cgcm_test_d2h(out.ctypes.data, addr, n) != 0:
            raise CgcmError("device read failed")
        return out

    def dev_write(self, addr: int, data: np.ndarray):
        self.main.synchronize()
        b = np.ascontiguousarray(data).view(np.uint8).reshape(-1)
        if b.nbytes and samples().cgcm_test_h2d(addr, b.ctypes.data, b.nbytes) != 0:
            raise CgcmError("device write failed")

    def synchronize(self):
        self.main.synchronize()


def strerror(s: int) -> str:
    return lib().cgcm_strerror(s).decode()
