"""Seeded synthetic inputs shared by the oracle-side tests and the CUDA-side tests/bench.

This module holds NONE of the method's arithmetic (no lookup, translation, refcount or epoch
logic): only a stateless counter-based generator, splitmix64(seed, i), and the recipes that turn
its output into the shapes of SURVEY.md §8(d) configs A-E (DESIGN.md §5 states each recipe).
Both sides evaluate the same generator, so they see identical inputs without shipping arrays.
"""
from __future__ import annotations

import ctypes

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_G = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, idx) -> np.ndarray:
    """Stateless splitmix64: z = seed + (i+1)*golden; two xor-shift-multiply rounds."""
    i = np.asarray(idx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + (i + np.uint64(1)) * _G
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def key(seed: int, stream: int) -> int:
    """Derive an independent stream key from (seed, stream id)."""
    return int(splitmix64(seed, np.uint64(stream)))


def u01(seed: int, stream: int, idx) -> np.ndarray:
    """Uniform doubles in [0, 1) from the top 53 bits."""
    r = splitmix64(key(seed, stream), idx)
    return (r >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def randint(seed: int, stream: int, idx, n) -> np.ndarray:
    """Uniform integers in [0, n) (n may be an array), via floor(u01 * n)."""
    return np.minimum(np.floor(u01(seed, stream, idx) * np.asarray(n, dtype=np.float64)).astype(np.uint64),
                      np.asarray(n, dtype=np.uint64) - np.uint64(1))


def permutation(seed: int, stream: int, n: int) -> np.ndarray:
    """A seeded permutation of range(n): argsort of splitmix64 keys."""
    return np.argsort(splitmix64(key(seed, stream), np.arange(n, dtype=np.uint64)), kind="stable")


# ---------------------------------------------------------------------------------------------
# Config C / E: allocation table of U units, sizes log-uniform in [16, 65536) rounded down to 16 B,
# gaps uniform in {0, 16, ..., 4080} B (gap 0 = adjacency, p = 1/256); interior-pointer queries
# with the unit uniform by index and the offset uniform in [0, size).
# ---------------------------------------------------------------------------------------------
def table_layout(U: int, seed: int):
    """Return (offsets, sizes, span): unit k occupies [offsets[k], offsets[k]+sizes[k]) of a region."""
    idx = np.arange(U, dtype=np.uint64)
    sizes = (16.0 * np.power(4096.0, u01(seed, 1, idx))).astype(np.uint64) // np.uint64(16) * np.uint64(16)
    sizes = np.maximum(sizes, np.uint64(16))
    gaps = (splitmix64(key(seed, 2), idx) % np.uint64(256)) * np.uint64(16)
    gaps[0] = 0
    ends = np.cumsum(sizes + gaps, dtype=np.uint64)
    offsets = ends - sizes
    span = int(ends[-1]) + 4096
    return offsets, sizes, span


def queries(offsets: np.ndarray, sizes: np.ndarray, n: int, seed: int, stream: int = 3, start: int = 0):
    """n interior-pointer offsets (relative to the region start) for query indices [start, start+n)."""
    idx = np.arange(start, start + n, dtype=np.uint64)
    u = randint(seed, stream, idx, len(offsets))
    off = randint(seed, stream + 1000, idx, sizes[u])
    return offsets[u] + off, u


_libc = None


def _c():
    global _libc
    if _libc is None:
        _libc = ctypes.CDLL(None, use_errno=True)
        _libc.mmap.restype = ctypes.c_void_p
        _libc.mmap.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                               ctypes.c_long]
        _libc.munmap.restype = ctypes.c_int
        _libc.munmap.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
    return _libc


def reserve_readonly(span: int) -> int:
    """Reserve `span` bytes of PROT_READ anonymous memory (reads as zero pages, uses no RAM)."""
    PROT_READ, MAP_PRIVATE, MAP_ANONYMOUS, MAP_NORESERVE = 1, 0x02, 0x20, 0x4000
    a = _c().mmap(None, span, PROT_READ, MAP_PRIVATE | MAP_ANONYMOUS | MAP_NORESERVE, -1, 0)
    if a is None or a == ctypes.c_void_p(-1).value:
        raise OSError(ctypes.get_errno(), "mmap failed")
    return a


def release_reservation(addr: int, span: int) -> None:
    _c().munmap(addr, span)


# ---------------------------------------------------------------------------------------------
# Config A: double **rows, 256 x 256 fp64, values 1 + u01 in [1, 2)
# Config B: three jagged n x n fp64 matrices, values u01 in [0, 1)
# Config D: 2^k node tree, nodes {i64 key; f64 val; f64 sum; i64 pad}, allocation order permuted
# ---------------------------------------------------------------------------------------------
def config_A_values(nrows: int = 256, ncols: int = 256, seed: int = 1) -> np.ndarray:
    idx = np.arange(nrows * ncols, dtype=np.uint64)
    return (1.0 + u01(seed, 10, idx)).reshape(nrows, ncols)


def config_B_values(n: int, seed: int = 2, which: int = 0) -> np.ndarray:
    idx = np.arange(n * n, dtype=np.uint64)
    return u01(seed, 20 + which, idx).reshape(n, n)


def tree_children(N: int) -> np.ndarray:
    """child[2i] = 2i+1, child[2i+1] = 2i+2 (node indices), -1 when >= N.  Shape (2N,)."""
    c = np.arange(1, 2 * N + 1, dtype=np.int64)
    c[c >= N] = -1
    return c


def tree_values(N: int, seed: int = 4) -> np.ndarray:
    return u01(seed, 40, np.arange(N, dtype=np.uint64))


def tree_alloc_order(N: int, seed: int = 4) -> np.ndarray:
    """Seeded permutation: position k of the node arena holds node tree_alloc_order[k]."""
    return permutation(seed, 41, N)


# ---------------------------------------------------------------------------------------------
# The same generator on torch tensors (any device), for inputs too large to build in numpy
# (config E's 2^28 pointers).  int64 arithmetic wraps like u64; shifts are made logical.
# tests/test_workloads.py checks it equals the numpy version bit for bit.
# ---------------------------------------------------------------------------------------------
def _s64(x: int) -> int:
    x &= 0xFFFFFFFFFFFFFFFF
    return x - (1 << 64) if x >= (1 << 63) else x


def _srl(t, k: int):
    return (t >> k) & ((1 << (64 - k)) - 1)


def splitmix64_t(seed: int, idx):
    """splitmix64 over an int64 tensor of indices (bit-identical to splitmix64)."""
    z = (idx + 1) * _s64(0x9E3779B97F4A7C15) + _s64(seed)
    z = (z ^ _srl(z, 30)) * _s64(0xBF58476D1CE4E5B9)
    z = (z ^ _srl(z, 27)) * _s64(0x94D049BB133111EB)
    return z ^ _srl(z, 31)


def u01_t(seed: int, stream: int, idx):
    r = splitmix64_t(key(seed, stream), idx)
    return _srl(r, 11).double() * (1.0 / 9007199254740992.0)


def randint_t(seed: int, stream: int, idx, n):
    import torch
    u = u01_t(seed, stream, idx)
    nn = n.double() if torch.is_tensor(n) else float(n)
    v = torch.floor(u * nn).long()
    return torch.minimum(v, (n - 1) if torch.is_tensor(n) else torch.full_like(v, n - 1))


def queries_t(offsets_t, sizes_t, n: int, seed: int, stream: int = 3, start: int = 0, chunk: int = 1 << 24):
    """Torch version of queries(): returns (offsets int64 tensor, unit int64 tensor) on offsets_t.device."""
    import torch
    dev = offsets_t.device
    outq = torch.empty(n, dtype=torch.int64, device=dev)
    outu = torch.empty(n, dtype=torch.int64, device=dev)
    U = offsets_t.numel()
    for c0 in range(0, n, chunk):
        c1 = min(n, c0 + chunk)
        idx = torch.arange(start + c0, start + c1, dtype=torch.int64, device=dev)
        u = randint_t(seed, stream, idx, U)
        off = randint_t(seed, stream + 1000, idx, sizes_t[u])
        outq[c0:c1] = offsets_t[u] + off
        outu[c0:c1] = u
    return outq, outu
