"""Differential harness: run the same operation on the CUDA path (through the C ABI) and on the
CPU oracle, with the oracle fed the GPU's device addresses (replay mode, SURVEY §8(c) "Parity
definition"), and compare the full observable state after every step.

Compared exactly: every translated pointer (raw 64-bit), per-AU refcount / epoch / active /
arrayMapped / devptr, unit-level copy counters, and the host bytes of every AU.
"""
from __future__ import annotations

import ctypes

import numpy as np

COMPARED_STATS = ["h2d_units", "h2d_bytes", "d2h_units", "d2h_bytes", "activations", "frees",
                  "fwd_translations", "rev_translations", "null_slots", "passthrough"]


def host_read(addr: int, n: int) -> bytes:
    return ctypes.string_at(addr, n)


def host_write(addr: int, data) -> None:
    b = bytes(data) if not isinstance(data, np.ndarray) else np.ascontiguousarray(data).tobytes()
    ctypes.memmove(addr, b, len(b))


class HostBuf:
    """Plain (pageable) host memory with a stable address."""

    def __init__(self, nbytes: int, align: int = 256):
        self.raw = np.zeros(nbytes + align, dtype=np.uint8)
        off = (-self.raw.ctypes.data) % align
        self.arr = self.raw[off:off + nbytes]
        self.addr = self.arr.ctypes.data


class Pair:
    def __init__(self, ctx, oracle):
        self.g = ctx
        self.o = oracle
        self.units = {}   # base -> size

    # ---- registration ----
    def declare(self, base, size, data=None, readonly=False):
        if data is not None:
            host_write(base, data)
        s1 = self.g.declareAlloc(base, size, readonly)
        s2 = self.o.declareAlloc(base, size, readonly)
        assert s1 == s2, (s1, s2)
        if s1 == 0:
            self.units[base] = size
            self.o.host_write(base, np.frombuffer(host_read(base, size), dtype=np.uint8))
        return s1

    def malloc(self, n, data=None):
        """cgcm_malloc on the GPU side (pinned, auto-declared), mirrored into the oracle."""
        a = self.g.malloc(n)
        assert a, "cgcm_malloc failed"
        if data is not None:
            host_write(a, data)
        assert self.o.declareAlloc(a, n) == 0
        self.units[a] = n
        self.o.host_write(a, np.frombuffer(host_read(a, n), dtype=np.uint8))
        return a

    def declare_global(self, name, base, size, ro=False):
        s1 = self.g.declareGlobal(name, base, size, ro)
        s2 = self.o.declareGlobal(name, base, size, ro)
        assert s1 == s2, (s1, s2)
        if s1 == 0:
            self.units[base] = size
            self.o.host_write(base, np.frombuffer(host_read(base, size), dtype=np.uint8))
        return s1

    def undeclare(self, base):
        s1 = self.g.undeclare(base)
        s2 = self.o.undeclare(base)
        assert s1 == s2, (s1, s2)
        if s1 == 0:
            self.units.pop(base, None)
        return s1

    def sync_host_to_oracle(self, base, n):
        """After the test itself writes host memory (legal only for unmapped AUs)."""
        self.o.host_write(base, np.frombuffer(host_read(base, n), dtype=np.uint8))

    # ---- replay: feed the GPU's devbase of units the GPU activated ----
    def feed_replay(self):
        gd = {u["base"]: u for u in self.g.dump()}
        od = {u["base"]: u for u in self.o.dump()}
        for b, u in gd.items():
            if u["devptr"] and od.get(b, {}).get("devptr", 0) == 0:
                self.o.replay(b, u["devptr"])

    # ---- operations ----
    def run(self, name, *args):
        """Run op `name` on both sides; returns (status, gpu_result)."""
        g = getattr(self.g, name)(*args)
        self.feed_replay()
        o = getattr(self.o, name)(*args)
        gs = g[0] if isinstance(g, tuple) else g
        os_ = o[0] if isinstance(o, tuple) else o
        assert gs == os_, f"{name}{args}: gpu status {gs} != oracle {os_}"
        if isinstance(g, tuple):
            gv, ov = g[1], o[1]
            if isinstance(gv, np.ndarray):
                assert (gv == ov).all(), f"{name}: translated pointers differ"
            else:
                assert gv == ov, f"{name}: {hex(gv)} != {hex(ov)}"
        return g

    def advance(self):
        self.g.advanceEpoch()
        self.o.advanceEpoch()

    # ---- full-state comparison ----
    def check(self, what=""):
        gd, od = self.g.dump(), self.o.dump()
        assert len(gd) == len(od), what
        for a, b in zip(gd, od):
            assert a == b, f"{what}: unit mismatch gpu={a} oracle={b}"
        gs, os_ = self.g.stats(), self.o.stats()
        for f in COMPARED_STATS:
            assert gs[f] == os_[f], f"{what}: stat {f} gpu={gs[f]} oracle={os_[f]}"
        for b, n in self.units.items():
            hb = host_read(b, n)
            ob = self.o.host_read(b, n).tobytes()
            assert hb == ob, f"{what}: host bytes of unit {hex(b)} differ"
        assert self.g.epoch == self.o.epoch

    def check_device_units(self):
        """Device copies of active units equal the oracle's simulated device bytes."""
        for u in self.g.dump():
            if u["devptr"] and u["refCount"] > 0:
                gb = self.g.dev_read(u["devptr"], u["size"]).tobytes()
                ob = self.o.dev_read(u["devptr"], u["size"]).tobytes()
                assert gb == ob, f"device bytes of unit {hex(u['base'])} differ"
