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
                  "fwd_translations", "rev_translations", "null_slots", "passthrough", "peer_units", "peer_bytes"]


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


class _Current:
    """A context proxy that makes the context current before every use (several contexts driven from
    one thread: coherence groups, NEXT-3)."""

    def __init__(self, ctx):
        object.__setattr__(self, "_ctx", ctx)

    def __getattr__(self, name):
        ctx = self._ctx
        ctx.make_current()
        v = getattr(ctx, name)
        if callable(v):
            def call(*a, **k):
                ctx.make_current()
                return v(*a, **k)
            return call
        return v


class Pair:
    def __init__(self, ctx, oracle, switch=False):
        self.g = _Current(ctx) if switch else ctx
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
        self.check_structure(what)

    # ---- structural checks of the GPU's device addresses (implementation-defined values, A22) ----
    def check_structure(self, what=""):
        """The device addresses the GPU chose (and replays into the oracle) must satisfy what the
        paper and reading A7 require of ANY valid choice (SURVEY §8(c) "Exact device addresses"):
          * devptr == base (mod 256)                                   (A7, alignment of the copy)
          * copies of distinct units are disjoint, and touch (d1 + s1 == d2) only if their host AUs
            touch in the same order (b1 + s1 == b2): a one-past-the-end GPU pointer must reverse to the
            unit it came from (A7)
          * every copy lies in exactly one live device extent, each extent's `live` count equals the
            number of copies inside it (no extent outlives its units: no device-memory leak), and
            arena extents lie inside the arena (Alg. 1 cuMemAlloc / Alg. 3 cuMemFree)."""
        gd = self.g.dump()
        copies = sorted((u["devptr"], u["size"], u["base"]) for u in gd if u["devptr"])
        for d, n, b in copies:
            assert d % 256 == b % 256, f"{what}: devptr {hex(d)} of {hex(b)} not congruent mod 256"
        for (d1, s1, b1), (d2, s2, b2) in zip(copies, copies[1:]):
            assert d1 + s1 <= d2, f"{what}: device copies of {hex(b1)} and {hex(b2)} overlap"
            if d1 + s1 == d2:
                assert b1 + s1 == b2, f"{what}: copies of {hex(b1)}, {hex(b2)} adjacent but host AUs are not"
        ex = sorted(self.g.extents(), key=lambda e: e["addr"])
        for e1, e2 in zip(ex, ex[1:]):
            assert e1["addr"] + e1["bytes"] <= e2["addr"], f"{what}: device extents overlap"
        lo = self.g.arena.data_ptr()
        hi = lo + self.g.arena.numel()
        starts = [e["addr"] for e in ex]
        import bisect
        held = [0] * len(ex)
        for d, n, b in copies:
            k = bisect.bisect_right(starts, d) - 1
            assert k >= 0 and d + n <= ex[k]["addr"] + ex[k]["bytes"], f"{what}: copy of {hex(b)} in no extent"
            held[k] += 1
        for e, h in zip(ex, held):
            assert e["live"] == h and h > 0, f"{what}: extent {hex(e['addr'])} live={e['live']} holds {h} copies"
            if not e["external"]:
                assert lo <= e["addr"] and e["addr"] + e["bytes"] <= hi, f"{what}: extent outside the arena"

    def drain(self, shadows=True):
        """Release every outstanding reference with scalar cgcm_release calls (each one compared with
        the oracle), then check the balance: all refcounts 0 and no storage held (check_balance)."""
        for _ in range(64):
            live = [(u["base"], u["refCount"]) for u in self.g.dump() if u["refCount"] > 0]
            if not live:
                break
            for b, rc in live:
                for _k in range(rc):
                    assert self.run("release", b) == 0
            self.check("drain")
        assert self.check_balance("drained", shadows)

    def check_balance(self, what="end", shadows=True):
        """After every reference is released, the runtime holds no device storage for AUs beyond the
        globals' persistent copies (A14) and no live forward-map shadow (SURVEY §8(c) "Refcounts":
        arena usage returns to baseline).  Scratch buffers the runtime keeps for reuse are excluded."""
        gd = self.g.dump()
        if any(u["refCount"] > 0 for u in gd):
            return False
        self.check_structure(what)
        si = self.g.storage()
        glob = [u for u in gd if u["devptr"]]
        assert all(u["flags"] & 1 for u in glob), f"{what}: a released non-global unit keeps a copy"
        assert not shadows or si["shadows_live"] == 0, f"{what}: {si['shadows_live']} live shadows after all releases"
        if not glob:
            assert si["extents"] == 0 and si["extent_bytes"] == 0, f"{what}: leaked extents {si}"
        return True

    def check_device_units(self):
        """Device copies of active units equal the oracle's simulated device bytes."""
        for u in self.g.dump():
            if u["devptr"] and u["refCount"] > 0:
                gb = self.g.dev_read(u["devptr"], u["size"]).tobytes()
                ob = self.o.dev_read(u["devptr"], u["size"]).tobytes()
                assert gb == ob, f"device bytes of unit {hex(u['base'])} differ"
