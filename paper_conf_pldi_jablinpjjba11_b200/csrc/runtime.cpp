// runtime.cpp -- host side of the B200-native CGCM run-time library (C ABI: include/cgcm.h).
//
// What runs here: AU registration (the host half of "allocInfoMap maintenance"),
// device-arena and pinned-host-arena allocation, the transfer scheduler (coalesced
// cudaMemcpyAsync runs on the copy stream), orchestration of the kernels and all-or-nothing
// rollback.  What never runs here: pointer lookup, translation, refcount or epoch decisions --
// those are the kernels of kernels.cu.  Nothing in this file can fall back
// to a CPU computation of a kernel's result.
#include <cuda_runtime.h>
#include <signal.h>
#include <sys/mman.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cerrno>
#include <cstdint>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <thread>
#include <string>
#include <unordered_map>
#include <unordered_set>
#include <vector>

#include "../../include/cgcm.h"
#include "cgcm_dev.h"

namespace cgcm {

thread_local std::string g_last_cuda_error;

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e_ = (x);                                                            \
    if (e_ != cudaSuccess) {                                                         \
      g_last_cuda_error = std::string(#x) + " (runtime.cpp:" + std::to_string(__LINE__) + "): " + \
                          cudaGetErrorString(e_);                                    \
      return CGCM_E_CUDA;                                                            \
    }                                                                                \
  } while (0)
#define CKS(x)                    \
  do {                            \
    int s_ = (x);                 \
    if (s_ != CGCM_OK) return s_; \
  } while (0)

static inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// CGCM_TRACE=1: host-side phase timings on stderr (wall clock of the host thread, for finding where a
// call's time goes; off by default)
struct Trace {
  const char *what;
  std::chrono::steady_clock::time_point t0;
  static bool on() {
    static const bool e = std::getenv("CGCM_TRACE") != nullptr;
    return e;
  }
  explicit Trace(const char *w) : what(w), t0(std::chrono::steady_clock::now()) {}
  ~Trace() {
    if (on())
      std::fprintf(stderr, "[cgcm] %-28s %9.3f ms\n", what,
                   std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count());
  }
};

// ---------------------------------------------------------------------------------------------
// Device arena: best-fit free list over [base, base+cap) with 256-byte granularity.  All device
// memory of a context (AU copies, tables, scratch) comes from here; the arena itself is provided
// by the caller (PyTorch) or cudaMalloc'ed once.
// ---------------------------------------------------------------------------------------------
class Arena {
 public:
  void init(uint64_t base, uint64_t cap) {
    uint64_t b = align_up(base, 256);
    cap_ = (cap - (b - base)) / 256 * 256;
    base_ = b;
    by_off_.clear();
    by_len_.clear();
    if (cap_) insert(base_, cap_);
    used_ = 0;
  }
  uint64_t alloc(uint64_t bytes) {
    bytes = align_up(std::max<uint64_t>(bytes, 1), 256);
    auto it = by_len_.lower_bound(bytes);
    if (it == by_len_.end()) return 0;
    uint64_t off = it->second, len = it->first;
    erase(off, len);
    if (len > bytes) insert(off + bytes, len - bytes);
    used_ += bytes;
    return off;
  }
  void free(uint64_t addr, uint64_t bytes) {
    if (!addr) return;
    bytes = align_up(std::max<uint64_t>(bytes, 1), 256);
    used_ -= bytes;
    uint64_t off = addr, len = bytes;
    auto nx = by_off_.lower_bound(off);
    if (nx != by_off_.end() && nx->first == off + len) {
      len += nx->second;
      erase(nx->first, nx->second);
    }
    auto pv = by_off_.lower_bound(off);
    if (pv != by_off_.begin()) {
      --pv;
      if (pv->first + pv->second == off) {
        off = pv->first;
        len += pv->second;
        erase(pv->first, pv->second);
      }
    }
    insert(off, len);
  }
  uint64_t used() const { return used_; }
  uint64_t capacity() const { return cap_; }

 private:
  void insert(uint64_t off, uint64_t len) {
    by_off_[off] = len;
    by_len_.emplace(len, off);
  }
  void erase(uint64_t off, uint64_t len) {
    by_off_.erase(off);
    auto r = by_len_.equal_range(len);
    for (auto it = r.first; it != r.second; ++it)
      if (it->second == off) {
        by_len_.erase(it);
        break;
      }
  }
  uint64_t base_ = 0, cap_ = 0, used_ = 0;
  std::map<uint64_t, uint64_t> by_off_;
  std::multimap<uint64_t, uint64_t> by_len_;
};

// growable device scratch buffer carved from the arena
struct DevBuf {
  uint64_t addr = 0;
  size_t bytes = 0;
  template <class T>
  T *as() const { return reinterpret_cast<T *>(addr); }
};

// growable pinned host buffer
struct HostBuf {
  void *p = nullptr;
  size_t bytes = 0;
  int ensure(size_t need) {
    if (need <= bytes) return CGCM_OK;
    if (p) cudaFreeHost(p);
    size_t nb = std::max<size_t>(need, std::max<size_t>(bytes * 3 / 2, 1 << 16));
    if (cudaHostAlloc(&p, nb, cudaHostAllocPortable | cudaHostAllocMapped) != cudaSuccess) {
      p = nullptr;
      bytes = 0;
      return CGCM_E_NOMEM;
    }
    bytes = nb;
    return CGCM_OK;
  }
  template <class T>
  T *as() const { return reinterpret_cast<T *>(p); }
};

// host registry entry: one declared AU
struct HostUnit {
  uint64_t size = 0;
  uint32_t flags = 0;       // UF_GLOBAL | UF_READONLY
  uint64_t epoch0 = 0;      // globalEpoch at declaration (A20)
  int32_t idx = -1;         // rank in the device table (valid after a table build)
  std::string name;
  uint64_t sym = 0;         // declareGlobalSymbol: the bound __device__ symbol's address (NEXT-4)
};

// one device extent holding the copies of one or more host-adjacent units (mirrored layout)
struct Run {
  uint64_t addr = 0, bytes = 0;
  uint64_t delta = 0;  // host address - device address of every unit copy in the extent (mirrored)
  int64_t live = 0;
  bool external = false;  // a bound __device__ symbol: not arena memory, never freed by the runtime
};

// Search-index buffers: forward (all units by base) and reverse (live device extents by start)
struct IndexBufs {
  DevBuf top, wide, dir, skmin, smeta, keys, pay, rid;
  DevBuf lvl[MAXL];
  size_t lvl_cap[MAXL] = {0};
  int n = 0, h = 0, ntop = 0, nseg = 0, ndir = 0;
  bool any_wide = false;
  IndexDev view(const uint64_t *keys_dev) const {
    IndexDev ix;
    ix.top = top.as<uint64_t>();
    ix.wide = wide.as<uint32_t>();
    ix.dir = dir.as<uint32_t>();
    ix.seg_kmin = skmin.as<uint64_t>();
    ix.seg_meta = smeta.as<uint32_t>();
    for (int k = 0; k < MAXL; ++k) ix.lvl[k] = lvl[k].as<uint32_t>();
    ix.keys = keys_dev;
    ix.n = n;
    ix.h = h;
    ix.ntop = ntop;
    ix.nseg = nseg;
    ix.ndir = ndir;
    return ix;
  }
};

struct Context;
// NEXT-3 coherence group (include/cgcm.h): the member contexts in join order
struct Group {
  std::mutex mu;
  std::vector<Context *> members;
};

struct Context {
  int device = 0;
  Group *group = nullptr;
  cudaStream_t main = nullptr, copy = nullptr;
  bool own_streams = false;
  void *own_arena = nullptr;
  unsigned flags = 0;
  int nsm = 148;
  Arena arena;
  std::recursive_mutex mu;
  uint64_t epoch = 0;
  uint64_t origin = 0;  // device epochs are u32 relative to this origin (A28)
  // generation of device-storage releases, and per array outer (host base) the generation at which its
  // slots were last translated from host memory: a re-map may reverse-translate its device slots (A9)
  // only if no storage was released since -- otherwise a slot may point at a freed copy whose address
  // a newer unit now occupies (an element released through another path, A25), and the re-map must
  // re-translate from the host slots as the sequential mapArray does
  uint64_t free_gen = 0;
  std::unordered_map<uint64_t, uint64_t> arr_gen;
  uint32_t rel_epoch(uint64_t e) const { return e >= origin ? (uint32_t)(e - origin) : 0u; }

  // registry (host)
  std::map<uint64_t, HostUnit> reg;
  // per-unit host state by table rank (structure of arrays, rebuilt by ensure_table): the
  // activation / copy-back / release loops walk these contiguously instead of the registry's nodes
  std::vector<uint64_t> ubase, usize, udev;  // host base, size, device copy address (0: none)
  std::vector<uint32_t> uflags;              // UF_GLOBAL | UF_READONLY
  std::vector<int64_t> urun;                 // device extent holding the copy (-1: none)
  std::vector<uint64_t> usym;                // bound __device__ symbol of a global (0: none)
  // open map-promotion region (cgcm_regionBegin): the promoted pointers and their kinds
  bool region_open = false, region_checked = false;
  std::vector<std::pair<uint64_t, unsigned>> region;
  std::vector<uint8_t> uarr;                 // mirror of UF_ARRAYMAPPED
  std::unordered_set<std::string> names;
  bool table_dirty = true, rev_dirty = true;
  int U = 0;  // units in the device table (ids [0, U))
  // NEXT-1 batched merge: up to DELTA_MAX declarations between two calls are appended to the device table
  // as "delta" units (ids [Umain, U)) instead of a rebuild; the sorted main table (ids [0, Umain), base
  // order) keeps its index and page directory, and the kernels search the small sorted delta index only
  // where the main table misses or hits exactly one past the end of a unit (A7).  An undeclare of a unit
  // in the device table, or too many delta units, makes the next merge a full rebuild.
  static constexpr int DELTA_MAX = 4096;
  int Umain = 0;
  std::vector<uint64_t> pend;   // bases declared since the last merge, not in the device table yet
  bool pend_over = false;       // more than DELTA_MAX of them
  bool dirty_del = false;       // a unit of the device table was undeclared
  std::vector<uint64_t> dk;     // delta index on the host: bases (sorted) ...
  std::vector<uint32_t> di;     // ... and ids
  DevBuf dkeys, dids;
  size_t col_cap = 0;           // units the device table columns have room for

  // device table
  DevBuf hotb, hotcb, stb, rcb, size64, dbase, extd, extlo, extlen, snap_st, snap_rc;  // unit table columns + extent deltas
  size_t extd_n = 0;                          // entries uploaded to extd
  IndexBufs fwd, rev;
  // page directory over the unit bases (cgcm_dev.h PdDev; built with the table)
  DevBuf pd_ent, pd_ovf, pd_start, pd_meta;
  int pd_nseg = 0, pd_v3 = 0;
  // the entries' page-state words (cgcm_dev.h) must be recomputed before a kernel reads the directory:
  // set by every change of a unit's ACTIVE / STORAGE / extent (activations, frees, unit ops, rebuilds)
  bool pd_state_dirty = true;
  uint64_t pd_pages = 0, pd_ovf_pages = 0, pd_bytes = 0;
  uint32_t pd_minP = 0, pd_maxP = 0;

  // scratch
  DevBuf slowmask, slowcnt, wlist, dump_rc, glue_prog, glue_regs, glue_status;
  // device-side transfer planning (activation packs, copy-back runs) for lists of >= PLAN_MIN units
  static constexpr size_t PLAN_MIN = 1u << 16;
  DevBuf plan_S, plan_F, plan_G, plan_pid, plan_gscan, plan_tmp, plan_cnt, plan_desc, plan_run;
  size_t plan_tb = 0;
  // the per-unit host mirrors (udev, urun, uarr) are not written by planned activations: stale until
  // need_mirrors() rebuilds them from the device table (only host paths read them)
  bool mirror_stale = false;
  DevBuf status, lc, hitmask, act_list, journal, free_list, copy_list, segs, seg0, staging, staging2, staging_cb, points, ptrs, temp;
  DevBuf up_units, up_vals, up_exts, uops;
  HostBuf h_small, h_status, h_list, h_pack[2];
  // pinned staging ring for small uploads: two halves, each fenced by an event on the main stream --
  // an upload waits for the GPU only when it reuses a half whose copies may still be in flight
  static constexpr size_t RING_HALF = 1 << 20;
  HostBuf h_ring;
  cudaEvent_t ev_ring[2] = {nullptr, nullptr};
  bool ring_used[2] = {false, false};
  int ring_cur = 0;
  size_t ring_head = 0;
  int pack_k = 0;
  cudaEvent_t ev_copy = nullptr, ev_t0 = nullptr, ev_t1 = nullptr, ev_pack[2] = {nullptr, nullptr};

  // runs of device extents
  std::vector<Run> runs;
  std::vector<int64_t> free_runs;
  std::map<uint64_t, int64_t> live_runs;  // extent start -> run id (the reverse index's keys)

  // pinned host arena (cgcm_malloc)
  std::vector<std::pair<char *, size_t>> hchunks;
  std::map<uint64_t, uint64_t> hfree;                 // addr -> len
  std::unordered_map<uint64_t, uint64_t> hallocs;     // addr -> rounded len
  std::unordered_map<uint64_t, uint64_t> hsizes;      // addr -> requested size (realloc)
  std::vector<std::vector<uint64_t>> scopes;           // declareAlloca registrations per open scope

  cgcm_stats_t st{};

  // Small inputs that repeat call after call (a promoted loop's segment table and unit ops) are uploaded
  // only when the device bytes differ from the last upload to that range (put_memo: device address ->
  // bytes).  Every write to those buffers goes through ring_put_memo or forgets the range (memo_forget),
  // and so does every release or reallocation of a buffer.
  std::map<uint64_t, std::string> put_memo;
  void memo_forget(uint64_t lo, uint64_t n) {
    for (auto it = put_memo.begin(); it != put_memo.end();)
      it = (it->first < lo + n && lo < it->first + it->second.size()) ? put_memo.erase(it) : std::next(it);
  }
  int ring_put_memo(void *dst, const void *src, size_t n) {
    const uint64_t key = reinterpret_cast<uint64_t>(dst);
    auto it = put_memo.find(key);
    if (it != put_memo.end() && it->second.size() == n && std::memcmp(it->second.data(), src, n) == 0) return CGCM_OK;
    memo_forget(key, n);
    CKS(ring_put(dst, src, n));
    put_memo[key].assign(static_cast<const char *>(src), n);
    return CGCM_OK;
  }
  // ------------------------------------------------------------------------------------------
  int dalloc(DevBuf &b, size_t need) {  // ensure capacity (contents not preserved)
    if (need <= b.bytes && b.addr) return CGCM_OK;
    if (b.addr) memo_forget(b.addr, b.bytes);
    if (b.addr) arena.free(b.addr, b.bytes);
    size_t nb = std::max<size_t>(need, 256);
    nb = std::max(nb, b.bytes * 3 / 2);
    b.addr = arena.alloc(nb);
    if (!b.addr) {
      b.bytes = 0;
      return CGCM_E_NOMEM;
    }
    b.bytes = align_up(nb, 256);
    return CGCM_OK;
  }
  void dfree(DevBuf &b) {
    if (b.addr) memo_forget(b.addr, b.bytes);
    if (b.addr) arena.free(b.addr, b.bytes);
    b.addr = 0;
    b.bytes = 0;
  }
  TableDev tab() const {
    TableDev t;
    t.hot = hotb.as<uint64_t>();
    t.hotc = hotcb.as<uint32_t>();
    t.st = stb.as<uint64_t>();
    t.rc = rcb.as<int32_t>();
    t.base = dbase.as<uint64_t>();
    t.size64 = size64.as<uint64_t>();
    t.ext_delta = extd.as<uint64_t>();
    t.ext_lo = extlo.as<uint64_t>();
    t.ext_len = extlen.as<uint32_t>();
    t.n_ext = (int)extd_n;
    return t;
  }
  // device copy of the extent deltas (devbase - base) indexed by run id
  int sync_ext() {
    std::vector<uint64_t> d(std::max<size_t>(runs.size(), 1), 0), lo(d.size(), 0);
    std::vector<uint32_t> len(d.size(), 0);
    for (size_t r = 0; r < runs.size(); ++r) {
      d[r] = 0 - runs[r].delta;  // runs store host - device
      lo[r] = runs[r].addr;
      len[r] = runs[r].bytes < (1ull << 32) ? (uint32_t)runs[r].bytes : 0u;  // >= 4 GiB: shadows not used
    }
    CKS(upload(extd, d, true));  // input-only buffers: repeated contents are not re-sent
    CKS(upload(extlo, lo, true));
    CKS(upload(extlen, len, true));
    extd_n = runs.size();
    return CGCM_OK;
  }

  int64_t new_run(uint64_t addr, uint64_t bytes, uint64_t delta) {
    Run r;
    r.addr = addr;
    r.bytes = bytes;
    r.delta = delta;
    r.live = 0;
    int64_t id;
    if (!free_runs.empty()) {
      id = free_runs.back();
      free_runs.pop_back();
      runs[id] = r;
    } else {
      runs.push_back(r);
      id = (int64_t)runs.size() - 1;
    }
    live_runs[addr] = id;
    rev_dirty = true;
    return id;
  }
  void drop_run(int64_t id) {
    if (!runs[id].external) arena.free(runs[id].addr, runs[id].bytes);
    live_runs.erase(runs[id].addr);
    runs[id] = Run();
    free_runs.push_back(id);
    rev_dirty = true;
  }
  void run_release(int64_t id) {
    if (id < 0) return;
    free_gen += 1;  // device addresses of this unit may now be reused by another unit
    if (--runs[id].live <= 0) drop_run(id);
  }

  int sync_main() {
    CK(cudaStreamSynchronize(main));
    return CGCM_OK;
  }

  // ------------------------------------------------------------------------------------------
  // index build (a0)
  // Build a search index over n sorted keys (hkeys on the host, dkeys the same keys on the device):
  // top splitters, wide bits, segments and radix directory on the host; u32 levels on the device.
  int build_index(IndexBufs &ib, const uint64_t *hkeys, int n, const uint64_t *dkeys, int topmax, int dirmax) {
    int h = 0;
    while (n > 0 && ((((int64_t)n + (1ll << (3 * h)) - 1) >> (3 * h)) > topmax)) ++h;
    int ntop = n > 0 ? (int)((((int64_t)n + (1ll << (3 * h)) - 1) >> (3 * h))) : 0;
    std::vector<uint64_t> top(std::max(ntop, 1), 0);
    std::vector<uint32_t> wide((ntop + 31) / 32 + 1, 0);
    for (int t = 0; t < ntop; ++t) {
      int64_t first = (int64_t)t << (3 * h), last = std::min<int64_t>(n, (int64_t)(t + 1) << (3 * h)) - 1;
      top[t] = hkeys[first];
      if (hkeys[last] - hkeys[first] >= 0xFFFFFFFFull) wide[t >> 5] |= 1u << (t & 31);
    }
    // segments at large gaps (so that one far-away region does not flatten the directory)
    std::vector<int> segstart;
    for (int thr = 32; thr <= 64; ++thr) {
      segstart.assign(1, 0);
      for (int t = 1; t < ntop; ++t)
        if (thr < 64 && top[t] - top[t - 1] >= (1ull << thr)) segstart.push_back(t);
      if ((int)segstart.size() <= MAXSEG) break;
    }
    int nseg = ntop > 0 ? (int)segstart.size() : 0;
    std::vector<uint64_t> skmin(std::max(nseg, 1), 0);
    std::vector<uint32_t> smeta(4 * std::max(nseg, 1), 0), dir;
    for (int g = 0; g < nseg; ++g) {
      int t0 = segstart[g], t1 = g + 1 < nseg ? segstart[g + 1] : ntop;
      uint64_t kmin = top[t0], span = top[t1 - 1] - kmin;
      const int64_t dir_total = std::min<int64_t>(dirmax - nseg, std::max<int64_t>(64, 2 * (int64_t)ntop));
      int64_t nbt = std::max<int64_t>(1, dir_total * (t1 - t0) / std::max(ntop, 1));
      uint32_t shift = 0;
      while (shift < 63 && (int64_t)(span >> shift) + 1 > nbt) ++shift;
      uint32_t nb = (uint32_t)((span >> shift) + 1);
      skmin[g] = kmin;
      smeta[4 * g] = (uint32_t)dir.size();
      smeta[4 * g + 1] = nb;
      smeta[4 * g + 2] = (uint32_t)t1;
      smeta[4 * g + 3] = shift;
      for (uint32_t d = 0; d < nb; ++d) {
        uint64_t bstart = kmin + ((uint64_t)d << shift);
        dir.push_back((uint32_t)(std::lower_bound(top.begin() + t0, top.begin() + t1, bstart) - top.begin()));
      }
    }
    if (dir.empty()) dir.push_back(0);
    std::vector<uint64_t> topv(top.begin(), top.begin() + std::max(ntop, 1));
    CKS(upload(ib.top, topv));
    CKS(upload(ib.wide, wide));
    CKS(upload(ib.dir, dir));
    CKS(upload(ib.skmin, skmin));
    CKS(upload(ib.smeta, smeta));
    uint32_t *lv[MAXL];
    for (int k = 0; k < MAXL; ++k) {
      if (k < h) {
        int64_t cnt = ((int64_t)n + (1ll << (3 * k)) - 1) >> (3 * k);
        size_t need = (size_t)((cnt + 7) / 8 * 8 + 8);
        CKS(dalloc(ib.lvl[k], 4 * need));
        ib.lvl_cap[k] = need;
      }
      lv[k] = ib.lvl[k].as<uint32_t>();
    }
    if (h > 0) {
      launch_build_levels(dkeys, n, h, ib.wide.as<uint32_t>(), lv, ib.lvl_cap, main);
      st.kernel_launches += h;
      CK(cudaGetLastError());
    }
    ib.n = n;
    ib.h = h;
    ib.ntop = ntop;
    ib.nseg = nseg;
    ib.ndir = (int)dir.size();
    ib.any_wide = false;
    for (uint32_t w : wide) ib.any_wide = ib.any_wide || w != 0;
    return CGCM_OK;
  }

  // Page directory (a0): cut the sorted bases at the largest start-to-start distances (>= 1 MiB, at
  // most PD_MAXSEG segments; pages stop at a segment's last base, whose unit's tail is decided by
  // the segment's end), give each segment the largest page size 2^P (P <= PD_MAXSHIFT) whose crowded pages (more than
  // PD_K starts) hold at most CGCM_PD_OVF (default 1 %) of its units, within a budget of
  // max(4n, 2^20) entries overall; then one entry per page (cgcm_dev.h).  No directory (the level
  // index serves the hot kernels) when the budget cannot be met or CGCM_NO_PAGEDIR is set.
  int build_pd(const uint64_t *hb, const uint64_t *hs, int n) {
    pd_nseg = 0;
    pd_pages = pd_ovf_pages = pd_bytes = 0;
    pd_minP = pd_maxP = 0;
    static const bool env_off = std::getenv("CGCM_NO_PAGEDIR") != nullptr;  // A/B experiments
    if (n == 0 || (flags & CGCM_NO_PAGEDIR) || env_off) return CGCM_OK;
    static const double ovf_frac = [] {
      const char *e = std::getenv("CGCM_PD_OVF");
      return e ? std::atof(e) : 0.01;
    }();
    std::vector<std::pair<uint64_t, int>> gaps;
    for (int i = 0; i + 1 < n; ++i) {
      const uint64_t g = hb[i + 1] - hb[i];  // start to start: a huge unit's tail needs no pages
      if (g >= (1ull << 20)) gaps.emplace_back(g, i + 1);
    }
    if ((int)gaps.size() > PD_MAXSEG - 1) {
      std::nth_element(gaps.begin(), gaps.begin() + (PD_MAXSEG - 1), gaps.end(),
                       [](const std::pair<uint64_t, int> &a, const std::pair<uint64_t, int> &b) { return a.first > b.first; });
      gaps.resize(PD_MAXSEG - 1);
    }
    std::vector<int> cut{0};
    for (auto &g : gaps) cut.push_back(g.second);
    std::sort(cut.begin(), cut.end());
    cut.push_back(n);
    const int nseg = (int)cut.size() - 1;
    const uint64_t budget = std::max<uint64_t>(4ull * (uint64_t)n, 1ull << 20);
    std::vector<uint32_t> Ps(nseg);
    std::vector<uint64_t> npg(nseg);
    uint64_t total = 0;
    static const int force_fmt = [] {  // A/B: CGCM_PD_FORMAT=2 or 3
      const char *e = std::getenv("CGCM_PD_FORMAT");
      return e ? std::atoi(e) : 0;
    }();
    // v3 entries (PD_K3 candidates) when the directory they need stays L2-sized, else v2 (PD_K2 starts)
    int v3 = (force_fmt == 2 || (flags & CGCM_PD_V2)) ? 0 : 1;
  size_pages:
    const int PD_K = v3 ? PD_K3 : PD_K2;
    total = 0;
    for (int s = 0; s < nseg; ++s) {
      const int i0 = cut[s], i1 = cut[s + 1];
      const uint64_t S = hb[i0], span = hb[i1 - 1] - S;  // pages up to the last base; beyond: its tail
      const uint64_t cap = budget * (uint64_t)(i1 - i0) / (uint64_t)n + 1024;
      int sel = -1;
      for (int P = PD_MAXSHIFT; P >= 0; --P) {
        if ((span >> P) + 1 > cap) break;
        uint64_t ovf = 0;  // units in pages with more than PD_K starts after the page's first byte
        bool fits = true;  // every page: <= PD_CNT_MAX starts, none at offset PD_PAD (the padding value)
        for (int i = i0; i < i1 && fits;) {
          const uint64_t pg = (hb[i] - S) >> P;
          int k = i, c = 0;
          while (k < i1 && ((hb[k] - S) >> P) == pg) {
            const uint64_t o = (hb[k] - S) & ((1ull << P) - 1);
            c += o != 0;
            fits = fits && o != PD_PAD;
            ++k;
          }
          if (c > PD_K) ovf += (uint64_t)c;
          fits = fits && (uint32_t)c <= PD_CNT_MAX;
          i = k;
        }
        if (!fits) continue;
        sel = P;
        if ((double)ovf <= ovf_frac * (double)(i1 - i0)) break;
      }
      if (sel < 0) {  // too sparse for the budget: the other format, or the level index serves
        if (v3 && force_fmt != 3) {
          v3 = 0;
          goto size_pages;
        }
        return CGCM_OK;
      }
      Ps[s] = (uint32_t)sel;
      npg[s] = (span >> sel) + 1;
      total += npg[s];
    }
    if (v3 && force_fmt != 3 && 32 * total > PD_V3_MAX_BYTES) {
      v3 = 0;
      goto size_pages;
    }
    std::vector<uint32_t> ent(8 * total);
    std::vector<uint16_t> ovf;
    std::vector<uint64_t> starts(2 * nseg);  // [start_s..., last_end_s...]
    std::vector<uint32_t> meta(4 * nseg, 0);
    uint64_t e = 0, novf = 0;
    for (int s = 0; s < nseg; ++s) {
      const int i0 = cut[s], i1 = cut[s + 1];
      const uint64_t S = hb[i0], psz = 1ull << Ps[s];
      starts[s] = S;
      starts[nseg + s] = hb[i1 - 1] + hs[i1 - 1];
      meta[4 * s] = (uint32_t)e;
      meta[4 * s + 1] = (uint32_t)npg[s];
      meta[4 * s + 2] = Ps[s];
      meta[4 * s + 3] = (uint32_t)(i1 - 1);
      int i = i0;  // greatestLTE(A)
      for (uint64_t g = 0; g < npg[s]; ++g, ++e) {
        const uint64_t A = S + (g << Ps[s]);
        while (i + 1 < i1 && hb[i + 1] <= A) ++i;
        int k = i + 1;
        while (k < i1 && hb[k] < A + psz) ++k;
        const uint32_t cnt = (uint32_t)(k - (i + 1));
        const uint64_t e0 = hb[i] + hs[i];
        const uint32_t end0 = e0 < A ? 0u : (uint32_t)std::min<uint64_t>(e0 - A + 1, PD_END_MAX);
        uint32_t *w = &ent[8 * e];
        w[0] = (uint32_t)i;
        w[1] = cnt | (hb[i] == A ? PD_EXACT : 0u) | (end0 << PD_END_SHIFT);
        if (!v3) {  // v2: up to PD_K2 sorted u16 starts in w[2..7]
          uint16_t *o16 = reinterpret_cast<uint16_t *>(w + 2);
          if (cnt <= (uint32_t)PD_K2) {
            for (int t = 0; t < PD_K2; ++t) o16[t] = t < (int)cnt ? (uint16_t)(hb[i + 1 + t] - A) : (uint16_t)PD_PAD;
          } else {
            w[2] = (uint32_t)ovf.size();
            w[3] = w[4] = w[5] = w[6] = w[7] = 0xFFFFFFFFu;
            for (uint32_t t = 0; t < cnt; ++t) ovf.push_back((uint16_t)(hb[i + 1 + t] - A));
            while (ovf.size() % 16) ovf.push_back((uint16_t)PD_PAD);
            ++novf;
          }
          continue;
        }
        w[2] = 0;  // page state: computed on the device (k_pd_state)
        if (cnt <= (uint32_t)PD_K3) {
          for (int t = 0; t < PD_K3; ++t) {
            if (t < (int)cnt) {
              const uint64_t st0 = hb[i + 1 + t] - A, en = std::min<uint64_t>(hb[i + 1 + t] + hs[i + 1 + t] - A, PD_PAD);
              w[3 + t] = (uint32_t)st0 | ((uint32_t)en << 16);
            } else {
              w[3 + t] = PD_PAD;  // start PD_PAD (never <= a clamped p - A), end 0
            }
          }
        } else {
          w[3] = (uint32_t)ovf.size();
          w[4] = w[5] = w[6] = w[7] = 0xFFFFFFFFu;
          for (uint32_t t = 0; t < cnt; ++t) ovf.push_back((uint16_t)(hb[i + 1 + t] - A));
          while (ovf.size() % 16) ovf.push_back((uint16_t)PD_PAD);
          ++novf;
        }
      }
    }
    if (ovf.empty()) ovf.assign(16, (uint16_t)PD_PAD);
    CKS(upload(pd_ent, ent));
    CKS(upload(pd_ovf, ovf));
    CKS(upload(pd_start, starts));
    CKS(upload(pd_meta, meta));
    pd_nseg = nseg;
    pd_v3 = v3;
    pd_pages = total;
    pd_ovf_pages = novf;
    pd_bytes = 32 * total + 2 * ovf.size();
    pd_minP = *std::min_element(Ps.begin(), Ps.end());
    pd_maxP = *std::max_element(Ps.begin(), Ps.end());
    return CGCM_OK;
  }
  PdDev pd_view() const {
    PdDev p;
    p.ent = pd_ent.as<uint32_t>();
    p.ovf = pd_ovf.as<uint16_t>();
    p.seg_start = pd_start.as<uint64_t>();
    p.seg_meta = pd_meta.as<uint32_t>();
    p.nseg = pd_nseg;
    p.v3 = pd_v3;
    return p;
  }

  void note_declared(uint64_t b) {
    if (pend_over) return;
    if (pend.size() >= (size_t)DELTA_MAX) {
      pend_over = true;
      pend.clear();
    } else {
      pend.push_back(b);
    }
  }
  // A pending unit that starts exactly where a unit of the main table ends would win greatestLTE at that
  // unit's one-past-the-end address (A7), which the main lookup decides as a hit: such a declaration
  // takes the rebuild, so that the kernels consult the delta units only where the main table misses.
  bool delta_touches_main() const {
    for (uint64_t b : pend) {
      auto it = reg.lower_bound(b);
      if (it == reg.begin()) continue;
      --it;
      if (it->second.idx >= 0 && it->second.idx < Umain && it->first + it->second.size == b) return true;
    }
    return false;
  }
  // the batched merge of pending declarations (NEXT-1): append them to the columns as delta units and
  // re-sort the small delta index -- O(#pending + #delta) host work, no registry walk, no rebuild
  int append_delta() {
    Trace trace_("ensure_table(delta)");
    std::sort(pend.begin(), pend.end());
    const size_t t = pend.size();
    std::vector<uint64_t> nb(t), ns(t), nh(t), nst(t);
    std::vector<uint32_t> nhc(t);
    std::vector<int32_t> nrc(t, 0);
    for (size_t q = 0; q < t; ++q) {
      auto it = reg.find(pend[q]);
      HostUnit &u = it->second;
      const uint32_t id = (uint32_t)(U + q);
      u.idx = (int32_t)id;
      const uint32_t fl = u.flags & (UF_GLOBAL | UF_READONLY);
      nb[q] = pend[q];
      ns[q] = u.size;
      nh[q] = make_hot(u.size, NO_EXT, fl);
      nhc[q] = make_hotc(nh[q]);
      nst[q] = make_st(nh[q], rel_epoch(u.epoch0));
      ubase.push_back(pend[q]);
      usize.push_back(u.size);
      uflags.push_back(fl);
      usym.push_back(u.sym);
      udev.push_back(0);
      urun.push_back(-1);
      uarr.push_back(0);
      dk.push_back(pend[q]);
      di.push_back(id);
    }
    if (t) {
      CKS(ring_put(dbase.as<uint64_t>() + U, nb.data(), 8 * t));
      CKS(ring_put(size64.as<uint64_t>() + U, ns.data(), 8 * t));
      CKS(ring_put(hotb.as<uint64_t>() + U, nh.data(), 8 * t));
      CKS(ring_put(hotcb.as<uint32_t>() + U, nhc.data(), 4 * t));
      CKS(ring_put(stb.as<uint64_t>() + U, nst.data(), 8 * t));
      CKS(ring_put(rcb.as<int32_t>() + U, nrc.data(), 4 * t));
    }
    // the delta index, sorted by base
    std::vector<size_t> ord(dk.size());
    for (size_t q = 0; q < ord.size(); ++q) ord[q] = q;
    std::sort(ord.begin(), ord.end(), [&](size_t x, size_t y) { return dk[x] < dk[y]; });
    std::vector<uint64_t> k2(ord.size());
    std::vector<uint32_t> i2(ord.size());
    for (size_t q = 0; q < ord.size(); ++q) {
      k2[q] = dk[ord[q]];
      i2[q] = di[ord[q]];
    }
    dk.swap(k2);
    di.swap(i2);
    CKS(upload(dkeys, dk));
    CKS(upload(dids, di));
    U += (int)t;
    pend.clear();
    table_dirty = false;
    st.table_merges += 1;
    return CGCM_OK;
  }

  // merge pending declares/undeclares into the device table (A19: kernels only see a compacted table)
  struct Stage {
    std::vector<uint64_t> w;
    size_t size() const { return 8 * w.size(); }
    void resize(size_t bytes) { w.resize((bytes + 7) / 8); }
    uint64_t *data() { return w.data(); }
  } table_stage;
  int ensure_table() {
    if (table_dirty) leases.clear();  // a rebuild renumbers the units
    Trace trace_("ensure_table");
    if (!table_dirty) return CGCM_OK;
    if (!dirty_del && !pend_over && Umain > 0 && dk.size() + pend.size() <= (size_t)DELTA_MAX &&
        (size_t)U + pend.size() <= col_cap && !delta_touches_main())
      return append_delta();
    CKS(materialise_all());  // deferred references name units by their index in the table being replaced
    CKS(need_mirrors());     // the remap carries the per-unit host mirrors to the new indices
    int n = (int)reg.size();
    // host staging: base[n], size[n], epoch0[n] (u32, relative), old_idx[n], flags[n]
    size_t need = (size_t)n * (8 + 8 + 4 + 4 + 4) + 256;
    // pageable staging (the uploads below are followed by a host wait anyway): a pinned buffer sized to the
    // table would cost a cudaHostAlloc here, 8-600 ms on this pool (profiles/r02bw_trace.log)
    if (table_stage.size() < need) table_stage.resize(need);
    {
      Trace t1("ensure_table:wait");
      CK(cudaStreamSynchronize(main));
      CK(cudaStreamSynchronize(copy));
    }
    uint64_t *hb = reinterpret_cast<uint64_t *>(table_stage.data());
    uint64_t *hs = hb + n;
    uint32_t *he = reinterpret_cast<uint32_t *>(hs + n);
    int32_t *ho = reinterpret_cast<int32_t *>(he + n);
    uint32_t *hf = reinterpret_cast<uint32_t *>(ho + n);
    std::vector<uint64_t> ndev(n, 0);
    std::vector<int64_t> nrun(n, -1);
    std::vector<uint8_t> narr(n, 0);
    uflags.resize(n);
    usym.resize(n);
    int i = 0;
    for (auto it = reg.begin(); it != reg.end(); ++it, ++i) {
      int32_t o = it->second.idx;
      hb[i] = it->first;
      hs[i] = it->second.size;
      he[i] = rel_epoch(it->second.epoch0);
      ho[i] = o;
      hf[i] = it->second.flags & (UF_GLOBAL | UF_READONLY);
      uflags[i] = hf[i];
      usym[i] = it->second.sym;
      if (o >= 0) {
        ndev[i] = udev[o];
        nrun[i] = urun[o];
        narr[i] = uarr[o];
      }
      it->second.idx = i;
    }
    ubase.assign(hb, hb + n);
    usize.assign(hs, hs + n);
    udev.swap(ndev);
    urun.swap(nrun);
    uarr.swap(narr);
    DevBuf nhot, nhotc, nst, nrc, nsize, nbase, tmp;
    int cap = std::max(n, 1) + DELTA_MAX;  // room for delta units appended by later merges
    CKS(dalloc(nhot, 8 * (size_t)cap + 64));
    CKS(dalloc(nhotc, 4 * (size_t)cap + 64));
    CKS(dalloc(nst, 8 * (size_t)cap + 64));
    CKS(dalloc(nrc, 4 * (size_t)cap + 64));
    CKS(dalloc(nsize, 8 * (size_t)cap));
    CKS(dalloc(nbase, 8 * (size_t)cap));
    CKS(dalloc(tmp, (size_t)cap * 24 + 256));
    if (n > 0) {
      CK(cudaMemcpyAsync(nbase.as<void>(), hb, 8 * (size_t)n, cudaMemcpyHostToDevice, main));
      CK(cudaMemcpyAsync(nsize.as<void>(), hs, 8 * (size_t)n, cudaMemcpyHostToDevice, main));
      CK(cudaMemcpyAsync(tmp.as<void>(), he, (size_t)n * 12, cudaMemcpyHostToDevice, main));
      const uint32_t *depoch = tmp.as<uint32_t>();
      const int32_t *dold = reinterpret_cast<const int32_t *>(depoch + n);
      const uint32_t *dflags = reinterpret_cast<const uint32_t *>(dold + n);
      TableDev nt = tab();
      nt.hot = nhot.as<uint64_t>();
      nt.hotc = nhotc.as<uint32_t>();
      nt.st = nst.as<uint64_t>();
      nt.rc = nrc.as<int32_t>();
      launch_remap(n, dold, nsize.as<uint64_t>(), dflags, depoch, tab(), nt, main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
      CK(cudaStreamSynchronize(main));
    }
    dfree(tmp);
    dfree(hotb);
    dfree(hotcb);
    dfree(stb);
    dfree(rcb);
    dfree(size64);
    dfree(dbase);
    hotb = nhot;
    hotcb = nhotc;
    stb = nst;
    rcb = nrc;
    size64 = nsize;
    dbase = nbase;
    U = n;
    Umain = n;
    col_cap = (size_t)cap;
    pend.clear();
    pend_over = false;
    dirty_del = false;
    dk.clear();
    di.clear();
    {
      Trace t2("ensure_table:index");
      CKS(build_index(fwd, hb, n, dbase.as<uint64_t>(), TOPMAX, DIRMAX));
    }
    {
      Trace t3("ensure_table:pagedir");
      CKS(build_pd(hb, hs, n));
    }
    pd_state_dirty = true;
    CK(cudaStreamSynchronize(main));
    table_dirty = false;
    rev_dirty = true;
    table_gen += 1;  // unit indices changed: recorded shadows are stale
    st.table_rebuilds += 1;
    return CGCM_OK;
  }

  // reverse index: the live device extents by start address, payload = host - device delta
  int ensure_rev() {
    CKS(ensure_table());
    if (!rev_dirty) return CGCM_OK;
    std::vector<uint64_t> keys, pay;
    std::vector<uint32_t> rid;
    keys.reserve(live_runs.size() + 1);
    pay.reserve(live_runs.size() + 1);
    for (auto &kv : live_runs) {
      keys.push_back(kv.first);
      pay.push_back(runs[kv.second].delta);
      rid.push_back((uint32_t)kv.second);
    }
    std::vector<uint64_t> kup = keys, pup = pay;
    std::vector<uint32_t> rup = rid;
    if (kup.empty()) {
      kup.push_back(0);
      pup.push_back(0);
      rup.push_back(0);
    }
    CKS(upload(rev.keys, kup));
    CKS(upload(rev.pay, pup));
    CKS(upload(rev.rid, rup));
    CKS(build_index(rev, keys.data(), (int)keys.size(), rev.keys.as<uint64_t>(), RUN_SMEM, RUN_SMEM));
    rev_dirty = false;
    st.rev_rebuilds += 1;
    return CGCM_OK;
  }

  // ------------------------------------------------------------------------------------------
  // slot kernels
  struct SlotCall {
    int dir = DIR_FWD, ops = 0, sel = SEL_ALL;
    bool dec_red = false;  // OP_DEC through reductions + k_release_scan (large batches)
    bool no_journal = false;  // large gate passes snapshot the rc/epoch columns instead
    bool defer = false;       // deferred references (cgcm_dev.h SlotArgs::defer)
    bool lazy = false;        // counters into lazy_status (folded when read), not the call's Status block
    uint32_t rc_unit = 0;     // k_slots applies rc[rc_unit] += rc_delta once (the queued re-map / release)
    int32_t rc_delta = 0;
    std::vector<Seg> segs;
    uint64_t nchunks = 0;
    Status res{};
    // transfer overlap (mapArrays): segs are ordered by group (nondecreasing, -1 first); the chunks of
    // group g are translated by a launch that waits for group_ev[g] (the H2D copy of their extent)
    std::vector<int> seg_group;
    std::vector<cudaEvent_t> group_ev;
  };

  int list_capacity() const { return std::max(U, 1); }
  size_t slot_smem_estimate(const SlotCall &c) const {
    (void)c;
    return 8 * (size_t)fwd.ntop + 4 * (size_t)fwd.ndir + 12 * (size_t)rev.ntop + 4 * (size_t)rev.ndir + 8 * extd_n;
  }

  // upload segments, launch, (no sync).  slot st index = which Status block to use.
  int launch(SlotCall &c, int st_index, bool reuse_hitmask_layout = false, bool timed_fwd = false,
             bool timed_rev = false) {
    (void)reuse_hitmask_layout;
    if (c.ops & (OP_DEC | OP_DECPLAIN)) lease_break();
    lists_fresh = false;  // the kernels below may append to the unit lists
    int k = (int)c.segs.size();
    if (k == 0) return CGCM_OK;
    std::vector<uint64_t> c0(k + 1, 0);
    for (int s = 0; s < k; ++s) {
      uint64_t head = (c.segs[s].ptr & 15) / 8;
      c0[s + 1] = c0[s] + (c.segs[s].n ? (head + c.segs[s].n + 1) / 2 : 0);
    }
    c.nchunks = c0[k];
    if (c.nchunks == 0) return CGCM_OK;
    if (c.nchunks > (1u << 15)) launches_small = false;  // no list heads with the next status fetch
    if ((c.ops & OP_HITMASK) || c.sel != SEL_ALL) CKS(dalloc(hitmask, 4 * (size_t)(c.nchunks / 16 + 4)));
    if (c.dir == DIR_REV) CKS(dalloc(slowmask, 4 * (size_t)(c.nchunks / 16 + 4)));
    CKS(dalloc(slowcnt, 64));
    CKS(dalloc(wlist, 4 * (size_t)(c.nchunks / 32 + 8)));
    CKS(dalloc(segs, sizeof(Seg) * (size_t)k * 8 + 256));
    CKS(dalloc(seg0, 8 * (size_t)(k + 1) * 8 + 256));
    // each launch uses its own eighth of the segment buffers (st_index 0..7, up to 8 launches in flight)
    Seg *dsegs = segs.as<Seg>() + (size_t)st_index * k;
    uint64_t *dc0 = seg0.as<uint64_t>() + (size_t)st_index * (k + 1);
    // pinned ring: no host wait, and no DMA (read by a kernel) -- also while the outers' H2D copies
    // are in flight on the copy stream
    if (sizeof(Seg) * k + 8 * (size_t)(k + 1) <= RING_HALF / 2) {
      CKS(ring_put_memo(dsegs, c.segs.data(), sizeof(Seg) * k));
      CKS(ring_put_memo(dc0, c0.data(), 8 * (size_t)(k + 1)));
    } else {
      memo_forget(reinterpret_cast<uint64_t>(dsegs), sizeof(Seg) * k);
      memo_forget(reinterpret_cast<uint64_t>(dc0), 8 * (size_t)(k + 1));
      CK(cudaMemcpyAsync(dsegs, c.segs.data(), sizeof(Seg) * k, cudaMemcpyHostToDevice, main));
      CK(cudaMemcpyAsync(dc0, c0.data(), 8 * (size_t)(k + 1), cudaMemcpyHostToDevice, main));
      CK(cudaStreamSynchronize(main));  // the host vectors above are pageable and go out of scope
    }
    SlotArgs a;
    std::memset(&a, 0, sizeof(a));
    a.tab = tab();
    a.fx = fwd.view(dbase.as<uint64_t>());
    a.fx_nowide = fwd.any_wide ? 0 : 1;
    a.pd = pd_view();
    a.dkeys = dkeys.as<uint64_t>();
    a.dids = dids.as<uint32_t>();
    a.dn = (int)dk.size();
    if (c.dir == DIR_REV) {
      a.rx = rev.view(rev.keys.as<uint64_t>());
      a.runpay = rev.pay.as<uint64_t>();
      a.runid = rev.rid.as<uint32_t>();
    }
    a.segs = dsegs;
    a.segs_host_shadow = 0;
    for (auto &sg : c.segs) a.segs_host_shadow |= sg.shadow != 0 ? 1 : 0;
    a.seg_inplace = (k == 1 && c.segs[0].out == 0) ? 1 : 0;
    a.seg_chunk0 = dc0;
    a.nseg = k;
    a.sel = c.sel;
    a.nchunks = c.nchunks;
    a.hitmask = hitmask.as<uint32_t>();
    a.slowmask = slowmask.as<uint32_t>();
    a.slowcount = slowcnt.as<unsigned long long>();
    a.wlist = wlist.as<uint32_t>();
    a.wcount = slowcnt.as<unsigned long long>() + 1;
    a.rc_unit = c.rc_unit;
    a.rc_delta = c.rc_delta;
    a.dec_red = c.dec_red ? 1 : 0;
    a.no_journal = c.no_journal ? 1 : 0;
    a.defer = c.defer ? 1 : 0;
    a.epoch = rel_epoch(epoch);
    a.st = c.lazy ? lazy_status.as<Status>() : status.as<Status>() + st_index;
    a.lc = lc.as<unsigned long long>();
    a.act_list = act_list.as<uint32_t>();
    a.journal = journal.as<Journal>();
    a.copy_list = copy_list.as<uint32_t>();
    a.free_list = free_list.as<uint32_t>();
    a.lenient = (flags & CGCM_LENIENT) ? 1 : 0;
    if (pd_nseg > 0 && pd_v3 && pd_state_dirty) {
      launch_pd_state(pd_view(), pd_pages, tab(), main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
      pd_state_dirty = false;
    }
    const bool pieces = !c.seg_group.empty();
    bool timed = (flags & CGCM_PROFILE) && (timed_fwd || timed_rev) && !pieces;
    if (timed) CK(cudaEventRecord(ev_t0, main));
    int nl = 0;
    int r = 0;
    if (!pieces) {
      r = launch_slots(c.dir, c.ops, a, nsm, main, &nl);
    } else {
      // one launch per copy group, each after its group's H2D copy: translation of the extents that
      // have arrived overlaps the copies still in flight.  Piece boundaries are multiples of 32 chunks
      // (one warp's hit-mask words); chunks of group g below the boundary ride with group g + 1,
      // whose copy is issued after g's on the same stream.
      uint64_t cb = 0;
      for (int s0 = 0; s0 < k && r == 0;) {
        const int g = c.seg_group[s0];
        int s1 = s0;
        while (s1 < k && c.seg_group[s1] == g) ++s1;
        const uint64_t ce = s1 < k ? (c0[s1] & ~31ull) : c.nchunks;
        if (g >= 0) CK(cudaStreamWaitEvent(main, c.group_ev[g], 0));
        if (ce > cb) {
          SlotArgs b = a;
          b.cbeg = cb;
          b.nchunks = ce;
          int n1 = 0;
          r = launch_slots(c.dir, c.ops, b, nsm, main, &n1);
          nl += n1;
          cb = ce;
        }
        s0 = s1;
      }
    }
    if (r != 0) {
      g_last_cuda_error = r == -2 ? std::string("unsupported slot-kernel operation set")
                                  : std::string("k_slots launch (dir ") + std::to_string(c.dir) + ", ops " +
                                        std::to_string(c.ops) + ", smem " + std::to_string(slot_smem_estimate(c)) +
                                        "): " + cudaGetErrorString((cudaError_t)r);
      return CGCM_E_CUDA;
    }
    CK(cudaGetLastError());
    st.kernel_launches += (uint64_t)nl;
    if ((c.ops & OP_DEC) && c.dec_red) {  // underflow / 1 -> 0 detection after reductions
      launch_release_scan(tab(), U, status.as<Status>() + st_index, lc.as<unsigned long long>(),
                          free_list.as<uint32_t>(), main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
    }
    if (timed) {
      CK(cudaEventRecord(ev_t1, main));
      CK(cudaEventSynchronize(ev_t1));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, ev_t0, ev_t1));
      uint64_t slots = 0;
      for (auto &s : c.segs) slots += s.n;
      if (timed_fwd) {
        st.fwd_kernel_ms += ms;
        st.fwd_kernel_calls += 1;
        st.fwd_kernel_slots += slots;
      } else {
        st.rev_kernel_ms += ms;
        st.rev_kernel_calls += 1;
        st.rev_kernel_slots += slots;
      }
    }
    return CGCM_OK;
  }

  // scratch sized for n slots and the unit lists
  int prepare(uint64_t nslots_total) {
    (void)nslots_total;
    CKS(dalloc(status, sizeof(Status) * 8 + 256));
    CKS(dalloc(lc, 64));
    int cap = list_capacity();
    CKS(dalloc(act_list, 4 * (size_t)cap + 64));
    CKS(dalloc(free_list, 4 * (size_t)cap + 64));
    CKS(dalloc(copy_list, 4 * (size_t)cap + 64));
    CKS(dalloc(journal, sizeof(Journal) * (size_t)cap + 64));
    CK(cudaMemsetAsync(status.as<void>(), 0, sizeof(Status) * 8, main));
    CK(cudaMemsetAsync(lc.as<void>(), 0, 64, main));
    CKS(h_status.ensure(sizeof(Status) * 8 + 64));
    return CGCM_OK;
  }
  // fetch the 8 Status blocks + list counters (synchronizes main)
  // Small calls: the status fetch also brings back the head of the unit lists (activation, free, copy-back;
  // LIST_HEAD entries each), so sorting a short list needs neither a device sort nor a second host wait
  // (sorted_units).  Valid until the next slot launch.
  static constexpr size_t LIST_HEAD = 512;
  HostBuf h_lists;
  bool lists_fresh = false, launches_small = true;
  uint64_t list_addr[3] = {0, 0, 0};
  int fetch_status(Status out[8], unsigned long long lcs[4]) {
    Trace trace_("fetch_status(sync)");
    // a kernel writes them into mapped pinned memory: no DMA to queue behind other copies (cgcm_dev.h)
    launch_copy_small(h_status.p, status.as<void>(), sizeof(Status) * 8, h_status.as<char>() + sizeof(Status) * 8,
                      lc.as<void>(), 32, main);
    st.kernel_launches += 1;
    lists_fresh = false;
    if (launches_small && act_list.addr && free_list.addr && copy_list.addr) {
      const size_t m = std::min<size_t>(LIST_HEAD, (size_t)list_capacity());
      CKS(h_lists.ensure(3 * 4 * LIST_HEAD + 64));
      launch_copy_small(h_lists.p, act_list.as<void>(), 4 * m, h_lists.as<char>() + 4 * LIST_HEAD,
                        free_list.as<void>(), 4 * m, main);
      launch_copy_small(h_lists.as<char>() + 8 * LIST_HEAD, copy_list.as<void>(), 4 * m, nullptr, nullptr, 0, main);
      st.kernel_launches += 2;
      list_addr[0] = act_list.addr;
      list_addr[1] = free_list.addr;
      list_addr[2] = copy_list.addr;
      lists_fresh = true;
    }
    launches_small = true;
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(main));
    std::memcpy(out, h_status.p, sizeof(Status) * 8);
    std::memcpy(lcs, h_status.as<char>() + sizeof(Status) * 8, 32);
    return CGCM_OK;
  }

  template <class T>
  int download(std::vector<T> &out, const DevBuf &src, size_t n) {
    out.resize(n);
    if (!n) return CGCM_OK;
    CKS(h_list.ensure(sizeof(T) * n));
    if (sizeof(T) * n <= (64u << 10)) {  // small: by a kernel into mapped pinned memory (no DMA queueing)
      launch_copy_small(h_list.p, src.as<void>(), sizeof(T) * n, nullptr, nullptr, 0, main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
    } else {
      CK(cudaMemcpyAsync(h_list.p, src.as<void>(), sizeof(T) * n, cudaMemcpyDeviceToHost, main));
    }
    CK(cudaStreamSynchronize(main));
    std::memcpy(out.data(), h_list.p, sizeof(T) * n);
    return CGCM_OK;
  }
  // n <= RING_HALF bytes from pageable host memory to dst, stream-ordered on main, no host wait
  int ring_init() {
    if (h_ring.p) return CGCM_OK;
    CKS(h_ring.ensure(2 * RING_HALF));
    for (auto &e : ev_ring) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    return CGCM_OK;
  }
  int ring_put(void *dst, const void *src, size_t n) {
    CKS(ring_init());
    if (ring_head + n > RING_HALF) {
      CK(cudaEventRecord(ev_ring[ring_cur], main));
      ring_used[ring_cur] = true;
      ring_cur ^= 1;
      ring_head = 0;
      if (ring_used[ring_cur]) CK(cudaEventSynchronize(ev_ring[ring_cur]));
    }
    char *p = h_ring.as<char>() + (size_t)ring_cur * RING_HALF + ring_head;
    std::memcpy(p, src, n);
    ring_head += (n + 255) & ~(size_t)255;
    // read by a kernel from mapped pinned memory: no DMA to queue behind other H2D copies
    launch_copy_small(dst, p, n, nullptr, nullptr, 0, main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    return CGCM_OK;
  }
  // memo: dst is an input-only buffer (no kernel writes it), so an upload of the bytes it already holds
  // can be skipped (ring_put_memo)
  template <class T>
  int upload(DevBuf &dst, const std::vector<T> &v, bool memo = false) {
    CKS(dalloc(dst, sizeof(T) * v.size() + 64));
    if (v.empty()) return CGCM_OK;
    if (sizeof(T) * v.size() <= RING_HALF)
      return memo ? ring_put_memo(dst.as<void>(), v.data(), sizeof(T) * v.size())
                  : ring_put(dst.as<void>(), v.data(), sizeof(T) * v.size());
    memo_forget(dst.addr, dst.bytes);
    CKS(h_small.ensure(sizeof(T) * v.size()));
    CK(cudaStreamSynchronize(main));
    std::memcpy(h_small.p, v.data(), sizeof(T) * v.size());
    CK(cudaMemcpyAsync(dst.as<void>(), h_small.p, sizeof(T) * v.size(), cudaMemcpyHostToDevice, main));
    CK(cudaStreamSynchronize(main));
    return CGCM_OK;
  }
  int unit_ops(const std::vector<UnitOp> &ops) {
    if (ops.empty()) return CGCM_OK;
    for (auto &o : ops)
      if ((o.op == UOP_ADD_RC && (int64_t)o.val < 0) || o.op == UOP_SET_RC) lease_break();
    CKS(dalloc(uops, sizeof(UnitOp) * ops.size() + 64));
    if (sizeof(UnitOp) * ops.size() <= RING_HALF) {
      CKS(ring_put_memo(uops.as<void>(), ops.data(), sizeof(UnitOp) * ops.size()));
    } else {
      memo_forget(uops.addr, uops.bytes);
      CKS(upload(uops, ops));
    }
    // the compact unit words need rewriting only if an op changes ACTIVE or STORAGE (cgcm_dev.h make_hotc)
    bool hotc = false;
    for (auto &o : ops)
      hotc = hotc || (o.op == UOP_OR_FLAGS && (o.val & (UF_ACTIVE | UF_STORAGE))) ||
             (o.op == UOP_AND_FLAGS && (~o.val & (UF_ACTIVE | UF_STORAGE)));
    launch_unit_ops(uops.as<UnitOp>(), (int)ops.size(), tab(), main, hotc);
    st.kernel_launches += hotc ? 2 : 1;
    pd_state_dirty = pd_state_dirty || hotc;
    CK(cudaGetLastError());
    return CGCM_OK;
  }

  // sorted unique unit list from a device list of n entries
  int sorted_units(const DevBuf &src, size_t n, std::vector<uint32_t> &out) {
    Trace trace_("sorted_units");
    out.clear();
    if (!n) return CGCM_OK;
    if (lists_fresh && n <= std::min<size_t>(LIST_HEAD, (size_t)list_capacity()))
      for (int l = 0; l < 3; ++l)
        if (src.addr == list_addr[l]) {  // the head fetched with the status (fetch_status)
          const uint32_t *h = reinterpret_cast<const uint32_t *>(h_lists.as<char>() + 4 * LIST_HEAD * l);
          out.assign(h, h + n);
          std::sort(out.begin(), out.end());
          return CGCM_OK;
        }
    if (n > 1) {
      size_t tb = sort_keys_temp_bytes((int)n);
      CKS(dalloc(temp, tb + 256 + 4 * n + 64));
      uint32_t *sorted = reinterpret_cast<uint32_t *>(temp.addr + align_up(tb, 256));
      launch_sort_keys(temp.as<void>(), tb, src.as<uint32_t>(), sorted, (int)n, main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
      DevBuf view;
      view.addr = reinterpret_cast<uint64_t>(sorted);
      view.bytes = 4 * n;
      CKS(download(out, view, n));
    } else {
      CKS(download(out, src, n));
    }
    return CGCM_OK;
  }

  // ------------------------------------------------------------------------------------------
  // activation (refcount 0 -> 1 transitions collected by the map kernel): allocate device storage
  // with host-adjacent units mirrored into one extent, write devbase (+ epoch, A5 R1), and copy
  // the units host -> device as coalesced runs on the copy stream (transfer scheduler).
  // Activation (refcount 0 -> 1, collected by the map kernel): device storage + devbase (+ epoch,
  // A5 R1) + the host -> device copies (the transfer scheduler).  Index-consecutive units whose host
  // gaps are small go into one extent that MIRRORS the host span [h0, h1) (devptr == base mod 256,
  // host gaps kept as device gaps, so copies are device-adjacent iff host-adjacent, A7) and the extent
  // has >= 1 byte of slack at its end.  One delta (host - device) per extent is what the reverse
  // index stores.  A host-contiguous extent of >= 256 KiB is one direct DMA; any other extent is
  // gathered on the host into pinned staging (multithreaded) and sent as one DMA.
  std::vector<cudaEvent_t> evpool;  // per-copy-group events (transfer overlap)
  int pool_event(size_t i, cudaEvent_t &e) {
    while (evpool.size() <= i) {
      cudaEvent_t x;
      CK(cudaEventCreateWithFlags(&x, cudaEventDisableTiming));
      evpool.push_back(x);
    }
    e = evpool[i];
    return CGCM_OK;
  }
  // ---- NEXT-3: coherence-group peers as copy sources ------------------------------------------
  struct PeerSrc {
    Context *ctx = nullptr;  // null: the host
    uint64_t src = 0;        // the peer's device copy
  };
  int peer_sources(const std::vector<uint32_t> &units, std::vector<PeerSrc> &out);
  int copy_in_with_peers(const std::vector<uint32_t> &units, const std::vector<PeerSrc> &peer, uint64_t bytes);
  cudaEvent_t ev_peer = nullptr;
  DevBuf peer_idx, peer_state;

  // pack_ev (optional): one event per pack (h2d_out entry), recorded on the copy stream after its copy;
  // the main stream then does NOT wait for the copies -- the caller waits per pack (transfer overlap)
  int activate_units(const std::vector<uint32_t> &units, std::vector<std::pair<uint64_t, uint64_t>> *h2d_out,
                     std::vector<cudaEvent_t> *pack_ev = nullptr, bool allow_peer = false) {
    Trace trace_("activate_units");  // (mirrors: globals never take the planned path; the rest are written here)
    if (units.empty()) return CGCM_OK;
    const uint64_t PACK_SPAN = 64ull << 20, GAPMAX = 64ull << 10, PACK_MIN = 256ull << 10;
    struct Pack {
      size_t i, j;
      uint64_t h0, h1;
      bool global, gaps;
      int64_t run;
      uint64_t dev0;
    };
    std::vector<Pack> packs;
    uint64_t bytes = 0;
    auto tr_packs = std::make_unique<Trace>("  act:packs");
    for (size_t i = 0; i < units.size(); ++i) {
      uint64_t b = ubase[units[i]], sz = usize[units[i]];
      bytes += sz;
      bool g = (uflags[units[i]] & UF_GLOBAL) != 0;
      if (!g && !packs.empty() && !packs.back().global && b >= packs.back().h1 && b - packs.back().h1 <= GAPMAX &&
          b + sz - packs.back().h0 <= PACK_SPAN) {
        Pack &P = packs.back();
        P.gaps = P.gaps || b != P.h1;
        P.h1 = b + sz;
        P.j = i + 1;
      } else {
        packs.push_back({i, i + 1, b, b + sz, g, false, -1, 0});
      }
    }
    tr_packs.reset();
    auto tr_alloc = std::make_unique<Trace>("  act:alloc+mirrors");
    std::vector<uint64_t> devbases(units.size());
    std::vector<int64_t> created;
    for (auto &P : packs) {
      uint32_t x0 = units[P.i];
      if (P.global && urun[x0] >= 0) {  // named region allocated on an earlier activation (A14)
        P.dev0 = udev[x0];
        P.run = urun[x0];
        devbases[P.i] = udev[x0];
        continue;
      }
      if (P.global && usym[x0]) {  // bound to a __device__ symbol: its storage is the symbol (NEXT-4)
        P.dev0 = usym[x0];
        P.run = new_run(P.dev0, P.h1 - P.h0, P.h0 - P.dev0);
        runs[P.run].external = true;
        udev[x0] = P.dev0;
        urun[x0] = P.run;
        devbases[P.i] = P.dev0;
        runs[P.run].live += 1;
        continue;
      }
      uint64_t need = (P.h0 % 256) + (P.h1 - P.h0) + 1;
      uint64_t a = arena.alloc(need);
      if (!a) {
        for (int64_t r : created) drop_run(r);
        for (auto &Q : packs)
          for (size_t q = Q.i; q < Q.j && Q.run >= 0; ++q) {
            uint32_t x = units[q];
            if (std::find(created.begin(), created.end(), urun[x]) != created.end()) {
              urun[x] = -1;
              udev[x] = 0;
            }
          }
        return CGCM_E_NOMEM;
      }
      P.dev0 = a + (P.h0 % 256);
      P.run = new_run(a, need, P.h0 - P.dev0);
      created.push_back(P.run);
      for (size_t q = P.i; q < P.j; ++q) {
        uint32_t x = units[q];
        udev[x] = P.dev0 + (ubase[x] - P.h0);
        urun[x] = P.run;
        devbases[q] = udev[x];
      }
      runs[P.run].live += (int64_t)(P.j - P.i);
    }
    tr_alloc.reset();
    auto tr_up = std::make_unique<Trace>("  act:exts+upload+set_ext");
    std::vector<uint32_t> exts(units.size());
    for (size_t q = 0; q < units.size(); ++q) exts[q] = (uint32_t)urun[units[q]];
    if (runs.size() > EXT_MASK) return CGCM_E_NOMEM;  // 2^24 live extents
    CKS(sync_ext());
    CKS(upload(up_units, units, true));
    CKS(upload(up_exts, exts, true));
    launch_set_ext(up_units.as<uint32_t>(), up_exts.as<uint32_t>(), (int)units.size(), tab(), rel_epoch(epoch),
                   (flags & CGCM_LITERAL_EPOCH) ? 0 : 1, main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    tr_up.reset();
    Trace tr_copy("  act:copies");
    CK(cudaEventRecord(ev_copy, main));  // the copies wait for everything the main stream did before
    CK(cudaStreamWaitEvent(copy, ev_copy, 0));
    // NEXT-3 (A31): units a group peer holds active and dirty are copied from its device copy
    std::vector<PeerSrc> peer;
    if (allow_peer && group) CKS(peer_sources(units, peer));
    if (!peer.empty()) return copy_in_with_peers(units, peer, bytes);
    auto mark = [&]() -> int {
      if (!pack_ev) return CGCM_OK;
      cudaEvent_t e;
      CKS(pool_event(pack_ev->size(), e));
      CK(cudaEventRecord(e, copy));
      pack_ev->push_back(e);
      return CGCM_OK;
    };
    for (auto &P : packs) {
      uint64_t span = P.h1 - P.h0;
      if (P.global || (!P.gaps && span >= PACK_MIN)) {
        CKS(copy_run(P.dev0, P.h0, span, true, units, P.i, P.j, copy));
        if (h2d_out) h2d_out->push_back({P.dev0, span});
        CKS(mark());
        continue;
      }
      int k = pack_k;
      pack_k ^= 1;
      CK(cudaEventSynchronize(ev_pack[k]));  // this staging buffer's previous DMA is done
      CKS(h_pack[k].ensure(span));
      char *stg = h_pack[k].as<char>();
      gather(units, P.i, P.j, P.h0, stg);
      CK(cudaMemcpyAsync(reinterpret_cast<void *>(P.dev0), stg, span, cudaMemcpyHostToDevice, copy));
      CK(cudaEventRecord(ev_pack[k], copy));
      st.h2d_memcpy_calls += 1;
      if (h2d_out) h2d_out->push_back({P.dev0, span});
      CKS(mark());
    }
    CK(cudaEventRecord(ev_copy, copy));
    if (!pack_ev) CK(cudaStreamWaitEvent(main, ev_copy, 0));
    st.h2d_units += units.size();
    st.h2d_bytes += bytes;
    st.activations += units.size();
    rev_dirty = true;
    pd_state_dirty = true;
    return CGCM_OK;
  }
  // ---- A9 re-map without a host wait -------------------------------------------------------------
  // Counters of passes whose status nobody waits for accumulate on the device and are folded into the
  // host statistics when they are read (cgcm_stats) or at the next full call.
  DevBuf lazy_status;
  bool lazy_pending = false;
  int fold_lazy() {
    if (!lazy_pending) return CGCM_OK;
    std::vector<Status> v;
    CKS(download(v, lazy_status, 1));
    st.fwd_translations += v[0].hits;
    st.null_slots += v[0].nulls;
    if (flags & CGCM_LENIENT) st.passthrough += v[0].misses;
    CK(cudaMemsetAsync(lazy_status.as<void>(), 0, sizeof(Status), main));
    lazy_pending = false;
    return CGCM_OK;
  }
  // mapArrays whose outers are ALL array-mapped (host mirrors, fresh) with no device storage released
  // since each was last translated from its host slots (A30): its elements are held by its own slot
  // references, so the re-map is refcounts only -- +mult per non-null slot through the reverse index
  // and +mult on the outer -- and cannot fail for a legal program (R13-ii: GPU functions do not store
  // pointers).  Both kernels are queued without a host wait.  Returns 1 when another path must run.
  // Leases: references the asynchronous re-maps above added to an outer and its elements (unit -> (dec_gen,
  // count)).  While no other call has released a reference since (dec_gen unchanged; a table rebuild clears
  // them), the units hold those references on top of the array mapping's own, so a releaseArray of the outer
  // that consumes a lease cannot bring any of them to 0 or below (Alg. 3 frees nothing, no underflow):
  // release_arrays_async queues its decrements without a host wait.
  std::unordered_map<uint32_t, std::pair<uint64_t, uint64_t>> leases;
  uint64_t dec_gen = 1;
  bool lease_quiet = false;  // set while release_arrays_async issues its own decrements
  void lease_break() {
    if (!lease_quiet) ++dec_gen;
  }
  int release_arrays_async(const uint64_t *ptrs, size_t k) {
    if (table_dirty || mirror_stale || k > 64 || (flags & CGCM_LENIENT) || leases.empty()) return 1;
    std::vector<std::pair<uint32_t, uint64_t>> outs;  // unit, mult
    for (size_t j = 0; j < k; ++j) {
      auto it = reg.upper_bound(ptrs[j]);
      if (it == reg.begin()) return 1;
      --it;
      const HostUnit &u = it->second;
      if (u.idx < 0 || ptrs[j] - it->first > u.size) return 1;
      const uint32_t x = (uint32_t)u.idx;
      if (!uarr[x] || !udev[x]) return 1;
      size_t q = 0;
      while (q < outs.size() && outs[q].first != x) ++q;
      if (q == outs.size()) outs.push_back({x, 0});
      outs[q].second += 1;
    }
    for (auto &o : outs) {
      auto l = leases.find(o.first);
      if (l == leases.end() || l->second.first != dec_gen || l->second.second < o.second) return 1;
    }
    for (auto &o : outs) {
      auto l = leases.find(o.first);
      if ((l->second.second -= o.second) == 0) leases.erase(l);
    }
    std::vector<UnitOp> ops;
    std::vector<Seg> rsegs;
    for (auto &o : outs) {
      ops.push_back({o.first, UOP_ADD_RC, (uint64_t)(-(int64_t)o.second)});
      const uint64_t n = usize[o.first] / 8;
      if (n) rsegs.push_back(Seg{udev[o.first], n, 0, (int32_t)o.second, 0});
    }
    // one outer with slots: its own decrement rides with the slot pass (SlotArgs::rc_delta)
    const bool fold = outs.size() == 1 && rsegs.size() == 1;
    lease_quiet = true;
    int r = ensure_rev();
    if (r == CGCM_OK && !fold) r = unit_ops(ops);
    if (r == CGCM_OK && !rsegs.empty()) {
      r = prepare_small(false);
      SlotCall R;
      R.dir = DIR_REV;
      R.ops = OP_DEC;
      R.segs = rsegs;
      if (fold) {
        R.rc_unit = outs[0].first;
        R.rc_delta = -(int32_t)outs[0].second;
      }
      if (r == CGCM_OK) r = launch(R, 2);
    }
    lease_quiet = false;
    if (r != CGCM_OK) lease_break();
    return r;
  }
  int remap_arrays_async(const uint64_t *ptrs, size_t k, void ***gpu_out) {
    // (lenient mode: a stray word in the device slots could fall inside another unit's device copy, A18)
    if (table_dirty || mirror_stale || k > 64 || (flags & CGCM_LENIENT)) return 1;
    std::vector<std::pair<uint32_t, int>> outs;  // unit, mult
    std::vector<uint32_t> which(k);
    for (size_t j = 0; j < k; ++j) {
      auto it = reg.upper_bound(ptrs[j]);
      if (it == reg.begin()) return 1;
      --it;
      const HostUnit &u = it->second;
      if (u.idx < 0 || ptrs[j] - it->first > u.size) return 1;
      const uint32_t x = (uint32_t)u.idx;
      if (!uarr[x] || !udev[x]) return 1;
      auto g = arr_gen.find(ubase[x]);
      if (g == arr_gen.end() || g->second != free_gen) return 1;
      size_t q = 0;
      while (q < outs.size() && outs[q].first != x) ++q;
      if (q == outs.size()) outs.push_back({x, 0});
      outs[q].second += 1;
      which[j] = (uint32_t)q;
    }
    Trace trace_q("remap_async:queue");
    std::vector<UnitOp> ops;
    std::vector<Seg> rsegs;
    for (auto &o : outs) {
      ops.push_back({o.first, UOP_ADD_RC, (uint64_t)(int64_t)o.second});
      const uint64_t n = usize[o.first] / 8;
      if (n) rsegs.push_back(Seg{udev[o.first], n, 0, o.second, 0});
    }
    // one outer with slots: its own increment rides with the slot pass (SlotArgs::rc_delta)
    const bool fold = outs.size() == 1 && rsegs.size() == 1;
    {
      Trace t1("remap_async:unit_ops");
      CKS(ensure_rev());
      if (!fold) CKS(unit_ops(ops));
    }
    if (!rsegs.empty()) {
      Trace t2("remap_async:launch");
      CKS(dalloc(lazy_status, sizeof(Status) + 256));
      if (!lazy_pending) CK(cudaMemsetAsync(lazy_status.as<void>(), 0, sizeof(Status), main));
      CKS(prepare_small(false));
      SlotCall R;
      R.dir = DIR_REV;
      R.ops = OP_INCPLAIN;
      R.segs = rsegs;
      R.lazy = true;
      if (fold) {
        R.rc_unit = outs[0].first;
        R.rc_delta = (int32_t)outs[0].second;
      }
      CKS(launch(R, 0));
      lazy_pending = true;
    }
    for (size_t j = 0; j < k; ++j) {
      const uint32_t x = outs[which[j]].first;
      gpu_out[j] = reinterpret_cast<void **>(udev[x] + (ptrs[j] - ubase[x]));
    }
    for (auto &o : outs) {
      auto &l = leases[o.first];
      if (l.first != dec_gen) l = {dec_gen, 0};
      l.second += (uint64_t)o.second;
    }
    return CGCM_OK;
  }

  // ---- device-side transfer planning -----------------------------------------------------------
  int need_mirrors() {
    if (!mirror_stale) return CGCM_OK;
    Trace trace_("need_mirrors(sync)");
    std::vector<uint64_t> hots;
    CKS(download(hots, hotb, (size_t)U));
    for (int x = 0; x < U; ++x) {
      const uint32_t fl = hot_flags(hots[x]);
      const uint32_t e = hot_ext(hots[x]);
      if ((fl & UF_STORAGE) && e < runs.size()) {
        urun[x] = (int64_t)e;
        udev[x] = ubase[x] - runs[e].delta;
      } else {
        urun[x] = -1;
        udev[x] = 0;
      }
      uarr[x] = (fl & UF_ARRAYMAPPED) ? 1 : 0;
    }
    mirror_stale = false;
    return CGCM_OK;
  }
  // refresh the mirrors of just these units (their state words: extent + flags) -- O(|xs|)
  DevBuf mir_idx, mir_out;
  int mirror_units(const std::vector<uint32_t> &xs) {
    if (!mirror_stale || xs.empty()) return CGCM_OK;
    CKS(upload(mir_idx, xs));
    CKS(dalloc(mir_out, 8 * xs.size() + 64));
    launch_gather_state(tab(), mir_idx.as<uint32_t>(), (int)xs.size(), mir_out.as<uint64_t>(), main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    std::vector<uint64_t> w;
    CKS(download(w, mir_out, xs.size()));
    for (size_t q = 0; q < xs.size(); ++q) {
      const uint32_t x = xs[q], fl = hot_flags(w[q]), e = hot_ext(w[q]);
      if ((fl & UF_STORAGE) && e < runs.size()) {
        urun[x] = (int64_t)e;
        udev[x] = ubase[x] - runs[e].delta;
      } else {
        urun[x] = -1;
        udev[x] = 0;
      }
      uarr[x] = (fl & UF_ARRAYMAPPED) ? 1 : 0;
    }
    return CGCM_OK;
  }
  // host memory the driver has pinned (cudaHostAlloc / cudaHostRegister): a DMA may read it directly
  static bool host_pinned(uint64_t h) {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, reinterpret_cast<const void *>(h)) != cudaSuccess) {
      (void)cudaGetLastError();
      return false;
    }
    return at.type == cudaMemoryTypeHost;
  }
  // sort the n unit ids of a device list into plan_S (and size the planning scratch)
  int plan_sort(const DevBuf &list, size_t n) {
    plan_tb = std::max(sort_keys_temp_bytes((int)n), plan_temp_bytes((int)n)) + 256;
    CKS(dalloc(plan_tmp, plan_tb));
    for (DevBuf *b : {&plan_S, &plan_F, &plan_G, &plan_pid, &plan_gscan}) CKS(dalloc(*b, 4 * n + 64));
    CKS(dalloc(plan_cnt, 64));
    launch_sort_keys(plan_tmp.as<void>(), plan_tb, list.as<uint32_t>(), plan_S.as<uint32_t>(), (int)n, main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    return CGCM_OK;
  }
  // the sorted ids [first, last] of plan_S on the host (fallback paths of one pack / run)
  int plan_slice(uint32_t first, uint32_t last, std::vector<uint32_t> &out) {
    DevBuf v;
    v.addr = plan_S.addr + 4ull * first;
    v.bytes = 4ull * (last - first + 1);
    return download(out, v, last - first + 1);
  }
  // Activation of n units (a device list) planned on the device: packs of host-adjacent units, one
  // mirrored extent each, device addresses and extent ids written by a kernel; the host handles one
  // descriptor per pack (allocation + one DMA).  Globals take the host path.
  int activate_planned(const DevBuf &list, size_t n) {
    Trace trace_("activate(planned)");
    const uint64_t GAPMAX = 64ull << 10;
    auto tr1 = std::make_unique<Trace>("  plan:sort+scan+download");
    CKS(plan_sort(list, n));
    int r = launch_plan_packs1(plan_S.as<uint32_t>(), (int)n, tab(), GAPMAX, 26, plan_F.as<uint32_t>(),
                               plan_G.as<uint32_t>(), plan_pid.as<uint32_t>(), plan_gscan.as<uint32_t>(),
                               plan_cnt.as<unsigned long long>(), plan_tmp.as<void>(), plan_tb, main);
    st.kernel_launches += 4;
    if (r) return CGCM_E_CUDA;
    std::vector<unsigned long long> cnt;
    CKS(download(cnt, plan_cnt, 4));
    const size_t np = (size_t)(cnt[0] & 0xFFFFFFFFull);
    const uint64_t bytes = cnt[2];
    if (cnt[1]) {  // globals keep their named regions (A14): the host path
      std::vector<uint32_t> units;
      CKS(plan_slice(0, (uint32_t)n - 1, units));
      return activate_units(units, nullptr, nullptr, true);
    }
    CKS(dalloc(plan_desc, sizeof(PackDesc) * np + 64));
    if (launch_plan_packs2(plan_S.as<uint32_t>(), (int)n, tab(), plan_F.as<uint32_t>(), plan_pid.as<uint32_t>(),
                           plan_gscan.as<uint32_t>(), plan_desc.as<PackDesc>(), main))
      return CGCM_E_CUDA;
    st.kernel_launches += 2;
    std::vector<PackDesc> packs;
    CKS(download(packs, plan_desc, np));
    tr1.reset();
    auto tr2 = std::make_unique<Trace>("  plan:alloc+set_ext");
    // device extents, all or nothing
    std::vector<int64_t> created;
    std::vector<uint32_t> rid(np);
    std::vector<uint64_t> dev0(np);
    for (size_t p = 0; p < np; ++p) {
      const PackDesc &P = packs[p];
      const uint64_t need = (P.h0 % 256) + (P.h1 - P.h0) + 1;  // >= 1 byte of slack (A7)
      const uint64_t a = arena.alloc(need);
      if (!a) {
        for (int64_t x : created) drop_run(x);
        return CGCM_E_NOMEM;
      }
      dev0[p] = a + (P.h0 % 256);  // devptr == base (mod 256)
      const int64_t run = new_run(a, need, P.h0 - dev0[p]);
      runs[run].live = (int64_t)(P.last - P.first + 1);
      created.push_back(run);
      rid[p] = (uint32_t)run;
    }
    if (runs.size() > EXT_MASK) {
      for (int64_t x : created) drop_run(x);
      return CGCM_E_NOMEM;
    }
    CKS(sync_ext());
    CKS(upload(plan_run, rid));
    launch_plan_set_ext(plan_S.as<uint32_t>(), (int)n, plan_pid.as<uint32_t>(), plan_run.as<uint32_t>(), tab(),
                        rel_epoch(epoch), (flags & CGCM_LITERAL_EPOCH) ? 0 : 1, main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    tr2.reset();
    Trace tr3("  plan:copies(issue)");
    CK(cudaEventRecord(ev_copy, main));
    CK(cudaStreamWaitEvent(copy, ev_copy, 0));
    for (size_t p = 0; p < np; ++p) {  // the transfer scheduler: one DMA per pack
      const PackDesc &P = packs[p];
      const uint64_t span = P.h1 - P.h0;
      // a pack with host gaps in pinned memory: one DMA of the whole span (the gap bytes land in the
      // extent's mirrored gaps, which belong to no unit); pageable memory is gathered unit by unit
      // (its gap pages may not even be mapped)
      if (!P.gaps || (host_pinned(P.h0) && host_pinned(P.h1 - 1))) {  // (a span across two pinned
        // allocations is rejected by cudaMemcpyAsync, then gathered below)
        cudaError_t e = cudaMemcpyAsync(reinterpret_cast<void *>(dev0[p]), reinterpret_cast<const void *>(P.h0), span,
                                        cudaMemcpyHostToDevice, copy);
        if (e == cudaSuccess) {
          st.h2d_memcpy_calls += 1;
          continue;
        }
        (void)cudaGetLastError();  // e.g. a span across two host allocations: unit by unit below
      }
      std::vector<uint32_t> units;
      CKS(plan_slice(P.first, P.last, units));
      if (!P.gaps) {
        CKS(copy_run(dev0[p], P.h0, span, true, units, 0, units.size(), copy));
        continue;
      }
      int k = pack_k;
      pack_k ^= 1;
      CK(cudaEventSynchronize(ev_pack[k]));
      CKS(h_pack[k].ensure(span));
      gather(units, 0, units.size(), P.h0, h_pack[k].as<char>());
      CK(cudaMemcpyAsync(reinterpret_cast<void *>(dev0[p]), h_pack[k].p, span, cudaMemcpyHostToDevice, copy));
      CK(cudaEventRecord(ev_pack[k], copy));
      st.h2d_memcpy_calls += 1;
    }
    CK(cudaEventRecord(ev_copy, copy));
    CK(cudaStreamWaitEvent(main, ev_copy, 0));
    st.h2d_units += n;
    st.h2d_bytes += bytes;
    st.activations += n;
    rev_dirty = true;
    pd_state_dirty = true;
    mirror_stale = true;
    return CGCM_OK;
  }
  // Frees (Alg. 3) of the n units of a device list (+ extra host-listed units): for long lists planned on
  // the device -- per extent the number of copies it loses, the array-mapped units listed -- so the host
  // does O(#extents + #array-mapped) work.  Device-array shadows inside freed copies need the host path.
  DevBuf free_dec, free_arr;
  int free_units_list(const DevBuf &list, size_t n, const std::vector<uint32_t> &extra = {}) {
    if (n + extra.size() == 0) return CGCM_OK;
    if (n + extra.size() < PLAN_MIN || dev_shadows) {
      std::vector<uint32_t> f;
      CKS(download(f, list, n));
      f.insert(f.end(), extra.begin(), extra.end());
      std::sort(f.begin(), f.end());
      f.erase(std::unique(f.begin(), f.end()), f.end());
      return free_units(f);
    }
    Trace trace_("free_units(planned)");
    const size_t m = n + extra.size();
    // the list (+ extras) sorted into plan_S: duplicates adjacent
    CKS(dalloc(plan_S, 4 * m + 64));
    DevBuf tmpl;
    const DevBuf *src = &list;
    if (!extra.empty()) {  // append the extras behind a copy of the list
      CKS(dalloc(plan_G, 4 * m + 64));
      CK(cudaMemcpyAsync(plan_G.as<void>(), list.as<void>(), 4 * n, cudaMemcpyDeviceToDevice, main));
      CK(cudaMemcpyAsync(plan_G.as<uint32_t>() + n, extra.data(), 4 * extra.size(), cudaMemcpyHostToDevice, main));
      CK(cudaStreamSynchronize(main));  // (extra is pageable host memory)
      src = &plan_G;
    }
    CKS(plan_sort(*src, m));
    CKS(dalloc(free_dec, 4 * std::max<size_t>(runs.size(), 1) + 64));
    CKS(dalloc(free_arr, 8 * m + 64));
    launch_free_plan(plan_S.as<uint32_t>(), (int)m, tab(), free_dec.as<uint32_t>(), (int)runs.size(),
                     free_arr.as<uint32_t>(), plan_cnt.as<unsigned long long>(), main);
    launch_deactivate(plan_S.as<uint32_t>(), (int)m, tab(), main);
    st.kernel_launches += 2;
    CK(cudaGetLastError());
    std::vector<unsigned long long> cnt;
    CKS(download(cnt, plan_cnt, 4));
    std::vector<uint32_t> dec, arr;
    CKS(download(dec, free_dec, runs.size()));
    CKS(download(arr, free_arr, 2 * cnt[2]));
    for (size_t q = 0; q < cnt[2]; ++q) {  // array-mapped: their shadows go with their copies
      const uint32_t x = arr[2 * q], e = arr[2 * q + 1];
      arr_gen.erase(ubase[x]);
      if (e < runs.size()) drop_shadows(ubase[x] - runs[e].delta);
      else if (udev[x]) drop_shadows(udev[x]);  // a global: its named region stays
    }
    for (size_t r = 0; r < dec.size(); ++r) {
      if (!dec[r]) continue;
      free_gen += dec[r];
      runs[r].live -= (int64_t)dec[r];
      if (runs[r].live <= 0) drop_run((int64_t)r);
    }
    st.frees += cnt[0];
    rev_dirty = true;
    pd_state_dirty = true;
    mirror_stale = true;
    return CGCM_OK;
  }
  // Copy-back (Alg. 2's cuMemcpyDtoH) of the n units of a device list: plain units as one DMA per
  // host-adjacent mirrored run, array-mapped units reverse translated first (A12).  Planned on the
  // device for long lists.
  int copy_back_list(const DevBuf &list, size_t n) {
    if (n == 0) return CGCM_OK;
    if (n < PLAN_MIN) {
      std::vector<uint32_t> units;
      CKS(sorted_units(list, n, units));
      return copy_back(units);
    }
    Trace trace_("copy_back(planned)");
    CKS(plan_sort(list, n));
    if (launch_plan_copyback1(plan_S.as<uint32_t>(), (int)n, tab(), plan_F.as<uint32_t>(), plan_pid.as<uint32_t>(),
                              plan_cnt.as<unsigned long long>(), plan_tmp.as<void>(), plan_tb, main))
      return CGCM_E_CUDA;
    st.kernel_launches += 2;
    std::vector<unsigned long long> cnt;
    CKS(download(cnt, plan_cnt, 4));
    const size_t nr = (size_t)(cnt[0] & 0xFFFFFFFFull);
    CKS(dalloc(plan_desc, sizeof(CopyRun) * nr + 64));
    if (launch_plan_copyback2(plan_S.as<uint32_t>(), (int)n, tab(), plan_F.as<uint32_t>(), plan_pid.as<uint32_t>(),
                              plan_desc.as<CopyRun>(), main))
      return CGCM_E_CUDA;
    st.kernel_launches += 2;
    std::vector<CopyRun> rs;
    CKS(download(rs, plan_desc, nr));
    std::vector<std::pair<uint32_t, uint64_t>> arr;
    for (auto &R : rs)
      if (R.arr) arr.push_back({R.unit, R.dev});
    CKS(copy_back_arr(arr));  // validated before any plain byte moves
    for (auto &R : rs) {
      if (R.arr) continue;
      cudaError_t e = cudaMemcpyAsync(reinterpret_cast<void *>(R.host), reinterpret_cast<const void *>(R.dev), R.len,
                                      cudaMemcpyDeviceToHost, copy);
      if (e != cudaSuccess) {  // a run across two host allocations: unit by unit
        (void)cudaGetLastError();
        std::vector<uint32_t> units;
        CKS(plan_slice(R.first, R.last, units));
        for (uint32_t x : units)
          CK(cudaMemcpyAsync(reinterpret_cast<void *>(ubase[x]), reinterpret_cast<const void *>(R.dev + (ubase[x] - R.host)),
                             usize[x], cudaMemcpyDeviceToHost, copy));
        st.d2h_memcpy_calls += units.size();
      } else {
        st.d2h_memcpy_calls += 1;
      }
      st.d2h_units += R.last - R.first + 1;
      st.d2h_bytes += R.len;
    }
    CK(cudaStreamSynchronize(copy));
    return CGCM_OK;
  }

  // host gather of units [i, j) into staging at their mirrored offsets (base - h0)
  void gather(const std::vector<uint32_t> &units, size_t i, size_t j, uint64_t h0, char *stg) {
    size_t n = j - i;
    uint64_t total = 0;
    for (size_t q = i; q < j; ++q) total += usize[units[q]];
    unsigned T = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
    auto work = [&](size_t lo, size_t hi) {
      for (size_t q = lo; q < hi; ++q) {
        uint32_t x = units[q];
        std::memcpy(stg + (ubase[x] - h0), reinterpret_cast<const void *>(ubase[x]), usize[x]);
      }
    };
    if (total < (8ull << 20) || T == 1 || n < 64) {
      work(i, j);
      return;
    }
    std::vector<std::thread> th;
    for (unsigned t = 0; t < T; ++t) th.emplace_back(work, i + n * t / T, i + n * (t + 1) / T);
    for (auto &x : th) x.join();
  }

  // One host<->device copy of a host-contiguous run of units.  Host-adjacent units may live in two
  // different host allocations (cudaMemcpyAsync rejects a pinned range that crosses them): retry
  // unit by unit then.
  int copy_run(uint64_t dev, uint64_t host, uint64_t len, bool h2d, const std::vector<uint32_t> &units, size_t i,
               size_t j, cudaStream_t s) {
    cudaError_t e = h2d ? cudaMemcpyAsync(reinterpret_cast<void *>(dev), reinterpret_cast<const void *>(host), len,
                                          cudaMemcpyHostToDevice, s)
                        : cudaMemcpyAsync(reinterpret_cast<void *>(host), reinterpret_cast<const void *>(dev), len,
                                          cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) {
      (h2d ? st.h2d_memcpy_calls : st.d2h_memcpy_calls) += 1;
      return CGCM_OK;
    }
    if (e != cudaErrorInvalidValue || j - i < 2) {
      g_last_cuda_error = std::string("cudaMemcpyAsync (run): ") + cudaGetErrorString(e);
      return CGCM_E_CUDA;
    }
    (void)cudaGetLastError();
    for (size_t q = i; q < j; ++q) {
      uint64_t hb = ubase[units[q]], n = usize[units[q]], db = dev + (hb - host);
      if (h2d) CK(cudaMemcpyAsync(reinterpret_cast<void *>(db), reinterpret_cast<const void *>(hb), n,
                                  cudaMemcpyHostToDevice, s));
      else CK(cudaMemcpyAsync(reinterpret_cast<void *>(hb), reinterpret_cast<const void *>(db), n,
                              cudaMemcpyDeviceToHost, s));
      (h2d ? st.h2d_memcpy_calls : st.d2h_memcpy_calls) += 1;
    }
    return CGCM_OK;
  }

  // units whose refcount reached 0: free device storage (globals keep theirs), clear flags
  int free_units(const std::vector<uint32_t> &units) {
    if (!units.empty()) lease_break();
    Trace trace_("free_units");
    CKS(mirror_units(units));
    if (units.empty()) return CGCM_OK;
    CKS(upload(up_units, units, true));
    launch_deactivate(up_units.as<uint32_t>(), (int)units.size(), tab(), main);
    st.kernel_launches += 1;
    pd_state_dirty = true;
    CK(cudaGetLastError());
    CK(cudaStreamSynchronize(main));
    for (uint32_t x : units) {
      const bool was_arr = uarr[x] != 0;
      if (was_arr) arr_gen.erase(ubase[x]);  // no longer array-mapped: the next mapArray translates from host slots
      uarr[x] = 0;
      // an outer's shadows go with its copy (and a device array's, if one lived in this copy)
      if (udev[x] && (was_arr || dev_shadows)) drop_shadows(udev[x]);
      if (uflags[x] & UF_GLOBAL) continue;
      run_release(urun[x]);
      urun[x] = -1;
      udev[x] = 0;
      st.frees += 1;
    }
    rev_dirty = true;
    return CGCM_OK;
  }

  // copy-back of whole units device -> host (Alg. 2's cuMemcpyDtoH).  Array-mapped units are
  // reverse translated first (A12) -- validated before any byte moves.  Synchronous.
  // array-mapped units (unit, device copy): reverse translate their slots into staging (validated:
  // a reverse miss fails the call before any byte moves, A12), then copy slots + trailing bytes back
  int copy_back_arr(const std::vector<std::pair<uint32_t, uint64_t>> &arr) {
    if (arr.empty()) return CGCM_OK;
    uint64_t arr_bytes = 0;
    for (auto &a : arr) arr_bytes += align_up(usize[a.first] / 8 * 8, 32) + 32;
    CKS(ensure_rev());
    CKS(dalloc(staging_cb, arr_bytes + 256));
    SlotCall c;
    c.dir = DIR_REV;
    c.ops = OP_WRITE;
    uint64_t off = staging_cb.addr;
    std::vector<uint64_t> dst(arr.size());
    for (size_t q = 0; q < arr.size(); ++q) {
      const uint32_t x = arr[q].first;
      const uint64_t db = arr[q].second, n = usize[x] / 8;
      off = align_up(off, 32) + (db & 31);  // same alignment as the source
      dst[q] = off;
      Seg sg;
      sg.ptr = db;
      sg.n = n;
      sg.out = off;
      sg.inc = 0;
      sg.pad = 0;
      sg.shadow = 0;
      if (n) c.segs.push_back(sg);
      off += 8 * n;
    }
    CKS(prepare_small());
    CKS(launch(c, 7));
    Status sts[8];
    unsigned long long lcs[4];
    CKS(fetch_status(sts, lcs));
    if (sts[7].misses && !(flags & CGCM_LENIENT)) return CGCM_E_UNREGISTERED;
    st.rev_translations += sts[7].translated;
    st.passthrough += (flags & CGCM_LENIENT) ? sts[7].misses : 0;
    for (size_t q = 0; q < arr.size(); ++q) {
      const uint32_t x = arr[q].first;
      const uint64_t hb = ubase[x], sz = usize[x], db = arr[q].second, n = sz / 8;
      if (n) CK(cudaMemcpyAsync(reinterpret_cast<void *>(hb), reinterpret_cast<void *>(dst[q]), 8 * n,
                                cudaMemcpyDeviceToHost, copy));
      if (sz > 8 * n)
        CK(cudaMemcpyAsync(reinterpret_cast<void *>(hb + 8 * n), reinterpret_cast<void *>(db + 8 * n), sz - 8 * n,
                           cudaMemcpyDeviceToHost, copy));
      st.d2h_memcpy_calls += 1 + (sz > 8 * n);
      st.d2h_units += 1;
      st.d2h_bytes += sz;
    }
    return CGCM_OK;
  }
  int copy_back(const std::vector<uint32_t> &units) {
    Trace trace_("copy_back");
    if (units.empty()) return CGCM_OK;
    CKS(mirror_units(units));
    std::vector<uint32_t> plain;
    std::vector<std::pair<uint32_t, uint64_t>> arr;
    for (uint32_t x : units) {
      if (uarr[x]) arr.push_back({x, udev[x]});
      else plain.push_back(x);
    }
    CKS(copy_back_arr(arr));
    // plain units: coalesce host-adjacent units whose device copies are mirrored
    size_t i = 0;
    while (i < plain.size()) {
      uint32_t x0 = plain[i];
      uint64_t h0 = ubase[x0], d0 = udev[x0], hend = h0 + usize[x0];
      st.d2h_units += 1;
      st.d2h_bytes += usize[x0];
      size_t j = i + 1;
      while (j < plain.size() && plain[j] == plain[j - 1] + 1) {
        uint32_t x = plain[j];
        if (ubase[x] != hend || udev[x] != d0 + (ubase[x] - h0)) break;
        hend += usize[x];
        st.d2h_units += 1;
        st.d2h_bytes += usize[x];
        ++j;
      }
      CKS(copy_run(d0, h0, hend - h0, false, plain, i, j, copy));
      i = j;
    }
    CK(cudaStreamSynchronize(copy));
    return CGCM_OK;
  }
  // zero = false: for passes nobody fetches the status of (the queued re-map / release): every call that
  // reads a status block zeroes it first
  int prepare_small(bool zero = true) {
    CKS(dalloc(status, sizeof(Status) * 8 + 256));
    CKS(dalloc(lc, 64));
    if (zero) CK(cudaMemsetAsync(status.as<void>(), 0, sizeof(Status) * 8, main));
    CKS(h_status.ensure(sizeof(Status) * 8 + 64));
    int cap = list_capacity();
    CKS(dalloc(act_list, 4 * (size_t)cap + 64));
    CKS(dalloc(free_list, 4 * (size_t)cap + 64));
    CKS(dalloc(copy_list, 4 * (size_t)cap + 64));
    CKS(dalloc(journal, sizeof(Journal) * (size_t)cap + 64));
    return CGCM_OK;
  }

  // ------------------------------------------------------------------------------------------
  // forward map over device slot segments (in place or out of place): a1 + a2.
  // prelaunch: optional additional REV INCPLAIN segments (array-mapped outers re-mapped, A9).
  // On error everything this function did is undone; the caller undoes its own prologue.
  int map_core(const std::vector<Seg> &fsegs, const std::vector<Seg> &rsegs, uint64_t *translated_out,
               uint64_t *nulls_out, const std::vector<int> *seg_group = nullptr,
               const std::vector<cudaEvent_t> *group_ev = nullptr, bool defer = false) {
    Trace trace_("map_core");
    uint64_t total = 0;
    for (auto &s : fsegs) total += s.n;
    if (fsegs.empty() && rsegs.empty()) {  // nothing to translate (e.g. every outer was re-mapped, A9)
      if (translated_out) *translated_out = 0;
      if (nulls_out) *nulls_out = 0;
      return CGCM_OK;
    }
    CKS(prepare(total + 64));
    SlotCall F;
    F.dir = DIR_FWD;
    F.ops = OP_WRITE | OP_INC | OP_HITMASK;
    F.segs = fsegs;
    F.defer = defer && fsegs.size() == 1 && fsegs[0].shadow != 0;
    if (seg_group && group_ev) {
      F.seg_group = *seg_group;
      F.group_ev = *group_ev;
    }
    SlotCall R;
    R.dir = DIR_REV;
    R.ops = OP_INCPLAIN;
    R.segs = rsegs;
    if (!rsegs.empty()) CKS(ensure_rev());
    int lr = launch(F, 0, false, true, false);
    if (!F.seg_group.empty()) CK(cudaStreamWaitEvent(main, ev_copy, 0));  // every copy, whatever happened
    CKS(lr);
    // hitmask is per launch: the REV pass does not use it
    if (!rsegs.empty()) CKS(launch(R, 1));
    Status sts[8];
    unsigned long long lcs[4];
    CKS(fetch_status(sts, lcs));
    bool strict = !(flags & CGCM_LENIENT);
    // a failing call first turns the references it deferred into ordinary ones, which undo_map drops
    auto undo_deferred = [&]() -> int {
      if (F.defer) {
        launch_materialise(reinterpret_cast<const uint64_t *>(fsegs[0].shadow), fsegs[0].n,
                           rcb.as<int32_t>(), main);
        st.kernel_launches += 1;
        CK(cudaGetLastError());
      }
      return CGCM_OK;
    };
    if ((sts[0].misses || sts[1].misses) && strict) {
      CKS(undo_deferred());
      CKS(undo_map(F, R));
      return CGCM_E_UNREGISTERED;
    }
    // activations
    if (lcs[0] > 0) {
      int r;
      if (lcs[0] >= PLAN_MIN && !group) {  // planned on the device: one descriptor per pack
        r = activate_planned(act_list, lcs[0]);
      } else {
        std::vector<uint32_t> units;
        CKS(sorted_units(act_list, lcs[0], units));
        r = activate_units(units, nullptr, nullptr, true);
      }
      if (r != CGCM_OK) {
        CKS(undo_deferred());
        CKS(undo_map(F, R));
        return r;
      }
    }
    if (sts[0].pending > 0) {  // complete the slots whose unit was activated by this call
      SlotCall C;
      C.dir = DIR_FWD;
      C.ops = OP_WRITE;
      C.sel = SEL_NOTHIT;
      C.segs = fsegs;
      CKS(launch(C, 2));
    }
    CK(cudaStreamSynchronize(main));
    uint64_t tr = sts[0].hits + sts[1].hits;
    st.fwd_translations += tr;
    st.null_slots += sts[0].nulls + sts[1].nulls;
    if (!strict) st.passthrough += sts[0].misses + sts[1].misses;
    if (translated_out) *translated_out = tr;
    if (nulls_out) *nulls_out = sts[0].nulls + sts[1].nulls;
    return CGCM_OK;
  }
  // re-map of array-mapped outers (A9): +inc per non-null slot through the reverse index.  On a
  // reverse miss (an element lost its device copy: unbalanced release) the pass is undone and
  // E_UNREGISTERED returned so that the caller can re-translate those outers from host memory.
  int rev_addref(const std::vector<Seg> &rsegs, Status &res) {
    CKS(ensure_rev());
    CKS(prepare(64));
    SlotCall R;
    R.dir = DIR_REV;
    R.ops = OP_INCPLAIN;
    R.segs = rsegs;
    CKS(launch(R, 0));
    Status sts[8];
    unsigned long long lcs[4];
    CKS(fetch_status(sts, lcs));
    res = sts[0];
    // a reverse miss means an element lost its device copy (A25) -- or, in lenient mode, a slot that
    // passed through unregistered (A18): either way the caller re-translates from the host slots,
    // which is what a sequential mapArray does (the oracle's semantics), lenient or not
    if (sts[0].misses) {
      CKS(rev_decref(rsegs));
      return CGCM_E_UNREGISTERED;
    }
    return CGCM_OK;
  }
  int rev_decref(const std::vector<Seg> &rsegs) {
    CKS(prepare_small());
    SlotCall R;
    R.dir = DIR_REV;
    R.ops = OP_DECPLAIN;
    R.segs = rsegs;
    CKS(launch(R, 1));
    CK(cudaStreamSynchronize(main));
    return CGCM_OK;
  }
  int undo_map(SlotCall &F, SlotCall &R) {
    // forward maps are always in place: translated slots (hit bit set) hold GPU pointers again
    // turned back into CPU pointers (reverse lookup) and lose their reference; the other hits
    // (pending activations) only lose their reference.
    rev_dirty = true;  // refcounts changed: rebuild the reverse index over the current active set
    CKS(ensure_rev());
    CKS(prepare_small());
    SlotCall a;
    a.dir = DIR_REV;
    a.ops = OP_WRITE | OP_DECPLAIN;
    a.sel = SEL_HIT;
    a.segs = F.segs;  // same chunk numbering as the forward launch (hitmask)
    CKS(launch(a, 0));
    SlotCall b;
    b.dir = DIR_FWD;
    b.ops = OP_DECPLAIN;
    b.sel = SEL_NOTHIT;
    b.segs = F.segs;
    CKS(launch(b, 1));
    if (!R.segs.empty()) {
      SlotCall r;
      r.dir = DIR_REV;
      r.ops = OP_DECPLAIN;
      r.segs = R.segs;
      CKS(launch(r, 2));
    }
    CK(cudaStreamSynchronize(main));
    rev_dirty = true;
    return CGCM_OK;
  }

  // reverse unmap over device slot segments (GPU pointers): a3 + a4 (+ release)
  //   ops: OP_WRITE|OP_GATE|OP_HITMASK [|OP_DEC] or OP_GATE
  int unmap_rev_core(const std::vector<Seg> &segs, bool write, bool dec, std::vector<uint32_t> &copy_units,
                     std::vector<uint32_t> &freed, uint64_t &journal_count, Status &res, bool defer = false) {
    Trace trace_("unmap_rev_core");
    CKS(ensure_rev());
    uint64_t total = 0;
    for (auto &s : segs) total += s.n;
    CKS(prepare(total + 64));
    SlotCall c;
    c.dir = DIR_REV;
    c.ops = write ? (OP_WRITE | OP_GATE | OP_HITMASK | (dec ? OP_DEC : 0)) : (OP_GATE | (dec ? OP_DEC : 0));
    c.segs = segs;
    c.defer = defer;
    // large passes: snapshot the rc/epoch columns instead of journaling every gated unit; a pass over
    // deferred references always does (its rollback is: restore the snapshot, then materialise)
    c.no_journal = (total >= (uint64_t)U / 8 && U >= 4096) || defer;
    c.dec_red = dec && c.no_journal;
    if (c.no_journal) CKS(take_snapshot());
    CKS(launch(c, 0, false, false, true));
    Status sts[8];
    unsigned long long lcs[4];
    CKS(fetch_status(sts, lcs));
    res = sts[0];
    journal_count = c.no_journal ? 0 : lcs[1];
    snapshotted = c.no_journal;
    bool strict = !(flags & CGCM_LENIENT);
    int err = CGCM_OK;
    if (sts[0].misses && strict) err = CGCM_E_UNREGISTERED;
    else if (sts[0].underflow) err = CGCM_E_NOT_MAPPED;
    if (err) {
      if (c.no_journal) {
        CKS(restore_snapshot());
        CKS(undo_rev(c, 0, {}, write, false));  // refcounts came back with the snapshot
      } else {
        CKS(undo_rev(c, lcs[1], {}, write, dec));
      }
      return err;
    }
    rev_copy_n = lcs[3];  // the caller copies back copy_list[0, rev_copy_n) (copy_back_list)
    rev_free_n = dec ? lcs[2] : 0;  // and frees free_list[0, rev_free_n) (free_units_list)
    (void)copy_units;
    (void)freed;
    return CGCM_OK;
  }
  bool snapshotted = false;
  size_t rev_copy_n = 0, rev_free_n = 0;
  // forward-map shadows of device-resident pointer arrays, keyed by (slots, n)
  struct Shadow {
    DevBuf buf;
    uint64_t gen = 0;
    bool valid = false;
    bool deferred = false;  // its unit words may carry deferred references (SH_DEFER)
    bool device_array = false;  // cgcm_mapArrayDevice's (else a host-array outer's device copy)
  };
  size_t dev_shadows = 0;  // shadows of device arrays (free_units checks every freed copy only then)
  // Deferred references: the last cgcm_mapArrayDevice may have recorded references in
  // its shadow instead of rc.  Every other call that reads or changes refcounts (or replaces the table)
  // first adds them to rc -- only the matching cgcm_unmapArrayDevice(..., CGCM_RELEASE) drops them.
  int materialise(std::pair<const std::pair<uint64_t, uint64_t>, Shadow> &kv) {
    if (!kv.second.deferred) return CGCM_OK;
    const uint64_t n = kv.first.second;
    launch_materialise(reinterpret_cast<const uint64_t *>(kv.second.buf.addr), n, rcb.as<int32_t>(), main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    kv.second.deferred = false;
    return CGCM_OK;
  }
  int materialise_all(const Shadow *except = nullptr) {
    if (!any_deferred) return CGCM_OK;
    bool left = false;
    for (auto &kv : shadows) {
      if (&kv.second == except) {
        left = left || kv.second.deferred;
        continue;
      }
      CKS(materialise(kv));
    }
    any_deferred = left;
    return CGCM_OK;
  }
  bool any_deferred = false;
  std::map<std::pair<uint64_t, uint64_t>, Shadow> shadows;
  uint64_t table_gen = 0;
  // Record (CPU pointer, unit) per slot for the reverse passes (R13-ii) when a lookup costs more than
  // the 12-byte shadow: arrays of >= 2^16 slots and indexes with >= 2 levels (measured, config C
  // (h = 2): 48.5 vs 43.5 G/s); CGCM_FORCE_SHADOW: every array (tests).  Returns the buffer (invalid until the map
  // succeeds: commit_shadow) or 0.
  uint64_t begin_shadow(uint64_t ptr, uint64_t n, bool device_array = false) {
    static const int min_h = [] {  // CGCM_SHADOW_MIN_H: A/B override of the depth threshold
      const char *e = std::getenv("CGCM_SHADOW_MIN_H");
      return e ? std::atoi(e) : 2;
    }();
    if (!(flags & CGCM_FORCE_SHADOW) && (n < (1u << 16) || fwd.h < min_h)) return 0;
    auto key = std::make_pair(ptr, n);
    auto ins = shadows.emplace(key, Shadow());
    Shadow &sh = ins.first->second;
    if (ins.second && device_array) {
      sh.device_array = true;
      dev_shadows += 1;
    }
    sh.valid = false;
    if (dalloc(sh.buf, 8 * n + 64) != CGCM_OK) {  // one shadow word per slot (cgcm_dev.h make_shw)
      erase_shadow(shadows.find(key));
      return 0;
    }
    return sh.buf.addr;
  }
  void commit_shadow(uint64_t ptr, uint64_t n, bool ok) {
    auto it = shadows.find(std::make_pair(ptr, n));
    if (it == shadows.end()) return;
    if (ok) {
      it->second.valid = true;
      it->second.gen = table_gen;
    } else {
      erase_shadow(it);
    }
  }
  std::map<std::pair<uint64_t, uint64_t>, Shadow>::iterator erase_shadow(
      std::map<std::pair<uint64_t, uint64_t>, Shadow>::iterator it) {
    dfree(it->second.buf);
    if (it->second.device_array) dev_shadows -= 1;
    return shadows.erase(it);
  }
  // the valid shadow of (ptr, n), or 0
  uint64_t find_shadow(uint64_t ptr, uint64_t n) const {
    auto it = shadows.find(std::make_pair(ptr, n));
    return it != shadows.end() && it->second.valid && it->second.gen == table_gen ? it->second.buf.addr : 0;
  }
  // an outer's device copy is released: its shadows go with it
  void drop_shadows(uint64_t ptr) {
    for (auto it = shadows.lower_bound(std::make_pair(ptr, (uint64_t)0)); it != shadows.end() && it->first.first == ptr;) {
      materialise(*it);
      it = erase_shadow(it);
    }
  }
  int take_snapshot() {
    CKS(dalloc(snap_st, 8 * (size_t)U + 64));
    CKS(dalloc(snap_rc, 4 * (size_t)U + 64));
    CK(cudaMemcpyAsync(snap_rc.as<void>(), rcb.as<void>(), 4 * (size_t)U, cudaMemcpyDeviceToDevice, main));
    CK(cudaMemcpyAsync(snap_st.as<void>(), stb.as<void>(), 8 * (size_t)U, cudaMemcpyDeviceToDevice, main));
    return CGCM_OK;
  }
  int restore_snapshot() {
    // the pass does not touch hot words or flags: restoring the state words restores the epochs
    CK(cudaMemcpyAsync(rcb.as<void>(), snap_rc.as<void>(), 4 * (size_t)U, cudaMemcpyDeviceToDevice, main));
    CK(cudaMemcpyAsync(stb.as<void>(), snap_st.as<void>(), 8 * (size_t)U, cudaMemcpyDeviceToDevice, main));
    CK(cudaStreamSynchronize(main));
    return CGCM_OK;
  }
  // undo of a gate/reverse pass: epochs from the device journal (+ host-side extra entries), then
  // the slot side (re-translate in-place writes, re-add released references)
  int undo_rev(SlotCall &c, uint64_t journal_count, const std::vector<Journal> &extra, bool write, bool dec) {
    if (journal_count) {
      launch_restore_epochs(journal.as<Journal>(), (int)journal_count, tab(), main);
      st.kernel_launches += 1;
      CK(cudaGetLastError());
    }
    CKS(prepare_small());
    if (!extra.empty()) {
      DevBuf jb;
      CKS(upload(jb, extra));
      launch_restore_epochs(jb.as<Journal>(), (int)extra.size(), tab(), main);
      st.kernel_launches += 1;
      CK(cudaStreamSynchronize(main));
      dfree(jb);
    }
    bool inplace = true;
    for (auto &s : c.segs) inplace = inplace && s.out == 0;
    if (write && inplace) {
      // written slots now hold CPU pointers: forward-translate them back (+ re-add the reference)
      SlotCall f;
      f.dir = DIR_FWD;
      f.ops = dec ? (OP_WRITE | OP_INCPLAIN) : OP_WRITE;
      f.sel = SEL_HIT;
      f.segs = c.segs;
      CKS(launch(f, 1));
    } else if (dec) {
      SlotCall f;
      f.dir = DIR_REV;
      f.ops = OP_INCPLAIN;
      f.segs = c.segs;
      CKS(launch(f, 1));
    }
    CK(cudaStreamSynchronize(main));
    return CGCM_OK;
  }

  // outer-pointer lookups (one kernel, k pointers)
  int lookup_points(const uint64_t *ptrs, size_t k, std::vector<PointInfo> &out) {
    CKS(ensure_table());
    std::vector<uint64_t> v(ptrs, ptrs + k);
    CKS(upload(this->ptrs, v, true));
    CKS(dalloc(points, sizeof(PointInfo) * k + 64));
    launch_lookup_points(fwd.view(dbase.as<uint64_t>()), tab(), this->ptrs.as<uint64_t>(), (int)k,
                         points.as<PointInfo>(), dkeys.as<uint64_t>(), dids.as<uint32_t>(), (int)dk.size(), main);
    st.kernel_launches += 1;
    CK(cudaGetLastError());
    CKS(download(out, points, k));
    return CGCM_OK;
  }
};

// The state words (epoch | extent | flags) of units idx[] of a peer context, read on its device.
int Context::peer_sources(const std::vector<uint32_t> &units, std::vector<PeerSrc> &out) {
  std::vector<Context *> members;
  {
    std::lock_guard<std::mutex> g(group->mu);
    members = group->members;
  }
  out.assign(units.size(), PeerSrc());
  bool any = false;
  std::vector<size_t> todo(units.size());
  for (size_t q = 0; q < units.size(); ++q) todo[q] = q;
  for (Context *c : members) {
    if (c == this || todo.empty()) continue;
    std::lock_guard<std::recursive_mutex> lk(c->mu);
    if (cudaSetDevice(c->device) != cudaSuccess) return CGCM_E_CUDA;
    int r = c->ensure_table();

    std::vector<uint32_t> cidx;
    std::vector<size_t> which;
    if (r == CGCM_OK)
      for (size_t q : todo) {
        const uint32_t x = units[q];
        auto it = c->reg.find(ubase[x]);
        if (it != c->reg.end() && it->second.size == usize[x] && it->second.idx >= 0) {
          cidx.push_back((uint32_t)it->second.idx);
          which.push_back(q);
        }
      }
    std::vector<uint64_t> stw;
    if (r == CGCM_OK && !cidx.empty()) {
      r = c->upload(c->peer_idx, cidx);
      if (r == CGCM_OK) r = c->dalloc(c->peer_state, 8 * cidx.size() + 64);
      if (r == CGCM_OK) {
        launch_gather_state(c->tab(), c->peer_idx.as<uint32_t>(), (int)cidx.size(), c->peer_state.as<uint64_t>(),
                            c->main);
        c->st.kernel_launches += 1;
        r = c->download(stw, c->peer_state, cidx.size());
      }
    }
    if (r == CGCM_OK && !stw.empty()) {
      const uint32_t cur = c->rel_epoch(c->epoch);
      std::vector<size_t> left;
      size_t k = 0;
      for (size_t q : todo) {
        if (k < which.size() && which[k] == q) {
          const uint64_t w = stw[k];
          const uint32_t fl = hot_flags(w);
          const uint32_t ci = cidx[k];
          ++k;
          // active, holding a copy, writable, and dirty: c launched since the unit became coherent there
          const uint32_t ce = hot_ext(w);
          if ((fl & UF_ACTIVE) && (fl & UF_STORAGE) && !(fl & UF_READONLY) && st_epoch(w) != cur &&
              ce < c->runs.size()) {
            out[q].ctx = c;
            out[q].src = c->ubase[ci] - c->runs[ce].delta;  // the peer's copy (from its device table)
            any = true;
            continue;
          }
        }
        left.push_back(q);
      }
      todo.swap(left);
    }
    if (r == CGCM_OK && any) {  // the copies come after the GPU functions already queued on c
      if (!c->ev_peer && cudaEventCreateWithFlags(&c->ev_peer, cudaEventDisableTiming) != cudaSuccess) r = CGCM_E_CUDA;
      if (r == CGCM_OK && cudaEventRecord(c->ev_peer, c->main) != cudaSuccess) r = CGCM_E_CUDA;
    }
    if (cudaSetDevice(device) != cudaSuccess) return CGCM_E_CUDA;
    if (r != CGCM_OK) return r;
    if (any && out.size() && c->ev_peer) CK(cudaStreamWaitEvent(copy, c->ev_peer, 0));
  }
  if (!any) out.clear();
  return CGCM_OK;
}

// The copy-in of an activation where some units come from group peers: host-sourced units by runs of
// host-adjacent units (mirrored extents), peer-sourced units by runs contiguous on both sides.
int Context::copy_in_with_peers(const std::vector<uint32_t> &units, const std::vector<PeerSrc> &peer,
                                uint64_t bytes) {
  size_t i = 0;
  uint64_t pu = 0, pb = 0;
  while (i < units.size()) {
    const uint32_t x0 = units[i];
    size_t j = i + 1;
    uint64_t end = ubase[x0] + usize[x0];
    if (!peer[i].ctx) {
      while (j < units.size() && !peer[j].ctx && ubase[units[j]] == end &&
             udev[units[j]] == udev[x0] + (ubase[units[j]] - ubase[x0])) {
        end += usize[units[j]];
        ++j;
      }
      CKS(copy_run(udev[x0], ubase[x0], end - ubase[x0], true, units, i, j, copy));
      st.h2d_units += j - i;
      for (size_t q = i; q < j; ++q) st.h2d_bytes += usize[units[q]];
    } else {
      Context *c = peer[i].ctx;
      while (j < units.size() && peer[j].ctx == c && ubase[units[j]] == end &&
             udev[units[j]] == udev[x0] + (ubase[units[j]] - ubase[x0]) &&
             peer[j].src == peer[i].src + (ubase[units[j]] - ubase[x0])) {
        end += usize[units[j]];
        ++j;
      }
      const uint64_t n = end - ubase[x0];
      if (c->device == device)
        CK(cudaMemcpyAsync(reinterpret_cast<void *>(udev[x0]), reinterpret_cast<const void *>(peer[i].src), n,
                           cudaMemcpyDeviceToDevice, copy));
      else  // NVLink peer copy
        CK(cudaMemcpyPeerAsync(reinterpret_cast<void *>(udev[x0]), device, reinterpret_cast<const void *>(peer[i].src),
                               c->device, n, copy));
      st.peer_memcpy_calls += 1;
      pu += j - i;
      for (size_t q = i; q < j; ++q) pb += usize[units[q]];
    }
    i = j;
  }
  st.peer_units += pu;
  st.peer_bytes += pb;
  (void)bytes;
  CK(cudaEventRecord(ev_copy, copy));
  CK(cudaStreamWaitEvent(main, ev_copy, 0));
  st.activations += units.size();
  rev_dirty = true;
  pd_state_dirty = true;
  return CGCM_OK;
}

// ---------------------------------------------------------------------------------------------
std::mutex g_ctx_mu;
std::unordered_set<Context *> g_contexts;
thread_local Context *tl_ctx = nullptr;

// ---- map-promotion regions and their dynamic modOrRef checker (NEXT-2) ----
// While a checked region is open, the host pages of every promoted AU are PROT_NONE.  A CPU access
// to one faults; the handler reopens that page and, unless a runtime call is in progress (the
// runtime's own reads/writes of host AUs are not the program's), counts a violation: the loop did
// modify or reference a promoted AU, which makes the promotion illegal (P:L261 ¬modOrRef).  Pages
// the runtime touched are closed again when its call returns.  Process-wide (one signal handler).
struct ProtRange {
  uintptr_t lo, hi;
};
constexpr int PROT_MAX = 4096, TOUCH_MAX = 4096;
static ProtRange g_prot[PROT_MAX];
static std::atomic<int> g_nprot{0};
static std::atomic<int> g_rt_busy{0};
static std::atomic<unsigned long long> g_viol{0};
static std::atomic<uintptr_t> g_viol_first{0};
static uintptr_t g_touched[TOUCH_MAX];
static std::atomic<int> g_ntouched{0};
static struct sigaction g_old_segv;
static bool g_segv_installed = false;
static uintptr_t g_pagesz = 4096;

static void on_segv(int sig, siginfo_t *si, void *uc) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(si->si_addr);
  const int n = g_nprot.load(std::memory_order_acquire);
  for (int i = 0; i < n; ++i)
    if (a >= g_prot[i].lo && a < g_prot[i].hi) {
      const uintptr_t pg = a & ~(g_pagesz - 1);
      mprotect(reinterpret_cast<void *>(pg), g_pagesz, PROT_READ | PROT_WRITE);
      if (g_rt_busy.load() > 0) {
        const int k = g_ntouched.fetch_add(1);
        if (k < TOUCH_MAX) g_touched[k] = pg;
      } else if (g_viol.fetch_add(1) == 0) {
        g_viol_first.store(a);
      }
      return;  // the access re-executes on the reopened page
    }
  // not a promoted page: the previous handler (or the default action on the re-executed access)
  if ((g_old_segv.sa_flags & SA_SIGINFO) && g_old_segv.sa_sigaction) {
    g_old_segv.sa_sigaction(sig, si, uc);
    return;
  }
  if (!(g_old_segv.sa_flags & SA_SIGINFO) && g_old_segv.sa_handler != SIG_DFL && g_old_segv.sa_handler != SIG_IGN) {
    g_old_segv.sa_handler(sig);
    return;
  }
  sigaction(SIGSEGV, &g_old_segv, nullptr);
}
// every C-ABI call: pages the runtime itself touches in a checked region are closed again on return
struct RtScope {
  RtScope() { g_rt_busy.fetch_add(1); }
  ~RtScope() {
    if (g_rt_busy.fetch_sub(1) == 1) {
      const int n = std::min(g_ntouched.exchange(0), TOUCH_MAX);
      for (int i = 0; i < n && g_nprot.load() > 0; ++i) mprotect(reinterpret_cast<void *>(g_touched[i]), g_pagesz, PROT_NONE);
    }
  }
};

}  // namespace cgcm

using namespace cgcm;
using SlotCall = Context::SlotCall;

#define CTX()                                     \
  Context *C = tl_ctx;                            \
  if (!C) return CGCM_E_NOCTX;                    \
  RtScope rts_;                                   \
  std::lock_guard<std::recursive_mutex> lk_(C->mu); \
  if (cudaSetDevice(C->device) != cudaSuccess) return CGCM_E_CUDA;

// every call that reads or changes refcounts first materialises deferred references
#define CTXM() \
  CTX();       \
  CKS(C->materialise_all());

// ============================== C ABI ==========================================================
extern "C" {

const char *cgcm_strerror(int s) {
  switch (s) {
    case CGCM_OK: return "ok";
    case CGCM_E_INVALID: return "invalid argument";
    case CGCM_E_UNREGISTERED: return "pointer not inside a declared allocation unit";
    case CGCM_E_OVERLAP: return "allocation unit overlaps a declared one";
    case CGCM_E_NOT_MAPPED: return "allocation unit not mapped (refCount 0)";
    case CGCM_E_BUSY: return "allocation unit is mapped";
    case CGCM_E_DUPLICATE: return "global name already declared";
    case CGCM_E_NOMEM: return "out of memory";
    case CGCM_E_CUDA: return "CUDA error";
    case CGCM_E_MIXED: return "mixed";
    case CGCM_E_NOCTX: return "no current context";
    case CGCM_E_MODREF: return "the CPU accessed a promoted allocation unit inside a map-promotion region";
  }
  return "unknown";
}
const char *cgcm_lastCudaError(void) { return g_last_cuda_error.c_str(); }

int cgcm_init(int device, void *dev_arena, size_t arena_bytes, void *main_stream, void *copy_stream, unsigned flags) {
  if (arena_bytes < (1u << 20)) return CGCM_E_INVALID;
  CK(cudaSetDevice(device));
  Context *C = new Context();
  C->device = device;
  C->flags = flags;
  int nsm = 0;
  if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device) == cudaSuccess && nsm > 0) C->nsm = nsm;
  if (const char *e = std::getenv("CGCM_L2_FETCH")) {  // A/B experiments: L2 fetch granularity (bytes)
    size_t want = (size_t)std::atoi(e), got = 0;
    cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, want);
    cudaDeviceGetLimit(&got, cudaLimitMaxL2FetchGranularity);
    std::fprintf(stderr, "cgcm: L2 fetch granularity %zu (asked %zu)\n", got, want);
  }
  if (!dev_arena) {
    if (cudaMalloc(&C->own_arena, arena_bytes) != cudaSuccess) {
      delete C;
      g_last_cuda_error = "cudaMalloc of the device arena failed";
      return CGCM_E_NOMEM;
    }
    dev_arena = C->own_arena;
  }
  C->arena.init(reinterpret_cast<uint64_t>(dev_arena), arena_bytes);
  if (!main_stream || !copy_stream) {
    cudaStreamCreateWithFlags(&C->main, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&C->copy, cudaStreamNonBlocking);
    C->own_streams = true;
  } else {
    C->main = reinterpret_cast<cudaStream_t>(main_stream);
    C->copy = reinterpret_cast<cudaStream_t>(copy_stream);
  }
  cudaEventCreateWithFlags(&C->ev_copy, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&C->ev_pack[0], cudaEventDisableTiming);
  cudaEventCreateWithFlags(&C->ev_pack[1], cudaEventDisableTiming);
  cudaEventCreate(&C->ev_t0);
  cudaEventCreate(&C->ev_t1);
  // the small pinned, mapped host buffers every call path uses, allocated now: a cudaHostAlloc inside a
  // call costs 8-600 ms on this pool (profiles/r02bw_trace.log)
  // (best effort: a failure here only leaves the allocation to the first call that needs the buffer)
  (void)C->h_list.ensure(1 << 20);
  (void)C->h_status.ensure(sizeof(Status) * 8 + 64);
  (void)C->h_small.ensure(1 << 16);
  (void)C->h_lists.ensure(3 * 4 * Context::LIST_HEAD + 64);
  (void)C->ring_init();
  {
    std::lock_guard<std::mutex> g(g_ctx_mu);
    g_contexts.insert(C);
  }
  tl_ctx = C;
  std::lock_guard<std::recursive_mutex> lk(C->mu);
  return C->ensure_table();
}

int cgcm_groupCreate(void **group_out) {
  if (!group_out) return CGCM_E_INVALID;
  *group_out = new Group();
  return CGCM_OK;
}
int cgcm_groupJoin(void *group) {
  CTXM();
  if (!group || C->group) return CGCM_E_INVALID;
  Group *g = static_cast<Group *>(group);
  std::lock_guard<std::mutex> lk(g->mu);
  g->members.push_back(C);
  C->group = g;
  return CGCM_OK;
}
static int group_leave(Context *C) {
  if (!C->group) return CGCM_E_INVALID;
  Group *g = C->group;
  std::lock_guard<std::mutex> lk(g->mu);
  g->members.erase(std::remove(g->members.begin(), g->members.end(), C), g->members.end());
  C->group = nullptr;
  return CGCM_OK;
}
int cgcm_groupLeave(void) {
  CTX();
  return group_leave(C);
}
int cgcm_groupDestroy(void *group) {
  if (!group) return CGCM_E_INVALID;
  Group *g = static_cast<Group *>(group);
  {
    std::lock_guard<std::mutex> lk(g->mu);
    if (!g->members.empty()) return CGCM_E_BUSY;
  }
  delete g;
  return CGCM_OK;
}

int cgcm_finalize(void) {
  Context *C = tl_ctx;
  if (!C) return CGCM_E_NOCTX;
  if (C->group) group_leave(C);
  if (C->ev_peer) cudaEventDestroy(C->ev_peer);
  {
    std::lock_guard<std::mutex> g(g_ctx_mu);
    g_contexts.erase(C);
  }
  cudaSetDevice(C->device);
  cudaStreamSynchronize(C->main);
  cudaStreamSynchronize(C->copy);
  for (auto &c : C->hchunks) cudaFreeHost(c.first);
  if (C->h_small.p) cudaFreeHost(C->h_small.p);
  if (C->h_ring.p) cudaFreeHost(C->h_ring.p);
  for (auto &e : C->ev_ring)
    if (e) cudaEventDestroy(e);
  if (C->h_status.p) cudaFreeHost(C->h_status.p);
  if (C->h_list.p) cudaFreeHost(C->h_list.p);
  if (C->h_lists.p) cudaFreeHost(C->h_lists.p);
  cudaEventDestroy(C->ev_copy);
  cudaEventDestroy(C->ev_pack[0]);
  cudaEventDestroy(C->ev_pack[1]);
  for (auto &hp : C->h_pack)
    if (hp.p) cudaFreeHost(hp.p);
  cudaEventDestroy(C->ev_t0);
  cudaEventDestroy(C->ev_t1);
  if (C->own_streams) {
    cudaStreamDestroy(C->main);
    cudaStreamDestroy(C->copy);
  }
  if (C->own_arena) cudaFree(C->own_arena);
  delete C;
  tl_ctx = nullptr;
  return CGCM_OK;
}

void *cgcm_getContext(void) { return tl_ctx; }
int cgcm_setContext(void *ctx) {
  std::lock_guard<std::mutex> g(g_ctx_mu);
  if (ctx && !g_contexts.count(reinterpret_cast<Context *>(ctx))) return CGCM_E_INVALID;
  tl_ctx = reinterpret_cast<Context *>(ctx);
  return CGCM_OK;
}

// ---- registration --------------------------------------------------------------------------
static int declare_one(Context *C, uint64_t b, uint64_t s, uint32_t fl, const char *name, uint64_t sym = 0) {
  if (b == 0 || s == 0 || b + s < b || b + s >= ADDR_LIMIT) return CGCM_E_INVALID;
  auto succ = C->reg.lower_bound(b);
  if (succ != C->reg.end() && succ->first < b + s) return CGCM_E_OVERLAP;
  if (succ != C->reg.begin()) {
    auto pred = std::prev(succ);
    if (pred->first + pred->second.size > b) return CGCM_E_OVERLAP;
  }
  HostUnit u;
  u.size = s;
  u.flags = fl;
  u.epoch0 = C->epoch;
  if (name) u.name = name;
  u.sym = sym;
  C->reg.emplace_hint(succ, b, u);
  C->table_dirty = true;
  C->note_declared(b);
  return CGCM_OK;
}

int cgcm_declareAlloc(void *base, size_t size) {
  CTX();
  return declare_one(C, reinterpret_cast<uint64_t>(base), size, 0, nullptr);
}
int cgcm_declareAllocFlags(void *base, size_t size, unsigned unit_flags) {
  CTX();
  return declare_one(C, reinterpret_cast<uint64_t>(base), size, (unit_flags & CGCM_UNIT_READONLY) ? UF_READONLY : 0,
                     nullptr);
}
int cgcm_declareBatch(void *const *bases, const size_t *sizes, size_t n, unsigned unit_flags) {
  CTX();
  if (n && (!bases || !sizes)) return CGCM_E_INVALID;
  std::vector<size_t> ord(n);
  for (size_t i = 0; i < n; ++i) ord[i] = i;
  auto B = [&](size_t i) { return reinterpret_cast<uint64_t>(bases[i]); };
  std::sort(ord.begin(), ord.end(), [&](size_t a, size_t b) { return B(a) < B(b); });
  for (size_t q = 0; q < n; ++q) {  // validate everything first (all-or-nothing)
    uint64_t b = B(ord[q]), s = sizes[ord[q]];
    if (b == 0 || s == 0 || b + s < b || b + s >= ADDR_LIMIT) return CGCM_E_INVALID;
    if (q + 1 < n && b + s > B(ord[q + 1])) return CGCM_E_OVERLAP;
    auto succ = C->reg.lower_bound(b);
    if (succ != C->reg.end() && succ->first < b + s) return CGCM_E_OVERLAP;
    if (succ != C->reg.begin()) {
      auto pred = std::prev(succ);
      if (pred->first + pred->second.size > b) return CGCM_E_OVERLAP;
    }
  }
  uint32_t fl = (unit_flags & CGCM_UNIT_READONLY) ? UF_READONLY : 0;
  auto hint = C->reg.begin();
  for (size_t q = 0; q < n; ++q) {
    HostUnit u;
    u.size = sizes[ord[q]];
    u.flags = fl;
    u.epoch0 = C->epoch;
    hint = C->reg.lower_bound(B(ord[q]));
    hint = C->reg.emplace_hint(hint, B(ord[q]), u);
    C->note_declared(B(ord[q]));
  }
  if (n) C->table_dirty = true;
  return CGCM_OK;
}
int cgcm_declareGlobal(const char *name, void *base, size_t size, int isReadOnly) {
  CTX();
  if (!name || !*name) return CGCM_E_INVALID;
  if (C->names.count(name)) return CGCM_E_DUPLICATE;
  int s = declare_one(C, reinterpret_cast<uint64_t>(base), size, UF_GLOBAL | (isReadOnly ? UF_READONLY : 0), name);
  if (s == CGCM_OK) C->names.insert(name);
  return s;
}
int cgcm_declareGlobalSymbol(const char *name, void *base, size_t size, int isReadOnly, void *dev_symbol) {
  CTX();
  if (!name || !*name || !dev_symbol) return CGCM_E_INVALID;
  if (C->names.count(name)) return CGCM_E_DUPLICATE;
  const uint64_t b = reinterpret_cast<uint64_t>(base), d = reinterpret_cast<uint64_t>(dev_symbol);
  // A7: two device copies may touch only if their host units touch in the same order (a one-past-the-end
  // pointer of one must reverse to the same place).  Arena extents always keep >= 1 byte of slack, so
  // only other bound symbols can be adjacent or overlap.
  for (auto &kv : C->reg) {
    const HostUnit &o = kv.second;
    if (!o.sym) continue;
    const uint64_t ob = kv.first, os = o.size;
    if (d < o.sym + os && o.sym < d + size) return CGCM_E_OVERLAP;
    if (d + size == o.sym && b + size != ob) return CGCM_E_OVERLAP;
    if (o.sym + os == d && ob + os != b) return CGCM_E_OVERLAP;
  }
  int s = declare_one(C, b, size, UF_GLOBAL | (isReadOnly ? UF_READONLY : 0), name, d);
  if (s == CGCM_OK) C->names.insert(name);
  return s;
}
int cgcm_undeclare(void *base) {
  CTXM();
  uint64_t b = reinterpret_cast<uint64_t>(base);
  auto it = C->reg.find(b);
  if (it == C->reg.end()) return CGCM_E_UNREGISTERED;
  HostUnit &u = it->second;
  if (u.idx >= 0) CKS(C->mirror_units({(uint32_t)u.idx}));
  if (u.idx >= 0) {  // idx refers to the current device table until the next ensure_table()
    int32_t rc = 0;
    CK(cudaMemcpyAsync(&rc, C->rcb.as<int32_t>() + u.idx, 4, cudaMemcpyDeviceToHost, C->main));
    CK(cudaStreamSynchronize(C->main));
    if (rc > 0) return CGCM_E_BUSY;
  }
  if (u.flags & UF_GLOBAL) {
    C->names.erase(u.name);
    if (u.idx >= 0 && C->urun[u.idx] >= 0) {
      C->run_release(C->urun[u.idx]);
      C->urun[u.idx] = -1;
      C->udev[u.idx] = 0;
    }
  }
  C->arr_gen.erase(b);
  if (u.idx >= 0) {
    C->dirty_del = true;  // the device table changes shape: the next merge rebuilds it
  } else {                // declared and undeclared between two merges: never in the device table
    auto pe = std::find(C->pend.begin(), C->pend.end(), b);
    if (pe != C->pend.end()) C->pend.erase(pe);
  }
  C->reg.erase(it);
  C->table_dirty = true;
  return CGCM_OK;
}

// ---- pinned host arena (R10 heap wrappers) ---------------------------------------------------
void *cgcm_malloc(size_t n) {
  Context *C = tl_ctx;
  if (!C || n == 0) return nullptr;
  std::lock_guard<std::recursive_mutex> lk(C->mu);
  uint64_t len = align_up(n, 16);
  auto pick = C->hfree.end();
  for (auto it = C->hfree.begin(); it != C->hfree.end(); ++it)
    if (it->second >= len) {
      pick = it;
      break;
    }
  if (pick == C->hfree.end()) {
    size_t chunk = std::max<size_t>(align_up(len, 1 << 21), (size_t)256 << 20);
    void *p = nullptr;
    cudaSetDevice(C->device);
    if (cudaHostAlloc(&p, chunk, cudaHostAllocPortable) != cudaSuccess) return nullptr;
    C->hchunks.push_back({static_cast<char *>(p), chunk});
    pick = C->hfree.emplace(reinterpret_cast<uint64_t>(p), chunk).first;
  }
  uint64_t a = pick->first, l = pick->second;
  C->hfree.erase(pick);
  if (l > len) C->hfree.emplace(a + len, l - len);
  if (declare_one(C, a, n, 0, nullptr) != CGCM_OK) {
    C->hfree.emplace(a, len);
    return nullptr;
  }
  C->hallocs[a] = len;
  C->hsizes[a] = n;
  return reinterpret_cast<void *>(a);
}
int cgcm_free(void *p) {
  Context *C = tl_ctx;
  if (!C) return CGCM_E_NOCTX;
  if (!p) return CGCM_OK;
  std::lock_guard<std::recursive_mutex> lk(C->mu);
  uint64_t a = reinterpret_cast<uint64_t>(p);
  auto it = C->hallocs.find(a);
  if (it == C->hallocs.end()) return CGCM_E_INVALID;
  int s = cgcm_undeclare(p);
  if (s != CGCM_OK) return s;
  uint64_t len = it->second;
  C->hallocs.erase(it);
  C->hsizes.erase(a);
  // coalesce with neighbours
  auto nx = C->hfree.lower_bound(a);
  if (nx != C->hfree.end() && nx->first == a + len) {
    len += nx->second;
    C->hfree.erase(nx);
  }
  auto pv = C->hfree.lower_bound(a);
  if (pv != C->hfree.begin()) {
    --pv;
    if (pv->first + pv->second == a) {
      a = pv->first;
      len += pv->second;
      C->hfree.erase(pv);
    }
  }
  C->hfree.emplace(a, len);
  return CGCM_OK;
}

void *cgcm_calloc(size_t nmemb, size_t size) {
  if (nmemb && size > SIZE_MAX / nmemb) return nullptr;
  void *p = cgcm_malloc(nmemb * size);
  if (p) std::memset(p, 0, nmemb * size);
  return p;
}

void *cgcm_realloc(void *p, size_t n) {
  Context *C = tl_ctx;
  if (!C) return nullptr;
  if (!p) return cgcm_malloc(n);
  if (n == 0) {
    cgcm_free(p);
    return nullptr;
  }
  std::lock_guard<std::recursive_mutex> lk(C->mu);
  uint64_t a = reinterpret_cast<uint64_t>(p);
  auto it = C->hsizes.find(a);
  if (it == C->hsizes.end()) return nullptr;
  auto ru = C->reg.find(a);
  if (C->materialise_all() != CGCM_OK) return nullptr;
  if (ru != C->reg.end() && ru->second.idx >= 0) {  // a mapped AU cannot move (BUSY)
    int32_t rc = 0;
    if (cudaMemcpy(&rc, C->rcb.as<int32_t>() + ru->second.idx, 4, cudaMemcpyDeviceToHost) != cudaSuccess || rc > 0)
      return nullptr;
  }
  size_t old = it->second;
  void *q = cgcm_malloc(n);
  if (!q) return nullptr;
  std::memcpy(q, p, std::min(old, n));
  if (cgcm_free(p) != CGCM_OK) {
    cgcm_free(q);
    return nullptr;
  }
  return q;
}

int cgcm_scopeEnter(void) {
  CTX();
  C->scopes.emplace_back();
  return CGCM_OK;
}
void *cgcm_declareAlloca(size_t n) {
  Context *C = tl_ctx;
  if (!C) return nullptr;
  std::lock_guard<std::recursive_mutex> lk(C->mu);
  if (C->scopes.empty()) C->scopes.emplace_back();  // an implicit outermost scope
  void *p = cgcm_malloc(n);
  if (p) C->scopes.back().push_back(reinterpret_cast<uint64_t>(p));
  return p;
}
int cgcm_scopeExit(void) {
  CTXM();
  if (C->scopes.empty()) return CGCM_E_INVALID;
  auto &sc = C->scopes.back();
  // all-or-nothing: no registration expires while one of the scope's AUs is mapped
  CKS(C->ensure_table());
  for (uint64_t a : sc) {
    auto ru = C->reg.find(a);
    if (ru == C->reg.end() || ru->second.idx < 0) continue;
    int32_t rc = 0;
    CK(cudaMemcpy(&rc, C->rcb.as<int32_t>() + ru->second.idx, 4, cudaMemcpyDeviceToHost));
    if (rc > 0) return CGCM_E_BUSY;
  }
  for (auto it = sc.rbegin(); it != sc.rend(); ++it) CKS(cgcm_free(reinterpret_cast<void *>(*it)));
  C->scopes.pop_back();
  return CGCM_OK;
}

// ---- device-resident arrays -------------------------------------------------------------------

int cgcm_mapArrayDevice(uint64_t *d_slots, size_t n) {
  CTXM();
  if (n == 0) return CGCM_OK;
  if (!d_slots || (reinterpret_cast<uint64_t>(d_slots) & 7)) return CGCM_E_INVALID;
  CKS(C->ensure_table());
  Seg s{reinterpret_cast<uint64_t>(d_slots), n, 0, 1, 0};
  s.shadow = C->begin_shadow(s.ptr, n, true);
  // with a shadow, references to units already active are deferred into it
  int r = C->map_core({s}, {}, nullptr, nullptr, nullptr, nullptr, s.shadow != 0);
  if (s.shadow) {
    C->commit_shadow(s.ptr, n, r == CGCM_OK);
    if (r == CGCM_OK) {
      C->shadows[std::make_pair(s.ptr, (uint64_t)n)].deferred = true;
      C->any_deferred = true;
    }
  }
  return r;
}

int cgcm_unmapArrayDevice(uint64_t *d_slots, size_t n, unsigned flags) {
  CTX();
  if (n == 0) return CGCM_OK;
  if (!d_slots || (reinterpret_cast<uint64_t>(d_slots) & 7)) return CGCM_E_INVALID;
  Seg s{reinterpret_cast<uint64_t>(d_slots), n, 0, 1, 0};
  auto shk = std::make_pair(s.ptr, (uint64_t)n);
  auto shi = C->shadows.find(shk);
  bool rel = (flags & CGCM_RELEASE) != 0;
  // the references the matching mapArrayDevice deferred are dropped by this pass when it releases
  // them; in every other case they become ordinary references first (as all others do here)
  const bool defer = rel && shi != C->shadows.end() && shi->second.valid && shi->second.deferred &&
                     shi->second.gen == C->table_gen && !C->table_dirty;
  CKS(C->materialise_all(defer ? &shi->second : nullptr));
  if (shi != C->shadows.end()) {
    CKS(C->ensure_table());
    if (shi->second.valid && shi->second.gen == C->table_gen) s.shadow = shi->second.buf.addr;
    shi->second.valid = false;  // consumed: after this call the slots hold CPU pointers again
  }
  std::vector<uint32_t> copy_units, freed;
  uint64_t jcount = 0;
  Status res{};
  // (on failure the snapshot restores rc and the shadow keeps its deferred references: the next call
  // materialises them)
  CKS(C->unmap_rev_core({s}, true, rel, copy_units, freed, jcount, res, defer));
  int r = C->copy_back_list(C->copy_list, C->rev_copy_n);
  if (r != CGCM_OK) {
    // reverse translation of an array-mapped element failed: undo the whole call
    SlotCall c;
    c.dir = DIR_REV;
    c.ops = OP_WRITE | OP_GATE | OP_HITMASK | (rel ? OP_DEC : 0);
    c.segs = {s};
    if (C->snapshotted) {
      C->restore_snapshot();
      C->undo_rev(c, 0, {}, true, false);
    } else {
      C->undo_rev(c, jcount, {}, true, rel);
    }
    return r;
  }
  if (defer) {  // every deferred reference was dropped or materialised by the pass
    shi->second.deferred = false;
    C->any_deferred = false;
  }
  C->st.rev_translations += res.translated;
  if (C->flags & CGCM_LENIENT) C->st.passthrough += res.misses;
  CKS(C->free_units_list(C->free_list, C->rev_free_n));
  return CGCM_OK;
}

// ---- host-array batch forms ---------------------------------------------------------------------
static int stage_in(Context *C, const void *const *cpu, size_t n, uint64_t &dptr) {
  CKS(C->dalloc(C->staging, 8 * n + 64));
  CKS(C->h_small.ensure(8 * n));
  CK(cudaStreamSynchronize(C->main));
  std::memcpy(C->h_small.p, cpu, 8 * n);
  CK(cudaMemcpyAsync(C->staging.as<void>(), C->h_small.p, 8 * n, cudaMemcpyHostToDevice, C->main));
  dptr = C->staging.addr;
  return CGCM_OK;
}

int cgcm_mapBatch(const void *const *cpu, size_t n, void **gpu_out) {
  CTXM();
  if (n == 0) return CGCM_OK;
  if (!cpu || !gpu_out) return CGCM_E_INVALID;
  CKS(C->ensure_table());
  uint64_t d = 0;
  CKS(stage_in(C, cpu, n, d));
  Seg s{d, n, 0, 1, 0};
  CKS(C->map_core({s}, {}, nullptr, nullptr));
  CK(cudaMemcpyAsync(C->h_small.p, C->staging.as<void>(), 8 * n, cudaMemcpyDeviceToHost, C->main));
  CK(cudaStreamSynchronize(C->main));
  std::memcpy(gpu_out, C->h_small.p, 8 * n);
  return CGCM_OK;
}

int cgcm_unmapBatch(const void *const *cpu, size_t n) {
  CTXM();
  if (n == 0) return CGCM_OK;
  if (!cpu) return CGCM_E_INVALID;
  CKS(C->ensure_table());
  uint64_t d = 0;
  CKS(stage_in(C, cpu, n, d));
  CKS(C->prepare(n + 64));
  SlotCall c;
  c.dir = DIR_FWD;
  c.ops = OP_GATE | OP_CHECKMAPPED;
  c.segs = {Seg{d, n, 0, 1, 0}};
  CKS(C->launch(c, 0));
  Status sts[8];
  unsigned long long lcs[4];
  CKS(C->fetch_status(sts, lcs));
  int err = CGCM_OK;
  if (sts[0].misses && !(C->flags & CGCM_LENIENT)) err = CGCM_E_UNREGISTERED;
  else if (sts[0].notmapped) err = CGCM_E_NOT_MAPPED;
  if (!err) err = C->copy_back_list(C->copy_list, lcs[3]);
  if (err) {
    SlotCall u;
    CKS(C->undo_rev(u, lcs[1], {}, false, false));
    return err;
  }
  return CGCM_OK;
}

int cgcm_releaseBatch(const void *const *cpu, size_t n) {
  CTXM();
  if (n == 0) return CGCM_OK;
  if (!cpu) return CGCM_E_INVALID;
  CKS(C->ensure_table());
  uint64_t d = 0;
  CKS(stage_in(C, cpu, n, d));
  CKS(C->prepare(n + 64));
  SlotCall c;
  c.dir = DIR_FWD;
  c.ops = OP_DEC;
  c.segs = {Seg{d, n, 0, 1, 0}};
  c.dec_red = n >= (size_t)C->U / 8 && C->U >= 4096;  // small tables: returning atomics, no scan launch
  CKS(C->launch(c, 0));
  Status sts[8];
  unsigned long long lcs[4];
  CKS(C->fetch_status(sts, lcs));
  int err = CGCM_OK;
  if (sts[0].misses && !(C->flags & CGCM_LENIENT)) err = CGCM_E_UNREGISTERED;
  else if (sts[0].underflow) err = CGCM_E_NOT_MAPPED;
  if (err) {
    SlotCall u;
    u.dir = DIR_FWD;
    u.ops = OP_INCPLAIN;
    u.segs = c.segs;
    CKS(C->prepare_small());
    CKS(C->launch(u, 0));
    CK(cudaStreamSynchronize(C->main));
    return err;
  }
  return C->free_units_list(C->free_list, lcs[2]);
}

int cgcm_map(const void *cpu, void **gpu_out) {
  if (!gpu_out) return CGCM_E_INVALID;
  void *out = nullptr;
  int s = cgcm_mapBatch(&cpu, 1, &out);
  if (s == CGCM_OK) *gpu_out = out;
  return s;
}
int cgcm_unmap(const void *cpu) { return cgcm_unmapBatch(&cpu, 1); }
int cgcm_release(const void *cpu) { return cgcm_releaseBatch(&cpu, 1); }

// ---- array variants ---------------------------------------------------
namespace {
struct Outer {
  int unit;
  PointInfo info;
  int mult;
  int first;  // index of first appearance
};
int distinct_outers(const std::vector<PointInfo> &infos, std::vector<Outer> &out, std::vector<int> &which) {
  std::unordered_map<int, int> pos;
  which.resize(infos.size());
  for (size_t j = 0; j < infos.size(); ++j) {
    if (infos[j].unit < 0) return CGCM_E_UNREGISTERED;
    auto it = pos.find(infos[j].unit);
    if (it == pos.end()) {
      pos[infos[j].unit] = (int)out.size();
      which[j] = (int)out.size();
      out.push_back({infos[j].unit, infos[j], 1, (int)j});
    } else {
      out[it->second].mult += 1;
      which[j] = it->second;
    }
  }
  return CGCM_OK;
}
}  // namespace

int cgcm_mapArrays(void *const *const *arrays, size_t k, void ***gpu_out) {
  Trace tt_("cgcm_mapArrays");
  CTXM();

  if (k == 0) return CGCM_OK;
  if (!arrays || !gpu_out) return CGCM_E_INVALID;
  {  // the re-map of array-mapped outers in a promoted loop (A9): no host wait at all
    const int r = C->remap_arrays_async(reinterpret_cast<const uint64_t *>(arrays), k, gpu_out);
    if (r != 1) return r;  // 1: not that case, take the general path
  }
  std::vector<PointInfo> infos;
  CKS(C->lookup_points(reinterpret_cast<const uint64_t *>(arrays), k, infos));
  std::vector<Outer> outs;
  std::vector<int> which;
  CKS(distinct_outers(infos, outs, which));
  {
    std::vector<uint32_t> ou;
    for (auto &o : outs) ou.push_back((uint32_t)o.unit);
    CKS(C->mirror_units(ou));
  }
  // prologue: activate inactive outers (raw copy of the CPU pointer array, rewritten in place),
  // then refcount/flags of every outer -- the outer AU first (A9)
  std::vector<uint32_t> act;
  for (auto &o : outs)
    if (o.info.refcount == 0) act.push_back((uint32_t)o.unit);
  std::sort(act.begin(), act.end());
  std::vector<std::pair<uint64_t, uint64_t>> copies;
  std::vector<cudaEvent_t> pack_ev;  // transfer overlap: the outers' H2D copies, one event per extent
  CKS(C->activate_units(act, &copies, &pack_ev));
  std::vector<UnitOp> ops;
  std::vector<Seg> fsegs, rsegs;
  bool rev_stale = false;
  for (auto &o : outs) {
    const uint64_t hu_dev = C->udev[o.unit];
    ops.push_back({(uint32_t)o.unit, UOP_ADD_RC, (uint64_t)(int64_t)o.mult});
    ops.push_back({(uint32_t)o.unit, UOP_OR_FLAGS, UF_ARRAYMAPPED});
    uint64_t n = o.info.size / 8;
    if (!n) continue;
    Seg s{hu_dev, n, 0, o.mult, 0};
    if (o.info.refcount > 0 && (o.info.flags & UF_ARRAYMAPPED)) {
      rsegs.push_back(s);  // A9: refcounts only
      auto g = C->arr_gen.find(o.info.base);
      if (g == C->arr_gen.end() || g->second != C->free_gen) rev_stale = true;
    } else {
      fsegs.push_back(s);
    }
  }
  bool ops_applied = false;
  auto undo_prologue = [&]() {
    cudaStreamSynchronize(C->copy);  // the outers' copies land before their storage is released
    std::vector<UnitOp> undo;
    if (ops_applied)
      for (auto &o : outs) {
        undo.push_back({(uint32_t)o.unit, UOP_ADD_RC, (uint64_t)(int64_t)(-o.mult)});
        if (!(o.info.flags & UF_ARRAYMAPPED)) undo.push_back({(uint32_t)o.unit, UOP_AND_FLAGS, ~(uint64_t)UF_ARRAYMAPPED});
      }
    for (auto &o : outs)
      if (o.info.refcount == 0) undo.push_back({(uint32_t)o.unit, UOP_SET_EPOCH, o.info.epoch});
    C->unit_ops(undo);
    cudaStreamSynchronize(C->main);
    std::vector<uint32_t> deact;
    for (auto &o : outs)
      if (o.info.refcount == 0) deact.push_back((uint32_t)o.unit);
    // these activations are withdrawn, not reported
    uint64_t frees0 = C->st.frees;
    C->st.activations -= act.size();
    C->st.h2d_units -= act.size();
    for (uint32_t x : act) C->st.h2d_bytes -= C->usize[x];
    C->free_units(deact);
    C->st.frees = frees0;
  };
  // unit ops must not run before the outers' set_devbase: same stream, issued after
  {
    const int r = C->unit_ops(ops);
    if (r != CGCM_OK) {  // all-or-nothing: withdraw the activations
      undo_prologue();
      return r;
    }
    ops_applied = true;
  }
  // array-mapped outers: refcounts through the reverse index (no copy); if an element
  // lost its device copy, re-translate the outer from its host slots instead (oracle semantics)
  Status rres{};
  bool rev_done = false;
  struct Backup { uint64_t src, dst, n; };
  std::vector<Backup> backups;
  if (!rsegs.empty()) {
    int r = rev_stale ? CGCM_E_UNREGISTERED : C->rev_addref(rsegs, rres);
    if (r == CGCM_OK) {
      rev_done = true;
    } else if (r == CGCM_E_UNREGISTERED) {
      // keep the current device slots so that a failing call can put them back (all-or-nothing)
      // every failure from here on restores the slots backed up so far and withdraws the prologue
      auto fail = [&](int status) {
        for (auto &b : backups)
          cudaMemcpyAsync(reinterpret_cast<void *>(b.dst), reinterpret_cast<void *>(b.src), b.n,
                          cudaMemcpyDeviceToDevice, C->main);
        undo_prologue();
        return status;
      };
      uint64_t bytes = 0;
      for (auto &sg : rsegs) bytes += 8 * sg.n + 32;
      if (C->dalloc(C->staging2, bytes + 256) != CGCM_OK) return fail(CGCM_E_NOMEM);
      uint64_t off = C->staging2.addr;
      for (auto &sg : rsegs) {
        if (cudaMemcpyAsync(reinterpret_cast<void *>(off), reinterpret_cast<void *>(sg.ptr), 8 * sg.n,
                            cudaMemcpyDeviceToDevice, C->main) != cudaSuccess)
          return fail(CGCM_E_CUDA);
        backups.push_back({off, sg.ptr, 8 * sg.n});
        off += 8 * sg.n + 32;
      }
      for (auto &sg : rsegs) {
        for (auto &o : outs)
          if (C->udev[o.unit] == sg.ptr) {
            if (cudaMemcpyAsync(reinterpret_cast<void *>(sg.ptr), reinterpret_cast<const void *>(o.info.base),
                                8 * sg.n, cudaMemcpyHostToDevice, C->main) != cudaSuccess)
              return fail(CGCM_E_CUDA);
            C->st.h2d_memcpy_calls += 1;
          }
        fsegs.push_back(sg);
      }
    } else {
      undo_prologue();
      return r;
    }
  }
  // translate each outer once its extent has arrived (transfer scheduler: H2D on the copy stream
  // overlapped with translation on the main stream, one launch per extent)
  std::vector<int> group(fsegs.size(), -1);
  for (size_t q = 0; q < fsegs.size(); ++q)
    for (size_t p = 0; p < copies.size(); ++p)
      if (fsegs[q].ptr >= copies[p].first && fsegs[q].ptr < copies[p].first + copies[p].second) {
        group[q] = (int)p;
        break;
      }
  {
    std::vector<size_t> ord(fsegs.size());
    for (size_t q = 0; q < ord.size(); ++q) ord[q] = q;
    std::sort(ord.begin(), ord.end(), [&](size_t x, size_t y) {
      return group[x] != group[y] ? group[x] < group[y] : fsegs[x].ptr < fsegs[y].ptr;
    });
    std::vector<Seg> fs(ord.size());
    std::vector<int> gs(ord.size());
    for (size_t q = 0; q < ord.size(); ++q) {
      fs[q] = fsegs[ord[q]];
      gs[q] = group[ord[q]];
    }
    fsegs.swap(fs);
    group.swap(gs);
  }
  for (auto &sg : fsegs) sg.shadow = C->begin_shadow(sg.ptr, sg.n);  // for unmapArrays / releaseArrays
  uint64_t tr = 0, nl = 0;
  int r = C->map_core(fsegs, {}, &tr, &nl, &group, &pack_ev);
  for (auto &sg : fsegs)
    if (sg.shadow) C->commit_shadow(sg.ptr, sg.n, r == CGCM_OK);
  if (r != CGCM_OK) {
    if (rev_done) C->rev_decref(rsegs);
    for (auto &b : backups)
      cudaMemcpyAsync(reinterpret_cast<void *>(b.dst), reinterpret_cast<void *>(b.src), b.n, cudaMemcpyDeviceToDevice,
                      C->main);
    undo_prologue();
    return r;
  }
  if (rev_done) {
    C->st.fwd_translations += rres.hits;
    C->st.null_slots += rres.nulls;
    if (C->flags & CGCM_LENIENT) C->st.passthrough += rres.misses;
  }
  for (auto &o : outs) C->uarr[o.unit] = 1;
  if (!rev_done)  // every outer of the call was translated from its host slots just now
    for (auto &o : outs) C->arr_gen[o.info.base] = C->free_gen;
  else
    for (auto &sg : fsegs)
      for (auto &o : outs)
        if (C->udev[o.unit] == sg.ptr) C->arr_gen[o.info.base] = C->free_gen;
  for (size_t j = 0; j < k; ++j) {
    const Outer &o = outs[which[j]];
    uint64_t dev = C->udev[o.unit];
    gpu_out[j] = reinterpret_cast<void **>(dev + (reinterpret_cast<uint64_t>(arrays[j]) - o.info.base));
  }
  return CGCM_OK;
}

int cgcm_unmapArrays(void *const *const *arrays, size_t k) {
  CTXM();
  if (k == 0) return CGCM_OK;
  if (!arrays) return CGCM_E_INVALID;
  std::vector<PointInfo> infos;
  CKS(C->lookup_points(reinterpret_cast<const uint64_t *>(arrays), k, infos));
  std::vector<Outer> outs;
  std::vector<int> which;
  CKS(distinct_outers(infos, outs, which));
  for (auto &o : outs)
    if (o.info.refcount <= 0) return CGCM_E_NOT_MAPPED;
  CKS(C->ensure_rev());
  // prologue: every outer's epoch becomes current first, so that self-references and outers that
  // are elements of other outers are not copied twice (A12)
  std::vector<UnitOp> ops;
  std::vector<Journal> outer_jn;
  struct OC { int unit; uint64_t stage; };
  std::vector<OC> outer_copies;
  std::vector<Seg> rsegs_copy, rsegs_gate, fsegs_gate;
  uint64_t stage_bytes = 0;
  for (auto &o : outs) {
    const uint32_t cur = C->rel_epoch(C->epoch);
    bool copy_o = o.info.epoch != cur && !(o.info.flags & UF_READONLY);
    if (o.info.epoch != cur) {
      ops.push_back({(uint32_t)o.unit, UOP_SET_EPOCH, cur});
      outer_jn.push_back({(uint32_t)o.info.epoch, (uint32_t)o.unit, 0, 0});
    }
    uint64_t n = o.info.size / 8;
    if (copy_o) {
      outer_copies.push_back({o.unit, 0});
      if (o.info.flags & UF_ARRAYMAPPED) stage_bytes += align_up(8 * n, 32) + 64;
    }
  }
  CKS(C->dalloc(C->staging2, stage_bytes + 256));
  uint64_t off = C->staging2.addr;
  for (auto &oc : outer_copies) {
    auto &o = *std::find_if(outs.begin(), outs.end(), [&](const Outer &x) { return x.unit == oc.unit; });
    uint64_t n = o.info.size / 8;
    if (o.info.flags & UF_ARRAYMAPPED) {
      off = align_up(off, 32) + (o.info.devbase & 31);
      oc.stage = off;
      off += 8 * n;
    }
  }
  for (auto &o : outs) {
    uint64_t n = o.info.size / 8;
    if (!n) continue;
    auto oc = std::find_if(outer_copies.begin(), outer_copies.end(), [&](const OC &x) { return x.unit == o.unit; });
    if (o.info.flags & UF_ARRAYMAPPED) {
      const uint64_t sh = C->find_shadow(o.info.devbase, n);  // the device copy still holds what the map wrote
      if (oc != outer_copies.end()) rsegs_copy.push_back(Seg{o.info.devbase, n, oc->stage, 1, 0, sh});
      else rsegs_gate.push_back(Seg{o.info.devbase, n, 0, 1, 0, sh});
    } else {
      fsegs_gate.push_back(Seg{o.info.devbase, n, 0, 1, 0});  // raw CPU pointers (scalar-mapped outer)
    }
  }
  CKS(C->unit_ops(ops));
  uint64_t total = 0;
  for (auto &o : outs) total += o.info.size / 8;
  CKS(C->prepare(total + 64));
  SlotCall A, B, F;
  A.dir = DIR_REV; A.ops = OP_WRITE | OP_GATE | OP_HITMASK; A.segs = rsegs_copy;
  B.dir = DIR_REV; B.ops = OP_GATE; B.segs = rsegs_gate;
  F.dir = DIR_FWD; F.ops = OP_GATE | OP_CHECKMAPPED; F.segs = fsegs_gate;
  CKS(C->launch(A, 0, false, false, true));
  CKS(C->launch(B, 1));
  CKS(C->launch(F, 2));
  Status sts[8];
  unsigned long long lcs[4];
  CKS(C->fetch_status(sts, lcs));
  bool strict = !(C->flags & CGCM_LENIENT);
  int err = CGCM_OK;
  if ((sts[0].misses || sts[2].misses) && strict) err = CGCM_E_UNREGISTERED;
  else if (sts[2].notmapped || (sts[1].misses && strict)) err = CGCM_E_NOT_MAPPED;
  // element copy-backs (array-mapped elements are reverse translated and validated first, into
  // their own staging buffer); the outers' staged slots are copied below
  if (!err) err = C->copy_back_list(C->copy_list, lcs[3]);
  if (err) {
    SlotCall none;
    C->undo_rev(none, lcs[1], outer_jn, false, false);
    return err;
  }
  for (auto &oc : outer_copies) {
    auto &o = *std::find_if(outs.begin(), outs.end(), [&](const Outer &x) { return x.unit == oc.unit; });
    uint64_t n = o.info.size / 8;
    if (o.info.flags & UF_ARRAYMAPPED) {
      if (n) CK(cudaMemcpyAsync(reinterpret_cast<void *>(o.info.base), reinterpret_cast<void *>(oc.stage), 8 * n,
                                cudaMemcpyDeviceToHost, C->main));
      if (o.info.size > 8 * n)
        CK(cudaMemcpyAsync(reinterpret_cast<void *>(o.info.base + 8 * n),
                           reinterpret_cast<void *>(o.info.devbase + 8 * n), o.info.size - 8 * n,
                           cudaMemcpyDeviceToHost, C->main));
      C->st.d2h_memcpy_calls += 1 + (o.info.size > 8 * n);
    } else {
      CK(cudaMemcpyAsync(reinterpret_cast<void *>(o.info.base), reinterpret_cast<void *>(o.info.devbase), o.info.size,
                         cudaMemcpyDeviceToHost, C->main));
      C->st.d2h_memcpy_calls += 1;
    }
    C->st.d2h_units += 1;
    C->st.d2h_bytes += o.info.size;
  }
  CK(cudaStreamSynchronize(C->main));
  C->st.rev_translations += sts[0].translated;
  if (!strict) C->st.passthrough += sts[0].misses;
  return CGCM_OK;
}

int cgcm_releaseArrays(void *const *const *arrays, size_t k) {
  CTXM();
  if (k == 0) return CGCM_OK;
  if (!arrays) return CGCM_E_INVALID;
  {  // the release that matches a queued re-map (a lease): no host wait at all
    const int r = C->release_arrays_async(reinterpret_cast<const uint64_t *>(arrays), k);
    if (r != 1) return r;  // 1: not that case, take the general path
  }
  std::vector<PointInfo> infos;
  CKS(C->lookup_points(reinterpret_cast<const uint64_t *>(arrays), k, infos));
  std::vector<Outer> outs;
  std::vector<int> which;
  CKS(distinct_outers(infos, outs, which));
  for (auto &o : outs)
    if (o.info.refcount < o.mult) return CGCM_E_NOT_MAPPED;
  std::vector<Seg> rsegs, fsegs;
  for (auto &o : outs) {
    uint64_t n = o.info.size / 8;
    if (!n) continue;
    Seg s{o.info.devbase, n, 0, o.mult, 0};
    if (o.info.flags & UF_ARRAYMAPPED) {
      s.shadow = C->find_shadow(o.info.devbase, n);
      rsegs.push_back(s);
    } else {
      fsegs.push_back(s);
    }
  }
  if (!rsegs.empty()) CKS(C->ensure_rev());
  // the outers' own references go first (plain decrement); slot decrements detect underflow / zero
  std::vector<UnitOp> ops;
  std::vector<uint32_t> outer_zero;
  for (auto &o : outs) {
    ops.push_back({(uint32_t)o.unit, UOP_ADD_RC, (uint64_t)(int64_t)(-o.mult)});
    if (o.info.refcount == o.mult) outer_zero.push_back((uint32_t)o.unit);
  }
  CKS(C->unit_ops(ops));
  uint64_t total = 0;
  for (auto &o : outs) total += o.info.size / 8;
  CKS(C->prepare(total + 64));
  SlotCall R, F;
  R.dir = DIR_REV; R.ops = OP_DEC; R.segs = rsegs;
  F.dir = DIR_FWD; F.ops = OP_DEC; F.segs = fsegs;
  R.dec_red = F.dec_red = total >= (uint64_t)C->U / 8 && C->U >= 4096;
  CKS(C->launch(R, 0));
  CKS(C->launch(F, 1));
  Status sts[8];
  unsigned long long lcs[4];
  CKS(C->fetch_status(sts, lcs));
  bool strict = !(C->flags & CGCM_LENIENT);
  int err = CGCM_OK;
  if (sts[1].misses && strict) err = CGCM_E_UNREGISTERED;
  else if (sts[0].underflow || sts[1].underflow || (sts[0].misses && strict)) err = CGCM_E_NOT_MAPPED;
  if (err) {
    CKS(C->prepare_small());
    SlotCall r2, f2;
    r2.dir = DIR_REV; r2.ops = OP_INCPLAIN; r2.segs = rsegs;
    f2.dir = DIR_FWD; f2.ops = OP_INCPLAIN; f2.segs = fsegs;
    CKS(C->launch(r2, 0));
    CKS(C->launch(f2, 1));
    std::vector<UnitOp> undo;
    for (auto &o : outs) undo.push_back({(uint32_t)o.unit, UOP_ADD_RC, (uint64_t)(int64_t)o.mult});
    CKS(C->unit_ops(undo));
    CK(cudaStreamSynchronize(C->main));
    return err;
  }
  // an outer reaches 0 through its own decrement only if no slot pointed into it; outers whose zero came
  // from a slot decrement are in the list too (duplicates are freed once); outers with remaining slot
  // refs into them (self-reference) cannot be in outer_zero (their refcount exceeded mult)
  return C->free_units_list(C->free_list, lcs[2], outer_zero);
}

// ---- map-promotion regions (NEXT-2) ----
int cgcm_regionBegin(void *const *ptrs, const unsigned *kinds, size_t n, unsigned flags) {
  CTXM();
  if (C->region_open) return CGCM_E_BUSY;
  if (n && (!ptrs || !kinds)) return CGCM_E_INVALID;
  const bool check = (flags & CGCM_REGION_CHECK) != 0;
  if (check && g_nprot.load() > 0) return CGCM_E_BUSY;  // one checked region per process
  for (size_t i = 0; i < n; ++i)
    if (kinds[i] > CGCM_REGION_MAPARRAY) return CGCM_E_INVALID;
  // the hoisted maps (Listing 4: map/mapArray before the loop)
  size_t done = 0;
  int err = CGCM_OK;
  for (; done < n && err == CGCM_OK; ++done) {
    const void *p = ptrs[done];
    if (kinds[done] == CGCM_REGION_MAP) {
      void *out = nullptr;
      err = cgcm_mapBatch(&p, 1, &out);
    } else {
      void **out = nullptr;
      void *const *pp = reinterpret_cast<void *const *>(p);
      err = cgcm_mapArrays(&pp, 1, &out);
    }
  }
  auto undo = [&](size_t k) {
    for (size_t i = k; i-- > 0;) {
      const void *p = ptrs[i];
      if (kinds[i] == CGCM_REGION_MAP) {
        cgcm_releaseBatch(&p, 1);
      } else {
        void *const *pp = reinterpret_cast<void *const *>(p);
        cgcm_releaseArrays(&pp, 1);
      }
    }
  };
  if (err != CGCM_OK) {
    undo(done - 1);
    return err;
  }
  if (check) {  // the host pages of every promoted AU (array outers and the AUs their slots point into)
    std::vector<std::pair<uint64_t, uint64_t>> au;
    auto unit_of = [&](uint64_t q) {
      auto it = C->reg.upper_bound(q);
      if (it == C->reg.begin()) return;
      --it;
      if (q - it->first <= it->second.size) au.push_back({it->first, it->first + it->second.size});
    };
    for (size_t i = 0; i < n; ++i) {
      const uint64_t p = reinterpret_cast<uint64_t>(ptrs[i]);
      unit_of(p);
      if (kinds[i] == CGCM_REGION_MAPARRAY && !au.empty()) {
        const uint64_t b = au.back().first, e = au.back().second;
        for (uint64_t w = b; w + 8 <= e; w += 8) {
          uint64_t v;
          std::memcpy(&v, reinterpret_cast<const void *>(w), 8);
          if (v) unit_of(v);
        }
      }
    }
    g_pagesz = (uintptr_t)sysconf(_SC_PAGESIZE);
    std::vector<ProtRange> rr;
    for (auto &x : au) rr.push_back({x.first & ~(g_pagesz - 1), (x.second + g_pagesz - 1) & ~(g_pagesz - 1)});
    std::sort(rr.begin(), rr.end(), [](const ProtRange &a, const ProtRange &b) { return a.lo < b.lo; });
    std::vector<ProtRange> m;
    for (auto &r : rr) {
      if (r.hi <= r.lo) continue;
      if (!m.empty() && r.lo <= m.back().hi)
        m.back().hi = std::max(m.back().hi, r.hi);
      else
        m.push_back(r);
    }
    if (m.size() > (size_t)PROT_MAX) {
      undo(n);
      return CGCM_E_NOMEM;
    }
    if (!g_segv_installed) {
      struct sigaction sa;
      std::memset(&sa, 0, sizeof(sa));
      sa.sa_sigaction = on_segv;
      sa.sa_flags = SA_SIGINFO;
      sigemptyset(&sa.sa_mask);
      if (sigaction(SIGSEGV, &sa, &g_old_segv) != 0) {
        undo(n);
        return CGCM_E_INVALID;
      }
      g_segv_installed = true;
    }
    for (size_t i = 0; i < m.size(); ++i) g_prot[i] = m[i];
    g_viol.store(0);
    g_viol_first.store(0);
    g_nprot.store((int)m.size(), std::memory_order_release);
    for (size_t i = 0; i < m.size(); ++i)
      if (mprotect(reinterpret_cast<void *>(m[i].lo), m[i].hi - m[i].lo, PROT_NONE) != 0) {
        g_last_cuda_error = std::string("mprotect: ") + std::strerror(errno);
        for (size_t k = 0; k < i; ++k)
          mprotect(reinterpret_cast<void *>(m[k].lo), m[k].hi - m[k].lo, PROT_READ | PROT_WRITE);
        g_nprot.store(0);
        undo(n);
        return CGCM_E_INVALID;
      }
  }
  C->region.clear();
  for (size_t i = 0; i < n; ++i) C->region.push_back({reinterpret_cast<uint64_t>(ptrs[i]), kinds[i]});
  C->region_open = true;
  C->region_checked = check;
  return CGCM_OK;
}
int cgcm_regionEnd(size_t *violations) {
  CTXM();
  if (!C->region_open) return CGCM_E_INVALID;
  unsigned long long v = 0;
  if (C->region_checked) {  // reopen every page before the copy-backs write host memory
    const int np = g_nprot.exchange(0);
    for (int i = 0; i < np; ++i)
      mprotect(reinterpret_cast<void *>(g_prot[i].lo), g_prot[i].hi - g_prot[i].lo, PROT_READ | PROT_WRITE);
    v = g_viol.exchange(0);
  }
  // the hoisted unmaps and releases (Listing 4 after the loop, A11), in reverse order
  int err = CGCM_OK;
  for (size_t i = C->region.size(); i-- > 0;) {
    const void *p = reinterpret_cast<const void *>(C->region[i].first);
    int s1, s2;
    if (C->region[i].second == CGCM_REGION_MAP) {
      s1 = cgcm_unmapBatch(&p, 1);
      s2 = cgcm_releaseBatch(&p, 1);
    } else {
      void *const *pp = reinterpret_cast<void *const *>(p);
      s1 = cgcm_unmapArrays(&pp, 1);
      s2 = cgcm_releaseArrays(&pp, 1);
    }
    if (err == CGCM_OK) err = s1 != CGCM_OK ? s1 : s2;
  }
  C->region.clear();
  C->region_open = false;
  C->region_checked = false;
  if (violations) *violations = (size_t)v;
  if (err != CGCM_OK) return err;
  return v ? CGCM_E_MODREF : CGCM_OK;
}

int cgcm_mapArray(void *const *cpu, void ***gpu_out) {
  if (!gpu_out) return CGCM_E_INVALID;
  void **out = nullptr;
  int s = cgcm_mapArrays(&cpu, 1, &out);
  if (s == CGCM_OK) *gpu_out = out;
  return s;
}
int cgcm_unmapArray(void *const *cpu) { return cgcm_unmapArrays(&cpu, 1); }
int cgcm_releaseArray(void *const *cpu) { return cgcm_releaseArrays(&cpu, 1); }

int cgcm_advanceEpochs(uint64_t n) {
  CTX();
  if (n >= 0xFFFFFFE0ull) return CGCM_E_INVALID;
  if (C->epoch + n - C->origin >= 0xFFFFFFF0ull) {  // move the u32 epoch origin (A28)
    CKS(C->ensure_table());
    launch_rebase_epochs(C->tab(), C->U, C->rel_epoch(C->epoch), C->main);
    CK(cudaStreamSynchronize(C->main));
    C->origin = C->epoch - 1;
  }
  C->epoch += n;  // "increases every time the program launches a GPU function"
  return CGCM_OK;
}
int cgcm_advanceEpoch(void) { return cgcm_advanceEpochs(1); }
uint64_t cgcm_epoch(void) {
  Context *C = tl_ctx;
  return C ? C->epoch : 0;
}

// ---- introspection ------------------------------------------------------------------------------
int cgcm_stats(cgcm_stats_t *out) {
  CTX();
  if (!out) return CGCM_E_INVALID;
  CKS(C->fold_lazy());
  *out = C->st;
  return CGCM_OK;
}
int cgcm_resetStats(void) {
  CTX();
  CKS(C->fold_lazy());
  std::memset(&C->st, 0, sizeof(C->st));
  return CGCM_OK;
}
int cgcm_dumpTable(cgcm_unit_t *out, size_t cap, size_t *n) {
  CTX();
  CKS(C->ensure_table());
  if (n) *n = (size_t)C->U;
  if (!out || cap == 0) return (size_t)C->U <= cap ? CGCM_OK : CGCM_E_NOMEM;
  std::vector<uint64_t> hots, sts;
  std::vector<int32_t> rcs;
  std::vector<uint64_t> szs;
  CKS(C->download(hots, C->hotb, (size_t)C->U));
  CKS(C->download(sts, C->stb, (size_t)C->U));
  if (C->any_deferred) {
    // refcounts as the paper defines them (deferred references included), without changing any state:
    // the deferred references are added to a copy of rc (observing must not change the execution path)
    CKS(C->dalloc(C->dump_rc, 4 * (size_t)C->U + 64));
    CK(cudaMemcpyAsync(C->dump_rc.as<void>(), C->rcb.as<void>(), 4 * (size_t)C->U, cudaMemcpyDeviceToDevice, C->main));
    for (auto &kv : C->shadows)
      if (kv.second.deferred)
        launch_materialise(reinterpret_cast<const uint64_t *>(kv.second.buf.addr), kv.first.second,
                           C->dump_rc.as<int32_t>(), C->main);
    CK(cudaGetLastError());
    CKS(C->download(rcs, C->dump_rc, (size_t)C->U));
  } else {
    CKS(C->download(rcs, C->rcb, (size_t)C->U));
  }
  CKS(C->download(szs, C->size64, (size_t)C->U));
  // in base order: the registry's order (delta units sit at ids >= Umain, NEXT-1)
  std::vector<uint32_t> order;
  order.reserve(C->U);
  for (auto &kv : C->reg) order.push_back((uint32_t)kv.second.idx);
  size_t m = std::min(cap, (size_t)C->U);
  for (size_t q = 0; q < m; ++q) {
    const size_t i = order[q];
    cgcm_unit_t &u = out[q];
    const uint32_t fl = hot_flags(hots[i]);
    u.base = C->ubase[i];
    u.size = szs[i];
    bool act = rcs[i] > 0;
    uint32_t e = hot_ext(hots[i]);
    u.devptr = ((fl & UF_STORAGE) && (act || (fl & UF_GLOBAL)) && e < C->runs.size())
                   ? u.base - C->runs[e].delta
                   : 0;
    u.refCount = rcs[i];
    u.epoch = C->origin + st_epoch(sts[i]);
    u.flags = ((fl & UF_GLOBAL) ? CGCM_UNIT_GLOBAL : 0) | ((fl & UF_READONLY) ? CGCM_UNIT_READONLY : 0) |
              ((fl & UF_ARRAYMAPPED) ? CGCM_UNIT_ARRAYMAPPED : 0) | (act ? CGCM_UNIT_ACTIVE : 0);
    u.pad = 0;
  }
  return (size_t)C->U <= cap ? CGCM_OK : CGCM_E_NOMEM;
}
int cgcm_arenaUsage(size_t *used, size_t *capacity) {
  CTX();
  if (used) *used = C->arena.used();
  if (capacity) *capacity = C->arena.capacity();
  return CGCM_OK;
}

// ---- glue kernels (NEXT-4) --------------------------------------------------------------
int cgcm_launchGlue(const cgcm_glue_op_t *prog, size_t n, const void *const *cpu_ptrs, size_t nptrs,
                    uint64_t max_steps, uint64_t *regs_out) {
  CTXM();
  static_assert(sizeof(cgcm_glue_op_t) == sizeof(GlueOp), "glue op layout");
  if ((!prog && n) || n > (1u << 20) || nptrs > (size_t)GLUE_REGS || (nptrs && !cpu_ptrs)) return CGCM_E_INVALID;
  std::vector<uint64_t> regs(GLUE_REGS, 0);
  if (nptrs) {  // Alg. 1's translation of each pointer into its (already mapped) unit's device copy
    std::vector<PointInfo> info;
    std::vector<uint64_t> nz;
    for (size_t i = 0; i < nptrs; ++i)
      if (cpu_ptrs[i]) nz.push_back(reinterpret_cast<uint64_t>(cpu_ptrs[i]));
    if (!nz.empty()) CKS(C->lookup_points(nz.data(), nz.size(), info));
    size_t k = 0;
    for (size_t i = 0; i < nptrs; ++i) {
      if (!cpu_ptrs[i]) continue;
      const PointInfo &pi = info[k++];
      if (pi.unit < 0) return CGCM_E_UNREGISTERED;
      if (pi.refcount <= 0 || !(pi.flags & UF_STORAGE)) return CGCM_E_NOT_MAPPED;
      regs[i] = pi.devbase + (reinterpret_cast<uint64_t>(cpu_ptrs[i]) - pi.base);
    }
  }
  CKS(C->ensure_rev());
  std::vector<GlueOp> ops(n);
  if (n) std::memcpy(ops.data(), prog, n * sizeof(GlueOp));
  if (ops.empty()) ops.push_back(GlueOp{13, 0, 0, 0, 0});
  CKS(C->upload(C->glue_prog, ops));
  CKS(C->upload(C->glue_regs, regs));
  CKS(C->dalloc(C->glue_status, 64));
  GlueArgs g;
  g.prog = C->glue_prog.as<GlueOp>();
  g.n = (int)n;
  g.regs = C->glue_regs.as<uint64_t>();
  g.max_steps = max_steps;
  g.status = C->glue_status.as<int>();
  g.tab = C->tab();
  g.ext_keys = C->rev.keys.as<uint64_t>();
  g.ext_pay = C->rev.pay.as<uint64_t>();
  g.ext_id = C->rev.rid.as<uint32_t>();
  g.n_ext_keys = (int)C->live_runs.size();
  g.U = C->Umain;
  g.dkeys = C->dkeys.as<uint64_t>();
  g.dids = C->dids.as<uint32_t>();
  g.dn = (int)C->dk.size();
  launch_glue(g, C->main);
  C->st.kernel_launches += 1;
  CK(cudaGetLastError());
  std::vector<int> st;
  CKS(C->download(st, C->glue_status, 2));
  if (regs_out) {
    std::vector<uint64_t> ro;
    CKS(C->download(ro, C->glue_regs, GLUE_REGS));
    std::memcpy(regs_out, ro.data(), 8 * GLUE_REGS);
  }
  return st[0];
}

int cgcm_dumpExtents(cgcm_extent_t *out, size_t cap, size_t *n) {
  CTX();
  if (!n) return CGCM_E_INVALID;
  *n = C->live_runs.size();
  if (cap < *n) return out || cap ? CGCM_E_NOMEM : CGCM_OK;
  size_t k = 0;
  for (auto &kv : C->live_runs) {
    const Run &r = C->runs[kv.second];
    cgcm_extent_t e{};
    e.addr = r.addr;
    e.bytes = r.bytes;
    e.live = r.live;
    e.external = r.external ? 1u : 0u;
    out[k++] = e;
  }
  return CGCM_OK;
}

int cgcm_storageInfo(cgcm_storage_t *out) {
  CTX();
  if (!out) return CGCM_E_INVALID;
  std::memset(out, 0, sizeof(*out));
  for (auto &kv : C->live_runs) {
    const Run &r = C->runs[kv.second];
    if (r.external) {
      out->external_extents += 1;
    } else {
      out->extents += 1;
      out->extent_bytes += r.bytes;
    }
  }
  for (auto &kv : C->shadows) {
    if (kv.second.valid) {
      out->shadows_live += 1;
      out->shadow_live_bytes += kv.second.buf.bytes;
    } else {
      out->shadows_cached += 1;
      out->shadow_cached_bytes += kv.second.buf.bytes;
    }
  }
  out->arena_used = C->arena.used();
  out->arena_capacity = C->arena.capacity();
  return CGCM_OK;
}

int cgcm_indexInfo(cgcm_index_info_t *out) {
  CTX();
  if (!out) return CGCM_E_INVALID;
  CKS(C->ensure_table());
  std::memset(out, 0, sizeof(*out));
  out->units = (uint64_t)C->U;
  out->levels = (uint32_t)C->fwd.h;
  out->pd_segments = (uint32_t)C->pd_nseg;
  out->pd_pages = C->pd_pages;
  out->pd_overflow_pages = C->pd_ovf_pages;
  out->pd_bytes = C->pd_bytes;
  out->pd_min_shift = C->pd_minP;
  out->pd_max_shift = C->pd_maxP;
  out->pd_format = C->pd_nseg ? (C->pd_v3 ? 3u : 2u) : 0u;
  return CGCM_OK;
}

}  // extern "C"
