// kernels.cu -- sm_100a kernels of the CGCM hot path.
//
//   k_slots<DIR, OPS>   the per-pointer kernel.  a1: interval lookup (greatestLTE of P:L169-170)
//                       over the sorted AU bases: shared-memory radix directory + top splitters,
//                       then h 32-byte sector levels of u32 keys, then one 16-byte record gather.
//                       Then any of a2 forward rewrite + refcount (Alg. 1), a3 reverse rewrite,
//                       a4 epoch gate (Alg. 2), release (Alg. 3).  Reverse lookups find the device
//                       extent (mirrored layout: one host-device delta per extent, shared memory),
//                       then run the forward lookup on the host address and verify it.
//                       Pointer arrays stream through 128-bit loads/stores with an L2 evict-first
//                       policy so the table stays L2-resident; 2 slots per thread per step.
//   k_build_level       u32 sector levels of an index (a0, off the per-pointer path).
//   small kernels       activation bookkeeping, rollback, release scan, outer-pointer lookup.
// DESIGN.md §7 gives the roofline of each kernel and its algorithmic bytes.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdlib>

#include "cgcm_dev.h"

namespace cgcm {

namespace {

constexpr int SEG_SMEM = 256;

__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// two pointer slots, streamed (no L1 allocation, L2 evict-first)
__device__ __forceinline__ void ld_stream2(const void *p, uint64_t pol, uint64_t &a, uint64_t &b) {
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
               : "=l"(a), "=l"(b)
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ void st_stream2(void *p, uint64_t pol, uint64_t a, uint64_t b) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(p), "l"(a), "l"(b),
               "l"(pol)
               : "memory");
}
__device__ __forceinline__ void st_stream1(void *p, uint64_t pol, uint64_t v) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(pol) : "memory");
}
// index / record gathers, kept in L2 (evict-last)
__device__ __forceinline__ void ld_sector(const void *p, uint64_t pol, uint64_t v[4]) {
  asm volatile("ld.global.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld_pair(const void *p, uint64_t pol, uint64_t &a, uint64_t &b) {
  asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(a), "=l"(b) : "l"(p), "l"(pol));
}
__device__ __forceinline__ uint64_t ld_u64(const uint64_t *p, uint64_t pol) {
  uint64_t v;
  asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
  return v;
}
// unit-word gathers of the hot kernels (random: no L1 reuse)
__device__ __forceinline__ uint64_t ld_u64_hot(const uint64_t *p, uint64_t pol) {
  uint64_t v;
#ifdef CGCM_HOT_NOL1
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
#else
  asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
#endif
  return v;
}
__device__ __forceinline__ void red_add(int32_t *p, int32_t v) {
  asm volatile("red.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// warp-aggregated append (the whole warp executes it): this lane's slot in the list if pred
__device__ __forceinline__ unsigned long long warp_append(unsigned long long *counter, bool pred) {
  unsigned want = __ballot_sync(0xffffffffu, pred);
  unsigned long long base = 0;
  if (want) {
    int leader = __ffs(want) - 1;
    if ((int)(threadIdx.x & 31) == leader) base = atomicAdd(counter, (unsigned long long)__popc(want));
    base = __shfl_sync(0xffffffffu, base, leader);
  }
  return base + __popc(want & lanemask_lt());
}
__device__ __forceinline__ void flush_count(unsigned long long *dst, unsigned long long v) {
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
}
// interleave the low 16 bits of x with zeros (bit i -> bit 2i)
__device__ __forceinline__ uint32_t spread16(uint32_t x) {
  x &= 0xFFFFu;
  x = (x | (x << 8)) & 0x00FF00FFu;
  x = (x | (x << 4)) & 0x0F0F0F0Fu;
  x = (x | (x << 2)) & 0x33333333u;
  x = (x | (x << 1)) & 0x55555555u;
  return x;
}

// Position of the largest entry <= r among the 8 sorted u32 of one 32-byte level sector (entry 0 is
// always <= r on a lookup path: every group starts at its parent's key).  Branch-free 3-step binary
// search (3 compares + 3 selects) instead of 8 compares; last8 returns the entry itself (bottom level).
__device__ __forceinline__ int idx8(const uint64_t w[4], uint32_t r) {
  const bool b4 = (uint32_t)w[2] <= r;                                // entry 4
  const bool b2 = (uint32_t)(b4 ? w[3] : w[1]) <= r;                  // entry 6 or 2
  const uint64_t wq = b4 ? (b2 ? w[3] : w[2]) : (b2 ? w[1] : w[0]);  // entries (i, i+1), i = 4*b4 + 2*b2
  const bool b1 = (uint32_t)(wq >> 32) <= r;
  return (b4 ? 4 : 0) + (b2 ? 2 : 0) + (b1 ? 1 : 0);
}
__device__ __forceinline__ uint32_t last8(const uint64_t w[4], int i) {
  const uint64_t wq = (i & 4) ? ((i & 2) ? w[3] : w[2]) : ((i & 2) ? w[1] : w[0]);
  return (i & 1) ? (uint32_t)(wq >> 32) : (uint32_t)wq;
}
// number of entries <= r among 8 sorted u32 (one 32-byte level sector), and the largest of them
__device__ __forceinline__ int count8(const uint64_t w[4], uint32_t r, uint32_t &last) {
  int c = 0;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint32_t lo = (uint32_t)w[q], hi = (uint32_t)(w[q] >> 32);
    if (lo <= r) last = lo;
    if (hi <= r) last = hi;
    c += (lo <= r);
    c += (hi <= r);
  }
  return c;
}
// ---- an index's top level, staged in shared memory -------------------------------------------
struct SIdx {
  const uint64_t *top;
  const uint32_t *dir;
  const uint32_t *wide;
  const uint64_t *skmin;
  const uint32_t *smeta;
  const uint64_t *pay;  // reverse index with h == 0: per-extent delta, staged
  const uint32_t *rid;  // ... and the extent ids
  int ntop, nseg;
  uint64_t kfirst;
};

__host__ __device__ __forceinline__ size_t al16(size_t x) { return (x + 15) & ~size_t(15); }
__host__ __device__ __forceinline__ size_t stage_bytes(const IndexDev &ix, bool with_pay) {
  size_t b = al16(8 * (size_t)ix.ntop) + al16(4 * (size_t)ix.ndir) + al16(4 * (size_t)((ix.ntop + 31) / 32)) +
             al16(8 * (size_t)ix.nseg) + al16(16 * (size_t)ix.nseg);
  if (with_pay) b += al16(8 * (size_t)ix.ntop) + al16(4 * (size_t)ix.ntop);
  return b;
}

__device__ __forceinline__ unsigned char *stage(const IndexDev &ix, const uint64_t *pay, const uint32_t *rid,
                                                unsigned char *base, SIdx &S) {
  uint64_t *top = reinterpret_cast<uint64_t *>(base);
  base += al16(8 * (size_t)ix.ntop);
  uint32_t *dir = reinterpret_cast<uint32_t *>(base);
  base += al16(4 * (size_t)ix.ndir);
  uint32_t *wide = reinterpret_cast<uint32_t *>(base);
  base += al16(4 * (size_t)((ix.ntop + 31) / 32));
  uint64_t *skmin = reinterpret_cast<uint64_t *>(base);
  base += al16(8 * (size_t)ix.nseg);
  uint32_t *smeta = reinterpret_cast<uint32_t *>(base);
  base += al16(16 * (size_t)ix.nseg);
  uint64_t *spay = nullptr;
  uint32_t *srid = nullptr;
  if (pay) {
    spay = reinterpret_cast<uint64_t *>(base);
    base += al16(8 * (size_t)ix.ntop);
    srid = reinterpret_cast<uint32_t *>(base);
    base += al16(4 * (size_t)ix.ntop);
  }
  for (int t = threadIdx.x; t < ix.ntop; t += blockDim.x) top[t] = ix.top[t];
  for (int t = threadIdx.x; t < ix.ndir; t += blockDim.x) dir[t] = ix.dir[t];
  for (int t = threadIdx.x; t < (ix.ntop + 31) / 32; t += blockDim.x) wide[t] = ix.wide[t];
  for (int t = threadIdx.x; t < ix.nseg; t += blockDim.x) skmin[t] = ix.seg_kmin[t];
  for (int t = threadIdx.x; t < 4 * ix.nseg; t += blockDim.x) smeta[t] = ix.seg_meta[t];
  if (pay)
    for (int t = threadIdx.x; t < ix.ntop; t += blockDim.x) {
      spay[t] = pay[t];
      srid[t] = rid[t];
    }
  S.top = top;
  S.dir = dir;
  S.wide = wide;
  S.skmin = skmin;
  S.smeta = smeta;
  S.pay = spay;
  S.rid = srid;
  S.ntop = ix.ntop;
  S.nseg = ix.nseg;
  S.kfirst = ix.ntop > 0 ? ix.top[0] : ~0ull;
  return base;
}

// greatest t with top[t] <= p (-1 if p < top[0]); tk = top[t].  ONESEG: the index has one segment.
template <bool ONESEG = false>
__device__ __forceinline__ int top_search(const SIdx &S, uint64_t p, uint64_t &tk) {
  if (p < S.kfirst) return -1;
  int sg = 0;
  if (!ONESEG && S.nseg > 1) {
    int lo = 0, len = S.nseg;
    while (len > 1) {
      int half = len >> 1;
      if (S.skmin[lo + half] <= p) lo += half;
      len -= half;
    }
    sg = lo;
  }
  const uint32_t off = S.smeta[4 * sg], nb = S.smeta[4 * sg + 1], tend = S.smeta[4 * sg + 2],
                 sh = S.smeta[4 * sg + 3];
  uint64_t d = (p - S.skmin[sg]) >> sh;
  if (d >= nb) d = nb - 1;
  uint32_t first = S.dir[off + d];
  uint32_t last = (d + 1 < nb) ? S.dir[off + d + 1] : tend;
  uint32_t count = last - first;
  while (count > 0) {  // upper bound of p in top[first, last)
    uint32_t step = count >> 1, it = first + step;
    if (S.top[it] <= p) {
      first = it + 1;
      count -= step + 1;
    } else {
      count = step;
    }
  }
  int t = (int)first - 1;
  tk = S.top[t];
  return t;
}

// fixed-depth variant of level_lookup2 for indexes without wide buckets (the hot path)
template <int H>
__device__ __forceinline__ void level_lookup2_fixed(const IndexDev &ix, uint64_t pol, const uint64_t p[2], int j[2],
                                                    uint64_t key[2]) {
  uint32_t rel[2], last[2] = {0, 0};
  bool ok[2];
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    ok[m] = j[m] >= 0;
    uint64_t d = p[m] - key[m];
    rel[m] = d >= 0xFFFFFFFEull ? 0xFFFFFFFEu : (uint32_t)d;
    if (!ok[m]) j[m] = 0;
  }
#pragma unroll
  for (int k = H - 1; k >= 0; --k) {
    const uint32_t *L = ix.lvl[k];
    uint64_t w0[4], w1[4];
    ld_sector(L + 8 * (size_t)j[0], pol, w0);
    ld_sector(L + 8 * (size_t)j[1], pol, w1);
#ifdef CGCM_COUNT8_LINEAR
    j[0] = 8 * j[0] + count8(w0, rel[0], last[0]) - 1;
    j[1] = 8 * j[1] + count8(w1, rel[1], last[1]) - 1;
#else
    const int i0 = idx8(w0, rel[0]), i1 = idx8(w1, rel[1]);
    j[0] = 8 * j[0] + i0;
    j[1] = 8 * j[1] + i1;
    if (k == 0) {
      last[0] = last8(w0, i0);
      last[1] = last8(w1, i1);
    }
#endif
  }
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    key[m] += last[m];
    if (!ok[m]) j[m] = -1;
  }
}

// two interleaved greatestLTE lookups through the u32 sector levels.  In: j = t, key = top[t]
// from top_search (j < 0: no candidate).  Out: j = key index (or -1).
__device__ __forceinline__ void level_lookup2(const SIdx &S, const IndexDev &ix, uint64_t pol, const uint64_t p[2],
                                              int j[2], uint64_t key[2]) {
  if (ix.h == 0) return;
  uint32_t rel[2], last[2] = {0, 0};
  bool wide[2];
  int t0[2];
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    t0[m] = j[m];
    int tt = j[m] < 0 ? 0 : j[m];
    wide[m] = j[m] >= 0 && ((S.wide[tt >> 5] >> (tt & 31)) & 1u);
    uint64_t d = p[m] - key[m];
    rel[m] = d >= 0xFFFFFFFEull ? 0xFFFFFFFEu : (uint32_t)d;
    j[m] = tt;
  }
  for (int k = ix.h - 1; k >= 0; --k) {
    const uint32_t *L = ix.lvl[k];
    uint64_t w0[4], w1[4];
    ld_sector(L + 8 * (size_t)j[0], pol, w0);
    ld_sector(L + 8 * (size_t)j[1], pol, w1);
    j[0] = 8 * j[0] + count8(w0, rel[0], last[0]) - 1;
    j[1] = 8 * j[1] + count8(w1, rel[1], last[1]) - 1;
  }
  const int sh = 3 * ix.h;
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    key[m] += last[m];
    if (t0[m] < 0) {
      j[m] = -1;
    } else if (wide[m]) {  // bucket spanning >= 4 GiB: binary search over the full u64 keys
      int lo = t0[m] << sh, len = min(ix.n, (t0[m] + 1) << sh) - lo;
      while (len > 1) {
        int half = len >> 1;
        if (ix.keys[lo + half] <= p[m]) lo += half;
        len -= half;
      }
      j[m] = lo;
      key[m] = ix.keys[lo];
    }
  }
}

// ---- page directory (cgcm_dev.h PdDev): segment starts and metadata staged in shared memory ----
struct SPd {
  const uint64_t *start;  // [nseg] starts, then [nseg] ends
  const uint32_t *meta;
  int nseg;
};
__host__ __device__ __forceinline__ size_t pd_stage_bytes(const PdDev &pd) {
  return al16(16 * (size_t)pd.nseg) + al16(16 * (size_t)pd.nseg);
}
__device__ __forceinline__ unsigned char *stage_pd(const PdDev &pd, unsigned char *base, SPd &S) {
  uint64_t *st = reinterpret_cast<uint64_t *>(base);
  base += al16(16 * (size_t)pd.nseg);
  uint32_t *mt = reinterpret_cast<uint32_t *>(base);
  base += al16(16 * (size_t)pd.nseg);
  for (int t = threadIdx.x; t < 2 * pd.nseg; t += blockDim.x) st[t] = pd.seg_start[t];
  for (int t = threadIdx.x; t < 4 * pd.nseg; t += blockDim.x) mt[t] = pd.seg_meta[t];
  S.start = st;
  S.meta = mt;
  S.nseg = pd.nseg;
  return base;
}
// count and maximum of the u16 offsets <= r (r replicated in both halves) in one 32-bit word
__device__ __forceinline__ void cnt_max2(uint32_t w, uint32_t rr, uint32_t &cnt, uint32_t &mx) {
  const uint32_t m = __vcmpleu2(w, rr);
  cnt += __popc(m);
  mx = __vmaxu2(mx, w & m);
}

// ---- forward-map shadows (cgcm_dev.h make_shw) ----------------------------------------------------
// The CPU pointer an unchanged slot g reverses to, given its recorded shadow word and the unit's extent e
// (lo/len: the extent's device range), or 0 when g is not provably the recorded pointer's translation.
__device__ __forceinline__ uint64_t sh_reverse(uint64_t g, uint64_t shw, uint64_t delta, uint64_t lo, uint32_t len) {
  const uint64_t h = g - delta;  // mirrored layout: host = device - (devbase - base)
  return (g - lo < (uint64_t)len && (uint32_t)h == (uint32_t)shw) ? h : 0ull;
}

// ---- NEXT-1 delta units ---------------------------------------------------------------------------
// The delta unit with the greatest base <= q that contains q (A7: q - base <= size), or -1; base out.
__device__ __noinline__ int delta_hit(const uint64_t *dk, const uint32_t *di, int dn, const TableDev &tab, uint64_t q,
                                      uint64_t &base) {
  if (dn <= 0 || q < dk[0]) return -1;
  int lo = 0, len = dn;
  while (len > 1) {
    const int half = len >> 1;
    if (dk[lo + half] <= q) lo += half;
    len -= half;
  }
  const uint32_t id = di[lo];
  const uint64_t b = dk[lo];
  uint64_t sz = hot_size32(tab.hot[id]);
  if (sz == BIG_SIZE) sz = tab.size64[id];
  if (q - b > sz) return -1;
  base = b;
  return (int)id;
}
// After the main table's lookup of q missed: the delta unit containing q, if any.  (A delta unit that
// starts exactly where a main unit ends -- and so would win greatestLTE at that unit's one-past-the-end
// address, A7 -- never exists: such a declaration rebuilds the table, Context::delta_touches_main.)
__device__ __forceinline__ int delta_override(const SlotArgs &a, uint64_t q, bool hit, uint64_t &base) {
  if (a.dn <= 0 || hit) return -1;
  return delta_hit(a.dkeys, a.dids, a.dn, a.tab, q, base);
}

// #{starts <= r} among an entry's (at most PD_K = 5) candidates, and the candidate word (start | end << 16)
// of the last of them (k > 0).  The 64-bit words e[1..3] hold w[2..7]: lane 2 of e[1] and lanes 0, 2 of
// e[2], e[3] are starts; per lane 0x8000 + r - x keeps bit 15 iff x <= r and never borrows into the next
// lane (every lane < 0x8000: starts and ends are 15-bit, the state word of e[1] is masked off).
__device__ __forceinline__ uint32_t pd_count5(const uint64_t e[4], uint32_t r, uint32_t &word) {
  const uint32_t r2 = r | (r << 16);
  const uint64_t rg = ((uint64_t)r2 | ((uint64_t)r2 << 32)) | 0x8000800080008000ull;
  const uint32_t k = __popcll((rg - (e[1] & 0xFFFFFFFF00000000ull)) & 0x0000800000000000ull) +
                     __popcll((rg - e[2]) & 0x0000800000008000ull) + __popcll((rg - e[3]) & 0x0000800000008000ull);
  const uint64_t q = k <= 1 ? e[1] : (k <= 3 ? e[2] : e[3]);
  word = (k & 1) ? (uint32_t)(q >> 32) : (uint32_t)q;  // candidate k-1: w[3] (e1 hi), w[4] (e2 lo), ...
  return k;
}

// Front half of a page-directory lookup of host address q: the segment, the page, and the entry to
// gather (ok), or the tail of the segment's last unit (tail >= 0: that unit, -1: a miss).
struct PdFront {
  uint64_t A;      // the page's first address
  uint64_t e;      // entry index
  uint32_t poff;   // q - A
  int tail;        // -2: look the page up; -1: miss; >= 0: the tail of this unit (decided by the end)
  bool ok;         // gather entry e
};
__device__ __forceinline__ PdFront pd_front(const SPd &S, uint64_t q, bool look) {
  PdFront f;
  int s = 0;
  if (S.nseg > 1) {
    int lo = 0, len = S.nseg;
    while (len > 1) {
      const int half = len >> 1;
      if (S.start[lo + half] <= q) lo += half;
      len -= half;
    }
    s = lo;
  }
  const uint64_t rel = q - S.start[s];
  const uint32_t P = S.meta[4 * s + 2];
  const uint64_t pg = rel >> P;
  const bool in = look && q >= S.start[s];
  f.tail = in && pg >= S.meta[4 * s + 1] ? (q <= S.start[S.nseg + s] ? (int)S.meta[4 * s + 3] : -1) : -2;
  f.ok = in && f.tail == -2;
  if (!in) f.tail = -1;
  f.poff = (uint32_t)rel & ((1u << P) - 1u);
  f.A = q - f.poff;
  f.e = (uint64_t)S.meta[4 * s] + pg;
  return f;
}
// Back half: decode the gathered entry w (ignored unless f.ok).  Out: j (unit or -1), key (its base;
// for a hit on the page's j0: A if base(j0) == A, else A - 1, which no query equals), k0 (the hit
// was decided here from end0 or the segment end: no size check).
__device__ __forceinline__ void pd_back(const PdDev &pd, uint64_t pol, const PdFront &f, uint64_t q,
                                        const uint64_t w_in[4], int &j, uint64_t &key, bool &k0) {
  if (!f.ok) {  // tail of the segment's last unit, or a miss
    k0 = true;
    j = f.tail;
    key = q - 1;
    return;
  }
  const uint32_t j0 = (uint32_t)w_in[0], w1 = (uint32_t)(w_in[0] >> 32);
  const uint32_t cnt = w1 & PD_CNT_MAX, end0 = w1 >> PD_END_SHIFT;
  // padding is PD_PAD and no start sits at offset PD_PAD (build_pd): counting with min(poff, PD_PAD - 1)
  // never counts padding and counts the same starts
  const uint32_t rr = min(f.poff, PD_PAD - 1u) * 0x10001u;
  uint32_t c = 0, mx = 0;
  if (pd.v3 && cnt <= (uint32_t)PD_K3) {
    uint32_t word;
    const uint32_t kk = pd_count5(w_in, min(f.poff, PD_PAD - 1u), word);
    c = kk << 4;  // (16 per counted start, as below)
    mx = kk ? (word & 0xFFFFu) : 0u;
  } else if (!pd.v3 && cnt <= (uint32_t)PD_K2) {  // v2: twelve starts in w[2..7]
#pragma unroll
    for (int t = 1; t < 4; ++t) {
      cnt_max2((uint32_t)w_in[t], rr, c, mx);
      cnt_max2((uint32_t)(w_in[t] >> 32), rr, c, mx);
    }
  } else {  // crowded page: the starts continue in ovf[], one sector per 16
    const uint16_t *o = pd.ovf + (pd.v3 ? (uint32_t)(w_in[1] >> 32) : (uint32_t)w_in[1]);
    for (uint32_t t = 0; t < cnt; t += 16) {
      uint64_t v[4];
      ld_sector(o + t, pol, v);
      const uint32_t c0 = c;
#pragma unroll
      for (int z = 0; z < 4; ++z) {
        cnt_max2((uint32_t)v[z], rr, c, mx);
        cnt_max2((uint32_t)(v[z] >> 32), rr, c, mx);
      }
      if (c - c0 < 16u * 16u) break;  // later sectors hold larger offsets only
    }
  }
  const uint32_t k = c >> 4;
  k0 = k == 0;
  if (k == 0) {
    j = (j0 != 0xFFFFFFFFu && f.poff < end0) ? (int)j0 : -1;  // A7 on the page's j0
    key = (w1 & PD_EXACT) ? f.A : f.A - 1;
  } else {
    j = (int)(j0 + k);
    key = f.A + max(mx & 0xFFFFu, mx >> 16);
  }
}

// Two interleaved greatestLTE lookups through the page directory (k_slots; written out rather than
// through pd_front/pd_back, which costs the reverse shadow variants ~90 bytes of spills).  In: q (host addresses), look.
// Out: j (unit or -1), key (its base, or for a hit on the page's j0: A if base(j0) == A, else A - 1,
// which no query equals), k0 (the unit is the page's j0: hit decided here, h0), h0.
__device__ __forceinline__ void pd_lookup2(const SPd &S, const PdDev &pd, uint64_t pol, const uint64_t q[2],
                                           const bool look[2], int j[2], uint64_t key[2], bool k0[2]) {
  uint64_t w[2][4];
  uint64_t A[2];
  uint32_t poff[2];
  bool ok[2];
  int tail[2];  // beyond the segment's pages: its last unit, or -1 (miss)
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    ok[m] = look[m];
    int s = 0;
    if (S.nseg > 1) {
      int lo = 0, len = S.nseg;
      while (len > 1) {
        const int half = len >> 1;
        if (S.start[lo + half] <= q[m]) lo += half;
        len -= half;
      }
      s = lo;
    }
    const uint64_t rel = q[m] - S.start[s];
    const uint32_t P = S.meta[4 * s + 2];
    const uint64_t pg = rel >> P;
    ok[m] = ok[m] && q[m] >= S.start[s];
    tail[m] = ok[m] && pg >= S.meta[4 * s + 1] ? (q[m] <= S.start[S.nseg + s] ? (int)S.meta[4 * s + 3] : -1) : -2;
    ok[m] = ok[m] && tail[m] == -2;
    poff[m] = (uint32_t)rel & ((1u << P) - 1u);
    A[m] = q[m] - poff[m];
    if (ok[m]) {
      ld_sector(pd.ent + 8 * ((uint64_t)S.meta[4 * s] + pg), pol, w[m]);
    } else {
      w[m][0] = w[m][1] = w[m][2] = w[m][3] = 0;
    }
  }
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    const uint32_t j0 = (uint32_t)w[m][0], w1 = (uint32_t)(w[m][0] >> 32);
    const uint32_t cnt = w1 & PD_CNT_MAX, end0 = w1 >> PD_END_SHIFT;
    const uint32_t rr = min(poff[m], PD_PAD - 1u) * 0x10001u;  // see pd_back
    uint32_t c = 0, mx = 0;
    if (pd.v3 && cnt <= (uint32_t)PD_K3) {
      uint32_t word;
      const uint32_t kk = pd_count5(w[m], min(poff[m], PD_PAD - 1u), word);
      c = kk << 4;
      mx = kk ? (word & 0xFFFFu) : 0u;
    } else if (!pd.v3 && cnt <= (uint32_t)PD_K2) {  // v2: twelve starts in w[2..7]
#pragma unroll
      for (int t = 1; t < 4; ++t) {
        cnt_max2((uint32_t)w[m][t], rr, c, mx);
        cnt_max2((uint32_t)(w[m][t] >> 32), rr, c, mx);
      }
    } else {  // crowded page: the starts continue in ovf[], one sector per 16
      const uint16_t *o = pd.ovf + (pd.v3 ? (uint32_t)(w[m][1] >> 32) : (uint32_t)w[m][1]);
      for (uint32_t t = 0; t < cnt; t += 16) {
        uint64_t v[4];
        ld_sector(o + t, pol, v);
        const uint32_t c0 = c;
#pragma unroll
        for (int z = 0; z < 4; ++z) {
          cnt_max2((uint32_t)v[z], rr, c, mx);
          cnt_max2((uint32_t)(v[z] >> 32), rr, c, mx);
        }
        if (c - c0 < 16u * 16u) break;  // later sectors hold larger offsets only
      }
    }
    const uint32_t k = c >> 4;
    const uint32_t off = max(mx & 0xFFFFu, mx >> 16);
    k0[m] = k == 0;
    if (tail[m] != -2) {  // the tail of the segment's last unit (decided by its end) or a miss
      k0[m] = true;
      j[m] = tail[m];
      key[m] = q[m] - 1;
    } else if (k == 0) {
      const bool h0 = ok[m] && j0 != 0xFFFFFFFFu && poff[m] < end0;  // A7 on the page's j0
      j[m] = h0 ? (int)j0 : -1;
      key[m] = (w1 & PD_EXACT) ? A[m] : A[m] - 1;
    } else {
      j[m] = ok[m] ? (int)(j0 + k) : -1;
      key[m] = A[m] + off;
    }
  }
}

}  // namespace

// -------------------------------------------------------------------------------------------------
// The slot kernel.  Each thread handles one 16-byte chunk (2 slots) per warp-uniform grid-stride
// step; the two lookups are interleaved level by level.
// -------------------------------------------------------------------------------------------------
// FH >= 0: the forward index has exactly FH levels, one address segment and no wide bucket (the
// common case, specialised for the hot operation sets); FH < 0: generic.
// threads per CTA: the shadow reverse variant keeps both paths live and gets more registers
template <int DIR, int SH>
struct SlotCfg {
#ifdef CGCM_SLOT_THREADS
  static constexpr int threads = CGCM_SLOT_THREADS;
#else
  static constexpr int threads = 768;  // measured: 768 > 1024 (spills) > 512 on configs C and E
#endif
};

constexpr int FH_PD = -2;  // forward lookups through the page directory

template <int DIR, int OPS, int FH, int SH>
__global__ void __launch_bounds__(SlotCfg<DIR, SH>::threads, 1) k_slots(SlotArgs a) {
  // the outer AU's own refcount change of a queued re-map / release, folded into its slot pass
  if (a.rc_delta && a.cbeg == 0 && blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(a.tab.rc + a.rc_unit, a.rc_delta);
  if (a.sel == SEL_SLOW && *a.slowcount == 0) return;  // the pipelined pass decided every slot
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ uint64_t s_seg0[SEG_SMEM + 1];
  SIdx F, R;
  SPd PD;
  unsigned char *sp = smem;
  if constexpr (FH == FH_PD) sp = stage_pd(a.pd, sp, PD);
  else sp = stage(a.fx, nullptr, nullptr, sp, F);
  if (DIR == DIR_REV) sp = stage(a.rx, a.rx.h == 0 ? a.runpay : nullptr, a.runid, sp, R);
  // extent deltas (devbase - base of every copy in the extent), staged when few
  const bool ext_s = a.tab.n_ext <= EXT_SMEM;
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(sp);
  if (ext_s)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  const int nseg_s = a.nseg <= SEG_SMEM ? a.nseg : 0;
  for (int t = threadIdx.x; t <= nseg_s; t += blockDim.x) s_seg0[t] = a.seg_chunk0[t];
  __syncthreads();

  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const int lane = threadIdx.x & 31;
  // single-segment calls (the common case) keep the segment in registers
  Seg seg1 = a.segs[0];
  const uint64_t a0base = seg1.ptr & ~15ull;

  unsigned c_nulls = 0, c_hits = 0, c_miss = 0, c_pend = 0, c_notm = 0, c_under = 0, c_tr = 0;

  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  // software pipelining: the next iteration's two slots are loaded while this one is translated
  const bool pf = a.nseg == 1;
  uint64_t nv0 = 0, nv1 = 0;
  {
    const uint64_t c = a.cbeg + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (pf && c < a.nchunks) ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * c), pol_s, nv0, nv1);
  }
  for (uint64_t cb = a.cbeg + (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); cb < a.nchunks; cb += stride) {
    const uint64_t c = cb + lane;
    const bool live = c < a.nchunks;
    const uint64_t cv0 = nv0, cv1 = nv1;
    if (pf && c + stride < a.nchunks)
      ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * (c + stride)), pol_s, nv0, nv1);
    Seg sg = seg1;
    uint64_t a0 = a0base + 16ull * c;
    if (a.nseg > 1) {
      int s = 0;
      if (live) {
        const uint64_t *spp = nseg_s ? s_seg0 : a.seg_chunk0;
        int lo = 0, len = a.nseg;  // last s with seg0[s] <= c
        while (len > 1) {
          int half = len >> 1;
          if (spp[lo + half] <= c) lo += half;
          len -= half;
        }
        s = lo;
        sg = a.segs[s];
      }
      a0 = (sg.ptr & ~15ull) + 16ull * (c - (nseg_s ? s_seg0[s] : a.seg_chunk0[s]));
    }
    uint32_t valid = 0;
    uint64_t v[2] = {0, 0};
    if (live) {
      const uint64_t hi_addr = sg.ptr + 8ull * sg.n;
      valid = (a0 >= sg.ptr && a0 < hi_addr ? 1u : 0u) | (a0 + 8 >= sg.ptr && a0 + 8 < hi_addr ? 2u : 0u);
      if (a.sel != SEL_ALL) {
        const uint32_t *mk = a.sel == SEL_SLOW ? a.slowmask : a.hitmask;
        uint32_t hm = (mk[c >> 4] >> (2 * (c & 15))) & 3u;
        valid &= (a.sel == SEL_NOTHIT) ? ~hm : hm;
      }
      if (pf) {
        v[0] = cv0;
        v[1] = cv1;
      } else {
        ld_stream2(reinterpret_cast<const void *>(a0), pol_s, v[0], v[1]);
      }
    }

    // ---- a1: lookups ----
    uint64_t q[2], key[2], dx[2] = {0, 0};
    uint32_t rid[2] = {0, 0};
    int j[2];
    bool look[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      look[m] = ((valid >> m) & 1) && v[m] != 0;
      q[m] = look[m] ? v[m] : 0ull;
    }
    // reverse pass over slots the forward map recorded (unchanged since, R13-ii): one check
    bool sh[2] = {false, false};
    int jsh[2] = {0, 0};
    uint64_t hsh[2] = {0, 0};
    // the unit's hot word (size | extent | flags) and state word (epoch | extent | flags)
    uint64_t hw[2] = {0, 0}, rw[2] = {0, 0};
    const int64_t slot0 = ((int64_t)(a0 - sg.ptr)) >> 3;  // slot index of m = 0 (-1 for a head chunk)
    if (SH && DIR == DIR_REV && sg.shadow) {
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (!look[m]) continue;
        const int64_t i = slot0 + m;
        // (a deferred reference was materialised by k_unmap_sh or the runtime before this pass)
        const uint64_t shw = reinterpret_cast<const uint64_t *>(sg.shadow)[i];
        const uint32_t u = sh_unit(shw_unit(shw));
        if (u == SH_NONE) continue;
        const uint64_t w = ld_u64(a.tab.st + u, pol_t);  // extent, flags and epoch in one word
        const uint32_t e = hot_ext(w);
        const uint64_t h = (hot_flags(w) & UF_ACTIVE) && e < (uint32_t)a.tab.n_ext
                               ? sh_reverse(q[m], shw, ext_s ? s_ext[e] : a.tab.ext_delta[e], a.tab.ext_lo[e],
                                            a.tab.ext_len[e])
                               : 0ull;
        if (h) {
          sh[m] = true;
          jsh[m] = (int)u;
          hsh[m] = h;
          hw[m] = w;  // the size bits are not used on this path
          rw[m] = w;
          look[m] = false;
        }
      }
    }
    // full lookups only where a lane still needs one: after the shadow check most reverse warps skip
    // the whole search (a warp-uniform branch, not predication)
    j[0] = j[1] = -1;
    key[0] = key[1] = 0;
    bool k0[2] = {false, false};  // page directory: the hit on the page's j0 was decided by the lookup
    if (!(SH && DIR == DIR_REV) || __any_sync(0xffffffffu, look[0] || look[1])) {
    if (DIR == DIR_REV) {
      // the device extent holding the pointer, and the host address it mirrors
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        uint64_t tk = 0;
        j[m] = look[m] ? top_search(R, q[m], tk) : -1;
        key[m] = tk;
      }
      if (a.rx.h > 0) level_lookup2(R, a.rx, pol_t, q, j, key);
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (j[m] >= 0) {
          dx[m] = a.rx.h == 0 ? R.pay[j[m]] : a.runpay[j[m]];
          rid[m] = a.rx.h == 0 ? R.rid[j[m]] : a.runid[j[m]];
        } else {
          look[m] = false;
        }
        q[m] = look[m] ? q[m] + dx[m] : 0ull;  // host address
      }
    }
    if constexpr (FH == FH_PD) {
      pd_lookup2(PD, a.pd, pol_t, q, look, j, key, k0);
    } else {
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        uint64_t tk = 0;
        j[m] = look[m] ? top_search<(FH >= 0)>(F, q[m], tk) : -1;
        key[m] = tk;
      }
      if constexpr (FH > 0) level_lookup2_fixed<FH>(a.fx, pol_t, q, j, key);
      else if constexpr (FH < 0) level_lookup2(F, a.fx, pol_t, q, j, key);
    }

    // ---- the unit's hot word (size | extent | flags), and its state word where the epoch is needed ----
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      look[m] = look[m] && j[m] >= 0;
      if (look[m]) hw[m] = ld_u64(a.tab.hot + j[m], pol_t);
      if ((OPS & OP_GATE) && look[m]) rw[m] = ld_u64(a.tab.st + j[m], pol_t);
    }
    }  // full lookups
    bool hit[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      uint64_t sz = hot_size32(hw[m]);
      if (look[m] && sz == BIG_SIZE) sz = a.tab.size64[j[m]];
      hit[m] = look[m] && (k0[m] || q[m] - key[m] <= sz);  // A7: p - base <= size
      if (DIR == DIR_REV && look[m]) {
        // the unit must own this extent's copy: active, and its copy lives in that extent
        if (!(hit[m] && (hot_flags(hw[m]) & UF_ACTIVE) && hot_ext(hw[m]) == rid[m])) {
          hit[m] = false;
          if (j[m] > 0 && q[m] == key[m]) {  // one past the end of the previous unit (A7)
            const uint64_t h2 = a.tab.hot[j[m] - 1], b2 = a.tab.base[j[m] - 1];
            uint64_t s2 = hot_size32(h2);
            if (s2 == BIG_SIZE) s2 = a.tab.size64[j[m] - 1];
            if ((hot_flags(h2) & UF_ACTIVE) && hot_ext(h2) == rid[m] && q[m] == b2 + s2) {
              hit[m] = true;
              j[m] -= 1;
              key[m] = b2;
              hw[m] = h2;
              rw[m] = a.tab.st[j[m]];
            }
          }
        }
      }
    }
    if (a.dn > 0) {  // NEXT-1: delta units (q: the host address looked up; 0 if none)
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (q[m] == 0 || sh[m] || !((valid >> m) & 1) || hit[m]) continue;
        uint64_t db;
        const int d = delta_override(a, q[m], hit[m], db);
        if (d < 0) continue;
        const uint64_t h2 = a.tab.hot[d];
        // a reverse lookup: the unit must own the extent's copy (active, its copy in that extent)
        if (DIR == DIR_REV && !((hot_flags(h2) & UF_ACTIVE) && hot_ext(h2) == rid[m])) continue;
        hit[m] = true;
        j[m] = d;
        key[m] = db;
        hw[m] = h2;
        if (OPS & OP_GATE) rw[m] = a.tab.st[d];
      }
    }
    if (SH && DIR == DIR_REV) {
#pragma unroll
      for (int m = 0; m < 2; ++m)
        if (sh[m]) {
          hit[m] = true;
          j[m] = jsh[m];
          q[m] = hsh[m];  // hw, rw: gathered by the shadow check
        }
    }
    // forward map: record the shadow of every slot (CPU pointer, unit) for the reverse pass
    if (SH && (OPS & OP_INC) && sg.shadow && live) {
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (!((valid >> m) & 1)) continue;
        const int64_t i = slot0 + m;
        reinterpret_cast<uint64_t *>(sg.shadow)[i] = make_shw(v[m], hit[m] ? (uint32_t)j[m] : SH_NONE);
      }
    }
    // epoch (gate): from the record gathered with the hot word; refcount (unmap check) where needed
    uint32_t ep[2];
    int32_t rcv[2] = {0, 0};
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      ep[m] = st_epoch(rw[m]);
      if ((OPS & OP_CHECKMAPPED) && hit[m]) rcv[m] = a.tab.rc[j[m]];
    }

    // ---- a2/a3/a4 operations ----
    uint64_t outv[2] = {v[0], v[1]};
    uint32_t wrote = 0;
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const bool vm = (valid >> m) & 1;
      const bool hm = vm && hit[m];
      const bool nul = vm && v[m] == 0;
      // a forward pass with inc = k stands for k sequential mapArray calls of one outer (a batch
      // naming it k times): each call maps -- and counts -- every slot (Alg. 1 per slot, A8)
      const unsigned w = (OPS & (OP_INC | OP_INCPLAIN)) ? (unsigned)sg.inc : 1u;
      c_nulls += nul * w;
      c_hits += hm * w;
      c_miss += (vm && !nul && !hm) * w;
      const int unit = hm ? j[m] : 0;
      int32_t *RC = a.tab.rc + unit;
      const uint32_t fl = hot_flags(hw[m]);
      if (OPS & OP_CHECKMAPPED) c_notm += (hm && rcv[m] <= 0);
      bool act = false;
      if (OPS & OP_INC) {
        if (hm) {
          if (fl & UF_ACTIVE) {
            red_add(RC, sg.inc);
          } else {
            int old = atomicAdd(RC, sg.inc);
            act = (old == 0);  // refcount 0 -> 1: Alg. 1's activation
          }
        }
      }
      if (OPS & OP_INCPLAIN)
        if (hm) red_add(RC, sg.inc);
      if (OPS & OP_DECPLAIN)
        if (hm) red_add(RC, -sg.inc);
      bool freed = false;
      if (OPS & OP_DEC) {
        if (hm) {
          if (a.dec_red) {
            red_add(RC, -sg.inc);
          } else {
            int old = atomicAdd(RC, -sg.inc);
            c_under += (old < sg.inc);
            freed = (old == sg.inc);  // refcount 1 -> 0: Alg. 3's cuMemFree
          }
        }
      }
      bool gated = false;
      uint32_t old_ep = 0;
      if (OPS & OP_GATE) {
        if (hm && a.no_journal && (fl & UF_READONLY)) {
          // Alg. 2 line 3 for a read-only unit: epoch <- globalEpoch (skipped when already current)
          if (ep[m] != a.epoch) *lo_word(a.tab.st + unit) = a.epoch;
        } else if (hm && ep[m] != a.epoch) {
          old_ep = atomicExch(lo_word(a.tab.st + unit), a.epoch);
          gated = (old_ep != a.epoch);
        }
      }
      if (OPS & OP_WRITE) {
        if (hm) {
          if (DIR == DIR_FWD) {
            if (fl & UF_STORAGE) {
              const uint32_t e = hot_ext(hw[m]);
              outv[m] = q[m] + (ext_s ? s_ext[e] : a.tab.ext_delta[e]);  // Alg. 1: devptr + (ptr - base)
              wrote |= 1u << m;
            } else {
              c_pend += 1;  // activated by this call: completed after the allocation
            }
          } else {
            outv[m] = q[m];  // reverse: base + (g - devbase), the mirrored host address
            wrote |= 1u << m;
          }
        }
      }
      // list appends (the whole warp takes part)
      if (OPS & OP_INC) {
        unsigned long long ix = warp_append(&a.lc[0], act);
        if (act) a.act_list[ix] = (uint32_t)unit;
      }
      if (OPS & OP_DEC) {
        if (!a.dec_red) {
          unsigned long long ix = warp_append(&a.lc[2], freed);
          if (freed) a.free_list[ix] = (uint32_t)unit;
        }
      }
      if (OPS & OP_GATE) {
        const bool jg = gated && !a.no_journal;
        unsigned long long ix = warp_append(&a.lc[1], jg);
        const bool cp = gated && !(fl & UF_READONLY);  // Alg. 2: stale and not read-only
        if (jg) {
          Journal jn;
          jn.old_epoch = old_ep;
          jn.unit = (uint32_t)unit;
          jn.copy = cp ? 1u : 0u;
          jn.pad = 0;
          a.journal[ix] = jn;
        }
        unsigned long long cx = warp_append(&a.lc[3], cp);
        if (cp) a.copy_list[cx] = (uint32_t)unit;
      }
    }
    if (OPS & OP_WRITE) {
      c_tr += __popc(wrote);
      if (live) {
        if (sg.out == 0) {
          if (wrote == 3u) {
            st_stream2(reinterpret_cast<void *>(a0), pol_s, outv[0], outv[1]);
          } else {
#pragma unroll
            for (int m = 0; m < 2; ++m)
              if ((wrote >> m) & 1) st_stream1(reinterpret_cast<void *>(a0 + 8ull * m), pol_s, outv[m]);
          }
        } else {  // out of place: untranslated slots (NULL, lenient misses) are copied verbatim
#pragma unroll
          for (int m = 0; m < 2; ++m) {
            const bool vm = (valid >> m) & 1;
            const bool pend = DIR == DIR_FWD && hit[m] && !((wrote >> m) & 1);
            if (vm && !pend) {
              uint64_t dst = sg.out + (a0 + 8ull * m - sg.ptr);
              st_stream1(reinterpret_cast<void *>(dst), pol_s, outv[m]);
            }
          }
        }
      }
    }
    if (OPS & OP_HITMASK) {
      unsigned b0 = __ballot_sync(0xffffffffu, wrote & 1u), b1 = __ballot_sync(0xffffffffu, (wrote >> 1) & 1u);
      if (lane == 0) {
        uint32_t w0 = spread16(b0) | (spread16(b1) << 1);
        uint32_t w1 = spread16(b0 >> 16) | (spread16(b1 >> 16) << 1);
        uint64_t wi = cb >> 4;
        if (a.sel == SEL_SLOW) {  // the pipelined pass wrote the other hits of these words
          w0 |= a.hitmask[wi];
          if (cb + 16 < a.nchunks) w1 |= a.hitmask[wi + 1];
        }
        a.hitmask[wi] = w0;
        if (cb + 16 < a.nchunks) a.hitmask[wi + 1] = w1;
      }
    }
  }
  flush_count(&a.st->nulls, c_nulls);
  flush_count(&a.st->hits, c_hits);
  flush_count(&a.st->misses, c_miss);
  if (OPS & OP_WRITE) {
    flush_count(&a.st->pending, c_pend);
    flush_count(&a.st->translated, c_tr);
  }
  if (OPS & OP_CHECKMAPPED) flush_count(&a.st->notmapped, c_notm);
  if (OPS & OP_DEC) flush_count(&a.st->underflow, c_under);
}

// -------------------------------------------------------------------------------------------------
// k_map_pd: the forward map of one in-place segment (mapArrayDevice; a1 + a2 of Alg. 1) through the
// page directory.  Per slot: one 32-byte page-entry gather (a single LDG.256: the entry as two
// 16-byte cp.async cost 1.33 L2 requests, profiles/r01k_ab_ldg.log), one 8-byte unit-word gather,
// one refcount reduction -- the random L2 operations that bound it (profiles/r01j_l2_model.md).
// Both slots' entry gathers are in flight together, and the slot values of chunk t+2 are loaded
// while chunk t is translated.  Same results, counters and lists as
// k_slots<DIR_FWD, OP_WRITE | OP_INC | OP_HITMASK> (which serves every other case).
// -------------------------------------------------------------------------------------------------
#ifdef CGCM_MAP_PD_THREADS
constexpr int MAP_PD_THREADS = CGCM_MAP_PD_THREADS;
#else
constexpr int MAP_PD_THREADS = 768;  // measured: 768 > 1024 (5.42 ms at E) > 640 > 512
#endif

template <int SH>
__global__ void __launch_bounds__(MAP_PD_THREADS, 1) k_map_pd(SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  SPd PD;
  unsigned char *sp = stage_pd(a.pd, smem, PD);
  const bool ext_s = a.tab.n_ext <= EXT_SMEM;
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(sp);
  if (ext_s)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  __syncthreads();

  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const int lane = threadIdx.x & 31;
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi_addr = sg.ptr + 8ull * sg.n;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  unsigned c_nulls = 0, c_hits = 0, c_miss = 0, c_pend = 0, c_tr = 0;

  auto valid_of = [&](uint64_t c) -> uint32_t {
    const uint64_t a0 = a0base + 16ull * c;
    return c < a.nchunks ? ((a0 >= sg.ptr && a0 < hi_addr ? 1u : 0u) | (a0 + 8 >= sg.ptr && a0 + 8 < hi_addr ? 2u : 0u))
                         : 0u;
  };

  const uint64_t c_first = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t cv[2] = {0, 0}, nv[2] = {0, 0}, nnv[2] = {0, 0};
  if (c_first < a.nchunks) ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * c_first), pol_s, cv[0], cv[1]);
  if (c_first + stride < a.nchunks)
    ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * (c_first + stride)), pol_s, nv[0], nv[1]);
  for (uint64_t cb = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); cb < a.nchunks; cb += stride) {
    const uint64_t c = cb + lane;
    const bool live = c < a.nchunks;
    // pipeline: values of chunk t+2 into registers
    if (c + 2 * stride < a.nchunks)
      ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * (c + 2 * stride)), pol_s, nnv[0], nnv[1]);

    const uint64_t a0 = a0base + 16ull * c;
    const uint32_t valid = valid_of(c);
    const int64_t slot0 = ((int64_t)(a0 - sg.ptr)) >> 3;
    int j[2];
    uint64_t key[2], hw[2] = {0, 0};
    bool look[2], k0[2];
    PdFront fr[2];
    uint64_t ew[2][4] = {{0, 0, 0, 0}, {0, 0, 0, 0}};
#pragma unroll
    for (int m = 0; m < 2; ++m) {  // a1: both page-entry gathers in flight before either is decoded
      look[m] = ((valid >> m) & 1) && cv[m] != 0;
      fr[m] = pd_front(PD, cv[m], look[m]);
      if (fr[m].ok)  // one LDG.256, not allocated in L1 (random sectors: no reuse; measured 0.98 -> 0.97 ms at C)
        asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
                     : "=l"(ew[m][0]), "=l"(ew[m][1]), "=l"(ew[m][2]), "=l"(ew[m][3])
                     : "l"(a.pd.ent + 8 * fr[m].e), "l"(pol_t));
    }
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      pd_back(a.pd, pol_t, fr[m], cv[m], ew[m], j[m], key[m], k0[m]);
      look[m] = look[m] && j[m] >= 0;
#ifdef CGCM_NO_HOTC
      if (look[m]) hw[m] = ld_u64_hot(a.tab.hot + j[m], pol_t);
#else
      if (look[m]) {  // the 4-byte compact unit word (cgcm_dev.h make_hotc)
        uint32_t c;
        asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(c) : "l"(a.tab.hotc + j[m]), "l"(pol_t));
        hw[m] = c;  // decoded below, once both gathers are in flight
      }
#endif
    }
#ifndef CGCM_NO_HOTC
#pragma unroll
    for (int m = 0; m < 2; ++m)
      if (look[m]) {
        const uint32_t c = (uint32_t)hw[m];
        hw[m] = (c & HOTC_ESC) ? ld_u64_hot(a.tab.hot + j[m], pol_t) : hot_of_hotc(c);
      }
#endif
    bool hit[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      uint64_t sz = hot_size32(hw[m]);
      if (look[m] && sz == BIG_SIZE) sz = a.tab.size64[j[m]];
      hit[m] = look[m] && (k0[m] || cv[m] - key[m] <= sz);  // A7: p - base <= size
      if (a.dn > 0 && ((valid >> m) & 1) && cv[m] != 0 && !hit[m]) {  // NEXT-1: delta units
        uint64_t db;
        const int d = delta_override(a, cv[m], hit[m], db);
        if (d >= 0) {
          j[m] = d;
          hw[m] = a.tab.hot[d];
          hit[m] = look[m] = true;
        }
      }
    }
    // deferred reference (a.defer, SH): the unit was ACTIVE when the call began, so a reference held
    // elsewhere keeps it active until the runtime materialises this one -- the slot's
    // shadow word records it instead of a refcount reduction
    bool dfr[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) dfr[m] = SH && a.defer && hit[m] && (hot_flags(hw[m]) & UF_ACTIVE);
    if (SH && live) {  // forward-map shadow: (CPU pointer, unit) per slot for the reverse pass
      uint64_t *shp = reinterpret_cast<uint64_t *>(sg.shadow);
      const uint32_t u0 = hit[0] ? ((uint32_t)j[0] | (dfr[0] ? SH_DEFER : 0u)) : SH_NONE;
      const uint32_t u1 = hit[1] ? ((uint32_t)j[1] | (dfr[1] ? SH_DEFER : 0u)) : SH_NONE;
      if (valid == 3u && !(slot0 & 1)) {
        st_stream2(shp + slot0, pol_s, make_shw(cv[0], u0), make_shw(cv[1], u1));
      } else {
#pragma unroll
        for (int m = 0; m < 2; ++m)
          if ((valid >> m) & 1) shp[slot0 + m] = make_shw(cv[m], m ? u1 : u0);
      }
    }
    uint64_t outv[2] = {cv[0], cv[1]};
    uint32_t wrote = 0;
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const bool vm = (valid >> m) & 1;
      const bool nul = vm && cv[m] == 0;
      c_nulls += nul * (unsigned)sg.inc;  // inc = k: k sequential mapArray calls (see k_slots)
      c_hits += hit[m] * (unsigned)sg.inc;
      c_miss += (vm && !nul && !hit[m]) * (unsigned)sg.inc;
      const uint32_t fl = hot_flags(hw[m]);
      bool act = false;
      if (hit[m]) {
        int32_t *RC = a.tab.rc + j[m];
        if (fl & UF_ACTIVE) {
          if (!dfr[m]) red_add(RC, sg.inc);
        } else {
          act = atomicAdd(RC, sg.inc) == 0;  // refcount 0 -> 1: Alg. 1's activation
        }
        if (fl & UF_STORAGE) {
          const uint32_t e = hot_ext(hw[m]);
          outv[m] = cv[m] + (ext_s ? s_ext[e] : a.tab.ext_delta[e]);  // Alg. 1: devptr + (ptr - base)
          wrote |= 1u << m;
        } else {
          c_pend += 1;  // activated by this call: completed after the allocation
        }
      }
      const unsigned long long ix = warp_append(&a.lc[0], act);
      if (act) a.act_list[ix] = (uint32_t)j[m];
    }
    c_tr += __popc(wrote);
    if (live) {
      if (wrote == 3u) {
        st_stream2(reinterpret_cast<void *>(a0), pol_s, outv[0], outv[1]);
      } else {
#pragma unroll
        for (int m = 0; m < 2; ++m)
          if ((wrote >> m) & 1) st_stream1(reinterpret_cast<void *>(a0 + 8ull * m), pol_s, outv[m]);
      }
    }
    {  // hit mask: 2 bits per chunk
      const unsigned b0 = __ballot_sync(0xffffffffu, wrote & 1u), b1 = __ballot_sync(0xffffffffu, (wrote >> 1) & 1u);
      if (lane == 0) {
        const uint32_t w0 = spread16(b0) | (spread16(b1) << 1);
        const uint32_t w1 = spread16(b0 >> 16) | (spread16(b1 >> 16) << 1);
        const uint64_t wi = cb >> 4;
        a.hitmask[wi] = w0;
        if (cb + 16 < a.nchunks) a.hitmask[wi + 1] = w1;
      }
    }
    cv[0] = nv[0];
    cv[1] = nv[1];
    nv[0] = nnv[0];
    nv[1] = nnv[1];
  }
  flush_count(&a.st->nulls, c_nulls);
  flush_count(&a.st->hits, c_hits);
  flush_count(&a.st->misses, c_miss);
  flush_count(&a.st->pending, c_pend);
  flush_count(&a.st->translated, c_tr);
}

template <int SH>
static int launch_map_pd(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = pd_stage_bytes(a.pd) + (a.tab.n_ext <= EXT_SMEM ? al16(8 * (size_t)a.tab.n_ext) : 0);
  static bool configured = false;
  if (!configured) {
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaError_t e = cudaFuncSetAttribute(k_map_pd<SH>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  const uint64_t want = (a.nchunks + MAP_PD_THREADS - 1) / MAP_PD_THREADS;
  const int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  k_map_pd<SH><<<grid, MAP_PD_THREADS, smem, s>>>(a);
  return (int)cudaGetLastError();
}

// -------------------------------------------------------------------------------------------------
// k_unmap_sh: the reverse pass over slots whose forward map recorded a shadow (R13-ii: an unchanged
// slot reverses to its recorded CPU pointer): unmapArray (a3 + a4, OPS = WRITE | GATE | HITMASK),
// fused with releaseArray (| DEC), or releaseArray alone (OPS = DEC).  Any number of segments, in
// place or out of place.  Software-pipelined: the slot values and shadow of chunk t+2 stream into
// registers and the units' state words of chunk t+1 are gathered while chunk t is decided.  A slot
// whose shadow check fails (modified since the map, not translated by it, or in a segment without a
// shadow) is marked in the slow mask and left to k_slots<DIR_REV, OPS> with SEL_SLOW, launched right
// after (it returns at once when there is none).  Same results, counters and lists as k_slots.
// -------------------------------------------------------------------------------------------------
constexpr int UNMAP_SH_THREADS = 768;

template <int OPS, bool MS>  // MS: more than one segment
__global__ void __launch_bounds__(UNMAP_SH_THREADS, 1) k_unmap_sh(SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ uint64_t s_seg0[SEG_SMEM + 1];
  __shared__ Seg s_segs[SEG_SMEM];
  const bool ext_s = a.tab.n_ext <= EXT_SMEM;
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(smem);
  if (ext_s)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  const bool seg_s = a.nseg <= SEG_SMEM;
  if (seg_s) {
    for (int t = threadIdx.x; t <= a.nseg; t += blockDim.x) s_seg0[t] = a.seg_chunk0[t];
    for (int t = threadIdx.x; t < a.nseg; t += blockDim.x) s_segs[t] = a.segs[t];
  }
  __syncthreads();
  const uint64_t *seg0 = seg_s ? s_seg0 : a.seg_chunk0;
  const Seg *segs = seg_s ? s_segs : a.segs;
  const Seg seg1 = a.segs[0];  // the single segment (!MS), in registers

  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const int lane = threadIdx.x & 31;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  unsigned c_nulls = 0, c_hits = 0, c_tr = 0, c_under = 0, c_slow = 0;

  // chunk c -> its segment (last s with seg0[s] <= c)
  auto seg_of = [&](uint64_t c) -> int {
    if (!MS) return 0;
    int lo = 0, len = a.nseg;
    while (len > 1) {
      const int half = len >> 1;
      if (seg0[lo + half] <= c) lo += half;
      len -= half;
    }
    return lo;
  };
  // the streams of one chunk: slot values, recorded CPU pointers and units
  struct In {
    uint64_t a0;  // address of the chunk's first word (16-byte aligned)
    uint64_t g[2], h[2];  // slot values, shadow words (cgcm_dev.h make_shw)
    uint32_t valid;
    int s;
  };
  auto load_in = [&](uint64_t c, In &x) {
    x.g[0] = x.g[1] = 0;
    x.h[0] = x.h[1] = make_shw(0, SH_NONE);  // (the unit word is read where it is used: no stall at the load)
    x.valid = 0;
    x.s = 0;
    x.a0 = 0;
    if (c >= a.nchunks) return;
    const int s = seg_of(c);
    const Seg &sg = MS ? segs[s] : seg1;
    const uint64_t a0 = (sg.ptr & ~15ull) + 16ull * (c - (MS ? seg0[s] : 0ull)), hi = sg.ptr + 8ull * sg.n;
    x.s = s;
    x.a0 = a0;
    x.valid = (a0 >= sg.ptr && a0 < hi ? 1u : 0u) | (a0 + 8 >= sg.ptr && a0 + 8 < hi ? 2u : 0u);
    if (!x.valid) return;
    ld_stream2(reinterpret_cast<const void *>(a0), pol_s, x.g[0], x.g[1]);
    if (!sg.shadow) return;
    const uint64_t *shp = reinterpret_cast<const uint64_t *>(sg.shadow);  // shadow words (make_shw)
    const int64_t i0 = ((int64_t)(a0 - sg.ptr)) >> 3;
    if (x.valid == 3u && !(i0 & 1)) {
      ld_stream2(shp + i0, pol_s, x.h[0], x.h[1]);
    } else {
#pragma unroll
      for (int m = 0; m < 2; ++m)
        if ((x.valid >> m) & 1) x.h[m] = shp[i0 + m];
    }
  };
  // the state words (epoch | extent | flags) of the recorded units of x
  auto gather = [&](const In &x, uint64_t w[2]) {
#pragma unroll
    for (int m = 0; m < 2; ++m)
      w[m] = (shw_unit(x.h[m]) != SH_NONE && x.g[m] != 0) ? ld_u64_hot(a.tab.st + sh_unit(shw_unit(x.h[m])), pol_t) : 0ull;
  };

  const uint64_t c_first = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  In cur, nxt, nn;
  uint64_t cw[2], nw[2];
  load_in(c_first, cur);
  load_in(c_first + stride, nxt);
  gather(cur, cw);
  for (uint64_t cb = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); cb < a.nchunks; cb += stride) {
    load_in(cb + lane + 2 * stride, nn);
    gather(nxt, nw);

    const uint32_t valid = cur.valid;
    const Seg &sg = MS ? segs[cur.s] : seg1;
    bool hit[2], slow[2];
    uint64_t outv[2] = {cur.g[0], cur.g[1]};
    uint32_t wrote = 0;
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const bool vm = (valid >> m) & 1;
      const bool look = vm && cur.g[m] != 0;
      const uint64_t w = cw[m];
      const uint32_t e = hot_ext(w);
      const uint32_t su = sh_unit(shw_unit(cur.h[m]));
      const uint64_t hr = look && su != SH_NONE && (hot_flags(w) & UF_ACTIVE) && e < (uint32_t)a.tab.n_ext
                              ? sh_reverse(cur.g[m], cur.h[m], ext_s ? s_ext[e] : a.tab.ext_delta[e],
                                           a.tab.ext_lo[e], a.tab.ext_len[e])
                              : 0ull;
      hit[m] = hr != 0;
      slow[m] = look && !hit[m];
      c_nulls += vm && cur.g[m] == 0;
      c_hits += hit[m];
      const uint32_t unit = hit[m] ? su : 0u;
      const uint32_t fl = hot_flags(w);
      int32_t *RC = a.tab.rc + unit;
      bool freed = false;
      // a deferred reference (recorded by k_map_pd) is dropped by a released hit; any other slot turns
      // it into an ordinary reference first (the slow pass then treats the slot like any other)
      const bool dfr = a.defer && vm && sh_deferred(shw_unit(cur.h[m]));  // (also if a GPU function wrote NULL there)
      const bool drop = dfr && hit[m] && (OPS & OP_DEC);
      if (dfr && !drop) red_add(a.tab.rc + su, 1);
      if (OPS & OP_DEC) {
        if (hit[m] && !drop) {
          if (a.dec_red) {
            red_add(RC, -sg.inc);
          } else {
            const int old = atomicAdd(RC, -sg.inc);
            c_under += (old < sg.inc);
            freed = (old == sg.inc);  // refcount 1 -> 0: Alg. 3's cuMemFree
          }
        }
        if (!a.dec_red) {
          const unsigned long long ix = warp_append(&a.lc[2], freed);
          if (freed) a.free_list[ix] = unit;
        }
      }
      if (OPS & OP_GATE) {
        bool gated = false;
        uint32_t old_ep = 0;
        const uint32_t ep = st_epoch(w);
        if (hit[m] && a.no_journal && (fl & UF_READONLY)) {
          if (ep != a.epoch) *lo_word(a.tab.st + unit) = a.epoch;  // Alg. 2 line 3, read-only unit
        } else if (hit[m] && ep != a.epoch) {
          old_ep = atomicExch(lo_word(a.tab.st + unit), a.epoch);
          gated = (old_ep != a.epoch);
        }
        const bool jg = gated && !a.no_journal;
        const unsigned long long ix = warp_append(&a.lc[1], jg);
        const bool cp = gated && !(fl & UF_READONLY);  // Alg. 2: stale and not read-only
        if (jg) {
          Journal jn;
          jn.old_epoch = old_ep;
          jn.unit = unit;
          jn.copy = cp ? 1u : 0u;
          jn.pad = 0;
          a.journal[ix] = jn;
        }
        const unsigned long long cx = warp_append(&a.lc[3], cp);
        if (cp) a.copy_list[cx] = unit;
      }
      if ((OPS & OP_WRITE) && hit[m]) {
        outv[m] = hr;  // reverse: base + (g - devbase), the recorded CPU pointer
        wrote |= 1u << m;
      }
    }
    c_tr += __popc(wrote);
    c_slow += slow[0] + slow[1];
    if (OPS & OP_WRITE) {
      if (sg.out == 0) {
        if (wrote == 3u) {
          st_stream2(reinterpret_cast<void *>(cur.a0), pol_s, outv[0], outv[1]);
        } else {
#pragma unroll
          for (int m = 0; m < 2; ++m)
            if ((wrote >> m) & 1) st_stream1(reinterpret_cast<void *>(cur.a0 + 8ull * m), pol_s, outv[m]);
        }
      } else {  // out of place: NULL slots are copied verbatim, slow slots are left to the generic pass
#pragma unroll
        for (int m = 0; m < 2; ++m)
          if (((valid >> m) & 1) && !slow[m])
            st_stream1(reinterpret_cast<void *>(sg.out + (cur.a0 + 8ull * m - sg.ptr)), pol_s, outv[m]);
      }
    }
    {  // hit and slow masks: 2 bits per chunk
      const unsigned s0 = __ballot_sync(0xffffffffu, slow[0]), s1 = __ballot_sync(0xffffffffu, slow[1]);
      unsigned b0 = 0, b1 = 0;
      if (OPS & OP_HITMASK) {
        b0 = __ballot_sync(0xffffffffu, wrote & 1u);
        b1 = __ballot_sync(0xffffffffu, (wrote >> 1) & 1u);
      }
      if (lane == 0) {
        const uint64_t wi = cb >> 4;
        if (OPS & OP_HITMASK) a.hitmask[wi] = spread16(b0) | (spread16(b1) << 1);
        a.slowmask[wi] = spread16(s0) | (spread16(s1) << 1);
        if (cb + 16 < a.nchunks) {
          if (OPS & OP_HITMASK) a.hitmask[wi + 1] = spread16(b0 >> 16) | (spread16(b1 >> 16) << 1);
          a.slowmask[wi + 1] = spread16(s0 >> 16) | (spread16(s1 >> 16) << 1);
        }
      }
    }
    cur = nxt;
    nxt = nn;
    cw[0] = nw[0];
    cw[1] = nw[1];
  }
  flush_count(&a.st->nulls, c_nulls);
  flush_count(&a.st->hits, c_hits);
  if (OPS & OP_WRITE) flush_count(&a.st->translated, c_tr);
  flush_count(a.slowcount, c_slow);
  if (OPS & OP_DEC) flush_count(&a.st->underflow, c_under);
}

template <int OPS, bool MS>
static int launch_unmap_sh1(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = (a.tab.n_ext <= EXT_SMEM ? al16(8 * (size_t)a.tab.n_ext) : 0) + 64;
  static bool configured = false;
  if (!configured) {
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, k_unmap_sh<OPS, MS>);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(k_unmap_sh<OPS, MS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             optin - (int)fa.sharedSizeBytes);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  const uint64_t want = (a.nchunks + UNMAP_SH_THREADS - 1) / UNMAP_SH_THREADS;
  const int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  k_unmap_sh<OPS, MS><<<grid, UNMAP_SH_THREADS, smem, s>>>(a);
  return (int)cudaGetLastError();
}
template <int OPS>
static int launch_unmap_sh(const SlotArgs &a, int nsm, cudaStream_t s) {
  return a.nseg > 1 ? launch_unmap_sh1<OPS, true>(a, nsm, s) : launch_unmap_sh1<OPS, false>(a, nsm, s);
}

// ---- helpers of the pipelined single-segment passes ---------------------------------------------
__device__ __forceinline__ uint32_t warp_or(uint32_t v) { return __reduce_or_sync(0xffffffffu, v); }

// #{o <= r} among the four sorted 15-bit offsets packed in q (16-bit lanes): per lane
// 0x8000 + r - o keeps bit 15 iff o <= r, and never borrows from the next lane (r, o < 0x8000)
__device__ __forceinline__ uint32_t le4(uint64_t q, uint64_t r4) {
  return __popcll(((r4 | 0x8000800080008000ull) - q) & 0x8000800080008000ull);
}
__device__ __forceinline__ uint32_t off_at(uint64_t q1, uint64_t q2, uint64_t q3, uint32_t i) {  // offset i < 12
  const uint64_t q = i < 4 ? q1 : (i < 8 ? q2 : q3);
  return (uint32_t)(q >> (16 * (i & 3))) & 0xFFFFu;
}
// crowded page (more than PD_K starts): count in the side array, one sector per 16 offsets; returns
// k | (offset of start k - 1) << 32
__device__ __forceinline__ uint64_t pd_crowded_i(const uint16_t *ovf, uint32_t first, uint32_t cnt, uint32_t r) {
  const uint64_t r4 = (uint64_t)r * 0x0001000100010001ull;
  uint32_t k = 0, off = 0;
  for (uint32_t t = 0; t < cnt; t += 16) {
    uint64_t v[4];
    asm volatile("ld.global.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3]) : "l"(ovf + first + t));
    uint32_t c = 0;
#pragma unroll
    for (int z = 0; z < 4; ++z) c += le4(v[z], r4);
    if (c) {
      const uint32_t i = c - 1;
      off = (uint32_t)(v[i >> 2] >> (16 * (i & 3))) & 0xFFFFu;
    }
    k += c;
    if (c < 16) break;  // later sectors hold larger offsets only
  }
  return (uint64_t)k | ((uint64_t)off << 32);
}
__device__ __noinline__ uint64_t pd_crowded(const uint16_t *ovf, uint32_t first, uint32_t cnt, uint32_t r) {
  return pd_crowded_i(ovf, first, cnt, r);
}

// -------------------------------------------------------------------------------------------------
// k_fwd_fast: the forward map of cgcm_mapArrayDevice (a1 + a2 of Alg. 1) over ONE in-place segment with
// a shadow, through a page directory of ONE address segment (the case of every config-C/E-shaped table);
// same results, counters and lists as k_map_pd<1>.  Software pipeline: slot values two chunks ahead, the
// page entries (one LDG.256 each) one chunk ahead, the unit words of a chunk gathered as soon as its
// entries are decoded; the loop is unrolled twice with the buffers' roles swapped (no stage copies).  A
// warp translates a group of 32 chunks on the short path when all of its 64 slots are ordinary: a whole
// chunk, a page of this segment, a hit on a unit that is ACTIVE with its copy (its reference deferred
// into the shadow, a.defer), no escaped unit word.  The short path keeps no per-slot counters (a fast
// chunk is two hits, two translations), builds no masks (its hit-mask words are all ones) and takes no
// atomics; crowded pages stay on it (a divergent side-array count).  Any other group -- a NULL, a miss,
// an activation, a ragged end, a huge unit, a delta unit -- is left untouched and listed (a.wlist); the
// fix-up kernel k_fwd_fix then redoes it with fwd_chunk_slow, which recomputes every case from the two
// slot values.  Round 2 (profiles/r02t, r02x, r02z): 270 thread instructions per slot -> 148; E 3.28 ->
// 2.75 ms, C 0.709 -> 0.478 ms per launch; E is bound by its two dependent random L2 gathers per slot
// (DESIGN.md §7, §7.1).
// -------------------------------------------------------------------------------------------------
#ifdef CGCM_FWD_FAST_THREADS
constexpr int FWD_FAST_THREADS = CGCM_FWD_FAST_THREADS;
#else
constexpr int FWD_FAST_THREADS = 768;
#endif

// every case of chunk c (slot values cv) of the warp whose first chunk is cb; called by
// all 32 lanes of the warp (warp collectives: activation list, hit mask, counters)
template <bool ES, bool V3, bool DELTA>
__device__ __noinline__ void fwd_chunk_slow(const SlotArgs &a, const uint64_t *s_ext, uint64_t c, uint64_t cb,
                                            uint64_t cv0, uint64_t cv1) {
  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const int lane = threadIdx.x & 31;
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi = sg.ptr + 8ull * sg.n;
  uint64_t *shp = reinterpret_cast<uint64_t *>(sg.shadow);
  const uint64_t S0 = a.pd.seg_start[0], Send = a.pd.seg_start[1];
  const uint32_t P = a.pd.seg_meta[2], npages = a.pd.seg_meta[1], lastu = a.pd.seg_meta[3];
  const uint32_t *ent = a.pd.ent + 8ull * a.pd.seg_meta[0];
  const uint32_t pmask = (1u << P) - 1u;
  const int32_t inc = sg.inc;
  const bool defer = a.defer != 0;
  const uint64_t a0 = a0base + 16ull * c;
  const uint32_t valid = c < a.nchunks ? ((a0 >= sg.ptr ? 1u : 0u) | (a0 + 8 < hi ? 2u : 0u)) : 0u;
  const uint64_t cv[2] = {cv0, cv1};
  unsigned c_nulls = 0, c_hits = 0, c_miss = 0, c_pend = 0, c_tr = 0;
  // a1 front: the page of each slot, its entry, or the tail of the segment's last unit (A7)
  uint64_t ew[2][4];
  uint32_t poff[2];
  int jt[2];
  bool ok[2];
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    const bool look = ((valid >> m) & 1) && cv[m] != 0 && cv[m] >= S0;
    const uint64_t rel = cv[m] - S0;
    const uint64_t pg = rel >> P;
    ok[m] = look && pg < npages;
    poff[m] = (uint32_t)rel & pmask;
    jt[m] = look && !ok[m] && cv[m] <= Send ? (int)lastu : -1;
    ew[m][0] = ew[m][1] = ew[m][2] = ew[m][3] = 0;
    if (ok[m]) ld_sector(ent + 8 * pg, pol_t, ew[m]);
  }
  int j[2];
  bool k0[2], dec[2];
  uint64_t key[2];
  uint32_t cw[2], ps[2];
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    j[m] = jt[m];
    k0[m] = true;
    dec[m] = false;
    key[m] = 0;
    ps[m] = 0;
    if (ok[m]) {
      const uint32_t j0 = (uint32_t)ew[m][0], w1 = (uint32_t)(ew[m][0] >> 32);
      const uint32_t cnt = w1 & PD_CNT_MAX, end0 = w1 >> PD_END_SHIFT;
      const uint32_t r = min(poff[m], PD_PAD - 1u);
      if (V3 && cnt <= (uint32_t)PD_K3) {
        uint32_t word;
        const uint32_t k = pd_count5(ew[m], r, word);
        const bool h = k ? poff[m] <= (word >> 16) : (j0 != 0xFFFFFFFFu && poff[m] < end0);
        j[m] = h ? (int)(j0 + k) : -1;
        dec[m] = true;
        ps[m] = (uint32_t)ew[m][1];
      } else if (!V3 && cnt <= (uint32_t)PD_K2) {
        const uint32_t r2 = r | (r << 16);
        const uint64_t r4 = (uint64_t)r2 | ((uint64_t)r2 << 32);
        const uint32_t k = le4(ew[m][1], r4) + le4(ew[m][2], r4) + le4(ew[m][3], r4);
        const uint32_t off = k ? off_at(ew[m][1], ew[m][2], ew[m][3], k - 1) : 0u;
        k0[m] = k == 0;
        j[m] = k ? (int)(j0 + k) : (j0 != 0xFFFFFFFFu && poff[m] < end0 ? (int)j0 : -1);
        key[m] = cv[m] - poff[m] + off;
      } else {
        const uint64_t ko = pd_crowded(a.pd.ovf, V3 ? (uint32_t)(ew[m][1] >> 32) : (uint32_t)ew[m][1], cnt, r);
        const uint32_t k = (uint32_t)ko, off = (uint32_t)(ko >> 32);
        k0[m] = k == 0;
        j[m] = k ? (int)(j0 + k) : (j0 != 0xFFFFFFFFu && poff[m] < end0 ? (int)j0 : -1);
        key[m] = cv[m] - poff[m] + off;
      }
    }
    cw[m] = 0;
    if (j[m] >= 0 && !(V3 && (ps[m] & PD_STATE_VALID)))
      asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(cw[m]) : "l"(a.tab.hotc + j[m]), "l"(pol_t));
  }
  uint64_t outv[2] = {cv[0], cv[1]};
  uint32_t wrote = 0, su[2];
  bool act[2];
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    const bool vm = (valid >> m) & 1;
    const bool look = j[m] >= 0;
    uint64_t hw;
    if (V3 && (ps[m] & PD_STATE_VALID))
      hw = ((uint64_t)(ps[m] & EXT_MASK) << ESHIFT) | ((uint64_t)(UF_ACTIVE | UF_STORAGE) << FSHIFT);
    else
      hw = (cw[m] & HOTC_ESC) && look ? ld_u64_hot(a.tab.hot + j[m], pol_t) : hot_of_hotc(cw[m]);
    uint64_t sz = hot_size32(hw);
    if (look && !dec[m] && !k0[m] && sz == BIG_SIZE) sz = a.tab.size64[j[m]];
    bool hit = look && (dec[m] || k0[m] || cv[m] - key[m] <= sz);  // A7: p - base <= size
    if (DELTA && vm && cv[m] != 0 && !hit) {  // NEXT-1: delta units, where the main table missed
      uint64_t db;
      const int d = delta_override(a, cv[m], hit, db);
      if (d >= 0) {
        j[m] = d;
        hw = ld_u64_hot(a.tab.hot + d, pol_t);
        hit = true;
      }
    }
    const bool nul = vm && cv[m] == 0;
    c_nulls += nul;
    c_hits += hit;
    c_miss += vm && !nul && !hit;
    const uint32_t fl = hot_flags(hw);
    const bool active = (fl & UF_ACTIVE) != 0;
    const bool dfr = defer && hit && active;
    act[m] = false;
    if (hit && !dfr) {
      int32_t *RC = a.tab.rc + j[m];
      if (active) red_add(RC, inc);
      else act[m] = atomicAdd(RC, inc) == 0;  // refcount 0 -> 1: Alg. 1's activation
    }
    if (hit && (fl & UF_STORAGE)) {
      const uint32_t e = hot_ext(hw);
      outv[m] = cv[m] + (ES ? s_ext[e] : a.tab.ext_delta[e]);  // Alg. 1: devptr + (ptr - base)
      wrote |= 1u << m;
    } else {
      c_pend += hit;
    }
    su[m] = hit ? ((uint32_t)j[m] | (dfr ? SH_DEFER : 0u)) : SH_NONE;
  }
  c_tr += __popc(wrote);
  if (__any_sync(0xffffffffu, act[0] || act[1])) {
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const unsigned long long ix = warp_append(&a.lc[0], act[m]);
      if (act[m]) a.act_list[ix] = (uint32_t)j[m];
    }
  }
  const int64_t i0 = ((int64_t)(a0 - sg.ptr)) >> 3;
  if (valid == 3u) {
    st_stream2(reinterpret_cast<void *>(a0), pol_s, outv[0], outv[1]);
    if (!(i0 & 1)) {
      st_stream2(shp + i0, pol_s, make_shw(cv[0], su[0]), make_shw(cv[1], su[1]));
    } else {
#pragma unroll
      for (int m = 0; m < 2; ++m) shp[i0 + m] = make_shw(cv[m], su[m]);
    }
  } else if (valid) {
#pragma unroll
    for (int m = 0; m < 2; ++m)
      if ((valid >> m) & 1) {
        st_stream1(reinterpret_cast<void *>(a0 + 8ull * m), pol_s, outv[m]);
        shp[i0 + m] = make_shw(cv[m], su[m]);
      }
  }
  {  // hit mask: 2 bits per chunk, 16 chunks per word (lanes 0-15: word cb/16, lanes 16-31: the next)
    const uint32_t b = wrote << (2u * (lane & 15));
    const uint32_t w0 = warp_or(lane < 16 ? b : 0u), w1 = warp_or(lane < 16 ? 0u : b);
    const uint64_t wi = cb >> 4;
    if (lane == 0) a.hitmask[wi] = w0;
    else if (lane == 16 && cb + 16 < a.nchunks) a.hitmask[wi + 1] = w1;
  }
  flush_count(&a.st->nulls, (unsigned long long)c_nulls * (unsigned)inc);
  flush_count(&a.st->hits, (unsigned long long)c_hits * (unsigned)inc);
  flush_count(&a.st->misses, (unsigned long long)c_miss * (unsigned)inc);
  flush_count(&a.st->pending, c_pend);
  flush_count(&a.st->translated, c_tr);
}

template <bool ES, bool V3, bool DELTA>
__global__ void __launch_bounds__(FWD_FAST_THREADS, 1) k_fwd_fast(const __grid_constant__ SlotArgs a) {
#ifdef CGCM_FWD_S3
  constexpr bool S3 = true;
#else
  constexpr bool S3 = false;
#endif
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(smem);
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  __syncthreads();
  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const uint32_t lane = threadIdx.x & 31;
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull;
  uint64_t *shp = reinterpret_cast<uint64_t *>(sg.shadow) - ((sg.ptr >> 3) & 1);  // shp[2c]: chunk c's first slot
  const bool sh_odd = (sg.ptr >> 3) & 1;
  const uint64_t S0 = a.pd.seg_start[0];
  const uint32_t P = a.pd.seg_meta[2];
  const uint64_t npages = a.pd.seg_meta[1];
  const uint32_t *ent = a.pd.ent + 8ull * a.pd.seg_meta[0];
  const uint32_t pmask = (1u << P) - 1u;
  const uint32_t nch = (uint32_t)a.nchunks;  // < 2^31 (launch_fwd_fast1; larger calls: k_fwd_big)
  // whole chunks (both slots in the segment): [f0, f1)
  const uint32_t f0 = sh_odd ? 1u : 0u;
  const uint32_t f1 = (uint32_t)((sg.ptr + 8ull * sg.n - a0base) >> 4);
  const bool fast_ok = a.defer != 0;
  const uint32_t stride = gridDim.x * blockDim.x;
  uint32_t c_fast = 0;

  struct Fr {  // one chunk in flight: its slot values and page entries
    uint64_t v0, v1;
    uint64_t ew[2][4];
    uint32_t poff[2];
    bool ok[2];
  };
  auto front = [&](uint64_t p0, uint64_t p1, Fr &f) {
    const uint64_t p[2] = {p0, p1};
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const uint64_t rel = p[m] - S0;  // NULL and p < S0 wrap far beyond the pages
      const uint64_t pg = rel >> P;
      f.ok[m] = pg < npages;
      f.poff[m] = (uint32_t)rel & pmask;
      if (f.ok[m])
        asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
                     : "=l"(f.ew[m][0]), "=l"(f.ew[m][1]), "=l"(f.ew[m][2]), "=l"(f.ew[m][3])
                     : "l"(ent + 8 * pg), "l"(pol_t));
    }
  };
  // a decoded chunk: its slot values, units, unit words (in flight), and per slot x = the distance the unit
  // word's size must cover (A7: p - base <= size; 0 when the entry decided) or, with a valid page state,
  // the extent | 2^31
  struct Dc {
    uint64_t v0, v1;
    uint32_t j[2], cw[2], x[2];
    bool rare;
  };
  // decode chunk c: j = j0 + #{starts <= p - A}; issue the unit words the entry does not decide
  auto decode = [&](const Fr &fc, uint32_t c, Dc &d) {
    d.v0 = fc.v0;
    d.v1 = fc.v1;
    d.rare = !(fast_ok && c >= f0 && c < f1);
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const uint32_t j0 = (uint32_t)fc.ew[m][0], w1 = (uint32_t)(fc.ew[m][0] >> 32);
      const uint32_t cnt = w1 & PD_CNT_MAX, end0 = w1 >> PD_END_SHIFT, po = fc.poff[m];
      const uint32_t r = min(po, PD_PAD - 1u);
      const bool okj0 = j0 != 0xFFFFFFFFu && po < end0;  // j0's end decides (A7)
      uint32_t k, dl = 0;
      bool hit = false, known = false;  // known: decided by the entry (v3), with the page state
      uint32_t ps = 0;
      if (V3 && cnt <= (uint32_t)PD_K3) {
        uint32_t word;
        k = pd_count5(fc.ew[m], r, word);
        hit = k ? po <= (word >> 16) : okj0;
        ps = (uint32_t)fc.ew[m][1];
        known = true;
      } else {
        uint32_t off;
        if (!V3 && cnt <= (uint32_t)PD_K2) {
          const uint32_t r2 = r | (r << 16);
          const uint64_t r4 = (uint64_t)r2 | ((uint64_t)r2 << 32);
          k = le4(fc.ew[m][1], r4) + le4(fc.ew[m][2], r4) + le4(fc.ew[m][3], r4);
          off = k ? off_at(fc.ew[m][1], fc.ew[m][2], fc.ew[m][3], k - 1) : 0u;
        } else if (fc.ok[m]) {  // crowded page: the side array
          const uint64_t ko = pd_crowded_i(a.pd.ovf, V3 ? (uint32_t)(fc.ew[m][1] >> 32) : (uint32_t)fc.ew[m][1], cnt, r);
          k = (uint32_t)ko;
          off = (uint32_t)(ko >> 32);
        } else {
          k = off = 0;
        }
        dl = po - off;
        hit = k ? true : okj0;  // k > 0: decided by the candidate's size (unit word)
      }
      d.j[m] = j0 + k;
      d.rare = d.rare || !fc.ok[m] || !hit;
      const bool st_valid = V3 && known && (ps & PD_STATE_VALID);
      d.cw[m] = 0;
      if (fc.ok[m] && hit && !st_valid)  // the 4-byte compact unit word (cgcm_dev.h make_hotc)
        asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;"  // random: no L1 reuse (r02h1)
                     : "=r"(d.cw[m]) : "l"(a.tab.hotc + d.j[m]), "l"(pol_t));
      d.x[m] = st_valid ? ((ps & (uint32_t)EXT_MASK) | 0x80000000u) : (known || k == 0 ? 0u : dl);
    }
  };
  // translate decoded chunk cb + lane, or list the warp's group for k_fwd_fix (nothing written here)
  auto finish = [&](const Dc &d, uint32_t cb) {
    const uint32_t c = cb + lane;
    bool rare = d.rare;
    uint32_t e[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      if (d.x[m] & 0x80000000u) {
        e[m] = d.x[m] & 0x7FFFFFFFu;
      } else {  // ACTIVE with its copy, no escape, and within the unit's size
        const uint32_t w = d.cw[m];
        rare = rare || (w & (HOTC_ESC | (3u << 29))) != (3u << 29) || d.x[m] > (w & 0x3FFFFu);
        e[m] = (w >> 18) & 0x7FFu;
      }
    }
    if (__any_sync(0xffffffffu, rare)) {
      if (lane == 0) a.wlist[atomicAdd(a.wcount, 1ull)] = cb;
    } else {
      ++c_fast;
      const uint64_t o0 = d.v0 + (ES ? s_ext[e[0]] : a.tab.ext_delta[e[0]]);  // Alg. 1: devptr + (ptr - base)
      const uint64_t o1 = d.v1 + (ES ? s_ext[e[1]] : a.tab.ext_delta[e[1]]);
      st_stream2(reinterpret_cast<void *>(a0base + 16ull * c), pol_s, o0, o1);
      const uint64_t s0 = make_shw(d.v0, d.j[0] | SH_DEFER), s1 = make_shw(d.v1, d.j[1] | SH_DEFER);
      if (!sh_odd) {
        st_stream2(shp + 2ull * c, pol_s, s0, s1);
      } else {
        shp[2ull * c] = s0;
        shp[2ull * c + 1] = s1;
      }
      if (lane == 0) a.hitmask[cb >> 4] = 0xFFFFFFFFu;
      else if (lane == 16 && cb + 16 < nch) a.hitmask[(cb >> 4) + 1] = 0xFFFFFFFFu;
    }
  };
  // one pipeline step for the warp's chunk cb: the values two chunks ahead go to (ld0, ld1), the entries
  // of the next chunk (values pv0, pv1) to fn, and chunk fc is decoded into dn; S3 (three stages): the
  // chunk decoded by the previous step (dp) is translated, so its unit words had a step to arrive;
  // otherwise chunk fc is translated at once.  The loop runs the step twice with the roles of the
  // buffers swapped (no register copies).
  const uint32_t cb0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
  auto step = [&](Fr &fc, Fr &fn, Dc &dn, Dc &dp, uint64_t &ld0, uint64_t &ld1, uint64_t pv0, uint64_t pv1, uint32_t cb) {
    const uint32_t c = cb + lane;
    if (c + 2 * stride < nch)
      ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * (c + 2 * stride)), pol_s, ld0, ld1);
    fn.v0 = pv0;
    fn.v1 = pv1;
    front(pv0, pv1, fn);  // the next chunk's entries are in flight while this one finishes
    decode(fc, c, dn);
    if (S3) {
      if (cb != cb0) finish(dp, cb - stride);
    } else {
      finish(dn, cb);
    }
  };
  const uint32_t c_first = cb0 + lane;
  Fr F0, F1;
  Dc D0, D1;
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    F0.ew[m][0] = F0.ew[m][1] = F0.ew[m][2] = F0.ew[m][3] = 0;
    F1.ew[m][0] = F1.ew[m][1] = F1.ew[m][2] = F1.ew[m][3] = 0;
  }
  uint64_t va0 = 0, va1 = 0, vb0 = 0, vb1 = 0;
  F0.v0 = F0.v1 = 0;
  if (c_first < nch) ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * c_first), pol_s, F0.v0, F0.v1);
  if (c_first + stride < nch)
    ld_stream2(reinterpret_cast<const void *>(a0base + 16ull * (c_first + stride)), pol_s, vb0, vb1);
  front(F0.v0, F0.v1, F0);
  for (uint32_t cb = cb0; cb < nch;) {
    step(F0, F1, D0, D1, va0, va1, vb0, vb1, cb);
    cb += stride;
    if (cb >= nch) {
      if (S3) finish(D0, cb - stride);
      break;
    }
    step(F1, F0, D1, D0, vb0, vb1, va0, va1, cb);
    cb += stride;
    if (cb >= nch) {
      if (S3) finish(D1, cb - stride);
      break;
    }
  }
  const unsigned inc = (unsigned)sg.inc;
  flush_count(&a.st->hits, 2ull * c_fast * inc);  // inc = k: k sequential calls
  flush_count(&a.st->translated, 2ull * c_fast);
}

// the warp groups k_fwd_fast listed: every chunk through fwd_chunk_slow (a NULL, a miss, an activation,
// a ragged end ... anywhere in the group); usually none
template <bool ES, bool V3, bool DELTA>
__global__ void __launch_bounds__(FWD_FAST_THREADS, 1) k_fwd_fix(const __grid_constant__ SlotArgs a) {
  const uint32_t n = (uint32_t)*a.wcount;
  if (n == 0) return;
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(smem);
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  __syncthreads();
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi = sg.ptr + 8ull * sg.n;
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n; i += nw) {
    const uint64_t cb = a.wlist[i], c = cb + (threadIdx.x & 31);
    uint64_t v0 = 0, v1 = 0;
    if (c < a.nchunks) {
      const uint64_t a0 = a0base + 16ull * c;
      if (a0 >= sg.ptr) v0 = reinterpret_cast<const uint64_t *>(a0)[0];
      if (a0 + 8 < hi) v1 = reinterpret_cast<const uint64_t *>(a0)[1];
    }
    fwd_chunk_slow<ES, V3, DELTA>(a, s_ext, c, cb, v0, v1);
  }
}

template <bool ES, bool V3, bool DELTA>
static int launch_fwd_fast1(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = (ES ? al16(8 * (size_t)a.tab.n_ext) : 0) + 64;
  static bool configured = false;
  if (!configured) {
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaError_t e = cudaFuncSetAttribute(k_fwd_fast<ES, V3, DELTA>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  constexpr int T = FWD_FAST_THREADS;
  const uint64_t want = (a.nchunks + T - 1) / T;
  const int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  if (cudaMemsetAsync(a.wcount, 0, sizeof(unsigned long long), s) != cudaSuccess) return (int)cudaGetLastError();
  k_fwd_fast<ES, V3, DELTA><<<grid, T, smem, s>>>(a);
  k_fwd_fix<ES, V3, DELTA><<<grid, T, smem, s>>>(a);
  return (int)cudaGetLastError();
}

#ifdef CGCM_REV_THREADS
constexpr int REV_THREADS = CGCM_REV_THREADS;
#else
constexpr int REV_THREADS = 768;
#endif

// -------------------------------------------------------------------------------------------------
// k_rev_fast: the reverse pass of cgcm_unmapArrayDevice (a3 + a4 [+ Alg. 3 release]) over ONE in-place
// segment that carries the forward map's shadow, in snapshot mode (no per-unit journal; releases as
// reductions checked afterwards by k_release_scan); same decisions, counters and lists as
// k_unmap_sh<WRITE|GATE|HITMASK[|DEC], false> in that mode.  Pipeline: slot values and shadow words two
// chunks ahead, the units' 8-byte state words one ahead.  A warp takes the short path for a chunk when
// all of its 64 slots are ordinary: a whole chunk, a recorded unit that is ACTIVE with the slot provably
// unchanged (shadow check), and an epoch gate that needs no copy (current, or stale and read-only: the
// epoch store only); releases and deferred references are predicated reductions.  Any other chunk is
// redone by rev_chunk_slow (copy list under a warp vote, hit / slow masks by warp reductions); slots
// whose shadow check fails go to k_slots SEL_SLOW afterwards.  Round 2: E 1.71 -> 1.60 ms, C 0.468 ->
// 0.436 (profiles/r02v_ab.log).
// -------------------------------------------------------------------------------------------------
struct RevIn {
  uint64_t g[2], h[2];  // slot values, shadow words (cgcm_dev.h make_shw)
  uint32_t valid;
};

// every case of chunk c (inputs x, state words w) of the warp whose first chunk is cb;
// called by all 32 lanes of the warp
template <bool DEC, bool ES>
__device__ __noinline__ void rev_chunk_slow(const SlotArgs &a, const ulonglong2 *s_dl, const uint32_t *s_len, uint64_t c,
                                            uint64_t cb, RevIn cur, uint64_t w0, uint64_t w1) {
  const uint64_t pol_s = policy_evict_first();
  const int lane = threadIdx.x & 31;
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull;
  const uint32_t n_ext = (uint32_t)a.tab.n_ext, cur_ep = a.epoch;
  const uint64_t cw[2] = {w0, w1};
  unsigned c_nulls = 0, c_hits = 0, c_slow = 0;
  bool hit[2], slow[2], cp[2];
  uint64_t outv[2];
  bool rare = false;
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    const bool vm = (cur.valid >> m) & 1;
    const uint64_t g = cur.g[m], w = cw[m];
    const uint32_t e = hot_ext(w), fl = hot_flags(w), su = sh_unit(shw_unit(cur.h[m]));
    const bool look = vm && g != 0;
    uint64_t hr = 0;
    if (look && su != SH_NONE && (fl & UF_ACTIVE) && e < n_ext) {
      const ulonglong2 dl = ES ? s_dl[e] : make_ulonglong2(a.tab.ext_delta[e], a.tab.ext_lo[e]);
      hr = sh_reverse(g, cur.h[m], dl.x, dl.y, ES ? s_len[e] : a.tab.ext_len[e]);
    }
    hit[m] = hr != 0;
    slow[m] = look && !hit[m];
    c_nulls += vm && g == 0;
    c_hits += hit[m];
    outv[m] = hit[m] ? hr : g;  // reverse: base + (g - devbase), the recorded CPU pointer
    const bool stale = hit[m] && st_epoch(w) != cur_ep;  // Alg. 2's epoch gate
    cp[m] = false;
    if (stale) {
      if (fl & UF_READONLY) {
        *lo_word(a.tab.st + su) = cur_ep;  // Alg. 2 line 3 only: never copied back
      } else {
        cp[m] = atomicExch(lo_word(a.tab.st + su), cur_ep) != cur_ep;  // stale and not read-only: copy
      }
    }
    // references: a deferred one (a.defer) is dropped by a released hit, materialised otherwise
    const bool dfr = a.defer && vm && sh_deferred(shw_unit(cur.h[m]));
    const bool drop = DEC && dfr && hit[m];
    if (dfr && !drop) red_add(a.tab.rc + su, 1);
    if (DEC && hit[m] && !drop) red_add(a.tab.rc + su, -sg.inc);  // Alg. 3, checked by k_release_scan
    rare = rare || cp[m];
  }
  c_slow += slow[0] + slow[1];
  if (__any_sync(0xffffffffu, rare)) {  // copy list of this warp's stale writable units
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const unsigned long long cx = warp_append(&a.lc[3], cp[m]);
      if (cp[m]) a.copy_list[cx] = sh_unit(shw_unit(cur.h[m]));
    }
  }
  if (cur.valid == 3u) {
    st_stream2(reinterpret_cast<void *>(a0base + 16ull * c), pol_s, outv[0], outv[1]);
  } else {
#pragma unroll
    for (int m = 0; m < 2; ++m)
      if ((cur.valid >> m) & 1) st_stream1(reinterpret_cast<void *>(a0base + 16ull * c + 8ull * m), pol_s, outv[m]);
  }
  {  // 2 bits per chunk, 16 chunks per word: lanes 0-15 make word cb/16, lanes 16-31 the next
    const uint32_t sh = 2u * (lane & 15);
    const uint32_t hb = ((hit[0] ? 1u : 0u) | (hit[1] ? 2u : 0u)) << sh;
    const uint32_t sb = ((slow[0] ? 1u : 0u) | (slow[1] ? 2u : 0u)) << sh;
    const uint32_t lo = lane < 16;
    const uint32_t h0 = warp_or(lo ? hb : 0u), h1 = warp_or(lo ? 0u : hb);
    const uint32_t s0 = warp_or(lo ? sb : 0u), s1 = warp_or(lo ? 0u : sb);
    const uint64_t wi = cb >> 4;
    if (lane == 0) {
      a.hitmask[wi] = h0;
      a.slowmask[wi] = s0;
    } else if (lane == 16 && cb + 16 < a.nchunks) {
      a.hitmask[wi + 1] = h1;
      a.slowmask[wi + 1] = s1;
    }
  }
  flush_count(&a.st->nulls, c_nulls);
  flush_count(&a.st->hits, c_hits);
  flush_count(&a.st->translated, c_hits);
  flush_count(a.slowcount, c_slow);
}

template <bool DEC, bool ES>
__global__ void __launch_bounds__(REV_THREADS, 1) k_rev_fast(const __grid_constant__ SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  // per extent {delta, device start | 2^63 if the extent spans 4 GiB or more}: one LDS.128 per slot.  The
  // shadow check needs no length: a slot g with 0 <= g - lo < 2^32 whose g - delta has the recorded low 32
  // bits IS the recorded pointer p + delta (g - delta and p lie in one window of width 2^32 starting at the
  // extent's host start, since the extent is shorter than 2^32), so it lies in the extent; a big extent's
  // flag bit fails the check (its slots take k_rev_fix, as with the length check of sh_reverse)
  ulonglong2 *s_dl = reinterpret_cast<ulonglong2 *>(smem);
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x)
      s_dl[t] = make_ulonglong2(a.tab.ext_delta[t], a.tab.ext_lo[t] | (a.tab.ext_len[t] == 0 ? 1ull << 63 : 0ull));
  __syncthreads();
  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const uint32_t lane = threadIdx.x & 31;
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi = sg.ptr + 8ull * sg.n;
  const uint64_t *shp = reinterpret_cast<const uint64_t *>(sg.shadow);
  const bool sh_odd = (sg.ptr >> 3) & 1;
  const uint32_t nch = (uint32_t)a.nchunks;  // < 2^31 (launch_rev_fast1; larger calls: k_rev_big)
  const uint32_t f0 = sh_odd ? 1u : 0u, f1 = (uint32_t)((hi - a0base) >> 4);  // whole chunks [f0, f1)
  const uint32_t stride = gridDim.x * blockDim.x;
  const uint32_t n_ext = (uint32_t)a.tab.n_ext, cur_ep = a.epoch;
  const int32_t dec = -sg.inc;
  const bool defer = a.defer != 0;
  uint32_t c_fast = 0;

  const uint32_t f0w = sh_odd ? 0xFFFFFFFFu : f0;  // vector loads: whole chunks of a 16-byte-aligned shadow
  // a chunk in flight: slot values, shadow words, validity, and the units' state words (gathered later)
  struct Rx {
    uint64_t g[2], h[2], w[2];
    uint32_t valid;
  };
  auto load_in = [&](uint32_t c, Rx &x) {
    if (c >= f0w && c < f1) {
      const uint64_t a0 = a0base + 16ull * c;
      ld_stream2(reinterpret_cast<const void *>(a0), pol_s, x.g[0], x.g[1]);
      ld_stream2(shp + 2ull * c, pol_s, x.h[0], x.h[1]);
      x.valid = 3u;
      return;
    }
    x.g[0] = x.g[1] = 0;
    x.h[0] = x.h[1] = make_shw(0, SH_NONE);
    x.valid = 0;
    if (c >= nch) return;
    const uint64_t a0 = a0base + 16ull * c;
    x.valid = (a0 >= sg.ptr ? 1u : 0u) | (a0 + 8 < hi ? 2u : 0u);
    const int64_t i0 = ((int64_t)(a0 - sg.ptr)) >> 3;
#pragma unroll
    for (int m = 0; m < 2; ++m)
      if ((x.valid >> m) & 1) {
        x.g[m] = reinterpret_cast<const uint64_t *>(a0)[m];
        x.h[m] = shp[i0 + m];
      }
  };
  auto gather = [&](Rx &x) {
#pragma unroll
    for (int m = 0; m < 2; ++m)
      x.w[m] = (shw_unit(x.h[m]) != SH_NONE && x.g[m] != 0) ? ld_u64_hot(a.tab.st + sh_unit(shw_unit(x.h[m])), pol_t) : 0ull;
  };
  // one pipeline step for the warp's chunk cb: values and shadow words two chunks ahead into xl, the next
  // chunk's state words into xn, chunk xc reversed.  The loop runs it three times with the roles of the
  // three buffers rotated (no register copies).
  auto step = [&](Rx &xc, Rx &xn, Rx &xl, uint32_t cb) {
    const uint32_t c = cb + lane;
    load_in(c + 2 * stride, xl);
    gather(xn);
    bool rare = !(c >= f0 && c < f1);
    uint64_t hr[2];
    uint32_t su[2];
    bool stale[2], dfr[2];
#pragma unroll
    for (int m = 0; m < 2; ++m) {
      const uint64_t g = xc.g[m], w = xc.w[m];
      const uint32_t uw = shw_unit(xc.h[m]), e = hot_ext(w), fl = hot_flags(w);
      su[m] = uw & ~SH_DEFER;
      ulonglong2 dl = make_ulonglong2(0, ~0ull);
      if (e < n_ext)
        dl = ES ? s_dl[e]
                : make_ulonglong2(a.tab.ext_delta[e], a.tab.ext_lo[e] | (a.tab.ext_len[e] == 0 ? 1ull << 63 : 0ull));
      // unchanged since the forward map (cgcm_dev.h make_shw): the recorded CPU pointer
      hr[m] = g - dl.x;
      const bool ok = g != 0 && uw != SH_NONE && (fl & UF_ACTIVE) && e < n_ext && ((g - dl.y) >> 32) == 0 &&
                      (uint32_t)hr[m] == (uint32_t)xc.h[m] && hr[m] != 0;
      stale[m] = st_epoch(w) != cur_ep;
      dfr[m] = defer && (uw & SH_DEFER);
      rare = rare || !ok || (stale[m] && !(fl & UF_READONLY));
    }
    if (__any_sync(0xffffffffu, rare)) {  // the whole group to k_rev_fix (nothing written here)
      if (lane == 0) a.wlist[atomicAdd(a.wcount, 1ull)] = cb;
    } else {
      ++c_fast;
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        if (stale[m]) *lo_word(a.tab.st + su[m]) = cur_ep;  // Alg. 2 line 3 (read-only: never copied back)
        if (DEC && !dfr[m]) red_add(a.tab.rc + su[m], dec);  // Alg. 3 (a deferred reference is dropped)
        if (!DEC && dfr[m]) red_add(a.tab.rc + su[m], 1);   // materialised
      }
      st_stream2(reinterpret_cast<void *>(a0base + 16ull * c), pol_s, hr[0], hr[1]);
      if (lane == 0 || (lane == 16 && cb + 16 < nch)) {
        const uint32_t wi = (cb >> 4) + (lane >> 4);
        a.hitmask[wi] = 0xFFFFFFFFu;
        a.slowmask[wi] = 0u;
      }
    }
  };

  const uint32_t cb0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u);
  Rx X0, X1, X2;
  load_in(cb0 + lane, X0);
  load_in(cb0 + lane + stride, X1);
  gather(X0);
  for (uint32_t cb = cb0; cb < nch;) {
    step(X0, X1, X2, cb);
    if ((cb += stride) >= nch) break;
    step(X1, X2, X0, cb);
    if ((cb += stride) >= nch) break;
    step(X2, X0, X1, cb);
    cb += stride;
  }
  flush_count(&a.st->hits, 2ull * c_fast);
  flush_count(&a.st->translated, 2ull * c_fast);
}

// the warp groups k_rev_fast listed: every chunk through rev_chunk_slow; usually none
template <bool DEC, bool ES>
__global__ void __launch_bounds__(REV_THREADS, 1) k_rev_fix(const __grid_constant__ SlotArgs a) {
  const uint32_t n = (uint32_t)*a.wcount;
  if (n == 0) return;
  extern __shared__ __align__(16) unsigned char smem[];
  ulonglong2 *s_dl = reinterpret_cast<ulonglong2 *>(smem);
  uint32_t *s_len = reinterpret_cast<uint32_t *>(s_dl + (ES ? a.tab.n_ext : 0));
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) {
      s_dl[t] = make_ulonglong2(a.tab.ext_delta[t], a.tab.ext_lo[t]);
      s_len[t] = a.tab.ext_len[t];
    }
  __syncthreads();
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi = sg.ptr + 8ull * sg.n;
  const uint64_t *shp = reinterpret_cast<const uint64_t *>(sg.shadow);
  const uint32_t nw = gridDim.x * (blockDim.x >> 5);
  for (uint32_t i = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < n; i += nw) {
    const uint64_t cb = a.wlist[i], c = cb + (threadIdx.x & 31);
    RevIn x;
    x.g[0] = x.g[1] = 0;
    x.h[0] = x.h[1] = make_shw(0, SH_NONE);
    x.valid = 0;
    uint64_t w[2] = {0, 0};
    if (c < a.nchunks) {
      const uint64_t a0 = a0base + 16ull * c;
      x.valid = (a0 >= sg.ptr ? 1u : 0u) | (a0 + 8 < hi ? 2u : 0u);
      const int64_t i0 = ((int64_t)(a0 - sg.ptr)) >> 3;
      for (int m = 0; m < 2; ++m)
        if ((x.valid >> m) & 1) {
          x.g[m] = reinterpret_cast<const uint64_t *>(a0)[m];
          x.h[m] = shp[i0 + m];
          if (shw_unit(x.h[m]) != SH_NONE && x.g[m] != 0) w[m] = a.tab.st[sh_unit(shw_unit(x.h[m]))];
        }
    }
    rev_chunk_slow<DEC, ES>(a, s_dl, s_len, c, cb, x, w[0], w[1]);
  }
}

template <bool DEC, bool ES>
static int launch_rev_fast1(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = (ES ? al16(20 * (size_t)a.tab.n_ext) + 16 : 0) + 64;
  static bool configured = false;
  if (!configured) {
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaError_t e = cudaFuncSetAttribute(k_rev_fast<DEC, ES>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  const uint64_t want = (a.nchunks + REV_THREADS - 1) / REV_THREADS;
  const int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  if (cudaMemsetAsync(a.wcount, 0, sizeof(unsigned long long), s) != cudaSuccess) return (int)cudaGetLastError();
  k_rev_fast<DEC, ES><<<grid, REV_THREADS, smem, s>>>(a);
  k_rev_fix<DEC, ES><<<grid, REV_THREADS, smem, s>>>(a);
  return (int)cudaGetLastError();
}


// Calls of 2^31 chunks or more (32 GiB of slots): every chunk through the general per-chunk code
// (64-bit chunk indices; no pipeline).
template <bool ES, bool V3, bool DELTA>
__global__ void __launch_bounds__(FWD_FAST_THREADS, 1) k_fwd_big(const __grid_constant__ SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  uint64_t *s_ext = reinterpret_cast<uint64_t *>(smem);
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) s_ext[t] = a.tab.ext_delta[t];
  __syncthreads();
  const uint64_t a0base = a.segs[0].ptr & ~15ull, stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t cb = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); cb < a.nchunks; cb += stride) {
    const uint64_t c = cb + (threadIdx.x & 31);
    uint64_t v0 = 0, v1 = 0;
    if (c < a.nchunks) {
      const uint64_t a0 = a0base + 16ull * c;
      const Seg &sg = a.segs[0];
      if (a0 >= sg.ptr) v0 = reinterpret_cast<const uint64_t *>(a0)[0];
      if (a0 + 8 < sg.ptr + 8ull * sg.n) v1 = reinterpret_cast<const uint64_t *>(a0)[1];
    }
    fwd_chunk_slow<ES, V3, DELTA>(a, s_ext, c, cb, v0, v1);
  }
}
template <bool DEC, bool ES>
__global__ void __launch_bounds__(REV_THREADS, 1) k_rev_big(const __grid_constant__ SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  ulonglong2 *s_dl = reinterpret_cast<ulonglong2 *>(smem);
  uint32_t *s_len = reinterpret_cast<uint32_t *>(s_dl + (ES ? a.tab.n_ext : 0));
  if (ES)
    for (int t = threadIdx.x; t < a.tab.n_ext; t += blockDim.x) {
      s_dl[t] = make_ulonglong2(a.tab.ext_delta[t], a.tab.ext_lo[t]);
      s_len[t] = a.tab.ext_len[t];
    }
  __syncthreads();
  const Seg sg = a.segs[0];
  const uint64_t a0base = sg.ptr & ~15ull, hi = sg.ptr + 8ull * sg.n, stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t *shp = reinterpret_cast<const uint64_t *>(sg.shadow);
  for (uint64_t cb = (uint64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31u); cb < a.nchunks; cb += stride) {
    const uint64_t c = cb + (threadIdx.x & 31);
    RevIn x;
    x.g[0] = x.g[1] = 0;
    x.h[0] = x.h[1] = make_shw(0, SH_NONE);
    x.valid = 0;
    uint64_t w[2] = {0, 0};
    if (c < a.nchunks) {
      const uint64_t a0 = a0base + 16ull * c;
      x.valid = (a0 >= sg.ptr ? 1u : 0u) | (a0 + 8 < hi ? 2u : 0u);
      const int64_t i0 = ((int64_t)(a0 - sg.ptr)) >> 3;
      for (int m = 0; m < 2; ++m)
        if ((x.valid >> m) & 1) {
          x.g[m] = reinterpret_cast<const uint64_t *>(a0)[m];
          x.h[m] = shp[i0 + m];
          if (shw_unit(x.h[m]) != SH_NONE && x.g[m] != 0) w[m] = a.tab.st[sh_unit(shw_unit(x.h[m]))];
        }
    }
    rev_chunk_slow<DEC, ES>(a, s_dl, s_len, c, cb, x, w[0], w[1]);
  }
}
template <bool ES, bool V3, bool DELTA>
static int launch_fwd_big1(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = (ES ? al16(8 * (size_t)a.tab.n_ext) : 0) + 64;
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  cudaError_t e = cudaFuncSetAttribute(k_fwd_big<ES, V3, DELTA>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
  if (e != cudaSuccess) return (int)e;
  k_fwd_big<ES, V3, DELTA><<<nsm, FWD_FAST_THREADS, smem, s>>>(a);
  return (int)cudaGetLastError();
}
template <bool DEC, bool ES>
static int launch_rev_big1(const SlotArgs &a, int nsm, cudaStream_t s) {
  const size_t smem = (ES ? al16(20 * (size_t)a.tab.n_ext) + 16 : 0) + 64;
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  cudaError_t e = cudaFuncSetAttribute(k_rev_big<DEC, ES>, cudaFuncAttributeMaxDynamicSharedMemorySize, optin);
  if (e != cudaSuccess) return (int)e;
  k_rev_big<DEC, ES><<<nsm, REV_THREADS, smem, s>>>(a);
  return (int)cudaGetLastError();
}
template <bool DEC>
static int launch_rev_lean(const SlotArgs &a, int nsm, cudaStream_t s) {
  const bool es = a.tab.n_ext <= EXT_SMEM;
  static const bool force_big = std::getenv("CGCM_FORCE_BIG") != nullptr;  // tests: the general per-chunk code
  if (a.nchunks >= (1ull << 31) || force_big) return es ? launch_rev_big1<DEC, true>(a, nsm, s) : launch_rev_big1<DEC, false>(a, nsm, s);
  return es ? launch_rev_fast1<DEC, true>(a, nsm, s) : launch_rev_fast1<DEC, false>(a, nsm, s);
}

// the operation sets the runtime uses
#define CGCM_SLOT_OPS(X)                                                                          \
  X(DIR_FWD, OP_WRITE | OP_INC | OP_HITMASK)           /* map: forward rewrite + refcount (a2)   */ \
  X(DIR_FWD, OP_WRITE)                                 /* complete pending slots after alloc     */ \
  X(DIR_FWD, OP_DECPLAIN)                              /* rollback of pending increments         */ \
  X(DIR_FWD, OP_DEC)                                   /* release by CPU pointer (Alg. 3)        */ \
  X(DIR_FWD, OP_INCPLAIN)                              /* rollback of release                    */ \
  X(DIR_FWD, OP_GATE | OP_CHECKMAPPED)                 /* unmap by CPU pointer (Alg. 2, a4)      */ \
  X(DIR_FWD, OP_WRITE | OP_INCPLAIN)                   /* rollback of reverse+release            */ \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_HITMASK)          /* unmapArray: reverse (a3) + gate (a4)   */ \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_DEC | OP_HITMASK) /* unmapArray + releaseArray fused        */ \
  X(DIR_REV, OP_GATE)                                  /* gate only (outer up to date)           */ \
  X(DIR_REV, OP_WRITE)                                 /* reverse only (copy-back of a unit)     */ \
  X(DIR_REV, OP_WRITE | OP_DECPLAIN)                   /* rollback of forward map (in place)     */ \
  X(DIR_REV, OP_INCPLAIN)                              /* re-map of an array-mapped outer (A9)   */ \
  X(DIR_REV, OP_DEC)                                   /* releaseArray of an array-mapped outer  */ \
  X(DIR_REV, OP_DECPLAIN)                              /* rollback of REV INCPLAIN               */

static size_t slots_smem(const SlotArgs &a, int dir, bool pd) {
  return (pd ? pd_stage_bytes(a.pd) : stage_bytes(a.fx, false)) + (dir == DIR_REV ? stage_bytes(a.rx, a.rx.h == 0) : 0) +
         (a.tab.n_ext <= EXT_SMEM ? al16(8 * (size_t)a.tab.n_ext) : 0) + 64;
}

template <int DIR, int OPS, int FH, int SH>
static int launch_one(const SlotArgs &a, int nsm, cudaStream_t s) {
  size_t smem = slots_smem(a, DIR, FH == FH_PD);
  // the 48 KiB default covers static + dynamic shared memory: opt in to the full carve-out once
  static bool configured = false;
  if (!configured) {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, k_slots<DIR, OPS, FH, SH>);
    if (e != cudaSuccess) return (int)e;
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    e = cudaFuncSetAttribute(k_slots<DIR, OPS, FH, SH>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             optin - (int)fa.sharedSizeBytes);
    if (e != cudaSuccess) return (int)e;
    configured = true;
  }
  constexpr int T = SlotCfg<DIR, SH>::threads;
  uint64_t want = (a.nchunks - a.cbeg + T - 1) / T;
  int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  k_slots<DIR, OPS, FH, SH><<<grid, T, smem, s>>>(a);
  return (int)cudaGetLastError();  // 0 or the cudaError_t of the launch
}

// hot operation sets get depth-specialised forward lookups (and shadow variants)
#define CGCM_HOT_OPS(X)                             \
  X(DIR_FWD, OP_WRITE | OP_INC | OP_HITMASK)         \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_DEC | OP_HITMASK) \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_HITMASK)

int launch_slots(int dir, int ops, const SlotArgs &a, int nsm, cudaStream_t s, int *nlaunch) {
  *nlaunch = 1;
  static const bool no_pipe = std::getenv("CGCM_NO_PIPELINE") != nullptr;  // A/B experiments
  if (dir == DIR_FWD && ops == (OP_WRITE | OP_INC | OP_HITMASK) && a.pd.nseg > 0 && a.nseg == 1 && a.seg_inplace &&
      a.sel == SEL_ALL && a.cbeg == 0 && !no_pipe)
  {
    static const bool no_lean = std::getenv("CGCM_NO_LEAN") != nullptr;  // A/B experiments
    if (a.segs_host_shadow && a.pd.nseg == 1 && !no_lean) {
      const bool es = a.tab.n_ext <= EXT_SMEM, v3 = a.pd.v3 != 0, dl = a.dn > 0;
      static const bool force_big = std::getenv("CGCM_FORCE_BIG") != nullptr;  // tests: the general per-chunk code
      const bool big = a.nchunks >= (1ull << 31) || force_big;
      *nlaunch = big ? 1 : 2;  // k_fwd_fast + k_fwd_fix
#define FWD_PASS(E, V, D) \
  if (es == E && v3 == V && dl == D) return big ? launch_fwd_big1<E, V, D>(a, nsm, s) : launch_fwd_fast1<E, V, D>(a, nsm, s);
      FWD_PASS(true, true, false) FWD_PASS(true, false, false) FWD_PASS(false, true, false) FWD_PASS(false, false, false)
      FWD_PASS(true, true, true) FWD_PASS(true, false, true) FWD_PASS(false, true, true) FWD_PASS(false, false, true)
#undef FWD_PASS
    }
    return a.segs_host_shadow ? launch_map_pd<1>(a, nsm, s) : launch_map_pd<0>(a, nsm, s);
  }
  constexpr int UNMAP = OP_WRITE | OP_GATE | OP_HITMASK, UNMAP_REL = OP_WRITE | OP_GATE | OP_DEC | OP_HITMASK;
  if (dir == DIR_REV && (ops == UNMAP || ops == UNMAP_REL || ops == OP_DEC) && a.segs_host_shadow &&
      a.sel == SEL_ALL && a.cbeg == 0 && !no_pipe) {
    // pipelined pass over the recorded slots, then the generic kernel over the slots it left
    if (cudaMemsetAsync(a.slowcount, 0, sizeof(unsigned long long), s) != cudaSuccess) return (int)cudaGetLastError();
    static const bool no_lean = std::getenv("CGCM_NO_LEAN") != nullptr;  // A/B experiments
    // the lean pass: one in-place segment with a shadow, snapshot mode (releases as reductions)
    const bool lean = !no_lean && ops != OP_DEC && a.nseg == 1 && a.seg_inplace && a.no_journal &&
                      (ops == UNMAP || a.dec_red);
    int r = lean ? (ops == UNMAP ? launch_rev_lean<false>(a, nsm, s) : launch_rev_lean<true>(a, nsm, s))
            : ops == UNMAP ? launch_unmap_sh<UNMAP>(a, nsm, s)
            : ops == UNMAP_REL ? launch_unmap_sh<UNMAP_REL>(a, nsm, s)
                               : launch_unmap_sh<OP_DEC>(a, nsm, s);
    if (r != 0) return r;
    SlotArgs b = a;
    b.sel = SEL_SLOW;
    static const bool force_big = std::getenv("CGCM_FORCE_BIG") != nullptr;
    *nlaunch = lean && a.nchunks < (1ull << 31) && !force_big ? 3 : 2;  // (k_rev_fast + k_rev_fix) + k_slots
    return launch_slots(dir, ops, b, nsm, s, &r);
  }
  // the forward index qualifies for the specialised path: one segment, no wide bucket, h <= 3
  int fh = a.pd.nseg > 0 ? FH_PD : a.fx.nseg <= 1 && a.fx_nowide && a.fx.h <= 3 ? a.fx.h : -1;
  const bool sh = a.segs_host_shadow;
#define X(D, O)                                                        \
  if (dir == D && ops == (O)) {                                        \
    if (sh) {                                                          \
      switch (fh) {                                                    \
        case FH_PD: return launch_one<D, (O), FH_PD, 1>(a, nsm, s);    \
        case 2: return launch_one<D, (O), 2, 1>(a, nsm, s);            \
        case 3: return launch_one<D, (O), 3, 1>(a, nsm, s);            \
        default: return launch_one<D, (O), -1, 1>(a, nsm, s);          \
      }                                                                \
    }                                                                  \
    switch (fh) {                                                      \
      case FH_PD: return launch_one<D, (O), FH_PD, 0>(a, nsm, s);      \
      case 0: return launch_one<D, (O), 0, 0>(a, nsm, s);              \
      case 1: return launch_one<D, (O), 1, 0>(a, nsm, s);              \
      case 2: return launch_one<D, (O), 2, 0>(a, nsm, s);              \
      case 3: return launch_one<D, (O), 3, 0>(a, nsm, s);              \
      default: return launch_one<D, (O), -1, 0>(a, nsm, s);            \
    }                                                                  \
  }
  CGCM_HOT_OPS(X)
#undef X
#define X(D, O) \
  if (dir == D && ops == (O)) return launch_one<D, (O), -1, 0>(a, nsm, s);
  CGCM_SLOT_OPS(X)
#undef X
  return -2;  // unsupported combination
}

// -------------------------------------------------------------------------------------------------
// Index levels (a0): lvl[k][j] = keys[j*8^k] - keys[bucket start], u32, padded to groups of 8
// -------------------------------------------------------------------------------------------------
__global__ void k_build_level(const uint64_t *keys, int n, int h, const uint32_t *wide, int k, uint32_t *lvl,
                              size_t cap) {
  int64_t cnt = ((int64_t)n + (1ll << (3 * k)) - 1) >> (3 * k);
  int64_t padded = (cnt + 7) / 8 * 8;
  for (int64_t jj = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; jj < padded && jj < (int64_t)cap;
       jj += (int64_t)gridDim.x * blockDim.x) {
    uint32_t val = 0xFFFFFFFFu;
    if (jj < cnt) {
      int64_t idx = jj << (3 * k);
      int64_t t = idx >> (3 * h);
      bool w = (wide[t >> 5] >> (t & 31)) & 1u;
      val = w ? 0u : (uint32_t)(keys[idx] - keys[t << (3 * h)]);
    }
    lvl[jj] = val;
  }
}

void launch_build_levels(const uint64_t *keys, int n, int h, const uint32_t *wide, uint32_t *const *lvl,
                         const size_t *lvl_cap, cudaStream_t s) {
  for (int k = 0; k < h; ++k) {
    int64_t cnt = ((int64_t)n + (1ll << (3 * k)) - 1) >> (3 * k);
    int grid = (int)std::min<int64_t>((cnt + 255) / 256 + 1, 4096);
    (void)cudaGetLastError();
    k_build_level<<<grid, 256, 0, s>>>(keys, n, h, wide, k, lvl[k], lvl_cap[k]);
  }
}

// new table row i = old row old_idx[i] (surviving unit) or a fresh row (declared since the last build)
__global__ void k_remap(int n, const int32_t *old_idx, const uint64_t *size, const uint32_t *flags,
                        const uint32_t *epoch0, TableDev o, TableDev t) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  int k = old_idx[i];
  if (k >= 0) {
    t.hot[i] = o.hot[k];
    t.hotc[i] = make_hotc(o.hot[k]);
    t.st[i] = o.st[k];
    t.rc[i] = o.rc[k];
  } else {
    const uint64_t h = make_hot(size[i], NO_EXT, flags[i]);
    t.hot[i] = h;
    t.hotc[i] = make_hotc(h);
    t.st[i] = make_st(h, epoch0[i]);
    t.rc[i] = 0;
  }
}
void launch_remap(int n, const int32_t *old_idx, const uint64_t *size, const uint32_t *flags, const uint32_t *epoch0,
                  TableDev old_tab, TableDev new_tab, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_remap<<<(n + 255) / 256, 256, 0, s>>>(n, old_idx, size, flags, epoch0, old_tab, new_tab);
  }
}

size_t sort_keys_temp_bytes(int n) {
  size_t bytes = 0;
  cub::DeviceRadixSort::SortKeys(nullptr, bytes, (const uint32_t *)nullptr, (uint32_t *)nullptr, n);
  return bytes;
}
void launch_sort_keys(void *temp, size_t temp_bytes, const uint32_t *kin, uint32_t *kout, int n, cudaStream_t s) {
  cub::DeviceRadixSort::SortKeys(temp, temp_bytes, kin, kout, n, 0, 32, s);
}

// -------------------------------------------------------------------------------------------------
// Transfer planning on the device (activation packs, copy-back runs): segmented scans over the sorted
// unit list, so that the host handles one descriptor per DMA instead of one entry per unit.
// -------------------------------------------------------------------------------------------------
size_t plan_temp_bytes(int n) {
  size_t a = 0;
  cub::DeviceScan::InclusiveSum(nullptr, a, (const uint32_t *)nullptr, (uint32_t *)nullptr, n);
  return a;
}
__device__ __forceinline__ uint64_t unit_size(const TableDev &t, uint32_t u) {
  const uint32_t s = hot_size32(t.hot[u]);
  return s == BIG_SIZE ? t.size64[u] : s;
}
__global__ void k_pack_flags(const uint32_t *S, int n, TableDev tab, uint64_t gapmax, int window, uint32_t *F,
                             uint32_t *G, unsigned long long *cnt) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t sz = 0;
  bool glob = false;
  if (i < n) {
    const uint32_t u = S[i];
    const uint64_t b = tab.base[u];
    sz = unit_size(tab, u);
    glob = hot_flags(tab.hot[u]) & UF_GLOBAL;
    uint32_t f = 1, g = 0;
    if (i > 0) {
      const uint32_t v = S[i - 1];
      const uint64_t e = tab.base[v] + unit_size(tab, v);
      const bool gv = hot_flags(tab.hot[v]) & UF_GLOBAL;
      f = (glob || gv || b < e || b - e > gapmax || (b >> window) != (tab.base[v] >> window)) ? 1u : 0u;
      g = (!f && b != e) ? 1u : 0u;
    }
    F[i] = f;
    G[i] = g;
  }
  // bytes and globals of the whole list: one atomic per warp
  unsigned long long ws = sz, wg = glob ? 1 : 0;
  for (int o = 16; o; o >>= 1) {
    ws += __shfl_xor_sync(0xffffffffu, ws, o);
    wg += __shfl_xor_sync(0xffffffffu, wg, o);
  }
  if ((threadIdx.x & 31) == 0) {
    if (ws) atomicAdd(&cnt[2], ws);
    if (wg) atomicAdd(&cnt[1], wg);
  }
}
__global__ void k_pack_first(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *pid,
                             PackDesc *packs) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n || !F[i]) return;
  PackDesc &P = packs[pid[i] - 1];
  P.first = (uint32_t)i;
  P.h0 = tab.base[S[i]];
}
__global__ void k_pack_last(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *pid,
                            const uint32_t *gscan, PackDesc *packs) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  if (i + 1 < n && !F[i + 1]) return;
  PackDesc &P = packs[pid[i] - 1];
  P.last = (uint32_t)i;
  P.h1 = tab.base[S[i]] + unit_size(tab, S[i]);
  P.gaps = gscan[i] - gscan[P.first] > 0 ? 1u : 0u;
  P.pad = 0;
}
int launch_plan_packs1(const uint32_t *S, int n, TableDev tab, uint64_t gapmax, int window, uint32_t *F, uint32_t *G,
                       uint32_t *pid, uint32_t *gscan, unsigned long long *cnt, void *temp, size_t temp_bytes,
                       cudaStream_t s) {
  if (n <= 0) return 0;
  (void)cudaGetLastError();
  cudaMemsetAsync(cnt, 0, 32, s);
  const int g = (n + 255) / 256;
  k_pack_flags<<<g, 256, 0, s>>>(S, n, tab, gapmax, window, F, G, cnt);
  size_t tb = temp_bytes;
  cub::DeviceScan::InclusiveSum(temp, tb, F, pid, n, s);
  tb = temp_bytes;
  cub::DeviceScan::InclusiveSum(temp, tb, G, gscan, n, s);
  cudaMemcpyAsync(cnt, pid + (n - 1), 4, cudaMemcpyDeviceToDevice, s);  // cnt[0] (low word) = #packs
  return (int)cudaGetLastError();
}
int launch_plan_packs2(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *pid,
                       const uint32_t *gscan, PackDesc *packs, cudaStream_t s) {
  if (n <= 0) return 0;
  (void)cudaGetLastError();
  const int g = (n + 255) / 256;
  k_pack_first<<<g, 256, 0, s>>>(S, n, tab, F, pid, packs);
  k_pack_last<<<g, 256, 0, s>>>(S, n, tab, F, pid, gscan, packs);
  return (int)cudaGetLastError();
}
__global__ void k_plan_set_ext(const uint32_t *S, int n, const uint32_t *pid, const uint32_t *run, TableDev tab,
                               uint32_t epoch, int set_epoch) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t u = S[i], p = pid[i] - 1;
  uint64_t h = tab.hot[u];
  h = (h & ~(EXT_MASK << ESHIFT)) | ((uint64_t)(run[p] & EXT_MASK) << ESHIFT);
  h |= (uint64_t)(UF_STORAGE | UF_ACTIVE) << FSHIFT;
  tab.hot[u] = h;
  tab.hotc[u] = make_hotc(h);
  tab.st[u] = make_st(h, set_epoch ? epoch : st_epoch(tab.st[u]));
}
void launch_plan_set_ext(const uint32_t *S, int n, const uint32_t *pid, const uint32_t *run, TableDev tab,
                         uint32_t epoch, int set_epoch, cudaStream_t s) {
  if (n <= 0) return;
  (void)cudaGetLastError();
  k_plan_set_ext<<<(n + 255) / 256, 256, 0, s>>>(S, n, pid, run, tab, epoch, set_epoch);
}

// copy-back runs: a new run unless the unit directly follows the previous one in index order, starts
// where it ends on the host, lives in the same (mirrored) extent, and neither is array-mapped
__global__ void k_cb_flags(const uint32_t *S, int n, TableDev tab, uint32_t *F) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t u = S[i];
  const uint64_t hu = tab.hot[u];
  uint32_t f = 1;
  if (i > 0) {
    const uint32_t v = S[i - 1];
    const uint64_t hv = tab.hot[v];
    const bool arr = (hot_flags(hu) | hot_flags(hv)) & UF_ARRAYMAPPED;
    f = (arr || u != v + 1 || tab.base[u] != tab.base[v] + unit_size(tab, v) || hot_ext(hu) != hot_ext(hv)) ? 1u : 0u;
  }
  F[i] = f;
}
__global__ void k_cb_first(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *rid,
                           CopyRun *runs) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n || !F[i]) return;
  const uint32_t u = S[i];
  const uint64_t h = tab.hot[u];
  CopyRun &R = runs[rid[i] - 1];
  R.first = (uint32_t)i;
  R.unit = u;
  R.arr = (hot_flags(h) & UF_ARRAYMAPPED) ? 1u : 0u;
  R.host = tab.base[u];
  R.dev = tab.base[u] + tab.ext_delta[hot_ext(h)];  // Alg. 1's devptr of the run's first unit
  R.pad = 0;
}
__global__ void k_cb_last(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *rid,
                          CopyRun *runs) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  if (i + 1 < n && !F[i + 1]) return;
  CopyRun &R = runs[rid[i] - 1];
  R.last = (uint32_t)i;
  R.len = tab.base[S[i]] + unit_size(tab, S[i]) - R.host;
}
int launch_plan_copyback1(const uint32_t *S, int n, TableDev tab, uint32_t *F, uint32_t *rid, unsigned long long *cnt,
                          void *temp, size_t temp_bytes, cudaStream_t s) {
  if (n <= 0) return 0;
  (void)cudaGetLastError();
  cudaMemsetAsync(cnt, 0, 32, s);
  const int g = (n + 255) / 256;
  k_cb_flags<<<g, 256, 0, s>>>(S, n, tab, F);
  size_t tb = temp_bytes;
  cub::DeviceScan::InclusiveSum(temp, tb, F, rid, n, s);
  cudaMemcpyAsync(cnt, rid + (n - 1), 4, cudaMemcpyDeviceToDevice, s);  // cnt[0] (low word) = #runs
  return (int)cudaGetLastError();
}
int launch_plan_copyback2(const uint32_t *S, int n, TableDev tab, const uint32_t *F, const uint32_t *rid,
                          CopyRun *runs, cudaStream_t s) {
  if (n <= 0) return 0;
  (void)cudaGetLastError();
  const int g = (n + 255) / 256;
  k_cb_first<<<g, 256, 0, s>>>(S, n, tab, F, rid, runs);
  k_cb_last<<<g, 256, 0, s>>>(S, n, tab, F, rid, runs);
  return (int)cudaGetLastError();
}

// page state words (w[2] of every page entry): valid with the extent when every unit a lookup in the page
// can return is ACTIVE with its copy in that one extent (cgcm_dev.h "Page directory")
__global__ void k_pd_state(PdDev pd, uint64_t npages, TableDev tab) {
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < npages; e += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t *w = const_cast<uint32_t *>(pd.ent) + 8 * e;
    const uint32_t j0 = w[0], w1 = w[1], cnt = w1 & PD_CNT_MAX, end0 = w1 >> PD_END_SHIFT;
    uint32_t state = 0;
    if (cnt <= (uint32_t)PD_K3) {
      bool ok = true, any = false;
      uint32_t ext = 0;
      auto take = [&](uint32_t u) {
        const uint64_t h = tab.hot[u];
        const uint32_t fl = hot_flags(h), x = hot_ext(h);
        ok = ok && (fl & UF_ACTIVE) && (fl & UF_STORAGE) && (!any || x == ext);
        ext = x;
        any = true;
      };
      if (j0 != 0xFFFFFFFFu && end0 > 0) take(j0);
      for (uint32_t t = 0; t < cnt; ++t) take(j0 + 1 + t);
      if (ok && any) state = PD_STATE_VALID | (ext & (uint32_t)EXT_MASK);
    }
    w[2] = state;
  }
}
void launch_pd_state(PdDev pd, uint64_t npages, TableDev tab, cudaStream_t s) {
  if (npages == 0) return;
  (void)cudaGetLastError();
  const uint64_t want = (npages + 255) / 256;
  k_pd_state<<<(int)std::min<uint64_t>(want, 148 * 16), 256, 0, s>>>(pd, npages, tab);
}

// frees of a sorted unit list (Alg. 3's cuMemFree at refCount 0), planned before k_deactivate clears the
// flags: per extent the number of copies it loses (warp-aggregated), the array-mapped units (the host
// drops their shadows), counts of frees and of globals (which keep their named region)
__global__ void k_free_plan(const uint32_t *S, int n, TableDev tab, uint32_t *run_dec, uint32_t *arr_out,
                            unsigned long long *cnt) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  bool fr = false, glob = false, arr = false;
  uint32_t x = 0, e = 0xFFFFFFFFu;
  if (i < n) {
    x = S[i];
    if ((i == 0 || S[i - 1] != x) && tab.rc[x] == 0) {
      const uint64_t h = tab.hot[x];
      glob = hot_flags(h) & UF_GLOBAL;
      fr = !glob && (hot_flags(h) & UF_STORAGE);
      arr = hot_flags(h) & UF_ARRAYMAPPED;
      if (fr) e = hot_ext(h);
    }
  }
  const unsigned peers = __match_any_sync(0xffffffffu, e);
  if (fr && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(run_dec + e, (uint32_t)__popc(peers));
  const unsigned nf = __popc(__ballot_sync(0xffffffffu, fr)), ng = __popc(__ballot_sync(0xffffffffu, glob));
  if ((threadIdx.x & 31) == 0) {
    if (nf) atomicAdd(&cnt[0], (unsigned long long)nf);
    if (ng) atomicAdd(&cnt[1], (unsigned long long)ng);
  }
  const unsigned long long ix = warp_append(&cnt[2], arr);
  if (arr) {
    arr_out[2 * ix] = x;
    arr_out[2 * ix + 1] = fr ? e : 0xFFFFFFFFu;
  }
}
void launch_free_plan(const uint32_t *S, int n, TableDev tab, uint32_t *run_dec, int nruns, uint32_t *arr_out,
                      unsigned long long *cnt, cudaStream_t s) {
  (void)cudaGetLastError();
  cudaMemsetAsync(cnt, 0, 32, s);
  cudaMemsetAsync(run_dec, 0, 4 * (size_t)(nruns > 0 ? nruns : 1), s);
  if (n > 0) k_free_plan<<<(n + 255) / 256, 256, 0, s>>>(S, n, tab, run_dec, arr_out, cnt);
}

// -------------------------------------------------------------------------------------------------
// small bookkeeping kernels
// -------------------------------------------------------------------------------------------------
__global__ void k_unit_ops(const UnitOp *ops, int n, TableDev tab) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  UnitOp o = ops[i];
  switch (o.op) {
    case UOP_ADD_RC: atomicAdd(tab.rc + o.unit, (int32_t)(int64_t)o.val); break;
    case UOP_SET_EPOCH: *lo_word(tab.st + o.unit) = (uint32_t)o.val; break;
    case UOP_OR_FLAGS:
      atomicOr(hi_word(tab.hot + o.unit), (uint32_t)o.val << (FSHIFT - 32));
      atomicOr(hi_word(tab.st + o.unit), (uint32_t)o.val << (FSHIFT - 32));
      break;
    case UOP_AND_FLAGS:
      atomicAnd(hi_word(tab.hot + o.unit), ((uint32_t)o.val << (FSHIFT - 32)) | ((1u << (FSHIFT - 32)) - 1));
      atomicAnd(hi_word(tab.st + o.unit), ((uint32_t)o.val << (FSHIFT - 32)) | ((1u << (FSHIFT - 32)) - 1));
      break;
    case UOP_SET_RC: tab.rc[o.unit] = (int32_t)(int64_t)o.val; break;
  }
}
// after k_unit_ops: the compact words of every unit whose flags an op changed (from the final hot word)
__global__ void k_hotc_ops(const UnitOp *ops, int n, TableDev tab) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const UnitOp o = ops[i];
  if (o.op == UOP_OR_FLAGS || o.op == UOP_AND_FLAGS) tab.hotc[o.unit] = make_hotc(tab.hot[o.unit]);
}
void launch_unit_ops(const UnitOp *ops, int n, TableDev tab, cudaStream_t s, bool hotc) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_unit_ops<<<(n + 255) / 256, 256, 0, s>>>(ops, n, tab);
    if (hotc) k_hotc_ops<<<(n + 255) / 256, 256, 0, s>>>(ops, n, tab);
  }
}

// activation: the unit's copy is in extent ext[i]; epoch = globalEpoch (A5 reading R1)
__global__ void k_set_ext(const uint32_t *units, const uint32_t *exts, int n, TableDev tab, uint32_t epoch,
                          int set_epoch) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t u = units[i];
  uint64_t h = tab.hot[u];
  h = (h & ~(EXT_MASK << ESHIFT)) | ((uint64_t)(exts[i] & EXT_MASK) << ESHIFT);
  h |= (uint64_t)(UF_STORAGE | UF_ACTIVE) << FSHIFT;
  tab.hot[u] = h;
  tab.hotc[u] = make_hotc(h);
  tab.st[u] = make_st(h, set_epoch ? epoch : st_epoch(tab.st[u]));
}
void launch_set_ext(const uint32_t *units, const uint32_t *exts, int n, TableDev tab, uint32_t epoch, int set_epoch,
                    cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_set_ext<<<(n + 255) / 256, 256, 0, s>>>(units, exts, n, tab, epoch, set_epoch);
  }
}

__global__ void k_deactivate(const uint32_t *units, int n, TableDev tab) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t u = units[i];
  if (tab.rc[u] != 0) return;
  uint64_t h = tab.hot[u];
  if (hot_flags(h) & UF_GLOBAL) {
    h &= ~((uint64_t)(UF_ARRAYMAPPED | UF_ACTIVE) << FSHIFT);  // named region persists
  } else {
    h &= ~((uint64_t)(UF_ARRAYMAPPED | UF_ACTIVE | UF_STORAGE) << FSHIFT);  // cuMemFree (Alg. 3)
    h |= NO_EXT << ESHIFT;
  }
  tab.hot[u] = h;
  tab.hotc[u] = make_hotc(h);
  tab.st[u] = make_st(h, st_epoch(tab.st[u]));
}
void launch_deactivate(const uint32_t *units, int n, TableDev tab, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_deactivate<<<(n + 255) / 256, 256, 0, s>>>(units, n, tab);
  }
}

__global__ void k_restore_epochs(const Journal *j, int n, TableDev tab) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  *lo_word(tab.st + j[i].unit) = j[i].old_epoch;
}
void launch_restore_epochs(const Journal *j, int n, TableDev tab, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_restore_epochs<<<(n + 255) / 256, 256, 0, s>>>(j, n, tab);
  }
}

// after a release pass through reductions: units whose refcount went negative (underflow) or
// reached 0 while active (freed by this call)
__global__ void k_release_scan(TableDev tab, int n, Status *st, unsigned long long *lc, uint32_t *free_list) {
  unsigned under = 0;
  for (int base = blockIdx.x * blockDim.x; base < n; base += gridDim.x * blockDim.x) {
    int i = base + threadIdx.x;
    bool fr = false;
    if (i < n) {
      int32_t rc = tab.rc[i];
      under += rc < 0;
      fr = rc == 0 && (hot_flags(tab.hot[i]) & UF_ACTIVE);
    }
    unsigned long long ix = warp_append(&lc[2], fr);
    if (fr) free_list[ix] = (uint32_t)i;
  }
  flush_count(&st->underflow, under);
}
void launch_release_scan(TableDev tab, int n, Status *st, unsigned long long *lc, uint32_t *free_list,
                         cudaStream_t s) {
  if (n > 0) {
    int grid = std::min((n + 255) / 256, 1184);
    (void)cudaGetLastError();
    k_release_scan<<<grid, 256, 0, s>>>(tab, n, st, lc, free_list);
  }
}

__global__ void k_gather_state(TableDev tab, const uint32_t *idx, int n, uint64_t *out) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = tab.st[idx[i]];
}
void launch_gather_state(TableDev tab, const uint32_t *idx, int n, uint64_t *out, cudaStream_t s) {
  if (n <= 0) return;
  (void)cudaGetLastError();
  k_gather_state<<<(n + 255) / 256, 256, 0, s>>>(tab, idx, n, out);
}

// deferred references of one shadow become ordinary references (DESIGN.md §6 "Deferred references")
__global__ void k_materialise(const uint64_t *shadow, uint64_t n, int32_t *rc) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t w = shw_unit(shadow[i]);
    if (sh_deferred(w)) red_add(rc + sh_unit(w), 1);
  }
}
void launch_materialise(const uint64_t *shadow_units, uint64_t n, int32_t *rc, cudaStream_t s) {
  if (n == 0) return;
  const uint64_t want = (n + 255) / 256;
  const int grid = (int)std::min<uint64_t>(want, 148 * 8);
  (void)cudaGetLastError();
  k_materialise<<<grid, 256, 0, s>>>(shadow_units, n, rc);
}

// epoch origin moves (once per 2^32 - 16 launches): the current epoch becomes 1, every other 0
__global__ void k_rebase_epochs(TableDev tab, int n, uint32_t cur) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    *lo_word(tab.st + i) = st_epoch(tab.st[i]) == cur ? 1u : 0u;
}
void launch_rebase_epochs(TableDev tab, int n, uint32_t cur, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_rebase_epochs<<<std::min((n + 255) / 256, 1184), 256, 0, s>>>(tab, n, cur);
  }
}

// outer-pointer lookup for mapArray/unmapArray/releaseArray: one thread per pointer, plain
// binary search over the full u64 key array (few pointers: latency, not bandwidth)
__global__ void k_lookup_points(IndexDev ix, TableDev tab, const uint64_t *ptrs, int n, PointInfo *out,
                                const uint64_t *dkeys, const uint32_t *dids, int dn) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t p = ptrs[i];
  int nk = ix.n;
  PointInfo r;
  r.unit = -1;
  r.base = r.size = r.devbase = r.epoch = 0;
  r.refcount = 0;
  r.flags = 0;
  r.pad = 0;
  if (nk > 0 && p >= ix.keys[0]) {
    int lo = 0, len = nk;
    while (len > 1) {
      int half = len >> 1;
      if (ix.keys[lo + half] <= p) lo += half;
      len -= half;
    }
    const uint64_t b = ix.keys[lo], sz = tab.size64[lo];
    if (p - b <= sz) r.unit = lo;
  }
  {  // NEXT-1: a delta unit containing p when the main table missed
    uint64_t db = 0;
    const int d = (dn > 0 && r.unit < 0) ? delta_hit(dkeys, dids, dn, tab, p, db) : -1;
    if (d >= 0) r.unit = d;
  }
  if (r.unit >= 0) {
    const int lo = r.unit;
    const uint64_t h = tab.hot[lo], b = tab.base[lo], sz = tab.size64[lo];
    {
      r.base = b;
      r.size = sz;
      r.flags = hot_flags(h);
      r.devbase = (r.flags & UF_STORAGE) ? b + tab.ext_delta[hot_ext(h)] : 0;
      r.epoch = st_epoch(tab.st[lo]);
      r.refcount = tab.rc[lo];
    }
  }
  out[i] = r;
}
void launch_lookup_points(IndexDev ix, TableDev tab, const uint64_t *ptrs, int n, PointInfo *out,
                          const uint64_t *dkeys, const uint32_t *dids, int dn, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_lookup_points<<<(n + 127) / 128, 128, 0, s>>>(ix, tab, ptrs, n, out, dkeys, dids, dn);
  }
}

// ---- glue kernels (NEXT-4): one GPU thread runs a short CPU region over mapped data ----
// is [g, g + 8) inside the device copy of an active unit?  (extent by device start, then the unit by the
// mirrored host address, then: the unit is ACTIVE and its copy lives in that extent)
__device__ bool glue_ok(const GlueArgs &A, uint64_t g) {
  if (A.n_ext_keys <= 0 || g < A.ext_keys[0]) return false;
  int lo = 0, len = A.n_ext_keys;
  while (len > 1) {
    const int half = len >> 1;
    if (A.ext_keys[lo + half] <= g) lo += half;
    len -= half;
  }
  const uint64_t h = g + A.ext_pay[lo];
  const uint32_t eid = A.ext_id[lo];
  auto owns = [&](int j) {
    const uint64_t w = A.tab.hot[j];
    return (hot_flags(w) & UF_ACTIVE) && (hot_flags(w) & UF_STORAGE) && hot_ext(w) == eid &&
           h - A.tab.base[j] <= A.tab.size64[j] && A.tab.size64[j] - (h - A.tab.base[j]) >= 8;
  };
  if (A.U > 0 && h >= A.tab.base[0]) {
    int j = 0;
    len = A.U;
    while (len > 1) {
      const int half = len >> 1;
      if (A.tab.base[j + half] <= h) j += half;
      len -= half;
    }
    if (owns(j)) return true;
  }
  uint64_t db;  // NEXT-1: the delta units
  const int d = delta_hit(A.dkeys, A.dids, A.dn, A.tab, h, db);
  return d >= 0 && owns(d);
}
__global__ void k_glue(GlueArgs A) {
  uint64_t r[GLUE_REGS];
  for (int i = 0; i < GLUE_REGS; ++i) r[i] = A.regs[i];
  int st = 0, pc = 0;
  uint64_t steps = 0;
  while (pc < A.n) {
    if (++steps > A.max_steps) {
      st = -1;  // CGCM_E_INVALID
      break;
    }
    const GlueOp o = A.prog[pc];
    if (o.dst >= GLUE_REGS || o.a >= GLUE_REGS || o.b >= GLUE_REGS) {
      st = -1;
      break;
    }
    const uint64_t x = r[o.a], y = r[o.b];
    int next = pc + 1;
    switch (o.op) {
      case 1: r[o.dst] = (uint64_t)o.imm; break;
      case 2: r[o.dst] = x + y; break;
      case 3: r[o.dst] = x + (uint64_t)o.imm; break;
      case 4: r[o.dst] = x - y; break;
      case 5: r[o.dst] = x * y; break;
      case 6: r[o.dst] = __double_as_longlong(__dadd_rn(__longlong_as_double(x), __longlong_as_double(y))); break;
      case 7: r[o.dst] = __double_as_longlong(__dsub_rn(__longlong_as_double(x), __longlong_as_double(y))); break;
      case 8: r[o.dst] = __double_as_longlong(__dmul_rn(__longlong_as_double(x), __longlong_as_double(y))); break;
      case 9: r[o.dst] = __double_as_longlong(__ddiv_rn(__longlong_as_double(x), __longlong_as_double(y))); break;
      case 10:
      case 11: {
        const uint64_t g = x + (uint64_t)o.imm;
        if ((g & 7) || !glue_ok(A, g)) {
          st = -2;  // CGCM_E_UNREGISTERED
          break;
        }
        if (o.op == 10) r[o.dst] = *reinterpret_cast<volatile uint64_t *>(g);
        else *reinterpret_cast<volatile uint64_t *>(g) = y;
        break;
      }
      case 12:
        if (o.imm < 0 || o.imm >= A.n) {
          st = -1;
          break;
        }
        if (x != 0) next = (int)o.imm;
        break;
      case 13: next = A.n; break;
      default: st = -1; break;
    }
    if (st) break;
    pc = next;
  }
  for (int i = 0; i < GLUE_REGS; ++i) A.regs[i] = r[i];
  A.status[0] = st;
  A.status[1] = pc;
}
void launch_glue(const GlueArgs &g, cudaStream_t s) {
  (void)cudaGetLastError();
  k_glue<<<1, 1, 0, s>>>(g);
}

// up to two byte ranges (either side may be mapped pinned host memory); 16-byte words when aligned
__global__ void k_copy_small(unsigned char *dst, const unsigned char *src, size_t n, unsigned char *dst2,
                             const unsigned char *src2, size_t n2) {
  const size_t t = (size_t)blockIdx.x * blockDim.x + threadIdx.x, str = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < 2; ++r) {
    unsigned char *d = r ? dst2 : dst;
    const unsigned char *q = r ? src2 : src;
    const size_t m = r ? n2 : n;
    if (!m) continue;
    if ((((uintptr_t)d | (uintptr_t)q) & 15) == 0) {
      const size_t w = m / 16;
      for (size_t i = t; i < w; i += str) reinterpret_cast<uint4 *>(d)[i] = reinterpret_cast<const uint4 *>(q)[i];
      for (size_t i = 16 * w + t; i < m; i += str) d[i] = q[i];
    } else {
      for (size_t i = t; i < m; i += str) d[i] = q[i];
    }
  }
}
void launch_copy_small(void *dst, const void *src, size_t n, void *dst2, const void *src2, size_t n2, cudaStream_t s) {
  const size_t words = (std::max(n, n2) + 15) / 16;
  const int threads = 256;
  const int blocks = (int)std::min<size_t>((words + threads - 1) / threads, 64);
  k_copy_small<<<blocks > 0 ? blocks : 1, threads, 0, s>>>(static_cast<unsigned char *>(dst),
                                                            static_cast<const unsigned char *>(src), n,
                                                            static_cast<unsigned char *>(dst2),
                                                            static_cast<const unsigned char *>(src2), n2);
}

}  // namespace cgcm
