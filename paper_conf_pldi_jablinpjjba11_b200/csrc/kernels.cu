// kernels.cu -- sm_100a kernels of the CGCM hot path.
//
//   k_slots<DIR, OPS>   the per-pointer kernel: interval lookup (a1, greatestLTE of P:L169-170 over
//                       a sorted u64 key array, shared-memory top level + 8-ary u32 sector levels),
//                       then any of: forward rewrite + refcount (a2, Alg. 1), reverse rewrite (a3),
//                       epoch gate (a4, Alg. 2), release (Alg. 3).  Pointer arrays are streamed with
//                       256-bit loads/stores (LDG/STG.E.ENL2.256) under an L2 evict-first policy so
//                       the table stays resident in L2.
//   k_build_*           table / index build (a0, off the per-pointer path).
//   small kernels       activation bookkeeping, rollback, outer-pointer lookup.
// DESIGN.md §7 gives the roofline of each kernel and its algorithmic bytes.
#include <cub/cub.cuh>

#include "cgcm_dev.h"

namespace cgcm {

namespace {

constexpr int SLOT_THREADS = 1024;
constexpr int SEG_SMEM = 512;

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

// 256-bit streaming load/store of four pointer slots (sm_100: LDG.E.ENL2.256 / STG.E.ENL2.256)
__device__ __forceinline__ void ld_stream4(const void *p, uint64_t pol, uint64_t v[4]) {
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ void st_stream4(void *p, uint64_t pol, const uint64_t v[4]) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u64 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p),
               "l"(v[0]), "l"(v[1]), "l"(v[2]), "l"(v[3]), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void st_stream1(void *p, uint64_t pol, uint64_t v) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(pol)
               : "memory");
}
// one 32-byte sector of the index / record arrays, kept in L2 (evict-last)
__device__ __forceinline__ void ld_sector(const void *p, uint64_t pol, uint64_t v[4]) {
  asm volatile("ld.global.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld_pair(const void *p, uint64_t pol, uint64_t &a, uint64_t &b) {
  asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(a), "=l"(b) : "l"(p), "l"(pol));
}
__device__ __forceinline__ void red_add(int32_t *p, int32_t v) {
  asm volatile("red.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// warp-aggregated append: returns this lane's slot in the list (valid only if pred)
__device__ __forceinline__ unsigned long long warp_append(unsigned long long *counter, bool pred) {
  unsigned active = __activemask();
  unsigned want = __ballot_sync(active, pred);
  unsigned long long base = 0;
  if (want) {
    int leader = __ffs(want) - 1;
    if ((threadIdx.x & 31) == leader) base = atomicAdd(counter, (unsigned long long)__popc(want));
    base = __shfl_sync(active, base, leader);
  }
  return base + __popc(want & lanemask_lt());
}

// per-warp reduction of a counter, one atomic per warp (all lanes are converged at kernel end)
__device__ __forceinline__ void flush_count(unsigned long long *dst, unsigned long long v) {
  unsigned active = __activemask();
  if (active == 0xffffffffu) {
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(active, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(dst, v);
  } else if (v) {
    atomicAdd(dst, v);
  }
}

// number of entries <= r among 8 sorted u32 and the largest such entry
__device__ __forceinline__ void count8(const uint64_t w[4], uint32_t r, int &c, uint32_t &last) {
  c = 0;
  last = 0;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint32_t lo = (uint32_t)w[q], hi = (uint32_t)(w[q] >> 32);
    if (lo <= r) { ++c; last = lo; }
    if (hi <= r) { ++c; last = hi; }
  }
}

}  // namespace

// -------------------------------------------------------------------------------------------------
// The slot kernel.  One thread handles one 32-byte-aligned chunk (4 slots) per grid-stride step;
// the 4 lookups are interleaved level by level so their sector loads are in flight together.
// -------------------------------------------------------------------------------------------------
template <int DIR, int OPS>
__global__ void __launch_bounds__(SLOT_THREADS, 1) k_slots(SlotArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ uint64_t s_seg0[SEG_SMEM + 1];
  uint64_t *s_top = reinterpret_cast<uint64_t *>(smem);
  uint32_t *s_wide = reinterpret_cast<uint32_t *>(smem + 8 * (size_t)a.smem_top);

  const int n = a.ix.meta[0], h = a.ix.meta[1], ntop = a.ix.meta[2];
  for (int t = threadIdx.x; t < ntop; t += blockDim.x) s_top[t] = a.ix.top[t];
  for (int t = threadIdx.x; t < (ntop + 31) / 32; t += blockDim.x) s_wide[t] = a.ix.wide[t];
  const int nseg_s = a.nseg <= SEG_SMEM ? a.nseg : 0;
  for (int t = threadIdx.x; t <= nseg_s; t += blockDim.x) s_seg0[t] = a.seg_chunk0[t];
  __syncthreads();

  const uint64_t pol_s = policy_evict_first();
  const uint64_t pol_t = policy_evict_last();
  const uint64_t top0 = ntop > 0 ? s_top[0] : ~0ull;
  const int sh = 3 * h;

  unsigned long long c_nulls = 0, c_hits = 0, c_miss = 0, c_pend = 0, c_notm = 0, c_under = 0, c_tr = 0;

  for (uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; c < a.nchunks;
       c += (uint64_t)gridDim.x * blockDim.x) {
    // ---- which segment / which slots ----
    int s;
    if (a.nseg == 1) {
      s = 0;
    } else {
      const uint64_t *sp = nseg_s ? s_seg0 : a.seg_chunk0;
      int lo = 0, len = a.nseg;  // last s with seg0[s] <= c
      while (len > 1) {
        int half = len >> 1;
        if (sp[lo + half] <= c) lo += half;
        len -= half;
      }
      s = lo;
    }
    const Seg sg = a.segs[s];
    const uint64_t c0 = nseg_s ? s_seg0[s] : a.seg_chunk0[s];
    const uint64_t a0 = (sg.ptr & ~31ull) + 32ull * (c - c0);
    const uint64_t lo_addr = sg.ptr, hi_addr = sg.ptr + 8ull * sg.n;
    uint32_t valid = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      uint64_t ad = a0 + 8ull * m;
      if (ad >= lo_addr && ad < hi_addr) valid |= 1u << m;
    }
    if (a.sel != SEL_ALL) {
      uint32_t hm = a.hitmask[c];
      valid &= (a.sel == SEL_HIT) ? hm : ~hm;
    }
    uint64_t v[4];
    ld_stream4(reinterpret_cast<const void *>(a0), pol_s, v);

    // ---- a1: interval lookup, 4 interleaved searches ----
    uint64_t p[4];
    int b[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      p[m] = ((valid >> m) & 1) ? v[m] : 0ull;
      b[m] = 0;
    }
    for (int len = ntop; len > 1;) {
      int half = len >> 1;
#pragma unroll
      for (int m = 0; m < 4; ++m)
        if (s_top[b[m] + half] <= p[m]) b[m] += half;
      len -= half;
    }
    uint64_t key[4];
    uint32_t rel[4], last[4];
    int j[4];
    bool wide[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      uint64_t tk = ntop > 0 ? s_top[b[m]] : 0ull;
      key[m] = tk;
      uint64_t d = p[m] - tk;
      rel[m] = d >= 0xFFFFFFFEull ? 0xFFFFFFFEu : (uint32_t)d;
      j[m] = b[m];
      last[m] = 0;
      wide[m] = ntop > 0 && ((s_wide[b[m] >> 5] >> (b[m] & 31)) & 1u);
    }
    for (int k = h - 1; k >= 0; --k) {
      const uint32_t *L = a.ix.lvl[k];
      uint64_t w[4][4];
#pragma unroll
      for (int m = 0; m < 4; ++m) ld_sector(L + 8 * (size_t)j[m], pol_t, w[m]);
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        int cc;
        uint32_t lst;
        count8(w[m], rel[m], cc, lst);
        j[m] = 8 * j[m] + cc - 1;
        last[m] = lst;
      }
    }
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      key[m] += last[m];
      if (wide[m]) {  // bucket spanning >= 4 GiB: binary search over the full u64 keys
        int lo = b[m] << sh, len = min(n, (b[m] + 1) << sh) - lo;
        while (len > 1) {
          int half = len >> 1;
          if (a.ix.keys[lo + half] <= p[m]) lo += half;
          len -= half;
        }
        j[m] = lo;
        key[m] = a.ix.keys[lo];
      }
    }

    // ---- record sectors ----
    uint64_t r[4][4];
    uint64_t cbase[4];
    int unit[4];
    bool hit[4], nul[4];
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      nul[m] = ((valid >> m) & 1) && v[m] == 0;
      bool look = ((valid >> m) & 1) && v[m] != 0 && p[m] >= top0;
      if (DIR == DIR_FWD) {
        unit[m] = look ? j[m] : 0;
        cbase[m] = key[m];
      } else {
        uint64_t bb = 0, uu = 0;
        if (look) ld_pair(a.rev + j[m], pol_t, bb, uu);
        cbase[m] = bb;
        unit[m] = (int)(uint32_t)uu;
      }
      if (look) ld_sector(a.rec + unit[m], pol_t, r[m]);
      else r[m][0] = r[m][1] = r[m][2] = r[m][3] = 0;
      hit[m] = look && (p[m] - key[m] <= r[m][0]);  // A7: p - base <= size
    }

    // ---- a2/a3/a4 operations ----
    uint64_t outv[4];
    uint32_t wrote = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) {
      const bool vm = (valid >> m) & 1;
      const bool hm = vm && hit[m];
      const bool miss = vm && !nul[m] && !hit[m];
      c_nulls += nul[m];
      c_hits += hm;
      c_miss += miss;
      outv[m] = v[m];
      UnitRec *R = a.rec + unit[m];
      const uint64_t off = p[m] - key[m];
      const uint64_t devbase = r[m][1], ep = r[m][2];
      const int32_t rc = (int32_t)(uint32_t)r[m][3];
      const uint32_t fl = (uint32_t)(r[m][3] >> 32);
      if (OPS & OP_CHECKMAPPED) c_notm += (hm && rc <= 0);
      bool act = false;
      if (OPS & OP_INC) {
        if (hm) {
          if (rc > 0) {
            red_add(&R->refcount, sg.inc);
          } else {
            int old = atomicAdd(&R->refcount, sg.inc);
            act = (old == 0);
          }
        }
      }
      if (OPS & OP_INCPLAIN)
        if (hm) red_add(&R->refcount, sg.inc);
      if (OPS & OP_DECPLAIN)
        if (hm) red_add(&R->refcount, -sg.inc);
      bool freed = false;
      if (OPS & OP_DEC) {
        if (hm) {
          int old = atomicAdd(&R->refcount, -sg.inc);
          c_under += (old < sg.inc);
          freed = (old == sg.inc);
        }
      }
      bool gated = false;
      uint64_t old_ep = 0;
      if (OPS & OP_GATE) {
        if (hm && ep != a.epoch) {
          old_ep = atomicExch(reinterpret_cast<unsigned long long *>(&R->epoch), (unsigned long long)a.epoch);
          gated = (old_ep != a.epoch);
        }
      }
      if (OPS & OP_WRITE) {
        if (hm) {
          if (DIR == DIR_FWD) {
            if (devbase != 0) {
              outv[m] = devbase + off;  // Alg. 1: info.devptr + (ptr - info.base)
              wrote |= 1u << m;
            } else {
              c_pend += 1;  // activated in this call: completed after the allocation
            }
          } else {
            outv[m] = cbase[m] + off;  // reverse: base + (g - devbase)
            wrote |= 1u << m;
          }
        }
      }
      // list appends in convergent code
      if (OPS & OP_INC) {
        unsigned long long ix = warp_append(&a.lc[0], act);
        if (act) a.act_list[ix] = (uint32_t)unit[m];
      }
      if (OPS & OP_DEC) {
        unsigned long long ix = warp_append(&a.lc[2], freed);
        if (freed) a.free_list[ix] = (uint32_t)unit[m];
      }
      if (OPS & OP_GATE) {
        unsigned long long ix = warp_append(&a.lc[1], gated);
        const bool cp = gated && !(fl & UF_READONLY);  // Alg. 2: stale and not read-only
        if (gated) {
          Journal jn;
          jn.old_epoch = old_ep;
          jn.unit = (uint32_t)unit[m];
          jn.copy = cp ? 1u : 0u;
          a.journal[ix] = jn;
        }
        unsigned long long cx = warp_append(&a.lc[3], cp);
        if (cp) a.copy_list[cx] = (uint32_t)unit[m];
      }
    }
    if (OPS & OP_WRITE) {
      c_tr += __popc(wrote);
      if (wrote) {
        if (sg.out == 0 && valid == 0xFu) {
          st_stream4(reinterpret_cast<void *>(a0), pol_s, outv);
        } else {
#pragma unroll
          for (int m = 0; m < 4; ++m)
            if ((wrote >> m) & 1) {
              uint64_t dst = sg.out ? sg.out + (a0 + 8ull * m - sg.ptr) : a0 + 8ull * m;
              st_stream1(reinterpret_cast<void *>(dst), pol_s, outv[m]);
            }
        }
      }
      if (sg.out != 0) {  // out-of-place: untranslated slots (NULL, lenient misses) copied verbatim
#pragma unroll
        for (int m = 0; m < 4; ++m)
          if (((valid >> m) & 1) && !((wrote >> m) & 1) && !(hit[m] && DIR == DIR_FWD)) {
            uint64_t dst = sg.out + (a0 + 8ull * m - sg.ptr);
            st_stream1(reinterpret_cast<void *>(dst), pol_s, v[m]);
          }
      }
    }
    if (OPS & OP_HITMASK) a.hitmask[c] = (uint8_t)wrote;
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

// the operation sets the runtime uses
#define CGCM_SLOT_OPS(X)                                                                          \
  X(DIR_FWD, OP_WRITE | OP_INC | OP_HITMASK)           /* map: forward rewrite + refcount (a2)   */ \
  X(DIR_FWD, OP_WRITE)                                 /* complete pending slots after alloc     */ \
  X(DIR_FWD, OP_DECPLAIN)                              /* rollback of pending increments         */ \
  X(DIR_FWD, OP_DEC)                                   /* release by CPU pointer (Alg. 3)        */ \
  X(DIR_FWD, OP_INCPLAIN)                              /* rollback of release                    */ \
  X(DIR_FWD, OP_GATE | OP_CHECKMAPPED)                 /* unmap by CPU pointer (Alg. 2, a4)      */ \
  X(DIR_FWD, OP_WRITE | OP_INCPLAIN)                   /* rollback of reverse+release            */ \
  X(DIR_FWD, OP_WRITE | OP_HITMASK)                    /* translate only (no refcount)           */ \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_HITMASK)          /* unmapArray: reverse (a3) + gate (a4)   */ \
  X(DIR_REV, OP_WRITE | OP_GATE | OP_DEC | OP_HITMASK) /* unmapArray + releaseArray fused        */ \
  X(DIR_REV, OP_GATE)                                  /* gate only (outer up to date)           */ \
  X(DIR_REV, OP_WRITE)                                 /* reverse only (copy-back of a unit)     */ \
  X(DIR_REV, OP_WRITE | OP_DECPLAIN)                   /* rollback of forward map (in place)     */ \
  X(DIR_REV, OP_INCPLAIN)                              /* re-map of an array-mapped outer (A9)   */ \
  X(DIR_REV, OP_DEC)                                   /* releaseArray of an array-mapped outer  */ \
  X(DIR_REV, OP_DECPLAIN)                              /* rollback of REV INCPLAIN               */

size_t slots_smem_bytes(int smem_top) { return 8 * (size_t)smem_top + 4 * (size_t)((smem_top + 31) / 32) + 16; }

template <int DIR, int OPS>
static int launch_one(const SlotArgs &a, int nsm, cudaStream_t s) {
  size_t smem = slots_smem_bytes(a.smem_top);
  static size_t configured = 0;
  if (smem > 48 * 1024 && smem > configured) {
    cudaError_t e = cudaFuncSetAttribute(k_slots<DIR, OPS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return -1;
    configured = smem;
  }
  uint64_t want = (a.nchunks + SLOT_THREADS - 1) / SLOT_THREADS;
  int grid = (int)(want < (uint64_t)nsm ? (want ? want : 1) : (uint64_t)nsm);
  (void)cudaGetLastError();
  k_slots<DIR, OPS><<<grid, SLOT_THREADS, smem, s>>>(a);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int launch_slots(int dir, int ops, const SlotArgs &a, int nsm, cudaStream_t s) {
#define X(D, O) \
  if (dir == D && ops == (O)) return launch_one<D, (O)>(a, nsm, s);
  CGCM_SLOT_OPS(X)
#undef X
  return -2;  // unsupported combination
}

// -------------------------------------------------------------------------------------------------
// Index build (a0): top splitters, wide bits, u32 sector levels.  n may live on the device.
// -------------------------------------------------------------------------------------------------
__device__ __forceinline__ void index_shape(int n, int &h, int &ntop) {
  h = 0;
  while (n > 0 && ((((int64_t)n + (1ll << (3 * h)) - 1) >> (3 * h)) > TOPMAX)) ++h;
  ntop = n > 0 ? (int)(((int64_t)n + (1ll << (3 * h)) - 1) >> (3 * h)) : 0;
}

__global__ void k_build_top(const uint64_t *keys, const int *n_dev, uint64_t *top, uint32_t *wide, int *meta) {
  int n = *n_dev, h, ntop;
  index_shape(n, h, ntop);
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t == 0) { meta[0] = n; meta[1] = h; meta[2] = ntop; }
  if (t >= ntop) return;
  int first = t << (3 * h);
  int lastu = min(n, (t + 1) << (3 * h)) - 1;
  top[t] = keys[first];
  if (keys[lastu] - keys[first] >= 0xFFFFFFFFull) atomicOr(&wide[t >> 5], 1u << (t & 31));
}

__global__ void k_build_level(const uint64_t *keys, const int *meta, const uint32_t *wide, int k, uint32_t *lvl,
                              size_t cap) {
  int n = meta[0], h = meta[1];
  if (k >= h) return;
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

void launch_build_index(const uint64_t *keys, const int *n_dev, int n_cap, uint64_t *top, uint32_t *wide,
                        uint32_t *const *lvl, const size_t *lvl_cap, int *meta, cudaStream_t s) {
  cudaMemsetAsync(wide, 0, 4 * ((TOPMAX + 31) / 32), s);
  (void)cudaGetLastError();
  k_build_top<<<(TOPMAX + 255) / 256, 256, 0, s>>>(keys, n_dev, top, wide, meta);
  for (int k = 0; k < MAXL; ++k) {
    if (!lvl[k] || lvl_cap[k] == 0) continue;
    int64_t cnt = ((int64_t)n_cap + (1ll << (3 * k)) - 1) >> (3 * k);
    int grid = (int)std::min<int64_t>((cnt + 255) / 256 + 1, 4096);
    (void)cudaGetLastError();
    k_build_level<<<grid, 256, 0, s>>>(keys, meta, wide, k, lvl[k], lvl_cap[k]);
  }
}

// new_rec[i] = old_rec[old_idx[i]] (surviving unit) or a fresh record (declared since the last build)
__global__ void k_remap(int n, const int32_t *old_idx, const uint64_t *size, const uint32_t *flags,
                        const uint64_t *epoch0, const UnitRec *old_rec, UnitRec *new_rec) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  UnitRec r;
  int o = old_idx[i];
  if (o >= 0) {
    r = old_rec[o];
  } else {
    r.size = size[i];
    r.devbase = 0;
    r.epoch = epoch0[i];
    r.refcount = 0;
    r.flags = flags[i];
  }
  new_rec[i] = r;
}
void launch_remap(int n, const int32_t *old_idx, const uint64_t *size, const uint32_t *flags, const uint64_t *epoch0,
                  const UnitRec *old_rec, UnitRec *new_rec, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_remap<<<(n + 255) / 256, 256, 0, s>>>(n, old_idx, size, flags, epoch0, old_rec, new_rec);
  }
}

// reverse index: key = devbase of active units (refcount > 0), inactive sorted to the end
__global__ void k_rev_collect(const UnitRec *rec, int n, uint64_t *keys, uint32_t *vals, int *count) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  bool act = rec[i].refcount > 0;
  keys[i] = act ? rec[i].devbase : ~0ull;
  vals[i] = (uint32_t)i;
  unsigned m = __ballot_sync(__activemask(), act);
  if (act && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(count, __popc(m));
}
void launch_rev_collect(const UnitRec *rec, int n, uint64_t *keys, uint32_t *vals, int *count, cudaStream_t s) {
  cudaMemsetAsync(count, 0, sizeof(int), s);
  if (n > 0) {
    (void)cudaGetLastError();
    k_rev_collect<<<(n + 255) / 256, 256, 0, s>>>(rec, n, keys, vals, count);
  }
}
__global__ void k_rev_payload(const uint32_t *units, const uint64_t *base, const int *n_dev, int n_cap, RevRec *rev) {
  int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n_cap || j >= *n_dev) return;
  RevRec r;
  r.unit = units[j];
  r.base = base[r.unit];
  r.pad = 0;
  rev[j] = r;
}
void launch_rev_payload(const uint32_t *units, const uint64_t *base, const int *n_dev, int n_cap, RevRec *rev,
                        cudaStream_t s) {
  if (n_cap > 0) {
    (void)cudaGetLastError();
    k_rev_payload<<<(n_cap + 255) / 256, 256, 0, s>>>(units, base, n_dev, n_cap, rev);
  }
}

size_t sort_pairs_temp_bytes(int n) {
  size_t bytes = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, bytes, (const uint64_t *)nullptr, (uint64_t *)nullptr,
                                  (const uint32_t *)nullptr, (uint32_t *)nullptr, n);
  return bytes;
}
void launch_sort_pairs(void *temp, size_t temp_bytes, const uint64_t *kin, uint64_t *kout, const uint32_t *vin,
                       uint32_t *vout, int n, cudaStream_t s) {
  cub::DeviceRadixSort::SortPairs(temp, temp_bytes, kin, kout, vin, vout, n, 0, 64, s);
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
// small bookkeeping kernels
// -------------------------------------------------------------------------------------------------
__global__ void k_unit_ops(const UnitOp *ops, int n, UnitRec *rec) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  UnitOp o = ops[i];
  UnitRec &r = rec[o.unit];
  switch (o.op) {
    case UOP_ADD_RC: atomicAdd(&r.refcount, (int32_t)(int64_t)o.val); break;
    case UOP_SET_EPOCH: r.epoch = o.val; break;
    case UOP_OR_FLAGS: atomicOr(&r.flags, (uint32_t)o.val); break;
    case UOP_AND_FLAGS: atomicAnd(&r.flags, (uint32_t)o.val); break;
    case UOP_SET_DEVBASE: r.devbase = o.val; break;
    case UOP_SET_RC: r.refcount = (int32_t)(int64_t)o.val; break;
  }
}
void launch_unit_ops(const UnitOp *ops, int n, UnitRec *rec, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_unit_ops<<<(n + 255) / 256, 256, 0, s>>>(ops, n, rec);
  }
}

__global__ void k_set_devbase(const uint32_t *units, const uint64_t *devbases, int n, UnitRec *rec, uint64_t epoch,
                              int set_epoch) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  UnitRec &r = rec[units[i]];
  r.devbase = devbases[i];
  r.flags |= UF_STORAGE;
  if (set_epoch) r.epoch = epoch;  // A5 reading R1: an AU is coherent when it becomes active
}
void launch_set_devbase(const uint32_t *units, const uint64_t *devbases, int n, UnitRec *rec, uint64_t epoch,
                        int set_epoch, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_set_devbase<<<(n + 255) / 256, 256, 0, s>>>(units, devbases, n, rec, epoch, set_epoch);
  }
}

__global__ void k_deactivate(const uint32_t *units, int n, UnitRec *rec) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  UnitRec &r = rec[units[i]];
  if (r.refcount != 0) return;  // re-activated in the meantime (cannot happen inside one call)
  if (r.flags & UF_GLOBAL) {
    r.flags &= ~UF_ARRAYMAPPED;  // named region persists
  } else {
    r.devbase = 0;               // cuMemFree (Alg. 3)
    r.flags &= ~(UF_ARRAYMAPPED | UF_STORAGE);
  }
}
void launch_deactivate(const uint32_t *units, int n, UnitRec *rec, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_deactivate<<<(n + 255) / 256, 256, 0, s>>>(units, n, rec);
  }
}

__global__ void k_restore_epochs(const Journal *j, int n, UnitRec *rec) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  rec[j[i].unit].epoch = j[i].old_epoch;
}
void launch_restore_epochs(const Journal *j, int n, UnitRec *rec, cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_restore_epochs<<<(n + 255) / 256, 256, 0, s>>>(j, n, rec);
  }
}

// outer-pointer lookup for mapArray/unmapArray/releaseArray: one thread per pointer, plain
// binary search over the full u64 key array (few pointers: latency, not bandwidth)
__global__ void k_lookup_points(IndexDev ix, const UnitRec *rec, const uint64_t *ptrs, int n, PointInfo *out) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint64_t p = ptrs[i];
  int nk = ix.meta[0];
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
    UnitRec u = rec[lo];
    if (p - ix.keys[lo] <= u.size) {
      r.unit = lo;
      r.base = ix.keys[lo];
      r.size = u.size;
      r.devbase = u.devbase;
      r.epoch = u.epoch;
      r.refcount = u.refcount;
      r.flags = u.flags;
    }
  }
  out[i] = r;
}
void launch_lookup_points(IndexDev ix, const UnitRec *rec, const uint64_t *ptrs, int n, PointInfo *out,
                          cudaStream_t s) {
  if (n > 0) {
    (void)cudaGetLastError();
    k_lookup_points<<<(n + 127) / 128, 128, 0, s>>>(ix, rec, ptrs, n, out);
  }
}

}  // namespace cgcm
