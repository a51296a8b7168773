// l2_gather.cu -- microbenchmarks of the access patterns the slot kernels are made of (SURVEY §8(d):
// "measure a random-32-B-gather microbenchmark over an L2-resident buffer ... if L2 caps below that,
// the cap (not HBM) is the true roof").  Standalone:  nvcc -O3 -gencode arch=compute_100a,code=sm_100a
// tools/l2_gather.cu -o build/l2_gather && build/l2_gather  -> one JSON line per measurement.
//
//   gather32   independent random 32-B loads (8 in flight per thread), evict-last: L2 gather rate
//   chain<D>   2 interleaved dependent chains of D random 32-B loads per thread, 768 threads/CTA, one CTA
//              per SM (the slot kernels' shape): per-chain latency-bound rate
//   red        random 4-B reductions (RED.ADD) over a 16-MiB array
//   skeleton   the forward slot kernel's memory skeleton: per 2 slots, a streamed 16-B load, D dependent
//              32-B gathers per slot, one 16-B record gather, one RED, a streamed 16-B store -- no
//              compute: the ceiling the real kernel is measured against
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x)                                                                            \
  do {                                                                                   \
    cudaError_t e_ = (x);                                                                \
    if (e_ != cudaSuccess) {                                                             \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_));         \
      exit(1);                                                                           \
    }                                                                                    \
  } while (0)

__device__ __forceinline__ uint64_t pol_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void ld32(const void *p, uint64_t pol, uint64_t v[4]) {
  asm volatile("ld.global.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 31;
  x *= 0x7fb5d329728ea185ull;
  x ^= x >> 27;
  x *= 0x81dadef4bc2dd44dull;
  return x ^ (x >> 33);
}

__global__ void k_gather32(const uint64_t *buf, uint64_t nsec, int iters, uint64_t *sink) {
  const uint64_t pol = pol_last();
  uint64_t acc = 0, s = mix(blockIdx.x * 1315423911ull + threadIdx.x);
  for (int it = 0; it < iters; ++it) {
    uint64_t v[8][4];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      s = mix(s + q);
      ld32(buf + 4 * (s % nsec), pol, v[q]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) acc ^= v[q][0] ^ v[q][3];
  }
  if (acc == 42) sink[0] = acc;
}

template <int D>
__global__ void __launch_bounds__(768, 1) k_chain(const uint64_t *buf, uint64_t nsec, int iters, uint64_t *sink) {
  const uint64_t pol = pol_last();
  uint64_t a = mix(blockIdx.x * 77ull + threadIdx.x), b = mix(a + 1), acc = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int d = 0; d < D; ++d) {
      uint64_t va[4], vb[4];
      ld32(buf + 4 * (a % nsec), pol, va);
      ld32(buf + 4 * (b % nsec), pol, vb);
      a = mix(va[1] + a);
      b = mix(vb[1] + b);
    }
    acc += a ^ b;
  }
  if (acc == 42) sink[0] = acc;
}

__global__ void k_red(int32_t *rc, uint32_t n, int iters) {
  uint64_t s = mix(blockIdx.x * 99991ull + threadIdx.x);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      s = mix(s + q);
      asm volatile("red.global.add.s32 [%0], %1;" ::"l"(rc + (s % n)), "r"(1) : "memory");
    }
  }
}

// forward-map memory skeleton: slots streamed in place, D dependent level gathers, record, RED
template <int D>
__global__ void __launch_bounds__(768, 1)
    k_skeleton(uint64_t *slots, uint64_t nchunks, const uint64_t *lv, uint64_t nsec, const uint64_t *rec,
               uint64_t nrec, int32_t *rc) {
  const uint64_t pl = pol_last(), pf = pol_first();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += stride) {
    uint64_t x0, x1;
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                 : "=l"(x0), "=l"(x1)
                 : "l"(slots + 2 * c), "l"(pf));
    uint64_t a = mix(x0 + 2 * c), b = mix(x1 + 2 * c + 1);  // distinct random units per slot
#pragma unroll
    for (int d = 0; d < D; ++d) {
      uint64_t va[4], vb[4];
      ld32(lv + 4 * (a % nsec), pl, va);
      ld32(lv + 4 * (b % nsec), pl, vb);
      a = mix(a ^ va[0]);
      b = mix(b ^ vb[0]);
    }
    uint64_t ra0, ra1, rb0, rb1;
    const uint64_t ia = a % nrec, ib = b % nrec;
    asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(ra0), "=l"(ra1) : "l"(rec + 2 * ia), "l"(pl));
    asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(rb0), "=l"(rb1) : "l"(rec + 2 * ib), "l"(pl));
    asm volatile("red.global.add.s32 [%0], %1;" ::"l"(rc + ia), "r"(1) : "memory");  // own refcount array
    asm volatile("red.global.add.s32 [%0], %1;" ::"l"(rc + ib), "r"(1) : "memory");
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(slots + 2 * c),
                 "l"(x0 + ra0), "l"(x1 + rb0), "l"(pf)
                 : "memory");
  }
}

// reverse-unmap memory skeleton (shadow variant): slots and their shadow (u64 CPU pointer[n], u32 unit[n])
// streamed, one 16-B record gather per slot at the shadow's unit, one RED, slots stored
// NOALLOC: record gathers bypass L1 allocation; SEP: refcounts in their own array (not the record's line)
template <bool RED, bool GATHER, bool SHADOW, bool NOALLOC = false, bool SEP = false, bool SCALAR = false>
__global__ void __launch_bounds__(768, 1)
    k_skeleton_rev(uint64_t *slots, uint64_t nchunks, const uint64_t *shp, const uint32_t *shu, const uint64_t *rec,
                   uint64_t nrec, int32_t *rc) {
  const uint64_t pl = pol_last(), pf = pol_first();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += stride) {
    uint64_t x0, x1, h0, h1;
    uint32_t u0, u1;
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                 : "=l"(x0), "=l"(x1)
                 : "l"(slots + 2 * c), "l"(pf));
    if (SHADOW && SCALAR) {  // the slot kernel's shape: 4 scalar shadow loads per thread
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(h0) : "l"(shp + 2 * c), "l"(pf));
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(h1) : "l"(shp + 2 * c + 1), "l"(pf));
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(u0) : "l"(shu + 2 * c), "l"(pf));
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(u1) : "l"(shu + 2 * c + 1), "l"(pf));
    } else if (SHADOW) {
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                   : "=l"(h0), "=l"(h1)
                   : "l"(shp + 2 * c), "l"(pf));
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;"
                   : "=r"(u0), "=r"(u1)
                   : "l"(shu + 2 * c), "l"(pf));
    } else {
      h0 = x0 >> 3;
      h1 = x1 >> 3;
      u0 = (uint32_t)mix(x0 + 2 * c);
      u1 = (uint32_t)mix(x1 + 2 * c + 1);
    }
    const uint64_t ia = u0 % nrec, ib = u1 % nrec;
    uint64_t ra0 = 0, ra1 = 0, rb0 = 0, rb1 = 0;
    if (GATHER && !NOALLOC) {
      asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(ra0), "=l"(ra1) : "l"(rec + 2 * ia), "l"(pl));
      asm volatile("ld.global.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(rb0), "=l"(rb1) : "l"(rec + 2 * ib), "l"(pl));
    }
    if (GATHER && NOALLOC) {
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(ra0), "=l"(ra1) : "l"(rec + 2 * ia), "l"(pl));
      asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;" : "=l"(rb0), "=l"(rb1) : "l"(rec + 2 * ib), "l"(pl));
    }
    int32_t *R = SEP ? rc + (16u << 20) : rc;  // SEP: a separate i32 array after the records
    const uint64_t oa = SEP ? ia : 4 * ia + 2, ob = SEP ? ib : 4 * ib + 2;
    if (RED) {
      asm volatile("red.global.add.s32 [%0], %1;" ::"l"(R + oa), "r"(-1) : "memory");
      asm volatile("red.global.add.s32 [%0], %1;" ::"l"(R + ob), "r"(-1) : "memory");
    }
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(slots + 2 * c),
                 "l"(x0 == h0 + ra0 ? h0 : x0), "l"(x1 == h1 + rb0 ? h1 : x1), "l"(pf)
                 : "memory");
  }
}

// page-directory forward skeleton (k_map_pd's memory shape): a streamed 16-B load per 2 slots; per slot
// ENT: a 32-B entry gather (dependent on the slot value), HOT: a dependent 8-B unit-word gather, RED: one
// reduction into a separate refcount array, SH: a 12-B shadow store; the 16-B slot store.  No compute.
template <bool ENT, bool HOT, bool RED, bool SH, bool W64 = false>
__global__ void __launch_bounds__(768, 1)
    k_skel_pd(uint64_t *slots, uint64_t nchunks, const uint64_t *ent, uint64_t nent, const uint64_t *hot,
              uint64_t nunit, int32_t *rc, uint64_t *shp, uint32_t *shu) {
  const uint64_t pl = pol_last(), pf = pol_first();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += stride) {
    uint64_t x0, x1;
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                 : "=l"(x0), "=l"(x1)
                 : "l"(slots + 2 * c), "l"(pf));
    uint64_t a = mix(x0 + 2 * c), b = mix(x1 + 2 * c + 1);
    if (ENT && !W64) {
      uint64_t va[4], vb[4];
      ld32(ent + 4 * (a % nent), pl, va);
      ld32(ent + 4 * (b % nent), pl, vb);
      a = mix(a ^ va[0]);
      b = mix(b ^ vb[0]);
    }
    if (ENT && W64) {  // 64-byte entries: two 32-byte loads of one 64-byte block
      uint64_t va[4], vb[4], wa[4], wb[4];
      const uint64_t ea = 8 * (a % (nent / 2)), eb = 8 * (b % (nent / 2));
      ld32(ent + ea, pl, va);
      ld32(ent + ea + 4, pl, wa);
      ld32(ent + eb, pl, vb);
      ld32(ent + eb + 4, pl, wb);
      a = mix(a ^ va[0] ^ wa[3]);
      b = mix(b ^ vb[0] ^ wb[3]);
    }
    const uint64_t ia = a % nunit, ib = b % nunit;
    uint64_t ha = 0, hb = 0;
    if (HOT) {
      asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(ha) : "l"(hot + ia), "l"(pl));
      asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(hb) : "l"(hot + ib), "l"(pl));
    }
    if (RED) {
      asm volatile("red.global.add.s32 [%0], %1;" ::"l"(rc + ia), "r"(1) : "memory");
      asm volatile("red.global.add.s32 [%0], %1;" ::"l"(rc + ib), "r"(1) : "memory");
    }
    if (SH) {
      asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(shp + 2 * c), "l"(x0),
                   "l"(x1), "l"(pf)
                   : "memory");
      asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u32 [%0], {%1,%2}, %3;" ::"l"(shu + 2 * c),
                   "r"((uint32_t)ia), "r"((uint32_t)ib), "l"(pf)
                   : "memory");
    }
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(slots + 2 * c),
                 "l"(x0 + ha), "l"(x1 + hb), "l"(pf)
                 : "memory");
  }
}

// forward with ONE returning 64-bit atomic per slot on {rc | unit word} instead of unit-word gather + RED
__global__ void __launch_bounds__(768, 1)
    k_skel_atom(uint64_t *slots, uint64_t nchunks, const uint64_t *ent, uint64_t nent, unsigned long long *rch,
                uint64_t nunit, uint64_t *shp, uint32_t *shu) {
  const uint64_t pl = pol_last(), pf = pol_first();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += stride) {
    uint64_t x0, x1;
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                 : "=l"(x0), "=l"(x1)
                 : "l"(slots + 2 * c), "l"(pf));
    uint64_t a = mix(x0 + 2 * c), b = mix(x1 + 2 * c + 1);
    uint64_t va[4], vb[4];
    ld32(ent + 4 * (a % nent), pl, va);
    ld32(ent + 4 * (b % nent), pl, vb);
    a = mix(a ^ va[0]);
    b = mix(b ^ vb[0]);
    const uint64_t ia = a % nunit, ib = b % nunit;
    const unsigned long long ha = atomicAdd(rch + ia, 1ull), hb = atomicAdd(rch + ib, 1ull);
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(shp + 2 * c), "l"(x0),
                 "l"(x1), "l"(pf)
                 : "memory");
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u32 [%0], {%1,%2}, %3;" ::"l"(shu + 2 * c),
                 "r"((uint32_t)ia), "r"((uint32_t)ib), "l"(pf)
                 : "memory");
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(slots + 2 * c),
                 "l"(x0 + (ha >> 32)), "l"(x1 + (hb >> 32)), "l"(pf)
                 : "memory");
  }
}
__global__ void k_fill_units(uint32_t *u, uint64_t n, uint32_t nrec) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    u[i] = (uint32_t)(mix(i) % nrec);
}

static float time_ms(cudaEvent_t e0, cudaEvent_t e1) {
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, e0, e1));
  return ms;
}

int main(int argc, char **argv) {
  int nsm = 0, dev = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  int l2 = 0;
  CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
  printf("{\"device_sms\": %d, \"l2_bytes\": %d}\n", nsm, l2);
  const size_t sizes[] = {16ull << 20, 48ull << 20, 96ull << 20, 1ull << 30};
  uint64_t *buf, *sink;
  CK(cudaMalloc(&buf, 1ull << 30));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(buf, 0x5a, 1ull << 30));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  for (size_t S : sizes) {
    const uint64_t nsec = S / 32;
    // gather32
    {
      int grid = nsm * 2, threads = 1024, iters = 256;
      k_gather32<<<grid, threads>>>(buf, nsec, 8, sink);
      CK(cudaEventRecord(e0));
      k_gather32<<<grid, threads>>>(buf, nsec, iters, sink);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      double n = (double)grid * threads * iters * 8;
      printf("{\"test\": \"gather32\", \"buffer_MiB\": %zu, \"G_per_s\": %.1f, \"GB_per_s\": %.0f}\n", S >> 20,
             n / time_ms(e0, e1) / 1e6, 32 * n / time_ms(e0, e1) / 1e6);
    }
    // dependent chains, the slot kernel's shape
    {
      int grid = nsm, threads = 768, iters = 64;
      k_chain<4><<<grid, threads>>>(buf, nsec, 4, sink);
      CK(cudaEventRecord(e0));
      k_chain<4><<<grid, threads>>>(buf, nsec, iters, sink);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      double n = (double)grid * threads * iters * 4 * 2;
      double ms = time_ms(e0, e1);
      double lat = ms * 1e-3 / ((double)iters * 4) * 1.965e9;  // cycles per dependent step at max clock
      printf("{\"test\": \"chain4x2\", \"buffer_MiB\": %zu, \"G_loads_per_s\": %.1f, \"cycles_per_step\": %.0f}\n",
             S >> 20, n / ms / 1e6, lat);
    }
  }
  // reductions
  {
    int32_t *rc;
    const uint32_t n = 4u << 20;
    CK(cudaMalloc(&rc, 4ull * n));
    CK(cudaMemset(rc, 0, 4ull * n));
    int grid = nsm * 2, threads = 1024, iters = 256;
    k_red<<<grid, threads>>>(rc, n, 8);
    CK(cudaEventRecord(e0));
    k_red<<<grid, threads>>>(rc, n, iters);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    double cnt = (double)grid * threads * iters * 8;
    printf("{\"test\": \"red_s32\", \"array_MiB\": 16, \"G_per_s\": %.1f}\n", cnt / time_ms(e0, e1) / 1e6);
    CK(cudaFree(rc));
  }
  // skeleton of the forward slot kernel at config E: 2^28 slots, levels over 16 MiB + 2 MiB + 256 KiB
  // (modelled as D gathers over an 18-MiB buffer), 2^22 16-B records, refcounts inside the records
  {
    const uint64_t nslots = 1ull << 28;
    uint64_t *slots, *lv, *rec;
    CK(cudaMalloc(&slots, 8 * nslots));
    CK(cudaMalloc(&lv, 18ull << 20));
    CK(cudaMalloc(&rec, (16ull << 22) + (4ull << 22)));  // records + a separate refcount array
    CK(cudaMemset(slots, 0x33, 8 * nslots));
    CK(cudaMemset(lv, 0x11, 18ull << 20));
    CK(cudaMemset(rec, 0, (16ull << 22) + (4ull << 22)));
    for (int D = 2; D <= 3; ++D) {
      auto run = [&]() {
        if (D == 2)
          k_skeleton<2><<<nsm, 768>>>(slots, nslots / 2, lv, (18ull << 20) / 32, rec, 1ull << 22,
                                      reinterpret_cast<int32_t *>(rec) + (16u << 20));
        else
          k_skeleton<3><<<nsm, 768>>>(slots, nslots / 2, lv, (18ull << 20) / 32, rec, 1ull << 22,
                                      reinterpret_cast<int32_t *>(rec) + (16u << 20));
      };
      run();
      CK(cudaEventRecord(e0));
      for (int r = 0; r < 5; ++r) run();
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      double ms = time_ms(e0, e1) / 5;
      printf("{\"test\": \"skeleton_fwd\", \"levels\": %d, \"slots\": %llu, \"ms\": %.3f, \"G_slots_per_s\": %.1f}\n", D,
             (unsigned long long)nslots, ms, nslots / ms / 1e6);
    }
    // reverse skeleton: shadow = 8 B CPU pointer + 4 B unit per slot
    uint64_t *shp;
    uint32_t *shu;
    CK(cudaMalloc(&shp, 8 * nslots));
    CK(cudaMalloc(&shu, 4 * nslots));
    CK(cudaMemset(shp, 0x21, 8 * nslots));
    k_fill_units<<<nsm * 4, 1024>>>(shu, nslots, 1u << 22);
    auto rev = [&](auto kern, const char *what) {
      kern<<<nsm, 768>>>(slots, nslots / 2, shp, shu, rec, 1ull << 22, reinterpret_cast<int32_t *>(rec));
      CK(cudaEventRecord(e0));
      for (int r = 0; r < 5; ++r)
        kern<<<nsm, 768>>>(slots, nslots / 2, shp, shu, rec, 1ull << 22, reinterpret_cast<int32_t *>(rec));
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      double ms = time_ms(e0, e1) / 5;
      printf("{\"test\": \"skeleton_rev\", \"parts\": \"%s\", \"slots\": %llu, \"ms\": %.3f, \"G_slots_per_s\": %.1f}\n",
             what, (unsigned long long)nslots, ms, nslots / ms / 1e6);
    };
    rev(k_skeleton_rev<true, true, true>, "shadow+gather+red");
    rev(k_skeleton_rev<false, true, true>, "shadow+gather");
    rev(k_skeleton_rev<true, false, true>, "shadow+red");
    rev(k_skeleton_rev<false, false, true>, "shadow (streams only)");
    rev(k_skeleton_rev<true, true, false>, "gather+red (no shadow)");
    rev(k_skeleton_rev<false, false, false>, "slots only");
    rev(k_skeleton_rev<true, true, true, true, false>, "shadow+gather(L1 no_allocate)+red");
    rev(k_skeleton_rev<true, true, true, false, true>, "shadow+gather+red(separate array)");
    rev(k_skeleton_rev<true, true, true, true, true>, "shadow+gather(no_allocate)+red(separate)");
    rev(k_skeleton_rev<true, true, true, false, true, true>, "scalar shadow+gather+red(separate)");
    // page-directory forward skeletons: config E (39 MiB entries, 2^22 units) and C (10 MiB, 2^20)
    for (int cfg = 0; cfg < 2; ++cfg) {
      const uint64_t nent = cfg == 0 ? (39ull << 20) / 32 : (10ull << 20) / 32, nunit = cfg == 0 ? 1ull << 22 : 1ull << 20;
      uint64_t *ent, *hot;
      int32_t *rcs;
      CK(cudaMalloc(&ent, 32 * nent));
      CK(cudaMalloc(&hot, 8 * nunit));
      CK(cudaMalloc(&rcs, 4 * nunit));
      CK(cudaMemset(ent, 0x11, 32 * nent));
      CK(cudaMemset(hot, 0, 8 * nunit));
      CK(cudaMemset(rcs, 0, 4 * nunit));
      auto pd = [&](auto kern, const char *what) {
        kern<<<nsm, 768>>>(slots, nslots / 2, ent, nent, hot, nunit, rcs, shp, shu);
        CK(cudaEventRecord(e0));
        for (int r = 0; r < 5; ++r) kern<<<nsm, 768>>>(slots, nslots / 2, ent, nent, hot, nunit, rcs, shp, shu);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        double ms = time_ms(e0, e1) / 5;
        printf("{\"test\": \"skeleton_pd\", \"cfg\": \"%s\", \"parts\": \"%s\", \"slots\": %llu, \"ms\": %.3f, \"G_slots_per_s\": %.1f}\n",
               cfg == 0 ? "E" : "C", what, (unsigned long long)nslots, ms, nslots / ms / 1e6);
      };
      pd(k_skel_pd<true, true, true, true>, "ent+hot+red+shadow");
      {
        unsigned long long *rch;
        CK(cudaMalloc(&rch, 8 * nunit));
        CK(cudaMemset(rch, 0, 8 * nunit));
        k_skel_atom<<<nsm, 768>>>(slots, nslots / 2, ent, nent, rch, nunit, shp, shu);
        CK(cudaEventRecord(e0));
        for (int r = 0; r < 5; ++r) k_skel_atom<<<nsm, 768>>>(slots, nslots / 2, ent, nent, rch, nunit, shp, shu);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        double ms = time_ms(e0, e1) / 5;
        printf("{\"test\": \"skeleton_pd\", \"cfg\": \"%s\", \"parts\": \"ent+atom64(rc|unit)+shadow\", \"ms\": %.3f}\n",
               cfg == 0 ? "E" : "C", ms);
        CK(cudaFree(rch));
      }
      pd(k_skel_pd<true, false, true, true, true>, "ent64+red+shadow");
      pd(k_skel_pd<true, false, true, false, true>, "ent64+red");
      pd(k_skel_pd<true, false, true, true>, "ent+red+shadow");
      pd(k_skel_pd<true, true, true, false>, "ent+hot+red");
      pd(k_skel_pd<true, true, false, false>, "ent+hot");
      pd(k_skel_pd<true, false, true, false>, "ent+red");
      pd(k_skel_pd<false, true, true, false>, "hot+red");
      pd(k_skel_pd<true, false, false, false>, "ent");
      pd(k_skel_pd<false, false, true, false>, "red");
      pd(k_skel_pd<false, false, false, true>, "streams+shadow");
      pd(k_skel_pd<false, false, false, false>, "streams");
      CK(cudaFree(ent));
      CK(cudaFree(hot));
      CK(cudaFree(rcs));
    }
    CK(cudaGetLastError());
  }
  return 0;
}
