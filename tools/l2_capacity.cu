// l2_capacity.cu -- effective L2 capacity for random 32-byte sector gathers issued from every SM (the
// table accesses of the slot kernels), with and without a concurrent evict-first pointer stream
// (the slot arrays).  For working sets from 8 MiB to 192 MiB: gather rate (G sectors/s); the knee is
// the capacity the table columns must fit in.  Standalone:
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/l2_capacity.cu -o build/l2_capacity
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e_ = (x);                                                        \
    if (e_ != cudaSuccess) {                                                     \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      exit(1);                                                                   \
    }                                                                            \
  } while (0)

__device__ __forceinline__ uint64_t pol_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
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

// STREAM: per 8 gathers, also read and write 64 B of a large evict-first stream
template <int STREAM, int POL>
__global__ void k_gather(const uint64_t *buf, uint64_t nsec, int iters, uint64_t *stream, uint64_t nstream,
                         uint64_t *sink) {
  const uint64_t pol = POL == 0 ? pol_last() : pol_normal();
  const uint64_t pf = pol_first();
  uint64_t acc = 0, s = mix(blockIdx.x * 1315423911ull + threadIdx.x);
  uint64_t sp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 2;
  const uint64_t sstride = (uint64_t)gridDim.x * blockDim.x * 2;
  for (int it = 0; it < iters; ++it) {
    uint64_t v[8][4];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      s = mix(s + q);
      ld32(buf + 4 * (s % nsec), pol, v[q]);
    }
    if (STREAM) {
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        uint64_t a, b;
        const uint64_t *p = stream + (sp % nstream);
        asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v2.u64 {%0,%1}, [%2], %3;"
                     : "=l"(a), "=l"(b)
                     : "l"(p), "l"(pf));
        asm volatile("st.global.L1::no_allocate.L2::cache_hint.v2.u64 [%0], {%1,%2}, %3;" ::"l"(p), "l"(a + 1),
                     "l"(b), "l"(pf)
                     : "memory");
        sp += sstride;
      }
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) acc ^= v[q][0] ^ v[q][3];
  }
  if (acc == 42) sink[0] = acc;
}

static float time_ms(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0;
  CK(cudaEventElapsedTime(&ms, a, b));
  return ms;
}

int main() {
  int nsm = 0, l2 = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, 0));
  printf("{\"device_sms\": %d, \"l2_bytes\": %d}\n", nsm, l2);
  const size_t maxbuf = 192ull << 20, nstream = (2ull << 30) / 8;
  uint64_t *buf, *stream, *sink;
  CK(cudaMalloc(&buf, maxbuf));
  CK(cudaMalloc(&stream, nstream * 8));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMemset(buf, 0x5a, maxbuf));
  CK(cudaMemset(stream, 0x11, nstream * 8));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int grid = nsm * 2, threads = 1024, iters = 128;
  for (size_t mb = 8; mb <= 192; mb += 8) {
    const uint64_t nsec = (mb << 20) / 32;
    auto run = [&](auto kern, const char *what) {
      kern<<<grid, threads>>>(buf, nsec, 16, stream, nstream, sink);
      CK(cudaEventRecord(e0));
      kern<<<grid, threads>>>(buf, nsec, iters, stream, nstream, sink);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      const double n = (double)grid * threads * iters * 8;
      printf("{\"test\": \"%s\", \"buffer_MiB\": %zu, \"G_sectors_per_s\": %.1f}\n", what, mb,
             n / time_ms(e0, e1) / 1e6);
    };
    run(k_gather<0, 0>, "gather_evict_last");
    run(k_gather<0, 1>, "gather_evict_normal");
    run(k_gather<1, 0>, "gather_evict_last+stream");
  }
  return 0;
}
