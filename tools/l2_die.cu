// l2_die.cu -- does the B200's L2 hold twice as much table when each die's SMs gather from only
// half of it?  tools/l2_capacity.cu found the knee of random 32-byte sector gathers issued from every
// SM at ~56 MiB (about one die's half of the 126 MiB L2: a line read by both dies' SMs is cached on
// both).  Here the SMs are split into two groups by a function of %smid; group 0 gathers from the
// lower half of the buffer, group 1 from the upper half.  If a split matches the dies, the knee
// moves out to ~110 MiB.  Standalone:
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/l2_die.cu -o build/l2_die
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
__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

// mode: 0 = no split; 1 = smid < nsm/2; 2.. = bit (mode-2) of smid; 100+ = table lookup in grp[]
__global__ void k_gather(const uint64_t *buf, uint64_t nsec, int iters, int mode, int nsm, const uint8_t *grp,
                         uint64_t *sink) {
  const uint64_t pol = pol_last();
  const uint32_t sm = smid();
  uint64_t base = 0, n = nsec;
  if (mode != 0) {
    uint32_t g;
    if (mode == 1)
      g = sm >= (uint32_t)(nsm / 2);
    else if (mode < 100)
      g = (sm >> (mode - 2)) & 1u;
    else
      g = grp[sm];
    n = nsec / 2;
    base = g ? n : 0;
  }
  uint64_t acc = 0, s = mix(blockIdx.x * 1315423911ull + threadIdx.x);
  for (int it = 0; it < iters; ++it) {
    uint64_t v[8][4];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      s = mix(s + q);
      ld32(buf + 4 * (base + s % n), pol, v[q]);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) acc ^= v[q][0] ^ v[q][3];
  }
  if (acc == 42) sink[0] = acc;
}

// per-SM latency probe: one warp on each SM chases a pointer ring in a 4 MiB buffer that is L2
// resident; the average dependent-load latency per SM tells near from far L2 halves when the ring
// lives in lines homed on one die.  Reported as a histogram-free list (sm, ns).
__global__ void k_chase(const uint64_t *ring, int steps, uint64_t *out) {
  if (threadIdx.x) return;
  uint64_t p = 0;
  long long t0 = clock64();
  for (int i = 0; i < steps; ++i) asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(p) : "l"(ring + p));
  long long t1 = clock64();
  out[2 * blockIdx.x] = smid();
  out[2 * blockIdx.x + 1] = (uint64_t)(t1 - t0) + (p == 0xFFFFFFFFFFFFull);
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
  const size_t maxbuf = 160ull << 20;
  uint64_t *buf, *sink;
  uint8_t *grp;
  CK(cudaMalloc(&buf, maxbuf));
  CK(cudaMalloc(&sink, 64));
  CK(cudaMalloc(&grp, 256));
  CK(cudaMemset(buf, 0x5a, maxbuf));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));

  // 1. latency per SM: small single-line ring (L2 resident) -- cycles per dependent load, per SM, for
  //    a few ring placements (each placement's lines hash to some L2 slices)
  {
    const int steps = 4096;
    uint64_t *ring, *out;
    CK(cudaMalloc(&ring, 1 << 20));
    CK(cudaMalloc(&out, 16 * 1024));
    static uint64_t h[32768];
    double best_spread = -1;
    uint8_t best_grp[256] = {0};
    for (int place = 0; place < 8; ++place) {
      // a one-line ring (self loop) at line `place`: every SM chases the same L2 line
      for (int i = 0; i < 32768; ++i) h[i] = 0;
      const int off = place * 16;  // 128-byte lines
      h[off] = off;
      CK(cudaMemcpy(ring, h, sizeof(h), cudaMemcpyHostToDevice));
      k_chase<<<nsm, 32>>>(ring, steps, out);
      k_chase<<<nsm, 32>>>(ring, steps, out);
      CK(cudaDeviceSynchronize());
      uint64_t o[2 * 256];
      CK(cudaMemcpy(o, out, 16 * nsm, cudaMemcpyDeviceToHost));
      double lat[256] = {0};
      for (int b = 0; b < nsm; ++b) lat[o[2 * b] & 255] = (double)o[2 * b + 1] / steps;
      printf("{\"test\": \"chase\", \"place\": %d, \"cycles_per_load_by_smid\": [", place);
      for (int s = 0; s < nsm; ++s) printf("%s%.0f", s ? "," : "", lat[s]);
      printf("]}\n");
      double lo = 1e30, hi = 0;
      for (int s = 0; s < nsm; ++s) lo = lat[s] < lo ? lat[s] : lo, hi = lat[s] > hi ? lat[s] : hi;
      if (hi - lo > best_spread) {
        best_spread = hi - lo;
        for (int s = 0; s < nsm; ++s) best_grp[s] = lat[s] > 0.5 * (lo + hi);
      }
    }
    int n1 = 0;
    printf("{\"test\": \"latency_group\", \"spread_cycles\": %.0f, \"group_by_smid\": [", best_spread);
    for (int s = 0; s < nsm; ++s) printf("%s%d", s ? "," : "", best_grp[s]), n1 += best_grp[s];
    printf("], \"group1_sms\": %d}\n", n1);
    CK(cudaMemcpy(grp, best_grp, 256, cudaMemcpyHostToDevice));
  }

  // 2. gather throughput with and without a split
  const int grid = nsm * 2, threads = 1024, iters = 128;
  const int modes[] = {0, 1, 2, 3, 4, 5, 100};
  const char *names[] = {"none", "smid_half", "smid_bit0", "smid_bit1", "smid_bit2", "smid_bit3", "latency_group"};
  for (size_t mb : {32, 48, 64, 80, 96, 112, 128}) {
    const uint64_t nsec = (mb << 20) / 32;
    for (int k = 0; k < 7; ++k) {
      k_gather<<<grid, threads>>>(buf, nsec, 16, modes[k], nsm, grp, sink);
      CK(cudaEventRecord(e0));
      k_gather<<<grid, threads>>>(buf, nsec, iters, modes[k], nsm, grp, sink);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      const double n = (double)grid * threads * iters * 8;
      printf("{\"test\": \"split_%s\", \"buffer_MiB\": %zu, \"G_sectors_per_s\": %.1f}\n", names[k], mb,
             n / time_ms(e0, e1) / 1e6);
    }
  }
  return 0;
}
