// cpu_baseline.cpp -- a TIMING-ONLY multi-core CPU baseline of the bench step (SURVEY §8(d) "Oracle
// timing beside the GPU": "translate-only over a sorted std::vector with std::upper_bound, OpenMP over
// all host cores").  Not the oracle (oracle/ is the correctness reference) and not the product: it is
// what a straightforward all-cores CPU implementation of the same step costs on the GPU box's host.
//
// One step over n pointer slots, against a table of U units sorted by base (devptr[u] = the unit's
// device address, mirrored layout):
//   forward (Alg. 1): u = greatestLTE(p) (std::upper_bound - 1), accept iff p - base <= size
//     (A7), slot = devptr[u] + (p - base[u]), refcount[u] += 1 (atomic)
//   reverse (Table 2 unmapArray + Alg. 2/3): v = the unit whose device copy holds g (upper_bound over the
//     devptr-sorted index), slot = base[v] + (g - devptr[v]), epoch gate (epoch[v] = current), refcount -= 1
// Built with g++ -O3 -fopenmp; loaded by bench.py through ctypes.
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdint>
#include <vector>

extern "C" {

int cpu_baseline_threads(void) { return omp_get_max_threads(); }

// returns the best step time in seconds over reps (slots are restored by each step's reverse pass);
// errors (a miss) return a negative value
double cpu_baseline_step(const uint64_t *base, const uint64_t *size, const uint64_t *devptr, int U, uint64_t *slots,
                         uint64_t n, int threads, int reps, uint64_t *translations_out) {
  if (threads > 0) omp_set_num_threads(threads);
  std::vector<std::atomic<int32_t>> rc(U);
  std::vector<std::atomic<uint32_t>> epoch(U);
  for (int u = 0; u < U; ++u) {
    rc[u].store(1, std::memory_order_relaxed);  // the setup reference the GPU run holds
    epoch[u].store(0, std::memory_order_relaxed);
  }
  // devptr-sorted index for the reverse lookups (built once, like the device reverse index)
  std::vector<uint64_t> dkey(U);
  std::vector<int32_t> dunit(U);
  {
    std::vector<int32_t> ord(U);
    for (int u = 0; u < U; ++u) ord[u] = u;
    std::sort(ord.begin(), ord.end(), [&](int a, int b) { return devptr[a] < devptr[b]; });
    for (int k = 0; k < U; ++k) {
      dkey[k] = devptr[ord[k]];
      dunit[k] = ord[k];
    }
  }
  double best = -1.0;
  uint64_t tr = 0;
  for (int r = 0; r < reps; ++r) {
    const uint32_t cur = (uint32_t)r + 1;
    std::atomic<uint64_t> miss{0}, done{0};
    auto t0 = std::chrono::steady_clock::now();
#pragma omp parallel
    {
      uint64_t m = 0, d = 0;
#pragma omp for schedule(static)
      for (int64_t i = 0; i < (int64_t)n; ++i) {
        const uint64_t p = slots[i];
        if (!p) continue;
        const uint64_t *it = std::upper_bound(base, base + U, p);
        if (it == base) { ++m; continue; }
        const int u = (int)(it - base) - 1;
        if (p - base[u] > size[u]) { ++m; continue; }
        slots[i] = devptr[u] + (p - base[u]);
        rc[u].fetch_add(1, std::memory_order_relaxed);
        ++d;
      }
#pragma omp for schedule(static)
      for (int64_t i = 0; i < (int64_t)n; ++i) {
        const uint64_t g = slots[i];
        if (!g) continue;
        auto it = std::upper_bound(dkey.begin(), dkey.end(), g);
        if (it == dkey.begin()) { ++m; continue; }
        const int v = dunit[(it - dkey.begin()) - 1];
        if (g - devptr[v] > size[v]) { ++m; continue; }
        slots[i] = base[v] + (g - devptr[v]);
        if (epoch[v].load(std::memory_order_relaxed) != cur) epoch[v].store(cur, std::memory_order_relaxed);
        rc[v].fetch_sub(1, std::memory_order_relaxed);
        ++d;
      }
      miss += m;
      done += d;
    }
    auto t1 = std::chrono::steady_clock::now();
    if (miss.load()) return -1.0;
    const double s = std::chrono::duration<double>(t1 - t0).count();
    best = best < 0 || s < best ? s : best;
    tr = done.load();
  }
  if (translations_out) *translations_out = tr;
  return best;
}

}  // extern "C"
