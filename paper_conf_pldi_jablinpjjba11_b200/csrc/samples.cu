// samples.cu -- test-only sample GPU functions that run BETWEEN map and
// unmap, the way the paper's auto-parallelized DOALL kernels do.  They are not part
// of the hot path; they exist so that copy-back (a4) has real GPU writes to carry.
//   S1 scale:   x *= alpha over a jagged 2-D array reached through translated row pointers
//               (config A; one correctly rounded multiply, bit-exact, A21)
//   S2 gemm:    C = alpha*A*B + beta*C on jagged n x n fp64 matrices, a block of rows per launch
//               (config B; DFMA, judged at 1e-12 relative)
//   S3 treesum: one bottom-up level of subtree sums through translated child pointers (config D;
//               fixed association, two adds per node, bit-exact)
#include <cuda_runtime.h>
#include <stdint.h>

// a module-scope __device__ variable, for symbol-bound globals (cgcm_declareGlobalSymbol, NEXT-4):
// GPU code names it directly, the way the paper's glue kernels reach globals
__device__ double cgcm_sample_global[512];

namespace {

__global__ void k_scale_global(double alpha) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < 512; i += gridDim.x * blockDim.x)
    cgcm_sample_global[i] = __dmul_rn(cgcm_sample_global[i], alpha);
}

__global__ void k_scale(const double *const *rows, uint64_t nrows, uint64_t ncols, double alpha) {
  uint64_t total = nrows * ncols;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    double *row = const_cast<double *>(rows[i / ncols]);
    uint64_t c = i % ncols;
    row[c] = __dmul_rn(row[c], alpha);
  }
}

__global__ void k_treesum_level(const uint64_t *child, uint64_t root, uint64_t nnodes, uint64_t lo, uint64_t hi) {
  uint64_t i = lo + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= hi || i >= nnodes) return;
  const double *node = reinterpret_cast<const double *>(i == 0 ? root : child[i - 1]);
  uint64_t l = child[2 * i], r = child[2 * i + 1];
  double s = node[1];
  if (l) s = __dadd_rn(s, reinterpret_cast<const double *>(l)[2]);
  if (r) s = __dadd_rn(s, reinterpret_cast<const double *>(r)[2]);
  const_cast<double *>(node)[2] = s;
}

// one thread per output element of the row block; k-loop with DFMA
__global__ void k_gemm_rows(const double *const *A, const double *const *B, double *const *Cm, int n, int row0,
                            int nrows, double alpha, double beta) {
  int j = blockIdx.x * blockDim.x + threadIdx.x;
  int i = row0 + blockIdx.y;
  if (j >= n || i >= row0 + nrows) return;
  const double *a = A[i];
  double acc = 0.0;
  for (int k = 0; k < n; ++k) acc = fma(a[k], B[k][j], acc);
  double *c = Cm[i];
  c[j] = alpha * acc + beta * c[j];
}

}  // namespace

extern "C" {

int cgcm_sample_scale(uint64_t rows_dev, uint64_t nrows, uint64_t ncols, double alpha, void *stream) {
  uint64_t total = nrows * ncols;
  if (!total) return 0;
  int grid = (int)((total + 255) / 256 < 4096 ? (total + 255) / 256 : 4096);
  k_scale<<<grid, 256, 0, (cudaStream_t)stream>>>(reinterpret_cast<const double *const *>(rows_dev), nrows, ncols,
                                                    alpha);
  return cudaGetLastError() == cudaSuccess ? 0 : -8;
}

int cgcm_sample_treesum_level(uint64_t child_dev, uint64_t root_dev, uint64_t nnodes, uint64_t lo, uint64_t hi,
                              void *stream) {
  if (hi <= lo) return 0;
  uint64_t cnt = hi - lo;
  k_treesum_level<<<(unsigned)((cnt + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      reinterpret_cast<const uint64_t *>(child_dev), root_dev, nnodes, lo, hi);
  return cudaGetLastError() == cudaSuccess ? 0 : -8;
}

int cgcm_sample_gemm_rows(uint64_t A_rows, uint64_t B_rows, uint64_t C_rows, int n, int row0, int nrows, double alpha,
                          double beta, void *stream) {
  dim3 grid((n + 127) / 128, nrows);
  k_gemm_rows<<<grid, 128, 0, (cudaStream_t)stream>>>(reinterpret_cast<const double *const *>(A_rows),
                                                       reinterpret_cast<const double *const *>(B_rows),
                                                       reinterpret_cast<double *const *>(C_rows), n, row0, nrows,
                                                       alpha, beta);
  return cudaGetLastError() == cudaSuccess ? 0 : -8;
}

// raw copies for tests that inspect or perturb device copies (e.g. the permutation test of a3)
int cgcm_test_d2h(void *dst, uint64_t src, uint64_t n) {
  return cudaMemcpy(dst, reinterpret_cast<const void *>(src), n, cudaMemcpyDeviceToHost) == cudaSuccess ? 0 : -8;
}
int cgcm_test_h2d(uint64_t dst, const void *src, uint64_t n) {
  return cudaMemcpy(reinterpret_cast<void *>(dst), src, n, cudaMemcpyHostToDevice) == cudaSuccess ? 0 : -8;
}

}  // extern "C"

extern "C" int cgcm_sample_global_addr(void **addr, size_t *bytes) {
  if (cudaGetSymbolAddress(addr, cgcm_sample_global) != cudaSuccess) return -8;
  return cudaGetSymbolSize(bytes, cgcm_sample_global) == cudaSuccess ? 0 : -8;
}
extern "C" int cgcm_sample_scale_global(double alpha, void *stream) {
  k_scale_global<<<2, 256, 0, (cudaStream_t)stream>>>(alpha);
  return cudaGetLastError() == cudaSuccess ? 0 : -8;
}
