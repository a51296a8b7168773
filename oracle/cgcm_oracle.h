/*
 * cgcm_oracle.h -- the CPU ORACLE for the CGCM run-time library (TEST INFRASTRUCTURE ONLY).
 *
 * This header and oracle/cgcm_oracle.cpp are a plain, slow, sequential C++17 statement of what the
 * run-time library of Jablin et al., "Automatic CPU-GPU Communication Management and Optimization"
 * (PLDI 2011) computes.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  The product (paper_conf_pldi_jablinpjjba11_b200/, include/cgcm.h)
 * never includes, links or calls anything in oracle/, and this file includes nothing from the product.
 *
 * Citations "P:Lnnn" are line numbers of the decoded `fulltext` of /root/reference/PAPER.md
 * (SURVEY.md §0 gives the one-liner).  The readings A1..A23 are listed in DESIGN.md §3.
 *
 * Memory model.  The oracle never dereferences the addresses it is given.  It keeps
 *   - a simulated HOST image (sparse, zero-filled pages) addressed by the caller's real CPU addresses;
 *     tests copy the initial bytes in with ref_hostWrite and read results with ref_hostRead;
 *   - a simulated DEVICE image (sparse) addressed by simulated device pointers.  Device pointers come
 *     from a bump allocator (devptr == base mod 256, >= 16 B guard + 1 B slack between copies) or, in
 *     replay mode, from ref_replayDevptr (the GPU path's own devbase for that unit).
 *
 * All entry points return 0 (REF_OK) or a negative status with the same numeric meaning as the
 * product ABI (DESIGN.md §4 lists the contract).  Every call is all-or-nothing: on error, no unit,
 * memory byte, epoch or counter changes (implemented with an undo journal, cgcm_oracle.cpp).
 */
#ifndef CGCM_ORACLE_H
#define CGCM_ORACLE_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum {
  REF_OK = 0,
  REF_E_INVALID = -1,
  REF_E_UNREGISTERED = -2,
  REF_E_OVERLAP = -3,
  REF_E_NOT_MAPPED = -4,
  REF_E_BUSY = -5,
  REF_E_DUPLICATE = -6,
  REF_E_NOMEM = -7,
};

/* context flags */
enum { REF_LITERAL_EPOCH = 1u, /* A5 literal: map never touches epoch */
       REF_LENIENT = 2u };     /* A18 lenient: uncovered non-null slots pass through */

/* unit flags (declare + dump) */
enum { REF_UNIT_GLOBAL = 1u, REF_UNIT_READONLY = 2u, REF_UNIT_ARRAYMAPPED = 4u, REF_UNIT_ACTIVE = 8u };

typedef struct {
  uint64_t base, size, devptr;
  int64_t refCount;
  uint64_t epoch;
  uint32_t flags;
  uint32_t pad;
} ref_unit_t;

typedef struct {
  uint64_t h2d_units, h2d_bytes, d2h_units, d2h_bytes;
  uint64_t activations, frees;
  uint64_t fwd_translations, rev_translations, null_slots, passthrough;
  uint64_t peer_units, peer_bytes;  /* NEXT-3: activations copied from a group peer's device copy */
} ref_stats_t;

void *ref_create(unsigned flags);
/* NEXT-3 coherence group: h joins the group of `leader` (which may be h itself: a group of one); the
 * members share one host memory (the leader's) and each keeps its own device, table and epochs. */
int ref_groupJoin(void *h, void *leader);
void ref_destroy(void *h);

int ref_declareAlloc(void *h, uint64_t base, uint64_t size);
int ref_declareAllocFlags(void *h, uint64_t base, uint64_t size, unsigned unit_flags);
int ref_declareGlobal(void *h, const char *name, uint64_t base, uint64_t size, int isReadOnly);
int ref_undeclare(void *h, uint64_t base);

int ref_hostWrite(void *h, uint64_t addr, const void *src, uint64_t n);
int ref_hostRead(void *h, uint64_t addr, void *dst, uint64_t n);
int ref_devWrite(void *h, uint64_t addr, const void *src, uint64_t n);
int ref_devRead(void *h, uint64_t addr, void *dst, uint64_t n);

int ref_map(void *h, uint64_t p, uint64_t *gpu_out);
int ref_unmap(void *h, uint64_t p);
int ref_release(void *h, uint64_t p);
int ref_mapArray(void *h, uint64_t pp, uint64_t *gpu_out);
int ref_unmapArray(void *h, uint64_t pp);
int ref_releaseArray(void *h, uint64_t pp);
int ref_advanceEpoch(void *h);
int ref_advanceEpochs(void *h, uint64_t n);
uint64_t ref_epoch(void *h);

int ref_mapBatch(void *h, const uint64_t *ps, size_t n, uint64_t *out);
int ref_unmapBatch(void *h, const uint64_t *ps, size_t n);
int ref_releaseBatch(void *h, const uint64_t *ps, size_t n);
int ref_mapArrays(void *h, const uint64_t *pps, size_t k, uint64_t *out);
int ref_unmapArrays(void *h, const uint64_t *pps, size_t k);
int ref_releaseArrays(void *h, const uint64_t *pps, size_t k);
/* device-resident pointer arrays, given here as plain caller memory:
   mapSlots:   slots[i] <- map(slots[i])                       (in place, all-or-nothing)
   unmapSlots: slots[i] <- reverse(slots[i]); unmap each unit; then (release != 0) release each. */
int ref_mapSlots(void *h, uint64_t *slots, size_t n);
int ref_unmapSlots(void *h, uint64_t *slots, size_t n, int release);

int ref_stats(void *h, ref_stats_t *out);
int ref_dumpTable(void *h, ref_unit_t *out, size_t cap, size_t *n);
int ref_replayDevptr(void *h, uint64_t base, uint64_t devptr);
int ref_lookup(void *h, uint64_t p, uint64_t *base, uint64_t *size); /* greatestLTE + A7 acceptance */
int ref_devLookup(void *h, uint64_t g, uint64_t *base, uint64_t *devptr);

/* sample GPU functions executed on the simulated device (test-only) */
int ref_kernel_scale(void *h, uint64_t rows_dev, uint64_t nrows, uint64_t ncols, double alpha);
int ref_runGlue(void *h, const void *prog, size_t n, const uint64_t *ptrs, size_t nptrs, uint64_t max_steps,
                uint64_t *regs_out);
int ref_kernel_treesum_level(void *h, uint64_t child_dev, uint64_t root_dev, uint64_t nnodes,
                             uint64_t lo, uint64_t hi);
/* S2 (config B): C[i][j] = alpha * sum_k A[i][k]*B[k][j] + beta * C[i][j] for rows [row0, row0+nrows),
   through translated row pointers; accumulated in long double (the accurate reference, A21) */
int ref_kernel_gemm_rows(void *h, uint64_t A_rows, uint64_t B_rows, uint64_t C_rows, uint64_t n, uint64_t row0,
                         uint64_t nrows, double alpha, double beta);

#ifdef __cplusplus
}
#endif
#endif
