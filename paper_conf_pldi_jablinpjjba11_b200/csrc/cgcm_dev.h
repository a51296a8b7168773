// cgcm_dev.h -- device-resident data layout shared by the kernels (kernels.cu) and the host
// runtime (runtime.cpp).  DESIGN.md §6 ("Data layout in HBM") describes every field.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace cgcm {

// Allocation-unit record (D3): one 32-byte sector per unit, indexed by the unit's rank
// in base order.  size/devbase drive translation, epoch the copy-back gate (Alg. 2), refcount
// Alg. 1/3.  devbase != 0 <=> the unit has device storage (active, or a global's named region).
struct __align__(32) UnitRec {
  uint64_t size;
  uint64_t devbase;
  uint64_t epoch;
  int32_t refcount;
  uint32_t flags;
};
static_assert(sizeof(UnitRec) == 32, "UnitRec must be one sector");

enum : uint32_t {
  UF_GLOBAL = 1u,
  UF_READONLY = 2u,
  UF_ARRAYMAPPED = 4u,
  UF_ACTIVE = 8u,   // only in dumps
  UF_STORAGE = 16u  // devbase valid
};

// Sorted-key search index ("device-resident sorted interval array with a shared-memory-staged
// top-level search index", north_star).  Keys are sorted u64 (AU bases for the forward index,
// device bases of active AUs for the reverse index).
//   top[t]  = keys[t * 8^h]                      (u64, staged in shared memory by every CTA)
//   lvl[k][j] = keys[j * 8^k] - top[bucket]      (u32, groups of 8 = one 32-byte sector)
//   wide bit t: bucket t spans >= 2^32-1 bytes -> binary search over keys[] instead
// A lookup costs the shared-memory search + h sector loads (+ the record sector).
constexpr int MAXL = 6;
constexpr int TOPMAX = 16384;  // 128 KiB of u64 splitters in shared memory
struct IndexDev {
  const uint64_t *top;
  const uint32_t *wide;
  const uint32_t *lvl[MAXL];
  const uint64_t *keys;
  const int *meta;  // meta[0] = n, meta[1] = h, meta[2] = ntop (written by the build kernels)
};

// Reverse-index payload: position j of the devbase-sorted order -> the unit and its CPU base.
struct __align__(16) RevRec {
  uint64_t base;
  uint32_t unit;
  uint32_t pad;
};

// One input segment of a slot kernel: n u64 slots at device address ptr (8-byte aligned),
// translated in place (out == 0) or into out.  inc = refcount delta per non-null slot.
struct Seg {
  uint64_t ptr, n, out;
  int32_t inc;
  uint32_t pad;
};

// per-call status, written by the kernels with warp-aggregated atomics
struct Status {
  unsigned long long nulls, hits, misses, pending, notmapped, underflow, translated, pad;
};

// gate journal entry: the unit whose epoch this call changed, its old epoch, and whether it needs
// a copy-back (stale and not read-only)
struct __align__(16) Journal {
  uint64_t old_epoch;
  uint32_t unit;
  uint32_t copy;
};

// outer-pointer lookup result (mapArray & friends)
struct PointInfo {
  uint64_t base, size, devbase, epoch;
  int32_t unit, refcount;
  uint32_t flags, pad;
};

// single-unit bookkeeping ops applied by k_unit_ops (one thread per op)
enum : uint32_t { UOP_ADD_RC = 1, UOP_SET_EPOCH = 2, UOP_OR_FLAGS = 3, UOP_AND_FLAGS = 4,
                  UOP_SET_DEVBASE = 5, UOP_SET_RC = 6 };
struct UnitOp {
  uint32_t unit, op;
  uint64_t val;
};

// slot-kernel operations (compile-time bit set)
enum : int {
  OP_WRITE = 1,      // write the translation to the output
  OP_INC = 2,        // refcount += inc, detect 0 -> 1 activations (forward map)
  OP_INCPLAIN = 4,   // refcount += inc (rollbacks, re-map of an array-mapped outer)
  OP_DEC = 8,        // refcount -= inc, detect underflow and 1 -> 0 (release)
  OP_GATE = 16,      // epoch gate of Alg. 2 + journal / copy list
  OP_CHECKMAPPED = 32,  // refcount must be > 0 (unmap of a CPU pointer)
  OP_HITMASK = 64,   // record which slots were translated (rollback / completion)
  OP_DECPLAIN = 128  // refcount -= inc (rollback of OP_INC)
};
enum : int { DIR_FWD = 0, DIR_REV = 1 };
enum : int { SEL_ALL = 0, SEL_HIT = 1, SEL_NOTHIT = 2 };

struct SlotArgs {
  IndexDev ix;
  UnitRec *rec;
  const RevRec *rev;
  const Seg *segs;
  const uint64_t *seg_chunk0;  // [nseg+1] prefix of 4-slot chunks per segment
  int nseg;
  int sel;
  uint64_t nchunks;
  uint8_t *hitmask;            // [nchunks], bit m = slot m of the chunk was translated
  uint64_t epoch;
  Status *st;
  unsigned long long *lc;      // shared list counters of the call: [0] act, [1] journal, [2] free, [3] copy
  uint32_t *act_list;
  Journal *journal;            // every epoch this call changed (rollback)
  uint32_t *copy_list;         // units that need a copy-back (stale, not read-only)
  uint32_t *free_list;
  int lenient;
  int smem_top;                // capacity of the shared-memory splitter array
};

// ---- host-callable launchers (kernels.cu) ----------------------------------------------------
int launch_slots(int dir, int ops, const SlotArgs &a, int nsm, cudaStream_t s);
size_t slots_smem_bytes(int smem_top);
void launch_build_index(const uint64_t *keys, const int *n_dev, int n_cap, uint64_t *top, uint32_t *wide,
                        uint32_t *const *lvl, const size_t *lvl_cap, int *meta, cudaStream_t s);
void launch_remap(int n, const int32_t *old_idx, const uint64_t *size, const uint32_t *flags,
                  const uint64_t *epoch0, const UnitRec *old_rec, UnitRec *new_rec, cudaStream_t s);
void launch_rev_collect(const UnitRec *rec, int n, uint64_t *keys, uint32_t *vals, int *meta, cudaStream_t s);
void launch_rev_payload(const uint32_t *units_sorted, const uint64_t *base, const int *n_dev, int n_cap,
                        RevRec *rev, cudaStream_t s);
size_t sort_pairs_temp_bytes(int n);
void launch_sort_pairs(void *temp, size_t temp_bytes, const uint64_t *kin, uint64_t *kout, const uint32_t *vin,
                       uint32_t *vout, int n, cudaStream_t s);
size_t sort_keys_temp_bytes(int n);
void launch_sort_keys(void *temp, size_t temp_bytes, const uint32_t *kin, uint32_t *kout, int n, cudaStream_t s);
void launch_unit_ops(const UnitOp *ops, int n, UnitRec *rec, cudaStream_t s);
void launch_set_devbase(const uint32_t *units, const uint64_t *devbases, int n, UnitRec *rec, uint64_t epoch,
                        int set_epoch, cudaStream_t s);
void launch_deactivate(const uint32_t *units, int n, UnitRec *rec, cudaStream_t s);
void launch_restore_epochs(const Journal *j, int n, UnitRec *rec, cudaStream_t s);
void launch_lookup_points(IndexDev ix, const UnitRec *rec, const uint64_t *ptrs, int n, PointInfo *out,
                          cudaStream_t s);

}  // namespace cgcm
