/*
 * cgcm.h -- C ABI of the B200-native CGCM run-time library (libcgcm.so, sm_100a).
 *
 * Re-creates the data-parallel hot path of the run-time library of Jablin et al., "Automatic
 * CPU-GPU Communication Management and Optimization", PLDI 2011 (CGCM): batched map/unmap of
 * allocation units (AUs) with CPU<->GPU pointer translation.  "P:Lnnn" cites line nnn of the
 * decoded fulltext of the paper; "Annn" cites a reading of DESIGN.md §3.
 *
 * Conventions (all entry points):
 *   - return int status: CGCM_OK (0) or a negative CGCM_E_* code; out-params are written only on
 *     success; every call is ALL-OR-NOTHING: on error no refcount, epoch, table entry, host byte or
 *     device byte changes (the GPU applies optimistically and rolls back).
 *   - pointers are plain 64-bit addresses.  "host" = CPU virtual address the caller owns;
 *     "device" = CUDA device address (UVA).  No torch types cross this boundary.
 *   - calls act on the calling thread's current context (one per device, cgcm_init makes it current).
 *   - lookups, translations, refcounts and epoch decisions all run in CUDA kernels on the context's
 *     device; the host side only registers AUs, allocates device storage and issues the copies.
 *   - If a batch contains several invalid elements, the status is one of their error codes (A24).
 */
#ifndef CGCM_H
#define CGCM_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* ---- status codes (the same numeric contract as the CPU oracle) ------------ */
enum {
  CGCM_OK = 0,
  CGCM_E_INVALID = -1,      /* bad argument, size 0, NULL where a pointer is required, overflow     */
  CGCM_E_UNREGISTERED = -2, /* greatestLTE miss: below the first AU, in a gap, past the end (A7)    */
  CGCM_E_OVERLAP = -3,      /* declared range overlaps a registered AU                              */
  CGCM_E_NOT_MAPPED = -4,   /* unmap/release at refCount 0, release underflow (A13)                 */
  CGCM_E_BUSY = -5,         /* undeclare while mapped                                               */
  CGCM_E_DUPLICATE = -6,    /* declareGlobal name reused                                            */
  CGCM_E_NOMEM = -7,        /* device arena / pinned host arena exhausted                           */
  CGCM_E_CUDA = -8,         /* a CUDA runtime call failed: cgcm_lastCudaError() has the detail      */
  CGCM_E_MIXED = -9,        /* reserved                                                             */
  CGCM_E_NOCTX = -10,       /* no current context on this thread                                    */
  CGCM_E_MODREF = -11       /* cgcm_regionEnd: the CPU accessed a promoted AU inside the region     */
};

/* ---- cgcm_init flags ----------------------------------------------------------------------- */
enum {
  CGCM_LITERAL_EPOCH = 1u, /* A5 literal reading: map never sets the AU epoch (default: R1, set at
                              activation so map->unmap with no launch copies nothing)             */
  CGCM_LENIENT = 2u,       /* A18: uncovered non-null words in pointer arrays pass through (counted) */
  CGCM_PROFILE = 4u,       /* time every hot kernel with CUDA events on its launch stream (stats)  */
  CGCM_FORCE_SHADOW = 8u,  /* always record the forward-map shadow of device arrays (tests)        */
  CGCM_NO_PAGEDIR = 16u,   /* hot kernels search the level index instead of the page directory     */
  CGCM_PD_V2 = 32u         /* page directory in the v2 entry format even when v3 would fit (tests) */
};

/* ---- AU flags (declare + dump) ------------------------------------------------------------- */
enum {
  CGCM_UNIT_GLOBAL = 1u,      /* declared with cgcm_declareGlobal: persistent device storage (A14) */
  CGCM_UNIT_READONLY = 2u,    /* never copied back (Alg. 2 `isReadOnly`)           */
  CGCM_UNIT_ARRAYMAPPED = 4u, /* device copy holds translated pointers (mapArray), A12             */
  CGCM_UNIT_ACTIVE = 8u       /* refCount > 0                                                       */
};

typedef struct {
  uint64_t base, size, devptr; /* devptr: device copy (0 when inactive, except globals, A14)        */
  int64_t refCount;
  uint64_t epoch;
  uint32_t flags, pad;
} cgcm_unit_t;

typedef struct {
  /* unit-level copy counters: compared EXACTLY with the oracle */
  uint64_t h2d_units, h2d_bytes, d2h_units, d2h_bytes;
  uint64_t activations, frees;
  uint64_t fwd_translations, rev_translations, null_slots, passthrough;
  /* implementation counters (reported, not compared, A22) */
  uint64_t h2d_memcpy_calls, d2h_memcpy_calls, kernel_launches, table_rebuilds, rev_rebuilds;
  double fwd_kernel_ms, rev_kernel_ms; /* CGCM_PROFILE: summed event time of the hot slot kernels */
  uint64_t fwd_kernel_calls, rev_kernel_calls;
  uint64_t fwd_kernel_slots, rev_kernel_slots; /* slots processed by those launches               */
  /* NEXT-3 coherence groups: activations copied from a peer context's device copy (compared
   * exactly with the oracle), and the device-to-device copies that moved them (reported) */
  uint64_t peer_units, peer_bytes, peer_memcpy_calls;
  /* NEXT-1: declarations merged into the device table without a rebuild (delta appends) */
  uint64_t table_merges;
} cgcm_stats_t;

/* ================================ lifecycle =================================================
 * cgcm_init: create a context on `device` and make it current for the calling thread.
 *   dev_arena/arena_bytes: device memory the runtime sub-allocates for AU copies and its own
 *     scratch (PyTorch provides it: torch.empty(arena_bytes, uint8, device)).  NULL -> cudaMalloc.
 *     Owned by the caller; must outlive the context.
 *   main_stream: cudaStream_t on which translation kernels run and which user kernels must use
 *     (stream-ordered results).  copy_stream: side stream for the coalesced host<->device copies.
 *     NULL -> the runtime creates its own.
 * cgcm_finalize: destroy the current context (device storage of globals is released). */
int cgcm_init(int device, void *dev_arena, size_t arena_bytes, void *main_stream, void *copy_stream,
              unsigned flags);
int cgcm_finalize(void);
void *cgcm_getContext(void);           /* opaque handle of the current context (NULL if none)   */
int cgcm_setContext(void *ctx);        /* make `ctx` current on this thread                      */
const char *cgcm_strerror(int status);
const char *cgcm_lastCudaError(void);  /* text of the last CUDA failure on this thread          */

/* ================================ registration (Table 2) ======================
 * cgcm_declareAlloc: register the heap/stack AU [base, base+size), size >= 1, no overlap (adjacent
 *   is allowed).  Its epoch starts at the current globalEpoch (A20).  The CPU bytes stay owned by
 *   the caller and must stay valid while declared; the CPU must not write an AU while it is mapped
 *   (A16).  cgcm_declareAllocFlags additionally takes CGCM_UNIT_READONLY (an AU in read-only memory).
 * cgcm_declareBatch: n AUs at once (bases need not be sorted); all-or-nothing.
 * cgcm_undeclare: exact base; CGCM_E_BUSY if refCount > 0 (declareAlloca scope exit, free()).
 * cgcm_declareGlobal: a global: persistent device storage allocated on first map and
 *   reused (A14); unique name (CGCM_E_DUPLICATE); isReadOnly -> never copied back.             */
int cgcm_declareAlloc(void *base, size_t size);
int cgcm_declareAllocFlags(void *base, size_t size, unsigned unit_flags);
int cgcm_declareBatch(void *const *bases, const size_t *sizes, size_t n, unsigned unit_flags);
int cgcm_undeclare(void *base);
int cgcm_declareGlobal(const char *name, void *base, size_t size, int isReadOnly);
/* cgcm_declareGlobalSymbol (NEXT-4; Alg. 1's `cuModuleGetGlobal(name)` branch, P:L214-215,
 *   P:L219-222, and the glue-kernel globals of P:L305-310): as cgcm_declareGlobal, but the device
 *   copy IS the __device__ variable at dev_symbol (a device address the caller obtained with
 *   cudaGetSymbolAddress / cuModuleGetGlobal, >= size bytes, owned by its module and never freed by
 *   the runtime).  map() returns dev_symbol + (p - base); activation copies the host bytes into the
 *   symbol and copy-back reads them out of it, so GPU code that names the variable directly sees the
 *   mapped data.  CGCM_E_INVALID for a NULL symbol; CGCM_E_OVERLAP if its range overlaps another
 *   bound symbol or touches one whose host unit does not touch this one in the same order (A7:
 *   adjacent device copies must mirror adjacent host units).                                      */
int cgcm_declareGlobalSymbol(const char *name, void *base, size_t size, int isReadOnly, void *dev_symbol);
/* Heap wrappers (R10): a header-free pinned host arena; every block is declared as one AU, so
 * consecutive blocks are host-adjacent and their copies coalesce.  cgcm_free undeclares (BUSY if
 * mapped -> the block is not freed).  NULL on failure.                                           */
void *cgcm_malloc(size_t n);
int cgcm_free(void *p);
/* calloc/realloc wrappers (NEXT-1).  cgcm_realloc keeps the AU registered under its new
 * base (the old registration expires); a mapped AU cannot move: NULL, nothing changes (BUSY).      */
void *cgcm_calloc(size_t nmemb, size_t size);
void *cgcm_realloc(void *p, size_t n);
/* declareAlloca (Table 2): an escaping "stack" variable of n bytes, from the
 * pinned arena, registered until the innermost scope opened with cgcm_scopeEnter exits.  Scopes nest;
 * cgcm_scopeExit returns CGCM_E_BUSY (and keeps the scope) if one of its AUs is still mapped.        */
void *cgcm_declareAlloca(size_t n);
int cgcm_scopeEnter(void);
int cgcm_scopeExit(void);

/* ================================ mapping (Alg. 1-3, Table 2) ==============================
 * cgcm_map (Alg. 1): *gpu_out = devptr + (cpu - base) of the AU containing `cpu`;
 *   refCount += 1; on 0 -> 1 the AU gets device storage and one host->device copy.  NULL -> NULL.
 *   Data is ready for work enqueued on main_stream after the call returns.
 * cgcm_unmap (Alg. 2, A1/A3/A4): copy the device copy back iff the AU's epoch is not
 *   current and it is not read-only (array-mapped AUs are reverse translated, A12); then
 *   epoch = globalEpoch.  Synchronous: host memory is updated when it returns.
 * cgcm_release (Alg. 3): refCount -= 1; at 0 the device copy is freed (not globals).
 * cgcm_mapArray: `cpu` points into an AU of pointers (all floor(size/8)
 *   words are slots, A10).  The outer AU is activated first (A9), every non-null slot is mapped
 *   (+1 refCount per slot, A8) and the outer's device copy receives the translated pointers,
 *   rewritten IN PLACE on the device.  *gpu_out = device address of `cpu` in that copy.
 * cgcm_unmapArray: unmap of the outer (reverse GPU->CPU rewrite when copied back, a3) and then of
 *   every element.  cgcm_releaseArray: release every element, then the outer.
 * cgcm_advanceEpoch: globalEpoch += 1; call once after every GPU function launch.
 * cgcm_advanceEpochs: globalEpoch += n, exactly as n calls of cgcm_advanceEpoch (n launches with no
 *   runtime call between them); n < 2^32 - 32, else CGCM_E_INVALID and nothing changes.  Used by the
 *   tests to reach the u32 device-epoch origin move (DESIGN A28) without 4e9 calls.  */
int cgcm_map(const void *cpu, void **gpu_out);
int cgcm_unmap(const void *cpu);
int cgcm_release(const void *cpu);
int cgcm_mapArray(void *const *cpu, void ***gpu_out);
int cgcm_unmapArray(void *const *cpu);
int cgcm_releaseArray(void *const *cpu);
int cgcm_advanceEpoch(void);
int cgcm_advanceEpochs(uint64_t n);
uint64_t cgcm_epoch(void);

/* ================================ data-parallel batch forms ================================
 * Same semantics as the sequential loop over the elements (validate, then apply in index order).
 * Host arrays: cpu[n] / gpu_out[n] are host memory.                                              */
int cgcm_mapBatch(const void *const *cpu, size_t n, void **gpu_out);
int cgcm_unmapBatch(const void *const *cpu, size_t n);
int cgcm_releaseBatch(const void *const *cpu, size_t n);
int cgcm_mapArrays(void *const *const *arrays, size_t k, void ***gpu_out);
int cgcm_unmapArrays(void *const *const *arrays, size_t k);
int cgcm_releaseArrays(void *const *const *arrays, size_t k);
/* Device-resident pointer arrays (the hot kernels without the host<->device copy of the array):
 * d_slots is a DEVICE pointer to n 8-byte-aligned u64 words, rewritten in place.
 * cgcm_mapArrayDevice:   d_slots[i] <- map(d_slots[i])   (CPU -> GPU; refcount, activation)
 * cgcm_unmapArrayDevice: d_slots[i] <- reverse(d_slots[i]) (GPU -> CPU), unmap every AU hit
 *   (epoch-gated copy-back), and with CGCM_RELEASE also release each slot (Listing 3's
 *   unmapArray + releaseArray, fused).  Stream-ordered on main_stream, synchronous on return.   */
enum { CGCM_RELEASE = 1u };
int cgcm_mapArrayDevice(uint64_t *d_slots, size_t n);
int cgcm_unmapArrayDevice(uint64_t *d_slots, size_t n, unsigned flags);

/* ===================== map promotion at run time (NEXT-2) ===================================
 * The paper's map promotion (§5.1) hoists a loop's map/mapArray calls above
 * it and its unmaps below it, so in-loop maps find their AUs active (no copies, A2) and in-loop
 * releases never reach refCount 0; it is legal only if the CPU neither modifies nor references the
 * promoted AUs inside the loop (¬modOrRef).  Without the compiler pass:
 * cgcm_regionBegin: map (kind CGCM_REGION_MAP) or mapArray (CGCM_REGION_MAPARRAY) each of ptrs[0..n)
 *   once and hold those references until cgcm_regionEnd.  All-or-nothing.  CGCM_E_BUSY if a region
 *   is open on this context (or, with CGCM_REGION_CHECK, anywhere in the process).
 *   CGCM_REGION_CHECK: the dynamic modOrRef checker -- the host pages of every promoted AU (for
 *   arrays: the outer AU and every AU its slots point into) are made PROT_NONE; a CPU access to them
 *   outside a runtime call is counted (a SIGSEGV handler reopens the page and lets the access
 *   proceed).  Whole pages are protected, so an access to other data sharing a page also counts
 *   (conservative).  CGCM_E_INVALID if mprotect refuses the pages (cgcm_lastCudaError has errno).
 * cgcm_regionEnd: reopen the pages, then unmap/unmapArray + release/releaseArray every promoted
 *   pointer (reverse order; epoch-gated copy-backs as usual).  *violations = accesses counted.
 *   Returns CGCM_E_MODREF if any (the promoted execution may differ from the naive one: the caller's
 *   loop must not be promoted), else the first unmap/release error, else OK.                      */
enum { CGCM_REGION_MAP = 0u, CGCM_REGION_MAPARRAY = 1u };
enum { CGCM_REGION_CHECK = 1u };
int cgcm_regionBegin(void *const *ptrs, const unsigned *kinds, size_t n, unsigned flags);
int cgcm_regionEnd(size_t *violations);

/* ================================ coherence groups (NEXT-3) ================================
 * The paper maps AUs between the CPU and ONE GPU (one GTX 480).  A coherence
 * group extends that to several contexts (one per GPU, or several on one GPU) over one CPU address
 * space: each context keeps its own table, refcounts and epochs (an epoch per GPU), and a writable AU
 * may be active on several of them.  Reading A31: when a context activates an AU (Alg. 1's
 * refCount 0 -> 1 copy), and another member -- the first in join order -- holds the same AU (same base
 * and size) active and DIRTY, i.e. it launched a GPU function since the AU became coherent there (its
 * unmap would copy the AU back, Alg. 2) and the AU is not read-only, the copy comes from that member's
 * device copy (device to device: NVLink peer copy across GPUs) instead of the host.  Ordered after the
 * work already on the source context's main stream.  Counted in peer_units / peer_bytes, not h2d_*.
 * Two members writing one AU between their unmaps is undefined, as CPU writes to a mapped AU are (A16).
 * cgcm_groupCreate: a new empty group.  cgcm_groupJoin: the current context joins (at most one group).
 * cgcm_groupLeave: the current context leaves (also done by cgcm_finalize).  cgcm_groupDestroy: the
 * group must be empty.  The members of a group must not be called concurrently from several threads
 * (an activation reads the peers' tables under their locks).                                      */
int cgcm_groupCreate(void **group_out);
int cgcm_groupJoin(void *group);
int cgcm_groupLeave(void);
int cgcm_groupDestroy(void *group);

/* ================================ glue kernels (NEXT-4) ====================================
 * P:L305-310 (§5.3 "Glue Kernels"): "Sometimes small CPU code regions between two GPU functions prevent
 * map promotion.  The performance of this code is inconsequential, but transforming it into a
 * single-threaded GPU function obviates the need to copy the allocation units between GPU and CPU
 * memories."  The paper's compiler lowers such a region; at run time the region is given as a short
 * program for a single GPU thread over 32 64-bit registers:
 *   r[0..nptrs) = the GPU translations of cpu_ptrs[] (Alg. 1's devptr + (ptr - base) of AUs that must
 *                 be mapped: refCount > 0, else CGCM_E_NOT_MAPPED; not in an AU: CGCM_E_UNREGISTERED;
 *                 NULL stays 0), the other registers 0;
 *   ops (dst, a, b are register numbers < 32, imm a signed 64-bit immediate):
 *     MOVI  r[dst] = imm                      ADD/SUB/MUL  r[dst] = r[a] op r[b] (u64, wrapping)
 *     ADDI  r[dst] = r[a] + imm               FADD/FSUB/FMUL/FDIV  binary64 op of r[a], r[b] (RN, no FMA)
 *     LD    r[dst] = *(u64 *)(r[a] + imm)     ST  *(u64 *)(r[a] + imm) = r[b]
 *     BNZ   if r[a] != 0: continue at instruction imm (0 <= imm < n)      HALT  stop
 *   Every LD/ST address must lie, with its 8 bytes, inside the device copy of an ACTIVE unit (a pointer
 *   loaded from an array-mapped AU is a GPU pointer, so pointer chasing works on device data);
 *   otherwise CGCM_E_UNREGISTERED.  More than max_steps executed instructions, an unknown op, a
 *   register >= 32 or a jump out of range: CGCM_E_INVALID.  A failed program may have executed some
 *   stores (a GPU function is not transactional).
 * The program runs on main_stream, one thread, and the call returns when it is done.  It is a GPU
 * function launch: call cgcm_advanceEpoch() after it like after any launch.  regs_out
 * (optional, 32 entries) receives the final registers.                                          */
typedef struct {
  uint32_t op, dst, a, b;
  int64_t imm;
} cgcm_glue_op_t;
enum {
  CGCM_GLUE_MOVI = 1, CGCM_GLUE_ADD = 2, CGCM_GLUE_ADDI = 3, CGCM_GLUE_SUB = 4, CGCM_GLUE_MUL = 5,
  CGCM_GLUE_FADD = 6, CGCM_GLUE_FSUB = 7, CGCM_GLUE_FMUL = 8, CGCM_GLUE_FDIV = 9, CGCM_GLUE_LD = 10,
  CGCM_GLUE_ST = 11, CGCM_GLUE_BNZ = 12, CGCM_GLUE_HALT = 13
};
int cgcm_launchGlue(const cgcm_glue_op_t *prog, size_t n, const void *const *cpu_ptrs, size_t nptrs,
                    uint64_t max_steps, uint64_t *regs_out);

/* ================================ introspection ===========================================
 * cgcm_stats: counters since init.  cgcm_dumpTable: the AU table in base order (cap entries; *n
 *   = total; CGCM_E_NOMEM if cap < total).  cgcm_resetStats zeroes the counters.                */
int cgcm_stats(cgcm_stats_t *out);
int cgcm_resetStats(void);
int cgcm_dumpTable(cgcm_unit_t *out, size_t cap, size_t *n);
/* arena usage in bytes (AU copies + runtime scratch), for balance checks */
int cgcm_arenaUsage(size_t *used, size_t *capacity);
/* the forward search structures of the current table (built on demand, like a map would):
 * the level index (top splitters + `levels` u32 sector levels) always exists; the page directory
 * is what the hot kernels search when pd_segments > 0.  Implementation detail
 * (A22), for tests and the bench.                                                              */
typedef struct {
  uint64_t units;             /* AUs in the device table                                          */
  uint32_t levels;            /* sector levels below the shared-memory top of the level index     */
  uint32_t pd_segments;       /* page-directory address segments (0: none built)                 */
  uint64_t pd_pages;          /* 32-byte page entries                                             */
  uint64_t pd_overflow_pages; /* pages with more than 12 unit starts (offsets in a side array)    */
  uint64_t pd_bytes;          /* entries + overflow offsets                                       */
  uint32_t pd_min_shift, pd_max_shift; /* page sizes 2^shift of the segments                     */
  uint32_t pd_format, pad;    /* page-entry format: 3 (candidates with ends + page state) or 2      */
} cgcm_index_info_t;
int cgcm_indexInfo(cgcm_index_info_t *out);
/* The device storage the runtime holds for AU copies (for leak / balance checks; the paper's
 * counterpart is Alg. 1's cuMemAlloc and Alg. 3's cuMemFree): one entry per live device
 * extent -- its device range [addr, addr + bytes), the number of AU copies it still holds (`live`;
 * an extent is freed when that reaches 0) and whether it is a bound __device__ symbol (external, not
 * arena memory).  *n = total; CGCM_E_NOMEM if cap < total (out may be NULL with cap 0).
 * cgcm_storageInfo: totals, plus the forward-map shadows (12 B per slot) that currently
 * record a mapped array (`shadows_live`) and the cached buffers of consumed ones (`shadows_cached`,
 * reused by the next map of the same device array).                                               */
typedef struct {
  uint64_t addr, bytes;
  int64_t live;
  uint32_t external, pad;
} cgcm_extent_t;
int cgcm_dumpExtents(cgcm_extent_t *out, size_t cap, size_t *n);
typedef struct {
  uint64_t extents, extent_bytes;        /* live arena extents (not external)                      */
  uint64_t external_extents;             /* bound __device__ symbols                               */
  uint64_t shadows_live, shadow_live_bytes;
  uint64_t shadows_cached, shadow_cached_bytes;
  uint64_t arena_used, arena_capacity;
} cgcm_storage_t;
int cgcm_storageInfo(cgcm_storage_t *out);

#ifdef __cplusplus
}
#endif
#endif /* CGCM_H */
