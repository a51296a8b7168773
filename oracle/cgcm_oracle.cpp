// cgcm_oracle.cpp -- CPU ORACLE of the CGCM run-time library.  TEST INFRASTRUCTURE ONLY.
//
// Plain sequential C++17.  It follows the paper's Algorithms 1-3, the interface of
// Table 2 and the array variants of P:L203-207 step by step, with the readings A1..A23
// of DESIGN.md §3 where the extracted text is silent or garbled.  There is no blocking, batching,
// fusion or reordering: a batch is "validate lookups, then apply the scalar semantics in index
// order", and a failing call is rolled back by an undo journal so that it has no effect at all.
//
// Shares no code with the product (paper_conf_pldi_jablinpjjba11_b200/csrc, include/cgcm.h).
//
// Parity status per function (DESIGN.md §3.2 lists the pins):
//   greatestLTE / lookup / devLookup ......... pinned (brute force, tests/test_oracle_lookup.py)
//   map / mapArray / mapBatch / mapSlots ..... pinned (closed form, invariants, golden Listing 1)
//   unmap / unmapArray / unmapSlots .......... pinned (round trip, permutation, closed-form counts)
//   release / releaseArray ................... pinned (balance, closed-form refcounts)
//   epoch gate ............................... pinned (closed-form copy counts configs A/B/D)
//   error paths (A6/A7/A13 readings) ......... parity unpinned by the paper: only state-unchanged checks
//   sample kernels S1/S3 ..................... pinned (numpy repeated multiply / recursive sum)
#include "cgcm_oracle.h"

#include <algorithm>
#include <array>
#include <climits>
#include <cstring>
#include <map>
#include <memory>
#include <string>
#include <unordered_map>
#include <unordered_set>
#include <vector>

namespace {

typedef uint64_t u64;
typedef int64_t i64;

// ------------------------------------------------------------------------------------------------
// Sparse byte memory: 4 KiB pages, an absent page reads as zero.  Used for both the simulated host
// image (keys = the caller's CPU addresses) and the simulated device (keys = simulated devptrs).
// ------------------------------------------------------------------------------------------------
const u64 PAGE = 4096;
typedef std::array<uint8_t, PAGE> Page;

struct Txn;

struct SparseMem {
  std::unordered_map<u64, std::unique_ptr<Page>> pages;
  Txn *txn = nullptr;

  void read(u64 addr, void *dst, u64 n) const {
    uint8_t *d = static_cast<uint8_t *>(dst);
    while (n) {
      u64 pg = addr / PAGE, off = addr % PAGE, k = std::min(n, PAGE - off);
      auto it = pages.find(pg);
      if (it == pages.end()) std::memset(d, 0, k);
      else std::memcpy(d, it->second->data() + off, k);
      addr += k; d += k; n -= k;
    }
  }
  Page *touch(u64 pg);  // page for writing (journaled when a transaction is open)
  void write(u64 addr, const void *src, u64 n) {
    const uint8_t *s = static_cast<const uint8_t *>(src);
    while (n) {
      u64 pg = addr / PAGE, off = addr % PAGE, k = std::min(n, PAGE - off);
      std::memcpy(touch(pg)->data() + off, s, k);
      addr += k; s += k; n -= k;
    }
  }
  bool present(u64 pg) const { return pages.count(pg) != 0; }
  void zero(u64 addr, u64 n) {  // write zeros, but never materialise an absent page
    while (n) {
      u64 pg = addr / PAGE, off = addr % PAGE, k = std::min(n, PAGE - off);
      if (present(pg)) std::memset(touch(pg)->data() + off, 0, k);
      addr += k; n -= k;
    }
  }
  u64 get64(u64 addr) const { u64 v; read(addr, &v, 8); return v; }
  void put64(u64 addr, u64 v) { write(addr, &v, 8); }
  double getf(u64 addr) const { double v; read(addr, &v, 8); return v; }
  void putf(u64 addr, double v) { write(addr, &v, 8); }
};

// copy n bytes src[sa..] -> dst[da..] (chunked so that zero pages stay absent)
void copyMem(SparseMem &dst, u64 da, const SparseMem &src, u64 sa, u64 n) {
  std::vector<uint8_t> buf;
  while (n) {
    u64 k = std::min(n, std::min(PAGE - sa % PAGE, PAGE - da % PAGE));
    if (!src.present(sa / PAGE)) {
      dst.zero(da, k);
    } else {
      buf.resize(k);
      src.read(sa, buf.data(), k);
      dst.write(da, buf.data(), k);
    }
    sa += k; da += k; n -= k;
  }
}

// ------------------------------------------------------------------------------------------------
// Allocation-unit record (D3): the fields Algorithms 1-3 use + arrayMapped (A12).
// ------------------------------------------------------------------------------------------------
struct Unit {
  u64 base = 0, size = 0, devptr = 0;
  i64 refCount = 0;
  u64 epoch = 0;
  bool isGlobal = false, isReadOnly = false, arrayMapped = false;
  bool hasStorage = false;  // globals: named region allocated once, never freed (A14)
  std::string name;
};

// Undo journal: everything a failing call may have touched is restored on rollback.
struct Txn {
  bool on = false;
  std::unordered_map<u64, Unit> savedUnits;  // base -> unit before its first change
  std::vector<std::pair<bool, std::pair<u64, u64>>> activeOps;  // (inserted?, (devptr, base))
  std::map<std::pair<SparseMem *, u64>, std::unique_ptr<Page>> savedPages;  // null = was absent
  ref_stats_t stats{};
  u64 cursor = 0;
  std::unordered_map<u64, u64> replay;
};

Page *SparseMem::touch(u64 pg) {
  auto it = pages.find(pg);
  if (txn && txn->on) {
    auto key = std::make_pair(this, pg);
    if (!txn->savedPages.count(key)) {
      std::unique_ptr<Page> old;
      if (it != pages.end()) old.reset(new Page(*it->second));
      txn->savedPages.emplace(key, std::move(old));
    }
  }
  if (it == pages.end()) {
    std::unique_ptr<Page> p(new Page());
    p->fill(0);
    Page *raw = p.get();
    pages.emplace(pg, std::move(p));
    return raw;
  }
  return it->second.get();
}

const u64 DEV0 = 0x0100000000000000ull;  // simulated device address space (never dereferenced)

struct Oracle {
  unsigned flags = 0;
  std::map<u64, Unit> table;   // allocInfoMap: self-balancing tree keyed by base
  std::map<u64, u64> active;   // devptr -> base of units with refCount > 0 (for devLookup, a3)
  std::unordered_set<std::string> globalNames;
  u64 globalEpoch = 0;         // P:L233-234; starts at 0 (A20)
  SparseMem ownHost, dev;
  SparseMem *hostp = &ownHost;  // the host memory (a coherence group's members share the leader's)
  SparseMem &host() { return *hostp; }
  // NEXT-3 coherence group (reading A31): the members in join order, shared by all of them
  std::shared_ptr<std::vector<Oracle *>> group;
  u64 cursor = DEV0;
  std::unordered_map<u64, u64> replay;  // base -> devptr to use at the next activation
  ref_stats_t st{};
  Txn txn;

  Oracle() { ownHost.txn = &txn; dev.txn = &txn; }

  // ---- transactions ------------------------------------------------------------------------
  void begin() {
    hostp->txn = &txn;  // a shared host journals into the member whose call is running
    txn.on = true;
    txn.savedUnits.clear(); txn.activeOps.clear(); txn.savedPages.clear();
    txn.stats = st; txn.cursor = cursor; txn.replay = replay;
  }
  void commit() { txn.on = false; txn.savedUnits.clear(); txn.activeOps.clear(); txn.savedPages.clear(); }
  void rollback() {
    for (auto &kv : txn.savedUnits) table[kv.first] = kv.second;
    for (auto it = txn.activeOps.rbegin(); it != txn.activeOps.rend(); ++it) {
      if (it->first) active.erase(it->second.first);
      else active[it->second.first] = it->second.second;
    }
    for (auto &kv : txn.savedPages) {
      SparseMem *m = kv.first.first;
      u64 pg = kv.first.second;
      if (kv.second) *m->pages[pg] = *kv.second;
      else m->pages.erase(pg);
    }
    st = txn.stats; cursor = txn.cursor; replay = txn.replay;
    txn.on = false; txn.savedUnits.clear(); txn.activeOps.clear(); txn.savedPages.clear();
  }
  Unit &mut(Unit &u) {
    if (txn.on && !txn.savedUnits.count(u.base)) txn.savedUnits.emplace(u.base, u);
    return u;
  }
  void activeInsert(u64 d, u64 b) { active[d] = b; if (txn.on) txn.activeOps.push_back({true, {d, b}}); }
  void activeErase(u64 d) {
    auto it = active.find(d);
    if (it == active.end()) return;
    if (txn.on) txn.activeOps.push_back({false, {d, it->second}});
    active.erase(it);
  }

  // ---- R1 greatestLTE (first line of Alg. 1/2/3) + A7 acceptance ------------------
  Unit *lookup(u64 p) {
    auto it = table.upper_bound(p);          // first key > p
    if (it == table.begin()) return nullptr;  // no key <= p
    --it;                                     // greatest key <= p
    Unit &u = it->second;
    return (p - u.base <= u.size) ? &u : nullptr;  // A7: p == base+size (one past the end) accepted
  }
  // device-side lookup over ACTIVE units for reverse translation (a3, R6)
  Unit *devLookup(u64 g) {
    auto it = active.upper_bound(g);
    if (it == active.begin()) return nullptr;
    --it;
    Unit &u = table.at(it->second);
    return (g - u.devptr <= u.size) ? &u : nullptr;
  }

  // ---- device storage ------------------------------------------------------------------------
  u64 devAlloc(const Unit &u) {  // cuMemAlloc (Alg. 1) simulated
    auto it = replay.find(u.base);
    if (it != replay.end()) { u64 d = it->second; replay.erase(it); return d; }
    u64 d = ((cursor + 255) / 256) * 256 + (u.base % 256);  // devptr == base (mod 256)
    cursor = d + u.size + 1 + 16;                           // 1 B slack (A7) + 16 B guard
    return d;
  }
  // NEXT-3 (A31): the first other member of the group (join order) holding the same AU active and dirty
  // -- it launched a GPU function since the AU became coherent there (epoch != its globalEpoch, the
  // condition under which its unmap would copy back, Alg. 2) -- and writable; else none (the host is current)
  Oracle *peerSource(const Unit &u) {
    if (!group) return nullptr;
    for (Oracle *c : *group) {
      if (c == this) continue;
      auto it = c->table.find(u.base);
      if (it == c->table.end() || it->second.size != u.size) continue;
      const Unit &cu = it->second;
      if (cu.refCount > 0 && cu.epoch != c->globalEpoch && !cu.isReadOnly) return c;
    }
    return nullptr;
  }
  // refCount 0 -> 1 transition of Alg. 1 (allocation/named region + optional HtoD copy)
  void activate(Unit &u, bool copyHtoD) {
    Unit &m = mut(u);
    if (m.isGlobal) {
      if (!m.hasStorage) { m.devptr = devAlloc(m); m.hasStorage = true; }  // cuModuleGetGlobal
    } else {
      m.devptr = devAlloc(m);                                               // cuMemAlloc
    }
    if (copyHtoD) {
      Oracle *src = peerSource(m);
      if (src) {  // NEXT-3 (A31): the newest copy is on a group peer's device -- copy it from there
        const Unit &pu = src->table.at(m.base);
        copyMem(dev, m.devptr, src->dev, pu.devptr, m.size);
        st.peer_units += 1; st.peer_bytes += m.size;
      } else {                                                              // cuMemcpyHtoD
        copyMem(dev, m.devptr, host(), m.base, m.size);
        st.h2d_units += 1; st.h2d_bytes += m.size;
      }
    }
    if (!(flags & REF_LITERAL_EPOCH)) m.epoch = globalEpoch;  // A5 reading R1
    st.activations += 1;
    activeInsert(m.devptr, m.base);
  }

  // ---- Algorithm 1: map (A2: copy only inside `if refCount = 0`) ---------------
  int map(u64 p, u64 *out) {
    if (p == 0) { st.null_slots += 1; *out = 0; return REF_OK; }  // A6
    Unit *u = lookup(p);
    if (!u) {
      if (flags & REF_LENIENT) { st.passthrough += 1; *out = p; return REF_OK; }
      return REF_E_UNREGISTERED;
    }
    if (u->refCount == 0) activate(*u, true);
    if (u->refCount >= INT32_MAX) return REF_E_INVALID;  // A20: i32 refcounts
    mut(*u).refCount += 1;
    st.fwd_translations += 1;
    *out = u->devptr + (p - u->base);  // "return info.devptr + (ptr - info.base)"
    return REF_OK;
  }

  // copy the device copy of u back to the host (the cuMemcpyDtoH of Alg. 2).  An array-mapped
  // unit holds GPU pointers: its slots are reverse translated (R6, A12); trailing bytes verbatim.
  int copyBack(Unit &u) {
    if (u.arrayMapped) {
      u64 n = u.size / 8;
      for (u64 i = 0; i < n; ++i) {
        u64 g = dev.get64(u.devptr + 8 * i), h = 0;
        if (g != 0) {
          Unit *v = devLookup(g);
          if (!v) {
            if (!(flags & REF_LENIENT)) return REF_E_UNREGISTERED;
            st.passthrough += 1; h = g;
          } else {
            h = v->base + (g - v->devptr);
            st.rev_translations += 1;
          }
        }
        host().put64(u.base + 8 * i, h);
      }
      copyMem(host(), u.base + 8 * n, dev, u.devptr + 8 * n, u.size - 8 * n);
    } else {
      copyMem(host(), u.base, dev, u.devptr, u.size);
    }
    st.d2h_units += 1; st.d2h_bytes += u.size;
    return REF_OK;
  }

  // ---- Algorithm 2: unmap (A1 "!=", A3 info.base, A4 epoch set unconditionally) -
  int unmap(u64 p) {
    if (p == 0) return REF_OK;
    Unit *u = lookup(p);
    if (!u) return (flags & REF_LENIENT) ? REF_OK : REF_E_UNREGISTERED;
    if (u->refCount == 0) return REF_E_NOT_MAPPED;  // A13
    if (u->epoch != globalEpoch && !u->isReadOnly) {
      int s = copyBack(*u);
      if (s) return s;
    }
    mut(*u).epoch = globalEpoch;
    return REF_OK;
  }

  // ---- Algorithm 3: release (globals never freed P:L236-238) -------------------
  int release(u64 p) {
    if (p == 0) return REF_OK;
    Unit *u = lookup(p);
    if (!u) return (flags & REF_LENIENT) ? REF_OK : REF_E_UNREGISTERED;
    if (u->refCount == 0) return REF_E_NOT_MAPPED;  // A13: underflow is an error
    Unit &m = mut(*u);
    m.refCount -= 1;
    if (m.refCount == 0) {
      m.arrayMapped = false;
      activeErase(m.devptr);
      if (!m.isGlobal) st.frees += 1;  // cuMemFree
    }
    return REF_OK;
  }

  int checkLookups(const u64 *ps, size_t n) {  // "validate all" pre-pass of the batch forms
    if (flags & REF_LENIENT) return REF_OK;
    for (size_t i = 0; i < n; ++i)
      if (ps[i] != 0 && !lookup(ps[i])) return REF_E_UNREGISTERED;
    return REF_OK;
  }
  std::vector<u64> hostSlots(const Unit &o) {
    std::vector<u64> q(o.size / 8);
    for (u64 i = 0; i < q.size(); ++i) q[i] = host().get64(o.base + 8 * i);
    return q;
  }

  // ---- mapArray (Table 2; A8, A9, A10) --------------------------------
  int mapArray(u64 pp, u64 *out) {
    Unit *o = lookup(pp);
    if (!o) return REF_E_UNREGISTERED;
    u64 n = o->size / 8;
    std::vector<u64> q = hostSlots(*o);
    int s = checkLookups(q.data(), q.size());
    if (s) return s;
    if (o->refCount == 0) {
      // activate without the raw copy: the "new array" of translated pointers is o's HtoD
      activate(*o, false);
      copyMem(dev, o->devptr + 8 * n, host(), o->base + 8 * n, o->size - 8 * n);  // trailing bytes
      st.h2d_units += 1; st.h2d_bytes += o->size;
    }
    if (o->refCount >= INT32_MAX) return REF_E_INVALID;
    Unit &m = mut(*o);
    m.refCount += 1;
    m.arrayMapped = true;  // A9: the outer AU first, then its elements
    for (u64 i = 0; i < n; ++i) {
      u64 t;
      s = map(q[i], &t);  // A8: +1 per non-null slot
      if (s) return s;
      dev.put64(o->devptr + 8 * i, t);
    }
    *out = o->devptr + (pp - o->base);
    return REF_OK;
  }

  // ---- unmapArray (Table 2; A12) ---------------------------------------
  int unmapArray(u64 pp) {
    Unit *o = lookup(pp);
    if (!o) return REF_E_UNREGISTERED;
    if (o->refCount == 0) return REF_E_NOT_MAPPED;
    // the element pointers the element unmaps will see: host[o] after unmap(o)
    std::vector<u64> h(o->size / 8);
    bool copy_o = o->epoch != globalEpoch && !o->isReadOnly;
    for (u64 i = 0; i < h.size(); ++i) {
      if (!copy_o) { h[i] = host().get64(o->base + 8 * i); continue; }
      u64 g = dev.get64(o->devptr + 8 * i);
      if (!o->arrayMapped || g == 0) { h[i] = g; continue; }
      Unit *v = devLookup(g);
      if (!v) {
        if (!(flags & REF_LENIENT)) return REF_E_UNREGISTERED;
        h[i] = g;
        continue;
      }
      h[i] = v->base + (g - v->devptr);
    }
    int s = checkLookups(h.data(), h.size());
    if (s) return s;
    for (u64 x : h)
      if (x != 0) { Unit *u = lookup(x); if (u && u->refCount == 0) return REF_E_NOT_MAPPED; }
    s = unmap(o->base);  // the outer first: a self-reference is then skipped by its epoch (A12)
    if (s) return s;
    for (u64 x : h) { s = unmap(x); if (s) return s; }
    return REF_OK;
  }

  // ---- releaseArray (Table 2) --------------------------------------------------------
  int releaseArray(u64 pp) {
    Unit *o = lookup(pp);
    if (!o) return REF_E_UNREGISTERED;
    if (o->refCount == 0) return REF_E_NOT_MAPPED;
    u64 base = o->base;
    std::vector<u64> q = hostSlots(*o);
    int s = checkLookups(q.data(), q.size());
    if (s) return s;
    for (u64 x : q) { s = release(x); if (s) return s; }
    return release(base);
  }

  // ---- device-resident pointer arrays ------------------------------------------------------------
  int mapSlots(u64 *slots, size_t n) {
    int s = checkLookups(slots, n);
    if (s) return s;
    std::vector<u64> out(n);
    for (size_t i = 0; i < n; ++i) { s = map(slots[i], &out[i]); if (s) return s; }
    std::memcpy(slots, out.data(), n * 8);
    return REF_OK;
  }
  int unmapSlots(u64 *slots, size_t n, bool rel) {
    std::vector<u64> h(n), unitBase(n, 0);
    for (size_t i = 0; i < n; ++i) {  // reverse lookups against the active set at call time
      u64 g = slots[i];
      if (g == 0) { h[i] = 0; continue; }
      Unit *v = devLookup(g);
      if (!v) {
        if (!(flags & REF_LENIENT)) return REF_E_UNREGISTERED;
        h[i] = g;
        continue;
      }
      h[i] = v->base + (g - v->devptr);
      unitBase[i] = v->base;
    }
    int s;
    for (size_t i = 0; i < n; ++i) {
      if (slots[i] == 0) continue;
      if (!unitBase[i]) { st.passthrough += 1; continue; }
      st.rev_translations += 1;
      s = unmap(unitBase[i]);
      if (s) return s;
    }
    if (rel)
      for (size_t i = 0; i < n; ++i)
        if (unitBase[i]) { s = release(unitBase[i]); if (s) return s; }
    std::memcpy(slots, h.data(), n * 8);
    return REF_OK;
  }

  // ---- registration (Table 2) ----------------------------------------
  int declare(u64 b, u64 s, bool isGlobal, bool ro, const char *name) {
    if (b == 0 || s == 0 || b + s < b) return REF_E_INVALID;
    auto succ = table.lower_bound(b);  // first base >= b
    if (succ != table.end() && succ->first < b + s) return REF_E_OVERLAP;
    if (succ != table.begin()) {
      auto pred = std::prev(succ);
      if (pred->first + pred->second.size > b) return REF_E_OVERLAP;
    }
    Unit u;
    u.base = b; u.size = s; u.epoch = globalEpoch;  // A20
    u.isGlobal = isGlobal; u.isReadOnly = ro;
    if (name) u.name = name;
    table.emplace(b, u);
    return REF_OK;
  }
};

template <class F>
int txn(Oracle *o, F f) {  // all-or-nothing wrapper
  o->begin();
  int s = f();
  if (s) o->rollback();
  else o->commit();
  return s;
}

Oracle *O(void *h) { return static_cast<Oracle *>(h); }

}  // namespace

extern "C" {

int ref_groupJoin(void *h, void *leader) {
  Oracle *o = O(h), *l = O(leader);
  if (o->group) return REF_E_INVALID;
  if (!l->group) l->group = std::make_shared<std::vector<Oracle *>>(1, l);
  if (o != l) {
    l->group->push_back(o);
    o->group = l->group;
    o->hostp = l->hostp;
  }
  return REF_OK;
}

void *ref_create(unsigned flags) {
  Oracle *o = new Oracle();
  o->flags = flags;
  return o;
}
void ref_destroy(void *h) {
  Oracle *o = O(h);
  if (o->group) {  // leave the group (destroy the members before the leader, whose host they share)
    auto &g = *o->group;
    g.erase(std::remove(g.begin(), g.end(), o), g.end());
  }
  delete o;
}

int ref_declareAlloc(void *h, uint64_t base, uint64_t size) {
  return O(h)->declare(base, size, false, false, nullptr);
}
int ref_declareAllocFlags(void *h, uint64_t base, uint64_t size, unsigned f) {
  return O(h)->declare(base, size, false, (f & REF_UNIT_READONLY) != 0, nullptr);
}
int ref_declareGlobal(void *h, const char *name, uint64_t base, uint64_t size, int ro) {
  Oracle *o = O(h);
  if (!name || !*name) return REF_E_INVALID;
  if (o->globalNames.count(name)) return REF_E_DUPLICATE;
  int s = o->declare(base, size, true, ro != 0, name);
  if (!s) o->globalNames.insert(name);
  return s;
}
int ref_undeclare(void *h, uint64_t base) {
  Oracle *o = O(h);
  auto it = o->table.find(base);
  if (it == o->table.end()) return REF_E_UNREGISTERED;
  if (it->second.refCount > 0) return REF_E_BUSY;
  if (it->second.isGlobal) o->globalNames.erase(it->second.name);
  o->table.erase(it);
  return REF_OK;
}

int ref_hostWrite(void *h, uint64_t a, const void *s, uint64_t n) { O(h)->host().write(a, s, n); return 0; }
int ref_hostRead(void *h, uint64_t a, void *d, uint64_t n) { O(h)->host().read(a, d, n); return 0; }
int ref_devWrite(void *h, uint64_t a, const void *s, uint64_t n) { O(h)->dev.write(a, s, n); return 0; }
int ref_devRead(void *h, uint64_t a, void *d, uint64_t n) { O(h)->dev.read(a, d, n); return 0; }

int ref_map(void *h, uint64_t p, uint64_t *out) {
  Oracle *o = O(h);
  u64 t = 0;
  int s = txn(o, [&] { return o->map(p, &t); });
  if (!s && out) *out = t;
  return s;
}
int ref_unmap(void *h, uint64_t p) { Oracle *o = O(h); return txn(o, [&] { return o->unmap(p); }); }
int ref_release(void *h, uint64_t p) { Oracle *o = O(h); return txn(o, [&] { return o->release(p); }); }
int ref_mapArray(void *h, uint64_t pp, uint64_t *out) {
  Oracle *o = O(h);
  u64 t = 0;
  int s = txn(o, [&] { return o->mapArray(pp, &t); });
  if (!s && out) *out = t;
  return s;
}
int ref_unmapArray(void *h, uint64_t pp) { Oracle *o = O(h); return txn(o, [&] { return o->unmapArray(pp); }); }
int ref_releaseArray(void *h, uint64_t pp) { Oracle *o = O(h); return txn(o, [&] { return o->releaseArray(pp); }); }
int ref_advanceEpoch(void *h) { O(h)->globalEpoch += 1; return 0; }  // +1 per GPU launch
int ref_advanceEpochs(void *h, uint64_t n) {  // n launches: n times +1; u64 epochs (A20)
  O(h)->globalEpoch += n;
  return 0;
}
uint64_t ref_epoch(void *h) { return O(h)->globalEpoch; }

int ref_mapBatch(void *h, const uint64_t *ps, size_t n, uint64_t *out) {
  Oracle *o = O(h);
  std::vector<u64> t(n);
  int s = txn(o, [&] {
    int r = o->checkLookups(ps, n);
    if (r) return r;
    for (size_t i = 0; i < n; ++i) { r = o->map(ps[i], &t[i]); if (r) return r; }
    return 0;
  });
  if (!s && n) std::memcpy(out, t.data(), n * 8);
  return s;
}
int ref_unmapBatch(void *h, const uint64_t *ps, size_t n) {
  Oracle *o = O(h);
  return txn(o, [&] {
    int r = o->checkLookups(ps, n);
    if (r) return r;
    for (size_t i = 0; i < n; ++i)
      if (ps[i]) { Unit *u = o->lookup(ps[i]); if (u && u->refCount == 0) return (int)REF_E_NOT_MAPPED; }
    for (size_t i = 0; i < n; ++i) { r = o->unmap(ps[i]); if (r) return r; }
    return 0;
  });
}
int ref_releaseBatch(void *h, const uint64_t *ps, size_t n) {
  Oracle *o = O(h);
  return txn(o, [&] {
    int r = o->checkLookups(ps, n);
    if (r) return r;
    for (size_t i = 0; i < n; ++i) { r = o->release(ps[i]); if (r) return r; }
    return 0;
  });
}
int ref_mapArrays(void *h, const uint64_t *pps, size_t k, uint64_t *out) {
  Oracle *o = O(h);
  std::vector<u64> t(k);
  int s = txn(o, [&] {
    for (size_t j = 0; j < k; ++j) { int r = o->mapArray(pps[j], &t[j]); if (r) return r; }
    return 0;
  });
  if (!s && k) std::memcpy(out, t.data(), k * 8);
  return s;
}
int ref_unmapArrays(void *h, const uint64_t *pps, size_t k) {
  Oracle *o = O(h);
  return txn(o, [&] {
    for (size_t j = 0; j < k; ++j) { int r = o->unmapArray(pps[j]); if (r) return r; }
    return 0;
  });
}
int ref_releaseArrays(void *h, const uint64_t *pps, size_t k) {
  Oracle *o = O(h);
  return txn(o, [&] {
    for (size_t j = 0; j < k; ++j) { int r = o->releaseArray(pps[j]); if (r) return r; }
    return 0;
  });
}
int ref_mapSlots(void *h, uint64_t *slots, size_t n) {
  Oracle *o = O(h);
  return txn(o, [&] { return o->mapSlots(slots, n); });
}
int ref_unmapSlots(void *h, uint64_t *slots, size_t n, int release) {
  Oracle *o = O(h);
  return txn(o, [&] { return o->unmapSlots(slots, n, release != 0); });
}

int ref_stats(void *h, ref_stats_t *out) { *out = O(h)->st; return 0; }
int ref_dumpTable(void *h, ref_unit_t *out, size_t cap, size_t *n) {
  Oracle *o = O(h);
  size_t i = 0;
  for (auto &kv : o->table) {
    if (i < cap && out) {
      const Unit &u = kv.second;
      ref_unit_t &r = out[i];
      r.base = u.base; r.size = u.size;
      bool act = u.refCount > 0;
      r.devptr = (act || (u.isGlobal && u.hasStorage)) ? u.devptr : 0;
      r.refCount = u.refCount; r.epoch = u.epoch;
      r.flags = (u.isGlobal ? REF_UNIT_GLOBAL : 0) | (u.isReadOnly ? REF_UNIT_READONLY : 0) |
                (u.arrayMapped ? REF_UNIT_ARRAYMAPPED : 0) | (act ? REF_UNIT_ACTIVE : 0);
      r.pad = 0;
    }
    ++i;
  }
  if (n) *n = i;
  return i <= cap ? 0 : REF_E_NOMEM;
}
int ref_replayDevptr(void *h, uint64_t base, uint64_t devptr) { O(h)->replay[base] = devptr; return 0; }
int ref_lookup(void *h, uint64_t p, uint64_t *base, uint64_t *size) {
  Unit *u = O(h)->lookup(p);
  if (!u) return REF_E_UNREGISTERED;
  *base = u->base; *size = u->size;
  return 0;
}
int ref_devLookup(void *h, uint64_t g, uint64_t *base, uint64_t *devptr) {
  Unit *u = O(h)->devLookup(g);
  if (!u) return REF_E_UNREGISTERED;
  *base = u->base; *devptr = u->devptr;
  return 0;
}

// Glue kernel (NEXT-4; §5.3: a small CPU region "transform[ed] ... into a single-threaded GPU
// function"): the glue program of the C ABI (cgcm_launchGlue), run by one interpreter loop on the
// simulated device.  r[i] = Alg. 1's devptr + (p - base) of cpu_ptrs[i], whose unit must be mapped.
// Every LD/ST of 8 bytes must lie in the device copy of an active unit (devLookup).  Plain C++ doubles
// (round to nearest; the file is compiled with -ffp-contract=off, so no FMA).
int ref_runGlue(void *h, const void *prog_v, size_t n, const uint64_t *ptrs, size_t nptrs, uint64_t max_steps,
                uint64_t *regs_out) {
  struct Op { uint32_t op, dst, a, b; int64_t imm; };
  const Op *prog = static_cast<const Op *>(prog_v);
  Oracle *o = O(h);
  const size_t NR = 32;
  if (nptrs > NR) return REF_E_INVALID;
  u64 r[32] = {0};
  for (size_t i = 0; i < nptrs; ++i) {
    if (ptrs[i] == 0) continue;
    Unit *u = o->lookup(ptrs[i]);
    if (!u) return REF_E_UNREGISTERED;
    if (u->refCount <= 0) return REF_E_NOT_MAPPED;
    r[i] = u->devptr + (ptrs[i] - u->base);
  }
  auto dbl = [](u64 x) { double d; std::memcpy(&d, &x, 8); return d; };
  auto bits = [](double d) { u64 x; std::memcpy(&x, &d, 8); return x; };
  auto inside = [&](u64 g) {  // 8 bytes inside an active unit's device copy
    Unit *v = o->devLookup(g);
    return v && (g % 8) == 0 && g - v->devptr + 8 <= v->size;
  };
  int st = REF_OK;
  u64 steps = 0;
  size_t pc = 0;
  while (pc < n) {
    if (++steps > max_steps) { st = REF_E_INVALID; break; }
    const Op &x = prog[pc];
    if (x.dst >= NR || x.a >= NR || x.b >= NR) { st = REF_E_INVALID; break; }
    size_t next = pc + 1;
    const u64 a = r[x.a], b = r[x.b];
    if (x.op == 1) r[x.dst] = (u64)x.imm;
    else if (x.op == 2) r[x.dst] = a + b;
    else if (x.op == 3) r[x.dst] = a + (u64)x.imm;
    else if (x.op == 4) r[x.dst] = a - b;
    else if (x.op == 5) r[x.dst] = a * b;
    else if (x.op == 6) r[x.dst] = bits(dbl(a) + dbl(b));
    else if (x.op == 7) r[x.dst] = bits(dbl(a) - dbl(b));
    else if (x.op == 8) r[x.dst] = bits(dbl(a) * dbl(b));
    else if (x.op == 9) r[x.dst] = bits(dbl(a) / dbl(b));
    else if (x.op == 10 || x.op == 11) {
      const u64 g = a + (u64)x.imm;
      if (!inside(g)) { st = REF_E_UNREGISTERED; break; }
      if (x.op == 10) r[x.dst] = o->dev.get64(g);
      else o->dev.put64(g, b);
    } else if (x.op == 12) {
      if (x.imm < 0 || (u64)x.imm >= n) { st = REF_E_INVALID; break; }
      if (a != 0) next = (size_t)x.imm;
    } else if (x.op == 13) next = n;
    else { st = REF_E_INVALID; break; }
    pc = next;
  }
  if (regs_out) std::memcpy(regs_out, r, sizeof(r));
  return st;
}

// S1: x *= alpha over a jagged 2-D array reached through its translated row pointers (config A).
int ref_kernel_scale(void *h, uint64_t rows_dev, uint64_t nrows, uint64_t ncols, double alpha) {
  Oracle *o = O(h);
  for (u64 r = 0; r < nrows; ++r) {
    u64 row = o->dev.get64(rows_dev + 8 * r);
    for (u64 c = 0; c < ncols; ++c) {
      double x = o->dev.getf(row + 8 * c);
      o->dev.putf(row + 8 * c, x * alpha);
    }
  }
  return 0;
}

// S3: one bottom-up level of subtree sums (config D).  Node i (32 B: key, val, sum, pad) is
// child[i-1] for i >= 1 and root_dev for i == 0; its children are child[2i], child[2i+1].
// sum = (val + sum(left)) + sum(right), absent children skipped (fixed association, A21).
int ref_kernel_treesum_level(void *h, uint64_t child_dev, uint64_t root_dev, uint64_t nnodes,
                             uint64_t lo, uint64_t hi) {
  Oracle *o = O(h);
  for (u64 i = lo; i < hi && i < nnodes; ++i) {
    u64 node = i == 0 ? root_dev : o->dev.get64(child_dev + 8 * (i - 1));
    u64 l = o->dev.get64(child_dev + 8 * (2 * i)), r = o->dev.get64(child_dev + 8 * (2 * i + 1));
    double s = o->dev.getf(node + 8);
    if (l) s = s + o->dev.getf(l + 16);
    if (r) s = s + o->dev.getf(r + 16);
    o->dev.putf(node + 16, s);
  }
  return 0;
}

// S2: PolyBench-shaped gemm on jagged fp64 matrices (config B), long-double accumulation.
int ref_kernel_gemm_rows(void *h, uint64_t A_rows, uint64_t B_rows, uint64_t C_rows, uint64_t n, uint64_t row0,
                         uint64_t nrows, double alpha, double beta) {
  Oracle *o = O(h);
  std::vector<u64> brow(n);
  for (u64 k = 0; k < n; ++k) brow[k] = o->dev.get64(B_rows + 8 * k);
  for (u64 i = row0; i < row0 + nrows && i < n; ++i) {
    u64 arow = o->dev.get64(A_rows + 8 * i), crow = o->dev.get64(C_rows + 8 * i);
    std::vector<double> a(n);
    o->dev.read(arow, a.data(), 8 * n);
    for (u64 j = 0; j < n; ++j) {
      long double acc = 0.0L;
      for (u64 k = 0; k < n; ++k) acc += (long double)a[k] * (long double)o->dev.getf(brow[k] + 8 * j);
      double c = o->dev.getf(crow + 8 * j);
      o->dev.putf(crow + 8 * j, (double)((long double)alpha * acc + (long double)beta * (long double)c));
    }
  }
  return 0;
}

}  // extern "C"
