// oracle_sanitize_driver.cpp -- TEST INFRASTRUCTURE: drives the CPU oracle (oracle/cgcm_oracle.cpp, compiled
// into this binary) through every entry point family -- declarations, scalar and array maps, batch forms,
// device slots, rollbacks of failing calls, lenient mode, glue programs, coherence groups -- so that
// tests/test_oracle_sanitize.py can run it under -fsanitize=address,undefined.  Exits non-zero on any
// unexpected status; the sanitizers abort on any memory error or undefined behaviour.
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>

#include "../oracle/cgcm_oracle.h"

#define CHECK(x)                                                    \
  do {                                                              \
    if (!(x)) {                                                     \
      std::fprintf(stderr, "check failed: %s (line %d)\n", #x, __LINE__); \
      return 1;                                                     \
    }                                                               \
  } while (0)

struct GlueOp {
  uint32_t op, dst, a, b;
  int64_t imm;
};

static int run(unsigned flags) {
  void *o = ref_create(flags);
  std::vector<uint64_t> rows;
  for (int r = 0; r < 64; ++r) {
    const uint64_t b = 0x100000 + 0x1000ull * r;
    CHECK(ref_declareAlloc(o, b, 256 + 8 * r) == 0);
    std::vector<uint8_t> v(256 + 8 * r, (uint8_t)r);
    ref_hostWrite(o, b, v.data(), v.size());
    rows.push_back(b + 8 * (r % 5));
  }
  const uint64_t pp = 0x900000;
  rows.push_back(0);
  CHECK(ref_declareAlloc(o, pp, 8 * rows.size()) == 0);
  ref_hostWrite(o, pp, rows.data(), 8 * rows.size());
  CHECK(ref_declareAlloc(o, 0x100000 + 8, 8) == REF_E_OVERLAP);
  uint64_t d = 0;
  CHECK(ref_mapArray(o, pp, &d) == 0);
  CHECK(ref_mapArray(o, pp, &d) == 0);
  ref_advanceEpoch(o);
  CHECK(ref_unmapArray(o, pp) == 0);
  CHECK(ref_releaseArray(o, pp) == 0);
  // batch forms, with a failing batch rolled back
  std::vector<uint64_t> ps(rows.begin(), rows.end() - 1), out(ps.size());
  CHECK(ref_mapBatch(o, ps.data(), ps.size(), out.data()) == 0);
  std::vector<uint64_t> bad = ps;
  bad.push_back(0x7777777);
  std::vector<uint64_t> out2(bad.size());
  const int sb = ref_mapBatch(o, bad.data(), bad.size(), out2.data());
  CHECK((flags & REF_LENIENT) ? sb == 0 : sb == REF_E_UNREGISTERED);
  if (sb == 0) CHECK(ref_releaseBatch(o, bad.data(), bad.size()) == 0);
  CHECK(ref_unmapBatch(o, ps.data(), ps.size()) == 0);
  CHECK(ref_releaseBatch(o, ps.data(), ps.size()) == 0);
  CHECK(ref_releaseArray(o, pp) == 0);
  // device slots
  std::vector<uint64_t> slots(ps);
  CHECK(ref_mapSlots(o, slots.data(), slots.size()) == 0);
  ref_advanceEpoch(o);
  CHECK(ref_unmapSlots(o, slots.data(), slots.size(), 1) == 0);
  CHECK(slots == ps);
  // a glue program over a mapped row: sum of its first 4 words into word 5
  uint64_t g = 0;
  CHECK(ref_map(o, 0x100000, &g) == 0);
  GlueOp prog[] = {{10, 1, 0, 0, 0}, {10, 2, 0, 0, 8}, {2, 1, 1, 2, 0}, {11, 0, 0, 1, 40}, {10, 3, 0, 0, 4096}};
  uint64_t ptr = 0x100000, regs[32];
  CHECK(ref_runGlue(o, prog, 4, &ptr, 1, 100, regs) == 0);
  CHECK(ref_runGlue(o, prog, 5, &ptr, 1, 100, regs) == REF_E_UNREGISTERED);
  CHECK(ref_release(o, 0x100000) == 0);
  CHECK(ref_undeclare(o, pp) == 0);
  ref_stats_t st;
  ref_stats(o, &st);
  size_t n = 0;
  ref_dumpTable(o, nullptr, 0, &n);
  std::vector<ref_unit_t> units(n);
  CHECK(ref_dumpTable(o, units.data(), n, &n) == 0);
  for (auto &u : units) CHECK(u.refCount == 0);
  ref_destroy(o);
  return 0;
}

static int run_group() {
  void *a = ref_create(0), *b = ref_create(0);
  CHECK(ref_groupJoin(a, a) == 0 && ref_groupJoin(b, a) == 0);
  for (void *o : {a, b}) CHECK(ref_declareAlloc(o, 0x10000, 64) == 0);
  uint64_t d = 0, v = 7;
  ref_hostWrite(a, 0x10000, &v, 8);
  CHECK(ref_map(a, 0x10000, &d) == 0);
  ref_devWrite(a, d, &v, 8);
  ref_advanceEpoch(a);
  CHECK(ref_map(b, 0x10000, &d) == 0);
  ref_stats_t st;
  ref_stats(b, &st);
  CHECK(st.peer_units == 1);
  CHECK(ref_release(b, 0x10000) == 0 && ref_release(a, 0x10000) == 0);
  ref_destroy(b);
  ref_destroy(a);
  return 0;
}

int main() {
  for (unsigned f : {0u, (unsigned)REF_LITERAL_EPOCH, (unsigned)REF_LENIENT})
    if (run(f)) return 1;
  if (run_group()) return 1;
  std::puts("oracle sanitize driver: ok");
  return 0;
}
