// CPU pin of the copy-engine run builder (csrc/ce_run.h): which chunk lists
// become one 1-D copy, one 2-D copy, or several copies.  Expected runs are
// written out by hand from the rules in ce_run.h (R4 interleaved layout).
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../../paper_conf_eurosys_wulywdyfwwj26_b200/csrc/ce_run.h"

struct Item { uint64_t src, dst, n; int x; };
struct Copy { uint64_t src, dst, width, height, spitch, dpitch; };

static std::vector<Copy> build(const std::vector<Item> &items) {
  std::vector<Copy> out;
  gr::CeRun r;
  auto flush = [&] {
    if (r.empty()) return;
    out.push_back({r.src, r.dst, r.width, r.height, r.height > 1 ? r.spitch : 0, r.height > 1 ? r.dpitch : 0});
    r.height = 0;
  };
  static int tag[64];
  for (auto &it : items)
    if (!r.add(it.src, it.dst, it.n, &tag[it.x])) {
      flush();
      r.add(it.src, it.dst, it.n, &tag[it.x]);
    }
  flush();
  return out;
}

static int fails = 0;
static void expect(const char *what, const std::vector<Item> &items, const std::vector<Copy> &want) {
  const std::vector<Copy> got = build(items);
  bool ok = got.size() == want.size();
  for (size_t i = 0; ok && i < got.size(); ++i)
    ok = got[i].src == want[i].src && got[i].dst == want[i].dst && got[i].width == want[i].width &&
         got[i].height == want[i].height && got[i].spitch == want[i].spitch && got[i].dpitch == want[i].dpitch;
  printf("%s: %s (%zu copies)\n", what, ok ? "ok" : "MISMATCH", got.size());
  if (!ok) {
    ++fails;
    for (auto &c : got)
      printf("  got src %llu dst %llu w %llu h %llu sp %llu dp %llu\n", (unsigned long long)c.src,
             (unsigned long long)c.dst, (unsigned long long)c.width, (unsigned long long)c.height,
             (unsigned long long)c.spitch, (unsigned long long)c.dpitch);
  }
}

int main() {
  const uint64_t M = 1 << 20, C = 2 * M;
  // one route, contiguous 2 MiB chunks of one transfer: one 1-D copy of 10 MiB
  expect("contiguous", {{0, 1000, C, 0}, {C, 1000 + C, C, 0}, {2 * C, 1000 + 2 * C, C, 0},
                        {3 * C, 1000 + 3 * C, C, 0}, {4 * C, 1000 + 4 * C, C, 0}},
         {{0, 1000, 5 * C, 1, 0, 0}});
  // route 1 of 4 equal routes (interleaved layout): chunks 1, 5, 9 -> one 2-D copy, pitch 4C both sides
  expect("interleaved route", {{1 * C, 7 + 1 * C, C, 0}, {5 * C, 7 + 5 * C, C, 0}, {9 * C, 7 + 9 * C, C, 0}},
         {{C, 7 + C, C, 3, 4 * C, 4 * C}});
  // the route's last chunk is short: it ends the 2-D run and goes alone
  expect("ragged tail", {{C, 0, C, 0}, {5 * C, 4 * C, C, 0}, {9 * C, 8 * C, 12345, 0}},
         {{C, 0, C, 2, 4 * C, 4 * C}, {9 * C, 8 * C, 12345, 1, 0, 0}});
  // equal chunks of TWO transfers at equal spacing (spills of equal victims): never one 2-D copy
  expect("two transfers", {{0, 0, C, 0}, {3 * C, 3 * C, C, 1}, {6 * C, 6 * C, C, 1}},
         {{0, 0, C, 1, 0, 0}, {3 * C, 3 * C, C, 2, 3 * C, 3 * C}});
  // a stride that breaks (third chunk not at src + 2 * pitch): the run ends there
  expect("broken stride", {{0, 0, C, 0}, {4 * C, 4 * C, C, 0}, {9 * C, 8 * C, C, 0}},
         {{0, 0, C, 2, 4 * C, 4 * C}, {9 * C, 8 * C, C, 1, 0, 0}});
  // source strided, destination contiguous (the staging ring): a 2-D copy with dpitch = width
  expect("strided to contiguous", {{0, 500, C, 0}, {3 * C, 500 + C, C, 0}, {6 * C, 500 + 2 * C, C, 0}},
         {{0, 500, C, 3, 3 * C, C}});
  // overlapping rows (pitch below the width) or going backwards: separate copies
  expect("backwards", {{4 * C, 4 * C, C, 0}, {0, 0, C, 0}}, {{4 * C, 4 * C, C, 1, 0, 0}, {0, 0, C, 1, 0, 0}});
  // a pitch above the 2-D copy limit (2^31 - 1): separate copies
  expect("pitch limit", {{0, 0, C, 0}, {1ull << 31, 1ull << 31, C, 0}},
         {{0, 0, C, 1, 0, 0}, {1ull << 31, 1ull << 31, C, 1, 0, 0}});
  // contiguous growth first, then an equal-width row cannot follow a widened run
  expect("1-D then stride", {{0, 0, C, 0}, {C, C, C, 0}, {8 * C, 8 * C, C, 0}},
         {{0, 0, 2 * C, 1, 0, 0}, {8 * C, 8 * C, C, 1, 0, 0}});
  return fails ? 1 : 0;
}
