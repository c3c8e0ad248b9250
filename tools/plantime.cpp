// Diagnostic (not product code): host cost of grouter_plan on an 8-GPU HGX
// calibration (R(0) = 4 routes), first call (the exact O6 split) vs repeated
// calls (cached).  Runs without a GPU (GROUTER_PLAN_ONLY).  Build:
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/plantime.cpp -o tools/plantime \
//       -L paper_conf_eurosys_wulywdyfwwj26_b200 -l:libgrouter.so \
//       -Wl,-rpath,'$ORIGIN/../paper_conf_eurosys_wulywdyfwwj26_b200'
#include <chrono>
#include <cstdio>
#include <vector>

#include "grouter.h"

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  grouter_config cfg;
  grouter_config_default(&cfg);
  cfg.n_gpus = 8;
  for (int i = 0; i < 8; ++i) {
    cfg.device_map[i] = i;
    cfg.h2d_Bps[i] = 55000000000ull;
    cfg.uplink_group[i] = i / 2;  // two GPUs per PCIe uplink (HGX)
  }
  cfg.flags = GROUTER_PLAN_ONLY;
  grouter_ctx *ctx = nullptr;
  if (grouter_init(&cfg, &ctx) != GROUTER_OK) return 1;
  std::vector<grouter_chunk> out(4096);
  for (uint64_t n : {4096ull, 2097152ull, 38535168ull, 268435456ull, 1073741824ull}) {
    uint64_t k = 0;
    double t0 = now_us();
    grouter_plan(ctx, GROUTER_HOST, 0, n, out.data(), out.size(), &k);
    double first = now_us() - t0;
    t0 = now_us();
    for (int i = 0; i < 1000; ++i) grouter_plan(ctx, GROUTER_HOST, 0, n, out.data(), out.size(), &k);
    const double cached = (now_us() - t0) / 1000;
    t0 = now_us();  // 300 distinct nearby sizes: every call is a cold (exact) split
    for (int i = 1; i <= 300; ++i) grouter_plan(ctx, GROUTER_HOST, 0, n + 4096ull * i, out.data(), out.size(), &k);
    printf("n=%llu: first %.1f us, cold avg %.1f us, cached %.2f us\n", (unsigned long long)n, first,
           (now_us() - t0) / 300, cached);
  }
  grouter_finalize(ctx);
  return 0;
}
