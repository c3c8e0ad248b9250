// Diagnostic (not product code): blocking cFn put / get of small objects
// through libgrouter from a plain C++ process (no Python, no torch), to split
// the library's host path from the binding's.  Build:
//   g++ -O2 -std=c++17 -I include tools/putlat.cpp -o tools/putlat \
//       -L paper_conf_eurosys_wulywdyfwwj26_b200 -lgrouter -Wl,-rpath,'$ORIGIN/../paper_conf_eurosys_wulywdyfwwj26_b200' \
//       -L /usr/local/cuda/lib64 -lcudart
// Run with GROUTER_HOST_PROFILE=1 for the per-stage split.
#include <cuda_runtime.h>

#include <algorithm>
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
  cfg.n_gpus = 1;
  cfg.device_map[0] = 0;
  cfg.host_store_bytes = 64 << 20;
  cfg.pool_cap_bytes[0] = 0;
  grouter_ctx *ctx = nullptr;
  if (grouter_init(&cfg, &ctx) != GROUTER_OK) {
    printf("init failed: %s\n", grouter_last_error());
    return 1;
  }
  void *h = nullptr;
  cudaHostAlloc(&h, 4 << 20, cudaHostAllocPortable);
  grouter_fn cfn{1, 1, GROUTER_HOST};
  for (size_t n : {size_t(4096), size_t(262144)}) {
    std::vector<double> tp, tg;
    for (int i = 0; i < 600; ++i) {
      grouter_oid oid = 0;
      double t0 = now_us();
      if (grouter_put(ctx, &cfn, h, n, 0, 0, nullptr, &oid) != GROUTER_OK) {
        printf("put failed: %s\n", grouter_last_error());
        return 1;
      }
      double t1 = now_us();
      const void *p = nullptr;
      uint64_t nn = 0;
      grouter_get(ctx, &cfn, oid, nullptr, &p, &nn);
      double t2 = now_us();
      grouter_release(ctx, &cfn, oid, p, nullptr);
      grouter_free(ctx, &cfn, oid);
      if (i >= 100) {
        tp.push_back(t1 - t0);
        tg.push_back(t2 - t1);
      }
    }
    std::sort(tp.begin(), tp.end());
    std::sort(tg.begin(), tg.end());
    printf("C++ n=%zu put H2D blocking p10 %.2f p50 %.2f us; get D2H blocking p10 %.2f p50 %.2f us\n", n,
           tp[50], tp[250], tg[50], tg[250]);
  }
  grouter_finalize(ctx);
  return 0;
}
