// Diagnostic (not product code): the library's host-path cost per call from
// plain C++ (no Python): blocking cFn put (H2D) / cFn get (D2H) vs a bare
// cudaMemcpyAsync + completion wait (grouter_test_memcpy), and a gFn's
// same-GPU get_into single call (CUDA events around the call on an idle
// stream) vs a bare cudaMemcpyAsync D2D, per size.  Run with
// GROUTER_HOST_PROFILE=1 for the per-stage split printed at finalize.  Build:
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include tools/libcost.cpp -o tools/libcost \
//       -L paper_conf_eurosys_wulywdyfwwj26_b200 -lgrouter \
//       -Wl,-rpath,'$ORIGIN/../paper_conf_eurosys_wulywdyfwwj26_b200' -L /usr/local/cuda/lib64 -lcudart
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <vector>

#include "grouter.h"
#include "grouter_testing.h"

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
static double p50(std::vector<double> v) {
  std::sort(v.begin(), v.end());
  return v[v.size() / 2];
}

int main(int argc, char **argv) {
  grouter_config cfg;
  grouter_config_default(&cfg);
  cfg.n_gpus = 1;
  cfg.device_map[0] = 0;
  cfg.host_store_bytes = 512ull << 20;
  cfg.pool_cap_bytes[0] = 0;
  grouter_ctx *ctx = nullptr;
  if (grouter_init(&cfg, &ctx) != GROUTER_OK) {
    printf("init failed: %s\n", grouter_last_error());
    return 1;
  }
  const size_t maxn = 64ull << 20;
  void *h = nullptr, *d0 = nullptr, *d1 = nullptr;
  cudaHostAlloc(&h, maxn, cudaHostAllocPortable);
  cudaMalloc(&d0, maxn);
  cudaMalloc(&d1, maxn);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  grouter_fn cfn{1, 1, GROUTER_HOST}, gfn{1, 2, 0};
  const int reps = argc > 1 ? atoi(argv[1]) : 400;
  for (size_t n : {size_t(4096), size_t(65536), size_t(1) << 20, size_t(4) << 20, size_t(38535168)}) {
    std::vector<double> tp, tg, bh, bd, gi, bgi;
    grouter_oid obj = 0;
    grouter_put(ctx, &cfn, h, n, 0, 0, nullptr, &obj);
    for (int i = 0; i < reps + 20; ++i) {
      grouter_oid oid = 0;
      double t0 = now_us();
      if (grouter_put(ctx, &cfn, h, n, 0, 0, nullptr, &oid) != GROUTER_OK) {
        printf("put failed: %s\n", grouter_last_error());
        return 1;
      }
      double t1 = now_us();
      grouter_free(ctx, &cfn, oid);
      const void *p = nullptr;
      uint64_t nn = 0;
      double t2 = now_us();
      grouter_get(ctx, &cfn, obj, nullptr, &p, &nn);
      double t3 = now_us();
      grouter_release(ctx, &cfn, obj, p, nullptr);
      double t4 = now_us();
      grouter_test_memcpy(d0, h, n, nullptr, 1);
      double t5 = now_us();
      grouter_test_memcpy(h, d0, n, nullptr, 1);
      double t6 = now_us();
      cudaStreamSynchronize(s);
      cudaEventRecord(a, s);
      grouter_get_into(ctx, &gfn, obj, (i & 1) ? d1 : d0, n, s, nullptr);
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms_gi = 0;
      cudaEventElapsedTime(&ms_gi, a, b);
      cudaEventRecord(a, s);
      cudaMemcpyAsync((i & 1) ? d1 : d0, (i & 1) ? d0 : d1, n, cudaMemcpyDeviceToDevice, s);
      cudaEventRecord(b, s);
      cudaEventSynchronize(b);
      float ms_b = 0;
      cudaEventElapsedTime(&ms_b, a, b);
      if (i >= 20) {
        tp.push_back(t1 - t0);
        tg.push_back(t3 - t2);
        bh.push_back(t5 - t4);
        bd.push_back(t6 - t5);
        gi.push_back(ms_gi * 1e3);
        bgi.push_back(ms_b * 1e3);
      }
    }
    grouter_free(ctx, &cfn, obj);
    printf("n=%9zu  put %.2f vs bare H2D %.2f | get %.2f vs bare D2H %.2f | get_into %.2f vs memcpy D2D %.2f (us p50)\n",
           n, p50(tp), p50(bh), p50(tg), p50(bd), p50(gi), p50(bgi));
    fflush(stdout);
  }
  grouter_finalize(ctx);
  return 0;
}
