// Diagnostic: the library's copy engines through grouter_test_copy, driven
// from C++ (no Python), cold 38.5 MB copies back to back.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -o tools/enginebench tools/enginebench.cu -ldl
#include <dlfcn.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "grouter_testing.h"

int main(int argc, char **argv) {
  void *h = dlopen("paper_conf_eurosys_wulywdyfwwj26_b200/libgrouter.so", RTLD_NOW | RTLD_LOCAL);
  if (!h) { printf("dlopen: %s\n", dlerror()); return 1; }
  auto test_copy = (decltype(&grouter_test_copy))dlsym(h, "grouter_test_copy");
  const size_t n = argc > 1 ? strtoull(argv[1], 0, 0) : 38535168ull;
  const int nbuf = (int)(1536ull << 20) / (int)std::min<size_t>(n, 1ull << 30) + 2 > 40 ? 40 : (int)((1536ull << 20) / n + 2);
  std::vector<char *> b(nbuf);
  for (auto &p : b) { cudaMalloc(&p, n); cudaMemset(p, 1, n); }
  cudaStream_t A;
  cudaStreamCreateWithFlags(&A, cudaStreamNonBlocking);
  cudaEvent_t t0, t1;
  cudaEventCreate(&t0);
  cudaEventCreate(&t1);
  std::vector<grouter_chunk> ch;
  for (size_t o = 0; o < n; o += 2 << 20) ch.push_back({o, std::min<size_t>(2 << 20, n - o), 0, 0});
  const int reps = 200;
  for (int i = 0; i < 10; ++i) test_copy(b[i % nbuf], b[(i + 17) % nbuf], ch.data(), (uint32_t)ch.size(), nullptr, 0, A);
  cudaStreamSynchronize(A);
  cudaEventRecord(t0, A);
  for (int i = 0; i < reps; ++i) test_copy(b[i % nbuf], b[(i + 17) % nbuf], ch.data(), (uint32_t)ch.size(), nullptr, 0, A);
  cudaEventRecord(t1, A);
  cudaEventSynchronize(t1);
  float ms;
  cudaEventElapsedTime(&ms, t0, t1);
  double us = ms * 1e3 / reps;
  printf("engine=%s n=%zu us=%.2f TBps_rw=%.3f\n", getenv("GR_COPY") ? getenv("GR_COPY") : "default", n, us,
         2.0 * n / us / 1e6);
  return 0;
}
