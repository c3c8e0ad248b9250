// Diagnostic (not product code): does splitting a 38.5 MB pinned H2D into
// 10 MiB batch copies (the O8 preemption granularity) cost link time, and do
// two copy-engine streams used alternately hide the per-copy setup?  Per
// pattern: back-to-back GB/s over 40 puts and the single-put latency.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 tools/ce2.cu -lcuda -o tools/ce2
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <vector>

int main() {
  const size_t n = 38535168, batch = 10u << 20;
  void *h, *d;
  cudaHostAlloc(&h, n, cudaHostAllocPortable);
  cudaMalloc(&d, n);
  cudaStream_t s[3];
  for (auto &x : s) cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking);
  cudaEvent_t a, b, j;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventCreateWithFlags(&j, cudaEventDisableTiming);
  std::vector<cudaEvent_t> evs(8);
  for (auto &e : evs) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  unsigned int *word;
  cudaHostAlloc(&word, 64, cudaHostAllocMapped);
  CUdeviceptr dword;
  cudaHostGetDevicePointer((void **)&dword, word, 0);
  static unsigned int seq = 0;
  auto put = [&](int mode) {
    if (mode == 0) {
      cudaMemcpyAsync(d, h, n, cudaMemcpyHostToDevice, s[0]);
      return;
    }
    int k = 0;
    for (size_t off = 0; off < n; off += batch, ++k) {
      size_t len = std::min(batch, n - off);
      cudaStream_t st = mode == 2 ? s[k & 1] : s[0];
      cudaMemcpyAsync((char *)d + off, (char *)h + off, len, cudaMemcpyHostToDevice, st);
      if (mode == 3) cudaEventRecord(evs[k & 7], st);           // the library's per-round event
      if (mode == 4) cuStreamWriteValue32(st, dword, ++seq, 0);  // or a completion word
      if (mode == 5) cuStreamWriteValue32(st, dword, ++seq, CU_STREAM_WRITE_VALUE_NO_MEMORY_BARRIER);
      if (mode == 6) {  // the word written from a side stream after an event (the CE stream runs on)
        cudaEventRecord(evs[k & 7], st);
        cudaStreamWaitEvent(s[2], evs[k & 7], 0);
        cuStreamWriteValue32(s[2], dword, ++seq, 0);
      }
    }
    if (mode == 2) {  // join the second stream back into the first
      cudaEventRecord(j, s[1]);
      cudaStreamWaitEvent(s[0], j, 0);
    }
  };
  const char *names[] = {"1 copy of 38.5 MB", "4 x 10 MiB, one stream", "4 x 10 MiB, two streams alternating",
                         "4 x 10 MiB, event after each", "4 x 10 MiB, stream write after each",
                         "4 x 10 MiB, write (no barrier) after each", "4 x 10 MiB, event + side-stream write"};
  for (int mode = 0; mode < 7; ++mode) {
    for (int i = 0; i < 3; ++i) put(mode);
    cudaDeviceSynchronize();
    cudaEventRecord(a, s[0]);
    for (int i = 0; i < 40; ++i) put(mode);
    cudaEventRecord(b, s[0]);
    cudaEventSynchronize(b);
    cudaDeviceSynchronize();
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    std::vector<double> lat;
    for (int i = 0; i < 100; ++i) {
      cudaDeviceSynchronize();
      auto t0 = std::chrono::steady_clock::now();
      put(mode);
      cudaStreamSynchronize(s[0]);
      lat.push_back(std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count());
    }
    std::sort(lat.begin(), lat.end());
    printf("%-40s b2b %7.2f GB/s  %8.1f us/put | single p50 %8.1f us\n", names[mode], 40.0 * n / (ms * 1e6),
           ms * 1e3 / 40, lat[50]);
  }
  return 0;
}
