// Diagnostic (not product code): one cold same-GPU copy split between an SM
// grid-stride kernel (stream A) and the copy engine (stream B), fork/join
// with events, back to back.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ int4 ldg(const int4 *p) {
  int4 r;
  asm volatile("ld.global.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__global__ void cp(int4 *__restrict__ d, const int4 *__restrict__ s, size_t nv) {
  size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += st * 8) {
    int4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) if (i + u * st < nv) v[u] = ldg(s + i + u * st);
#pragma unroll
    for (int u = 0; u < 8; ++u) if (i + u * st < nv) d[i + u * st] = v[u];
  }
}
int main() {
  const size_t n = 38535168;
  const int nbuf = 40;
  std::vector<char *> b(nbuf);
  for (auto &p : b) { cudaMalloc(&p, n); cudaMemset(p, 1, n); }
  cudaStream_t A, B;
  cudaStreamCreateWithFlags(&A, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&B, cudaStreamNonBlocking);
  cudaEvent_t t0, t1;
  cudaEventCreate(&t0);
  cudaEventCreate(&t1);
  std::vector<cudaEvent_t> fork(2000), join(2000);
  for (auto &e : fork) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  for (auto &e : join) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
  for (int ctas : {296, 592}) {
    for (double f : {1.0, 0.0, 0.85, 0.75, 0.65, 0.55, 0.45}) {
      size_t k = (size_t)(n * f) / 4096 * 4096;
      const int reps = 200;
      auto one = [&](int i) {
        char *d = b[i % nbuf], *s = b[(i + 17) % nbuf];
        cudaEventRecord(fork[i], A);
        cudaStreamWaitEvent(B, fork[i], 0);
        if (k) cp<<<ctas, 256, 0, A>>>((int4 *)d, (const int4 *)s, k / 16);
        if (k < n) cudaMemcpyAsync(d + k, s + k, n - k, cudaMemcpyDeviceToDevice, B);
        cudaEventRecord(join[i], B);
        cudaStreamWaitEvent(A, join[i], 0);
      };
      for (int i = 0; i < 10; ++i) one(i);
      cudaStreamSynchronize(A);
      cudaEventRecord(t0, A);
      for (int i = 0; i < reps; ++i) one(i);
      cudaEventRecord(t1, A);
      cudaEventSynchronize(t1);
      float ms;
      cudaEventElapsedTime(&ms, t0, t1);
      double us = ms * 1e3 / reps;
      printf("ctas=%d kernel_share=%.2f us=%.2f TBps_rw=%.3f\n", ctas, f, us, 2.0 * n / us / 1e6);
    }
  }
  return 0;
}
