// Diagnostic (not product code): SM streaming read-only / write-only / copy
// kernels at several grid sizes, cold data, to see which half of a copy is
// slow on this B200.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ int4 ldg(const int4 *p) {
  int4 r;
  asm volatile("ld.global.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
template <int U>
__global__ void rd(const int4 *__restrict__ s, size_t nv, int *sink) {
  int acc = 0;
  size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += st * U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = (i + u * st < nv) ? ldg(s + i + u * st) : make_int4(0, 0, 0, 0);
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  if (acc == 0x12345678) *sink = acc;
}
template <int U>
__global__ void wr(int4 *__restrict__ d, size_t nv) {
  size_t st = (size_t)gridDim.x * blockDim.x;
  int4 z = make_int4(threadIdx.x, 1, 2, 3);
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += st * U)
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (i + u * st < nv) d[i + u * st] = z;
}
template <int U>
__global__ void cp(int4 *__restrict__ d, const int4 *__restrict__ s, size_t nv) {
  size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += st * U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) if (i + u * st < nv) v[u] = ldg(s + i + u * st);
#pragma unroll
    for (int u = 0; u < U; ++u) if (i + u * st < nv) d[i + u * st] = v[u];
  }
}

int main() {
  const size_t sizes[] = {38535168, 268435456};
  int *sink;
  cudaMalloc(&sink, 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (size_t n : sizes) {
    int nbuf = (int)(1536ull * 1024 * 1024 / n) + 2;
    if (nbuf > 40) nbuf = 40;
    std::vector<int4 *> bufs(nbuf);
    for (auto &p : bufs) { cudaMalloc(&p, n); cudaMemset(p, 1, n); }
    size_t nv = n / 16;
    for (int ctas : {148, 296, 592, 1184, 2368}) {
      for (int kind = 0; kind < 4; ++kind) {
        const int reps = 40;
        for (int w = 0; w < 3; ++w) {
          if (kind == 0) rd<8><<<ctas, 256>>>(bufs[w % nbuf], nv, sink);
          else if (kind == 1) wr<8><<<ctas, 256>>>(bufs[w % nbuf], nv);
          else if (kind == 2) cp<8><<<ctas, 256>>>(bufs[(w + 1) % nbuf], bufs[w % nbuf], nv);
          else cudaMemcpyAsync(bufs[(w + 1) % nbuf], bufs[w % nbuf], n, cudaMemcpyDeviceToDevice);
        }
        cudaEventRecord(a);
        for (int r = 0; r < reps; ++r) {
          if (kind == 0) rd<8><<<ctas, 256>>>(bufs[r % nbuf], nv, sink);
          else if (kind == 1) wr<8><<<ctas, 256>>>(bufs[r % nbuf], nv);
          else if (kind == 2) cp<8><<<ctas, 256>>>(bufs[(r + 1) % nbuf], bufs[r % nbuf], nv);
          else cudaMemcpyAsync(bufs[(r + 1) % nbuf], bufs[r % nbuf], n, cudaMemcpyDeviceToDevice);
        }
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        double us = ms * 1e3 / reps;
        double bytes = (kind >= 2 ? 2.0 : 1.0) * n;
        const char *nm[] = {"read", "write", "copy", "memcpy"};
        if (kind == 3 && ctas != 148) continue;
        printf("n=%zu ctas=%d %s us=%.2f TB/s=%.3f\n", n, ctas, nm[kind], us, bytes / us / 1e6);
      }
    }
    for (auto &p : bufs) cudaFree(p);
  }
  return 0;
}
