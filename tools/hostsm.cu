// Diagnostic (not product code): can the SMs move host<->device bytes over
// PCIe as fast as the copy engine, and with less latency for small payloads?
// Decides the small-transfer path and the fused host-read relay.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/hostsm.cu -lcuda -o tools/hostsm
// Bandwidth: back to back, CUDA events, rotating buffers.  Latency: host-timed
// from the call to the host knowing the bytes landed (event spin, or a
// host-mapped flag the kernel's last CTA releases).
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  printf("CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); return 1; } } while (0)

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

__device__ __forceinline__ int4 ld_nc(const int4 *p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ int4 ld_vol(const int4 *p) {
  int4 r;
  asm volatile("ld.volatile.global.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// grid-stride, U 16 B loads in flight per thread
template <int U>
__global__ void __launch_bounds__(256) sm_copy(int4 *__restrict__ d, const int4 *__restrict__ s, size_t nv,
                                               unsigned *flag, unsigned val, unsigned *done) {
  size_t st = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < nv; i += st * U) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (i + u * st < nv) v[u] = ld_nc(s + i + u * st);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (i + u * st < nv) d[i + u * st] = v[u];
  }
  if (flag) {
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence_system();
      unsigned prev = atomicAdd(done, 1u);
      if (prev == gridDim.x - 1) {
        *done = 0;
        __threadfence_system();
        asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(val) : "memory");
      }
    }
  }
}

// per-warp contiguous tiles: warp w takes 8 KiB tile w, w+W, ... ; 16 loads of 16 B per lane
__global__ void __launch_bounds__(256) sm_copy_tiles(int4 *__restrict__ d, const int4 *__restrict__ s, size_t nv) {
  const size_t tile = 512;  // int4s = 8 KiB
  size_t W = (size_t)gridDim.x * 8;
  size_t w = blockIdx.x * 8 + threadIdx.x / 32;
  int lane = threadIdx.x & 31;
  for (size_t t = w; t * tile < nv; t += W) {
    size_t b = t * tile;
    int4 v[16];
#pragma unroll
    for (int u = 0; u < 16; ++u)
      if (b + u * 32 + lane < nv) v[u] = ld_nc(s + b + u * 32 + lane);
#pragma unroll
    for (int u = 0; u < 16; ++u)
      if (b + u * 32 + lane < nv) d[b + u * 32 + lane] = v[u];
  }
}

// TMA bulk ring: one elected thread, S stages of 16 KiB, global(any) -> smem -> global(any)
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
template <int S>
__global__ void __launch_bounds__(32) tma_copy(char *__restrict__ d, const char *__restrict__ s, size_t n) {
  extern __shared__ __align__(128) char buf[];
  __shared__ __align__(8) unsigned long long bar[S];
  const size_t U = 16384;
  if (threadIdx.x != 0) return;
  for (int i = 0; i < S; ++i)
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[i])));
  asm volatile("fence.mbarrier_init.release.cluster;");
  size_t units = (n + U - 1) / U;
  size_t first = blockIdx.x, step = gridDim.x;
  unsigned phase[S] = {0};
  // prologue
  size_t u = first;
  int k = 0;
  for (; k < S && u < units; ++k, u += step) {
    size_t bytes = (u == units - 1) ? n - u * U : U;
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[k])), "r"((unsigned)bytes));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(buf + k * U)), "l"(s + u * U), "r"((unsigned)bytes), "r"(smem_u32(&bar[k])) : "memory");
  }
  size_t cu = first;
  int slot = 0;
  while (cu < units) {
    size_t bytes = (cu == units - 1) ? n - cu * U : U;
    asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared.b64 p, [%0], %1; @!p bra W; }"
                 ::"r"(smem_u32(&bar[slot])), "r"(phase[slot]));
    phase[slot] ^= 1;
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(d + cu * U), "r"(smem_u32(buf + slot * U)), "r"((unsigned)bytes) : "memory");
    asm volatile("cp.async.bulk.commit_group;");
    if (u < units) {
      asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(0) : "memory");
      size_t b2 = (u == units - 1) ? n - u * U : U;
      asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[slot])), "r"((unsigned)b2));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(smem_u32(buf + slot * U)), "l"(s + u * U), "r"((unsigned)b2), "r"(smem_u32(&bar[slot])) : "memory");
      u += step;
    }
    cu += step;
    slot = (slot + 1) % S;
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

struct Bufs {
  std::vector<char *> h, d;
};

int main(int argc, char **argv) {
  CK(cudaSetDevice(0));
  CK(cudaFree(0));
  cudaStream_t s, s2;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  const int NB = 4;
  const size_t MAXN = 256u << 20;
  Bufs B;
  for (int i = 0; i < NB; ++i) {
    char *h, *d;
    CK(cudaHostAlloc((void **)&h, MAXN, cudaHostAllocPortable | cudaHostAllocMapped));
    CK(cudaMalloc(&d, MAXN));
    memset(h, i + 1, MAXN);
    CK(cudaMemset(d, i + 7, MAXN));
    B.h.push_back(h);
    B.d.push_back(d);
  }
  unsigned *flag, *done;
  CK(cudaHostAlloc((void **)&flag, 64, cudaHostAllocPortable | cudaHostAllocMapped));
  CK(cudaMalloc(&done, 64));
  CK(cudaMemset(done, 0, 64));
  *flag = 0;
  cudaEvent_t e0, e1, ev;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  CK(cudaFuncSetAttribute(tma_copy<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 16384));
  CK(cudaFuncSetAttribute(tma_copy<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 16384));

  // ---------------- bandwidth
  auto bw = [&](const char *name, size_t n, int reps, auto &&launch) -> int {
    for (int i = 0; i < 3; ++i) launch(i, n);
    CK(cudaStreamSynchronize(s));
    CK(cudaEventRecord(e0, s));
    for (int i = 0; i < reps; ++i) launch(i, n);
    CK(cudaEventRecord(e1, s));
    CK(cudaEventSynchronize(e1));
    CK(cudaGetLastError());
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    printf("BW %-34s n=%10zu  %8.2f us  %7.2f GB/s\n", name, n, ms * 1e3 / reps, (double)n * reps / (ms * 1e6));
    return 0;
  };
  for (size_t n : {size_t(38535168), size_t(256u << 20)}) {
    int reps = n > (64u << 20) ? 10 : 40;
    bw("CE H2D", n, reps, [&](int i, size_t n) { cudaMemcpyAsync(B.d[i % NB], B.h[i % NB], n, cudaMemcpyHostToDevice, s); });
    bw("CE D2H", n, reps, [&](int i, size_t n) { cudaMemcpyAsync(B.h[i % NB], B.d[i % NB], n, cudaMemcpyDeviceToHost, s); });
    for (int g : {8, 16, 32, 64, 148, 296}) {
      char nm[64];
      snprintf(nm, sizeof nm, "SM H2D ldnc U8 G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], n / 16, nullptr, 0, nullptr); });
      snprintf(nm, sizeof nm, "SM H2D ldnc U4 G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { sm_copy<4><<<g, 256, 0, s>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], n / 16, nullptr, 0, nullptr); });
      snprintf(nm, sizeof nm, "SM H2D tiles8K G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { sm_copy_tiles<<<g, 256, 0, s>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], n / 16); });
      snprintf(nm, sizeof nm, "TMA4 H2D G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { tma_copy<4><<<g, 32, 4 * 16384, s>>>(B.d[i % NB], B.h[i % NB], n); });
      snprintf(nm, sizeof nm, "TMA8 H2D G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { tma_copy<8><<<g, 32, 8 * 16384, s>>>(B.d[i % NB], B.h[i % NB], n); });
      snprintf(nm, sizeof nm, "SM D2H U8 G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.h[i % NB], (const int4 *)B.d[i % NB], n / 16, nullptr, 0, nullptr); });
      snprintf(nm, sizeof nm, "TMA4 D2H G=%d", g);
      bw(nm, n, reps, [&](int i, size_t n) { tma_copy<4><<<g, 32, 4 * 16384, s>>>(B.h[i % NB], B.d[i % NB], n); });
    }
    // CE + SM split of one H2D (does the link have headroom above the CE?)
    for (double f : {0.2, 0.35, 0.5}) {
      char nm[64];
      snprintf(nm, sizeof nm, "CE+SM(G=32) H2D sm=%.2f", f);
      size_t k = (size_t)(n * f) / 4096 * 4096;
      bw(nm, n, reps, [&](int i, size_t n) {
        cudaEventRecord(ev, s);
        cudaStreamWaitEvent(s2, ev, 0);
        sm_copy<8><<<32, 256, 0, s2>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], k / 16, nullptr, 0, nullptr);
        cudaMemcpyAsync(B.d[i % NB] + k, B.h[i % NB] + k, n - k, cudaMemcpyHostToDevice, s);
        cudaEventRecord(ev, s2);
        cudaStreamWaitEvent(s, ev, 0);
      });
    }
  }

  // ---------------- latency (host-timed, call -> host knows)
  unsigned val = 0;
  auto lat = [&](const char *name, size_t n, auto &&one) {
    std::vector<double> ts;
    for (int it = 0; it < 300; ++it) {
      cudaStreamSynchronize(s);
      double t0 = now_us();
      one(it, n);
      double t1 = now_us();
      if (it >= 20) ts.push_back(t1 - t0);
    }
    std::sort(ts.begin(), ts.end());
    printf("LAT %-40s n=%9zu  p50 %7.2f us  p99 %7.2f us\n", name, n, ts[ts.size() / 2], ts[(ts.size() * 99 + 99) / 100 - 1]);
  };
  auto spin_ev = [&]() { cudaEventRecord(ev, s); while (cudaEventQuery(ev) != cudaSuccess) {} };
  auto spin_flag = [&](unsigned v) { while ((int)(*(volatile unsigned *)flag - v) < 0) {} };
  for (size_t n : {size_t(4096), size_t(65536), size_t(262144), size_t(1) << 20, size_t(4) << 20}) {
    lat("CE H2D + event spin", n, [&](int i, size_t n) { cudaMemcpyAsync(B.d[i % NB], B.h[i % NB], n, cudaMemcpyHostToDevice, s); spin_ev(); });
    lat("CE D2H + event spin", n, [&](int i, size_t n) { cudaMemcpyAsync(B.h[i % NB], B.d[i % NB], n, cudaMemcpyDeviceToHost, s); spin_ev(); });
    for (int g : {1, 4, 16, 32, 64}) {
      if ((size_t)g * 256 * 16 > n * 4 && g > 1) continue;
      char nm[64];
      snprintf(nm, sizeof nm, "SM H2D G=%d + event spin", g);
      lat(nm, n, [&](int i, size_t n) { sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], n / 16, nullptr, 0, nullptr); spin_ev(); });
      snprintf(nm, sizeof nm, "SM H2D G=%d + flag poll", g);
      lat(nm, n, [&](int i, size_t n) { ++val; sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.d[i % NB], (const int4 *)B.h[i % NB], n / 16, flag, val, done); spin_flag(val); });
      snprintf(nm, sizeof nm, "SM D2H G=%d + flag poll", g);
      lat(nm, n, [&](int i, size_t n) { ++val; sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.h[i % NB], (const int4 *)B.d[i % NB], n / 16, flag, val, done); spin_flag(val); });
      snprintf(nm, sizeof nm, "SM D2D G=%d + flag poll", g);
      lat(nm, n, [&](int i, size_t n) { ++val; sm_copy<8><<<g, 256, 0, s>>>((int4 *)B.d[(i + 1) % NB], (const int4 *)B.d[i % NB], n / 16, flag, val, done); spin_flag(val); });
    }
    lat("CE D2D + event spin", n, [&](int i, size_t n) { cudaMemcpyAsync(B.d[(i + 1) % NB], B.d[i % NB], n, cudaMemcpyDeviceToDevice, s); spin_ev(); });
    lat("empty kernel + flag poll", n, [&](int i, size_t n) { ++val; sm_copy<8><<<1, 256, 0, s>>>((int4 *)B.d[1], (const int4 *)B.d[0], 0, flag, val, done); spin_flag(val); });
  }
  // correctness spot check of the SM H2D
  sm_copy<8><<<32, 256, 0, s>>>((int4 *)B.d[0], (const int4 *)B.h[2], 38535168 / 16, nullptr, 0, nullptr);
  tma_copy<4><<<32, 32, 4 * 16384, s>>>(B.d[1], B.h[3], 38535168);
  CK(cudaStreamSynchronize(s));
  std::vector<char> chk(38535168);
  CK(cudaMemcpy(chk.data(), B.d[0], chk.size(), cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (char c : chk) bad += c != 3;
  CK(cudaMemcpy(chk.data(), B.d[1], chk.size(), cudaMemcpyDeviceToHost));
  for (char c : chk) bad += c != 4;
  printf("check bad=%zu\n", bad);
  return 0;
}
