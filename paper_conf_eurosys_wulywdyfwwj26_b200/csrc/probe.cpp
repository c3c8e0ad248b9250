// probe.cpp -- calibration probe (PAPER.md L131, L178:
// GPUs behind one PCIe switch share one link to host memory; L203: the
// topology matrix the path planner consumes).  Everything is measured with
// CUDA events on dedicated streams; results are integers (B/s, ps).
#include <algorithm>
#include <chrono>
#include <cstring>
#include <vector>

#include "../../include/grouter.h"
#include "common.h"

namespace {

struct Dev {
  int ord;
  cudaStream_t s = nullptr;
  void *d = nullptr;
  cudaEvent_t a = nullptr, b = nullptr;
};

double time_h2d(Dev &g, const void *host, uint64_t bytes, int reps) {
  gr::DeviceGuard dg(g.ord);
  GR_CUDA(cudaMemcpyAsync(g.d, host, bytes, cudaMemcpyHostToDevice, g.s));  // warm
  GR_CUDA(cudaEventRecord(g.a, g.s));
  for (int r = 0; r < reps; ++r) GR_CUDA(cudaMemcpyAsync(g.d, host, bytes, cudaMemcpyHostToDevice, g.s));
  GR_CUDA(cudaEventRecord(g.b, g.s));
  GR_CUDA(cudaEventSynchronize(g.b));
  float ms = 0;
  GR_CUDA(cudaEventElapsedTime(&ms, g.a, g.b));
  return ms * 1e-3 / reps;  // seconds per copy
}

}  // namespace

extern "C" grouter_status grouter_probe(grouter_config *cfg, uint64_t probe_bytes) {
  if (!cfg || cfg->n_gpus == 0 || cfg->n_gpus > GROUTER_MAX_GPUS) return GROUTER_EINVAL;
  if (probe_bytes < (4u << 20)) probe_bytes = 256ull << 20;
  const int n = (int)cfg->n_gpus;
  int prev = 0;
  cudaGetDevice(&prev);
  std::vector<Dev> devs(n);
  void *host = nullptr;
  try {
    GR_CUDA(cudaHostAlloc(&host, probe_bytes * 2, cudaHostAllocPortable));
    std::memset(host, 0x5a, probe_bytes * 2);
    for (int i = 0; i < n; ++i) {
      devs[i].ord = cfg->device_map[i];
      gr::DeviceGuard dg(devs[i].ord);
      GR_CUDA(cudaStreamCreateWithFlags(&devs[i].s, cudaStreamNonBlocking));
      GR_CUDA(cudaMalloc(&devs[i].d, probe_bytes));
      GR_CUDA(cudaEventCreate(&devs[i].a));
      GR_CUDA(cudaEventCreate(&devs[i].b));
    }
    // solo bandwidth, per-chunk cost, first-chunk latency
    for (int i = 0; i < n; ++i) {
      const double t_big = time_h2d(devs[i], host, probe_bytes, 4);
      const uint64_t bw = (uint64_t)(probe_bytes / t_big);
      const double t_small = time_h2d(devs[i], host, 4096, 200);            // per-copy overhead
      const double t_2m = time_h2d(devs[i], host, 2ull << 20, 1);          // one chunk, cold-ish
      cfg->h2d_Bps[i] = bw;
      cfg->h2d_alpha_ps[i] = (uint64_t)std::max(0.0, (t_small - 4096.0 / bw) * 1e12);
      cfg->h2d_phi_ps[i] = (uint64_t)std::max(0.0, (t_2m - (double)(2ull << 20) / bw) * 1e12);
    }
    // pairwise concurrent H2D (shared uplinks show no gain)
    for (int i = 0; i < n; ++i) {
      cfg->h2d_pair_Bps[i][i] = cfg->h2d_Bps[i];
      for (int j = i + 1; j < n; ++j) {
        Dev &A = devs[i], &B = devs[j];
        const int reps = 4;
        for (Dev *g : {&A, &B}) {  // both idle before the clock starts
          gr::DeviceGuard dg(g->ord);
          GR_CUDA(cudaStreamSynchronize(g->s));
        }
        auto t0 = std::chrono::steady_clock::now();
        for (Dev *g : {&A, &B}) {
          gr::DeviceGuard dg(g->ord);
          for (int r = 0; r < reps; ++r)
            GR_CUDA(cudaMemcpyAsync(g->d, (char *)host + (g == &B ? probe_bytes : 0), probe_bytes,
                                    cudaMemcpyHostToDevice, g->s));
        }
        for (Dev *g : {&A, &B}) {
          gr::DeviceGuard dg(g->ord);
          GR_CUDA(cudaStreamSynchronize(g->s));
        }
        const double tmax = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        const uint64_t sum = (uint64_t)(2.0 * reps * probe_bytes / tmax);
        cfg->h2d_pair_Bps[i][j] = cfg->h2d_pair_Bps[j][i] = sum;
      }
    }
    // peer access and a D2D peer copy
    uint64_t nvl = 0;
    for (int i = 0; i < n; ++i)
      for (int j = 0; j < n; ++j) {
        int ok = (i == j);
        if (i != j) cudaDeviceCanAccessPeer(&ok, devs[i].ord, devs[j].ord);
        cfg->p2p[i][j] = (uint8_t)(ok != 0);
        if (i != j && ok && nvl == 0 && devs[i].ord != devs[j].ord) {
          gr::DeviceGuard dg(devs[i].ord);
          cudaDeviceEnablePeerAccess(devs[j].ord, 0);
          cudaGetLastError();
          GR_CUDA(cudaMemcpyPeerAsync(devs[j].d, devs[j].ord, devs[i].d, devs[i].ord, probe_bytes, devs[i].s));
          GR_CUDA(cudaEventRecord(devs[i].a, devs[i].s));
          for (int r = 0; r < 4; ++r)
            GR_CUDA(cudaMemcpyPeerAsync(devs[j].d, devs[j].ord, devs[i].d, devs[i].ord, probe_bytes, devs[i].s));
          GR_CUDA(cudaEventRecord(devs[i].b, devs[i].s));
          GR_CUDA(cudaEventSynchronize(devs[i].b));
          float ms = 0;
          GR_CUDA(cudaEventElapsedTime(&ms, devs[i].a, devs[i].b));
          nvl = (uint64_t)(4.0 * probe_bytes / (ms * 1e-3));
        }
      }
    if (nvl) cfg->nvl_Bps = nvl;
    for (int i = 0; i < GROUTER_MAX_GPUS; ++i) cfg->uplink_group[i] = -1;
  } catch (const gr::Error &e) {
    gr::set_error(e.what());
    for (auto &g : devs) {
      gr::DeviceGuard dg(g.ord < 0 ? 0 : g.ord);
      if (g.s) cudaStreamDestroy(g.s);
      if (g.d) cudaFree(g.d);
    }
    if (host) cudaFreeHost(host);
    cudaSetDevice(prev);
    return e.st;
  }
  for (auto &g : devs) {
    gr::DeviceGuard dg(g.ord);
    cudaStreamDestroy(g.s);
    cudaFree(g.d);
    cudaEventDestroy(g.a);
    cudaEventDestroy(g.b);
  }
  cudaFreeHost(host);
  cudaSetDevice(prev);
  return GROUTER_OK;
}
