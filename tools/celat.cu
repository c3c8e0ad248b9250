// Diagnostic (not product code): latency of a small pinned H2D / D2H copy on
// an idle copy-engine stream with different completion mechanisms, host-timed
// (call -> the host knows the bytes landed).  Decides how blocking cFn puts /
// gets complete.  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 tools/celat.cu -lcuda -o tools/celat
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdint>
#include <vector>

static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  cudaSetDevice(0);
  cudaFree(0);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  const size_t maxn = 4 << 20;
  void *h, *d;
  cudaHostAlloc(&h, maxn, cudaHostAllocPortable | cudaHostAllocMapped);
  cudaMalloc(&d, maxn);
  volatile uint32_t *word;
  cudaHostAlloc((void **)&word, 64, cudaHostAllocPortable | cudaHostAllocMapped);
  *word = 0;
  cudaEvent_t ev, evb;
  cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&evb, cudaEventDisableTiming | cudaEventBlockingSync);
  uint32_t val = 0;
  const char *names[] = {"memcpy+streamSync", "memcpy+event+eventSync", "memcpy+event+query-spin",
                         "memcpy+writeValue+poll", "memcpy+writeValue+event+poll (current)",
                         "memcpy+hostFunc? (skip)", "cuMemcpyHtoDAsync+event+query-spin",
                         "memcpy only (host call cost)", "event record only", "writeValue only"};
  for (size_t n : {size_t(4096), size_t(65536), size_t(262144), size_t(1) << 20}) {
    for (int dir = 0; dir < 2; ++dir) {
      cudaMemcpyKind k = dir == 0 ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost;
      void *dst = dir == 0 ? d : h;
      void *src = dir == 0 ? h : d;
      for (int mode = 0; mode < 10; ++mode) {
        if (mode == 5) continue;
        std::vector<double> ts;
        for (int it = 0; it < 400; ++it) {
          cudaStreamSynchronize(s);
          double t0 = now_us();
          switch (mode) {
            case 0:
              cudaMemcpyAsync(dst, src, n, k, s);
              cudaStreamSynchronize(s);
              break;
            case 1:
              cudaMemcpyAsync(dst, src, n, k, s);
              cudaEventRecord(ev, s);
              cudaEventSynchronize(ev);
              break;
            case 2:
              cudaMemcpyAsync(dst, src, n, k, s);
              cudaEventRecord(ev, s);
              while (cudaEventQuery(ev) != cudaSuccess) {
              }
              break;
            case 3:
              cudaMemcpyAsync(dst, src, n, k, s);
              ++val;
              cuStreamWriteValue32((CUstream)s, (CUdeviceptr)(uintptr_t)word, val, 0);
              while ((int32_t)(*word - val) < 0) {
              }
              break;
            case 4:
              cudaMemcpyAsync(dst, src, n, k, s);
              ++val;
              cuStreamWriteValue32((CUstream)s, (CUdeviceptr)(uintptr_t)word, val, 0);
              cudaEventRecord(ev, s);
              while ((int32_t)(*word - val) < 0) {
              }
              break;
            case 6:
              if (dir == 0) cuMemcpyHtoDAsync((CUdeviceptr)d, h, n, (CUstream)s);
              else cuMemcpyDtoHAsync(h, (CUdeviceptr)d, n, (CUstream)s);
              cudaEventRecord(ev, s);
              while (cudaEventQuery(ev) != cudaSuccess) {
              }
              break;
            case 7:
              cudaMemcpyAsync(dst, src, n, k, s);
              break;
            case 8:
              cudaEventRecord(ev, s);
              break;
            case 9:
              ++val;
              cuStreamWriteValue32((CUstream)s, (CUdeviceptr)(uintptr_t)word, val, 0);
              break;
          }
          ts.push_back(now_us() - t0);
        }
        std::sort(ts.begin(), ts.end());
        printf("%s n=%zu %-45s p10 %6.2f p50 %6.2f p90 %6.2f us\n", dir ? "D2H" : "H2D", n, names[mode], ts[40],
               ts[200], ts[360]);
      }
    }
  }
  // VMM destination (how the pool maps its pages) vs cudaMalloc: host cost of
  // the memcpy call and the full latency
  {
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    prop.location.id = 0;
    prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    size_t gran = 0;
    cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_MINIMUM);
    size_t sz = 64 << 20;
    CUdeviceptr va;
    cuMemAddressReserve(&va, 2 * sz, 0, 0, 0);
    CUmemGenericAllocationHandle hd;
    cuMemCreate(&hd, sz, &prop, 0);
    cuMemMap(va, sz, 0, hd, 0);
    CUmemAccessDesc acc = {};
    acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc.location.id = 0;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    cuMemSetAccess(va, sz, &acc, 1);
    for (int dst_kind = 0; dst_kind < 2; ++dst_kind) {
      for (int dir = 0; dir < 2; ++dir) {
        void *dv = dst_kind ? (void *)va : d;
        std::vector<double> tc, tl;
        for (int it = 0; it < 400; ++it) {
          cudaStreamSynchronize(s);
          double t0 = now_us();
          if (dir == 0) cudaMemcpyAsync(dv, h, 4096, cudaMemcpyHostToDevice, s);
          else cudaMemcpyAsync(h, dv, 4096, cudaMemcpyDeviceToHost, s);
          double t1 = now_us();
          cudaEventRecord(ev, s);
          while (cudaEventQuery(ev) != cudaSuccess) {
          }
          tc.push_back(t1 - t0);
          tl.push_back(now_us() - t0);
        }
        std::sort(tc.begin(), tc.end());
        std::sort(tl.begin(), tl.end());
        printf("%s 4096 dst=%s memcpy call p50 %.2f p90 %.2f, total p50 %.2f us\n", dir ? "D2H" : "H2D",
               dst_kind ? "VMM" : "cudaMalloc", tc[200], tc[360], tl[200]);
      }
    }
    // the same with cudaMemcpyDefault kind and with the driver API
    std::vector<double> tc;
    for (int it = 0; it < 400; ++it) {
      cudaStreamSynchronize(s);
      double t0 = now_us();
      cuMemcpyHtoDAsync(va, h, 4096, (CUstream)s);
      tc.push_back(now_us() - t0);
    }
    std::sort(tc.begin(), tc.end());
    printf("H2D 4096 dst=VMM cuMemcpyHtoDAsync call p50 %.2f\n", tc[200]);
    int lo, hi;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStream_t sp;
    cudaStreamCreateWithPriority(&sp, cudaStreamNonBlocking, hi);
    for (int dst_kind = 0; dst_kind < 2; ++dst_kind) {
      std::vector<double> tc2, tl2;
      void *dv = dst_kind ? (void *)va : d;
      for (int it = 0; it < 400; ++it) {
        cudaStreamSynchronize(sp);
        double t0 = now_us();
        cudaMemcpyAsync(dv, h, 4096, cudaMemcpyHostToDevice, sp);
        double t1 = now_us();
        cudaEventRecord(ev, sp);
        while (cudaEventQuery(ev) != cudaSuccess) {
        }
        tc2.push_back(t1 - t0);
        tl2.push_back(now_us() - t0);
      }
      std::sort(tc2.begin(), tc2.end());
      std::sort(tl2.begin(), tl2.end());
      printf("H2D 4096 high-priority stream dst=%s memcpy call p50 %.2f, total p50 %.2f us\n",
             dst_kind ? "VMM" : "cudaMalloc", tc2[200], tl2[200]);
    }
  }
  return 0;
}
