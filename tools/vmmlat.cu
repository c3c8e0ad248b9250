// Diagnostic (not product code): what does growing a VMM pool by one 64 MiB
// segment cost while copies are in flight, and does it block a concurrent
// cudaMemcpyAsync issue from another thread?  (bench sweep put p99: the
// background pre-warm's grow took ~90 ms while a 1 GiB put was streaming.)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 tools/vmmlat.cu -lcuda -o tools/vmmlat
#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <thread>
#include <vector>

static double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main() {
  cudaSetDevice(0);
  cudaFree(0);
  const size_t big = 1ull << 30, seg = 64ull << 20;
  void *h, *d;
  cudaHostAlloc(&h, big, cudaHostAllocPortable);
  cudaMalloc(&d, big);
  cudaStream_t s;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  CUdeviceptr base;
  cuMemAddressReserve(&base, 64 * seg, 2 << 20, 0, 0);
  CUmemAllocationProp prop = {};
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = 0;
  prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  CUmemAccessDesc ad = {};
  ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ad.location.id = 0;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  for (int busy = 0; busy < 2; ++busy) {
    for (int k = 0; k < 4; ++k) {
      const int i = busy * 4 + k;
      if (busy) {  // 10 MiB batches back to back, like the H2D server (~20 ms of copies)
        for (size_t off = 0; off < big; off += 10u << 20)
          cudaMemcpyAsync((char *)d + off, (char *)h + off, std::min<size_t>(10u << 20, big - off),
                          cudaMemcpyHostToDevice, s);
      }
      std::atomic<double> issue_ms{0};
      std::thread other([&] {  // a concurrent copy issue (the dispatcher) during the grow
        std::this_thread::sleep_for(std::chrono::microseconds(200));
        double t = now_ms();
        cudaMemcpyAsync(d, h, 4096, cudaMemcpyHostToDevice, s);
        issue_ms = now_ms() - t;
      });
      CUmemGenericAllocationHandle hd;
      double t0 = now_ms();
      cuMemCreate(&hd, seg, &prop, 0);
      double t1 = now_ms();
      cuMemMap(base + i * seg, seg, 0, hd, 0);
      double t2 = now_ms();
      cuMemSetAccess(base + i * seg, seg, &ad, 1);
      double t3 = now_ms();
      other.join();
      cudaStreamSynchronize(s);
      printf("%s create %7.2f ms  map %6.2f ms  setAccess %7.2f ms  | concurrent memcpy issue %7.2f ms\n",
             busy ? "copies in flight" : "idle            ", t1 - t0, t2 - t1, t3 - t2, issue_ms.load());
    }
  }
  return 0;
}
