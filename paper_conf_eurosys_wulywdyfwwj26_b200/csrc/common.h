// common.h -- internal helpers shared by the libgrouter translation units.
//
// The library links cudart statically and reaches the driver API through
// cudaGetDriverEntryPoint, so libgrouter.so loads (and exports its symbols)
// on a machine without libcuda.so.1; nothing touches CUDA before
// grouter_init().
#pragma once

#include <atomic>

#include <cuda.h>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <cstdint>
#include <cstring>
#include <memory>
#include <mutex>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/grouter.h"

namespace gr {

constexpr uint64_t kPage = 2ull << 20;   // R14: 2 MiB pool pages (= VMM granularity)

inline uint64_t charge(uint64_t n) { return (n + kPage - 1) / kPage * kPage; }
inline uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// thread-local last error text (grouter_last_error)
void set_error(const std::string &msg);
const char *last_error();

// An internal failure that maps to a status at the ABI boundary.
struct Error : std::runtime_error {
  grouter_status st;
  Error(grouter_status s, const std::string &m) : std::runtime_error(m), st(s) {}
};

#define GR_CUDA(call)                                                                   \
  do {                                                                                  \
    cudaError_t e_ = (call);                                                            \
    if (e_ != cudaSuccess)                                                              \
      throw ::gr::Error(GROUTER_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

#define GR_CU(call)                                                                     \
  do {                                                                                  \
    CUresult r_ = (call);                                                               \
    if (r_ != CUDA_SUCCESS)                                                             \
      throw ::gr::Error(GROUTER_ECUDA, std::string(#call) + ": CUresult " + std::to_string((int)r_)); \
  } while (0)

// Driver entry points (resolved once, lazily, through the runtime).
struct Driver {
  CUresult (*memCreate)(CUmemGenericAllocationHandle *, size_t, const CUmemAllocationProp *,
                        unsigned long long);
  CUresult (*memRelease)(CUmemGenericAllocationHandle);
  CUresult (*memAddressReserve)(CUdeviceptr *, size_t, size_t, CUdeviceptr, unsigned long long);
  CUresult (*memAddressFree)(CUdeviceptr, size_t);
  CUresult (*memMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
  CUresult (*memUnmap)(CUdeviceptr, size_t);
  CUresult (*memSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc *, size_t);
  CUresult (*memGetAllocationGranularity)(size_t *, const CUmemAllocationProp *,
                                          CUmemAllocationGranularity_flags);
  CUresult (*memExportToShareableHandle)(void *, CUmemGenericAllocationHandle, CUmemAllocationHandleType,
                                         unsigned long long);
  CUresult (*memImportFromShareableHandle)(CUmemGenericAllocationHandle *, void *, CUmemAllocationHandleType);
  CUresult (*streamWaitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
  CUresult (*streamWriteValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
  CUresult (*launchKernelEx)(const CUlaunchConfig *, CUfunction, void **, void **);
};
const Driver &drv();

// NVTX ranges (SURVEY §5 tracing): one per data-path call and one per
// dispatch round / direct launch, in the "grouter" domain, with the bytes as
// payload.  nvtx3 is header-only: without an attached tool (nsys, ncu range
// replay) a push/pop costs a few ns.
nvtxDomainHandle_t nvtx_domain();
struct NvtxRange {
  explicit NvtxRange(const char *name, uint64_t bytes = 0) {
    nvtxEventAttributes_t a = {};
    a.version = NVTX_VERSION;
    a.size = NVTX_EVENT_ATTRIB_STRUCT_SIZE;
    a.messageType = NVTX_MESSAGE_TYPE_ASCII;
    a.message.ascii = name;
    a.payloadType = NVTX_PAYLOAD_TYPE_UNSIGNED_INT64;
    a.payload.ullValue = bytes;
    nvtxDomainRangePushEx(nvtx_domain(), &a);
  }
  ~NvtxRange() { nvtxDomainRangePop(nvtx_domain()); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};

// Saves/restores the caller's current device around library work.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  void set(int dev) {
    int cur = -1;
    cudaGetDevice(&cur);
    if (cur != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

// A pooled CUDA event; returns itself to its pool when the last reference drops.
struct EventPool;
struct Event {
  cudaEvent_t ev = nullptr;
  int phys = -1;
  EventPool *pool = nullptr;
  // completion memo shared by every fence holding this event (an event query
  // costs ~1 us of host time); reset when the pool hands the event out again
  std::atomic<bool> fired{false};
};
using EventRef = std::shared_ptr<Event>;

struct EventPool {
  int phys = -1;
  std::mutex mu;
  std::vector<Event *> free_list;
  EventRef get();                  // caller must have `phys` current
  ~EventPool();
};

struct Xfer;  // ctx.h

// Something the library can wait for: a CUDA event, or a completion word
// (host-mapped u32) reaching a target value (wrap-safe compare, the same
// rule as CU_STREAM_WAIT_VALUE_GEQ).  `epoch` = replay epoch of creation.
struct Waitable {
  EventRef ev;
  volatile uint32_t *word = nullptr;
  uint32_t target = 0;
  uint64_t epoch = 0;
  // transfer whose chunks publish `word`; null when the producing GPU work is
  // already submitted (events, caller-stream signals).  A wait is never
  // enqueued before its producer is submitted (see engine.cpp).
  std::shared_ptr<Xfer> producer;
  // stream the event was recorded on (events only): fences of one stream
  // complete in order, so a newer one stands for the older ones
  cudaStream_t origin = nullptr;
  bool done() const {
    if (word) return (int32_t)(*word - target) >= 0;
    if (ev) {
      if (ev->fired.load(std::memory_order_relaxed)) return true;
      if (cudaEventQuery(ev->ev) != cudaSuccess) return false;
      ev->fired.store(true, std::memory_order_relaxed);
      return true;
    }
    return true;
  }
};

// Appends w to a fence list, replacing the last entry when both are events of
// the same stream (the newer completes after the older).
inline void push_fence(std::vector<Waitable> &f, const Waitable &w) {
  if (!w.ev && !w.word) return;  // the completed fence (an idle stream's point)
  if (!f.empty() && w.ev && !w.word && f.back().ev && !f.back().word && w.origin && f.back().origin == w.origin)
    f.back() = w;
  else
    f.push_back(w);
}
using Fences = std::vector<Waitable>;

// Drops completed fences (keeps long-lived objects' reader lists short).
inline void prune(Fences &f) {
  size_t w = 0;
  for (size_t i = 0; i < f.size(); ++i)
    if (!f[i].done()) {
      if (w != i) f[w] = std::move(f[i]);
      ++w;
    }
  f.resize(w);
}

// GROUTER_HOST_PROFILE=1: per-stage host time of the data-path calls,
// printed to stderr at grouter_finalize (tuning aid).
struct HostProf {
  bool on = false;
  uint64_t calls = 0, put_calls = 0;
  uint64_t rounds[2] = {};  // SM-copy rounds, copy-engine rounds (H2D and D2H) timed in t[19], t[20]
  double t[24] = {};  // [0..7] get_into stages, [8..15] blocking put stages, [16..18] put -> H2D copy,
                     // [19..23] dispatch rounds: host ns / count per server kind (copy, h2d, d2h) and relayed chunks
};
HostProf &hprof();
uint64_t now_ns();
extern thread_local uint64_t tl_put_t0;  // profiling: start of the current blocking put

}  // namespace gr
