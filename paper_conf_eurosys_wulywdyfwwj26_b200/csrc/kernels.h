// kernels.h -- host-side launch interface of the sm_100a data-movement kernels.
//
// gr_copy (SURVEY K2'/K4'): one launch moves a whole dispatch ROUND -- a list
// of chunks in stride order (L229) -- with one of three engines (kernels.cu:
// wv8 / tmas4 split the round statically over warps / CTAs, ldst8 claims
// tiles from a ticket in device scratch).  The same
// kernel is the NVLink D2D push (dst = peer VA), the same-GPU HBM copy, and
// the relay forward hop of striped host->GPU transfers (src = staging slot
// on the route GPU, dst = lease on the destination).  When the last CTA
// finishes it publishes per-(transfer, path) completion values with
// system-scope release stores (L182 "synchronization primitives ensuring
// in-order delivery": consumers see nothing until the whole payload landed).
#pragma once

#include <cstdint>

namespace gr {

constexpr int kMaxRoundChunks = 128;
constexpr int kMaxPublish = 64;

struct KChunk {
  uint64_t src, dst, bytes;
};
struct KPublish {
  uint64_t word;   // address of a u32 completion word (host-mapped or device)
  uint32_t value;
  uint32_t pad;
};

constexpr uint32_t kFlagPdl = 1;        // launched with programmatic stream serialization
constexpr uint32_t kFlagLocalDst = 2;   // every destination is in this GPU's memory
constexpr uint32_t kFlagNoPublish = 4;  // completion written by the host after the launch
constexpr uint32_t kFlagLocalSrc = 8;   // every source is in this GPU's memory (L2 prefetch is safe)
constexpr uint32_t kPfShift = 8;        // flags >> kPfShift & 0xff: units per warp prefetched to L2

// Kernel parameters (passed by value, __grid_constant__).  Two capacities:
// the large one for rounds with many distinct chunks, a small one (a few
// hundred bytes -- cheaper to launch) for the common round whose chunks
// coalesce into a handful of contiguous runs.
template <int C, int P>
struct KParams {
  static constexpr int kChunks = C, kPubs = P;
  uint32_t n_chunks = 0, n_pub = 0;
  uint32_t tile_log2 = 16;
  uint32_t flags = 0;            // kFlag* below
  uint32_t *scratch = nullptr;   // [0] tile ticket, [1] finished CTAs; zero between launches
  uint32_t *counts = nullptr;    // test only: bytes written per 16 B granule
  uint64_t count_base = 0;
  // GROUTER_PROFILE: [0] = earliest CTA start, [1] = latest CTA end, in
  // %globaltimer ns (device memory; the kernel's own duration, independent of
  // the host's submission timing); null otherwise
  unsigned long long *stamp = nullptr;
  uint64_t tile_prefix[C + 1] = {};
  KChunk chunk[C];
  KPublish pub[P];
};
using CopyParams = KParams<kMaxRoundChunks, kMaxPublish>;   // host-side builder
using SmallParams = KParams<8, 8>;

// Launch gr_copy on `stream` (current device must own the stream).  grid =
// min(tiles, sm_count * ctas_per_sm).  Returns cudaError_t as int.  When
// `host_publish` is non-null and the engine chosen has static work
// assignment (no ticket scratch to reset), the kernel skips its completion
// protocol and *host_publish = true: the CALLER must publish p.pub with
// stream writes right after the launch on the same stream.
// GROUTER_HOST_PROFILE tuning aid: host ns inside launch_copy
// [0] before the launch call, [1] the launch call, [2] cudaGetLastError.
extern double g_launch_prof[3];
extern uint64_t g_launch_prof_n;
extern bool g_launch_prof_on;
void launch_prof_percentiles(double *p10, double *p50, double *p90);  // us, launch call

int launch_copy(CopyParams &p, int sm_count, int ctas_per_sm, bool tma, void *stream,
                bool *host_publish = nullptr);

}  // namespace gr
