// ce_run.h -- builder of the copy-engine copies of a dispatch round (host
// logic only: engine.cpp issues each finished run as one cudaMemcpyAsync or
// cudaMemcpy2DAsync; tests/c/ce_run_test.cpp pins the rules on the CPU).
#pragma once

#include <cstdint>

namespace gr {

// Copy-engine runs of a round: contiguous chunks become ONE copy, and chunks
// of equal size at a constant source and destination stride -- a route's
// share of an interleaved plan (R4: chunk i of route r sits Σ_routes c
// after chunk i-1), whose source AND destination are strided alike when the
// route's copy engine writes the destination directly (its own chunks, or
// GROUTER_CE_RELAY) -- become ONE 2-D copy (cudaMemcpy2DAsync).  Each copy
// costs the engine ~3 us of setup (tools/ce2.cu, probe), so five 2 MiB
// chunks per round copied one by one cost a relayed link ~8% of its rate.
// A 2-D run never spans two transfers: its pitched source and destination
// ranges must each lie inside one allocation (the transfer's source buffer
// and its destination object), which chunks of unrelated transfers at equal
// spacing would not (spills of equal-sized victims, say).
struct CeRun {
  static constexpr uint64_t kMaxPitch = (1ull << 31) - 1;  // cudaMemcpy2D pitch limit
  uint64_t src = 0, dst = 0, width = 0, height = 0, spitch = 0, dpitch = 0;
  const void *owner = nullptr;  // the transfer of the run's first chunk
  bool add(uint64_t s, uint64_t d, uint64_t n, const void *x) {  // true: absorbed into this run
    if (!height) {
      src = s, dst = d, width = n, height = 1, owner = x;
      return true;
    }
    if (height == 1 && s == src + width && d == dst + width) {
      width += n;
      return true;
    }
    if (n != width || x != owner) return false;
    if (height == 1) {
      if (s <= src || d <= dst) return false;
      const uint64_t sp = s - src, dp = d - dst;
      if (sp < width || dp < width || sp > kMaxPitch || dp > kMaxPitch) return false;
      spitch = sp, dpitch = dp, height = 2;
      return true;
    }
    if (s != src + height * spitch || d != dst + height * dpitch) return false;
    ++height;
    return true;
  }
  bool empty() const { return height == 0; }
};


}  // namespace gr
