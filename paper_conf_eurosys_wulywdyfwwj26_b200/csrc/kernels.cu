// kernels.cu -- sm_100a data-movement kernels (no tensor cores: pure bytes).
//
// gr_copy (SURVEY K2'/K4', kernels.h) has three engines, chosen per launch
// in launch_copy:
//   * wv8   -- warp-strided, 256-bit LDG/STG over 8 KiB units, L2 prefetch
//              of each warp's first unit before the PDL wait (default);
//   * tmas4 -- static-assignment TMA bulk ring (cp.async.bulk global ->
//              shared -> global, 4 x 16 KiB mbarrier stages, one elected
//              thread per CTA) for large 16 B-aligned local rounds;
//   * ldst8 -- 256-thread tiles claimed from a ticket, 128-bit LD/ST with
//              co-aligned and funnel-shift paths for misaligned user buffers.
// All serve local HBM, peer (NVLink) and host-mapped addresses: the data
// path never interprets bytes.  The round-1 tuning variants (ws/wd/gs, the
// ticketed TMA ring, L2 eviction hints, prefetch-ahead) were measured and
// dropped; their numbers are in DESIGN.md §6 and profiles/r01_*.
#include <cuda_runtime.h>

#include <cstdint>
#include <chrono>
#include <cstdlib>
#include <string>
#include <vector>
#include <algorithm>

#include "../../include/grouter.h"
#include "../../include/grouter_testing.h"
#include "kernels.h"
#include "common.h"

typedef int CUresult_t;

namespace gr {

constexpr int kThreads = 256;
constexpr int kTmaThreads = 32;
constexpr uint32_t kTmaStage = 16384;

// ------------------------------------------------------------------ helpers
__host__ __device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ int4 ld_stream(const int4 *p) {
  int4 r;
  asm volatile("ld.global.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st_stream(int4 *p, const int4 &v) {
  asm volatile("st.global.v4.s32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}
// Programmatic dependent launch (sm_90+): a copy kernel is launched while
// its predecessor on the stream drains; it waits here (before touching any
// memory or its scratch) until the predecessor completed and flushed, and
// lets its own successor launch once its main loop is done.
__device__ __forceinline__ void pdl_wait_raw() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
#define pdl_wait() \
  do {                                   \
    if (p.flags & kFlagPdl) pdl_wait_raw(); \
  } while (0)
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void prefetch_l2(uint64_t addr, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(addr), "r"(bytes) : "memory");
}

__device__ __forceinline__ void st_release_sys(uint64_t addr, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(addr), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// GROUTER_PROFILE stamps: every CTA after its PDL wait, and once all its
// threads are done (p.stamp is grid-uniform, so the barrier is too)
// (separate kernel instantiations: launches without stamps carry no trace of them)
template <bool STAMP, class KP>
__device__ __forceinline__ void stamp_begin(const KP &p) {
  if (STAMP && threadIdx.x == 0) atomicMin(&p.stamp[0], gtimer());
}
template <bool STAMP, class KP>
__device__ __forceinline__ void stamp_end(const KP &p) {
  if (STAMP) {
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(&p.stamp[1], gtimer());
  }
}

template <bool COUNT, class KP>
__device__ __forceinline__ void count_bytes(const KP &p, uint64_t dst_addr, uint32_t nbytes) {
  if (COUNT) atomicAdd(&p.counts[(dst_addr - p.count_base) >> 4], nbytes);
}

// dst[0,len) <- src[0,len), all threads of the CTA; any alignment.
template <bool COUNT, int U, class KP>
__device__ void tile_ldst(const KP &p, uint8_t *dst, const uint8_t *src, uint64_t len) {
  const uint32_t tid = threadIdx.x;
  uintptr_t d = (uintptr_t)dst, s = (uintptr_t)src;
  // head: bytes until dst is 16-aligned
  uint64_t head = (16 - (d & 15)) & 15;
  if (head > len) head = len;
  if (tid < head) {
    dst[tid] = src[tid];
    count_bytes<COUNT>(p, d + tid, 1);
  }
  dst += head;
  src += head;
  len -= head;
  d += head;
  s += head;
  const uint64_t nvec = len >> 4;
  int4 *vd = reinterpret_cast<int4 *>(dst);
  if ((s & 15) == 0) {
    // 8 x 16 B in flight per thread before the first store (32 KiB per
    // CTA pass); tiles are 8-64 KiB, chosen per launch to balance waves
    const int4 *vs = reinterpret_cast<const int4 *>(src);
    uint64_t i = tid;
    for (; i + (U - 1) * kThreads < nvec; i += U * kThreads) {
      int4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ld_stream(vs + i + u * kThreads);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        st_stream(vd + i + u * kThreads, v[u]);
        count_bytes<COUNT>(p, (uint64_t)(vd + i + u * kThreads), 16);
      }
    }
    for (; i < nvec; i += kThreads) {
      st_stream(vd + i, ld_stream(vs + i));
      count_bytes<COUNT>(p, (uint64_t)(vd + i), 16);
    }
  } else {
    // shifted: each aligned 16 B dst word is assembled from two aligned src
    // words; the shift is uniform across the CTA (no divergence).
    const uint32_t r = (uint32_t)(s & 15);
    const uint32_t q = r >> 2, b = (r & 3) * 8;
    const uint4 *as = reinterpret_cast<const uint4 *>(s - r);
    auto shift = [&](const uint4 &lo, const uint4 &hi) {
      uint32_t w[8] = {lo.x, lo.y, lo.z, lo.w, hi.x, hi.y, hi.z, hi.w};
      uint32_t o[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        uint32_t a0, a1;
        switch (q) {  // warp-uniform
          case 0: a0 = w[k]; a1 = w[k + 1]; break;
          case 1: a0 = w[k + 1]; a1 = w[k + 2]; break;
          case 2: a0 = w[k + 2]; a1 = w[k + 3]; break;
          default: a0 = w[k + 3]; a1 = w[k + 4]; break;
        }
        o[k] = b ? __funnelshift_r(a0, a1, b) : a0;
      }
      return make_int4((int)o[0], (int)o[1], (int)o[2], (int)o[3]);
    };
    uint64_t i = tid;
    // 4 output vectors (8 aligned loads) in flight per thread
    for (; i + 3 * kThreads < nvec; i += 4 * kThreads) {
      uint4 lo[4], hi[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        lo[u] = as[i + u * kThreads];
        hi[u] = as[i + u * kThreads + 1];
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        st_stream(vd + i + u * kThreads, shift(lo[u], hi[u]));
        count_bytes<COUNT>(p, (uint64_t)(vd + i + u * kThreads), 16);
      }
    }
    for (; i < nvec; i += kThreads) {
      st_stream(vd + i, shift(as[i], as[i + 1]));
      count_bytes<COUNT>(p, (uint64_t)(vd + i), 16);
    }
  }
  // tail
  const uint64_t tail = len & 15, base = nvec << 4;
  if (tid < tail) {
    dst[base + tid] = src[base + tid];
    count_bytes<COUNT>(p, d + base + tid, 1);
  }
}

// ------------------------------------------------------------------ TMA bulk engine
__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE;\n"
      "bra LAB_WAIT;\n"
      "DONE:\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(phase)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *sdst, const void *gsrc, uint32_t bytes, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(sdst)),
      "l"(gsrc), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}
__device__ __forceinline__ void bulk_s2g(void *gdst, const void *ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst),
               "r"(smem_addr(ssrc)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ------------------------------------------------------------------ round kernels
template <class KP>
__device__ __forceinline__ int find_chunk(const KP &p, uint32_t t) {
  int lo = 0, hi = (int)p.n_chunks - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (p.tile_prefix[mid] <= t) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// Round completion: the CTA barrier orders every thread's stores before
// thread 0's system-scope fence (fences are cumulative), so ONE fence per
// CTA suffices; the last CTA to finish publishes the completion words with
// release stores (no partial visibility).
template <class KP>
__device__ __forceinline__ void finish_round(const KP &p) {
  if (p.flags & kFlagNoPublish) return;  // a stream write after the launch publishes
  __syncthreads();
  if (threadIdx.x == 0) {
    // local destinations only need GPU-scope ordering before the counter;
    // peer (NVLink) destinations need the system-scope fence
    if ((p.flags & kFlagLocalDst) || p.n_pub == 0) __threadfence();  // n_pub 0: only the scratch reset
    else __threadfence_system();
    unsigned prev = atomicAdd(&p.scratch[1], 1u);
    if (prev == gridDim.x - 1) {
      if (p.n_pub) __threadfence_system();
      for (uint32_t i = 0; i < p.n_pub; ++i) st_release_sys(p.pub[i].word, p.pub[i].value);
      // every CTA has stopped claiming: reset for the next launch on this stream
      p.scratch[0] = 0;
      p.scratch[1] = 0;
      __threadfence();
    }
  }
}

template <bool COUNT, int U, int MINB, bool STAMP, class KP>
__global__ void __launch_bounds__(kThreads, MINB) gr_copy_ldst(const __grid_constant__ KP p) {
  pdl_wait();
  stamp_begin<STAMP>(p);
  __shared__ uint32_t s_tile;
  const uint32_t total = (uint32_t)p.tile_prefix[p.n_chunks];
  for (;;) {
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.scratch[0], 1u);
    __syncthreads();
    const uint32_t t = s_tile;
    __syncthreads();
    if (t >= total) break;
    const int c = find_chunk(p, t);
    const KChunk &ch = p.chunk[c];
    const uint64_t off = (uint64_t)(t - (uint32_t)p.tile_prefix[c]) << p.tile_log2;
    const uint64_t len = umin64(ch.bytes - off, 1ull << p.tile_log2);
    tile_ldst<COUNT, U>(p, reinterpret_cast<uint8_t *>(ch.dst + off),
                     reinterpret_cast<const uint8_t *>(ch.src + off), len);
  }
  pdl_trigger();
  stamp_end<STAMP>(p);
  finish_round(p);
}

// Static-assignment TMA ring ("tmas"): CTA b of G moves the 16 KiB units
// b, b+G, b+2G ... of the round (no ticket, so no scratch to reset and the
// completion can be published by the host after the launch), through a
// STAGES-deep cp.async.bulk ring small enough (STAGES x 16 KiB <= 96 KiB)
// that the NEXT launch's CTA is co-resident under PDL.  Before
// griddepcontrol.wait it initialises its barriers and pulls its first
// STAGES units of SOURCE into L2 (local sources only, like wv), so the DRAM
// read ramp of launch i+1 overlaps the tail of launch i.  16 B-aligned
// rounds only (bulk copies need 16 B addresses and sizes).
template <int STAGES, bool STAMP, class KP>
__global__ void __launch_bounds__(kTmaThreads) gr_copy_tmas(const __grid_constant__ KP p) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bars[STAGES];
  const uint32_t total = (uint32_t)p.tile_prefix[p.n_chunks];
  const uint32_t G = gridDim.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < STAGES; ++i) mbar_init(&bars[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (p.flags & kFlagLocalSrc)
      for (uint32_t k = 0, id = blockIdx.x; k < (uint32_t)STAGES && id < total; ++k, id += G) {
        const int c = find_chunk(p, id);
        const uint64_t off = (uint64_t)(id - (uint32_t)p.tile_prefix[c]) * kTmaStage;
        prefetch_l2(p.chunk[c].src + off, (uint32_t)umin64(p.chunk[c].bytes - off, kTmaStage));
      }
  }
  pdl_wait();
  stamp_begin<STAMP>(p);
  if (threadIdx.x == 0) {
    uint64_t dst_of[STAGES];
    uint32_t bytes_of[STAGES];
    uint32_t phase = 0;
    auto load = [&](uint32_t k) {  // unit number k of this CTA -> stage k % STAGES
      const uint32_t id = blockIdx.x + k * G;
      const int c = find_chunk(p, id);
      const uint64_t off = (uint64_t)(id - (uint32_t)p.tile_prefix[c]) * kTmaStage;
      const uint32_t st = k % STAGES;
      const uint32_t pb = (uint32_t)umin64(p.chunk[c].bytes - off, kTmaStage);
      dst_of[st] = p.chunk[c].dst + off;
      bytes_of[st] = pb;
      mbar_expect_tx(&bars[st], pb);
      bulk_g2s(smem + st * kTmaStage, reinterpret_cast<const void *>(p.chunk[c].src + off), pb, &bars[st]);
    };
    const uint32_t mine = blockIdx.x < total ? (total - blockIdx.x + G - 1) / G : 0;
    uint32_t loaded = 0;
    for (; loaded < mine && loaded < (uint32_t)STAGES; ++loaded) load(loaded);
    for (uint32_t k = 0; k < mine; ++k) {
      const uint32_t st = k % STAGES;
      mbar_wait(&bars[st], (phase >> st) & 1u);
      phase ^= (1u << st);
      bulk_s2g(reinterpret_cast<void *>(dst_of[st]), smem + st * kTmaStage, bytes_of[st]);
      bulk_commit();
      if (k >= 1 && loaded < mine) {
        bulk_wait_read<1>();  // the store of unit k-1 has left its stage
        load(loaded);
        ++loaded;
      }
    }
    bulk_wait_all();
    asm volatile("fence.proxy.async.global;" ::: "memory");
  }
  __syncthreads();
  pdl_trigger();
  stamp_end<STAMP>(p);
  finish_round(p);
}

// Before waiting on the predecessor grid (PDL), a warp may pull the first
// units of its OWN source into L2 with bulk prefetches: L2 is the point of
// coherence for this GPU's memory, so a prefetch can never return stale
// data (a line the predecessor still writes is updated in L2), and the
// DRAM read ramp of this launch overlaps the predecessor's tail.  Only for
// rounds whose sources are all in this GPU's memory (kFlagLocalSrc).
template <int LG, class KP>
__device__ __forceinline__ void prefetch_units(const KP &p, uint32_t w0, uint32_t W, uint32_t total,
                                               uint32_t lane) {
  const uint32_t n = (p.flags >> kPfShift) & 0xffu;
  if (!n || !(p.flags & kFlagLocalSrc) || lane != 0) return;
  for (uint32_t k = 0, id = w0; k < n && id < total; ++k, id += W) {
    const int c = find_chunk(p, id);
    const KChunk &ch = p.chunk[c];
    const uint64_t off = (uint64_t)(id - (uint32_t)p.tile_prefix[c]) << LG;
    const uint64_t src = ch.src + off;
    const uint32_t len = (uint32_t)umin64(ch.bytes - off, 1ull << LG);
    if (((src | len) & 15) == 0) prefetch_l2(src, len);
  }
}

// 256-bit global accesses (sm_100: LDG.256 / STG.256; L1 no-allocate: a
// source byte is read once).  L2 eviction hints measured no gain
// and are not used.
struct alignas(32) V8 {
  uint32_t x[8];
};
__device__ __forceinline__ V8 ld256(const V8 *p) {
  V8 r;
  asm volatile("ld.global.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(r.x[0]), "=r"(r.x[1]), "=r"(r.x[2]), "=r"(r.x[3]), "=r"(r.x[4]), "=r"(r.x[5]),
                 "=r"(r.x[6]), "=r"(r.x[7])
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st256(V8 *p, const V8 &v) {
  asm volatile("st.global.L1::no_allocate.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v.x[0]),
               "r"(v.x[1]), "r"(v.x[2]), "r"(v.x[3]), "r"(v.x[4]), "r"(v.x[5]), "r"(v.x[6]), "r"(v.x[7])
               : "memory");
}

// wv8: warp-strided copy with 256-bit accesses over 8 KiB units (LG = 13);
// warp w of W takes units w, w+W, ...; each lane keeps 8 x 32 B loads in
// flight per unit.  32 B co-aligned full units take the 256-bit path, 16 B
// co-aligned ones a 16 B path with 8 loads in flight per lane, anything else
// bytes (misaligned rounds go to ldst8 instead, see launch_copy).  Small
// rounds (<= 4 MiB) use 1 KiB units (LG = 10, one 32 B load per lane): the
// copy spreads over 8x more warps and SMs, so a latency-bound small copy
// waits for one DRAM round trip per lane instead of eight in a row.
template <bool COUNT, int LG, bool STAMP, class KP>
__global__ void __launch_bounds__(kThreads) gr_copy_wv(const __grid_constant__ KP p) {
  constexpr uint32_t kUnit = 1u << LG;
  constexpr int kPer = (int)(kUnit / (32 * 32));  // 32 B loads per lane per unit
  const uint32_t total = (uint32_t)p.tile_prefix[p.n_chunks];
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t W = gridDim.x * (kThreads / 32);
  prefetch_units<LG>(p, blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5), W, total, lane);
  pdl_wait();
  stamp_begin<STAMP>(p);
  for (uint32_t id = blockIdx.x * (kThreads / 32) + (threadIdx.x >> 5); id < total; id += W) {
    const int c = find_chunk(p, id);
    const KChunk &ch = p.chunk[c];
    const uint64_t off = (uint64_t)(id - (uint32_t)p.tile_prefix[c]) << LG;
    const uint64_t src = ch.src + off, dst = ch.dst + off;
    const uint32_t len = (uint32_t)umin64(ch.bytes - off, kUnit);
    if (len == kUnit && ((src | dst) & 31) == 0) {
      const V8 *sv = reinterpret_cast<const V8 *>(src);
      V8 *dv = reinterpret_cast<V8 *>(dst);
      V8 v[kPer];
#pragma unroll
      for (int j = 0; j < kPer; ++j) v[j] = ld256(sv + j * 32 + lane);
#pragma unroll
      for (int j = 0; j < kPer; ++j) {
        st256(dv + j * 32 + lane, v[j]);
        count_bytes<COUNT>(p, (uint64_t)(dv + j * 32 + lane), 16);
        count_bytes<COUNT>(p, (uint64_t)(dv + j * 32 + lane) + 16, 16);
      }
    } else if (((src | dst) & 15) == 0) {
      const uint32_t nv = len >> 4;
      const int4 *sv = reinterpret_cast<const int4 *>(src);
      int4 *dv = reinterpret_cast<int4 *>(dst);
      uint32_t i = lane;
      // 16 B co-aligned (not 32 B): 8 x 16 B loads in flight per lane
      for (; i + 7 * 32 < nv; i += 8 * 32) {
        int4 w[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) w[j] = ld_stream(sv + i + j * 32);
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          st_stream(dv + i + j * 32, w[j]);
          count_bytes<COUNT>(p, (uint64_t)(dv + i + j * 32), 16);
        }
      }
      for (; i < nv; i += 32) {
        st_stream(dv + i, ld_stream(sv + i));
        count_bytes<COUNT>(p, (uint64_t)(dv + i), 16);
      }
      uint8_t *d = reinterpret_cast<uint8_t *>(dst);
      const uint8_t *sp = reinterpret_cast<const uint8_t *>(src);
      for (uint32_t i = (nv << 4) + lane; i < len; i += 32) {
        d[i] = sp[i];
        count_bytes<COUNT>(p, (uint64_t)(d + i), 1);
      }
    } else {
      uint8_t *d = reinterpret_cast<uint8_t *>(dst);
      const uint8_t *sp = reinterpret_cast<const uint8_t *>(src);
      for (uint32_t i = lane; i < len; i += 32) {
        d[i] = sp[i];
        count_bytes<COUNT>(p, (uint64_t)(d + i), 1);
      }
    }
  }
  pdl_trigger();
  stamp_end<STAMP>(p);
  finish_round(p);
}

// Launch with programmatic stream serialization (PDL; GR_PDL=0 disables):
// the next copy's CTAs are scheduled while this one drains and block in
// griddepcontrol.wait before touching memory, which hides the inter-kernel
// gap (~1.2-2.2 us per 38.5 MB launch measured, tools/pubbench.sh).  It pays
// only when nothing but kernels/events sit between launches: a stream write
// (cuStreamWriteValue32) after a kernel breaks the overlap, which is why
// direct launches complete by an event (engine.cpp try_direct).
template <class KP>
static void launch_pdl(void (*kern)(KP), uint64_t grid, int block, int smem, cudaStream_t s, const KP &p) {
  static int pdl = -1;
  if (pdl < 0) {
    const char *e = getenv("GR_PDL");
    pdl = (e && e[0] == '0') ? 0 : 1;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  if (pdl) const_cast<KP &>(p).flags |= kFlagPdl;
  if (pdl) cudaLaunchKernelEx(&cfg, kern, p);
  else kern<<<cfg.gridDim, cfg.blockDim, cfg.dynamicSmemBytes, s>>>(p);
}

// Tile size per launch.  Tiles are claimed dynamically, so the makespan is
// ~ceil(tiles / grid) tiles: take the LARGEST tile (fewest claims, longest
// streams per claim) whose wave quantisation costs <= 5% over a perfect
// split of the round's bytes; min_lg keeps a tile at least one full pass of
// the engine (LD/ST: U x 256 x 16 B; TMA: 4 pieces).
template <class KP>
static void choose_tiles(KP &p, uint64_t grid_cap, uint32_t min_lg, uint32_t max_lg) {
  uint64_t total = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) total += p.chunk[i].bytes;
  uint32_t best = min_lg;
  double best_q = 1e30;
  for (uint32_t lg = max_lg; lg >= min_lg; --lg) {
    uint64_t tiles = 0;
    for (uint32_t i = 0; i < p.n_chunks; ++i) tiles += (p.chunk[i].bytes + (1ull << lg) - 1) >> lg;
    // makespan in bytes per CTA slot vs a perfect split over ALL slots
    const double q = (double)(((tiles + grid_cap - 1) / grid_cap) << lg) * (double)grid_cap / (double)total;
    if (q <= 1.05) {
      best = lg;
      break;
    }
    if (q < best_q) {
      best_q = q;
      best = lg;
    }
  }
  p.tile_log2 = best;
  uint64_t t = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) {
    p.tile_prefix[i] = t;
    t += (p.chunk[i].bytes + (1ull << best) - 1) >> best;
  }
  p.tile_prefix[p.n_chunks] = t;
}

// Engine: GR_COPY env (tests / tuning) = wv8 | tmas4 | ldst8; unset = the
// product choice in launch_copy.
enum Engine { kEngDefault = -1, kEngLdst8 = 0, kEngTmas4 = 1, kEngWv8 = 2 };
static int engine_from_env() {
  static int v = -2;
  if (v == -2) {
    const char *e = getenv("GR_COPY");
    v = kEngDefault;
    if (e) {
      std::string s(e);
      v = s == "ldst8" ? kEngLdst8 : s == "tmas4" ? kEngTmas4 : s == "wv8" ? kEngWv8 : kEngDefault;
    }
  }
  return v;
}

// tmas4: one 32-thread CTA per SM, 4 x 16 KiB stages (64 KiB of shared
// memory, so the next launch's CTA co-resides under PDL).
template <class KP>
static void launch_tmas(KP &p, int sm_count, cudaStream_t s) {
  constexpr int STAGES = 4;
  static bool attr_set = false;
  const int smem = STAGES * kTmaStage;
  if (!attr_set) {
    cudaFuncSetAttribute(gr_copy_tmas<STAGES, false, KP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(gr_copy_tmas<STAGES, true, KP>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr_set = true;
  }
  p.tile_log2 = 14;  // units of kTmaStage bytes
  uint64_t t = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) {
    p.tile_prefix[i] = t;
    t += (p.chunk[i].bytes + kTmaStage - 1) / kTmaStage;
  }
  p.tile_prefix[p.n_chunks] = t;
  uint64_t grid = (uint64_t)sm_count;
  if (grid > t) grid = t;
  if (grid == 0) grid = 1;
  if (p.stamp) launch_pdl(gr_copy_tmas<STAGES, true, KP>, grid, kTmaThreads, smem, s, p);
  else launch_pdl(gr_copy_tmas<STAGES, false, KP>, grid, kTmaThreads, smem, s, p);
}

// ldst8: 256-thread CTAs claim 32-256 KiB tiles from a ticket, 8 x 16 B in
// flight per thread; co-aligned and funnel-shift paths for misaligned rounds.
template <class KP>
static void launch_ldst(KP &p, int sm_count, int ctas_per_sm, cudaStream_t s) {
  static int occ = 0;
  if (!occ) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, gr_copy_ldst<false, 8, 1, false, KP>, kThreads, 0);
    if (occ <= 0) occ = 1;
  }
  const int per_sm = ctas_per_sm < occ ? ctas_per_sm : occ;
  const uint64_t cap = (uint64_t)sm_count * (uint64_t)per_sm;
  choose_tiles(p, cap, 15, 18);
  uint64_t tiles = p.tile_prefix[p.n_chunks];
  uint64_t grid = cap > tiles ? tiles : cap;
  if (p.counts) launch_pdl(gr_copy_ldst<true, 8, 1, false, KP>, grid, kThreads, 0, s, p);
  else if (p.stamp) launch_pdl(gr_copy_ldst<false, 8, 1, true, KP>, grid, kThreads, 0, s, p);
  else launch_pdl(gr_copy_ldst<false, 8, 1, false, KP>, grid, kThreads, 0, s, p);
}

template <int LG, class KP>
static void launch_wv(KP &p, int sm_count, int ctas_per_sm, cudaStream_t s) {
  static int occ = 0;
  if (!occ) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, gr_copy_wv<false, LG, false, KP>, kThreads, 0);
    if (occ <= 0) occ = 1;
  }
  const int per_sm = ctas_per_sm < occ ? ctas_per_sm : occ;
  p.tile_log2 = LG;
  uint64_t t = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) {
    p.tile_prefix[i] = t;
    t += (p.chunk[i].bytes + (1ull << LG) - 1) >> LG;
  }
  p.tile_prefix[p.n_chunks] = t;
  uint64_t grid = (t + (kThreads / 32) - 1) / (kThreads / 32);
  const uint64_t cap = (uint64_t)sm_count * per_sm;
  if (grid > cap) grid = cap;
  if (grid == 0) grid = 1;
  if (p.counts) launch_pdl(gr_copy_wv<true, LG, false, KP>, grid, kThreads, 0, s, p);
  else if (p.stamp) launch_pdl(gr_copy_wv<false, LG, true, KP>, grid, kThreads, 0, s, p);
  else launch_pdl(gr_copy_wv<false, LG, false, KP>, grid, kThreads, 0, s, p);
}

static bool getenv_wv_big() {  // GR_WV_BIG=1: 8 KiB units at every size (measurement only)
  static const bool b = getenv("GR_WV_BIG") != nullptr;
  return b;
}

template <class KP>
static void launch_engine(KP &p, int v, int sm_count, int ctas_per_sm, cudaStream_t s) {
  switch (v) {
    case kEngTmas4: launch_tmas(p, sm_count, s); break;
    case kEngWv8: {
      uint64_t total = 0;
      for (uint32_t i = 0; i < p.n_chunks; ++i) total += p.chunk[i].bytes;
      if (total <= (4ull << 20) && !getenv_wv_big()) launch_wv<10>(p, sm_count, ctas_per_sm, s);
      else launch_wv<13>(p, sm_count, ctas_per_sm, s);
      break;
    }
    default: launch_ldst(p, sm_count, ctas_per_sm, s); break;
  }
}

double g_launch_prof[3] = {};
uint64_t g_launch_prof_n = 0;
bool g_launch_prof_on = [] {
  const char *e = getenv("GROUTER_HOST_PROFILE");
  return e && e[0] == '1';
}();
static std::vector<uint32_t> g_launch_ns;
void launch_prof_percentiles(double *p10, double *p50, double *p90) {
  std::vector<uint32_t> v = g_launch_ns;
  std::sort(v.begin(), v.end());
  auto at = [&](double q) { return v.empty() ? 0.0 : v[(size_t)(q * (v.size() - 1))] / 1e3; };
  *p10 = at(0.1);
  *p50 = at(0.5);
  *p90 = at(0.9);
}
static inline uint64_t lp_now() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int launch_copy(CopyParams &p, int sm_count, int ctas_per_sm, bool tma, void *stream, bool *host_publish) {
  const uint64_t lp0 = g_launch_prof_on ? lp_now() : 0;
  uint64_t lp1 = 0, lp2 = 0;
  if (host_publish) *host_publish = false;
  if (p.n_chunks == 0) return (int)cudaSuccess;
  cudaStream_t s = (cudaStream_t)stream;
  // coalesce chunks that are contiguous in both source and destination (the
  // plan's 2 MiB chunks of one transfer are): fewer, longer runs per launch
  uint32_t w = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) {
    if (w && p.chunk[w - 1].src + p.chunk[w - 1].bytes == p.chunk[i].src &&
        p.chunk[w - 1].dst + p.chunk[w - 1].bytes == p.chunk[i].dst)
      p.chunk[w - 1].bytes += p.chunk[i].bytes;
    else
      p.chunk[w++] = p.chunk[i];
  }
  p.n_chunks = w;
  bool aligned = true, addr_aligned = true;
  for (uint32_t i = 0; i < p.n_chunks; ++i) {
    aligned &= ((p.chunk[i].src | p.chunk[i].dst | p.chunk[i].bytes) & 15) == 0;
    addr_aligned &= ((p.chunk[i].src | p.chunk[i].dst) & 15) == 0;
  }
  uint64_t total = 0;
  for (uint32_t i = 0; i < p.n_chunks; ++i) total += p.chunk[i].bytes;
  // Product choice (measured; tools/engine_sizes.py):
  //  * tmas4 for 16 B-aligned rounds >= 96 MiB whose sources and destinations
  //    are all in the launching GPU's memory (128 MiB 45.1 us, 256 MiB 84.9 us,
  //    1 GiB 329.6 us back to back = the copy engine's 44.4 / 84.3 / 329.3);
  //    GROUTER_COPY_TMA takes it for every aligned round;
  //  * wv8 otherwise (38.5 MB get_into back to back 11.8 us, 0.997 of the
  //    measured HBM copy peak); peer rounds (NVLink push/pull) stay on wv8;
  //  * ldst8 for rounds with a source or destination not 16 B aligned (a
  //    tensor view, a by-copy put of a host structure): co-aligned and
  //    funnel-shift 16 B paths instead of the warp engines' byte fallback.
  const bool local_round = (p.flags & kFlagLocalDst) && (p.flags & kFlagLocalSrc);
  int v = engine_from_env();
  if (v == kEngDefault) {
    if (!addr_aligned) v = kEngLdst8;
    else if (aligned && (tma || (local_round && total >= (96ull << 20)))) v = kEngTmas4;
    else v = kEngWv8;
  }
  if (v == kEngTmas4 && (!aligned || p.counts)) v = kEngWv8;  // bulk copies: 16 B only; counting is LD/ST
  // L2 prefetch of each warp's first 8 KiB unit before the PDL wait (wv8;
  // measured best at one unit, tools/exp_hints.sh in round 1)
  p.flags &= ~(0xffu << kPfShift);
  if (v == kEngWv8) p.flags |= 1u << kPfShift;
  // static-assignment engines (wv8, tmas4) need no scratch: their completion
  // can be published by the host after the launch (an event), which costs
  // the GPU ~2 us less than the in-kernel fence + counter + last-CTA protocol
  const bool is_static = v == kEngWv8 || v == kEngTmas4;
  p.flags &= ~kFlagNoPublish;
  if (host_publish && is_static && !p.counts) {
    p.flags |= kFlagNoPublish;
    *host_publish = true;
  } else if (p.n_pub == 0 && is_static && !p.counts) {
    p.flags |= kFlagNoPublish;  // nothing to publish and no ticket scratch to reset
  }
  if (p.n_chunks <= (uint32_t)SmallParams::kChunks && p.n_pub <= (uint32_t)SmallParams::kPubs) {
    SmallParams q;
    q.flags = p.flags;
    q.n_chunks = p.n_chunks;
    q.n_pub = p.n_pub;
    q.scratch = p.scratch;
    q.counts = p.counts;
    q.count_base = p.count_base;
    q.stamp = p.stamp;
    for (uint32_t i = 0; i < p.n_chunks; ++i) q.chunk[i] = p.chunk[i];
    for (uint32_t i = 0; i < p.n_pub; ++i) q.pub[i] = p.pub[i];
    if (g_launch_prof_on) lp1 = lp_now();
    launch_engine(q, v, sm_count, ctas_per_sm, s);
  } else {
    if (g_launch_prof_on) lp1 = lp_now();
    launch_engine(p, v, sm_count, ctas_per_sm, s);
  }
  if (g_launch_prof_on) lp2 = lp_now();
  const int err = (int)cudaGetLastError();
  if (g_launch_prof_on) {
    g_launch_prof[0] += lp1 - lp0;
    g_launch_prof[1] += lp2 - lp1;
    if (g_launch_ns.size() < (1u << 20)) g_launch_ns.push_back((uint32_t)(lp2 - lp1));
    g_launch_prof[2] += lp_now() - lp2;
    g_launch_prof_n++;
  }
  return err;
}

// ------------------------------------------------------------------ test kernels (K9)
__device__ __forceinline__ uint64_t splitmix(uint64_t seed, uint64_t i) {
  uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Each thread owns stream word w; writes the bytes of w that fall in
// [offset, offset+n) to dst[8w - offset + k].
__global__ void gr_fill_kernel(uint8_t *dst, uint64_t n, uint64_t seed, uint64_t offset) {
  const uint64_t w0 = offset >> 3, w1 = (offset + n + 7) >> 3;
  const bool aligned = (((uintptr_t)dst - offset) & 7) == 0;
  for (uint64_t w = w0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w1;
       w += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t v = splitmix(seed, w);
    const uint64_t b0 = w << 3;
    if (aligned && b0 >= offset && b0 + 8 <= offset + n) {
      *reinterpret_cast<uint64_t *>(dst + (b0 - offset)) = v;
    } else {
      for (int k = 0; k < 8; ++k) {
        uint64_t b = b0 + k;
        if (b >= offset && b < offset + n) dst[b - offset] = (uint8_t)(v >> (8 * k));
      }
    }
  }
}

__global__ void gr_verify_kernel(const uint8_t *src, uint64_t n, uint64_t seed, uint64_t offset,
                                 unsigned long long *out /* [0]=count, [1]=first */) {
  const uint64_t w0 = offset >> 3, w1 = (offset + n + 7) >> 3;
  unsigned long long bad = 0, first = ~0ull;
  for (uint64_t w = w0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w1;
       w += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t v = splitmix(seed, w);
    for (int k = 0; k < 8; ++k) {
      uint64_t b = (w << 3) + k;
      if (b >= offset && b < offset + n && src[b - offset] != (uint8_t)(v >> (8 * k))) {
        ++bad;
        if (b - offset < first) first = b - offset;
      }
    }
  }
  if (bad) {
    atomicAdd(&out[0], bad);
    atomicMin(&out[1], first);
  }
}

}  // namespace gr

// ------------------------------------------------------------------ testing ABI
using namespace gr;

static unsigned fill_grid(uint64_t words) {
  uint64_t g = (words + 255) / 256;
  if (g > 148 * 16) g = 148 * 16;
  return (unsigned)(g ? g : 1);
}

__global__ void gr_empty_kernel(const __grid_constant__ SmallParams p) { (void)p; }
__global__ void gr_empty_kernel_big(const __grid_constant__ CopyParams p) { (void)p; }
__global__ void gr_empty_kernel_tiny(int x) { (void)x; }

extern "C" grouter_status grouter_test_launch_cost(int kind, int n, int blocks, void *stream, double *us_per_launch) {
  if (!us_per_launch || n <= 0) return GROUTER_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  static SmallParams sp;
  static CopyParams bp;
  // kinds 3/4: small block via cudaLaunchKernelEx with / without the PDL
  // attribute; 5: cudaEventRecord only; 6: cudaEventQuery of a recorded event
  static cudaEvent_t ev = nullptr;
  if (!ev) cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(blocks);
  cfg.blockDim = dim3(256);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  if (kind == 6) cudaEventRecord(ev, s);
  // kind >= 100: latency mode -- the stream is drained before every launch
  // and only the launch call itself is timed
  // kind >= 200: like 100 plus a 50 us host spin after the drain (GPU and
  // link left idle as between latency-mode requests)
  const bool spin = kind >= 200;
  if (spin) kind -= 100;
  const bool idle = kind >= 100;
  if (idle) kind -= 100;
  double idle_us = 0;
  auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) {
    auto ti = std::chrono::steady_clock::now();
    if (idle) {
      cudaStreamSynchronize(s);
      if (spin)
        while (std::chrono::steady_clock::now() - ti < std::chrono::microseconds(50)) {
        }
      ti = std::chrono::steady_clock::now();
    }
    if (kind == 0) gr_empty_kernel_tiny<<<blocks, 256, 0, s>>>(i);
    else if (kind == 1) gr_empty_kernel<<<blocks, 256, 0, s>>>(sp);
    else if (kind == 2) gr_empty_kernel_big<<<blocks, 256, 0, s>>>(bp);
    else if (kind == 3 || kind == 4) {
      cfg.numAttrs = kind == 3 ? 1 : 0;
      cudaLaunchKernelEx(&cfg, gr_empty_kernel, sp);
    } else if (kind == 10 || kind == 11) {  // driver API cuLaunchKernelEx (with / without PDL)
      static CUfunction f = nullptr;
      if (!f) cudaGetFuncBySymbol(&f, (const void *)gr_empty_kernel);
      CUlaunchAttribute at[1];
      at[0].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
      at[0].value.programmaticStreamSerializationAllowed = 1;
      CUlaunchConfig lc = {};
      lc.gridDimX = blocks;
      lc.gridDimY = lc.gridDimZ = 1;
      lc.blockDimX = 256;
      lc.blockDimY = lc.blockDimZ = 1;
      lc.hStream = (CUstream)s;
      lc.attrs = at;
      lc.numAttrs = kind == 10 ? 1 : 0;
      void *args[] = {(void *)&sp};
      drv().launchKernelEx(&lc, f, args, nullptr);
    } else if (kind == 5) cudaEventRecord(ev, s);
    else if (kind == 6) (void)cudaEventQuery(ev);
    else {  // 7: launch_copy of 4 KiB, 8: of 38.5 MB (the production launch path), 9: event + 8
      static uint8_t *buf = nullptr;
      static uint32_t *scr = nullptr;
      if (!buf) {
        cudaMalloc(&buf, 2 * 38535168ull);
        cudaMalloc(&scr, 64);
        cudaMemset(scr, 0, 64);
      }
      if (kind == 9) cudaEventRecord(ev, s);
      CopyParams &q = bp;
      q.flags = kFlagLocalDst | kFlagLocalSrc;
      q.n_chunks = 1;
      q.n_pub = 0;
      q.scratch = scr;
      q.counts = nullptr;
      q.chunk[0] = {(uint64_t)buf, (uint64_t)buf + 38535168ull, kind == 7 ? 4096ull : 38535168ull};
      bool hp = false;
      launch_copy(q, 148, 4, false, s, &hp);
    }
    if (idle) idle_us += std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - ti).count();
  }
  auto t1 = std::chrono::steady_clock::now();
  cudaStreamSynchronize(s);
  *us_per_launch = idle ? idle_us / n : std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
  return cudaGetLastError() == cudaSuccess ? GROUTER_OK : GROUTER_ECUDA;
}

extern "C" grouter_status grouter_test_memcpy(void *dst, const void *src, uint64_t n, void *stream, int32_t wait) {
  if (n && (!dst || !src)) return GROUTER_EINVAL;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev >= 64) return GROUTER_ECUDA;
  static cudaStream_t own[64] = {};
  static cudaEvent_t ev[64] = {};
  cudaStream_t s = (cudaStream_t)stream;
  if (!s) {
    if (!own[dev] && cudaStreamCreateWithFlags(&own[dev], cudaStreamNonBlocking) != cudaSuccess)
      return GROUTER_ECUDA;
    s = own[dev];
  }
  if (!ev[dev] && cudaEventCreateWithFlags(&ev[dev], cudaEventDisableTiming) != cudaSuccess) return GROUTER_ECUDA;
  if (n && cudaMemcpyAsync(dst, src, n, cudaMemcpyDefault, s) != cudaSuccess) return GROUTER_ECUDA;
  if (wait) {
    if (cudaEventRecord(ev[dev], s) != cudaSuccess) return GROUTER_ECUDA;
    cudaError_t e;
    int spins = 0;
    while ((e = cudaEventQuery(ev[dev])) == cudaErrorNotReady)
      if (++spins > 24) {  // the library's host_wait: spin briefly, then block in the driver
        e = cudaEventSynchronize(ev[dev]);
        break;
      }
    if (e != cudaSuccess) return GROUTER_ECUDA;
  }
  return GROUTER_OK;
}

extern "C" grouter_status grouter_test_fill(void *dst, uint64_t n, uint64_t seed, uint64_t offset,
                                            void *stream) {
  if (n == 0) return GROUTER_OK;
  if (!dst) return GROUTER_EINVAL;
  const uint64_t words = ((offset + n + 7) >> 3) - (offset >> 3);
  gr_fill_kernel<<<fill_grid(words), 256, 0, (cudaStream_t)stream>>>((uint8_t *)dst, n, seed, offset);
  return cudaGetLastError() == cudaSuccess ? GROUTER_OK : GROUTER_ECUDA;
}

extern "C" grouter_status grouter_test_verify(const void *src, uint64_t n, uint64_t seed,
                                              uint64_t offset, void *stream, uint64_t *mismatches,
                                              uint64_t *first_bad) {
  if (!mismatches || !first_bad) return GROUTER_EINVAL;
  *mismatches = 0;
  *first_bad = UINT64_MAX;
  if (n == 0) return GROUTER_OK;
  cudaStream_t s = (cudaStream_t)stream;
  unsigned long long *d = nullptr, h[2] = {0, ~0ull};
  if (cudaMalloc(&d, sizeof(h)) != cudaSuccess) return GROUTER_ECUDA;
  cudaMemcpyAsync(d, h, sizeof(h), cudaMemcpyHostToDevice, s);
  const uint64_t words = ((offset + n + 7) >> 3) - (offset >> 3);
  gr_verify_kernel<<<fill_grid(words), 256, 0, s>>>((const uint8_t *)src, n, seed, offset, d);
  cudaMemcpyAsync(h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
  cudaError_t e = cudaStreamSynchronize(s);
  cudaFree(d);
  if (e != cudaSuccess) return GROUTER_ECUDA;
  *mismatches = h[0];
  *first_bad = h[1] == ~0ull ? UINT64_MAX : h[1];
  return GROUTER_OK;
}

extern "C" grouter_status grouter_test_copy(void *dst_base, const void *src_base,
                                            const grouter_chunk *chunks, uint32_t n_chunks,
                                            uint32_t *counts, int tma, void *stream) {
  if (n_chunks > (uint32_t)kMaxRoundChunks || (n_chunks && !chunks)) return GROUTER_EINVAL;
  if (n_chunks == 0) return GROUTER_OK;
  static uint32_t *scratch[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 64) return GROUTER_EINVAL;
  if (!scratch[dev]) {
    if (cudaMalloc(&scratch[dev], 2 * sizeof(uint32_t)) != cudaSuccess) return GROUTER_ECUDA;
    cudaMemset(scratch[dev], 0, 2 * sizeof(uint32_t));
  }
  CopyParams *p = new CopyParams();
  p->flags = kFlagLocalDst | kFlagLocalSrc;  // test copies stay on the current device
  p->n_chunks = n_chunks;
  p->scratch = scratch[dev];
  p->counts = counts;
  p->count_base = (uint64_t)dst_base & ~15ull;
  uint64_t t = 0;
  for (uint32_t i = 0; i < n_chunks; ++i) {
    p->chunk[i] = {(uint64_t)src_base + chunks[i].offset, (uint64_t)dst_base + chunks[i].offset,
                   chunks[i].bytes};
    p->tile_prefix[i] = t;
    t += (chunks[i].bytes + (1ull << p->tile_log2) - 1) >> p->tile_log2;
  }
  p->tile_prefix[n_chunks] = t;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // diagnostic knob GR_TEST_PUB: 0 = in-kernel completion (default), 1 = no
  // completion, 2 = host-published (stream write after the launch), 3 =
  // event record after the launch
  static int pub = getenv("GR_TEST_PUB") ? atoi(getenv("GR_TEST_PUB")) : 0;
  static uint32_t *word = nullptr;
  static cudaEvent_t ev = nullptr;
  typedef CUresult_t (*WriteFn)(cudaStream_t, unsigned long long, unsigned, unsigned);
  static WriteFn wv = nullptr;
  if (pub >= 2 && !word) {
    cudaHostAlloc(&word, 64, cudaHostAllocMapped);
    cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuStreamWriteValue32", (void **)&wv, cudaEnableDefault, &q);
  }
  bool host_pub = false;
  int e = launch_copy(*p, sms, 2, tma && !counts, stream, pub >= 1 ? &host_pub : nullptr);
  if (pub == 2 && wv) {
    void *dptr = nullptr;
    cudaHostGetDevicePointer(&dptr, word, 0);
    wv((cudaStream_t)stream, (unsigned long long)dptr, 1, 0);
  } else if (pub == 3) {
    cudaEventRecord(ev, (cudaStream_t)stream);
  }
  delete p;
  return e == 0 ? GROUTER_OK : GROUTER_ECUDA;
}
