// kernels.cu -- sm_100a data-movement kernels (no tensor cores: pure bytes).
//
// gr_copy: see kernels.h.  Two tile engines:
//   * LD/ST: 256 threads, 128-bit vector loads/stores, 4 in flight per
//     thread before the first store (coalesced, L1 no-allocate), with
//     co-aligned and shifted (funnel-shift) paths for misaligned user
//     buffers and byte head/tail;
//   * TMA bulk: one elected thread streams the tile global -> shared ->
//     global with cp.async.bulk through a 4-stage mbarrier ring (16 KiB per
//     stage), used for 16-byte aligned tiles.
// Both serve local HBM, peer (NVLink) and host-mapped addresses: the data
// path never interprets bytes.
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/grouter.h"
#include "../../include/grouter_testing.h"
#include "kernels.h"

namespace gr {

constexpr int kThreads = 256;
constexpr int kTmaThreads = 32;
constexpr uint32_t kTmaStage = 16384;
constexpr int kTmaStages = 4;

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
__device__ __forceinline__ void st_release_sys(uint64_t addr, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(addr), "r"(v) : "memory");
}

template <bool COUNT>
__device__ __forceinline__ void count_bytes(const CopyParams &p, uint64_t dst_addr, uint32_t nbytes) {
  if (COUNT) atomicAdd(&p.counts[(dst_addr - p.count_base) >> 4], nbytes);
}

// dst[0,len) <- src[0,len), all threads of the CTA; any alignment.
template <bool COUNT>
__device__ void tile_ldst(const CopyParams &p, uint8_t *dst, const uint8_t *src, uint64_t len) {
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
    const int4 *vs = reinterpret_cast<const int4 *>(src);
    constexpr int U = 4;
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
    for (uint64_t i = tid; i < nvec; i += kThreads) {
      uint4 lo = as[i], hi = as[i + 1];
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
      int4 v = make_int4((int)o[0], (int)o[1], (int)o[2], (int)o[3]);
      st_stream(vd + i, v);
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

struct TmaState {
  uint32_t phase_bits;  // one parity bit per stage
};

// One elected thread moves [src, src+len) -> [dst, ...) in kTmaStage pieces.
// Requires 16 B alignment of src, dst and len.  Stage s is refilled with
// piece k+S only after the store of piece k has finished READING shared
// memory (wait_group.read 1 while the newest store may still be reading).
__device__ void tile_tma(uint8_t *dst, const uint8_t *src, uint64_t len, uint8_t *smem,
                         uint64_t *bars, TmaState &st) {
  const uint32_t pieces = (uint32_t)((len + kTmaStage - 1) / kTmaStage);
  auto piece_bytes = [&](uint32_t k) {
    return (uint32_t)umin64(kTmaStage, len - (uint64_t)k * kTmaStage);
  };
  auto load = [&](uint32_t k) {
    const uint32_t s = k % kTmaStages;
    mbar_expect_tx(&bars[s], piece_bytes(k));
    bulk_g2s(smem + s * kTmaStage, src + (uint64_t)k * kTmaStage, piece_bytes(k), &bars[s]);
  };
  for (uint32_t k = 0; k < pieces && k < (uint32_t)kTmaStages; ++k) load(k);
  for (uint32_t k = 0; k < pieces; ++k) {
    const uint32_t s = k % kTmaStages;
    mbar_wait(&bars[s], (st.phase_bits >> s) & 1u);
    st.phase_bits ^= (1u << s);
    bulk_s2g(dst + (uint64_t)k * kTmaStage, smem + s * kTmaStage, piece_bytes(k));
    bulk_commit();
    if (k >= 1 && k - 1 + kTmaStages < pieces) {
      bulk_wait_read<1>();
      load(k - 1 + kTmaStages);
    }
  }
  bulk_wait_read<0>();  // stages free for the next tile
}

// ------------------------------------------------------------------ round kernel
__device__ __forceinline__ int find_chunk(const CopyParams &p, uint32_t t) {
  int lo = 0, hi = (int)p.n_chunks - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (p.tile_prefix[mid] <= t) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ void finish_round(const CopyParams &p) {
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned prev = atomicAdd(&p.scratch[1], 1u);
    if (prev == gridDim.x - 1) {
      __threadfence_system();
      for (uint32_t i = 0; i < p.n_pub; ++i) st_release_sys(p.pub[i].word, p.pub[i].value);
      // every CTA has stopped claiming: reset for the next launch on this stream
      p.scratch[0] = 0;
      p.scratch[1] = 0;
      __threadfence();
    }
  }
}

template <bool COUNT>
__global__ void __launch_bounds__(kThreads) gr_copy_ldst(const __grid_constant__ CopyParams p) {
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
    tile_ldst<COUNT>(p, reinterpret_cast<uint8_t *>(ch.dst + off),
                     reinterpret_cast<const uint8_t *>(ch.src + off), len);
  }
  finish_round(p);
}

__global__ void __launch_bounds__(kTmaThreads) gr_copy_tma(const __grid_constant__ CopyParams p) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bars[kTmaStages];
  __shared__ uint32_t s_tile;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kTmaStages; ++i) mbar_init(&bars[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  TmaState st{0};
  const uint32_t total = (uint32_t)p.tile_prefix[p.n_chunks];
  for (;;) {
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.scratch[0], 1u);
    __syncwarp();
    __syncthreads();
    const uint32_t t = s_tile;
    __syncthreads();
    if (t >= total) break;
    const int c = find_chunk(p, t);
    const KChunk &ch = p.chunk[c];
    const uint64_t off = (uint64_t)(t - (uint32_t)p.tile_prefix[c]) << p.tile_log2;
    const uint64_t len = umin64(ch.bytes - off, 1ull << p.tile_log2);
    uint8_t *dst = reinterpret_cast<uint8_t *>(ch.dst + off);
    const uint8_t *src = reinterpret_cast<const uint8_t *>(ch.src + off);
    if ((((uintptr_t)dst | (uintptr_t)src | len) & 15) == 0) {
      if (threadIdx.x == 0) tile_tma(dst, src, len, smem, bars, st);
      __syncwarp();
    } else {
      // rare misaligned tile: plain byte copy by the warp
      for (uint64_t i = threadIdx.x; i < len; i += kTmaThreads) dst[i] = src[i];
    }
  }
  if (threadIdx.x == 0) {
    bulk_wait_all();
    asm volatile("fence.proxy.async.global;" ::: "memory");
  }
  __syncthreads();
  finish_round(p);
}

int launch_copy(CopyParams &p, int sm_count, int ctas_per_sm, bool tma, void *stream) {
  const uint64_t tiles = p.tile_prefix[p.n_chunks];
  if (tiles == 0) return (int)cudaSuccess;
  cudaStream_t s = (cudaStream_t)stream;
  if (tma) {
    static bool attr_set = false;
    const int smem = kTmaStages * kTmaStage;
    if (!attr_set) {
      cudaFuncSetAttribute(gr_copy_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      attr_set = true;
    }
    uint64_t grid = (uint64_t)sm_count * 3;
    if (grid > tiles) grid = tiles;
    gr_copy_tma<<<(unsigned)grid, kTmaThreads, smem, s>>>(p);
  } else {
    uint64_t grid = (uint64_t)sm_count * (uint64_t)ctas_per_sm;
    if (grid > tiles) grid = tiles;
    if (p.counts) gr_copy_ldst<true><<<(unsigned)grid, kThreads, 0, s>>>(p);
    else gr_copy_ldst<false><<<(unsigned)grid, kThreads, 0, s>>>(p);
  }
  return (int)cudaGetLastError();
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
  int e = launch_copy(*p, sms, 2, tma && !counts, stream);
  delete p;
  return e == 0 ? GROUTER_OK : GROUTER_ECUDA;
}
