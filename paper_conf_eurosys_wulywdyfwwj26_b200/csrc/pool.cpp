// pool.cpp -- elastic GPU object pool, pinned host store, error/driver plumbing.
//
// PAPER.md L248 (cudaMalloc/cudaFree are millisecond-level -> pool), L256
// (minimum warm pool "e.g., 300 MB", scale with demand), L262 (storage kept
// under 50% of free memory), L269 (per-GPU elastic pool; an I/O thread
// reclaims unused memory), L394 ("enforced alignment" of mapped storage).
//
// Device pool = one CUDA VMM virtual range per logical GPU, backed by
// physical segments mapped contiguously from its base; objects and leases
// are page-aligned runs (2 MiB, R14) of that range.  Freed runs go to a
// quarantine until every GPU operation that may still touch them has
// completed (stream-ordered reuse without host synchronisation on the hot
// path); the pool grows by mapping more segments at its end and trims
// trailing free segments back toward the warm floor.
#include <algorithm>
#include <csignal>
#include <cstdio>
#include <dlfcn.h>
#include <execinfo.h>
#include <chrono>
#include <cstdio>
#include <thread>

#include "ctx.h"

namespace gr {

// ------------------------------------------------------------------ host profile
// GROUTER_BT=1: print a raw backtrace on SIGABRT/SIGSEGV (debug aid; map
// the offsets with addr2line -e libgrouter.so).
static void bt_handler(int sig) {
  void *fr[64];
  int n = backtrace(fr, 64);
  Dl_info di;
  for (int i = 0; i < n; ++i) {
    if (dladdr(fr[i], &di) && di.dli_fname)
      fprintf(stderr, "  #%d %s +0x%lx\n", i, di.dli_fname, (unsigned long)((char *)fr[i] - (char *)di.dli_fbase));
  }
  ::signal(sig, SIG_DFL);
  ::raise(sig);
}
static int bt_init = [] {
  const char *e = getenv("GROUTER_BT");
  if (e && e[0] == '1') {
    ::signal(SIGABRT, bt_handler);
    ::signal(SIGSEGV, bt_handler);
  }
  return 0;
}();

thread_local uint64_t tl_put_t0 = 0;
HostProf &hprof() {
  static HostProf h = [] {
    HostProf x;
    const char *e = getenv("GROUTER_HOST_PROFILE");
    x.on = e && e[0] == '1';
    return x;
  }();
  return h;
}
uint64_t now_ns() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

nvtxDomainHandle_t nvtx_domain() {
  static nvtxDomainHandle_t d = nvtxDomainCreateA("grouter");
  return d;
}

// ------------------------------------------------------------------ errors
static thread_local std::string tl_error;
void set_error(const std::string &msg) { tl_error = msg; }
const char *last_error() { return tl_error.c_str(); }

// ------------------------------------------------------------------ driver
template <class F>
static void resolve(const char *name, F &fn) {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || !p)
    throw Error(GROUTER_ECUDA, std::string("driver entry point missing: ") + name);
  fn = reinterpret_cast<F>(p);
}

const Driver &drv() {
  static Driver d;
  static std::once_flag once;
  static std::string err;
  std::call_once(once, [] {
    try {
      resolve("cuMemCreate", d.memCreate);
      resolve("cuMemRelease", d.memRelease);
      resolve("cuMemAddressReserve", d.memAddressReserve);
      resolve("cuMemAddressFree", d.memAddressFree);
      resolve("cuMemMap", d.memMap);
      resolve("cuMemUnmap", d.memUnmap);
      resolve("cuMemSetAccess", d.memSetAccess);
      resolve("cuMemGetAllocationGranularity", d.memGetAllocationGranularity);
      resolve("cuMemExportToShareableHandle", d.memExportToShareableHandle);
      resolve("cuMemImportFromShareableHandle", d.memImportFromShareableHandle);
      resolve("cuStreamWaitValue32", d.streamWaitValue32);
      resolve("cuStreamWriteValue32", d.streamWriteValue32);
      resolve("cuLaunchKernelEx", d.launchKernelEx);
    } catch (const Error &e) {
      err = e.what();
    }
  });
  if (!err.empty()) throw Error(GROUTER_ECUDA, err);
  return d;
}

// ------------------------------------------------------------------ events
EventRef EventPool::get() {
  Event *e = nullptr;
  {
    std::lock_guard<std::mutex> g(mu);
    if (!free_list.empty()) {
      e = free_list.back();
      free_list.pop_back();
    }
  }
  if (e) e->fired.store(false, std::memory_order_relaxed);
  if (!e) {
    e = new Event();
    e->phys = phys;
    e->pool = this;
    GR_CUDA(cudaEventCreateWithFlags(&e->ev, cudaEventDisableTiming));
  }
  return EventRef(e, [](Event *ev) {
    std::lock_guard<std::mutex> g(ev->pool->mu);
    ev->pool->free_list.push_back(ev);
  });
}

EventPool::~EventPool() {
  for (Event *e : free_list) {
    cudaEventDestroy(e->ev);
    delete e;
  }
}

// ------------------------------------------------------------------ page heap
bool PageHeap::take(uint64_t len, uint64_t *off) {
  for (auto it = free_runs.begin(); it != free_runs.end(); ++it) {
    if (it->second >= len) {
      *off = it->first;
      uint64_t rest = it->second - len, o = it->first;
      free_runs.erase(it);
      if (rest) free_runs[o + len] = rest;
      return true;
    }
  }
  return false;
}

void PageHeap::give(uint64_t off, uint64_t len) {
  if (!len) return;
  auto nx = free_runs.lower_bound(off);
  if (nx != free_runs.end() && off + len == nx->first) {
    len += nx->second;
    nx = free_runs.erase(nx);
  }
  if (nx != free_runs.begin()) {
    auto pv = std::prev(nx);
    if (pv->first + pv->second == off) {
      pv->second += len;
      return;
    }
  }
  free_runs[off] = len;
}

void PageHeap::reclaim() {
  size_t w = 0;
  for (size_t i = 0; i < quarantine.size(); ++i) {
    bool done = true;
    for (auto &f : quarantine[i].fences)
      if (!f.done()) {
        done = false;
        break;
      }
    if (done) {
      give(quarantine[i].off, quarantine[i].len);
    } else {
      if (w != i) quarantine[w] = std::move(quarantine[i]);  // never self-move: it empties the fences
      ++w;
    }
  }
  quarantine.resize(w);
}

uint64_t PageHeap::free_bytes() const {
  uint64_t s = 0;
  for (auto &kv : free_runs) s += kv.second;
  return s;
}

uint64_t PageHeap::tail_free(uint64_t end) const {
  if (free_runs.empty()) return 0;
  auto it = std::prev(free_runs.end());
  return it->first + it->second == end ? it->second : 0;
}

// ------------------------------------------------------------------ pool sizing (R44)
// Nearest-rank p99: the ceil(0.99 m)-th smallest sample.
static uint64_t p99(const std::deque<uint64_t> &xs) {
  if (xs.empty()) return 0;
  std::vector<uint64_t> v(xs.begin(), xs.end());
  const size_t k = (99 * v.size() + 99) / 100;
  std::nth_element(v.begin(), v.begin() + (k - 1), v.end());
  return v[k - 1];
}

void FuncHist::observe(uint64_t t, uint64_t size, uint64_t con) {
  arrivals.push_back(t);
  sizes.push_back(size);
  cons.push_back(con);
  if (arrivals.size() > kHist + 1) arrivals.pop_front();
  if (sizes.size() > kHist) sizes.pop_front();
  if (cons.size() > kHist) cons.pop_front();
}

uint64_t FuncHist::r_window() const {
  std::deque<uint64_t> iv;
  for (size_t i = 1; i < arrivals.size(); ++i) iv.push_back(arrivals[i] - arrivals[i - 1]);
  return p99(iv);
}

uint64_t FuncHist::data_size() const {
  const unsigned __int128 d = (unsigned __int128)p99(sizes) * p99(cons);
  return d > UINT64_MAX ? UINT64_MAX : (uint64_t)d;
}

static uint64_t clock_now(const grouter_ctx *c) { return c->clock_fixed ? c->clock_ns : now_ns(); }

// target(d, now) = min(cap, max(floor, MemPool_size)), MemPool_size = sum of
// Data_size over the functions whose reservation window is open (L254-L256).
uint64_t pool_target(grouter_ctx *c, int d) {
  const uint64_t t = clock_now(c);
  unsigned __int128 sum = 0;
  for (auto &kv : c->hists)
    if (std::get<2>(kv.first) == d && kv.second.active(t)) sum += kv.second.data_size();
  uint64_t m = sum > UINT64_MAX ? UINT64_MAX : (uint64_t)sum;
  m = std::max<uint64_t>(m, c->cfg.pool_floor_bytes);
  return std::min<uint64_t>(m, c->dev[d].cap);
}

// ------------------------------------------------------------------ device pool
void DevicePool::init(int lg, int ph, uint64_t va, const std::vector<int> &acc, uint64_t prewarm) {
  logical = lg;
  phys = ph;
  access = acc;
  va_size = va;
  GR_CU(drv().memAddressReserve(&base, va_size, kPage, 0, 0));
  if (prewarm) grow(prewarm);
}

DevicePool::Seg DevicePool::map_seg(CUdeviceptr base, uint64_t off, uint64_t size, int phys,
                                    const std::vector<int> &access, bool fallback_ok, uint64_t need) {
  CUmemAllocationProp prop = {};
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = phys;
  prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;  // IPC-exportable (L167)
  CUmemGenericAllocationHandle h;
  CUresult r = drv().memCreate(&h, size, &prop, 0);
  if (r != CUDA_SUCCESS && fallback_ok && size > need) {
    size = need;
    r = drv().memCreate(&h, size, &prop, 0);
  }
  if (r != CUDA_SUCCESS) throw Error(GROUTER_ENOMEM, "cuMemCreate failed (HBM exhausted)");
  if (drv().memMap(base + off, size, 0, h, 0) != CUDA_SUCCESS) {
    drv().memRelease(h);
    throw Error(GROUTER_ECUDA, "cuMemMap failed");
  }
  std::vector<CUmemAccessDesc> ad;
  for (int p : access) {
    CUmemAccessDesc a = {};
    a.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    a.location.id = p;
    a.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    ad.push_back(a);
  }
  if (drv().memSetAccess(base + off, size, ad.data(), ad.size()) != CUDA_SUCCESS) {
    drv().memUnmap(base + off, size);
    drv().memRelease(h);
    throw Error(GROUTER_ECUDA, "cuMemSetAccess failed");
  }
  return {off, size, h};
}

void DevicePool::publish(const Seg &s) {
  // segments stay in VA order (an on-demand grow may have mapped above a
  // pre-warm reservation meanwhile)
  auto it = std::upper_bound(segs.begin(), segs.end(), s.off,
                             [](uint64_t off, const Seg &x) { return off < x.off; });
  segs.insert(it, s);
  heap.give(s.off, s.size);
  mapped += s.size;
}

void DevicePool::grow(uint64_t need) {
  need = charge(need);
  uint64_t seg = std::max<uint64_t>(need, 64ull << 20);
  if (va_top + seg > va_size) seg = need;
  if (va_top + seg > va_size) throw Error(GROUTER_ENOMEM, "pool VA range exhausted");
  const uint64_t off = va_top;
  Seg s = map_seg(base, off, seg, phys, access, true, need);
  va_top = off + s.size;
  publish(s);
}

bool DevicePool::reserve(uint64_t size, uint64_t &off) {
  if (va_top + size > va_size) return false;
  off = va_top;
  va_top += size;
  return true;
}

void DevicePool::unreserve(uint64_t off, uint64_t size) {
  if (va_top == off + size) va_top = off;  // else a hole (never handed out)
}

// Detaches trailing segments that are entirely free while the mapping stays
// >= keep; their pages leave the heap at once (never handed out again).
std::vector<DevicePool::Seg> DevicePool::detach(uint64_t keep) {
  heap.reclaim();
  std::vector<Seg> out;
  uint64_t end = va_top;
  while (!segs.empty()) {
    Seg s = segs.back();
    if (mapped - s.size < keep) break;
    if (s.off + s.size != end || heap.tail_free(end) < s.size) break;  // (a hole above: stop)
    // carve the segment out of the trailing free run
    auto it = std::prev(heap.free_runs.end());
    uint64_t run_off = it->first;
    heap.free_runs.erase(it);
    if (s.off > run_off) heap.free_runs[run_off] = s.off - run_off;
    mapped -= s.size;
    segs.pop_back();
    out.push_back(s);
    end = s.off;
  }
  return out;
}

void DevicePool::unmap(CUdeviceptr base, const std::vector<Seg> &v) {
  for (auto &s : v) {
    drv().memUnmap(base + s.off, s.size);
    drv().memRelease(s.h);
  }
}

// out is in descending VA order; lower va_top only if nothing grew above it
void DevicePool::settle(const std::vector<Seg> &v) {
  if (v.empty()) return;
  const uint64_t hi = v.front().off + v.front().size, lo = v.back().off;
  if (va_top == hi) va_top = lo;
}

void DevicePool::trim(uint64_t keep) {
  auto v = detach(keep);
  unmap(base, v);
  settle(v);
}

void DevicePool::destroy() {
  for (auto &s : segs) {
    drv().memUnmap(base + s.off, s.size);
    drv().memRelease(s.h);
  }
  segs.clear();
  if (base) drv().memAddressFree(base, va_size);
  base = 0;
  mapped = 0;
  va_top = 0;
}

static bool all_grounded(const grouter_ctx *c, const Quarantined &q) {
  return grounded(c, q.fences);
}

// Physical pages for `len` bytes (a multiple of 2 MiB) on a logical GPU.
// Order: free runs; reclaimed quarantine; wait for grounded quarantine (after
// draining queued work so no wait depends on the caller); grow the mapping.
uint8_t *dev_alloc(grouter_ctx *c, int logical, uint64_t len, std::unique_lock<std::mutex> *lk) {
  if (c->cfg.flags & GROUTER_NO_POOL) {  // ablation: no pool (Fig. 16 "ES" off)
    nopool_sweep(c, false);
    DeviceGuard g(c->dev[logical].phys);
    void *p = nullptr;
    if (cudaMalloc(&p, len) != cudaSuccess) {
      cudaGetLastError();
      throw Error(GROUTER_ENOMEM, "cudaMalloc failed (GROUTER_NO_POOL)");
    }
    c->nopool_live[(uint8_t *)p] = c->dev[logical].phys;
    return (uint8_t *)p;
  }
  DevicePool &P = c->dev[logical].pool;
  uint64_t off;
  P.heap.reclaim();
  if (P.heap.take(len, &off)) return (uint8_t *)(P.base + off);
  bool any = false;
  for (auto &q : P.heap.quarantine) any |= all_grounded(c, q);
  if (any) {
    if (!c->replay) pump(c, true);
    for (auto &q : P.heap.quarantine)
      if (all_grounded(c, q)) host_wait(q.fences);
    P.heap.reclaim();
    if (P.heap.take(len, &off)) return (uint8_t *)(P.base + off);
  }
  if (lk && lk->owns_lock() && !c->replay) {
    // grow by a whole segment of its own without the context lock: cuMemCreate /
    // cuMemSetAccess took up to ~60 ms while copies streamed (tools/vmmlat.cu),
    // and meanwhile the dispatch thread and the other callers keep going
    const uint64_t seg = std::max<uint64_t>(len, 64ull << 20);
    uint64_t voff = 0;
    if (P.reserve(seg, voff)) {
      const CUdeviceptr base = P.base;
      const int phys = P.phys;
      const std::vector<int> access = P.access;
      lk->unlock();
      DevicePool::Seg sg{};
      bool ok = true;
      try {
        sg = DevicePool::map_seg(base, voff, seg, phys, access, true, len);
      } catch (const Error &) {
        ok = false;
      }
      lk->lock();
      if (ok) P.publish(sg);
      else P.unreserve(voff, seg);
      if (ok && P.heap.take(len, &off)) return (uint8_t *)(P.base + off);
    }
  }
  P.grow(len - std::min(len, P.heap.tail_free(P.va_top)));
  if (!P.heap.take(len, &off)) throw Error(GROUTER_ENOMEM, "pool fragmentation");
  return (uint8_t *)(P.base + off);
}

void dev_free(grouter_ctx *c, int logical, uint8_t *p, uint64_t len, Fences &&f) {
  if (!len) return;
  if (c->cfg.flags & GROUTER_NO_POOL) {  // ablation: cudaFree once the buffer's GPU work completed
    c->nopool_pending.push_back({p, std::move(f)});
    nopool_sweep(c, false);
    return;
  }
  if (!c->dedicated.empty() && ded_free(c, p, std::move(f))) return;  // an exported object's own allocation
  DevicePool &P = c->dev[logical].pool;
  uint64_t off = (uint64_t)p - P.base;
  bool done = true;
  for (auto &w : f) done &= w.done();
  if (done) P.heap.give(off, len);
  else P.heap.quarantine.push_back({off, len, std::move(f)});
}

// GROUTER_NO_POOL: cudaFree (which synchronizes the device -- the cost the
// pool exists to avoid, L248) every pending buffer whose fences completed;
// wait: first wait for all of them (shutdown).
void nopool_sweep(grouter_ctx *c, bool wait) {
  size_t k = 0;
  for (size_t i = 0; i < c->nopool_pending.size(); ++i) {
    auto &e = c->nopool_pending[i];
    bool done = true;
    if (wait) host_wait(e.f);
    else
      for (auto &w : e.f) done &= w.done();
    if (!done) {
      if (k != i) c->nopool_pending[k] = std::move(e);
      ++k;
      continue;
    }
    auto it = c->nopool_live.find(e.p);
    if (it != c->nopool_live.end()) {
      DeviceGuard g(it->second);
      GR_CUDA(cudaFree(e.p));
      c->nopool_live.erase(it);
    }
  }
  c->nopool_pending.resize(k);
}

uint8_t *host_alloc(grouter_ctx *c, uint64_t len) {
  uint64_t off;
  c->host.heap.reclaim();
  if (c->host.heap.take(len, &off)) return c->host.base + off;
  bool any = false;
  for (auto &q : c->host.heap.quarantine) any |= all_grounded(c, q);
  if (any) {
    if (!c->replay) pump(c, true);
    for (auto &q : c->host.heap.quarantine)
      if (all_grounded(c, q)) host_wait(q.fences);
    c->host.heap.reclaim();
    if (c->host.heap.take(len, &off)) return c->host.base + off;
  }
  throw Error(GROUTER_ENOMEM, "host store arena fragmented or busy");
}

void host_free(grouter_ctx *c, uint8_t *p, uint64_t len, Fences &&f) {
  if (!len) return;
  uint64_t off = (uint64_t)(p - c->host.base);
  bool done = true;
  for (auto &w : f) done &= w.done();
  if (done) c->host.heap.give(off, len);
  else c->host.heap.quarantine.push_back({off, len, std::move(f)});
}

}  // namespace gr
