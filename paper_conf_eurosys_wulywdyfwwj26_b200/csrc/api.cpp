// api.cpp -- the C ABI of include/grouter.h: object table, placement,
// authentication, refcounted lifetimes, queue-aware eviction.
//
// PAPER.md L165 (locality-aware Put, Get dispatch, one transfer per get),
// L167 (zero copy on the same GPU; allocate on the consumer GPU + NVLink;
// host data staged over parallel PCIe), L173 (id -> address/location table),
// L248-L262 (elastic pool, 50% cap, queue-aware migration, prompt removal),
// L394 (authentication by function id + workflow id).  Readings R14-R24 in
// DESIGN.md.  Byte movement is delegated to engine.cpp.
#include <unistd.h>

#include <algorithm>
#include <thread>
#include <cstring>

#include "../../include/grouter.h"
#include "../../include/grouter_testing.h"

#include <chrono>
#include <cstdio>
#include <sstream>
#include "ctx.h"
#include "kernels.h"

using namespace gr;

namespace {

struct Guard {
  grouter_ctx *c;
  std::unique_lock<std::mutex> lk;
  explicit Guard(grouter_ctx *c_) : c(c_), lk(c_->mu, std::defer_lock) {
    if (!lk.try_lock()) {
      c->lock_waiters.fetch_add(1, std::memory_order_relaxed);
      lk.lock();
      c->lock_waiters.fetch_sub(1, std::memory_order_relaxed);
    }
  }
};

grouter_status fail(grouter_status st, const char *msg) {
  set_error(msg);
  return st;
}

#define API_TRY try {
#define API_CATCH(ctx)                                                        \
  }                                                                           \
  catch (const gr::Error &e) {                                                \
    gr::set_error(e.what());                                                  \
    if (e.st == GROUTER_ECUDA && (ctx)) {                                    \
      (ctx)->sticky_error = true;                                             \
      (ctx)->submit_cv.notify_all();                                          \
    }                                                                         \
    return e.st;                                                              \
  }                                                                           \
  catch (const std::exception &e) {                                           \
    gr::set_error(e.what());                                                  \
    return GROUTER_EINVAL;                                                    \
  }

bool valid_gpu(const grouter_ctx *c, int d) { return d >= 0 && d < (int)c->cfg.n_gpus; }
bool valid_loc(const grouter_ctx *c, int d) { return d == GROUTER_HOST || valid_gpu(c, d); }

int phys_of(grouter_ctx *c, int logical) { return c->dev[logical].phys; }

bool dead(const Obj &o) { return o.state == OBJ_CONSUMED || o.state == OBJ_FREED; }

Obj *lookup_live(grouter_ctx *c, grouter_oid oid) {
  auto it = c->objects.find(oid);
  if (it == c->objects.end() || dead(it->second)) return nullptr;
  return &it->second;
}

// Resident-object counts per (wf, fid, gpu) and the pool-sizing sample of a
// placement (L250-L256, R44).
static void resident_add(grouter_ctx *c, const Obj &o, int64_t delta) {
  if (o.loc < 0) return;
  const auto key = std::make_tuple(o.wf, o.fid, o.loc);
  uint64_t &r = c->resident[key];
  r += delta;
  if (r == 0) c->resident.erase(key);  // an absent entry reads 0: bounded for short-lived workflows
}

static void observe(grouter_ctx *c, const Obj &o) {
  if (o.loc < 0) return;
  resident_add(c, o, 1);
  const auto key = std::make_tuple(o.wf, o.fid, o.loc);
  c->hists[key].observe(c->clock_fixed ? c->clock_ns : now_ns(), charge(o.n), c->resident[key]);
}

// Proactive restore (L260-L262, R42): once storage on GPU d is
// released (or its cap raised), objects migrated away from d come back while
// they fit under the cap -- objects with a next-use hint first, queue head
// first; then most recently used; then lower oid.  Stops at the first misfit.
void restore(grouter_ctx *c, int d) {
  if (!c->restore_on || d < 0) return;
  std::vector<Obj *> v;
  for (auto &kv : c->objects) {
    Obj &o = kv.second;
    if (o.loc == GROUTER_HOST && o.home == d && o.state == OBJ_SEALED && o.pins == 0 && o.n > 0)
      v.push_back(&o);
  }
  std::sort(v.begin(), v.end(), [](const Obj *a, const Obj *b) {
    if (a->has_next_use != b->has_next_use) return a->has_next_use;
    if (a->has_next_use && a->next_use != b->next_use) return a->next_use < b->next_use;
    if (a->last_access != b->last_access) return a->last_access > b->last_access;
    return a->oid < b->oid;
  });
  LogicalDev &D = c->dev[d];
  for (Obj *o : v) {
    const uint64_t ch = charge(o->n);
    if (D.cap != GROUTER_UNLIMITED && D.used + ch > D.cap) break;
    uint8_t *p = dev_alloc(c, d, ch);
    restore_copy(c, *o, d, p);   // frees the host pages behind the copy
    D.used += ch;
    c->host_used -= ch;
    o->loc = d;
    resident_add(c, *o, 1);
    o->ptr = p;
    o->home = -1;
    c->restored.push_back(o->oid);
  }
}

// Storage of a consumed/freed object goes back to its pool once no zero-copy
// lease pins it ("promptly removes intermediate data", L260).
void release_storage_if_dead(grouter_ctx *c, Obj &o) {
  if (!dead(o) || o.pins) return;
  const uint64_t ch = charge(o.n);
  Fences f = std::move(o.readers);
  for (auto &w : o.ready) f.push_back(w);
  if (o.loc == GROUTER_REMOTE) {  // imported mapping: unmap once local reads are done
    if (!c->replay) pump(c, true);
    host_wait(f);
    if (o.remote) ipc_unmap(*o.remote);
    c->objects.erase(o.oid);
    return;
  }
  if (o.loc == GROUTER_HOST) {
    c->host_used -= ch;
    host_free(c, o.ptr, ch, std::move(f));
  } else {
    const int d = o.loc;
    resident_add(c, o, -1);
    c->dev[d].used -= ch;
    dev_free(c, d, o.ptr, ch, std::move(f));
    c->objects.erase(o.oid);
    restore(c, d);
    return;
  }
  c->objects.erase(o.oid);
}

void consume(grouter_ctx *c, Obj &o) {
  if (o.consumers_left > 0 && --o.consumers_left == 0) {
    o.state = OBJ_CONSUMED;
    release_storage_if_dead(c, o);
  }
}

// Eviction order (L258 queue-aware; R15 tie-breaks): objects without a
// next-use hint first, then the TAIL of the request queue (largest
// next_use), then least recently accessed, then lower oid.
std::vector<Obj *> candidates(grouter_ctx *c, int d) {
  std::vector<Obj *> v;
  for (auto &kv : c->objects) {
    Obj &o = kv.second;
    if (o.loc == d && o.state == OBJ_SEALED && o.pins == 0 && o.n > 0) v.push_back(&o);
  }
  std::sort(v.begin(), v.end(), [](const Obj *a, const Obj *b) {
    if (a->has_next_use != b->has_next_use) return !a->has_next_use;
    if (a->has_next_use && a->next_use != b->next_use) return a->next_use > b->next_use;
    if (a->last_access != b->last_access) return a->last_access < b->last_access;
    return a->oid < b->oid;
  });
  return v;
}

// Migrates a victim to the pinned host store.
void spill(grouter_ctx *c, Obj &o) {
  const uint64_t ch = charge(o.n);
  uint8_t *h = host_alloc(c, ch);
  const int d = o.loc;
  spill_copy(c, o, h);            // D2H + device pages to quarantine
  resident_add(c, o, -1);
  o.home = d;
  o.loc = GROUTER_HOST;
  o.ptr = h;
  c->dev[d].used -= ch;
  c->host_used += ch;
  c->victims.push_back(o.oid);
}

// reserve(d, ch): admit if it fits under the cap; else evict in victim order
// until it fits -- all or nothing (no eviction when it cannot fit, or when
// the host store cannot take the victims).
bool reserve(grouter_ctx *c, int d, uint64_t ch) {
  LogicalDev &D = c->dev[d];
  if (D.cap == GROUTER_UNLIMITED || D.used + ch <= D.cap) {
    D.used += ch;
    return true;
  }
  const uint64_t need = D.used + ch - D.cap;
  uint64_t freed = 0;
  std::vector<Obj *> picked;
  for (Obj *o : candidates(c, d)) {
    picked.push_back(o);
    freed += charge(o->n);
    if (freed >= need) break;
  }
  if (freed < need || c->host_used + freed > c->host_cap) return false;
  for (Obj *o : picked) spill(c, *o);
  D.used += ch;
  return true;
}

bool host_reserve(grouter_ctx *c, uint64_t ch) {
  if (c->host_used + ch > c->host_cap) return false;
  c->host_used += ch;
  return true;
}

// Physical storage for a reservation already charged; undoes the charge on failure.
// lk: the caller's lock, which a pool growth may release (callers that hold no
// object-table reference across the call: put, alloc)
uint8_t *storage(grouter_ctx *c, int loc, uint64_t ch, std::unique_lock<std::mutex> *lk = nullptr) {
  if (!ch) return nullptr;
  try {
    return loc == GROUTER_HOST ? host_alloc(c, ch) : dev_alloc(c, loc, ch, lk);
  } catch (...) {
    if (loc == GROUTER_HOST) c->host_used -= ch;
    else c->dev[loc].used -= ch;
    throw;
  }
}

bool is_pageable(const void *p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return true;
  }
  return a.type == cudaMemoryTypeUnregistered;
}

// Blocking completion for host callers.  Replay mode: the call flushes
// (R31).  Real-time: the transfer competes in the servers'
// schedulers like any other (no forced dispatch); the context lock is
// dropped while the caller polls its completion words, so the daemon and
// other callers keep running.  Nothing touches context state afterwards.
void block_on(grouter_ctx *c, Guard &g, const Fences &f) {
  if (c->replay) {
    flush_all(c);
    host_wait(f);
    return;
  }
  const uint64_t t0 = hprof().on ? now_ns() : 0;
  pump(c, false);  // wakes the daemon itself when work stays queued (a futex wake costs ~2.6 us)
  static const bool always_notify = getenv("GR_BLOCK_NOTIFY") != nullptr;
  if (always_notify) c->cv.notify_one();
  g.lk.unlock();
  if (hprof().on) hprof().t[13] += now_ns() - t0;  // pump + daemon notify
  const uint64_t t1 = hprof().on ? now_ns() : 0;
  host_wait(f, 120.0, &c->sticky_error);
  if (hprof().on) hprof().t[15] += now_ns() - t1;
}

// Stream-ordered completion for device callers: work enqueued on `s` after
// the call sees the bytes.  A wait may only be enqueued once its producer
// is submitted, so in real-time mode the caller blocks (lock released,
// condition variable) until the servers have submitted the transfer --
// backpressure, not a forced dispatch that would bypass the tenant
// scheduler.  Replay mode: waits on unsubmitted transfers are attached to
// them and enqueued at grouter_flush() (R31).
void order_after(grouter_ctx *c, Guard &g, cudaStream_t s, const Fences &f) {
  if (!c->replay) {
    auto all_submitted = [&] {
      for (auto &w : f)
        if (!is_submitted(w)) return false;
      return true;
    };
    // a failed round (sticky error) or a shutdown never submits the rest:
    // wake up and fail instead of waiting forever (the daemon notifies)
    auto settled = [&] { return c->sticky_error.load() || c->stop || all_submitted(); };
    if (!all_submitted()) {
      pump(c, false);
      c->cv.notify_one();
      static const bool diag = getenv("GR_DIAG") != nullptr;
      if (!diag) {
        if (!c->submit_cv.wait_for(g.lk, std::chrono::seconds(120), settled))
          throw Error(GROUTER_ECUDA, "timeout waiting for a transfer's submission");
      } else {  // diagnostics: report the servers' state when a submission stalls
        const uint64_t t0 = now_ns();
        while (!c->submit_cv.wait_for(g.lk, std::chrono::milliseconds(50), settled)) {
          fprintf(stderr, "[grouter diag] order_after: transfer unsubmitted for %.0f ms\n", (now_ns() - t0) / 1e6);
          const char *kn[] = {"copy", "h2d", "d2h"};
          for (size_t i = 0; i < c->dev.size(); ++i) {
            Server *sv[] = {&c->dev[i].copy, &c->dev[i].h2d, &c->dev[i].d2h};
            for (int k = 0; k < 3; ++k) {
              Server &q = *sv[k];
              std::string inf;
              for (auto &f : q.inflight) {
                inf += f.w.done() ? "D" : "p";
                if (f.w.word) inf += "(w " + std::to_string(*f.w.word) + "/" + std::to_string(f.w.target) + ")";
              }
              fprintf(stderr, "  dev %zu %s: sched %llu carry %zu urgent %zu inflight [%s]\n", i, kn[k],
                      (unsigned long long)q.sched.backlog_items, q.carry.size(), q.urgent.size(), inf.c_str());
            }
          }
          for (auto &w : f)
            if (w.producer)
              fprintf(stderr, "  waiting on xfer %llu: %u/%u chunks submitted, %zu deps\n",
                      (unsigned long long)w.producer->id, w.producer->submitted_chunks, w.producer->nchunks,
                      w.producer->deps.size());
        }
      }
      if (!all_submitted())
        throw Error(GROUTER_ECUDA, c->stop ? "context shutting down" : "sticky CUDA error; see the first failure");
    }
  }
  caller_wait(c, s, f);
}

int server_kind_for(int src, int dst) {
  if (src == GROUTER_REMOTE) return SK_COPY;
  if (src == GROUTER_HOST) return SK_H2D;
  if (dst == GROUTER_HOST) return SK_D2H;
  return SK_COPY;
}

// Plans, enqueues and starts one transfer; returns it.  `caller` (a device
// caller's stream, else null): a same-GPU SM copy may run directly on it
// (*direct = true: stream order alone sequences it, no signal or wait
// needed); otherwise `caller_dep` adds a point on the caller's stream to the
// transfer's dependencies (the copy reads src / overwrites dst only after
// prior work on that stream).
XferRef start_transfer(grouter_ctx *c, uint32_t tenant, int src_loc, int dst_loc, uint64_t n,
                       const uint8_t *src, uint8_t *dst, Fences deps, bool pageable_src,
                       cudaStream_t caller = nullptr, int caller_logical = -1, bool caller_dep = false,
                       bool *direct = nullptr, bool pool_src = true) {
  const uint64_t tst = hprof().on ? now_ns() : 0;
  if ((c->cfg.flags & GROUTER_HOST_CENTRIC) && src_loc >= 0 && dst_loc >= 0 && src_loc != dst_loc && n &&
      pool_src) {
    // ablation "UF off" (R49): GPU -> pinned host bounce -> GPU, one engine per hop
    const uint64_t ch = charge(n);
    uint8_t *bounce = host_alloc(c, ch);  // library-internal: not charged to the host store (R49)
    std::vector<grouter_chunk> p1, p2;
    c->planner.plan_single(n, src_loc, p1);
    XferRef x1 = new_xfer(c, tenant, p1);
    x1->deps = std::move(deps);
    enqueue_plan(c, x1, p1, SK_D2H, (uint64_t)(uintptr_t)src, (uint64_t)(uintptr_t)bounce, GROUTER_HOST);
    c->planner.plan_single(n, dst_loc, p2);
    XferRef x2 = new_xfer(c, tenant, p2);
    done_fences(x1, x2->deps);
    enqueue_plan(c, x2, p2, SK_H2D, (uint64_t)(uintptr_t)bounce, (uint64_t)(uintptr_t)dst, dst_loc);
    if (caller && caller_dep) x2->deps.push_back(signal(c, caller, c->dev[caller_logical].phys));
    Fences f;
    done_fences(x2, f);
    host_free(c, bounce, ch, std::move(f));
    if (direct) *direct = false;
    if (hprof().on) hprof().t[4] += now_ns() - tst;
    pump(c, false);
    return x2;
  }
  // GROUTER_FORCE_REMOTE: a copy between two logical GPUs takes the path a
  // physical pair takes (the consumer's stream is on another device there, so
  // never a direct launch): the source's copy server pushes, the consumer
  // stream waits on the completion words
  const bool may_direct = !(c->cfg.flags & GROUTER_FORCE_REMOTE) || src_loc == dst_loc;
  if (caller && direct && n && server_kind_for(src_loc, dst_loc) == SK_COPY) {  // (small pulls: forced too)
    const int server = src_loc == GROUTER_REMOTE ? dst_loc : src_loc;
    XferRef fx = fast_direct(c, tenant, server, dst_loc, (uint64_t)(uintptr_t)src, (uint64_t)(uintptr_t)dst, n,
                             pool_src && src_loc >= 0, deps, caller, caller_logical);
    if (fx) {
      *direct = true;
      if (hprof().on) hprof().t[4] += now_ns() - tst;
      return fx;
    }
  }
  std::vector<grouter_chunk> plan;
  if (src_loc == GROUTER_REMOTE) c->planner.plan_single(n, dst_loc, plan);  // consumer GPU pulls
  else c->planner.plan(src_loc, dst_loc, n, plan, pool_src);
  const int kind0 = server_kind_for(src_loc, dst_loc);
  if (!caller && !pageable_src && (kind0 == SK_H2D || kind0 == SK_D2H)) {  // host caller, idle copy engine
    XferRef fx = fast_ce(c, tenant, kind0, plan, (uint64_t)(uintptr_t)src, (uint64_t)(uintptr_t)dst, n, deps);
    if (fx) {
      if (direct) *direct = false;
      if (hprof().on) hprof().t[4] += now_ns() - tst;
      return fx;
    }
  }
  XferRef x = new_xfer(c, tenant, plan);
  x->deps = std::move(deps);
  x->pageable_src = pageable_src;
  x->local_src = pool_src && src_loc >= 0;  // a GPU pool object, copied by that GPU's SMs
  const int kind = server_kind_for(src_loc, dst_loc);
  enqueue_plan(c, x, plan, kind, (uint64_t)(uintptr_t)src, (uint64_t)(uintptr_t)dst, dst_loc);
  if (hprof().on) hprof().t[4] += now_ns() - tst;
  if (direct) *direct = false;
  if (caller && kind == SK_COPY && direct && may_direct &&
      try_direct(c, x, src_loc == GROUTER_REMOTE ? dst_loc : src_loc, caller, c->dev[caller_logical].phys)) {
    *direct = true;
    return x;
  }
  if (caller && caller_dep) x->deps.push_back(signal(c, caller, c->dev[caller_logical].phys));
  pump(c, false);  // inline dispatch when the server has room (no-op in replay mode)
  return x;
}

bool check_ready(grouter_ctx *c) {
  if (c->sticky_error) {
    set_error("sticky CUDA error; see the first failure");
    return false;
  }
  return true;
}

}  // namespace

// O10 auto cap and the cap rule shared by set_pool_limit / refresh_cap (L262)
bool gr::apply_cap(grouter_ctx *c, int d, uint64_t bytes) {
  LogicalDev &D = c->dev[d];
  D.cap = bytes;
  if (bytes != GROUTER_UNLIMITED && D.used > bytes)
    for (Obj *o : candidates(c, d)) {  // migrate until under the new cap (L262)
      if (D.used <= D.cap) break;
      if (c->host_used + charge(o->n) > c->host_cap) break;
      spill(c, *o);
    }
  const bool ok = bytes == GROUTER_UNLIMITED || D.used <= D.cap;
  if (ok) restore(c, d);
  return ok;
}

uint64_t gr::auto_cap_bytes(uint32_t permille, uint64_t avail) {
  return (uint64_t)((unsigned __int128)avail * permille / 1000) / kPage * kPage;
}

uint64_t gr::refresh_cap(grouter_ctx *c, int d, uint64_t avail, bool *ok) {
  LogicalDev &D = c->dev[d];
  if (avail == GROUTER_AUTO_AVAIL) {  // free + the store's own device memory
    DeviceGuard g(D.phys);
    size_t fr = 0, tot = 0;
    GR_CUDA(cudaMemGetInfo(&fr, &tot));
    avail = (uint64_t)fr + D.pool.mapped;
    for (auto &kv : c->dedicated)
      if (kv.second.logical == d) avail += kv.second.size;
  }
  const uint64_t cap = auto_cap_bytes(c->cfg.pool_cap_permille, avail);
  D.auto_cap = true;
  c->stats.auto_avail[d] = avail;
  c->stats.auto_refreshes++;
  *ok = apply_cap(c, d, cap);
  return cap;
}

extern "C" {

const char *grouter_strerror(grouter_status st) {
  static const char *s[] = {"GROUTER_OK",     "GROUTER_EINVAL", "GROUTER_ENOENT", "GROUTER_EPERM",
                            "GROUTER_ENOMEM", "GROUTER_EBUSY",  "GROUTER_ECUDA",  "GROUTER_ESTATE"};
  return ((unsigned)st < 8) ? s[st] : "GROUTER_?";
}

const char *grouter_last_error(void) { return gr::last_error(); }

#ifndef GROUTER_SRC_HASH
#define GROUTER_SRC_HASH "unknown"
#endif
// the marker is found by a byte scan of the .so (_build.built_hash), no dlopen needed
static const char kSrcHashMarker[] __attribute__((used)) = "GROUTER_SRC_HASH=" GROUTER_SRC_HASH;
const char *grouter_build_hash(void) { return kSrcHashMarker + 17; }

static int64_t g_race_counter;  // deliberately unsynchronised (grouter_test_race)
static void race_body(int32_t iters) {
  for (int32_t i = 0; i < iters; ++i) {
    int64_t v = g_race_counter;
    asm volatile("" ::: "memory");
    g_race_counter = v + 1;
  }
}
// Positive control for AddressSanitizer builds: reads one element past the
// end of a heap array (an ASan build reports a heap-buffer-overflow here).
grouter_status grouter_test_oob(int32_t *out) {
  if (!out) return GROUTER_EINVAL;
  std::vector<int32_t> v(4, 7);
  volatile int32_t *p = v.data();
  *out = p[4];
  return GROUTER_OK;
}

grouter_status grouter_test_race(int32_t iters, int64_t *out) {
  if (!out || iters < 0) return GROUTER_EINVAL;
  g_race_counter = 0;
  std::thread a(race_body, iters), b(race_body, iters);
  a.join();
  b.join();
  *out = g_race_counter;
  return GROUTER_OK;
}

void grouter_config_default(grouter_config *cfg) {
  if (!cfg) return;
  std::memset(cfg, 0, sizeof(*cfg));
  for (int i = 0; i < GROUTER_MAX_GPUS; ++i) {
    cfg->device_map[i] = i;
    cfg->h2d_Bps[i] = 55000000000ull;
    cfg->h2d_alpha_ps[i] = 4000000ull;
    cfg->h2d_phi_ps[i] = 10000000ull;
    cfg->uplink_group[i] = i;  // uncalibrated: every GPU its own uplink
    for (int j = 0; j < GROUTER_MAX_GPUS; ++j) cfg->p2p[i][j] = 1;
  }
  cfg->nvl_Bps = 900000000000ull;
  cfg->relay_phi_ps = 20000000ull;
  cfg->chunk_bytes = 2ull << 20;
  cfg->batch_chunks = 5;
  cfg->granule = 4096;
  cfg->pool_floor_bytes = 300ull << 20;
  cfg->pool_cap_permille = 500;
  cfg->host_store_bytes = 1ull << 30;
  cfg->auto_cap_period_us = 20000;
  cfg->copy_ctas_per_sm = 4;
}

grouter_status grouter_init(const grouter_config *cfg_in, grouter_ctx **out) {
  if (!cfg_in || !out) return fail(GROUTER_EINVAL, "null argument");
  grouter_config cfg = *cfg_in;
  if (cfg.granule < 16 || cfg.chunk_bytes < cfg.granule || cfg.chunk_bytes % cfg.granule ||
      cfg.batch_chunks < 1 || cfg.batch_chunks > 8)
    return fail(GROUTER_EINVAL, "bad chunk/granule/batch configuration");
  if (!(cfg.flags & GROUTER_PLAN_ONLY) && cfg.n_gpus == 0) {
    int nd = 0;
    if (cudaGetDeviceCount(&nd) != cudaSuccess || nd == 0)
      return fail(GROUTER_ECUDA, "no CUDA device (the data path has no CPU fallback)");
    cfg.n_gpus = (uint32_t)std::min(nd, GROUTER_MAX_GPUS);
  }
  if (cfg.n_gpus == 0 || cfg.n_gpus > GROUTER_MAX_GPUS) return fail(GROUTER_EINVAL, "bad n_gpus");
  if (cfg.copy_ctas_per_sm == 0) cfg.copy_ctas_per_sm = 4;
  auto *c = new grouter_ctx();
  c->cfg = cfg;
  c->replay = (cfg.flags & GROUTER_REPLAY) != 0;
  c->restore_on = (cfg.flags & GROUTER_RESTORE) != 0;
  c->plan_only = (cfg.flags & GROUTER_PLAN_ONLY) != 0;
  c->planner.build(cfg);
  c->dev.resize(cfg.n_gpus);
  if (c->plan_only) {
    *out = c;
    return GROUTER_OK;
  }
  try {
    int prev = 0;
    cudaGetDevice(&prev);
    engine_init(c);
    cudaSetDevice(prev);
  } catch (const gr::Error &e) {
    set_error(e.what());
    grouter_status st = e.st;
    try {
      engine_shutdown(c);
    } catch (...) {
    }
    delete c;
    return st;
  }
  *out = c;
  return GROUTER_OK;
}

grouter_status grouter_finalize(grouter_ctx *c) {
  if (!c) return fail(GROUTER_EINVAL, "null ctx");
  if (hprof().on && (hprof().rounds[0] || hprof().rounds[1]))
    fprintf(stderr, "[grouter host profile] dispatch rounds: SM copy x%llu %.2f us each, copy engine x%llu %.2f us each\n",
            (unsigned long long)hprof().rounds[0], hprof().t[19] / std::max<uint64_t>(1, hprof().rounds[0]) / 1e3,
            (unsigned long long)hprof().rounds[1], hprof().t[20] / std::max<uint64_t>(1, hprof().rounds[1]) / 1e3);
  if (hprof().on && (hprof().calls || hprof().put_calls)) {
    HostProf &h = hprof();
    fprintf(stderr, "[grouter host profile] get_into calls %llu: lock+lookup %.2f us, transfer+launch %.2f us, "
                    "fences+consume %.2f us, ordering %.2f us\n",
            (unsigned long long)h.calls, h.t[0] / h.calls / 1e3, h.t[1] / h.calls / 1e3,
            h.t[2] / h.calls / 1e3, h.t[3] / h.calls / 1e3);
    if (g_launch_prof_n) {
      double q10, q50, q90;
      launch_prof_percentiles(&q10, &q50, &q90);
      fprintf(stderr, "[grouter host profile] launch_copy x%llu: prepare %.2f us, launch call %.2f us "
                      "(p10/p50/p90 %.2f/%.2f/%.2f), cudaGetLastError %.2f us\n",
              (unsigned long long)g_launch_prof_n, g_launch_prof[0] / g_launch_prof_n / 1e3,
              g_launch_prof[1] / g_launch_prof_n / 1e3, q10, q50, q90, g_launch_prof[2] / g_launch_prof_n / 1e3);
    }
    if (h.put_calls)
      fprintf(stderr, "[grouter host profile] blocking put calls %llu: reserve %.2f us, pageable check %.2f us, "
                      "transfer+dispatch %.2f us, observe %.2f us, block_on %.2f us (of it pump+notify %.2f us)\n",
              (unsigned long long)h.put_calls, h.t[8] / h.put_calls / 1e3, h.t[9] / h.put_calls / 1e3,
              h.t[10] / h.put_calls / 1e3, h.t[11] / h.put_calls / 1e3, h.t[12] / h.put_calls / 1e3,
              h.t[13] / h.put_calls / 1e3);
    if (h.put_calls)
      fprintf(stderr, "[grouter host profile] put call -> first H2D copy submitted %.2f us (to round %.2f, "
                      "take+guard %.2f, memcpy call %.2f), host wait %.2f us\n",
              h.t[14] / h.put_calls / 1e3, h.t[16] / h.put_calls / 1e3, h.t[17] / h.put_calls / 1e3,
              h.t[18] / h.put_calls / 1e3, h.t[15] / h.put_calls / 1e3);
    if (h.t[4] > 0)
      fprintf(stderr, "[grouter host profile] inside transfer: plan+xfer+enqueue %.2f us, take %.2f us, "
                      "params %.2f us, launch %.2f us\n",
              h.t[4] / h.calls / 1e3, h.t[5] / h.calls / 1e3, h.t[6] / h.calls / 1e3, h.t[7] / h.calls / 1e3);
  }
  if (!c->plan_only) {
    API_TRY
    ipc_shutdown(c);
    engine_shutdown(c);
    for (auto &kv : c->objects)
      if (kv.second.remote) ipc_unmap(*kv.second.remote);
    API_CATCH(c)
  }
  delete c;
  return GROUTER_OK;
}

// ------------------------------------------------------------------ put / alloc / seal
grouter_status grouter_put(grouter_ctx *c, const grouter_fn *fn, const void *src, uint64_t n,
                           int32_t hint, uint32_t consumers, void *stream, grouter_oid *out) {
  gr::NvtxRange nvtx_("grouter_put", n);
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->seq++;
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!check_ready(c)) return GROUTER_ECUDA;
  if (!fn || !out || !valid_loc(c, fn->device) ||
      !(hint == GROUTER_NOHINT || hint == GROUTER_HOST || valid_gpu(c, hint)) || (!src && n))
    return fail(GROUTER_EINVAL, "put: bad argument");
  HostProf &hp = hprof();
  uint64_t p0 = hp.on ? now_ns() : 0, p1 = 0, p2 = 0, p3 = 0, p4 = 0;
  if (hp.on) tl_put_t0 = p0;
  const int from = fn->device;
  const bool blocking = !stream || from == GROUTER_HOST;
  int home = from != GROUTER_HOST ? from : (hint >= 0 ? hint : GROUTER_HOST);  // L165, R23
  const uint64_t ch = charge(n);
  if (home != GROUTER_HOST && !reserve(c, home, ch)) home = GROUTER_HOST;    // R16
  if (home == GROUTER_HOST && !host_reserve(c, ch)) return fail(GROUTER_ENOMEM, "host store full");
  uint8_t *ptr = storage(c, home, ch, &g.lk);
  if (hp.on) p1 = p2 = now_ns();
  Obj o;
  o.oid = c->next_oid++;
  o.wf = fn->workflow_id;
  o.fid = fn->function_id;
  o.n = n;
  o.loc = home;
  o.ptr = ptr;
  o.state = OBJ_SEALED;
  o.consumers_left = consumers;
  o.last_access = c->seq;
  Fences done;
  if (n) {
    if (from == GROUTER_HOST && home == GROUTER_HOST) {
      std::memcpy(ptr, src, n);  // cFn -> host store: plain memcpy
    } else {
      bool pageable = from == GROUTER_HOST && is_pageable(src);
      if (hp.on) p2 = now_ns();
      bool direct = false;
      XferRef x;
      try {
        x = start_transfer(c, fn->workflow_id, from, home, n, (const uint8_t *)src, ptr, Fences{}, pageable,
                           blocking ? nullptr : (cudaStream_t)stream, from, true, &direct,
                           /*pool_src=*/false);  // the caller's buffer
      } catch (const Error &e) {
        if (e.st == GROUTER_ECUDA) throw;  // sticky: the context is unusable anyway
        if (home == GROUTER_HOST) {        // nothing was enqueued: give the storage back
          c->host_used -= ch;
          host_free(c, ptr, ch, Fences{});
        } else {
          c->dev[home].used -= ch;
          dev_free(c, home, ptr, ch, Fences{});
        }
        throw;
      }
      done_fences(x, done);
      o.ready = done;
      if (!blocking && !direct) order_after(c, g, (cudaStream_t)stream, done);
    }
  }
  if (hp.on) p3 = now_ns();
  *out = o.oid;
  observe(c, o);
  c->objects.emplace(o.oid, std::move(o));
  if (hp.on) p4 = now_ns();
  if (blocking && (c->replay || !done.empty())) block_on(c, g, done);
  if (hp.on && blocking) {
    const uint64_t p5 = now_ns();
    hp.put_calls++;
    hp.t[8] += p1 - p0;   // reserve + storage
    hp.t[9] += p2 - p1;   // pageable check
    hp.t[10] += p3 - p2;  // plan + transfer + dispatch
    hp.t[11] += p4 - p3;  // observe + object table
    hp.t[12] += p5 - p4;  // block_on (pump, notify, wait)
  }
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_alloc(grouter_ctx *c, const grouter_fn *fn, uint64_t n, int32_t hint,
                             uint32_t consumers, void **buf, grouter_oid *out) {
  gr::NvtxRange nvtx_("grouter_alloc", n);
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->seq++;
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!check_ready(c)) return GROUTER_ECUDA;
  if (!fn || !buf || !out || !valid_loc(c, fn->device) ||
      !(hint == GROUTER_NOHINT || hint == GROUTER_HOST || valid_gpu(c, hint)))
    return fail(GROUTER_EINVAL, "alloc: bad argument");
  const int home = fn->device;
  const uint64_t ch = charge(n);
  if (home != GROUTER_HOST ? !reserve(c, home, ch) : !host_reserve(c, ch))
    return fail(GROUTER_ENOMEM, "alloc: does not fit after eviction");
  uint8_t *ptr = storage(c, home, ch, &g.lk);
  Obj o;
  o.oid = c->next_oid++;
  o.wf = fn->workflow_id;
  o.fid = fn->function_id;
  o.n = n;
  o.loc = home;
  o.ptr = ptr;
  o.state = OBJ_OPEN;
  o.consumers_left = consumers;
  o.last_access = c->seq;
  *buf = ptr;
  *out = o.oid;
  observe(c, o);
  c->objects.emplace(o.oid, std::move(o));
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_seal(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid, void *stream) {
  gr::NvtxRange nvtx_("grouter_seal");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->seq++;
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!fn) return fail(GROUTER_EINVAL, "seal: null fn");
  auto it = c->objects.find(oid);
  if (it == c->objects.end() || dead(it->second)) return fail(GROUTER_ENOENT, "seal: unknown oid");
  Obj &o = it->second;
  if (o.wf != fn->workflow_id) return fail(GROUTER_EPERM, "seal: workflow mismatch");
  if (o.state != OBJ_OPEN) return fail(GROUTER_ESTATE, "seal: not open");
  o.state = OBJ_SEALED;
  o.last_access = c->seq;
  if (stream && o.loc != GROUTER_HOST)
    o.ready.push_back(signal(c, (cudaStream_t)stream, phys_of(c, o.loc)));
  return GROUTER_OK;
  API_CATCH(c)
}

// ------------------------------------------------------------------ get / get_into
static grouter_status get_common(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid, Obj **out) {
  if (!fn || !valid_loc(c, fn->device)) return fail(GROUTER_EINVAL, "get: bad function");
  auto it = c->objects.find(oid);
  if (it == c->objects.end() || dead(it->second)) return fail(GROUTER_ENOENT, "get: unknown oid");
  if (it->second.wf != fn->workflow_id) return fail(GROUTER_EPERM, "get: workflow mismatch (L394)");
  if (it->second.state == OBJ_OPEN) return fail(GROUTER_ENOENT, "get: object not sealed");
  // completed producer fences are dropped once: an event fence is re-queried
  // (~1 us of host time) by every later get otherwise (copies of a fence do
  // not share its completion memo)
  if (!it->second.ready.empty()) prune(it->second.ready);
  *out = &it->second;
  return GROUTER_OK;
}

grouter_status grouter_get(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid, void *stream,
                           const void **ptr, uint64_t *n_out) {
  gr::NvtxRange nvtx_("grouter_get");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->seq++;
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!check_ready(c)) return GROUTER_ECUDA;
  if (!ptr || !n_out) return fail(GROUTER_EINVAL, "get: null output");
  Obj *op = nullptr;
  grouter_status st = get_common(c, fn, oid, &op);
  if (st) return st;
  Obj &o = *op;
  const int d = fn->device;
  const bool blocking = !stream || d == GROUTER_HOST;
  const uint64_t n = o.n;
  Fences wait;
  const void *result = nullptr;
  const bool remote = o.loc == GROUTER_REMOTE;
  if (remote && d == GROUTER_HOST) return fail(GROUTER_EINVAL, "get: CPU get of an imported object");
  if (n == 0) {
    result = nullptr;
  } else if (o.loc == d || (remote && o.remote->phys == c->dev[d].phys)) {  // zero copy (L167 (1))
    o.pins++;
    result = o.ptr;
    wait = o.ready;
  } else {
    const uint64_t ch = charge(n);
    if (d == GROUTER_HOST ? !host_reserve(c, ch) : !reserve(c, d, ch))
      return fail(GROUTER_ENOMEM, "get: lease does not fit after eviction");
    // a lease that needs a new pool segment grows it without the context lock
    // (the driver calls take up to ~60 ms while copies stream; dev_alloc), so
    // the object is looked up again: freed or consumed meanwhile -> ENOENT;
    // moved (spilled, restored) -> copied from where it is now
    uint8_t *lease = storage(c, d, ch, d == GROUTER_HOST ? nullptr : &g.lk);
    if (d != GROUTER_HOST) {
      auto again = c->objects.find(oid);
      if (again == c->objects.end() || dead(again->second) || &again->second != op) {
        c->dev[d].used -= ch;
        dev_free(c, d, lease, ch, Fences{});
        return fail(GROUTER_ENOENT, "get: object freed while its lease's pages were mapped");
      }
    }
    bool direct = false;
    XferRef x;
    try {
      x = start_transfer(c, fn->workflow_id, o.loc, d, n, o.ptr, lease, o.ready, false,
                         blocking ? nullptr : (cudaStream_t)stream, d, false, &direct);
    } catch (const Error &e) {
      if (e.st == GROUTER_ECUDA) throw;  // sticky: the context is unusable anyway
      // nothing was enqueued: give the lease back before reporting (e.g. a
      // host-centric bounce that does not fit, R49)
      if (d == GROUTER_HOST) {
        c->host_used -= ch;
        host_free(c, lease, ch, Fences{});
      } else {
        c->dev[d].used -= ch;
        dev_free(c, d, lease, ch, Fences{});
      }
      throw;
    }
    Fences done;
    done_fences(x, done);
    if (o.readers.size() > 8) prune(o.readers);
    for (auto &w : done) push_fence(o.readers, w);
    Lease L{oid, o.wf, d, lease, n, done};
    c->leases[(uintptr_t)lease] = std::move(L);
    result = lease;
    if (!direct) wait = done;
  }
  o.last_access = c->seq;
  *ptr = result;
  *n_out = n;
  consume(c, o);  // may release the object's storage (quarantined behind `wait`)
  if (blocking) block_on(c, g, wait);
  else order_after(c, g, (cudaStream_t)stream, wait);
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_get_into(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid, void *dst,
                                uint64_t dst_cap, void *stream, uint64_t *n_out) {
  gr::NvtxRange nvtx_("grouter_get_into");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  HostProf &hp = hprof();
  uint64_t t0 = hp.on ? now_ns() : 0, t1 = 0, t2 = 0, t3 = 0;
  Guard g(c);
  c->seq++;
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!check_ready(c)) return GROUTER_ECUDA;
  Obj *op = nullptr;
  grouter_status st = get_common(c, fn, oid, &op);
  if (st) return st;
  Obj &o = *op;
  const uint64_t n = o.n;
  if (dst_cap < n || (!dst && n)) return fail(GROUTER_EINVAL, "get_into: dst too small");
  const int d = fn->device;
  if (o.loc == GROUTER_REMOTE && d == GROUTER_HOST)
    return fail(GROUTER_EINVAL, "get_into: CPU get of an imported object");
  const bool blocking = !stream || d == GROUTER_HOST;
  Fences wait;
  if (hp.on) t1 = t2 = now_ns();
  if (n) {
    if (o.loc == GROUTER_HOST && d == GROUTER_HOST) {
      if (c->replay) flush_all(c);
      else pump(c, true);
      host_wait(o.ready);
      std::memcpy(dst, o.ptr, n);
    } else {
      // the copy must not overwrite dst before prior work on the stream:
      // a direct launch on that stream, or a signal from it as a dependency
      bool direct = false;
      XferRef x = start_transfer(c, fn->workflow_id, o.loc, d, n, o.ptr, (uint8_t *)dst, o.ready,
                                 false, blocking ? nullptr : (cudaStream_t)stream, d, true, &direct);
      if (hp.on) t2 = now_ns();
      Fences done;
      done_fences(x, done);
      if (o.readers.size() > 8) prune(o.readers);
      for (auto &w : done) push_fence(o.readers, w);
      if (!direct) wait = done;
    }
  }
  o.last_access = c->seq;
  if (n_out) *n_out = n;
  consume(c, o);
  if (hp.on) t3 = now_ns();
  if (blocking) block_on(c, g, wait);
  else order_after(c, g, (cudaStream_t)stream, wait);
  if (hp.on) {
    const uint64_t t4 = now_ns();
    hp.calls++;
    hp.t[0] += t1 - t0;  // lock + lookup + checks
    hp.t[1] += t2 - t1;  // plan + transfer + enqueue + dispatch/launch
    hp.t[2] += t3 - t2;  // fences + consume
    hp.t[3] += t4 - t3;  // ordering
  }
  return GROUTER_OK;
  API_CATCH(c)
}

// ------------------------------------------------------------------ release / free
grouter_status grouter_release(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid,
                               const void *ptr, void *stream) {
  gr::NvtxRange nvtx_("grouter_release");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!fn || !ptr) return fail(GROUTER_EINVAL, "release: bad argument");
  const bool dev_stream = stream && fn->device != GROUTER_HOST && valid_gpu(c, fn->device);
  auto it = c->objects.find(oid);
  if (it != c->objects.end() && it->second.ptr == ptr && it->second.pins > 0) {
    Obj &o = it->second;  // zero-copy lease: drop the pin
    if (o.wf != fn->workflow_id) return fail(GROUTER_EPERM, "release: workflow mismatch");
    o.pins--;
    if (dev_stream)
      o.readers.push_back(signal(c, (cudaStream_t)stream, phys_of(c, fn->device)));
    release_storage_if_dead(c, o);
    return GROUTER_OK;
  }
  auto lt = c->leases.find((uintptr_t)ptr);
  if (lt == c->leases.end() || lt->second.oid != oid) return fail(GROUTER_EINVAL, "release: unknown lease");
  Lease &L = lt->second;
  if (L.wf != fn->workflow_id) return fail(GROUTER_EPERM, "release: workflow mismatch");
  Fences f = std::move(L.fill);
  if (dev_stream) f.push_back(signal(c, (cudaStream_t)stream, phys_of(c, fn->device)));
  const uint64_t ch = charge(L.n);
  if (L.dev == GROUTER_HOST) {
    c->host_used -= ch;
    host_free(c, L.ptr, ch, std::move(f));
    c->leases.erase(lt);
  } else {
    const int d = L.dev;
    c->dev[d].used -= ch;
    dev_free(c, d, L.ptr, ch, std::move(f));
    c->leases.erase(lt);
    restore(c, d);
  }
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_free(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid) {
  gr::NvtxRange nvtx_("grouter_free");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!fn) return fail(GROUTER_EINVAL, "free: null fn");
  Obj *o = lookup_live(c, oid);
  if (!o) return fail(GROUTER_ENOENT, "free: unknown oid");
  if (o->wf != fn->workflow_id) return fail(GROUTER_EPERM, "free: workflow mismatch");
  if (o->state == OBJ_OPEN) return fail(GROUTER_EBUSY, "free: object not sealed");
  o->state = OBJ_FREED;
  release_storage_if_dead(c, *o);
  return GROUTER_OK;
  API_CATCH(c)
}

// ------------------------------------------------------------------ cross-process handoff
grouter_status grouter_export_ipc(grouter_ctx *c, const grouter_fn *fn, grouter_oid oid,
                                  grouter_ipc_desc *desc) {
  gr::NvtxRange nvtx_("grouter_export_ipc");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!desc) return fail(GROUTER_EINVAL, "export_ipc: null desc");
  Obj *op = nullptr;
  grouter_status st = get_common(c, fn, oid, &op);
  if (st) return st;
  Obj &o = *op;
  if (o.loc < 0) return fail(GROUTER_EINVAL, "export_ipc: object is not in a GPU pool");
  if (c->cfg.flags & GROUTER_NO_POOL) return fail(GROUTER_EINVAL, "export_ipc: no pool segments (GROUTER_NO_POOL)");
  if (c->replay) flush_all(c);
  else pump(c, true);
  host_wait(o.ready);  // the importer sees finished bytes
  const bool dedicated = !o.n || c->dedicated.count((uint64_t)(uintptr_t)o.ptr);
  if (!dedicated && o.pins)
    return fail(GROUTER_EBUSY, "export_ipc: the object has zero-copy leases (export before leasing it)");
  if (!dedicated) ipc_dedicate(c, o);  // its own VMM allocation: the importer maps only this object (R52)
  ipc_serve_start(c);
  grouter_ipc_desc d{};
  d.magic = 0x47524f55u;
  d.version = 2;
  d.pid = (int32_t)getpid();
  d.ctx_id = c->ctx_id;
  cudaDeviceProp prop;
  GR_CUDA(cudaGetDeviceProperties(&prop, c->dev[o.loc].phys));
  std::memcpy(d.gpu_uuid, &prop.uuid, 16);
  d.workflow_id = o.wf;
  d.logical = o.loc;
  d.oid = oid;
  d.n = o.n;
  d.exporter_ptr = (uint64_t)(uintptr_t)o.ptr;
  if (o.n) {
    d.export_id = ipc_export_record(c, (uint64_t)(uintptr_t)o.ptr, d.nonce);
    d.alloc_bytes = charge(o.n);
  }
  o.pins++;  // like a zero-copy lease: released with grouter_release(ptr = exporter_ptr)
  o.last_access = c->seq;
  *desc = d;
  consume(c, o);
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_import_ipc(grouter_ctx *c, const grouter_fn *fn, const grouter_ipc_desc *d,
                                  uint32_t consumers, grouter_oid *out) {
  gr::NvtxRange nvtx_("grouter_import_ipc");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!fn || !d || !out || d->magic != 0x47524f55u || d->version != 2 || (d->n && d->alloc_bytes < d->n))
    return fail(GROUTER_EINVAL, "import_ipc: bad descriptor");
  if (!valid_loc(c, fn->device)) return fail(GROUTER_EINVAL, "import_ipc: bad function");
  if (d->workflow_id != fn->workflow_id) return fail(GROUTER_EPERM, "import_ipc: workflow mismatch (L394)");
  // which local GPU (if any) holds the bytes
  int local_phys = -1;
  for (auto &kv : c->phys) {
    cudaDeviceProp prop;
    GR_CUDA(cudaGetDeviceProperties(&prop, kv.first));
    if (std::memcmp(&prop.uuid, d->gpu_uuid, 16) == 0) local_phys = kv.first;
  }
  std::shared_ptr<RemoteMap> map;
  if (d->n) {
    // the round trip to the exporter runs WITHOUT our lock: two contexts may
    // import from each other at once, and each server thread needs its
    // context's lock to look its segments up
    g.lk.unlock();
    try {
      map = ipc_map(c, *d, local_phys);
    } catch (...) {
      g.lk.lock();
      throw;
    }
    g.lk.lock();
  } else {
    map = std::make_shared<RemoteMap>();
  }
  Obj o;
  o.oid = c->next_oid++;
  o.wf = fn->workflow_id;
  o.fid = fn->function_id;
  o.n = d->n;
  o.loc = GROUTER_REMOTE;
  o.ptr = d->n ? (uint8_t *)(uintptr_t)map->va : nullptr;
  o.state = OBJ_SEALED;
  o.consumers_left = consumers;
  o.last_access = c->seq;
  o.remote = map;
  *out = o.oid;
  c->objects.emplace(o.oid, std::move(o));
  return GROUTER_OK;
  API_CATCH(c)
}

// ------------------------------------------------------------------ control
static grouter_status reweight_slos(grouter_ctx *c);

grouter_status grouter_set_tenant_weight(grouter_ctx *c, uint32_t wf, uint32_t w) {
  if (!c) return fail(GROUTER_EINVAL, "null ctx");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  if (w < 1) return fail(GROUTER_EINVAL, "weight must be >= 1");
  c->weights[wf] = w;
  if (c->slos.erase(wf)) return reweight_slos(c);  // an explicit weight replaces an SLO (R43)
  return GROUTER_OK;
}

// Rate_least (L195) = ceil(data * 1e9 / (slo - infer)) B/s; Rate_idle (L197)
// to the tightest SLO (L227); weight = rate in MiB/s rounded up (R43).
grouter_status grouter_slo_weights(uint32_t n, const uint32_t *ids, const uint64_t *data,
                                   const uint64_t *slo, const uint64_t *infer, uint64_t bw_all,
                                   uint32_t *out) {
  if (n && (!ids || !data || !slo || !infer || !out)) return fail(GROUTER_EINVAL, "slo_weights: null");
  std::vector<unsigned __int128> least(n);
  unsigned __int128 sum = 0;
  uint32_t tight = 0;
  for (uint32_t i = 0; i < n; ++i) {
    if (slo[i] <= infer[i]) return fail(GROUTER_EINVAL, "slo_weights: slo_ns <= infer_ns");
    const unsigned __int128 num = (unsigned __int128)data[i] * 1000000000u, den = slo[i] - infer[i];
    least[i] = (num + den - 1) / den;
    sum += least[i];
    if (slo[i] < slo[tight] || (slo[i] == slo[tight] && ids[i] < ids[tight])) tight = i;
  }
  const unsigned __int128 idle = sum < bw_all ? bw_all - sum : 0;
  for (uint32_t i = 0; i < n; ++i) {
    const unsigned __int128 rate = least[i] + (i == tight ? idle : 0);
    unsigned __int128 w = (rate + (1u << 20) - 1) >> 20;
    if (w < 1) w = 1;
    if (w > 0xFFFFFFFFu) w = 0xFFFFFFFFu;
    out[i] = (uint32_t)w;
  }
  return GROUTER_OK;
}

grouter_status grouter_set_tenant_slo(grouter_ctx *c, uint32_t wf, uint64_t data, uint64_t slo_ns,
                                      uint64_t infer_ns) {
  if (!c) return fail(GROUTER_EINVAL, "null ctx");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  if (data == 0) {
    c->slos.erase(wf);
    c->weights.erase(wf);
  } else {
    if (slo_ns <= infer_ns) return fail(GROUTER_EINVAL, "set_tenant_slo: slo_ns <= infer_ns");
    c->slos[wf] = {data, slo_ns, infer_ns};
  }
  return reweight_slos(c);
}

static grouter_status reweight_slos(grouter_ctx *c) {
  const uint32_t n = (uint32_t)c->slos.size();
  std::vector<uint32_t> ids, w(n);
  std::vector<uint64_t> d, s, inf;
  for (auto &kv : c->slos) {
    ids.push_back(kv.first);
    d.push_back(kv.second[0]);
    s.push_back(kv.second[1]);
    inf.push_back(kv.second[2]);
  }
  uint64_t bw_all = 0;
  for (uint32_t i = 0; i < c->cfg.n_gpus; ++i) bw_all += c->cfg.h2d_Bps[i];
  grouter_status st = grouter_slo_weights(n, ids.data(), d.data(), s.data(), inf.data(), bw_all, w.data());
  if (st) return st;
  for (uint32_t i = 0; i < n; ++i) c->weights[ids[i]] = w[i];
  return GROUTER_OK;
}

grouter_status grouter_set_next_use(grouter_ctx *c, grouter_oid oid, uint64_t pos) {
  if (!c) return fail(GROUTER_EINVAL, "null ctx");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  Obj *o = lookup_live(c, oid);
  if (!o) return fail(GROUTER_ENOENT, "set_next_use: unknown oid");
  o->has_next_use = true;
  o->next_use = pos;
  return GROUTER_OK;
}

grouter_status grouter_set_pool_limit(grouter_ctx *c, int32_t d, uint64_t bytes) {
  gr::NvtxRange nvtx_("grouter_set_pool_limit");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!valid_gpu(c, d)) return fail(GROUTER_EINVAL, "set_pool_limit: bad device");
  c->dev[d].auto_cap = false;
  return apply_cap(c, d, bytes) ? GROUTER_OK : fail(GROUTER_ENOMEM, "pool above cap");
  API_CATCH(c)
}

grouter_status grouter_refresh_cap(grouter_ctx *c, int32_t d, uint64_t avail, uint64_t *cap_out) {
  gr::NvtxRange nvtx_("grouter_refresh_cap");
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (!valid_gpu(c, d)) return fail(GROUTER_EINVAL, "refresh_cap: bad device");
  bool ok = false;
  const uint64_t cap = refresh_cap(c, d, avail, &ok);
  if (cap_out) *cap_out = cap;
  return ok ? GROUTER_OK : fail(GROUTER_ENOMEM, "pool above cap");
  API_CATCH(c)
}

grouter_status grouter_flush(grouter_ctx *c) {
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  c->victims.clear();
  c->restored.clear();
  API_TRY
  if (c->replay) flush_all(c);
  else pump(c, true);
  return GROUTER_OK;
  API_CATCH(c)
}

grouter_status grouter_sync(grouter_ctx *c) {
  if (!c || c->plan_only) return fail(GROUTER_EINVAL, "no data-path context");
  Guard g(c);
  API_TRY
  if (!c->replay) pump(c, true);
  for (auto &d : c->dev) {
    DeviceGuard dg(d.phys);
    for (Server *s : {&d.copy, &d.h2d, &d.d2h}) {
      if (s->stream) GR_CUDA(cudaStreamSynchronize(s->stream));
      if (s->fwd_stream) GR_CUDA(cudaStreamSynchronize(s->fwd_stream));
    }
  }
  return c->sticky_error ? GROUTER_ECUDA : GROUTER_OK;
  API_CATCH(c)
}

// ------------------------------------------------------------------ introspection
grouter_status grouter_plan(grouter_ctx *c, int32_t src, int32_t dst, uint64_t n, grouter_chunk *out,
                            uint64_t cap, uint64_t *n_out) {
  if (!c || !n_out) return fail(GROUTER_EINVAL, "null argument");
  if (!valid_loc(c, src) || !valid_loc(c, dst)) return fail(GROUTER_EINVAL, "plan: bad location");
  std::vector<grouter_chunk> plan;
  c->planner.plan(src, dst, n, plan);
  *n_out = plan.size();
  if (plan.size() > cap || (!out && !plan.empty())) return fail(GROUTER_EINVAL, "plan: cap too small");
  if (!plan.empty()) std::memcpy(out, plan.data(), plan.size() * sizeof(grouter_chunk));
  return GROUTER_OK;
}

grouter_status grouter_route_set(grouter_ctx *c, int32_t d, int32_t *out, uint32_t cap, uint32_t *n_out) {
  if (!c || !n_out) return fail(GROUTER_EINVAL, "null argument");
  if (!valid_gpu(c, d)) return fail(GROUTER_EINVAL, "route_set: bad device");
  const auto &R = c->planner.routes[d];
  *n_out = (uint32_t)R.size();
  if (R.size() > cap || !out) return fail(GROUTER_EINVAL, "route_set: cap too small");
  for (size_t i = 0; i < R.size(); ++i) out[i] = R[i];
  return GROUTER_OK;
}

grouter_status grouter_where(grouter_ctx *c, grouter_oid oid, int32_t *loc) {
  if (!c || !loc) return fail(GROUTER_EINVAL, "null argument");
  Guard g(c);
  auto it = c->objects.find(oid);
  if (it == c->objects.end()) return fail(GROUTER_ENOENT, "where: unknown oid");
  *loc = it->second.loc;
  return GROUTER_OK;
}

grouter_status grouter_tenant_stats(grouter_ctx *c, uint32_t workflow_id, uint64_t bytes[3]) {
  if (!c || !bytes) return fail(GROUTER_EINVAL, "null argument");
  Guard g(c);
  auto it = c->tenant_bytes.find(workflow_id);
  for (int k = 0; k < 3; ++k) bytes[k] = it == c->tenant_bytes.end() ? 0 : it->second[k];
  return GROUTER_OK;
}

grouter_status grouter_tenant_rate(grouter_ctx *c, uint32_t wf, uint64_t window_ns, uint64_t *rate_Bps,
                                   uint64_t *rate_least_Bps, int32_t *backlogged) {
  if (!c || !rate_Bps || !rate_least_Bps || !backlogged) return fail(GROUTER_EINVAL, "null argument");
  if (window_ns < 1000000ull || window_ns > 10000000000ull) return fail(GROUTER_EINVAL, "tenant_rate: window");
  Guard g(c);
  const uint64_t now = c->clock_fixed ? c->clock_ns : now_ns();
  unsigned __int128 bytes = 0;
  auto it = c->tenant_log.find(wf);
  if (it != c->tenant_log.end())
    for (auto r = it->second.rbegin(); r != it->second.rend() && r->first + window_ns > now; ++r) bytes += r->second;
  *rate_Bps = (uint64_t)(bytes * 1000000000u / window_ns);
  uint64_t least = 0;
  auto s = c->slos.find(wf);
  if (s != c->slos.end()) {
    const unsigned __int128 num = (unsigned __int128)s->second[0] * 1000000000u, den = s->second[1] - s->second[2];
    least = (uint64_t)((num + den - 1) / den);
  }
  *rate_least_Bps = least;
  int32_t bl = 0;
  for (auto &d : c->dev)
    for (Server *sv : {&d.copy, &d.h2d, &d.d2h}) {
      auto t = sv->sched.tenants.find(wf);
      if (t != sv->sched.tenants.end() && !t->second.q.empty()) bl = 1;
      for (auto &ci : sv->carry) bl |= ci.x->tenant == wf;
    }
  *backlogged = bl;
  return GROUTER_OK;
}

grouter_status grouter_stats(grouter_ctx *c, grouter_stats_t *out) {
  if (!c || !out) return fail(GROUTER_EINVAL, "null argument");
  Guard g(c);
  if (!c->plan_only) {
    API_TRY
    harvest_profile(c, false);
    API_CATCH(c)
  }
  *out = c->stats;
  for (size_t i = 0; i < c->dev.size(); ++i) {
    out->used[i] = c->dev[i].used;
    out->cap[i] = c->dev[i].cap;
    out->mapped[i] = c->dev[i].pool.mapped;
    out->pool_target[i] = pool_target(c, (int)i);
    if (c->dev[i].auto_cap) out->auto_mode |= 1u << i;
  }
  out->host_used = c->host_used;
  out->host_cap = c->host_cap;
  out->tracked_functions = c->hists.size();
  out->tracked_tenants = c->tenant_bytes.size();
  return GROUTER_OK;
}

grouter_status grouter_pool_target(grouter_ctx *c, int32_t d, uint64_t *target) {
  if (!c || !target) return fail(GROUTER_EINVAL, "pool_target: null argument");
  Guard g(c);
  if (d < 0 || d >= (int)c->dev.size()) return fail(GROUTER_EINVAL, "pool_target: bad device");
  *target = pool_target(c, d);
  return GROUTER_OK;
}

grouter_status grouter_test_inject(grouter_ctx *c, int32_t what, int32_t count) {
  if (!c || what != 1 || count < 0) return fail(GROUTER_EINVAL, "test_inject: bad argument");
  Guard g(c);
  c->inject_round_failures = count;
  return GROUTER_OK;
}

grouter_status grouter_test_set_clock(grouter_ctx *c, int32_t fixed, uint64_t t_ns) {
  if (!c) return fail(GROUTER_EINVAL, "null ctx");
  Guard g(c);
  c->clock_fixed = fixed != 0;
  c->clock_ns = t_ns;
  return GROUTER_OK;
}

grouter_status grouter_restored(grouter_ctx *c, grouter_oid *out, uint64_t cap, uint64_t *n_out) {
  if (!c || !n_out) return fail(GROUTER_EINVAL, "restored: bad argument");
  Guard g(c);
  *n_out = c->restored.size();
  if (c->restored.size() > cap || (!out && !c->restored.empty()))
    return fail(GROUTER_EINVAL, "restored: cap too small");
  for (size_t i = 0; i < c->restored.size(); ++i) out[i] = c->restored[i];
  c->restored.clear();
  return GROUTER_OK;
}

grouter_status grouter_victims(grouter_ctx *c, grouter_oid *out, uint64_t cap, uint64_t *n_out) {
  if (!c || !n_out) return fail(GROUTER_EINVAL, "null argument");
  Guard g(c);
  *n_out = c->victims.size();
  if (c->victims.size() > cap || (!out && !c->victims.empty()))
    return fail(GROUTER_EINVAL, "victims: cap too small");
  for (size_t i = 0; i < c->victims.size(); ++i) out[i] = c->victims[i];
  c->victims.clear();
  return GROUTER_OK;
}

grouter_status grouter_dispatch_log(grouter_ctx *c, grouter_dispatch *out, uint64_t cap, uint64_t *n_out) {
  if (!c || !n_out) return fail(GROUTER_EINVAL, "null argument");
  Guard g(c);
  uint64_t k = 0;
  while (k < cap && !c->dlog.empty() && out) {
    out[k++] = c->dlog.front();
    c->dlog.pop_front();
  }
  *n_out = k;
  return GROUTER_OK;
}

// ------------------------------------------------------------------ standalone scheduler
struct grouter_sched {
  struct Item {
    uint64_t id, bytes;
  };
  gr::Stride<Item> s;
  std::map<uint32_t, uint32_t> w;
};

grouter_status grouter_sched_new(uint32_t batch, grouter_sched **out) {
  if (!out || batch < 1 || batch > 8) return fail(GROUTER_EINVAL, "sched_new: bad argument");
  *out = new grouter_sched();
  (*out)->s.batch = batch;
  return GROUTER_OK;
}

grouter_status grouter_sched_set_weight(grouter_sched *s, uint32_t t, uint32_t w) {
  if (!s || w < 1) return fail(GROUTER_EINVAL, "sched_set_weight: bad argument");
  s->w[t] = w;
  return GROUTER_OK;
}

grouter_status grouter_sched_enqueue(grouter_sched *s, uint32_t t, uint64_t id, uint64_t bytes) {
  if (!s) return fail(GROUTER_EINVAL, "null sched");
  s->s.enqueue(t, {id, bytes});
  return GROUTER_OK;
}

grouter_status grouter_sched_dispatch(grouter_sched *s, uint32_t *tenant, uint64_t *ids, uint32_t *n,
                                      uint64_t *bytes, uint64_t *pass_after) {
  if (!s || !tenant || !ids || !n || !bytes || !pass_after) return fail(GROUTER_EINVAL, "null argument");
  std::vector<grouter_sched::Item> b;
  uint32_t t = s->s.dispatch(
      [&](uint32_t x) {
        auto it = s->w.find(x);
        return it == s->w.end() ? 1u : it->second;
      },
      b, bytes, pass_after);
  if (t == UINT32_MAX) return GROUTER_ENOENT;
  *tenant = t;
  *n = (uint32_t)b.size();
  for (size_t i = 0; i < b.size(); ++i) ids[i] = b[i].id;
  return GROUTER_OK;
}

grouter_status grouter_sched_account_solo(grouter_sched *s, uint32_t tenant, uint64_t n, uint64_t chunk) {
  if (!s || !chunk) return fail(GROUTER_EINVAL, "sched_account_solo: bad argument");
  auto it = s->w.find(tenant);
  s->s.account_solo(tenant, n, chunk, it == s->w.end() ? 1u : it->second);
  return GROUTER_OK;
}

void grouter_sched_free(grouter_sched *s) { delete s; }

static void dump_fences(std::ostringstream &o, grouter_ctx *c, const Fences &f) {
  o << "[";
  for (auto &w : f) {
    if (w.word)
      o << " w" << (w.word - c->words) << "=" << *w.word << "/" << w.target << (w.done() ? "ok" : "WAIT");
    else if (w.ev)
      o << " ev" << (w.done() ? "ok" : "WAIT");
    o << "@" << w.epoch;
  }
  o << " ]";
}

grouter_status grouter_test_dump(grouter_ctx *c, char *buf, uint64_t cap, uint64_t *len) {
  if (!c) return GROUTER_EINVAL;
  Guard g(c);
  std::ostringstream o;
  o << "epoch " << c->epoch << " replay " << c->replay << " sticky " << c->sticky_error << "\n";
  for (size_t i = 0; i < c->dev.size(); ++i) {
    auto &d = c->dev[i];
    o << "dev " << i << " phys " << d.phys << " used " << d.used << " cap " << d.cap << " mapped "
      << d.pool.mapped << " quarantine " << d.pool.heap.quarantine.size() << "\n";
    for (Server *s : {&d.copy, &d.h2d, &d.d2h}) {
      o << "  server " << s->kind << " backlog " << s->sched.backlog_items << " inflight";
      for (auto &e : s->inflight) o << (e.w.done() ? " done" : " busy") << (e.direct ? "(direct)" : "");
      if (s->stream) o << " stream " << (cudaStreamQuery(s->stream) == cudaSuccess ? "idle" : "busy");
      if (s->fwd_stream) o << " fwd " << (cudaStreamQuery(s->fwd_stream) == cudaSuccess ? "idle" : "busy");
      o << "\n";
    }
  }
  for (auto &kv : c->objects) {
    const Obj &ob = kv.second;
    o << "obj " << ob.oid << " loc " << ob.loc << " n " << ob.n << " state " << ob.state << " pins "
      << ob.pins << " ready";
    dump_fences(o, c, ob.ready);
    o << " readers";
    dump_fences(o, c, ob.readers);
    o << "\n";
  }
  for (auto &kv : c->leases) {
    o << "lease " << kv.first << " oid " << kv.second.oid << " dev " << kv.second.dev << " fill";
    dump_fences(o, c, kv.second.fill);
    o << "\n";
  }
  for (uint32_t sl = 0; sl < c->n_slots; ++sl)
    for (int p = 0; p < GROUTER_MAX_PATHS; ++p) {
      uint32_t w = c->words[sl * GROUTER_MAX_PATHS + p];
      if ((int32_t)(w - c->slot_final[sl][p]) < 0)
        o << "pending slot " << sl << " path " << p << " word " << w << " final " << c->slot_final[sl][p] << "\n";
    }
  std::string str = o.str();
  if (len) *len = str.size();
  if (buf && cap) {
    uint64_t k = std::min<uint64_t>(cap - 1, str.size());
    std::memcpy(buf, str.data(), k);
    buf[k] = 0;
  }
  return GROUTER_OK;
}

}  // extern "C"
