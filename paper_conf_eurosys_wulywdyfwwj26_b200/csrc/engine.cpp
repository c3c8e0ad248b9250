// engine.cpp -- per-GPU servers: stride-ordered dispatch rounds, copy
// engines, SM copy/forward kernels, completion words, the daemon thread.
//
// chunks are "pipelined across GPU streams, with
// synchronization primitives ensuring in-order delivery".  L229: batches of
// 5 chunks so new functions preempt at batch boundaries; a circular pinned
// buffer is reused across batches.  L269-L271: one daemon per GPU with
// several streams for the different directions, plus an I/O thread that
// reclaims memory; fixed PCIe routes generated at init.
//
// B200 design:
//  * A transfer owns a completion SLOT of <= 8 u32 words in pinned,
//    host-mapped memory, one per path.  Producers publish ABSOLUTE values
//    (the host knows how many of the transfer's path-p chunks each round
//    carries): SM kernels with st.release.sys from the round's last CTA, copy
//    engines with cuStreamWriteValue32 after their memcpys (on the server's
//    publish stream behind an event, so the write's memory barrier does not
//    idle the copy engine).  Consumers wait
//    with cuStreamWaitValue32(GEQ) on their own stream, or poll from the
//    host -- no host round trip on the data path, no partial visibility.
//  * Each server (SM-copy egress of a GPU, H2D engine of a route GPU, D2H
//    engine) owns a Stride scheduler; a ROUND = ONE batch in stride order
//    (plus urgent unscheduled work), executed by one kernel launch (SM copy)
//    or one memcpy burst (CE).  <= 2 rounds -- so <= 2 batches, SURVEY O8 --
//    in flight per server in real-time mode; replay mode dispatches only at
//    grouter_flush().  Exceptions on an SM-copy server with nothing else
//    queued (R53 direct launches, R55 rounds of up to 7 batches of the one
//    queued transfer): a newcomer waits behind <= 2 of those.
//  * Host->GPU relay: CE copies a route's chunks of a round into consecutive
//    staging slots on route GPU r (one 2-D copy), an event hands them to r's
//    forward stream, one forward launch pushes them over NVLink into the
//    lease on d (the path's last chunk alone, so the tail is one chunk's
//    forward) and the launch with the last chunk publishes the word; the
//    slots are reused after that launch's event.
#include <algorithm>
#include <cstdio>
#include <chrono>
#include <cstring>
#include <thread>

#include <sys/prctl.h>

#include "ce_run.h"
#include "ctx.h"
#include "kernels.h"

namespace gr {

struct CopyParamsHost {
  CopyParams p;
};

static const uint32_t kSlots = 4096;
static const size_t kRoundItems = 1024;         // chunks popped per server-stream round
static const size_t kDirectItems = 1 << 16;     // direct launches: a whole transfer
static const uint64_t kDirectBytes = 4ull << 30;
XferRef new_xfer_slot(grouter_ctx *c, const std::vector<grouter_chunk> &plan);
static const uint32_t kBounceSlots = 16;

// ------------------------------------------------------------------ waits
// Deadlock rule: a stream wait (cuStreamWaitValue32 / cudaStreamWaitEvent) is
// only ever enqueued once the GPU work that satisfies it has been SUBMITTED.
// Streams share hardware channels, so a wait enqueued ahead of its producer
// can park the very channel the producer would run on.
bool is_submitted(const Waitable &w) { return !w.producer || w.producer->submitted(); }

bool grounded(const grouter_ctx *c, const Fences &f) {
  if (!c->replay) return true;
  for (auto &w : f)
    if (w.epoch >= c->epoch && !w.done()) return false;
  return true;
}

void stream_wait(grouter_ctx *c, cudaStream_t s, int phys, const Fences &f) {
  (void)c;
  (void)phys;
  for (auto &w : f) {
    if (w.done()) continue;  // fast path: already satisfied, no GPU wait
    if (!is_submitted(w)) throw Error(GROUTER_ECUDA, "internal: wait before submission");
    if (w.word) {
      GR_CU(drv().streamWaitValue32((CUstream)s, (CUdeviceptr)(uintptr_t)w.word, w.target,
                                    CU_STREAM_WAIT_VALUE_GEQ));
    } else if (w.ev) {
      GR_CUDA(cudaStreamWaitEvent(s, w.ev->ev, 0));
    }
  }
}

void caller_wait(grouter_ctx *c, cudaStream_t s, const Fences &f) {
  for (auto &w : f) {
    if (w.done()) continue;
    if (is_submitted(w)) stream_wait(c, s, -1, Fences{w});
    else w.producer->waiters.push_back({s, w});
  }
}

static Waitable ev_wait(grouter_ctx *c, EventRef e) {
  Waitable w;
  w.ev = std::move(e);
  w.epoch = c->epoch;
  return w;
}

EventRef record(grouter_ctx *c, cudaStream_t s, int phys) {
  EventRef e = c->phys.at(phys)->events.get();
  GR_CUDA(cudaEventRecord(e->ev, s));
  return e;
}

// A point on a CALLER's stream: an event recorded there (the caller's runtime
// and this library's share the device's primary context; the fast direct path
// records its completion on caller streams the same way).  Round 1 wrote a
// completion word from the caller's stream instead: cuStreamWriteValue32
// carries a memory barrier that idles the stream ~3.5-5 us (tools/ce2.cu; the
// launch_round note above), which every seal / release / stream-ordered put
// of a function would have paid on its own stream.
// A point on a caller's stream: "the work enqueued there so far".  When the
// stream is idle right now that point has passed, and the fence is the
// completed (empty) one: no event, and no cross-stream wait for whoever
// depends on it (a push on the source GPU's server stream would otherwise
// wait on an event of the consumer's stream, one more hand-off between
// engines -- between devices on a GPU pair).
Waitable signal(grouter_ctx *c, cudaStream_t s, int phys) {
  static const bool no_skip = getenv("GR_NO_IDLE_SKIP") != nullptr;
  DeviceGuard g(phys);  // a fresh pooled event is created on the current device
  if (!no_skip) {
    const cudaError_t q = cudaStreamQuery(s);
    if (q == cudaSuccess) return Waitable{};
    if (q != cudaErrorNotReady) cudaGetLastError();  // e.g. a stream under graph capture: record below
  }
  Waitable w = ev_wait(c, record(c, s, phys));
  w.origin = s;
  return w;
}

void host_wait(const Fences &f, double timeout_s, const std::atomic<bool> *abort) {
  auto t0 = std::chrono::steady_clock::now();
  for (auto &w : f) {
    if (w.ev && !w.word) {
      // event fence (a direct launch or a whole CE round): spin on the query
      // for a short transfer's worth of time, then block in the driver
      bool ok = false;
      for (int k = 0; k < 24 && !ok; ++k) ok = w.done();
      if (!ok) GR_CUDA(cudaEventSynchronize(w.ev->ev));
      continue;
    }
    uint32_t spins = 0;
    while (!w.done()) {
      if (++spins > 64) std::this_thread::yield();
      if ((spins & 1023) == 0) {
        if (abort && abort->load(std::memory_order_relaxed))
          throw Error(GROUTER_ECUDA, "sticky CUDA error while waiting for a transfer");
        double dt = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (dt > timeout_s) throw Error(GROUTER_ECUDA, "timeout waiting for a transfer");
      }
    }
  }
}

// ------------------------------------------------------------------ transfers
void done_fences(const XferRef &x, Fences &f) {
  if (x->done_ev) {
    Waitable w;
    w.ev = x->done_ev;
    w.epoch = x->epoch;
    w.origin = x->done_stream;
    f.push_back(w);
    return;
  }
  x->word_fenced = true;
  for (uint32_t p = 0; p < x->npath; ++p) {
    if (!x->total[p]) continue;
    Waitable w;
    w.word = &x->words[p];
    w.target = x->target[p];
    w.epoch = x->epoch;
    w.producer = x;
    f.push_back(w);
  }
}

bool Xfer::done() const {
  if (done_ev) {
    if (done_ev->fired.load(std::memory_order_relaxed)) return true;
    if (cudaEventQuery(done_ev->ev) != cudaSuccess) return false;
    done_ev->fired.store(true, std::memory_order_relaxed);
    return true;
  }
  for (uint32_t p = 0; p < npath; ++p)
    if (total[p] && (int32_t)(words[p] - target[p]) < 0) return false;
  return true;
}

XferRef new_xfer(grouter_ctx *c, uint32_t tenant, const std::vector<grouter_chunk> &plan) {
  XferRef x = new_xfer_slot(c, plan);
  x->id = ++c->xfer_seq;
  x->tenant = tenant;
  c->stats.xfer_count++;
  return x;
}

// Completion slot for `plan` (one word per path) without a transfer id.
XferRef new_xfer_slot(grouter_ctx *c, const std::vector<grouter_chunk> &plan) {
  auto x = std::make_shared<Xfer>();
  x->epoch = c->epoch;
  uint32_t np = 1;
  for (auto &ch : plan) {
    x->total[ch.path]++;
    np = std::max<uint32_t>(np, (uint32_t)ch.path + 1);
  }
  x->npath = np;
  x->nchunks = (uint32_t)plan.size();
  // a slot is reusable once its previous user has completed
  for (uint32_t tries = 0; tries < c->n_slots; ++tries) {
    uint32_t s = c->next_slot;
    c->next_slot = (c->next_slot + 1) % c->n_slots;
    volatile uint32_t *w = c->words + (uint64_t)s * GROUTER_MAX_PATHS;
    bool free_ = true;
    for (int p = 0; p < GROUTER_MAX_PATHS; ++p)
      if ((int32_t)(w[p] - c->slot_final[s][p]) < 0) free_ = false;
    if (!free_) continue;
    x->slot = s;
    x->words = w;
    for (uint32_t p = 0; p < np; ++p) {
      x->target[p] = c->slot_final[s][p] + x->total[p];
      c->slot_final[s][p] = x->target[p];
    }
    return x;
  }
  throw Error(GROUTER_EBUSY, "no free completion slot (too many transfers in flight)");
}

static Server &server_of(grouter_ctx *c, int kind, int logical) {
  LogicalDev &d = c->dev[logical];
  return kind == SK_COPY ? d.copy : kind == SK_H2D ? d.h2d : d.d2h;
}

static ChunkItem make_item(const XferRef &x, uint32_t i, const grouter_chunk &ch, uint64_t src_base,
                           uint64_t dst_base, int dst_logical) {
  ChunkItem it;
  it.x = x.get();
  it.idx = i;
  it.path = (uint32_t)ch.path;
  it.src = src_base + ch.offset;
  it.dst = dst_base + ch.offset;
  it.bytes = ch.bytes;
  it.dst_logical = dst_logical;
  return it;
}

void enqueue_plan(grouter_ctx *c, const XferRef &x, const std::vector<grouter_chunk> &plan, int kind,
                  uint64_t src_base, uint64_t dst_base, int dst_logical) {
  if (!plan.empty()) c->live.emplace(x.get(), x);
  for (uint32_t i = 0; i < plan.size(); ++i)
    server_of(c, kind, plan[i].route_gpu)
        .sched.enqueue(x->tenant, make_item(x, i, plan[i], src_base, dst_base, dst_logical));
}

// ------------------------------------------------------------------ rounds
static uint32_t weight_of(grouter_ctx *c, uint32_t t) {
  auto it = c->weights.find(t);
  return it == c->weights.end() ? 1u : it->second;
}

static void retire(Server &s);
static inline void cpu_relax() {
#if defined(__x86_64__) || defined(__i386__)
  __builtin_ia32_pause();
#else
  std::this_thread::yield();
#endif
}

static void log_batch(grouter_ctx *c, Server &s, uint32_t tenant,
                      const std::vector<ChunkItem> &b, uint64_t bytes) {
  if (!(c->replay || (c->cfg.flags & GROUTER_LOG))) return;
  grouter_dispatch d{};
  if (!c->replay) {  // batches still in flight on this server (logging mode only: retire costs queries)
    retire(s);
    for (auto &f : s.inflight) d.inflight += f.batches;
  }
  d.server_kind = s.kind;
  d.server_dev = s.logical;
  d.tenant = tenant;
  d.n_chunks = (uint32_t)b.size();
  for (size_t i = 0; i < b.size() && i < 8; ++i) d.chunk_ids[i] = (b[i].x->id << 32) | b[i].idx;
  d.bytes = bytes;
  c->dlog.push_back(d);
  if (c->dlog.size() > (1u << 20)) c->dlog.pop_front();
}

// Per-tenant accounting of dispatched bytes (grouter_tenant_stats) and the
// rate monitor's records (L197: 10 s of dispatch records per tenant).
static void note_dispatch(grouter_ctx *c, uint32_t tenant, int kind, uint64_t bytes) {
  c->tenant_bytes[tenant][kind] += bytes;
  auto &lg = c->tenant_log[tenant];
  const uint64_t now = c->clock_fixed ? c->clock_ns : now_ns();
  lg.emplace_back(now, bytes);
  while (!lg.empty() && (lg.size() > 65536 || lg.front().first + 10000000000ull < now)) lg.pop_front();
}

// Moves whole batches (stride order, logged) from the scheduler into the
// carry queue until the round budget is covered; returns how many.
static uint32_t refill(grouter_ctx *c, Server &s, uint32_t max_batches, uint64_t max_bytes,
                       size_t max_items = kRoundItems) {
  uint64_t bytes = 0;
  for (auto &it : s.carry) bytes += it.bytes;
  uint32_t nb = 0;
  std::vector<ChunkItem> b;
  const uint32_t batch = s.sched.batch;
  while (!s.sched.empty() && nb < max_batches && bytes < max_bytes &&
         s.carry.size() + batch <= max_items) {
    uint64_t bb = 0;
    uint32_t t = s.sched.dispatch([&](uint32_t tn) { return weight_of(c, tn); }, b, &bb);
    if (t == UINT32_MAX) break;
    log_batch(c, s, t, b, bb);
    note_dispatch(c, t, s.kind, bb);
    for (auto &it : b) s.carry.push_back(it);
    bytes += bb;
    ++nb;
  }
  return nb;
}

// One dispatch round carries at most ONE scheduled batch (and urgent
// unscheduled work, e.g. spills); with <= 2 rounds in flight per server that
// is SURVEY O8's "<= 2 batches in flight": a tenant that becomes backlogged
// waits behind at most two batches already handed to the engine (L229).
// A new batch is taken only when the previous one has left the carry queue.
static uint32_t refill_one(grouter_ctx *c, Server &s) {
  return s.carry.empty() ? refill(c, s, 1, 1) : 0;
}

static uint64_t batch_budget(const grouter_ctx *c, const Server &s) {
  return (uint64_t)s.sched.batch * c->cfg.chunk_bytes;
}

// Takes the longest submittable prefix of urgent + carry (bounded by the
// round limits).  An item is submittable unless it is the first item of a
// transfer on this server whose dependencies are not all submitted; cut[i]
// says a stream wait for the transfer's dependencies must precede item i.
static void take(Server &s, uint64_t max_bytes, std::vector<ChunkItem> &items, std::vector<char> &cut,
                 size_t max_items = kRoundItems) {
  items.clear();
  cut.clear();
  uint64_t bytes = 0;
  const Xfer *last_x = nullptr;
  uint32_t last_path = ~0u;
  for (int q = 0; q < 2; ++q) {
    std::deque<ChunkItem> &dq = q == 0 ? s.urgent : s.carry;
    while (!dq.empty() && items.size() < max_items && bytes < max_bytes) {
      const ChunkItem &it = dq.front();
      Xfer &x = *it.x;
      bool first = !(x.deps_waited & s.id_bit());
      bool need_wait = false;
      if (first) {
        for (auto &w : x.deps) {
          if (!is_submitted(w)) return;  // producer not submitted yet: stop here
          need_wait |= !w.done();
        }
        x.deps_waited |= s.id_bit();
      }
      (void)last_x;
      (void)last_path;
      items.push_back(it);
      cut.push_back(need_wait);
      bytes += it.bytes;
      dq.pop_front();
    }
    if (items.size() >= max_items || bytes >= max_bytes) return;
  }
}

// Marks the items as issued and returns the distinct (xfer, path) pairs.
struct Pub {
  Xfer *x;
  uint32_t path;
};
static std::vector<Pub> issue(const std::vector<ChunkItem> &items) {
  std::vector<Pub> pubs;
  for (auto &it : items) {
    Xfer *x = it.x;
    x->issued[it.path]++;
    bool found = false;
    for (auto &p : pubs) found |= (p.x == x && p.path == it.path);
    if (!found) pubs.push_back({x, it.path});
  }
  return pubs;
}

// After a round is submitted: count chunks, release caller-stream waits of
// transfers that are now fully submitted.
static void after_submit(grouter_ctx *c, const std::vector<ChunkItem> &items) {
  for (auto &it : items) it.x->submitted_chunks++;
  Xfer *last = nullptr;
  for (auto &it : items) {
    Xfer *x = it.x;
    if (x == last || !x->submitted()) continue;
    last = x;
    if (!x->waiters.empty()) {
      auto ws = std::move(x->waiters);
      x->waiters.clear();
      for (auto &wt : ws) stream_wait(c, wt.stream, -1, Fences{wt.w});
    }
  }
  // release ownership of fully submitted transfers (collect first: erasing
  // may destroy the transfer, and a round may hold several of its chunks)
  std::vector<Xfer *> fin;
  for (auto &it : items)
    if (it.x->submitted() && std::find(fin.begin(), fin.end(), it.x) == fin.end()) fin.push_back(it.x);
  for (Xfer *x : fin) c->live.erase(x);
  if (!fin.empty()) c->submit_cv.notify_all();
}

// One or more kernel launches for `items` (in order): contiguous chunks are
// coalesced into one run while the parameter block is built; a launch ends
// when its block is full (kMaxRoundChunks runs or kMaxPublish publishes).
// deferred_pub (direct launches of one whole transfer): when the engine needs
// a host-side publish, skip the stream writes and report it -- the caller
// records an event instead (a stream write after a kernel costs ~3.5 us of
// GPU time per launch and breaks programmatic dependent launch; an event
// record costs neither).
// GROUTER_PROFILE around one copy-kernel launch on stream st: timing events
// (pooled) and a %globaltimer stamp slot the kernel writes its first CTA start
// and last CTA end into (*stamp = null when every slot awaits harvesting).
static void prof_begin(PhysDev &pd, cudaStream_t st, ProfRec &pr, unsigned long long *&stamp) {
  for (cudaEvent_t *e : {&pr.start, &pr.stop}) {
    if (!pd.timing_free.empty()) {
      *e = pd.timing_free.back();
      pd.timing_free.pop_back();
    } else {
      GR_CUDA(cudaEventCreate(e));
    }
  }
  static const uint32_t kStampSlots = 4096;
  if (!pd.stamps) {  // [start, end] per slot: UINT64_MAX / 0 until a kernel stamps it
    std::vector<unsigned long long> init(2 * kStampSlots);
    for (uint32_t k = 0; k < kStampSlots; ++k) init[2 * k] = ~0ull, init[2 * k + 1] = 0;
    GR_CUDA(cudaMalloc(&pd.stamps, init.size() * sizeof(unsigned long long)));
    GR_CUDA(cudaMemcpy(pd.stamps, init.data(), init.size() * sizeof(unsigned long long), cudaMemcpyHostToDevice));
    pd.stamp_busy.assign(kStampSlots, 0);
  }
  stamp = nullptr;
  const uint32_t k = pd.next_stamp;
  if (!pd.stamp_busy[k]) {  // else: no stamp for this launch (slots not harvested yet)
    pd.next_stamp = (k + 1) % kStampSlots;
    pd.stamp_busy[k] = 1;
    pr.stamp = (int)k;
    stamp = pd.stamps + 2 * k;
  }
  GR_CUDA(cudaEventRecord(pr.start, st));
}

static void prof_end(grouter_ctx *c, cudaStream_t st, ProfRec &pr) {
  GR_CUDA(cudaEventRecord(pr.stop, st));
  c->prof.push_back(pr);
}

static void launch_round(grouter_ctx *c, Server &s, cudaStream_t st, uint32_t *scratch,
                         const std::vector<ChunkItem> &items, const uint64_t *src_override,
                         bool *deferred_pub = nullptr) {
  if (!c->params) c->params = new CopyParamsHost();
  CopyParams *p = &c->params->p;
  PhysDev &pd = *c->phys.at(s.phys);
  const bool prof = (c->cfg.flags & GROUTER_PROFILE) != 0;
  size_t i = 0;
  std::vector<ChunkItem> part;
  bool first = true;
  bool local = true;  // every destination in the launching GPU's memory -> GPU-scope fences
  for (auto &it : items)
    local &= it.dst_logical >= 0 && c->dev[it.dst_logical].phys == s.phys;
  bool local_src = true;  // relay forwards read this GPU's staging ring
  if (!src_override)
    for (auto &it : items) local_src &= it.x->local_src;
  if (c->cfg.flags & GROUTER_FORCE_REMOTE) local = local_src = false;  // test: the peer branch
  while (i < items.size()) {
    const uint64_t tparams = hprof().on ? now_ns() : 0;
    p->flags = (local ? kFlagLocalDst : 0) | (local_src ? kFlagLocalSrc : 0);
    p->n_chunks = 0;
    p->n_pub = 0;
    p->scratch = scratch;
    p->counts = nullptr;
    p->count_base = 0;
    part.clear();
    uint64_t bytes = 0;
    for (; i < items.size(); ++i) {
      const ChunkItem &it = items[i];
      const uint64_t src = src_override ? src_override[i] : it.src;
      // would this item need a new publish entry / a new run?
      bool new_pub = true;
      for (uint32_t k = 0; k < p->n_pub; ++k)
        if (p->pub[k].word == (uint64_t)(uintptr_t)&it.x->words[it.path]) new_pub = false;
      KChunk *prev = p->n_chunks ? &p->chunk[p->n_chunks - 1] : nullptr;
      const bool extend = prev && prev->src + prev->bytes == src && prev->dst + prev->bytes == it.dst;
      if ((!extend && p->n_chunks == (uint32_t)kMaxRoundChunks) || (new_pub && p->n_pub == (uint32_t)kMaxPublish))
        break;
      if (extend) prev->bytes += it.bytes;
      else p->chunk[p->n_chunks++] = {src, it.dst, it.bytes};
      if (new_pub) p->pub[p->n_pub++] = {(uint64_t)(uintptr_t)&it.x->words[it.path], 0, 0};
      part.push_back(it);
      bytes += it.bytes;
    }
    // publish values after this launch -- only for the (transfer, path)
    // words whose LAST chunk this launch carries: every fence on a word waits
    // for its final value (done_fences; R5, no partial visibility), and a
    // path's chunks run in stream order on one stream, so earlier launches
    // need not publish -- nor pay the in-kernel protocol (a system-scope
    // fence per CTA on the peer branch: ~12 us per launch measured through
    // GROUTER_FORCE_REMOTE, tools/peerpath.py)
    std::vector<Pub> pubs = issue(part);
    uint32_t npub = 0;
    for (uint32_t k = 0; k < p->n_pub; ++k)
      for (auto &pb : pubs)
        if (p->pub[k].word == (uint64_t)(uintptr_t)&pb.x->words[pb.path] &&
            pb.x->issued[pb.path] == pb.x->total[pb.path]) {
          p->pub[npub] = p->pub[k];
          p->pub[npub++].value = pb.x->value_after(pb.path);
        }
    p->n_pub = npub;
    ProfRec pr{s.phys, nullptr, nullptr, bytes};
    p->stamp = nullptr;
    if (prof) prof_begin(pd, st, pr, p->stamp);
    HostProf &hp = hprof();
    uint64_t tl = hp.on ? now_ns() : 0;
    if (hp.on) hp.t[6] += tl - tparams;
    // host-side completion only where an event can stand in for the words
    // (a whole direct transfer); elsewhere the kernel publishes in-kernel,
    // which costs less GPU time than a stream write after the launch
    bool host_pub = false;
    const bool only = first && i == items.size();  // one launch moves every item
    first = false;
    int e = launch_copy(*p, pd.sm_count, (int)c->cfg.copy_ctas_per_sm,
                        (c->cfg.flags & GROUTER_COPY_TMA) != 0, st,
                        deferred_pub && only ? &host_pub : nullptr);
    if (hp.on) hp.t[7] += now_ns() - tl;
    if (e != 0)
      throw Error(GROUTER_ECUDA, std::string("gr_copy launch: ") + cudaGetErrorString((cudaError_t)e));
    if (host_pub) *deferred_pub = true;
    if (prof) prof_end(c, st, pr);
    c->stats.kernel_launches++;
    if (!local) c->stats.peer_launches++;
  }
}

void harvest_profile(grouter_ctx *c, bool wait) {
  while (!c->prof.empty()) {
    ProfRec &r = c->prof.front();
    if (wait) GR_CUDA(cudaEventSynchronize(r.stop));
    else if (cudaEventQuery(r.stop) != cudaSuccess) break;
    float ms = 0.f;
    GR_CUDA(cudaEventElapsedTime(&ms, r.start, r.stop));
    c->stats.timed_launches++;
    c->stats.timed_ns += (uint64_t)((double)ms * 1e6);
    c->stats.timed_bytes += r.bytes;
    if (r.stamp >= 0) {  // the kernel's own start/end (completed: the stop event fired)
      PhysDev &pd = *c->phys.at(r.phys);
      unsigned long long t[2], init[2] = {~0ull, 0ull};
      DeviceGuard g(r.phys);
      GR_CUDA(cudaMemcpy(t, pd.stamps + 2 * r.stamp, sizeof(t), cudaMemcpyDeviceToHost));
      GR_CUDA(cudaMemcpy(pd.stamps + 2 * r.stamp, init, sizeof(init), cudaMemcpyHostToDevice));
      pd.stamp_busy[r.stamp] = 0;
      if (t[1] > t[0] && t[0] != ~0ull) {
        c->stats.timed_kernel_launches++;
        c->stats.timed_kernel_ns += t[1] - t[0];
      }
    }
    auto &fl = c->phys.at(r.phys)->timing_free;
    fl.push_back(r.start);
    fl.push_back(r.stop);
    c->prof.pop_front();
  }
}

// SM-copy server: one kernel launch per round segment (D2D push over
// NVLink, or a same-GPU HBM copy).
//
// A transfer that is the ONLY work queued on the server (one tenant, one
// transfer, no urgent work) goes out in rounds of up to 7 whole batches
// (70 MiB) -- whole when it fits (R55): e.g. a GPU -> other-GPU get, whose consumer stream lives on
// another device and so never takes the direct launch.  A batch per round
// costs a launch and a dispatch reaction per 10 MiB -- at NVLink rates
// (~14 us per batch) that, not the link, bounds a large push
// (tools/peerpath.py).  A tenant arriving later waits behind the <= 2 rounds
// in flight: <= 140 MiB, ~190 us over NVLink (10 MiB batches: ~28 us).
// Real-time mode without GROUTER_LOG only (replay and the log keep one batch
// per round).
static void complete_by_event(grouter_ctx *c, const std::vector<Xfer *> &xs, const EventRef &e, cudaStream_t st);
static const uint32_t kSoloBatches = 7;  // R55: at most 7 batches (70 MiB at 5 x 2 MiB) per solo round
static bool single_transfer(const Server &s) {
  if (!s.urgent.empty()) return false;
  const Xfer *only = nullptr;
  for (auto &it : s.carry) {  // the rest of a solo round's last batch
    if (only && it.x != only) return false;
    only = it.x;
  }
  bool queued = false;
  for (auto &kv : s.sched.tenants) {
    const auto &q = kv.second.q;
    if (q.empty()) continue;
    if (queued || q.front().x != q.back().x || (only && q.front().x != only)) return false;
    queued = true;
    only = q.front().x;
  }
  return only != nullptr;
}

static size_t round_copy(grouter_ctx *c, Server &s) {
  NvtxRange nvtx_("round copy");
  static const bool solo_off = getenv("GR_NO_FAST") != nullptr || getenv("GR_NO_SOLO") != nullptr;
  const bool solo = !solo_off && !c->replay && !(c->cfg.flags & GROUTER_LOG) && single_transfer(s);
  std::vector<ChunkItem> items, seg;
  std::vector<char> cut;
  uint32_t nb;
  if (solo) {  // whole batches only: no leftover in the carry for a newcomer to wait behind
    nb = refill(c, s, kSoloBatches, UINT64_MAX, kDirectItems);
    take(s, UINT64_MAX, items, cut, kDirectItems);
  } else {
    nb = refill_one(c, s);
    take(s, batch_budget(c, s), items, cut);
  }
  if (items.empty()) return 0;
  DeviceGuard g(s.phys);
  if (solo) {
    // one launch moves the whole transfer: complete it by an event, not words
    Xfer *x = items[0].x;
    static const bool ev_done = !getenv("GR_NO_EVDONE");
    const bool whole = ev_done && !x->word_fenced && x->submitted_chunks == 0 && x->waiters.empty() &&
                       items.size() == x->nchunks && std::count(cut.begin(), cut.end(), 1) <= (cut[0] ? 1 : 0) &&
                       !(c->cfg.flags & GROUTER_FORCE_REMOTE);  // forced remote: in-kernel publish
    if (whole) {
      if (cut[0]) stream_wait(c, s.stream, s.phys, x->deps);
      bool deferred = false;
      launch_round(c, s, s.stream, s.scratch, items, nullptr, &deferred);
      EventRef ev = record(c, s.stream, s.phys);
      if (deferred) complete_by_event(c, {x}, ev, s.stream);
      for (auto &it : items) c->stats.link_bytes[0][s.logical] += it.bytes;
      s.inflight.push_back({ev_wait(c, ev), nullptr, nb});
      c->stats.rounds++;
      after_submit(c, items);
      return items.size();
    }
  }
  for (size_t i = 0; i < items.size(); ++i) {
    if (cut[i]) {
      if (!seg.empty()) launch_round(c, s, s.stream, s.scratch, seg, nullptr);
      seg.clear();
      stream_wait(c, s.stream, s.phys, items[i].x->deps);
    }
    seg.push_back(items[i]);
    c->stats.link_bytes[0][s.logical] += items[i].bytes;
  }
  launch_round(c, s, s.stream, s.scratch, seg, nullptr);
  s.inflight.push_back({ev_wait(c, record(c, s.stream, s.phys)), nullptr, nb});
  c->stats.rounds++;
  after_submit(c, items);
  return items.size();
}

// Copies a pageable host chunk into the circular pinned buffer (L229) and
// returns the pinned address to DMA from; the slot is reused once the DMA
// that last read it has completed.
static uint64_t bounce(grouter_ctx *c, uint64_t src, uint64_t bytes, uint32_t *slot_out) {
  uint32_t k = c->bounce_next;
  c->bounce_next = (k + 1) % c->bounce_slots;
  if (c->bounce_ev[k]) GR_CUDA(cudaEventSynchronize(c->bounce_ev[k]->ev));
  uint8_t *slot = c->bounce + (uint64_t)k * c->cfg.chunk_bytes;
  std::memcpy(slot, (const void *)src, bytes);
  *slot_out = k;
  return (uint64_t)slot;
}

// Transfers a CE round moves WHOLE (every chunk in this round, none relayed,
// no word fences handed out yet, no deferred stream waits) complete by the
// round's closing event instead of stream-written words: a
// cuStreamWriteValue32 costs ~0.8 us of host time and ~1-2 us of latency
// per round (tools/celat.cu), the dominant cost of small blocking cFn puts
// and gets.  Real-time mode only (replay hands out word fences first).
static std::vector<Xfer *> whole_in_round(grouter_ctx *c, const Server &s, const std::vector<ChunkItem> &items) {
  std::vector<Xfer *> out;
  static const bool ev_done = !getenv("GR_NO_EVDONE");
  if (!ev_done || c->replay) return out;
  std::unordered_map<Xfer *, uint32_t> n;
  for (auto &it : items) {
    Xfer *x = it.x;
    if (x->word_fenced || x->submitted_chunks || !x->waiters.empty()) continue;
    if (s.kind == SK_H2D && it.dst_logical != s.logical && !(c->cfg.flags & GROUTER_CE_RELAY)) {
      n[x] = UINT32_MAX;  // a relayed chunk: the forward kernel publishes
      continue;
    }
    uint32_t &k = n[x];
    if (k != UINT32_MAX) ++k;
  }
  for (auto &kv : n)
    if (kv.second == kv.first->nchunks) out.push_back(kv.first);
  return out;
}

static void complete_by_event(grouter_ctx *c, const std::vector<Xfer *> &xs, const EventRef &e, cudaStream_t st) {
  for (Xfer *x : xs) {
    x->done_ev = e;
    x->done_stream = st;
    for (uint32_t p = 0; p < x->npath; ++p) c->slot_final[x->slot][p] -= x->total[p];  // slot back
  }
}

static void publish_ce(grouter_ctx *c, Server &s, std::vector<ChunkItem> &seg,
                       const std::vector<Xfer *> &evented) {
  if (!evented.empty())
    seg.erase(std::remove_if(seg.begin(), seg.end(),
                             [&](const ChunkItem &it) {
                               return std::find(evented.begin(), evented.end(), it.x) != evented.end();
                             }),
              seg.end());
  // Only the round that carries a path's LAST chunk writes that path's word
  // (consumers never see partial progress, R5; the copies of one path on one
  // server are in stream order, so the final write covers the earlier rounds):
  // a stream write costs ~1-2 us per round on a multi-round transfer.  Every
  // fence on a word waits for its final value (done_fences).
  // The write itself goes on the server's publish stream, behind an event on
  // the CE stream: a stream write carries a memory barrier that idles the copy
  // engine ~5 us before the next copy may start (tools/ce2.cu: 4 x 10 MiB H2D
  // back to back 52.8 GB/s with a write after each copy, 54.3 with an event,
  // 54.3 with the event + publish-stream write), while the event costs the
  // CE stream nothing and keeps the ordering (copies, then the word).
  std::vector<Pub> fin;
  for (auto &p : issue(seg))
    if (p.x->issued[p.path] == p.x->total[p.path]) fin.push_back(p);
  seg.clear();
  if (fin.empty()) return;
  cudaStream_t ws = s.stream;
  if (s.pub_stream) {
    EventRef e = record(c, s.stream, s.phys);
    GR_CUDA(cudaStreamWaitEvent(s.pub_stream, e->ev, 0));
    ws = s.pub_stream;
  }
  for (auto &p : fin)
    GR_CU(drv().streamWriteValue32((CUstream)ws, (CUdeviceptr)(uintptr_t)&p.x->words[p.path],
                                   p.x->value_after(p.path), 0));
}

// Issues a finished run as one copy (1-D) or one pitched copy (2-D).
static void flush_ce_run(CeRun &r, cudaMemcpyKind kind, cudaStream_t st) {
  if (!r.height) return;
  if (r.height == 1) GR_CUDA(cudaMemcpyAsync((void *)r.dst, (const void *)r.src, r.width, kind, st));
  else GR_CUDA(cudaMemcpy2DAsync((void *)r.dst, r.dpitch, (const void *)r.src, r.spitch, r.width, r.height, kind, st));
  r.height = 0;
}


// H2D server of route GPU r: CE copies of up to two batches (L229).  Chunks
// for r itself land in the lease; relayed chunks go through r's staging ring
// and a forward round kernel on r pushes them to their destination.
static size_t round_h2d(grouter_ctx *c, Server &s) {
  NvtxRange nvtx_("round h2d");
  const bool ce_relay = (c->cfg.flags & GROUTER_CE_RELAY) != 0;
  const uint64_t budget = batch_budget(c, s);
  const uint64_t tr0 = tl_put_t0 ? now_ns() : 0;
  const uint32_t nb = refill_one(c, s);
  std::vector<ChunkItem> items, direct;
  std::vector<char> cut;
  take(s, budget, items, cut);
  if (items.empty()) return 0;
  const std::vector<Xfer *> evented = whole_in_round(c, s, items);
  DeviceGuard g(s.phys);
  EventRef last_fwd;
  // contiguous direct chunks of a round go to the copy engine as ONE copy
  // (per-copy engine overhead ~3.6 us measured by the probe)
  CeRun run;
  auto flush_run = [&]() {
    if (!run.empty()) {
      const uint64_t tm = tl_put_t0 ? now_ns() : 0;
      flush_ce_run(run, cudaMemcpyDefault, s.stream);
      if (tl_put_t0) {  // profiling: put call -> its first H2D copy submitted
        const uint64_t te = now_ns();
        hprof().t[14] += te - tl_put_t0;
        hprof().t[16] += tr0 - tl_put_t0;  // put call -> round (after refill)
        hprof().t[17] += tm - tr0;         // take + DeviceGuard -> memcpy call
        hprof().t[18] += te - tm;          // the memcpy call
        tl_put_t0 = 0;
      }
    }
  };
  // Relay forward (K4', L182 "chunks are pipelined across GPU streams").  A
  // route's relayed chunks of one transfer in a round form a GROUP: they are
  // copied into consecutive staging slots by ONE 2-D copy (equal chunks at
  // the plan's interleave stride, R4) and pushed to the destination by ONE
  // forward launch on the route GPU's forward stream, which waits for exactly
  // that copy; the forward of round j overlaps the copies of round j+1.  In
  // the round that carries the path's LAST chunk, that chunk is copied and
  // forwarded on its own after the group, so the relay adds one chunk's
  // forward to the transfer's tail, not a round's.  Per chunk, a copy costs
  // the copy engine ~3 us of setup and the dispatch thread ~7 us of host time
  // (copy, event, stream wait, launch, event; tools/relaycost.py): one copy
  // and one forward per round instead of five.  The forward kernels run only
  // while a chunk is moving (no SMs parked polling for PCIe arrivals).
  // Measurement only: GR_CHUNK_FWD=1 (every relayed chunk copied and
  // forwarded alone, the previous design), GR_SEGMENT_FWD=1 (the round-1
  // design: one forward per segment after all of its chunk copies).
  static const bool segment_fwd = getenv("GR_SEGMENT_FWD") != nullptr;
  static const bool chunk_fwd = getenv("GR_CHUNK_FWD") != nullptr;
  std::vector<ChunkItem> seg_relay;
  std::vector<uint64_t> seg_src;
  std::vector<uint32_t> seg_slots;
  // slots [k0, k0 + g) of the staging ring, consecutive (a group never wraps:
  // the ring's tail slots are skipped instead); waits for their last readers
  auto take_slots = [&](uint32_t g) -> uint32_t {
    if (s.next_slot + g > s.n_slots) s.next_slot = 0;
    const uint32_t k0 = s.next_slot;
    s.next_slot = (k0 + g) % s.n_slots;
    EventRef last;
    for (uint32_t k = k0; k < k0 + g; ++k)
      if (s.slot_free[k] && s.slot_free[k] != last) {
        GR_CUDA(cudaStreamWaitEvent(s.stream, s.slot_free[k]->ev, 0));
        last = s.slot_free[k];
      }
    return k0;
  };
  auto forward = [&](const std::vector<ChunkItem> &its, const std::vector<uint64_t> &srcs, uint32_t k0) {
    EventRef ce = record(c, s.stream, s.phys);
    GR_CUDA(cudaStreamWaitEvent(s.fwd_stream, ce->ev, 0));
    launch_round(c, s, s.fwd_stream, s.fwd_scratch, its, srcs.data());
    last_fwd = record(c, s.fwd_stream, s.phys);
    for (uint32_t k = k0; k < k0 + (uint32_t)its.size(); ++k) s.slot_free[k] = last_fwd;
  };
  // a chunk on its own: one copy into one slot, one forward
  auto relay_one = [&](const ChunkItem &it, uint64_t src) {
    const uint32_t k = take_slots(1);
    uint8_t *slot = s.staging + (uint64_t)k * s.slot_bytes;
    GR_CUDA(cudaMemcpyAsync(slot, (const void *)src, it.bytes, cudaMemcpyHostToDevice, s.stream));
    if (segment_fwd) {
      seg_relay.push_back(it);
      seg_src.push_back((uint64_t)slot);
      seg_slots.push_back(k);
      return;
    }
    forward(std::vector<ChunkItem>(1, it), std::vector<uint64_t>(1, (uint64_t)slot), k);
  };
  std::vector<ChunkItem> grp;  // pending group: same transfer and path, equal chunks, one stride
  auto flush_group = [&]() {
    if (grp.empty()) return;
    const ChunkItem &l = grp.back();
    const bool has_last = l.x->total[l.path] - l.x->issued[l.path] == grp.size();
    const size_t g = grp.size() - (has_last && grp.size() > 1 ? 1 : 0);
    if (g == 1) {
      relay_one(grp[0], grp[0].src);
    } else {
      const uint32_t k0 = take_slots((uint32_t)g);
      uint8_t *slot0 = s.staging + (uint64_t)k0 * s.slot_bytes;
      const uint64_t spitch = grp[1].src - grp[0].src;
      GR_CUDA(cudaMemcpy2DAsync(slot0, s.slot_bytes, (const void *)grp[0].src, spitch, grp[0].bytes, g,
                                cudaMemcpyHostToDevice, s.stream));
      std::vector<ChunkItem> its(grp.begin(), grp.begin() + g);
      std::vector<uint64_t> srcs(g);
      for (size_t j = 0; j < g; ++j) srcs[j] = (uint64_t)(slot0 + j * s.slot_bytes);
      forward(its, srcs, k0);
    }
    if (g < grp.size()) relay_one(grp.back(), grp.back().src);
    grp.clear();
  };
  auto group_accepts = [&](const ChunkItem &it) {
    if (grp.empty()) return true;
    const ChunkItem &a = grp.front();
    if (it.x != a.x || it.path != a.path || it.bytes != a.bytes || grp.size() >= s.n_slots / 2) return false;
    if (grp.size() == 1) return it.src > a.src && it.src - a.src >= a.bytes && it.src - a.src <= CeRun::kMaxPitch;
    return it.src == a.src + grp.size() * (grp[1].src - a.src);
  };
  auto end_segment = [&]() {
    flush_group();
    flush_run();
    publish_ce(c, s, direct, evented);
    if (!seg_relay.empty()) {
      EventRef ce = record(c, s.stream, s.phys);
      GR_CUDA(cudaStreamWaitEvent(s.fwd_stream, ce->ev, 0));
      launch_round(c, s, s.fwd_stream, s.fwd_scratch, seg_relay, seg_src.data());
      last_fwd = record(c, s.fwd_stream, s.phys);
      for (uint32_t k : seg_slots) s.slot_free[k] = last_fwd;
      seg_relay.clear();
      seg_src.clear();
      seg_slots.clear();
    }
  };
  for (size_t i = 0; i < items.size(); ++i) {
    const ChunkItem &it = items[i];
    if (cut[i]) {
      end_segment();
      stream_wait(c, s.stream, s.phys, it.x->deps);
    }
    uint64_t src = it.src;
    uint32_t bslot = 0;
    if (it.x->pageable_src) src = bounce(c, it.src, it.bytes, &bslot);
    // GROUTER_CE_RELAY: the route GPU's copy engine reads host memory over its
    // own PCIe link and writes the destination's pages directly (over NVLink
    // on a multi-GPU box): no staging slot, no forward launch
    if (it.dst_logical == s.logical || ce_relay) {
      if (it.x->pageable_src) {  // bounce slot: copy now, the slot is reused
        flush_run();
        run.add(src, it.dst, it.bytes, it.x);
        flush_run();
      } else if (!run.add(src, it.dst, it.bytes, it.x)) {
        flush_run();
        run.add(src, it.dst, it.bytes, it.x);
      }
      direct.push_back(it);
    } else {
      flush_run();
      if (it.x->pageable_src || chunk_fwd || segment_fwd) {  // bounce slot reused at once; measurement modes
        flush_group();
        relay_one(it, src);
      } else {
        if (!group_accepts(it)) flush_group();
        grp.push_back(it);
      }
    }
    if (it.x->pageable_src) c->bounce_ev[bslot] = record(c, s.stream, s.phys);
    c->stats.link_bytes[1][s.logical] += it.bytes;
  }
  end_segment();
  EventRef ce_end = record(c, s.stream, s.phys);
  complete_by_event(c, evented, ce_end, s.stream);
  if (last_fwd) {  // one in-flight marker covering both the CE and the forward stream
    GR_CUDA(cudaStreamWaitEvent(s.fwd_stream, ce_end->ev, 0));
    s.inflight.push_back({ev_wait(c, record(c, s.fwd_stream, s.phys)), nullptr, nb});
  } else {
    s.inflight.push_back({ev_wait(c, ce_end), nullptr, nb});
  }
  c->stats.rounds++;
  after_submit(c, items);
  return items.size();
}

// D2H server: CE copies device -> host (host store, host leases, caller
// host buffers, and urgent spills).
static size_t round_d2h(grouter_ctx *c, Server &s) {
  NvtxRange nvtx_("round d2h");
  const uint32_t nb = refill_one(c, s);
  std::vector<ChunkItem> items, seg;
  std::vector<char> cut;
  take(s, batch_budget(c, s), items, cut);
  if (items.empty()) return 0;
  const std::vector<Xfer *> evented = whole_in_round(c, s, items);
  DeviceGuard g(s.phys);
  CeRun run;
  auto flush_run = [&]() { flush_ce_run(run, cudaMemcpyDefault, s.stream); };
  for (size_t i = 0; i < items.size(); ++i) {
    const ChunkItem &it = items[i];
    if (cut[i]) {
      flush_run();
      publish_ce(c, s, seg, evented);
      stream_wait(c, s.stream, s.phys, it.x->deps);
    }
    if (!run.add(it.src, it.dst, it.bytes, it.x)) {
      flush_run();
      run.add(it.src, it.dst, it.bytes, it.x);
    }
    seg.push_back(it);
    c->stats.link_bytes[2][s.logical] += it.bytes;
  }
  flush_run();
  publish_ce(c, s, seg, evented);
  EventRef ce_end = record(c, s.stream, s.phys);
  complete_by_event(c, evented, ce_end, s.stream);
  s.inflight.push_back({ev_wait(c, ce_end), nullptr, nb});
  c->stats.rounds++;
  after_submit(c, items);
  return items.size();
}

static void retire(Server &s) {
  while (!s.inflight.empty() && s.inflight.front().w.done()) s.inflight.pop_front();
}

static bool has_work(const Server &s) {
  return !s.sched.empty() || !s.carry.empty() || !s.urgent.empty();
}

static size_t pump_server(grouter_ctx *c, Server &s, bool force) {
  if (!s.stream || !has_work(s)) return 0;
  // retire only when the in-flight limit would hold the round back: every
  // completed-round check is an event query (~1 us of host time), and pump
  // runs on every call for every server of the node
  if (!force && s.inflight.size() >= 2) retire(s);
  size_t total = 0;
  while (has_work(s) && (force || s.inflight.size() < 2 || (retire(s), s.inflight.size() < 2))) {
    if (c->inject_round_failures > 0) {  // grouter_test_inject: fault injection (tests only)
      --c->inject_round_failures;
      throw Error(GROUTER_ECUDA, "injected dispatch-round failure (grouter_test_inject)");
    }
    const uint64_t tr = hprof().on ? now_ns() : 0;
    size_t n = s.kind == SK_COPY ? round_copy(c, s) : s.kind == SK_H2D ? round_h2d(c, s) : round_d2h(c, s);
    if (tr && n) {  // GROUTER_HOST_PROFILE: host time per dispatch round (the dispatch thread's budget)
      static std::mutex m;
      std::lock_guard<std::mutex> lk(m);
      hprof().t[s.kind == SK_COPY ? 19 : 20] += now_ns() - tr;
      hprof().rounds[s.kind == SK_COPY ? 0 : 1]++;
    }
    if (!n) break;  // blocked on another server's submission
    total += n;
  }
  return total;
}

// Dispatches rounds.  force: ignore the in-flight limit and iterate over the
// servers until every queued chunk is submitted (a server blocked on another
// server's submission is retried after that one progressed).
void pump(grouter_ctx *c, bool force_all) {
  if (c->replay && !force_all) return;
  for (;;) {
    size_t progress = 0;
    for (auto &d : c->dev) {
      progress += pump_server(c, d.copy, force_all);
      progress += pump_server(c, d.h2d, force_all);
      progress += pump_server(c, d.d2h, force_all);
    }
    if (!force_all || !progress) break;
  }
  bool backlog = false;
  for (auto &d : c->dev) backlog |= has_work(d.copy) || has_work(d.h2d) || has_work(d.d2h);
  if (backlog) c->cv.notify_one();
}

void flush_all(grouter_ctx *c) {
  pump(c, true);
  c->epoch++;  // everything created before is now submitted (grounded)
}

// Direct launch without the queues: one same-GPU (or same-device logical
// pair) SM copy of a contiguous single-path plan on an idle copy server, in
// real-time mode.  Does exactly what enqueue + try_direct would -- the
// tenant's stride passes advance as if its batches had been dispatched
// (Stride::account_solo), tenant bytes, the rate monitor and the stats are
// updated, the transfer completes by an event on the caller's stream -- but
// skips building chunk items, the scheduler queues, round assembly and the
// completion slot (~1.5 us of host time per call, tools/libcost.cpp).  Only
// for static-assignment engines (16 B-aligned addresses: wv8 / tmas4, no
// device scratch).  Returns null when the queued path must be used.
//
// Small GPU -> other-GPU copies (<= kPullMax) run here too, as a PULL on the
// consumer's stream (R56): the consumer GPU's SMs read the source over
// NVLink (pool pages and peer buffers are mapped for every GPU), so the
// consumer's stream needs no cross-device event, no completion words and no
// wait on the source GPU's server stream -- at these sizes that chain, not
// the link, is the latency (tools/peerpath.py).  Larger ones are pushed by
// the source GPU's copy server (R40, R55).  The source's server still does
// the stride accounting: the bytes use its NVLink egress.
static const uint64_t kPullMax = 4ull << 20;

XferRef fast_direct(grouter_ctx *c, uint32_t tenant, int server_logical, int dst_logical, uint64_t src,
                    uint64_t dst, uint64_t n, bool local_src, const Fences &deps, cudaStream_t caller,
                    int caller_logical) {
  static const bool off = getenv("GR_NO_FAST") != nullptr || getenv("GR_COPY") != nullptr;
  static const bool pull_off = getenv("GR_NO_PULL") != nullptr;
  const uint32_t never = GROUTER_LOG | GROUTER_COPY_TMA;
  if (off || c->replay || !caller || (c->cfg.flags & never) || !n || ((src | dst) & 15)) return nullptr;
  if (caller_logical < 0) return nullptr;
  Server &s = c->dev[server_logical].copy;
  const int caller_phys = c->dev[caller_logical].phys;
  // forced remote (test): logical GPUs stand for physical ones
  const bool forced = (c->cfg.flags & GROUTER_FORCE_REMOTE) != 0;
  const bool cross = forced ? server_logical != caller_logical : s.phys != caller_phys;
  if (forced && !cross) return nullptr;  // forced remote: same-GPU rounds take the queued path
  if (cross && (pull_off || (n > kPullMax && !(c->cfg.flags & GROUTER_PULL_ALL)))) return nullptr;
  if (!s.carry.empty() || !s.urgent.empty() || !s.sched.empty()) return nullptr;
  for (auto &f : s.inflight)
    if (f.direct != caller) {
      retire(s);
      for (auto &g : s.inflight)
        if (g.direct != caller) return nullptr;
      break;
    }
  for (auto &w : deps)
    if (!is_submitted(w)) return nullptr;
  NvtxRange nvtx_("fast direct copy", n);
  const uint64_t C = c->cfg.chunk_bytes;
  auto x = std::make_shared<Xfer>();
  x->id = ++c->xfer_seq;
  x->tenant = tenant;
  x->epoch = c->epoch;
  x->npath = 1;
  x->nchunks = x->submitted_chunks = (uint32_t)((n + C - 1) / C);
  local_src &= !cross;  // a pull reads the other GPU's memory
  x->local_src = local_src;
  c->stats.xfer_count++;
  DeviceGuard g(caller_phys);
  stream_wait(c, caller, caller_phys, deps);  // no-op for completed fences
  if (!c->params) c->params = new CopyParamsHost();
  CopyParams *p = &c->params->p;
  const bool local = !forced && dst_logical >= 0 && c->dev[dst_logical].phys == caller_phys;
  p->flags = (local ? kFlagLocalDst : 0) | (local_src ? kFlagLocalSrc : 0);
  p->n_chunks = 1;
  p->n_pub = 0;
  p->scratch = nullptr;
  p->counts = nullptr;
  p->count_base = 0;
  p->stamp = nullptr;
  p->chunk[0] = {src, dst, n};
  bool host_pub = false;
  PhysDev &pd = *c->phys.at(caller_phys);
  // Small same-device copies (<= 1 MiB; GR_SMALL_CE overrides for measurement)
  // go to the copy engine: its start latency beats a kernel launch's there
  // (C++ single calls, tools/libcost.cpp: 4 KiB 7.94 -> 7.14 us, 64 KiB
  // 8.80 -> 8.58 us; through Python, tools/smallce.py, 256 KiB-1 MiB p50
  // 9.0-9.9 us by kernel vs 7.7-9.2 us by copy engine; from 1.5 MiB on the
  // two are within run-to-run noise and the kernel keeps the HBM roofline)
  static const uint64_t small_ce =
      getenv("GR_SMALL_CE") ? strtoull(getenv("GR_SMALL_CE"), nullptr, 0) : (1ull << 20);
  if (n <= small_ce && !cross) {
    GR_CUDA(cudaMemcpyAsync((void *)dst, (const void *)src, n, cudaMemcpyDeviceToDevice, caller));
    host_pub = true;
  } else {
    const bool prof = (c->cfg.flags & GROUTER_PROFILE) != 0;  // the same events and stamps as launch_round
    ProfRec pr{caller_phys, nullptr, nullptr, n};
    if (prof) prof_begin(pd, caller, pr, p->stamp);
    int e = launch_copy(*p, pd.sm_count, (int)c->cfg.copy_ctas_per_sm, false, caller, &host_pub);
    if (e != 0) throw Error(GROUTER_ECUDA, std::string("gr_copy launch: ") + cudaGetErrorString((cudaError_t)e));
    if (prof) prof_end(c, caller, pr);
  }
  if (!host_pub) throw Error(GROUTER_ECUDA, "internal: fast direct launch needs a static engine");
  x->done_ev = record(c, caller, caller_phys);
  x->done_stream = caller;
  // the bookkeeping a queued dispatch would have done
  s.sched.account_solo(tenant, n, C, weight_of(c, tenant));
  note_dispatch(c, tenant, SK_COPY, n);
  c->stats.link_bytes[0][s.logical] += n;
  c->stats.rounds++;
  if (n > small_ce || cross) {
    c->stats.kernel_launches++;
    if (!local || cross) c->stats.peer_launches++;
  }
  Waitable w;
  w.ev = x->done_ev;
  w.epoch = x->epoch;
  w.origin = caller;
  const uint32_t nb = (uint32_t)((x->nchunks + s.sched.batch - 1) / s.sched.batch);
  if (!s.inflight.empty() && s.inflight.back().direct == caller && s.inflight.back().w.origin == caller)
    s.inflight.back().w = w;
  else
    s.inflight.push_back({w, caller, nb});
  return x;
}

// Copy-engine transfer of an idle H2D / D2H server without the queues, for
// a single-route plan of at most two batches (so <= 2 batches in flight
// holds): one cudaMemcpyAsync on the server's stream and an
// event, with the same scheduler accounting (Stride::account_solo), tenant
// bytes, rate monitor and stats as a queued dispatch.  Real-time mode only,
// no LOG (the dispatch log lists batches); null when the queued path must be used.
XferRef fast_ce(grouter_ctx *c, uint32_t tenant, int kind, const std::vector<grouter_chunk> &plan, uint64_t src,
                uint64_t dst, uint64_t n, const Fences &deps) {
  static const bool off = getenv("GR_NO_FAST") != nullptr;
  if (off || c->replay || (c->cfg.flags & GROUTER_LOG) || plan.empty()) return nullptr;
  const int route = plan[0].route_gpu;
  for (auto &ch : plan)
    if (ch.route_gpu != route || ch.path != 0) return nullptr;  // striped: the queued path relays
  Server &s = server_of(c, kind, route);
  if (plan.size() > 2ull * s.sched.batch || !s.carry.empty() || !s.urgent.empty() || !s.sched.empty())
    return nullptr;  // more than two batches: the queued path keeps them preemptible (O8)
  if (!s.inflight.empty()) {
    retire(s);
    if (!s.inflight.empty()) return nullptr;
  }
  for (auto &w : deps)
    if (!is_submitted(w)) return nullptr;
  NvtxRange nvtx_(kind == SK_H2D ? "fast ce h2d" : "fast ce d2h", n);
  auto x = std::make_shared<Xfer>();
  x->id = ++c->xfer_seq;
  x->tenant = tenant;
  x->epoch = c->epoch;
  x->npath = 1;
  x->nchunks = x->submitted_chunks = (uint32_t)plan.size();
  c->stats.xfer_count++;
  DeviceGuard g(s.phys);
  stream_wait(c, s.stream, s.phys, deps);
  GR_CUDA(cudaMemcpyAsync((void *)dst, (const void *)src, n,
                          kind == SK_H2D ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToHost, s.stream));
  x->done_ev = record(c, s.stream, s.phys);
  x->done_stream = s.stream;
  s.sched.account_solo(tenant, n, plan[0].bytes, weight_of(c, tenant));
  note_dispatch(c, tenant, kind, n);
  c->stats.link_bytes[kind][s.logical] += n;
  c->stats.rounds++;
  s.inflight.push_back({ev_wait(c, x->done_ev), nullptr,
                        (uint32_t)((plan.size() + s.sched.batch - 1) / s.sched.batch)});
  return x;
}

bool try_direct(grouter_ctx *c, const XferRef &x, int server_logical, cudaStream_t caller, int caller_phys) {
  NvtxRange nvtx_("direct launch");
  if (c->replay || !caller) return false;
  Server &s = c->dev[server_logical].copy;
  if (s.phys != caller_phys || !s.carry.empty() || !s.urgent.empty()) return false;
  if (s.sched.backlog_items != x->nchunks) return false;  // only this transfer is queued
  // server-stream or other-stream work in flight: keep order there (retire
  // only when needed: an event query costs host time)
  bool foreign = false;
  for (auto &f : s.inflight) foreign |= f.direct != caller;
  if (foreign) {
    retire(s);
    for (auto &f : s.inflight)
      if (f.direct != caller) return false;
  }
  for (auto &w : x->deps)
    if (!is_submitted(w)) return false;
  PhysDev &pd = *c->phys.at(s.phys);
  DeviceGuard g(s.phys);
  std::vector<ChunkItem> items;
  std::vector<char> cut;
  HostProf &hp = hprof();
  while (has_work(s)) {
    uint64_t ta = hp.on ? now_ns() : 0;
    const uint32_t nb = refill(c, s, UINT32_MAX, kDirectBytes, kDirectItems);
    take(s, kDirectBytes, items, cut, kDirectItems);
    if (hp.on) hp.t[5] += now_ns() - ta;
    if (items.empty()) throw Error(GROUTER_ECUDA, "internal: direct launch made no progress");
    if (cut[0]) stream_wait(c, caller, s.phys, x->deps);
    // scratch pair for this launch (the server's own pair belongs to its stream)
    uint32_t k = pd.next_scratch;
    pd.next_scratch = (k + 1) % pd.n_scratch;
    for (auto &w : pd.scratch_busy[k])
      if (!w.done()) host_wait(Fences{w});
    pd.scratch_busy[k].clear();
    // one launch moves the whole transfer: complete it by an event, not words
    static const bool ev_done = !getenv("GR_NO_EVDONE");
    const bool whole = ev_done && x->submitted_chunks == 0 && items.size() == x->nchunks && x->waiters.empty() &&
                       !(c->cfg.flags & GROUTER_FORCE_REMOTE);  // forced remote: in-kernel publish
    bool deferred = false;
    launch_round(c, s, caller, pd.scratch + 2 * k, items, nullptr, whole ? &deferred : nullptr);
    if (deferred) {
      x->done_ev = record(c, caller, s.phys);
      x->done_stream = caller;
      for (uint32_t p = 0; p < x->npath; ++p) c->slot_final[x->slot][p] -= x->total[p];  // slot back
    }
    for (auto &it : items) c->stats.link_bytes[0][s.logical] += it.bytes;
    c->stats.rounds++;
    after_submit(c, items);
    Fences done;
    done_fences(x, done);
    if (!deferred) pd.scratch_busy[k] = done;  // an in-kernel publish used the pair
    // one entry per caller stream: its newest launch stands for the older ones
    Waitable w = done.empty() ? Waitable{} : done.front();
    if (!s.inflight.empty() && s.inflight.back().direct == caller && deferred && s.inflight.back().w.origin == caller)
      s.inflight.back().w = w;
    else
      s.inflight.push_back({w, caller, nb});
  }
  return true;
}

// D2H of an eviction victim (L258-L262; the per-GPU I/O path of L269): an
// urgent, unscheduled transfer on the victim GPU's D2H engine.
// GROUTER_STRIPED_MIGRATION (R47): the victim leaves over R(src), each route
// GPU's copy engine reading its share straight from the source pool pages
// (mapped for every GPU) -- the gFn-host plan of L178 / R45.
void spill_copy(grouter_ctx *c, Obj &o, uint8_t *host_dst) {
  NvtxRange nvtx_("spill", o.n);
  std::vector<grouter_chunk> plan;
  if (c->cfg.flags & GROUTER_STRIPED_MIGRATION) c->planner.plan_h2d(o.loc, o.n, plan);
  else c->planner.plan_single(o.n, o.loc, plan);
  XferRef x = new_xfer_slot(c, plan);
  x->deps = o.ready;
  for (uint32_t i = 0; i < plan.size(); ++i)
    c->dev[plan[i].route_gpu].d2h.urgent.push_back(
        make_item(x, i, plan[i], (uint64_t)(uintptr_t)o.ptr, (uint64_t)(uintptr_t)host_dst, GROUTER_HOST));
  Fences done;
  done_fences(x, done);
  Fences old = std::move(o.readers);
  for (auto &f : o.ready) old.push_back(f);
  for (auto &f : done) old.push_back(f);
  dev_free(c, o.loc, o.ptr, charge(o.n), std::move(old));
  o.ready = done;
  o.readers.clear();
  c->stats.spill_count++;
  c->stats.spill_bytes += o.n;
  pump(c, false);
}

// H2D of a proactively restored object (L260-L262) back to its home GPU d: an
// urgent, unscheduled transfer, single-path on d's own H2D engine (R42), or
// striped over R(d) with relays under GROUTER_STRIPED_MIGRATION (R47).
void restore_copy(grouter_ctx *c, Obj &o, int d, uint8_t *dev_dst) {
  NvtxRange nvtx_("restore", o.n);
  std::vector<grouter_chunk> plan;
  if (c->cfg.flags & GROUTER_STRIPED_MIGRATION) c->planner.plan_h2d(d, o.n, plan);
  else c->planner.plan_single(o.n, d, plan);
  XferRef x = new_xfer_slot(c, plan);
  x->deps = o.ready;
  for (uint32_t i = 0; i < plan.size(); ++i)
    c->dev[plan[i].route_gpu].h2d.urgent.push_back(
        make_item(x, i, plan[i], (uint64_t)(uintptr_t)o.ptr, (uint64_t)(uintptr_t)dev_dst, d));
  Fences done;
  done_fences(x, done);
  Fences old = std::move(o.readers);
  for (auto &f : o.ready) old.push_back(f);
  for (auto &f : done) old.push_back(f);
  host_free(c, o.ptr, charge(o.n), std::move(old));
  o.ready = done;
  o.readers.clear();
  c->stats.restore_count++;
  c->stats.restore_bytes += o.n;
  pump(c, false);
}

// ------------------------------------------------------------------ lifecycle
static constexpr uint64_t kTrimDelayNs = 1000000000ull;  // 1 s of sustained excess before a trim

// Dispatch thread (L269-L271 I/O daemon): pumps the servers' queues and
// retires completed rounds.  Nothing here may block in a slow driver call:
// while a blocking host put waits, this thread alone issues its next batches.
//
// Poll period while work is queued.  A copy engine's round (one 10 MiB batch
// over PCIe) lasts ~190 us, so a 20 us sleep keeps its two-round window
// full.  An SM-copy round is one 10 MiB batch over NVLink (~14 us) or HBM
// (~3 us): with two rounds in flight the next launch must follow a
// completion within a few microseconds, or the link idles between rounds
// (measured on the forced-remote path, tools/peerpath.py: a 20 us sleep --
// ~70 us with the default 50 us timer slack -- left 1 GiB pushes at 0.08 of
// the HBM copy rate).  So while an SM-copy server's backlog waits for a free
// slot in its window the thread spins with the lock released (~1 us between
// polls; one core, only then), with the full retire sweep every 64 polls.
static void daemon_main(grouter_ctx *c) {
  prctl(PR_SET_TIMERSLACK, 1000UL, 0, 0, 0);  // 1 us: sleeps close to what they ask for
  std::unique_lock<std::mutex> lk(c->mu);
  uint32_t spins = 0;
  while (!c->stop) {
    bool backlog = false, busy = false, sm_backlog = false;
    try {
      if (!c->replay) pump(c, false);
      // spin only while a copy server's queued work waits for its in-flight
      // window (work blocked on another server's submission sleeps as before)
      for (auto &d : c->dev) sm_backlog |= !c->replay && has_work(d.copy) && d.copy.inflight.size() >= 2;
      // full retire sweep (event queries on every server) only when not
      // spinning, or every 64th spin
      const bool sweep = !sm_backlog || (++spins & 63) == 0;
      for (auto &d : c->dev) {
        backlog |= has_work(d.copy) || has_work(d.h2d) || has_work(d.d2h);
        busy |= !d.copy.inflight.empty() || !d.h2d.inflight.empty() || !d.d2h.inflight.empty();
        if (!c->replay && sweep) {
          retire(d.copy);
          retire(d.h2d);
          retire(d.d2h);
        }
      }
    } catch (const Error &e) {
      set_error(e.what());
      c->sticky_error = true;
      c->submit_cv.notify_all();  // callers blocked in order_after fail with ECUDA
      sm_backlog = false;
    }
    if (sm_backlog) {
      lk.unlock();
      // ~1 us between polls; longer (up to 100 us) while an API caller waits
      // for the lock, so the unfair mutex is not re-taken ahead of it
      const uint64_t t0 = now_ns();
      for (uint64_t t = t0; t - t0 < 1000 || (c->lock_waiters.load(std::memory_order_relaxed) > 0 && t - t0 < 100000);
           t = now_ns())
        cpu_relax();
      lk.lock();
    } else if (backlog && !c->replay) {
      lk.unlock();
      std::this_thread::sleep_for(std::chrono::microseconds(20));
      lk.lock();
    } else {
      c->cv.wait_for(lk, busy ? std::chrono::milliseconds(1) : std::chrono::milliseconds(20));
    }
  }
}

// One pool tick of logical GPU i (L250-L256 histogram-driven size, R44; L269
// reclaim): pre-warm one segment toward the target, trim back to
// max(used, target) once the excess has lasted kTrimDelay and the GPU's
// servers are idle.  The slow driver calls (create / map / set access;
// unmap) run WITHOUT the context lock.
static void pool_tick(grouter_ctx *c, size_t i, std::unique_lock<std::mutex> &lk) {
  static const bool diag = getenv("GR_DIAG") != nullptr;
  LogicalDev &d = c->dev[i];
  DeviceGuard g(d.phys);
  d.pool.heap.reclaim();
  const uint64_t tgt = pool_target(c, (int)i);
  const uint64_t t0 = diag ? now_ns() : 0, m0 = d.pool.mapped;
  if (d.pool.mapped < tgt && !(c->cfg.flags & GROUTER_NO_POOL)) {
    const uint64_t need = charge(std::min<uint64_t>(tgt - d.pool.mapped, 64ull << 20));
    const uint64_t seg = std::max<uint64_t>(need, 64ull << 20);
    uint64_t off = 0;
    if (d.pool.reserve(seg, off)) {
      const CUdeviceptr base = d.pool.base;
      const int phys = d.pool.phys;
      const std::vector<int> access = d.pool.access;
      lk.unlock();
      bool ok = true;
      DevicePool::Seg sg{};
      try {
        sg = DevicePool::map_seg(base, off, seg, phys, access, false, need);
      } catch (const Error &) {
        ok = false;  // HBM short: pre-warming is best effort
      }
      lk.lock();
      if (ok) d.pool.publish(sg);
      else d.pool.unreserve(off, seg);
    }
  }
  const uint64_t t1 = diag ? now_ns() : 0, m1 = d.pool.mapped;
  const uint64_t keep = std::max<uint64_t>(d.used, tgt) + (64ull << 20);
  const uint64_t tnow = now_ns();
  if (d.pool.mapped <= keep) d.pool.excess_since = 0;
  else if (!d.pool.excess_since) d.pool.excess_since = tnow;
  const bool idle = d.copy.inflight.empty() && d.h2d.inflight.empty() && d.d2h.inflight.empty() &&
                    !has_work(d.copy) && !has_work(d.h2d) && !has_work(d.d2h);
  if (d.pool.excess_since && tnow - d.pool.excess_since >= kTrimDelayNs && idle) {
    std::vector<DevicePool::Seg> v = d.pool.detach(keep);
    if (!v.empty()) {
      const CUdeviceptr base = d.pool.base;
      lk.unlock();
      DevicePool::unmap(base, v);
      lk.lock();
      d.pool.settle(v);
    }
    d.pool.excess_since = 0;
  }
  if (diag && now_ns() - t0 > 5000000)
    fprintf(stderr, "[grouter diag] pool tick dev %zu: grow %.1f ms (%llu -> %llu MiB), trim %.1f ms "
                    "(-> %llu MiB), used %llu MiB, target %llu MiB\n",
            i, (t1 - t0) / 1e6, (unsigned long long)(m0 >> 20), (unsigned long long)(m1 >> 20),
            (now_ns() - t1) / 1e6, (unsigned long long)(d.pool.mapped >> 20),
            (unsigned long long)(d.used >> 20), (unsigned long long)(tgt >> 20));
}

// Housekeeping thread: the auto cap (O10), pool pre-warm / trim, quarantine
// reclaim, bounded bookkeeping -- off the dispatch thread, so a slow driver
// call here never holds back a batch.
static void pool_main(grouter_ctx *c) {
  std::unique_lock<std::mutex> lk(c->mu);
  auto last_trim = std::chrono::steady_clock::now();
  auto last_cap = last_trim;
  while (!c->stop) {
    try {
      auto now = std::chrono::steady_clock::now();
      // auto cap (O10, L262): re-read available memory and migrate / restore
      // to stay within permille of it
      if (!c->replay && c->cfg.auto_cap_period_us &&
          now - last_cap >= std::chrono::microseconds(c->cfg.auto_cap_period_us)) {
        last_cap = now;
        for (size_t i = 0; i < c->dev.size(); ++i)
          if (c->dev[i].auto_cap) {
            bool ok = false;
            const size_t nv = c->victims.size(), nr = c->restored.size();
            refresh_cap(c, (int)i, GROUTER_AUTO_AVAIL, &ok);
            c->victims.resize(nv);  // grouter_victims lists the API calls' own victims
            c->restored.resize(nr);
          }
      }
      if (now - last_trim > std::chrono::milliseconds(50)) {  // I/O thread: reclaim (L269)
        last_trim = now;
        for (size_t i = 0; i < c->dev.size() && !c->stop; ++i) {
          if (i == 0 && !c->nopool_pending.empty()) nopool_sweep(c, false);
          for (Server *sv : {&c->dev[i].copy, &c->dev[i].h2d, &c->dev[i].d2h})
            sv->sched.prune();  // idle tenants (no-op for dispatch)
          if (i == 0) {  // rate-monitor records older than its 10 s horizon; bounded per-tenant counters
            const uint64_t tn = c->clock_fixed ? c->clock_ns : now_ns();
            for (auto it = c->tenant_log.begin(); it != c->tenant_log.end();)
              if (it->second.empty() || it->second.back().first + 10000000000ull < tn) it = c->tenant_log.erase(it);
              else ++it;
            // pool-sizing histograms (R44, R50): with more than 4096 functions
            // tracked, forget those whose window closed over 60 s ago (one
            // workflow id per request would otherwise grow the table -- and
            // this tick's pool_target scan -- without bound)
            if (c->hists.size() > 4096)
              for (auto it = c->hists.begin(); it != c->hists.end();) {
                const FuncHist &h = it->second;
                if (!h.arrivals.empty() && !h.active(tn) && h.arrivals.back() + h.r_window() + 60000000000ull < tn)
                  it = c->hists.erase(it);
                else ++it;
              }
            if (c->tenant_bytes.size() > (1u << 16))
              for (auto it = c->tenant_bytes.begin(); it != c->tenant_bytes.end();)
                if (!c->tenant_log.count(it->first)) it = c->tenant_bytes.erase(it);
                else ++it;
          }
          pool_tick(c, i, lk);
        }
        c->host.heap.reclaim();
        if (!c->ded_retire.empty()) ded_sweep(c, &lk, false);  // exported objects' own allocations
      }
    } catch (const Error &e) {
      set_error(e.what());
      c->sticky_error = true;
      c->submit_cv.notify_all();  // callers blocked in order_after fail with ECUDA
    }
    c->pool_cv.wait_for(lk, std::chrono::milliseconds(10));
  }
}

void engine_init(grouter_ctx *c) {
  const int n = (int)c->cfg.n_gpus;
  int ndev = 0;
  GR_CUDA(cudaGetDeviceCount(&ndev));
  for (int i = 0; i < n; ++i) {
    int p = c->cfg.device_map[i];
    if (p < 0 || p >= ndev) throw Error(GROUTER_EINVAL, "device_map entry out of range");
    if (!c->phys.count(p)) {
      auto pd = std::make_unique<PhysDev>();
      pd->ordinal = p;
      pd->events.phys = p;
      GR_CUDA(cudaDeviceGetAttribute(&pd->sm_count, cudaDevAttrMultiProcessorCount, p));
      {
        DeviceGuard g(p);
        pd->n_scratch = 256;
        GR_CUDA(cudaMalloc(&pd->scratch, (size_t)pd->n_scratch * 2 * sizeof(uint32_t)));
        GR_CUDA(cudaMemset(pd->scratch, 0, (size_t)pd->n_scratch * 2 * sizeof(uint32_t)));
        pd->scratch_busy.assign(pd->n_scratch, {});
      }
      c->phys[p] = std::move(pd);
    }
  }
  // peer access between every pair of physical GPUs that supports it
  std::vector<int> phys_list;
  for (auto &kv : c->phys) phys_list.push_back(kv.first);
  for (int a : phys_list)
    for (int b : phys_list) {
      if (a == b) continue;
      int ok = 0;
      cudaDeviceCanAccessPeer(&ok, a, b);
      if (ok) {
        DeviceGuard g(a);
        cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
          throw Error(GROUTER_ECUDA, "cudaDeviceEnablePeerAccess failed");
        cudaGetLastError();
      }
    }
  // completion words (pinned, mapped; written by kernels and copy engines)
  c->n_slots = kSlots;
  GR_CUDA(cudaHostAlloc((void **)&c->words, (size_t)kSlots * GROUTER_MAX_PATHS * 4,
                        cudaHostAllocMapped | cudaHostAllocPortable));
  std::memset(c->words, 0, (size_t)kSlots * GROUTER_MAX_PATHS * 4);
  c->slot_final.assign(kSlots, {});
  // circular pinned bounce ring for pageable host sources (L229)
  c->bounce_slots = kBounceSlots;
  GR_CUDA(cudaHostAlloc((void **)&c->bounce, (size_t)kBounceSlots * c->cfg.chunk_bytes,
                        cudaHostAllocPortable));
  c->bounce_ev.assign(kBounceSlots, nullptr);
  // pinned host store (+ headroom so page fragmentation does not decide a
  // placement that the capacity accounting admitted)
  c->host_cap = c->cfg.host_store_bytes / kPage * kPage;
  c->host.size = (c->host_cap + c->host_cap / 4 + (64ull << 20)) / kPage * kPage;
  GR_CUDA(cudaHostAlloc((void **)&c->host.base, c->host.size,
                        cudaHostAllocMapped | cudaHostAllocPortable));
  c->host.heap.give(0, c->host.size / kPage * kPage);
  // per logical GPU: pool, servers
  const bool multi = n > 1 && !(c->cfg.flags & GROUTER_NO_MULTIPATH);
  for (int i = 0; i < n; ++i) {
    gr::LogicalDev &d = c->dev[i];
    d.phys = c->cfg.device_map[i];
    DeviceGuard g(d.phys);
    size_t fr = 0, tot = 0;
    GR_CUDA(cudaMemGetInfo(&fr, &tot));
    if (c->cfg.pool_cap_bytes[i]) {
      d.cap = c->cfg.pool_cap_bytes[i];
    } else {  // auto mode (O10): nothing mapped yet, so available = free
      d.auto_cap = true;
      d.cap = auto_cap_bytes(c->cfg.pool_cap_permille, fr);
      c->stats.auto_avail[i] = fr;
    }
    uint64_t prewarm = std::min<uint64_t>(c->cfg.pool_floor_bytes, d.cap == GROUTER_UNLIMITED ? c->cfg.pool_floor_bytes : d.cap);
    if (c->cfg.flags & GROUTER_NO_POOL) prewarm = 0;  // ablation: nothing pooled
    d.pool.init(i, d.phys, (uint64_t)tot * 2 / kPage * kPage, phys_list, prewarm / kPage * kPage);
    Server *ss[3] = {&d.copy, &d.h2d, &d.d2h};
    for (int k = 0; k < 3; ++k) {
      Server &s = *ss[k];
      s.kind = k;
      s.logical = i;
      s.phys = d.phys;
      s.sched.batch = c->cfg.batch_chunks;
      int lo = 0, hi = 0;
      cudaDeviceGetStreamPriorityRange(&lo, &hi);
      // SM-copy rounds run at the highest priority (they share SMs with the
      // functions' kernels); copy-engine streams at the default one: a memcpy
      // on a high-priority stream costs ~2.2 us more host time and ~2 us more
      // latency per call (tools/celat.cu), and priority buys a CE nothing
      static const bool ce_hi = getenv("GR_CE_PRIO_HI") != nullptr;
      GR_CUDA(cudaStreamCreateWithPriority(&s.stream, cudaStreamNonBlocking, (k == SK_COPY || ce_hi) ? hi : lo));
      if (k != SK_COPY) GR_CUDA(cudaStreamCreateWithFlags(&s.pub_stream, cudaStreamNonBlocking));  // publish_ce
    }
    GR_CUDA(cudaMalloc(&d.copy.scratch, 64));
    GR_CUDA(cudaMemset(d.copy.scratch, 0, 64));
    if (multi) {
      int lo = 0, hi = 0;
      cudaDeviceGetStreamPriorityRange(&lo, &hi);
      GR_CUDA(cudaStreamCreateWithPriority(&d.h2d.fwd_stream, cudaStreamNonBlocking, hi));
      GR_CUDA(cudaMalloc(&d.h2d.fwd_scratch, 64));
      GR_CUDA(cudaMemset(d.h2d.fwd_scratch, 0, 64));
      d.h2d.n_slots = 4 * c->cfg.batch_chunks;  // two rounds of two batches in flight
      d.h2d.slot_bytes = c->cfg.chunk_bytes;
      GR_CUDA(cudaMalloc(&d.h2d.staging, (size_t)d.h2d.n_slots * d.h2d.slot_bytes));
      d.h2d.slot_free.assign(d.h2d.n_slots, nullptr);
    }
    GR_CUDA(cudaDeviceSynchronize());
  }
  c->daemon = std::thread(daemon_main, c);
  c->pool_thread = std::thread(pool_main, c);
}

void engine_shutdown(grouter_ctx *c) {
  {
    std::lock_guard<std::mutex> lk(c->mu);
    c->stop = true;
  }
  c->cv.notify_all();
  c->pool_cv.notify_all();
  c->submit_cv.notify_all();
  if (c->daemon.joinable()) c->daemon.join();
  if (c->pool_thread.joinable()) c->pool_thread.join();
  // drain the library's own streams (never the device: a caller stream may be
  // parked on a completion word that will not arrive after an error)
  auto t0 = std::chrono::steady_clock::now();
  for (auto &d : c->dev) {
    DeviceGuard g(d.phys);
    for (Server *s : {&d.copy, &d.h2d, &d.d2h})
      for (cudaStream_t st : {s->stream, s->fwd_stream, s->pub_stream})
        while (st && cudaStreamQuery(st) == cudaErrorNotReady &&
               std::chrono::steady_clock::now() - t0 < std::chrono::seconds(10))
          std::this_thread::sleep_for(std::chrono::microseconds(100));
  }
  try {  // GROUTER_NO_POOL: every buffer still allocated goes back
    if (!c->sticky_error && !c->nopool_pending.empty()) {
      pump(c, true);  // replay: submit what the pending buffers wait for
      nopool_sweep(c, true);
    }
  } catch (const Error &) {
  }
  for (auto &kv : c->nopool_live) {
    DeviceGuard g(kv.second);
    cudaFree(kv.first);
  }
  c->nopool_live.clear();
  c->nopool_pending.clear();
  for (auto &d : c->dev) {
    DeviceGuard g(d.phys);
    Server *ss[3] = {&d.copy, &d.h2d, &d.d2h};
    for (Server *s : ss) {
      s->inflight.clear();
      s->slot_free.clear();
      if (s->stream) cudaStreamDestroy(s->stream);
      if (s->fwd_stream) cudaStreamDestroy(s->fwd_stream);
      if (s->pub_stream) cudaStreamDestroy(s->pub_stream);
      if (s->scratch) cudaFree(s->scratch);
      if (s->fwd_scratch) cudaFree(s->fwd_scratch);
      if (s->staging) cudaFree(s->staging);
    }
    d.pool.heap.quarantine.clear();
    d.pool.destroy();
  }
  for (auto &kv : c->phys) {
    DeviceGuard g(kv.first);
    if (kv.second->scratch) cudaFree(kv.second->scratch);
    for (cudaEvent_t e : kv.second->timing_free) cudaEventDestroy(e);
    if (kv.second->stamps) cudaFree(kv.second->stamps);
    kv.second->scratch_busy.clear();
  }
  ipc_release_all(c);  // dedicated (exported) allocations; their fences hold pooled events
  c->prof.clear();
  c->live.clear();
  delete c->params;
  c->params = nullptr;
  c->bounce_ev.clear();
  c->host.heap.quarantine.clear();
  if (c->host.base) cudaFreeHost(c->host.base);
  if (c->bounce) cudaFreeHost(c->bounce);
  if (c->words) cudaFreeHost(c->words);
  // fences may hold pooled events: drop them while the pools are alive
  for (auto &kv : c->objects) {
    kv.second.ready.clear();
    kv.second.readers.clear();
  }
  for (auto &kv : c->leases) kv.second.fill.clear();
  c->phys.clear();
}

}  // namespace gr
