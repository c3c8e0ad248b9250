// ctx.h -- the libgrouter runtime: pools, servers, transfers, object table.
//
// Layering: api.cpp (the C ABI, object table, auth, refcounts,
// eviction: PAPER.md L165-L173, L248-L262, L394) sits on engine.cpp (per-GPU
// servers, stride scheduling, dispatch rounds, completion words: L182,
// L193-L229, L269-L271) which drives the sm_100a kernels of kernels.cu and
// the copy engines; pool.cpp holds the VMM device pools, the pinned host
// store and the staging rings (L229, L248-L256, L269).
#pragma once

#include <array>
#include <atomic>
#include <condition_variable>
#include <deque>
#include <map>
#include <memory>
#include <set>
#include <thread>
#include <unordered_map>
#include <vector>

#include "common.h"
#include "plan.h"
#include "stride.h"

namespace gr {

// ------------------------------------------------------------------ pages
struct Quarantined {
  uint64_t off, len;
  Fences fences;
};

// Page-granular first-fit allocator over offsets, with a quarantine of
// freed runs that in-flight GPU work may still touch.
struct PageHeap {
  std::map<uint64_t, uint64_t> free_runs;  // offset -> length
  std::vector<Quarantined> quarantine;
  bool take(uint64_t len, uint64_t *off);
  void give(uint64_t off, uint64_t len);
  void reclaim();                           // returns quarantined runs whose fences are done
  uint64_t free_bytes() const;
  uint64_t tail_free(uint64_t end) const;   // length of the free run ending at `end`
};

struct DevicePool {
  int logical = -1, phys = -1;
  CUdeviceptr base = 0;
  // mapped: physical bytes mapped; va_top: VA offset where the next segment
  // maps (> mapped only while detached segments are being unmapped, or after
  // a grow raced an unmap and left a hole that is never handed out)
  uint64_t va_size = 0, mapped = 0, va_top = 0;
  uint64_t excess_since = 0;  // ns since mapped first exceeded the trim mark (0 = not over)
  struct Seg {
    uint64_t off, size;
    CUmemGenericAllocationHandle h;
  };
  std::vector<Seg> segs;
  PageHeap heap;
  std::vector<int> access;  // physical devices that may access the pages
  void init(int logical, int phys, uint64_t va, const std::vector<int> &access, uint64_t prewarm);
  void grow(uint64_t need);  // on demand, lock held
  // pre-warm in three steps so the driver calls (cuMemCreate / cuMemSetAccess
  // took up to ~60 ms while copies streamed, tools/vmmlat.cu) run without the
  // context lock and off the dispatch thread: reserve() takes a VA range
  // (lock held), map_seg() creates and maps it (lock NOT held), publish()
  // hands it to the heap (lock held); unreserve() after a failed map_seg
  bool reserve(uint64_t size, uint64_t &off);
  static Seg map_seg(CUdeviceptr base, uint64_t off, uint64_t size, int phys, const std::vector<int> &access,
                     bool fallback_ok, uint64_t need);
  void publish(const Seg &s);
  void unreserve(uint64_t off, uint64_t size);
  // trim in two steps so the (slow, up to ~0.8 s measured) cuMemUnmap runs
  // without the context lock: detach() takes trailing free segments out of
  // the heap (lock held), unmap() releases them (lock NOT held), settle()
  // lowers va_top again when nothing mapped above them meanwhile (lock held)
  std::vector<Seg> detach(uint64_t keep);
  static void unmap(CUdeviceptr base, const std::vector<Seg> &segs);
  void settle(const std::vector<Seg> &segs);
  void trim(uint64_t keep);  // all three steps with the lock held (tests, shutdown)
  void destroy();
};

// Pool-sizing samples of one function on one GPU (L250-L256, Fig. 11a; R44):
// arrival times, page charges and resident-object counts, last kHist each.
struct FuncHist {
  static constexpr size_t kHist = 1024;
  std::deque<uint64_t> arrivals, sizes, cons;
  void observe(uint64_t t, uint64_t size, uint64_t con);
  uint64_t r_window() const;   // p99 inter-arrival interval, 0 with < 2 arrivals
  uint64_t data_size() const;  // Data_size = R_size * R_con (saturating)
  bool active(uint64_t t) const { return !arrivals.empty() && t <= arrivals.back() + r_window(); }
};

struct HostStore {
  uint8_t *base = nullptr;
  uint64_t size = 0;
  PageHeap heap;
};

// ------------------------------------------------------------------ transfers
enum ServerKind { SK_COPY = 0, SK_H2D = 1, SK_D2H = 2 };

struct Xfer {
  uint64_t id = 0;
  uint32_t tenant = 0;
  uint32_t slot = 0;
  volatile uint32_t *words = nullptr;       // host-mapped completion words of the slot
  uint32_t target[GROUTER_MAX_PATHS] = {};  // final word value per path
  uint32_t total[GROUTER_MAX_PATHS] = {};   // chunks per path
  uint32_t issued[GROUTER_MAX_PATHS] = {};  // chunks dispatched so far per path
  // absolute word value once the first `issued` chunks of `path` are done
  uint32_t value_after(uint32_t path) const { return target[path] - total[path] + issued[path]; }
  uint32_t npath = 0;
  Fences deps;                              // must complete before the first chunk moves
  uint64_t deps_waited = 0;                 // bitmask of servers that already waited
  uint64_t epoch = 0;
  bool pageable_src = false;
  bool local_src = false;                   // source = pool pages of the copying GPU (L2 prefetch safe)
  uint32_t nchunks = 0, submitted_chunks = 0;
  bool submitted() const { return submitted_chunks == nchunks; }
  struct Waiter {
    cudaStream_t stream;
    Waitable w;
  };
  std::vector<Waiter> waiters;              // caller-stream waits deferred until submission
  // completion evidence when no word is published: an event recorded on the
  // caller stream after a direct launch that moved the whole transfer (its
  // completion slot is handed back at once)
  EventRef done_ev;
  cudaStream_t done_stream = nullptr;      // stream done_ev was recorded on
  // word fences were handed out (done_fences before the transfer's rounds
  // ran): its words must be published, an event may not stand in for them
  mutable bool word_fenced = false;
  bool done() const;
};
using XferRef = std::shared_ptr<Xfer>;

struct ChunkItem {
  Xfer *x;            // kept alive by grouter_ctx::live until fully submitted
  uint32_t idx;       // chunk index in the plan
  uint32_t path;
  uint64_t src, dst;  // absolute addresses (device VA or host)
  uint64_t bytes;
  int dst_logical;    // destination device (H2D: relay if != server device)
};

struct Server {
  int kind = 0, logical = -1, phys = -1;
  Stride<ChunkItem> sched;
  cudaStream_t stream = nullptr;      // SM-copy stream / CE stream
  cudaStream_t fwd_stream = nullptr;  // H2D: relay forward kernel stream
  cudaStream_t pub_stream = nullptr;  // CE servers: completion-word writes (publish_ce)
  uint32_t *scratch = nullptr;        // device scratch of the copy kernel on `stream`
  uint32_t *fwd_scratch = nullptr;    // ... on `fwd_stream`
  struct Inflight {
    Waitable w;                  // completion of a dispatched round
    cudaStream_t direct;         // caller stream of a direct launch, null for the server stream
    uint32_t batches = 0;        // scheduled batches the round carries (O8: <= 2 in flight)
  };
  std::deque<Inflight> inflight;
  std::deque<ChunkItem> carry;        // scheduled (stride order) but not yet submitted
  std::deque<ChunkItem> urgent;       // unscheduled work (spills), FIFO
  // H2D relay staging ring on this GPU (device memory)
  uint8_t *staging = nullptr;
  uint32_t n_slots = 0, next_slot = 0;
  uint64_t slot_bytes = 0;
  std::vector<EventRef> slot_free;
  uint64_t id_bit() const { return 1ull << (kind * GROUTER_MAX_GPUS + logical); }
};

// ------------------------------------------------------------------ objects
// An object imported from another process (grouter_import_ipc): its bytes
// live in the exporter's pool; this process maps the exporter's segments.
struct RemoteMap {
  CUdeviceptr va = 0;
  uint64_t size = 0;
  std::vector<CUmemGenericAllocationHandle> handles;
  std::vector<uint64_t> sizes;
  int phys = -1;   // local CUDA ordinal holding the bytes, -1 if not visible
};

// An exported object's own VMM allocation (ipc.cpp, R52): the
// importer can map it and nothing else; it never returns to the pool.
struct Dedicated {
  int logical = -1, phys = -1;
  CUdeviceptr va = 0;
  uint64_t size = 0;
  CUmemGenericAllocationHandle h = 0;
  int fd = -1;                        // POSIX fd of h, created at the first export
  std::vector<uint64_t> export_ids;   // live exports (grouter_ctx::exports)
};
struct ExportRec {
  uint64_t nonce[2];                  // 128-bit random capability carried by the descriptor
  uint64_t va;                        // the Dedicated it serves
};
struct DedRetire {
  Dedicated d;
  Fences f;                           // unmapped once these complete
};

enum ObjState { OBJ_OPEN, OBJ_SEALED, OBJ_CONSUMED, OBJ_FREED };

struct Obj {
  grouter_oid oid = 0;
  uint32_t wf = 0, fid = 0;
  uint64_t n = 0;
  int loc = GROUTER_HOST;
  uint8_t *ptr = nullptr;          // device VA or host-store address
  ObjState state = OBJ_OPEN;
  uint32_t consumers_left = 0;
  uint32_t pins = 0;
  uint64_t last_access = 0;
  bool has_next_use = false;
  uint64_t next_use = 0;
  int home = -1;                   // GPU it was migrated away from (proactive restore)
  Fences ready;                    // the bytes are in place once these complete
  Fences readers;                  // in-flight library reads of the bytes
  std::shared_ptr<RemoteMap> remote;  // loc == GROUTER_REMOTE
};

struct Lease {
  grouter_oid oid;
  uint32_t wf;
  int dev;
  uint8_t *ptr;
  uint64_t n;
  Fences fill;                     // the copy into the lease
};

struct LogicalDev {
  int phys = -1;
  DevicePool pool;
  uint64_t used = 0, cap = GROUTER_UNLIMITED;
  bool auto_cap = false;  // cap follows available memory (O10, grouter_refresh_cap)
  Server copy, h2d, d2h;
};

struct CopyParamsHost;  // kernels.h CopyParams, boxed (keeps kernels.h out of this header)

struct PhysDev {
  int ordinal = -1;
  int sm_count = 148;
  EventPool events;
  // copy-kernel scratch pairs for direct launches on caller streams; a pair
  // is reusable once the launch that used it has completed
  uint32_t *scratch = nullptr;
  uint32_t n_scratch = 0, next_scratch = 0;
  std::vector<Fences> scratch_busy;
  std::vector<cudaEvent_t> timing_free;  // timing-enabled events (GROUTER_PROFILE)
  // GROUTER_PROFILE kernel stamps (%globaltimer start/end per launch, device
  // memory, a ring of slots; a slot is reused once its launch was harvested)
  unsigned long long *stamps = nullptr;
  std::vector<char> stamp_busy;
  uint32_t next_stamp = 0;
};

struct ProfRec {
  int phys;
  cudaEvent_t start, stop;
  uint64_t bytes;
  int stamp = -1;  // slot of PhysDev::stamps, -1 if none was free
};

}  // namespace gr

struct grouter_ctx {
  grouter_config cfg;
  gr::Planner planner;
  bool plan_only = false, replay = false;
  std::mutex mu;                                       // the big lock
  // API callers blocked on `mu` (Guard): the dispatch thread's spin leaves the
  // lock alone while any wait, so a spinning dispatch loop cannot starve them
  std::atomic<int> lock_waiters{0};
  std::vector<gr::LogicalDev> dev;
  std::map<int, std::unique_ptr<gr::PhysDev>> phys;
  gr::HostStore host;
  uint64_t host_used = 0, host_cap = 0;
  // completion slots (host-mapped pinned memory)
  uint32_t *words = nullptr;
  uint32_t n_slots = 0, next_slot = 0;
  std::vector<std::array<uint32_t, GROUTER_MAX_PATHS>> slot_final;
  // pageable-source bounce ring (the circular pinned buffer of L229)
  uint8_t *bounce = nullptr;
  uint32_t bounce_slots = 0, bounce_next = 0;
  std::vector<gr::EventRef> bounce_ev;
  // object table (L173)
  std::unordered_map<grouter_oid, gr::Obj> objects;
  std::unordered_map<uintptr_t, gr::Lease> leases;     // copy leases by address
  std::unordered_map<uint32_t, uint32_t> weights;
  std::unordered_map<uint32_t, std::array<uint64_t, 3>> tenant_bytes;  // dispatched, per server kind
  // rate monitor (L197): (dispatch time ns, bytes) per dispatched batch, last 10 s
  std::unordered_map<uint32_t, std::deque<std::pair<uint64_t, uint64_t>>> tenant_log;
  // GROUTER_NO_POOL (ablation): live cudaMalloc'ed buffers (ptr -> physical
  // device) and frees waiting for the buffer's GPU work to complete
  struct NoPoolFree {
    uint8_t *p;
    gr::Fences f;
  };
  std::unordered_map<uint8_t *, int> nopool_live;
  std::vector<NoPoolFree> nopool_pending;
  std::map<uint32_t, std::array<uint64_t, 3>> slos;    // wf -> (data, slo_ns, infer_ns), R43
  // pool sizing (R44): per (wf, fid, gpu) histograms and resident counts
  std::map<std::tuple<uint32_t, uint32_t, int>, gr::FuncHist> hists;
  std::map<std::tuple<uint32_t, uint32_t, int>, uint64_t> resident;
  bool clock_fixed = false;                            // grouter_test_set_clock
  uint64_t clock_ns = 0;
  uint64_t seq = 0, next_oid = 1, xfer_seq = 0;
  uint64_t epoch = 1, flushed_epoch = 0;               // replay grounding
  std::vector<grouter_oid> victims;
  std::vector<grouter_oid> restored;                   // GROUTER_RESTORE (L260)
  bool restore_on = false;
  std::deque<gr::ProfRec> prof;                        // GROUTER_PROFILE launches not yet harvested
  std::unordered_map<gr::Xfer *, gr::XferRef> live;    // transfers with chunks not yet submitted
  gr::CopyParamsHost *params = nullptr;                // reused kernel-parameter builder (engine.cpp)
  std::deque<grouter_dispatch> dlog;
  grouter_stats_t stats{};
  // background I/O + dispatch thread (L269, L271)
  std::thread daemon;
  std::thread pool_thread;               // pool pre-warm / trim, auto cap, housekeeping
  std::condition_variable pool_cv;
  std::condition_variable cv;
  std::condition_variable submit_cv;                   // a transfer became fully submitted
  bool stop = false;
  std::atomic<bool> sticky_error{false};
  int inject_round_failures = 0;                       // grouter_test_inject (tests only)
  // cross-process export (ipc.cpp)
  uint32_t ctx_id = 0;
  int ipc_listen = -1;
  std::thread ipc_thread;
  std::map<uint64_t, gr::Dedicated> dedicated;         // by VA: exported objects' own allocations
  std::unordered_map<uint64_t, gr::ExportRec> exports;   // live exports by id
  uint64_t next_export_id = 1;
  std::vector<gr::DedRetire> ded_retire;                 // freed dedicated allocations
};

namespace gr {
struct CopyParamsHost;
// engine.cpp
void engine_init(grouter_ctx *c);
void engine_shutdown(grouter_ctx *c);
XferRef new_xfer(grouter_ctx *c, uint32_t tenant, const std::vector<grouter_chunk> &plan);
// Enqueue every chunk of a planned transfer to its server.  src_base/dst_base
// are the absolute base addresses; kind = server kind for single-path plans,
// SK_H2D for host->GPU plans.
void enqueue_plan(grouter_ctx *c, const XferRef &x, const std::vector<grouter_chunk> &plan,
                  int kind, uint64_t src_base, uint64_t dst_base, int dst_logical);
void pump(grouter_ctx *c, bool force_all);            // dispatch rounds (caller holds mu)
void flush_all(grouter_ctx *c);                        // replay flush
void nopool_sweep(grouter_ctx *c, bool wait);            // GROUTER_NO_POOL deferred cudaFree
void harvest_profile(grouter_ctx *c, bool wait);       // completed timed launches -> stats
// Same-GPU SM copy run directly on the caller's stream when its copy server
// is idle (or only busy with direct launches on that same stream).  Returns
// false (nothing done) when the server path must be used.
bool try_direct(grouter_ctx *c, const XferRef &x, int server_logical, cudaStream_t caller, int caller_phys);
XferRef fast_ce(grouter_ctx *c, uint32_t tenant, int kind, const std::vector<grouter_chunk> &plan, uint64_t src,
                uint64_t dst, uint64_t n, const Fences &deps);
XferRef fast_direct(grouter_ctx *c, uint32_t tenant, int server_logical, int dst_logical, uint64_t src,
                    uint64_t dst, uint64_t n, bool local_src, const Fences &deps, cudaStream_t caller,
                    int caller_logical);
void stream_wait(grouter_ctx *c, cudaStream_t s, int phys, const Fences &f);  // submitted fences only
// Waits on a CALLER stream: submitted fences now, the others as soon as their
// producer transfer is submitted.
void caller_wait(grouter_ctx *c, cudaStream_t s, const Fences &f);
void done_fences(const XferRef &x, Fences &f);
bool is_submitted(const Waitable &w);
EventRef record(grouter_ctx *c, cudaStream_t s, int phys);       // library streams only
Waitable signal(grouter_ctx *c, cudaStream_t s, int phys);       // caller streams
// abort (optional): a sticky-error flag; a wait on words that will never be
// written (the producing round failed) ends with ECUDA instead of the timeout
void host_wait(const Fences &f, double timeout_s = 120.0, const std::atomic<bool> *abort = nullptr);
bool grounded(const grouter_ctx *c, const Fences &f);
void spill_copy(grouter_ctx *c, Obj &o, uint8_t *host_dst);  // D2H of a victim (unscheduled)
void restore_copy(grouter_ctx *c, Obj &o, int d, uint8_t *dev_dst);  // H2D back home (unscheduled)
// ipc.cpp
void ipc_serve_start(grouter_ctx *c);
void ipc_shutdown(grouter_ctx *c);
std::shared_ptr<RemoteMap> ipc_map(grouter_ctx *c, const grouter_ipc_desc &d, int local_phys);
void ipc_unmap(RemoteMap &m);
void ipc_dedicate(grouter_ctx *c, Obj &o);                       // move into an own allocation
uint64_t ipc_export_record(grouter_ctx *c, uint64_t va, uint64_t nonce[2]);
bool ded_free(grouter_ctx *c, uint8_t *p, Fences &&f);          // false: not dedicated
// cap_d := bytes; migrate victims until used <= cap, then restore what fits
// (L262); false when unevictable data keeps the pool above the cap
bool apply_cap(grouter_ctx *c, int d, uint64_t bytes);
// O10 (R12, R54): cap = floor(avail * permille / 1000 / page) * page
uint64_t auto_cap_bytes(uint32_t permille, uint64_t avail);
// auto mode on d: measure (avail == GROUTER_AUTO_AVAIL) or take avail, apply
// the O10 cap; *ok = apply_cap's result; returns the cap
uint64_t refresh_cap(grouter_ctx *c, int d, uint64_t avail, bool *ok);
void ded_sweep(grouter_ctx *c, std::unique_lock<std::mutex> *lk, bool wait);
void ipc_release_all(grouter_ctx *c);
// pool.cpp
uint64_t pool_target(grouter_ctx *c, int logical);   // R44 target at the current clock
// may grow the pool; with `lk` (the caller's hold on c->mu, real-time mode)
// the growth's driver calls run with the lock released -- only for callers
// that hold no reference into the object table across the call (put, alloc)
uint8_t *dev_alloc(grouter_ctx *c, int logical, uint64_t len, std::unique_lock<std::mutex> *lk = nullptr);
void dev_free(grouter_ctx *c, int logical, uint8_t *p, uint64_t len, Fences &&f);
uint8_t *host_alloc(grouter_ctx *c, uint64_t len);
void host_free(grouter_ctx *c, uint8_t *p, uint64_t len, Fences &&f);
}  // namespace gr
