/*
 * grouter.h -- C ABI of the B200-native GROUTER data-passing hot path.
 *
 * What this library is (PAPER.md = marker text of Wu et al., EuroSys '26):
 *   L165 §4.2.1  Put() stores an intermediate object locally and returns a
 *                globally unique id; Get(id) retrieves it and picks the
 *                transfer method from the consumer's placement.
 *   L167 §4.2.2  same GPU -> zero copy (share the address); other GPU ->
 *                allocate on the consumer GPU and copy over NVLink; host ->
 *                stage over parallel PCIe links, then map.
 *   L178-L182    host<->GPU traffic striped over route GPUs' PCIe links,
 *                forwarded over NVLink; payloads cut in 2 MB chunks under a
 *                precomputed plan; in-order delivery.
 *   L193-L229    per-function bandwidth shares; batches of 5 chunks.
 *   L248-L262    elastic GPU pool (2 MiB pages here), 50%-of-free cap,
 *                queue-aware migration to pinned host memory.
 *   L260         data no longer needed is removed promptly.
 *   L394 §7      every access is authenticated by function id + workflow id.
 * Readings of silent/ambiguous points (R1 onward) are listed in DESIGN.md §3.
 *
 * Conventions (all calls):
 *   - Every call returns a grouter_status; on error outputs are untouched
 *     and no C++ exception crosses the ABI.  CUDA failures -> GROUTER_ECUDA
 *     (sticky; grouter_last_error() has the text).
 *   - "stream" arguments are a cudaStream_t (CUstream) of the caller's
 *     device passed as void*.  Device callers are stream-ordered: a put reads
 *     `src` after prior work on the stream, and the stream cannot overwrite
 *     `src` before the library's copy completes; a get returns at once and
 *     work enqueued on the stream afterwards sees the data.  A NULL stream
 *     means a host caller: the call blocks until the bytes are in place.
 *   - Ownership: the caller owns put `src` and get_into `dst`; the library
 *     owns object pages, leases, staging rings and the host store.  A lease
 *     stays valid until grouter_release(); a zero-copy lease aliases the
 *     object and must not be written.
 *   - n == 0 is valid: empty plan, get returns ptr = NULL, n = 0, GROUTER_OK.
 *   - All calls are thread-safe.
 */
#ifndef GROUTER_H
#define GROUTER_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GROUTER_MAX_GPUS 16
#define GROUTER_MAX_PATHS 8
#define GROUTER_HOST (-1)          /* location / device of a CPU function  */
#define GROUTER_NOHINT (-2)        /* put: no placement hint               */
#define GROUTER_REMOTE (-3)        /* location of an object imported from another process */
#define GROUTER_UNLIMITED UINT64_MAX

/* flags for grouter_config.flags */
#define GROUTER_REPLAY        0x1u /* dispatch only at grouter_flush() (deterministic log) */
#define GROUTER_NO_MULTIPATH  0x2u /* host->GPU uses the direct PCIe link only (ablation)  */
#define GROUTER_PLAN_ONLY     0x4u /* no CUDA at all: planner/introspection only            */
#define GROUTER_LOG           0x8u /* keep the dispatch log in real-time mode too           */
#define GROUTER_COPY_TMA      0x10u/* SM copy kernel uses cp.async.bulk (TMA) staging       */
#define GROUTER_PROFILE       0x20u/* time every copy-kernel launch with CUDA events on its stream
                                      (measurement mode: the events sit between launches and
                                      cost the programmatic-dependent-launch overlap)           */
#define GROUTER_D2H_MULTIPATH 0x80u/* gFn-host striping (L178, Fig. 5a; R45): a GPU
                                      object read into host memory is split over R(src) like a
                                      host->GPU plan; route r's copy engine moves its share      */
#define GROUTER_RESTORE       0x40u/* proactive restore (L260-L262): when pool storage is released
                                      or a cap is raised, objects migrated away from that GPU come
                                      back while they fit (R42)                      */
#define GROUTER_NO_POOL       0x200u/* ablation "ES off" (Fig. 16; L248 "cudaMalloc/cudaFree
                                      ... millisecond-level"): every object / lease is its own
                                      cudaMalloc, freed by cudaFree once its GPU work completed;
                                      accounting, caps and eviction unchanged; no IPC export  */
#define GROUTER_NO_TOPOLOGY   0x400u/* ablation "TA off" (Fig. 16; L131, L178): route sets
                                      ignore shared PCIe uplinks (every GPU its own uplink group,
                                      DESIGN.md R48), so GPUs behind one switch both stage data */
#define GROUTER_HOST_CENTRIC  0x800u/* ablation "UF off" (Fig. 16) / the host-centric data
                                      passing of L90: a GPU -> other-GPU copy goes through
                                      pinned host memory (D2H on the source's engine, then H2D on
                                      the destination's), one path each (R49)        */
#define GROUTER_STRIPED_MIGRATION 0x100u /* spills leave over R(src) on the route GPUs' D2H
                                      engines (the gFn-host plan, L178), restores come back over
                                      R(d) with relays like a fetch (L178, L366 "parallel PCIe
                                      transfers ... mitigate the overhead"); R47      */
#define GROUTER_CE_RELAY      0x2000u/* host->GPU striping without the staging hop: route GPU r's copy
                                      engine reads its share from host memory over r's PCIe link
                                      and writes the destination's pages directly (over NVLink on
                                      a multi-GPU box) -- no staging slot, no forward launch.
                                      Opt-in until measured on a multi-GPU box */
#define GROUTER_FORCE_REMOTE  0x1000u/* TEST ONLY: every copy-kernel round is launched as if its
                                      sources and destinations were on another GPU (the NVLink
                                      branch: system-scope fences, no L2 prefetch, no TMA bulk
                                      engine, completion published in-kernel), and a copy between
                                      two logical GPUs takes the dispatch of a physical pair: the
                                      source's copy server pushes it (the consumer waits on
                                      completion words), or, <= 4 MiB on an idle server, the
                                      consumer's stream pulls it (R55, R56), so one-GPU
                                      test boxes execute the code a physical peer transfer runs */
#define GROUTER_PULL_ALL      0x4000u/* MEASUREMENT: every GPU -> other-GPU copy requested on a
                                      consumer stream while the source's copy server is idle is
                                      pulled by the consumer GPU (R56 without its 4 MiB bound),
                                      so bench.py can time pull against push per size on a
                                      multi-GPU box (d2d_sweep_pull)                          */

typedef uint64_t grouter_oid;      /* opaque, 0 never valid: (node << 48) | seq, node 0 */
typedef struct grouter_ctx grouter_ctx;

typedef enum {
  GROUTER_OK = 0,
  GROUTER_EINVAL = 1,  /* bad argument, unknown device, dst_cap < n, unknown lease */
  GROUTER_ENOENT = 2,  /* unknown, freed, consumed or unsealed object            */
  GROUTER_EPERM = 3,   /* workflow mismatch (L394)                               */
  GROUTER_ENOMEM = 4,  /* pool/lease/alloc cannot fit after eviction; host full  */
  GROUTER_EBUSY = 5,   /* free of an unsealed object; no completion slot free    */
  GROUTER_ECUDA = 6,   /* CUDA error (sticky)                                    */
  GROUTER_ESTATE = 7   /* wrong object state (e.g. seal twice)                   */
} grouter_status;

/* A serverless function: its workflow, its id, and its resident device
 * (a logical GPU index 0..n_gpus-1, or GROUTER_HOST for a CPU function).
 * Placement is given explicitly by the caller (L110: virtualised device ids
 * make it unobservable from inside a container). */
typedef struct {
  uint32_t workflow_id;
  uint32_t function_id;
  int32_t device;
} grouter_fn;

/* One chunk of a transfer plan (L182).  path = index into the route set
 * R(dst) for host->GPU plans (0 = direct link of dst), 0 otherwise;
 * route_gpu = GPU whose link/engine moves the chunk. */
typedef struct {
  uint64_t offset;
  uint64_t bytes;
  int32_t path;
  int32_t route_gpu;
} grouter_chunk;

/* Node calibration (the topology matrix of Alg. 1) plus knobs.
 * Fill with grouter_config_default(), then override. */
typedef struct {
  uint32_t n_gpus;                                   /* logical GPUs            */
  int32_t device_map[GROUTER_MAX_GPUS];              /* logical -> CUDA ordinal */
  uint64_t nvl_Bps;                                  /* NVLink B/s per direction*/
  uint64_t h2d_Bps[GROUTER_MAX_GPUS];                /* solo pinned H2D, B/s    */
  uint64_t h2d_alpha_ps[GROUTER_MAX_GPUS];           /* per-chunk CE cost, ps   */
  uint64_t h2d_phi_ps[GROUTER_MAX_GPUS];             /* first-chunk latency, ps */
  uint64_t relay_phi_ps;                             /* extra fill of a relay   */
  uint64_t h2d_pair_Bps[GROUTER_MAX_GPUS][GROUTER_MAX_GPUS]; /* concurrent sums */
  int32_t uplink_group[GROUTER_MAX_GPUS];            /* explicit group id or -1 */
  uint8_t p2p[GROUTER_MAX_GPUS][GROUTER_MAX_GPUS];   /* peer access matrix      */
  uint64_t chunk_bytes;        /* C, default 2 MiB (L182, R1)                 */
  uint32_t batch_chunks;       /* default 5 (L229)                            */
  uint64_t granule;            /* split granule g, default 4096               */
  uint64_t pool_floor_bytes;   /* trim floor, default 300 MiB (L256, R13)     */
  uint32_t pool_cap_permille;  /* auto cap = permille of available, default 500 (L262) */
  uint64_t pool_cap_bytes[GROUTER_MAX_GPUS]; /* explicit cap; 0 = auto (O10) */
  uint64_t host_store_bytes;   /* pinned host store H, default 1 GiB          */
  uint64_t auto_cap_period_us; /* auto-mode GPUs: the background thread re-reads
                                  free memory and re-applies the cap this often
                                  (grouter_refresh_cap); default 20000; 0 = only
                                  on explicit grouter_refresh_cap calls; never
                                  in GROUTER_REPLAY mode                      */
  uint32_t copy_ctas_per_sm;   /* SM copy kernel CTAs per SM cap, default 4   */
  uint32_t flags;              /* GROUTER_* flags                              */
} grouter_config;

typedef struct {
  uint64_t used[GROUTER_MAX_GPUS];       /* sum of charges (objects + leases)   */
  uint64_t cap[GROUTER_MAX_GPUS];        /* current cap                         */
  uint64_t mapped[GROUTER_MAX_GPUS];     /* physical bytes mapped in the pool   */
  uint64_t host_used, host_cap;
  uint64_t spill_count, spill_bytes;     /* migrations to host (L258)           */
  uint64_t xfer_count;                   /* transfers planned                   */
  uint64_t link_bytes[3][GROUTER_MAX_GPUS]; /* [0]=SM copy egress, [1]=H2D, [2]=D2H */
  uint64_t kernel_launches;              /* copy/forward kernels launched       */
  uint64_t rounds;                       /* dispatch rounds                     */
  /* GROUTER_PROFILE: completed, timed copy-kernel launches (CUDA events
   * recorded on the launching stream around each launch) */
  uint64_t timed_launches;
  uint64_t timed_ns;                     /* sum of their durations              */
  uint64_t timed_bytes;                  /* sum of the bytes they moved         */
  uint64_t restore_count, restore_bytes; /* host -> home GPU restores (L260)    */
  uint64_t pool_target[GROUTER_MAX_GPUS]; /* histogram-driven pool size (R44)    */
  uint64_t tracked_functions;            /* pool-sizing histograms held (R50)   */
  uint64_t tracked_tenants;              /* per-tenant counters held (R50)      */
  uint64_t peer_launches;                /* copy-kernel launches on the peer (NVLink) branch:
                                            a destination or source outside the launching GPU,
                                            or GROUTER_FORCE_REMOTE                         */
  uint64_t timed_kernel_launches;        /* GROUTER_PROFILE: launches with kernel stamps     */
  uint64_t timed_kernel_ns;              /* their summed kernel time: latest CTA end minus
                                            earliest CTA start, %globaltimer (the kernel's
                                            own duration, host submission excluded)         */
  /* auto cap (O10, R54): the input of the last grouter_refresh_cap of each GPU
   * (explicit or by the background thread): available = free + the pool's own
   * mapped bytes; cap[] is then the O10 function of it */
  uint64_t auto_avail[GROUTER_MAX_GPUS];
  uint64_t auto_refreshes;               /* refreshes applied (all GPUs)                     */
  uint32_t auto_mode;                    /* bit d set: GPU d's cap follows free memory       */
  uint32_t pad_;
} grouter_stats_t;

/* One dispatched batch (L229: <= batch_chunks chunks of ONE tenant on ONE
 * server; a dispatch round carries one batch and each server keeps <= 2
 * rounds in flight -- SURVEY O8 -- except a direct launch, which moves the
 * whole transfer of the only tenant queued on an idle SM-copy server).  server_kind: 0 = SM copy egress of server_dev, 1 = H2D engine of
 * route GPU server_dev, 2 = D2H engine of server_dev.  Chunk ids are
 * (xfer << 32 | chunk index) where xfer numbers transfers from 1 in call order. */
typedef struct {
  int32_t server_kind;
  int32_t server_dev;
  uint32_t tenant;
  uint32_t n_chunks;
  uint64_t chunk_ids[8];
  uint64_t bytes;
  uint32_t inflight;  /* real-time mode: batches of this server dispatched earlier whose
                         completion had not been observed when this one was dispatched
                         (an upper bound; SURVEY O8 keeps it <= 1, i.e. <= 2 in flight).
                         Replay flushes dispatch everything at once: not meaningful there */
  uint32_t pad;
} grouter_dispatch;

/* ------------------------------------------------------------ lifecycle */
void grouter_config_default(grouter_config *cfg);
/* Calibration probe (the topology matrix of Alg. 1,
 * and the PCIe-switch sharing of L131/L178, measured on this box): for the
 * n_gpus CUDA ordinals in cfg->device_map, measures solo pinned H2D
 * bandwidth (h2d_Bps, from `probe_bytes` copies), per-chunk copy-engine cost
 * (h2d_alpha_ps, from back-to-back 4 KiB copies), first-chunk latency
 * (h2d_phi_ps), concurrent H2D sums for every pair (h2d_pair_Bps; uplink
 * groups are then derived by grouter_init), peer access (p2p) and a D2D
 * peer copy (nvl_Bps, if any pair has P2P).  Writes into *cfg (sets
 * uplink_group to -1 so groups come from the pair matrix).  Blocking; uses
 * the GPUs exclusively for a few seconds. */
grouter_status grouter_probe(grouter_config *cfg, uint64_t probe_bytes);
/* Creates the context: per-GPU pools (VMM reservations), host store, streams,
 * route sets R(d) (precomputed, L271).  cfg is copied. */
grouter_status grouter_init(const grouter_config *cfg, grouter_ctx **out);
/* Waits for all library work, releases every resource. */
grouter_status grouter_finalize(grouter_ctx *ctx);

/* ------------------------------------------------------------ data path */
/* Put by copy (L165).  fn->device GPU: stored on that GPU (locality, hint
 * ignored).  CPU fn: stored on `hint` GPU if given (eager striped H2D, R23),
 * else in the pinned host store.  If the home GPU cannot fit even after
 * eviction the object goes to the host store (R16).  `consumers` = k: the
 * object is freed after k completed gets (0 = explicit free only). */
grouter_status grouter_put(grouter_ctx *ctx, const grouter_fn *fn, const void *src, uint64_t n,
                           int32_t hint, uint32_t consumers, void *stream, grouter_oid *out);
/* Zero-copy put, step 1: library-owned, page-aligned buffer on fn->device
 * (or the host store for a CPU fn).  ENOMEM if it cannot fit. */
grouter_status grouter_alloc(grouter_ctx *ctx, const grouter_fn *fn, uint64_t n, int32_t hint,
                             uint32_t consumers, void **buf, grouter_oid *out);
/* Zero-copy put, step 2: the object becomes visible once prior work on
 * `stream` (which wrote the buffer) completes.  ESTATE if already sealed. */
grouter_status grouter_seal(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid, void *stream);
/* Get (L165, L167): read-only lease on fn->device.  Same location -> the
 * object's own address (zero copy, pins the object).  Otherwise a copy lease
 * (D2D over NVLink, striped H2D, or D2H for a CPU fn).  *ptr, *n out. */
grouter_status grouter_get(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid, void *stream,
                           const void **ptr, uint64_t *n);
/* Get into caller memory `dst` (device memory of fn->device, or host memory
 * for a CPU fn); always copies.  EINVAL if dst_cap < n. *n_out may be NULL.
 * A GPU -> other-GPU copy is pushed by the source GPU's SMs over NVLink
 * (in rounds of up to 7 batches when it is the only work of that copy server,
 * R55), or, <= 4 MiB on
 * an idle server with a non-NULL `stream`, pulled by the consumer GPU's SMs
 * on `stream` (R56); either way `stream` sees the bytes in order. */
grouter_status grouter_get_into(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid, void *dst,
                                uint64_t dst_cap, void *stream, uint64_t *n_out);
/* Drops a lease (ptr as returned by grouter_get).  Stream-ordered: pages are
 * reused only after prior work on `stream` completes (NULL: now). */
grouter_status grouter_release(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid,
                               const void *ptr, void *stream);
/* Frees an object (L260); later gets fail with ENOENT.  Pages are reclaimed
 * once zero-copy pins drain.  EBUSY if unsealed. */
grouter_status grouter_free(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid);

/* ------------------------------------------------------------ cross-process handoff
 * L167 (1) / L269: GROUTER maps stored data into the address space of the
 * consuming function through CUDA IPC; L394: only pre-mapped storage is
 * exposed, and access is authenticated.  An exported object lives in its own
 * CUDA VMM allocation (exactly its 2 MiB pages; R52), so an importer
 * maps that object and nothing else.  The descriptor below is plain bytes that
 * any channel can carry; it is the capability: the exporting context serves
 * the allocation's file descriptor over an abstract Unix socket only for a
 * live export whose random nonce matches, and only to a process of the same
 * uid (or root). */
#define GROUTER_IPC_MAX_SEGS 8  /* unused since descriptor version 2 */
typedef struct {
  uint32_t magic, version;        /* 0x47524f55, 2                               */
  int32_t pid;                    /* exporting process                          */
  uint32_t ctx_id;                /* exporting context (socket name)            */
  uint8_t gpu_uuid[16];           /* GPU holding the bytes                      */
  uint32_t workflow_id;           /* owner workflow: importer must match (L394) */
  int32_t logical;                /* exporter's logical GPU                     */
  grouter_oid oid;                /* exporter-side object id                    */
  uint64_t n;                     /* bytes                                      */
  uint64_t exporter_ptr;          /* object address in the exporter (release)   */
  uint64_t export_id;             /* the exporter's export record               */
  uint64_t nonce[2];              /* 128-bit random capability                  */
  uint64_t alloc_bytes;           /* size of the object's own allocation        */
} grouter_ipc_desc;

/* Exports a sealed object resident on a GPU for use by another process.
 * Blocks until the object's bytes are in place.  The first export of an
 * object moves it out of the shared pool into its own allocation (one
 * same-GPU copy); EBUSY if the object still has zero-copy leases then (their
 * pointers would dangle).  Pins the object like a zero-copy lease and
 * consumes one consumer; the exporter drops the pin with
 * grouter_release(fn, oid, (void*)desc.exporter_ptr, stream).  The export
 * ends when the object is freed: later imports fail with ENOENT, existing
 * importer mappings stay valid (the pages live until the importer unmaps). */
grouter_status grouter_export_ipc(grouter_ctx *ctx, const grouter_fn *fn, grouter_oid oid,
                                  grouter_ipc_desc *desc);
/* Imports an exported object as a local, sealed, read-only object owned by
 * fn's workflow (EPERM if desc's workflow differs).  No bytes move: gets on
 * the GPU that holds the bytes alias them (zero copy); gets on another GPU
 * copy them with the SM copy kernel on the consumer GPU reading over
 * NVLink.  Its location is GROUTER_REMOTE; grouter_free (or `consumers`)
 * unmaps it.  consumers as in grouter_put. */
grouter_status grouter_import_ipc(grouter_ctx *ctx, const grouter_fn *fn, const grouter_ipc_desc *desc,
                                  uint32_t consumers, grouter_oid *out);

/* ------------------------------------------------------------ control */
/* Tenant (workflow) bandwidth weight, >= 1 (north star; L193-L197). */
grouter_status grouter_set_tenant_weight(grouter_ctx *ctx, uint32_t workflow_id, uint32_t weight);
/* Transfer rate control (§4.3.2; R43):
 * declares workflow wf's SLO -- it must move data_bytes within
 * slo_ns - infer_ns.  Rate_least = ceil(data_bytes * 1e9 / (slo_ns - infer_ns))
 * B/s; Rate_idle = max(0, BW_all - sum Rate_least) with BW_all = sum of the
 * calibrated h2d_Bps; the tightest SLO (min slo_ns, ties -> lower id) also
 * gets Rate_idle; every SLO workflow's stride weight becomes its rate in
 * MiB/s, rounded up (>= 1).  Workflows without an SLO keep their weight.
 * data_bytes == 0 removes wf's SLO (weight back to 1); a later
 * grouter_set_tenant_weight(wf) also removes it; both re-weight the other SLO
 * workflows.  EINVAL if slo_ns <= infer_ns. */
grouter_status grouter_set_tenant_slo(grouter_ctx *ctx, uint32_t workflow_id, uint64_t data_bytes,
                                      uint64_t slo_ns, uint64_t infer_ns);
/* The same allocation as a pure function (no context, no GPU): n workflows
 * with ids[i] and SLO triples; writes weights_out[i].  EINVAL on a null
 * pointer with n > 0 or slo_ns[i] <= infer_ns[i]. */
grouter_status grouter_slo_weights(uint32_t n, const uint32_t *ids, const uint64_t *data_bytes,
                                   const uint64_t *slo_ns, const uint64_t *infer_ns, uint64_t bw_all_Bps,
                                   uint32_t *weights_out);

/* Queue position of the object's next consumer (D8; L258 queue-aware eviction).
 * CONTROL PLANE: called by the function scheduler that owns the request
 * queue, not by functions, so it takes no grouter_fn and performs no
 * workflow check (L394 authenticates the data-path calls). */
grouter_status grouter_set_next_use(grouter_ctx *ctx, grouter_oid oid, uint64_t queue_pos);
/* Pool cap of a GPU (GROUTER_UNLIMITED = no cap); evicts at once until used <= cap
 * (L262).  ENOMEM if unevictable data keeps the pool above the cap.  An
 * explicit limit takes the GPU out of auto mode (grouter_refresh_cap puts it
 * back). */
grouter_status grouter_set_pool_limit(grouter_ctx *ctx, int32_t device, uint64_t bytes);
/* Auto cap (O10; "GROUTER triggers data migration and
 * restoration automatically based on available GPU memory, maintaining storage
 * usage within a fixed threshold (50% of free memory in our experiments)";
 * readings R12, R54).  Puts GPU `device` in auto mode and applies
 *   cap = floor(avail * pool_cap_permille / 1000 / 2 MiB) * 2 MiB
 * exactly as grouter_set_pool_limit(device, cap) would: victims migrate to the
 * host in queue-aware order until used <= cap, and with GROUTER_RESTORE host
 * objects come back while they fit.  avail_bytes = memory available to the
 * store; GROUTER_AUTO_AVAIL = measure it now: cudaMemGetInfo's free bytes of
 * the GPU's device plus the bytes its pool has mapped (the pool's own memory
 * is the store's, so its growth does not shrink its cap; logical GPUs sharing
 * one device each see that device's free bytes).  Any other value is taken as
 * the measurement (a platform that accounts function memory itself, tests).
 * The background thread repeats the measured form every auto_cap_period_us
 * for every auto-mode GPU; its victims count in stats but are not listed by
 * grouter_victims.  *cap_out (nullable) = the cap applied.  EINVAL: bad
 * device; ENOMEM as grouter_set_pool_limit (the cap stays). */
#define GROUTER_AUTO_AVAIL UINT64_MAX
grouter_status grouter_refresh_cap(grouter_ctx *ctx, int32_t device, uint64_t avail_bytes, uint64_t *cap_out);
/* Replay mode: dispatch every queued chunk (stride order); no-op otherwise. */
grouter_status grouter_flush(grouter_ctx *ctx);
/* Blocks until all library work issued so far has completed. */
grouter_status grouter_sync(grouter_ctx *ctx);

/* ------------------------------------------------------------ introspection */
/* Transfer plan (L182) for n bytes of pool data from src_loc (GPU or
 * GROUTER_HOST) to dst_dev (GPU or GROUTER_HOST); GPU -> host plans are
 * striped when GROUTER_D2H_MULTIPATH is set.  *n_out = chunk count even if cap is short
 * (then EINVAL and nothing written). */
grouter_status grouter_plan(grouter_ctx *ctx, int32_t src_loc, int32_t dst_dev, uint64_t n,
                            grouter_chunk *out, uint64_t cap, uint64_t *n_out);
/* Route set R(dst) (L178, precomputed at init, L271). */
grouter_status grouter_route_set(grouter_ctx *ctx, int32_t dst_dev, int32_t *out, uint32_t cap,
                                 uint32_t *n_out);
/* Histogram-driven pool size of GPU dev at the current clock (PAPER.md
 * §4.4.1, Fig. 11a; R44): per function (workflow,
 * function id, GPU) the library samples, at every put/alloc placed in that
 * GPU's pool, the arrival time, the page charge and the function's resident
 * object count; R_window/R_size/R_con are nearest-rank p99s over the last
 * 1024 samples; target = min(cap, max(pool_floor_bytes, sum of
 * R_size * R_con over functions with now <= last arrival + R_window)).
 * The background thread pre-maps the pool up to the target (pre-warming)
 * and trims it down to max(used, target) + one 64 MiB segment. */
grouter_status grouter_pool_target(grouter_ctx *ctx, int32_t dev, uint64_t *target);
/* Current location of an object: GPU index or GROUTER_HOST.  CONTROL PLANE
 * (scheduler / introspection): no workflow check, like grouter_set_next_use. */
grouter_status grouter_where(grouter_ctx *ctx, grouter_oid oid, int32_t *loc);
grouter_status grouter_stats(grouter_ctx *ctx, grouter_stats_t *out);
/* Per-tenant share accounting (L193: "data chunks of each function are
 * scheduled proportionally to their allocated bandwidth"; L227-L229):
 * bytes[k] = bytes of workflow_id's chunks the servers of kind k dispatched
 * so far (0 = SM-copy egress, 1 = H2D engines, 2 = D2H engines), summed over
 * GPUs.  Scheduled transfers only: spills and restores are unscheduled
 * (R41, R42).  An unknown tenant reads zeros.  EINVAL on null arguments.
 * Once more than 65,536 tenants are tracked, tenants idle for over 10 s are
 * forgotten (they read zeros again). */
grouter_status grouter_tenant_stats(grouter_ctx *ctx, uint32_t workflow_id, uint64_t bytes[3]);
/* Real-time rate monitor (L197: GROUTER "monitors the transfer rate of each
 * function in real time, ensuring that it does not fall below Rate_least"):
 * *rate_Bps = bytes of workflow_id's chunks dispatched by every server in
 * the last window_ns nanoseconds (1 ms <= window_ns <= 10 s, else EINVAL),
 * times 1e9 / window_ns (integer, rounded down); *rate_least_Bps =
 * ceil(data * 1e9 / (slo - infer)) from grouter_set_tenant_slo, 0 without an
 * SLO; *backlogged = 1 if chunks of the tenant are queued and not yet
 * dispatched (a tenant below Rate_least only misses it while backlogged).
 * Dispatch times use the library clock (grouter_test_set_clock fixes it). */
grouter_status grouter_tenant_rate(grouter_ctx *ctx, uint32_t workflow_id, uint64_t window_ns, uint64_t *rate_Bps,
                                   uint64_t *rate_least_Bps, int32_t *backlogged);
/* Takes (and clears) the objects spilled since the last call, in order. */
grouter_status grouter_victims(grouter_ctx *ctx, grouter_oid *out, uint64_t cap, uint64_t *n_out);
/* Takes (and clears) the objects proactively restored to a GPU pool since the
 * last call, in order (GROUTER_RESTORE, R42).
 * Like grouter_victims the list is also reset at the start of every data-path
 * call, so it reports the restores of the latest call (the background auto-cap
 * refresh's migrations and restores are counted in grouter_stats only). */
grouter_status grouter_restored(grouter_ctx *ctx, grouter_oid *out, uint64_t cap, uint64_t *n_out);
/* Takes (and clears) up to cap dispatch records, oldest first. */
grouter_status grouter_dispatch_log(grouter_ctx *ctx, grouter_dispatch *out, uint64_t cap,
                                    uint64_t *n_out);

/* ------------------------------------------------------------ NVLink path planner
 * Contention-aware path selection, Algorithm 1 in full (§4.3.3
 * L199-L242; R11, R46).  Host-only planner state, no GPU needed.
 * The graph has n_nodes nodes: GPUs 0..n_gpus-1, then switch nodes (an
 * NVSwitch is one node every GPU links to); topo is row-major n_nodes x
 * n_nodes, topo[u*n_nodes+v] = capacity u -> v in B/s (0 = no link; the
 * diagonal is ignored).  Paths are simple, <= max_edges edges.  On an
 * NVSwitch topology every pair receives exactly its direct path. */
#define GROUTER_MAX_PATH_NODES 8
#define GROUTER_MAX_PATH_GRAPH 32
typedef struct {
  uint64_t bw_Bps;                         /* b_min(path) when it was taken  */
  uint32_t func;                           /* owning function                */
  uint32_t n_nodes;                        /* path length in nodes (edges+1) */
  int32_t nodes[GROUTER_MAX_PATH_NODES];   /* g_s, ..., g_d                  */
} grouter_path;
typedef struct grouter_paths grouter_paths;
/* NULL on bad arguments (n_nodes > GROUTER_MAX_PATH_GRAPH, max_edges + 1 >
 * GROUTER_MAX_PATH_NODES, n_gpus > n_nodes).  Caller owns; free with
 * grouter_paths_free. */
grouter_paths *grouter_paths_new(uint32_t n_nodes, uint32_t n_gpus, const uint64_t *topo, uint32_t max_edges);
void grouter_paths_free(grouter_paths *t);
/* Alg. 1 for func moving data g_s -> g_d (GPUs): may move other functions'
 * allocations (direct priority, balancing; they re-run the free phase).
 * Writes func's paths (allocation order) to out[0..cap); *n_out = count
 * (EINVAL if > cap).  ESTATE if func already holds paths (release first). */
grouter_status grouter_paths_select(grouter_paths *t, uint32_t func, int32_t gs, int32_t gd, grouter_path *out,
                                    uint32_t cap, uint32_t *n_out);
/* The function finished: its bandwidth returns to BW. */
grouter_status grouter_paths_release(grouter_paths *t, uint32_t func);
/* Every active allocation in allocation order (EINVAL if cap is short). */
grouter_status grouter_paths_table(grouter_paths *t, grouter_path *out, uint32_t cap, uint32_t *n_out);
/* Chunk plan of n bytes over func's current paths (L182, L242, O6 split):
 * path p -> grouter_chunk.path = p (allocation order), beta = its bw, alpha 0,
 * phi = (GPU relays on p) * relay_phi_ps; route_gpu = first relay GPU (the
 * source for a direct or switch-only path). */
grouter_status grouter_paths_plan(grouter_paths *t, uint32_t func, uint64_t n, uint64_t chunk_bytes,
                                  uint64_t granule, uint64_t relay_phi_ps, grouter_chunk *out, uint64_t cap,
                                  uint64_t *n_out);

/* ------------------------------------------------------------ stride scheduler
 * The tenant-share scheduler used by every server (L229 batches, stride
 * order), exposed standalone for host-side tests; needs no GPU. */
typedef struct grouter_sched grouter_sched;
grouter_status grouter_sched_new(uint32_t batch_chunks, grouter_sched **out);
grouter_status grouter_sched_set_weight(grouter_sched *s, uint32_t tenant, uint32_t weight);
grouter_status grouter_sched_enqueue(grouter_sched *s, uint32_t tenant, uint64_t chunk_id,
                                     uint64_t bytes);
/* Next batch: *tenant, up to 8 ids, *n, *bytes, tenant's pass after it.
 * ENOENT when nothing is backlogged. */
grouter_status grouter_sched_dispatch(grouter_sched *s, uint32_t *tenant, uint64_t *ids,
                                      uint32_t *n, uint64_t *bytes, uint64_t *pass_after);
/* The pass / virtual-time updates the dispatch of `tenant`'s n bytes (in
 * chunks of `chunk` bytes, the last one partial) would make if the tenant
 * were alone on the server -- what the library applies when a transfer
 * bypasses the queues of an idle server (direct launches, idle copy
 * engines), so later contention sees the same state.  The tenant must have
 * nothing queued.  EINVAL on a null scheduler or chunk == 0. */
grouter_status grouter_sched_account_solo(grouter_sched *s, uint32_t tenant, uint64_t n, uint64_t chunk);
void grouter_sched_free(grouter_sched *s);

const char *grouter_strerror(grouter_status st);
/* Text of the last error seen by this thread (thread-local). */
const char *grouter_last_error(void);
/* SHA-256 (hex) of the sources this library was built from (static string);
 * the Python binding refuses a library whose hash differs from the tree. */
const char *grouter_build_hash(void);

#ifdef __cplusplus
}
#endif
#endif /* GROUTER_H */
