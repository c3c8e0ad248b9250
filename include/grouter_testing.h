/*
 * grouter_testing.h -- test-infrastructure kernels.
 *
 * Not part of the data path.  These implement, on the device, the
 * SplitMix64 counter-mode payload generator of SURVEY §8(c) O11 (the same
 * input recipe synth/payload.py implements on the host) so large payloads
 * can be produced and verified in HBM, plus an exactly-once probe that runs
 * the PRODUCTION copy kernel over a chunk list while counting every 16-byte
 * destination granule it writes.
 *
 * All functions take device pointers (or host-mapped pinned pointers), are
 * stream-ordered on `stream` (a cudaStream_t as void*), and return
 * grouter_status (ECUDA on CUDA failure, EINVAL on bad arguments).
 */
#ifndef GROUTER_TESTING_H
#define GROUTER_TESTING_H

#include "grouter.h"

#ifdef __cplusplus
extern "C" {
#endif

/* dst[i] = byte (offset + i) of stream `seed`, i in [0, n). */
grouter_status grouter_test_fill(void *dst, uint64_t n, uint64_t seed, uint64_t offset,
                                 void *stream);
/* Counts bytes of src[0, n) that differ from stream `seed` at `offset`.
 * Blocking: synchronizes `stream`; *mismatches and *first_bad (UINT64_MAX if
 * none) are host outputs. */
grouter_status grouter_test_verify(const void *src, uint64_t n, uint64_t seed, uint64_t offset,
                                   void *stream, uint64_t *mismatches, uint64_t *first_bad);
/* Runs the production SM copy kernel over `n_chunks` chunks
 * (dst_base + chunk.offset <- src_base + chunk.offset, chunk.bytes) on the
 * current device.  If counts != NULL (device array of ceil((max_end)/16)
 * uint32), every 16-byte destination granule touched is counted (exactly-once
 * probe, invariant I1).  tma != 0 selects the cp.async.bulk variant. */
grouter_status grouter_test_copy(void *dst_base, const void *src_base, const grouter_chunk *chunks,
                                 uint32_t n_chunks, uint32_t *counts, int tma, void *stream);

/* Host cost of kernel launches from this library (tuning probe): kind 0 =
 * empty kernel with an int parameter, 1 = small copy-parameter block, 2 =
 * large copy-parameter block; n launches of `blocks` x 256 on `stream`;
 * *us_per_launch = host time per launch call. */
grouter_status grouter_test_launch_cost(int kind, int n, int blocks, void *stream, double *us_per_launch);

/* Measured BASELINE, not the data path: one bare cudaMemcpyAsync(dst, src, n,
 * cudaMemcpyDefault) on `stream` (a cudaStream_t as void*; NULL = a
 * library-internal non-blocking stream of the current device).  wait != 0:
 * the call returns once the copy has completed (an event recorded after it,
 * polled like the library's blocking callers poll theirs); wait == 0: it
 * returns after the enqueue.  The bench times it through the same binding as
 * the library calls it is compared with (SURVEY §8(d) baselines). */
grouter_status grouter_test_memcpy(void *dst, const void *src, uint64_t n, void *stream, int32_t wait);

/* Positive control for the race detector (sanitizer builds):
 * two threads increment one plain int `iters` times each, unsynchronised --
 * a ThreadSanitizer build must report exactly this data race.  Returns the
 * final count in *out (any value; the race is the point). */
grouter_status grouter_test_race(int32_t iters, int64_t *out);
/* Positive control for AddressSanitizer builds: a deliberate one-past-the-end
 * heap read (the sanitizer must report it; a product build just returns). */
grouter_status grouter_test_oob(int32_t *out);

/* Text dump of the context's internal state (servers, objects, leases,
 * pending completion words) for debugging; truncated to cap bytes.  Returns
 * the full length needed in *len (may be NULL). */
grouter_status grouter_test_dump(grouter_ctx *ctx, char *buf, uint64_t cap, uint64_t *len);

/* Fault injection (tests only): what = 1 -- the next `count` dispatch rounds
 * fail as a CUDA error would (the context turns sticky-ECUDA; callers blocked
 * waiting for a submission wake up and fail instead of hanging). */
grouter_status grouter_test_inject(grouter_ctx *ctx, int32_t what, int32_t count);

/* Fixes the clock the pool-sizing samples and targets use (fixed != 0) to
 * t_ns, or returns to the monotonic clock (fixed == 0).  For deterministic
 * parity traces (R44). */
grouter_status grouter_test_set_clock(grouter_ctx *ctx, int32_t fixed, uint64_t t_ns);

#ifdef __cplusplus
}
#endif
#endif /* GROUTER_TESTING_H */
