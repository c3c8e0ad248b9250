/* A plain C99 consumer of include/grouter.h (tests/test_c_abi.py compiles it
 * with gcc -std=c99 -Wall -Wextra -Werror and runs it on a machine without a
 * GPU): the header is valid C, the library links from C, a planner-only
 * context plans host->GPU transfers, and a data-path context fails loudly
 * with GROUTER_ECUDA instead of falling back to the CPU. */
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#include "grouter.h"
#include "grouter_testing.h"

int main(void) {
  grouter_config cfg;
  grouter_config_default(&cfg);
  cfg.n_gpus = 8;
  for (int i = 0; i < 8; ++i) {
    cfg.device_map[i] = i;
    cfg.uplink_group[i] = i / 2;
  }
  cfg.flags = GROUTER_PLAN_ONLY;
  grouter_ctx *ctx = NULL;
  if (grouter_init(&cfg, &ctx) != GROUTER_OK) {
    printf("plan-only init failed: %s\n", grouter_last_error());
    return 1;
  }
  grouter_chunk chunks[64];
  uint64_t k = 0;
  const uint64_t n = 38535168u;
  if (grouter_plan(ctx, GROUTER_HOST, 0, n, chunks, 64, &k) != GROUTER_OK || k == 0 || k > 64) return 2;
  uint64_t covered = 0;
  int routes = 0;
  for (uint64_t i = 0; i < k; ++i) {
    covered += chunks[i].bytes;
    routes |= 1 << chunks[i].route_gpu;
  }
  if (covered != n) return 3;
  /* a data-path call on a planner-only context is rejected, not emulated */
  grouter_fn fn = {1, 1, GROUTER_HOST};
  grouter_oid oid = 0;
  if (grouter_put(ctx, &fn, chunks, 16, 0, 0, NULL, &oid) == GROUTER_OK) return 4;
  grouter_finalize(ctx);
  /* a data-path context without a GPU fails loudly */
  grouter_config dcfg;
  grouter_config_default(&dcfg);
  dcfg.n_gpus = 1;
  grouter_ctx *dctx = NULL;
  grouter_status st = grouter_init(&dcfg, &dctx);
  printf("plan %llu chunks over route mask 0x%x; data-path init: %s (%s)\n", (unsigned long long)k, routes,
         grouter_strerror(st), st == GROUTER_OK ? "" : grouter_last_error());
  if (st == GROUTER_OK) grouter_finalize(dctx);
  return 0;
}
