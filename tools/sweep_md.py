"""Renders a tests/harness/sweep.py JSON document as the profiles/<round>_sweep.md table.
usage: python tools/sweep_md.py SWEEP_JSON > profiles/rNN_sweep.md"""
import json
import sys

d = json.load(open(sys.argv[1]))
P = d["patterns"]


def row(name, n):
    for r in P.get(name, []):
        if r["n"] == n:
            return r
    return None


def cell(name, n, gbps=True, p99=False):
    r = row(name, n)
    if r is None:
        return "—"
    s = f"{r['p50_us']}" + (f"/{r['p99_us']}" if p99 else "")
    return s + (f" ({r['GBps']})" if gbps else "")


print(f"# cfg3 sweep ({d['gpu']}, host cores {d['host_cores']})\n")
print("`python tests/harness/sweep.py` (device-event timing for get_into / baselines on the consumer stream; host clock "
      "for blocking cFn calls and the zero-copy get+release pair). Latency mode: one call at a time on an idle "
      "GPU, so every number includes the library's host path. GB/s = payload bytes / p50. Probe of this GPU: "
      f"{json.dumps(d['probe'])}\n")
print("| bytes | get_into same-GPU p50/p99 µs (GB/s) | cudaMemcpy D2D p50 µs | zero-copy get µs | put H2D (hint GPU0) "
      "p50 µs (GB/s) | pinned H2D p50 µs | get D2H p50 µs (GB/s) | pinned D2H p50 µs | oracle get_into µs | "
      "oracle put H2D µs (1 thread / striped, threads) |")
print("|---|---|---|---|---|---|---|---|---|---|")
for r in P["get_into_same"]:
    n = r["n"]
    print(f"| {n:,} | {cell('get_into_same', n, True, True)} | {cell('base_memcpy_d2d', n, False)} | "
          f"{cell('zero_copy_get', n, False)} | {cell('put_h2d', n)} | {cell('base_h2d_pinned', n, False)} | "
          f"{cell('get_d2h', n)} | {cell('base_d2h_pinned', n, False)} | {cell('oracle_get_into', n, False)} | "
          f"{cell('oracle_put_h2d', n, False)} / {cell('oracle_put_striped', n, False)}"
          f"{', T=' + str(row('oracle_put_striped', n)['threads']) if row('oracle_put_striped', n) else ''} |")
