"""Turns an `ncu --page raw --csv` export and an ncu launch list into the
committed profile summaries (profiles/<round>_ncu_full_gr_copy.json,
ncu_traffic.json, <round>_ncu_launches_summary.csv).

usage: python tools/ncu_extract.py RAW_CSV LAUNCHES_CSV ROUND
"""
import collections
import csv
import json
import sys

KEYS = ["Kernel Name", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__cycles_active.avg", "sm__cycles_active.min", "sm__cycles_active.max",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio",
        "smsp__average_warp_latency_issue_stalled_barrier.ratio",
        "smsp__average_warp_latency_issue_stalled_membar.ratio",
        "smsp__average_warp_latency_issue_stalled_lg_throttle.ratio",
        "lts__t_sectors_srcunit_ltcfabric.sum", "smsp__inst_executed.sum"]


def scale(v, unit):
    f = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit)
    return float(v.replace(",", "")) * f if f else None


def main(raw, launches, rnd):
    rows = list(csv.reader(open(raw)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    head, units = rows[hi], rows[hi + 1]
    out = []
    for r in rows[hi + 2:]:
        if len(r) != len(head):
            continue
        out.append({k: [r[head.index(k)] if k in head else None, units[head.index(k)] if k in head else ""]
                    for k in KEYS})
    json.dump(out, open(f"profiles/{rnd}_ncu_full_gr_copy.json", "w"), indent=1)
    rd = [scale(*x["dram__bytes_read.sum"]) for x in out]
    wr = [scale(*x["dram__bytes_write.sum"]) for x in out]
    tr = {"kernel": out[0]["Kernel Name"][0], "dram_bytes_per_launch": (sum(rd) + sum(wr)) / len(out),
          "dram_read": sum(rd) / len(out), "dram_write": sum(wr) / len(out),
          "note": "ncu --set full, cache flushed per replay: writes of a 38.5 MB copy stay in the 126 MB "
                  "L2 and are written back after the kernel, so traffic per launch ~= the read half of "
                  "the algorithmic 2 x 38.5 MB",
          "source": f"profiles/{rnd}_ncu_full_gr_copy.json"}
    json.dump(tr, open("profiles/ncu_traffic.json", "w"), indent=1)
    rows = list(csv.reader(open(launches)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = collections.defaultdict(list)
    for r in rows[hi + 1:]:
        if len(r) > vi and r[vi]:
            try:
                agg[r[ki]].append(float(r[vi].replace(",", "")) / 1e3)
            except ValueError:
                pass
    tot = sum(sum(v) for v in agg.values())
    with open(f"profiles/{rnd}_ncu_launches_summary.csv", "w") as f:
        w = csv.writer(f)
        w.writerow(["kernel", "launches", "avg_us", "total_us", "share"])
        for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
            w.writerow([k, len(v), round(sum(v) / len(v), 3), round(sum(v), 1), round(sum(v) / tot, 3)])
    print(json.dumps(tr))


if __name__ == "__main__":
    main(*sys.argv[1:4])
