"""Steady-state DRAM traffic of the leg-B copy kernel (bench.py `roofline.traffic_steady`).

Reads the `ncu --cache-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,
gpu__time_duration.sum -k regex:gr_copy` CSV of tools/round_run.sh, averages the per-launch
bytes, writes profiles/<round>_ncu_steady_traffic.json and merges the figure into
profiles/ncu_traffic.json (which bench.py reads).
Usage: python tools/ncu_steady.py gpurun_out/final/steady.csv r02
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ALG = 2 * 38535168


def main(path, rnd):
    rows = [ln for ln in open(path) if ln.startswith('"')]
    per = {}
    for r in csv.DictReader(rows):
        if "gr_copy" not in r["Kernel Name"]:
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r["Metric Unit"]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "ns": 1, "usecond": 1e3, "us": 1e3,
                 "msecond": 1e6}[unit]
        per.setdefault(r["ID"], {})[r["Metric Name"]] = v * scale
    n = len(per)
    rd = sum(p["dram__bytes_read.sum"] for p in per.values()) / n
    wr = sum(p["dram__bytes_write.sum"] for p in per.values()) / n
    us = sum(p["gpu__time_duration.sum"] for p in per.values()) / n / 1e3
    out = {"launches": n, "dram_read_per_launch": rd, "dram_write_per_launch": wr,
           "steady_dram_bytes_per_launch": rd + wr, "alg_bytes_per_launch": ALG,
           "ratio_to_alg": (rd + wr) / ALG, "avg_duration_us": us,
           "how": "ncu --cache-control none --clock-control none, consecutive gr_copy launches of leg B back to "
                  "back (bench.py --b2b region), per-launch dram bytes; durations are serialised by ncu"}
    dst = os.path.join(ROOT, "profiles", f"{rnd}_ncu_steady_traffic.json")
    json.dump(out, open(dst, "w"), indent=1)
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    tj = json.load(open(tp)) if os.path.exists(tp) else {}
    tj["steady_dram_bytes_per_launch"] = rd + wr
    tj["steady_source"] = f"profiles/{rnd}_ncu_steady_traffic.json ({n} back-to-back leg-B launches, " \
                          "--cache-control none)"
    json.dump(tj, open(tp, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
