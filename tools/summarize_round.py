#!/usr/bin/env python
"""Turn a tools/measure_round.sh batch (gpurun_out/<TAG>_*) into the tracked summaries under profiles/:
<TAG>_bench.json, <TAG>_bench_reference.json, <TAG>_workloads.jsonl, <TAG>_launches.csv, <TAG>_launch_summary.md,
<TAG>_br6_bench_dram.csv and ncu_br_kernel_summary.json (the `traffic` bench.py reports).

  python tools/summarize_round.py TAG
"""
import collections
import csv
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
src, dst = os.path.join(ROOT, "gpurun_out"), os.path.join(ROOT, "profiles")


def rows(path):
    lines = [l for l in open(path) if l.startswith('"')]
    return list(csv.DictReader(lines))


for a, b in (("bench.json", "bench.json"), ("ref.json", "bench_reference.json"), ("workloads.jsonl", "workloads.jsonl"),
             ("launches.csv", "launches.csv"), ("br6_dram.csv", "br6_bench_dram.csv")):
    shutil.copy(os.path.join(src, "%s_%s" % (tag, a)), os.path.join(dst, "%s_%s" % (tag, b)))

bench = json.loads(open(os.path.join(src, tag + "_bench.json")).read())
d = {r["Metric Name"]: float(r["Metric Value"].replace(",", "")) for r in rows(os.path.join(src, tag + "_br6_dram.csv"))}
r0 = rows(os.path.join(src, tag + "_br6_dram.csv"))[0]
lanes = bench["config"]["gates_per_gpu"]
summary = {
    "kernel": "br6_kernel<2>",
    "command": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum "
               "--clock-control none -k regex:br6_kernel -s 3 -c 1 python bench.py --steps 1 --no-cpu-baseline --no-e2e",
    "lanes": lanes, "lanes_per_cta": bench["config"]["lanes_per_cta"], "br_variant": bench["config"]["br_variant"],
    "grid": r0["Grid Size"], "block": r0["Block Size"],
    "dram_bytes_read": d["dram__bytes_read.sum"], "dram_bytes_write": d["dram__bytes_write.sum"],
    "dram_bytes_per_launch": d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"],
    "lts_bytes_per_launch": d["lts__t_bytes.sum"], "gpu_time_ns_cold_serialised": d["gpu__time_duration.sum"],
    "note": "DRAM traffic %.0f GB/s over the launch (BK re-read from HBM about twice per wave of 592 lanes); L2 "
            "traffic %.2f TB/s.  Neither is near its roof: the kernel is bound by the integer-multiply pipe "
            "(DESIGN.md 7.1)." % ((d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"]) / d["gpu__time_duration.sum"],
                                  d["lts__t_bytes.sum"] / d["gpu__time_duration.sum"] / 1e3),
    "source_csv": "profiles/%s_br6_bench_dram.csv" % tag,
}
json.dump(summary, open(os.path.join(dst, "ncu_br_kernel_summary.json"), "w"), indent=2)

agg = collections.OrderedDict()
for r in rows(os.path.join(src, tag + "_launches.csv")):
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    k = (r["Kernel Name"][:110], r["Grid Size"])
    t = float(r["Metric Value"].replace(",", "")) / 1e6
    n, s = agg.get(k, (0, 0.0))
    agg[k] = (n + 1, s + t)
out = ["# %s launch list: `ncu --metrics gpu__time_duration.sum --clock-control none python bench.py "
       "--no-cpu-baseline --steps 2 --warmup 3`" % tag, "",
       "Cold-cache, serialised per-launch device times (compare shares, not absolutes). Full CSV: %s_launches.csv" % tag,
       "", "| kernel | grid | launches | ms/launch (mean) | total ms |", "|---|---|---|---|---|"]
br = ks = 0.0
for (name, grid), (n, s) in agg.items():
    out.append("| %s | %s | %d | %.3f | %.1f |" % (name, grid, n, s / n, s))
    if "br6_kernel" in name and grid.startswith("(32768"):
        br += s
    if "ks_kernel" in name and grid.startswith("(8192"):
        ks += s
out += ["", "Bench-level launches (%d lanes): blind rotation %.1f ms, key switch %.1f ms -> BR share %.1f %% (live "
        "CUDA-event share in the bench line: %.1f %%)." % (lanes, br, ks, 100 * br / (br + ks),
                                                           100 * bench["roofline"]["kernel_share_of_step"])]
open(os.path.join(dst, tag + "_launch_summary.md"), "w").write("\n".join(out) + "\n")
print("\n".join(out))
