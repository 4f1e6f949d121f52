#!/usr/bin/env python
"""Key metrics and a barrier-delimited phase split (warp samples per SASS range of the main loop) from an
ncu --set full report:  python tools/ncu_summary.py report.ncu-rep [kernel-regex]"""
import csv
import io
import re
import subprocess
import sys

rep = sys.argv[1]
METRICS = [("duration (ms)", "gpu__time_duration.sum"), ("SM cycles", "sm__cycles_elapsed.avg"),
           ("warp instructions", "smsp__inst_executed.sum"),
           ("issue active % (per active SMSP)", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
           ("FMA-heavy pipe % (elapsed)", "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed"),
           ("FP64 pipe % (elapsed)", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_elapsed"),
           ("ALU pipe % (active)", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"),
           ("shared wavefronts", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
           ("DRAM read (bytes as printed)", "dram__bytes_read.sum"), ("registers", "launch__registers_per_thread"),
           ("grid", "launch__grid_size"), ("block", "launch__block_size")]


def run(*args):
    return subprocess.run(["ncu", "-i", rep] + list(args), capture_output=True, text=True).stdout


rows = list(csv.reader(io.StringIO(run("--page", "raw", "--csv"))))
h, v = rows[0], rows[2]
print("| metric | value |\n|---|---|")
for label, name in METRICS:
    if name in h:
        print("| %s (`%s`) | %s |" % (label, name, v[h.index(name)]))
src = [r for r in csv.reader(io.StringIO(run("--page", "source", "--csv")))]
hdr = src[1]
ia, isrc, iss = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
stall = [i for i, n in enumerate(hdr) if n.startswith("stall_")]
segs, cur, tot = [], {"s": 0.0, "st": {}}, 0.0
for r in src[2:]:
    try:
        x = float(r[iss] or 0)
    except (ValueError, IndexError):
        continue
    cur["s"] += x
    tot += x
    for i in stall:
        try:
            cur["st"][hdr[i]] = cur["st"].get(hdr[i], 0.0) + float(r[i] or 0)
        except ValueError:
            pass
    if re.search(r"BAR\.SYNC|EXIT|SYNCS|try_wait|BAR\.RED", r[isrc]):
        cur["end"] = r[isrc].strip()[:48]
        segs.append(cur)
        cur = {"s": 0.0, "st": {}}
print("\n| SASS range ending at | share of warp samples | top stalls |\n|---|---|---|")
for sg in segs:
    if sg["s"] < 0.01 * tot:
        continue
    top = sorted(sg["st"].items(), key=lambda t: -t[1])[:3]
    print("| `%s` | %.1f %% | %s |" % (sg.get("end", ""), 100 * sg["s"] / tot,
                                     ", ".join("%s %.0f %%" % (k[6:], 100 * val / sg["s"]) for k, val in top)))
