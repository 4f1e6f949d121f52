#!/usr/bin/env python
"""Warp-stall samples and executed instructions of one kernel per CUDA source line, from an ncu --set full
report (SASS page) and the line table of the built library (nvdisasm -gi of its sm_100a cubin):

    python tools/ncu_lines.py report.ncu-rep kernel_symbol_substring [file_substring] [top]

The library must be the one the report was taken with (build, run, then read)."""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile
from collections import defaultdict

rep, ksub = sys.argv[1], sys.argv[2]
fsub = sys.argv[3] if len(sys.argv) > 3 else ""
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
so = os.path.join(ROOT, "paper_conf_ispass_maxw23_b200", "libtfhe_b200.so")

tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", so], cwd=tmp, capture_output=True)
cubin = [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")][0]
dis = subprocess.run(["nvdisasm", "-gi", "-c", cubin], capture_output=True, text=True).stdout
# address -> (file, line) inside the kernel's function
line_of, cur_fn, loc, fresh = {}, None, None, True
for ln in dis.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", ln)
    if m:
        cur_fn = m.group(1)
        continue
    if "//## File" in ln:
        if not fresh:             # -gi prints the inlined frame first, then the bare outer line: keep the first
            continue
        fresh = False
        # innermost first: File "a", line x inlined at "b", line y ...; keep the first frame in the wanted file
        frames = [(os.path.basename(f), int(n)) for f, n in re.findall(r'"([^"]+)", line (\d+)', ln)]
        pick = [fr for fr in frames if fsub and fsub in fr[0]]
        loc = pick[0] if pick else frames[0]
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m:
        fresh = True
        if cur_fn and ksub in cur_fn:
            line_of[int(m.group(1), 16)] = loc

txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr = rows[1]
ia, iw, ii = hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
stall = [i for i, n in enumerate(hdr) if n.startswith("stall_") and "Not Issued" not in n]
agg = defaultdict(lambda: {"s": 0.0, "i": 0.0, "st": defaultdict(float)})
tot_s = tot_i = 0.0
base = None
for r in rows[2:]:
    try:
        addr = int(r[ia], 16)
    except (ValueError, IndexError):
        continue
    base = addr if base is None else base
    off = addr - base
    s, i = float(r[iw] or 0), float(r[ii] or 0)
    key = line_of.get(off) or ("?", 0)
    if fsub and fsub not in key[0]:
        key = ("other", 0)
    a = agg[key]
    a["s"] += s
    a["i"] += i
    tot_s += s
    tot_i += i
    for k in stall:
        try:
            a["st"][hdr[k][6:]] += float(r[k] or 0)
        except ValueError:
            pass
print("| file:line | warp samples | instructions | top stalls |\n|---|---|---|---|")
for key, a in sorted(agg.items(), key=lambda t: -t[1]["s"])[:top]:
    st = sorted(a["st"].items(), key=lambda t: -t[1])[:3]
    print("| %s:%d | %.1f %% | %.1f %% | %s |" % (key[0], key[1], 100 * a["s"] / tot_s, 100 * a["i"] / max(tot_i, 1),
                                               ", ".join("%s %.0f%%" % (k, 100 * v / max(a["s"], 1)) for k, v in st)))
