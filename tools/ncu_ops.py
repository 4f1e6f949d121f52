#!/usr/bin/env python
"""Executed warp instructions of one profiled kernel per SASS opcode and per CUDA source line range
(from the ncu source page; same line table as ncu_lines.py):

    python tools/ncu_ops.py report.ncu-rep kernel_substring [range_spec ...]

range_spec = name:file:first-last (e.g. fwd:tb_br6t.cu:131-215); instructions inlined from other files are
attributed to the outermost frame that lies in a named file range, else to 'other'."""
import csv, io, os, re, subprocess, sys, tempfile
from collections import defaultdict

rep, ksub = sys.argv[1], sys.argv[2]
ranges = []
for spec in sys.argv[3:]:
    name, f, rg = spec.split(":")
    a, b = rg.split("-")
    ranges.append((name, f, int(a), int(b)))
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
so = os.path.join(ROOT, "paper_conf_ispass_maxw23_b200", "libtfhe_b200.so")
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", so], cwd=tmp, capture_output=True)
cubin = [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")][0]
dis = subprocess.run(["nvdisasm", "-gi", "-c", cubin], capture_output=True, text=True).stdout
reg_of, cur_fn, frames, fresh = {}, None, [], True
for ln in dis.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", ln)
    if m:
        cur_fn = m.group(1)
        continue
    if "//## File" in ln:
        if not fresh:
            continue
        fresh = False
        frames = [(os.path.basename(f), int(n)) for f, n in re.findall(r'"([^"]+)", line (\d+)', ln)]
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m:
        fresh = True
        if cur_fn and ksub in cur_fn:
            reg = "other"
            for fr in reversed(frames):           # outermost frame first (the kernel's own line)
                hit = [r[0] for r in ranges if r[1] == fr[0] and r[2] <= fr[1] <= r[3]]
                if hit:
                    reg = hit[0]
                    break
            reg_of[int(m.group(1), 16)] = reg
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr = rows[1]
ia, ii, isrc = hdr.index("Address"), hdr.index("Instructions Executed"), hdr.index("Source")
ops = defaultdict(lambda: defaultdict(float))
base = None
for r in rows[2:]:
    try:
        addr = int(r[ia], 16)
    except (ValueError, IndexError):
        continue
    base = addr if base is None else base
    reg = reg_of.get(addr - base, "other")
    op = r[isrc].strip().split()
    op = [t for t in op if not t.startswith("@")]
    name = op[0].split(".")[0] if op else "?"
    if op and op[0].startswith("IMAD"):
        name = op[0]
    ops[reg][name] += float(r[ii] or 0)
tot = sum(sum(d.values()) for d in ops.values())
for reg, d in sorted(ops.items(), key=lambda t: -sum(t[1].values())):
    s = sum(d.values())
    top = ", ".join("%s %.1f%%" % (k, 100 * v / tot) for k, v in sorted(d.items(), key=lambda t: -t[1])[:9])
    print("%-8s %5.1f%% | %s" % (reg, 100 * s / tot, top))
