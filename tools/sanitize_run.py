#!/usr/bin/env python
"""Small run of every kernel (all blind-rotation variants incl. the tensor-core brt, every latency-mode kernel,
tiled and split key switch at 3 / 7 / 37 gates, a mixed netlist through the device and the overlapped host path,
and the fused-exchange peer stores into a second array) for compute-sanitizer:
    compute-sanitizer --tool {memcheck,racecheck,synccheck} python tools/sanitize_run.py
TB_SAN_BRT=1: only the tensor-core kernels brt / br6t / brq / brtl (racecheck on their shared-memory hand-offs).
TB_SAN_NOBRT=1: everything but the tensor-core kernels (synccheck does not model tcgen05.commit arrivals)."""
import ctypes
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ispass_maxw23_b200 as tb  # noqa: E402
import synth  # noqa: E402

ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 1), synth.random_words(tb.KSK_WORDS, 2))
g = torch.Generator(device="cuda")
g.manual_seed(3)
ct = ctx.empty(5)
ct.random_(-2 ** 31, 2 ** 31 - 1, generator=g)
outs = []
QUICK = os.environ.get("TB_SAN_QUICK") == "1"                # racecheck: key switch, netlist and peer stores only
LAT = os.environ.get("TB_SAN_LATENCY") == "1"                # racecheck: the latency kernels on one lane only
BRT = os.environ.get("TB_SAN_BRT") == "1"                    # racecheck: the tensor-core kernel only
if BRT:
    ctx.set_narrow_lanes(0)
    ctx.set_br_variant(6)
    a = ctx.bootstrap_wo_ks(ct)
    bs = []
    for v in (12, 14, 15):
        ctx.set_br_variant(v)
        bs.append(ctx.bootstrap_wo_ks(ct))
    ctx.set_br_variant(6)
    ctx.set_narrow_lanes(148)
    ctx.set_narrow_kernel(13)
    bs.append(ctx.bootstrap_wo_ks(ct))
    torch.cuda.synchronize()
    ok = all(torch.equal(a[:, :1025], b[:, :1025]) for b in bs)
    print("brt / br6t / brq / brtl agree with br6:", ok)
    sys.exit(0 if ok else 1)
if LAT:
    one = ct[:1]
    res = []
    for k in (11, 9, 16):
        ctx.set_narrow_kernel(k)
        res.append(ctx.bootstrap_wo_ks(one))
    torch.cuda.synchronize()
    ok = all(torch.equal(res[0][:, :1025], r[:, :1025]) for r in res[1:])
    print("latency kernels agree:", ok)
    sys.exit(0 if ok else 1)
NOBRT = os.environ.get("TB_SAN_NOBRT") == "1"                # synccheck: the tool does not model tcgen05.commit
for variant in ((6,) if QUICK else ((6, 10) if NOBRT else (6, 10, 12, 14, 15))):
    ctx.set_br_variant(variant)
    ctx.set_narrow_lanes(0)
    outs.append(ctx.bootstrap_wo_ks(ct))
ctx.set_br_variant(6)
ctx.set_narrow_lanes(148)
for k in (() if QUICK else ((11, 9, 16) if NOBRT else (11, 9, 13, 16))):   # latency: brl, br9, brtl, brl2
    ctx.set_narrow_kernel(k)
    outs.append(ctx.bootstrap_wo_ks(ct))
ctx.set_narrow_kernel(0)
ext = ctx.empty(37, stride=1028)
ext.random_(-2 ** 31, 2 ** 31 - 1, generator=g)
ks = [ctx.keyswitch(ext[:c]) for c in (3, 7, 37)]           # split KS: 64 / 32 / 16 slices per gate
ctx.set_narrow_lanes(0)
ks.append(ctx.keyswitch(ext))                               # tiled KS
ctx.set_narrow_lanes(148)
n = synth.ripple_carry_adder(2)
net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"])
d = ctx.upload(net)
w = ctx.wire_array(d)
w[:n["n_inputs"]].random_(-2 ** 31, 2 ** 31 - 1, generator=g)
ctx.run_netlist(d, w)
hin = w[:n["n_inputs"], :631].cpu().contiguous()
hout = ctx.run_netlist_host(d, hin.numpy().view("uint32"), [d.n_rows - 1, 0])   # overlapped host path
mirror = ctx.wire_array(d)                                  # fused exchange: peer stores into a second array
arr = (ctypes.c_void_p * 1)(mirror.data_ptr())
tb._native.check(tb._native.lib().tb_set_peer_wires(ctx._h, ctypes.c_void_p(w.data_ptr()), arr, 1))
ctx.run_netlist(d, w)
tb._native.check(tb._native.lib().tb_set_peer_wires(ctx._h, None, None, 0))
torch.cuda.synchronize()
same_rows = torch.equal(mirror[n["n_inputs"]:d.n_rows, :631], w[n["n_inputs"]:d.n_rows, :631])
print("peer mirror equal:", same_rows)
same = all(torch.equal(outs[0][:, :1025], o[:, :1025]) for o in outs[1:])
print("variants agree:", same)
sys.exit(0 if same and same_rows else 1)
