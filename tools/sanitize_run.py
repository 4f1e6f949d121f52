#!/usr/bin/env python
"""Small run of every kernel (all blind-rotation variants, latency mode, key switch, a mixed netlist) for
compute-sanitizer:  compute-sanitizer --tool {memcheck,racecheck,synccheck} python tools/sanitize_run.py"""
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
for variant in (6, 7, 8):
    ctx.set_br_variant(variant)
    ctx.set_narrow_lanes(0)
    outs.append(ctx.bootstrap_wo_ks(ct))
ctx.set_br_variant(6)
ctx.set_narrow_lanes(148)
outs.append(ctx.bootstrap_wo_ks(ct))                        # latency mode (br7<1>)
ks = ctx.keyswitch(outs[0])
n = synth.ripple_carry_adder(2)
net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"])
d = ctx.upload(net)
w = ctx.wire_array(d)
w[:n["n_inputs"]].random_(-2 ** 31, 2 ** 31 - 1, generator=g)
ctx.run_netlist(d, w)
torch.cuda.synchronize()
same = all(torch.equal(outs[0][:, :1025], o[:, :1025]) for o in outs[1:])
print("variants agree:", same)
sys.exit(0 if same else 1)
