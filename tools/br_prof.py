"""one throughput launch of the selected blind-rotation variant (for ncu): python tools/br_prof.py VARIANT LANES"""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ispass_maxw23_b200 as tb, synth
variant, lanes = int(sys.argv[1]), int(sys.argv[2])
ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 11), synth.random_words(tb.KSK_WORDS, 12))
ctx.set_br_variant(variant)
ctx.set_narrow_lanes(0)
a = ctx.empty(lanes); a.random_(-2**31, 2**31-1)
for _ in range(2):
    ctx.bootstrap_wo_ks(a)
torch.cuda.synchronize()
