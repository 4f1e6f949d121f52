"""one-gate-level launches of the latency kernel K (default 11 = brl) for ncu: python tools/brl_prof.py [K]"""
import os, sys, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ispass_maxw23_b200 as tb, synth
ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 11), synth.random_words(tb.KSK_WORDS, 12))
ctx.set_narrow_kernel(int(sys.argv[1]) if len(sys.argv) > 1 else 11)
a = ctx.empty(2); a.random_(-2**31, 2**31-1)
for _ in range(3):
    ctx.bootstrap_wo_ks(a[:1])
torch.cuda.synchronize()
