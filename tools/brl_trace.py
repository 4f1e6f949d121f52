"""Per-phase clock64 trace of brl_kernel (one lane, steps 100-115, per cluster rank): build with
  bash tools/buildvar.sh WORK trace -DTB_BRL_TRACE, then TB_LIB=scratch/lib_trace.so python tools/brl_trace.py
(DESIGN.md latency mode: A 2,100 / MAC 1,500 / inverse 1,530 / half swap + ACC update 750 of ~6,100 cycles)."""
import ctypes, os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ispass_maxw23_b200 as tb, synth
from paper_conf_ispass_maxw23_b200 import _native
ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 11), synth.random_words(tb.KSK_WORDS, 12))
ctx.set_narrow_kernel(11)
a = ctx.empty(1); b = ctx.empty(1); out = ctx.empty(1)
for _ in range(3): ctx.gates(tb.NAND, a, b, out=out)
torch.cuda.synchronize()
buf = np.zeros((4, 8, 16), np.int64)
assert _native.lib().tb_debug_brl_trace(ctypes.c_void_p(buf.ctypes.data)) == 0
names = ["start", "A done", "BK ok", "rows ok", "MAC done", "C done", "half ok", "ACC done"]
for r in range(4):
    d = buf[r] - buf[r][0]                      # relative to step start
    step = np.diff(buf[r][0])
    print("rank", r, "step cycles median", int(np.median(step)))
    print("   ", "  ".join("%s=%d" % (names[p], int(np.median(d[p]))) for p in range(1, 8)))
