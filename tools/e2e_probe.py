"""Where the end-to-end (host buffer) time of the bench level goes: device-only level, host path overlapped and
serial, bare pinned copies of the same bytes.  python tools/e2e_probe.py [G]"""
import os, sys, time
import numpy as np
import torch
sys.path.insert(0, os.getcwd())
import paper_conf_ispass_maxw23_b200 as tb, synth
G = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 1), synth.random_words(tb.KSK_WORDS, 2))
nr = synth.independent_level(G, seed=15)
net = tb.Netlist(nr["n_inputs"], nr["type"], nr["in0"], nr["in1"], nr["in2"])
d = ctx.upload(net)
hin = torch.empty((nr["n_inputs"], tb.CT_WORDS), dtype=torch.int32, pin_memory=True); hin.random_(-2**31, 2**31 - 1)
hout = torch.empty((G, tb.CT_WORDS), dtype=torch.int32, pin_memory=True)
ow = np.ascontiguousarray(nr["outputs"], np.int64)
w = ctx.wire_array(d); w[:nr["n_inputs"], :631] = hin.cuda()
def t(f, k=3):
    f(); torch.cuda.synchronize(); ts = []
    for _ in range(k):
        t0 = time.perf_counter(); f(); torch.cuda.synchronize(); ts.append((time.perf_counter() - t0) * 1e3)
    return round(min(ts), 2), round(float(np.median(ts)), 2)
res = {"G": G}
res["device_level_ms"] = t(lambda: ctx.run_netlist(d, w))
for ov in (True, False):
    ctx.set_host_overlap(ov)
    res["host_path_ms_overlap_%d" % ov] = t(lambda: ctx.run_netlist_host_into(d, hin, ow, hout))
ctx.set_host_overlap(True)
dev_in = torch.empty_like(hin, device="cuda"); dev_out = torch.empty_like(hout, device="cuda")
res["h2d_only_ms"] = t(lambda: dev_in.copy_(hin, non_blocking=True))
res["d2h_only_ms"] = t(lambda: hout.copy_(dev_out, non_blocking=True))
res["h2d_GBps"] = round(hin.numel() * 4 / res["h2d_only_ms"][0] / 1e6, 1)
print(res)
# the host path's copy shape: 631-word host rows (2,524 B) into 632-word device rows (2,528 B)
dw = torch.empty((nr["n_inputs"], 632), dtype=torch.int32, device="cuda")
def h2d_2d():
    dw[:, :631].copy_(hin, non_blocking=True)
def h2d_2d_host_wall():
    t0 = time.perf_counter(); dw[:, :631].copy_(hin, non_blocking=True); return (time.perf_counter() - t0) * 1e3
res2 = {"h2d_2d_ms": t(h2d_2d)}
torch.cuda.synchronize(); res2["h2d_2d_issue_wall_ms"] = round(h2d_2d_host_wall(), 2); torch.cuda.synchronize()
def staged():
    dev_in.copy_(hin, non_blocking=True); dw[:, :631].copy_(dev_in)
res2["h2d_staged_ms"] = t(staged)
ho = torch.empty((G, 631), dtype=torch.int32, pin_memory=True)
res2["d2h_2d_ms"] = t(lambda: ho.copy_(dw[:G, :631], non_blocking=True))
print(res2)
# per-kernel CUDA-event times inside both paths
def host_serial():
    ctx.set_host_overlap(False)
    try:
        ctx.run_netlist_host_into(d, hin, ow, hout)
    finally:
        ctx.set_host_overlap(True)
for name, f in (("device", lambda: ctx.run_netlist(d, w)), ("host", lambda: ctx.run_netlist_host_into(d, hin, ow, hout)),
                ("host_serial", host_serial)):
    f(); torch.cuda.synchronize()
    ctx.profile(True)
    t0 = time.perf_counter(); f(); torch.cuda.synchronize(); wall = (time.perf_counter() - t0) * 1e3
    recs = ctx.profile_read(); ctx.profile(False)
    print(name, "wall %.2f ms" % wall, recs if not isinstance(recs, dict) else {k: (round(v[0], 2) if isinstance(v, (list, tuple)) else v) for k, v in recs.items()})
