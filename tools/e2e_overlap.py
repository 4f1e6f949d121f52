#!/usr/bin/env python
"""End-to-end (host buffers) time of multi-level BASELINE netlists with the host copies overlapped with the level
loop (tb_run_netlist_host, default) vs serialised (tb_set_host_overlap(0)): SURVEY 8(f) f1.  Keys and input
ciphertexts are seeded uniform words (timing does not depend on them); pinned host buffers.
    python tools/e2e_overlap.py            -> one JSON line per (netlist, mode)"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ispass_maxw23_b200 as tb  # noqa: E402
import synth  # noqa: E402

tb.build()
ctx = tb.Context(0)
ctx.load_keys(synth.random_words(tb.BK_WORDS, 1), synth.random_words(tb.KSK_WORDS, 2))
nets = {"cfg4a multiplier 32x32": synth.array_multiplier(32, full=True), "cfg5 Fig.4 MNIST": synth.mnist_fig4()}
for name, n in nets.items():
    dnet = ctx.upload(tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]))
    hin = torch.empty((n["n_inputs"], tb.CT_WORDS), dtype=torch.int32).pin_memory()
    hin.random_(-2 ** 31, 2 ** 31 - 1)
    ow = np.ascontiguousarray(n["outputs"], np.int64)
    hout = torch.empty((ow.size, tb.CT_WORDS), dtype=torch.int32).pin_memory()
    reps = 3 if n["type"].size < 100000 else 1
    for overlap in (False, True, False, True):
        ctx.set_host_overlap(overlap)
        ctx.run_netlist_host_into(dnet, hin, ow, hout)                   # warm
        t0 = time.perf_counter()
        for _ in range(reps):
            ctx.run_netlist_host_into(dnet, hin, ow, hout)
        dt = (time.perf_counter() - t0) / reps
        print(json.dumps({"netlist": name, "gates": int(n["type"].size), "levels": dnet.n_levels,
                          "inputs": int(n["n_inputs"]), "h2d_mb": n["n_inputs"] * 2524 / 1e6,
                          "overlap": overlap, "e2e_s": dt, "gates_per_s": n["type"].size / dt}), flush=True)
    dnet.free()
