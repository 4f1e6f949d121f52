#!/usr/bin/env python
"""Time every BASELINE.json configuration end to end on one GPU (device-timed, CUDA events) and print one
JSON line per config: gates, bootstraps, levels, total ms, per-level latency (median / p90 / max), gates/s.

Timing only: keys and input ciphertexts are seeded uniform words (TFHE evaluation is data-oblivious);
bit-exactness of the same netlists is covered by tests/test_gpu_parity.py and tests/test_gpu_workloads.py.

  python tools/workloads.py [--only cfg3] [--reps 2]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ispass_maxw23_b200 as tb  # noqa: E402
import synth  # noqa: E402


def configs():
    yield "cfg1_nand_truth_table", synth.independent_level(4, 1, kinds=(synth.NAND,))
    yield "cfg2_rca8", synth.ripple_carry_adder(8)
    for G in (1024, 4096, 16384, 65536, 262144):
        yield "cfg3_level_%d" % G, synth.independent_level(G, 2)
    yield "cfg4a_mul32x32", synth.array_multiplier(32)
    yield "cfg4b_sort16x16", synth.bubble_sort(16, 16)
    yield "cfg5_mnist_fig4", synth.mnist_fig4()
    yield "f3_attention_S", synth.attention(4, 32, 4)          # Attention_S shape (hidden 32)
    yield "f3_attention_L", synth.attention(4, 64, 4)          # Attention_L shape (hidden 64)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default=None)
    ap.add_argument("--reps", type=int, default=1)
    args = ap.parse_args()
    tb.build()
    ctx = tb.Context(0)
    ctx.load_keys(synth.random_words(tb.BK_WORDS, 1), synth.random_words(tb.KSK_WORDS, 2))
    for name, n in configs():
        if args.only and args.only not in name:
            continue
        net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"])
        d = ctx.upload(net)
        w = ctx.wire_array(d)
        w[:n["n_inputs"]].random_(-2 ** 31, 2 ** 31 - 1)
        ctx.run_level(d, 1, 0, d.levels[0][1], w)            # warm-up (allocations, attributes)
        torch.cuda.synchronize()
        best = None
        for _ in range(args.reps):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(d.n_levels + 1)]
            ev[0].record()
            for L, (_, ng, _, _) in enumerate(d.levels, start=1):
                ctx.run_level(d, L, 0, ng, w)
                ev[L].record()
            torch.cuda.synchronize()
            per = np.array([ev[k].elapsed_time(ev[k + 1]) for k in range(d.n_levels)])
            if best is None or per.sum() < best.sum():
                best = per
        tot = float(best.sum())
        print(json.dumps({"config": name, "gates": net.n_gates, "bootstrapped_gates": d.n_boot,
                          "bootstraps": sum(lv[3] for lv in d.levels), "levels": d.n_levels,
                          "max_width": max(lv[1] for lv in d.levels), "total_ms": round(tot, 2),
                          "level_ms_median": round(float(np.median(best)), 3),
                          "level_ms_p90": round(float(np.percentile(best, 90)), 3),
                          "level_ms_max": round(float(best.max()), 3),
                          "gates_per_s": round(d.n_boot / tot * 1e3, 1),
                          "bootstraps_per_s": round(sum(lv[3] for lv in d.levels) / tot * 1e3, 1)}), flush=True)
        d.free()
        del w
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
