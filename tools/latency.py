"""Narrow-level latency of each latency-mode kernel: device time of one level of L NAND gates (BR + KS).

  python tools/latency.py [kernels...]     (default: 9 11; 6 = the throughput kernel br6, latency mode off)
Inputs are seeded uniform words (evaluation is data-oblivious); parity is tests/test_gpu_parity.py's job.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ispass_maxw23_b200 as tb  # noqa: E402
import synth  # noqa: E402


def main():
    kernels = [int(a) for a in sys.argv[1:]] or [9, 11]
    ctx = tb.Context(0)
    ctx.load_keys(synth.random_words(tb.BK_WORDS, 11), synth.random_words(tb.KSK_WORDS, 12))
    g = torch.Generator(device=ctx.device)
    g.manual_seed(3)
    for k in kernels:
        if k == 6:
            ctx.set_narrow_lanes(0)
        else:
            ctx.set_narrow_lanes(1000)                     # latency mode for every width measured here
            ctx.set_narrow_kernel(k)
        for lanes in (1, 4, 16, 32, 37, 74, 100, 148) + ((200, 222, 296, 400, 592) if k in (6, 16) else ()):
            a, b = ctx.empty(lanes), ctx.empty(lanes)
            a.random_(-2 ** 31, 2 ** 31 - 1, generator=g)
            b.random_(-2 ** 31, 2 ** 31 - 1, generator=g)
            out = ctx.empty(lanes)
            ctx.gates(tb.NAND, a, b, out=out)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(3):
                ctx.gates(tb.NAND, a, b, out=out)
            e1.record()
            torch.cuda.synchronize()
            print(json.dumps({"narrow_kernel": k, "lanes": lanes, "level_ms": e0.elapsed_time(e1) / 3}), flush=True)


if __name__ == "__main__":
    main()
