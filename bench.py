#!/usr/bin/env python
"""bench.py -- bootstrapped gates/s of the B200 TFHE hot path (BASELINE.json metric), one JSON line.

Workload (BASELINE configs[2], the throughput sweep): one Algorithm-1 level of
G independent NAND/XOR gates per GPU (seeded 50/50 mix, two fresh input ciphertexts per gate), tfhe-lib
128-bit parameters.  A step = the whole hot path over that level: linear combination, mod switch, 630 CMux
blind rotation, extraction, key switch, and for N > 1 the in-place NCCL all-gather of the
level's output rows.  Weak scaling: G gates per GPU, N*G in total.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--gates-per-gpu G] [--impl ours|reference]

`value` = N*G*K / (max over ranks of the CUDA-event time of the K steps).  `e2e` = the same metric through the
C ABI with HOST buffers (tb_run_netlist_host: pinned inputs H2D, all levels, outputs D2H, synchronise) per
step.  `cpu_baseline` = the CPU oracle (oracle/, schoolbook TFHE) timed on this host's cores on a bounded
sample of the same workload.  --impl reference times that oracle alone as the reference arm.
Key material and ciphertexts in the timed GPU arm are seeded uniform words: TFHE evaluation is
data-oblivious, so timing does not depend on them; bit-exactness on this exact configuration is
checked by tests/test_gpu_parity.py::test_throughput_level_bench_size_sampled.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "bootstrapped gates/sec (box, device-timed) at 1/2/4/8 B200; % of roofline"
UNIT = "gates/s"
CMUX_BFLY = 12 * 5 * 1024          # 12 negacyclic NTTs of N = 1024 per CMux step (6 forward + 6 inverse)
CMUX_MAC = 6 * 6 * 1024            # pointwise 64-bit multiply-accumulates per CMux step
# FP64 variant (--br-variant 10): FP64-pipe warp instructions per CMux step and lane of the implemented
# structure (10 transforms of 9 radix-2 stages with 6-DFMA CT / 8-op GS butterflies and constant twiddle
# factors, 1,536 MAC DFMAs, digit conversions), counted by ncu smsp__inst_executed_pipe_fp64 / (lanes x 630)
# on a 4,736-lane launch (profiles/r01_ncu_brf_summary.md)
CMUX_FP64_INSTR = 7032
N_LWE = 630


def workload_name(G):
    return ("cfg3 throughput sweep: one level of %d independent NAND/XOR gates per GPU (seeded 50/50), "
            "tfhe-lib 128-bit params n=630 N=1024 k=1 l=3 Bgbit=7 KS t=8 base 4" % G)


# ------------------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampled every 200 ms while the timed region runs (B200_PROFILING.md clocks line)."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_id: str):
        self.gpu_id, self.rows, self.proc = gpu_id, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", self.gpu_id, "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if len(r) >= 7 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 7 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows if len(r) >= 7 for k in range(4) if r[3 + k] == "Active"})
        pw = [float(r[2]) for r in self.rows if len(r) >= 7 and r[2].replace(".", "").isdigit()]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm), "power_w_max": max(pw) if pw else None}


def gpu_id_for(dev: int) -> str:
    import torch
    try:
        u = str(torch.cuda.get_device_properties(dev).uuid)
        return u if u.startswith("GPU-") else "GPU-" + u
    except Exception:
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        return vis.split(",")[dev] if vis else str(dev)


# ------------------------------------------------------------------------------------------------ oracle
def host_threads():
    """the host cores this process may use (torchrun sets OMP_NUM_THREADS=1 per rank; the oracle legs run on
    rank 0 alone while the other ranks wait, so they take every core)"""
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_rate(G_types, seconds_hint=None):
    """Time the CPU oracle on a bounded sample of the workload: 4 gates per host thread (NAND/XOR as in
    the GPU arm) with real seeded keys; returns (gates/s, threads, sample description)."""
    import numpy as np
    import oracle as O
    import synth
    threads = host_threads()
    keys = O.keygen(O.DEFAULT, seed=99)
    ns = 4 * threads
    types = np.asarray(G_types[:ns], np.int32)
    bits = synth.random_bits(2 * ns, 98)
    ca, cb = O.encrypt_bits(keys, bits[0::2], 1), O.encrypt_bits(keys, bits[1::2], 2)
    t0 = time.perf_counter()
    O.gates(keys, types, ca, cb, nthreads=threads)
    dt = time.perf_counter() - t0
    return ns / dt, threads, "%d NAND/XOR gates of the same workload (4 per thread) on %d host threads, %.1f s" % (
        ns, threads, dt)


def run_reference(args, rank):
    """--impl reference: the CPU oracle as it stands, on this host's cores (rank 0 only)."""
    if rank != 0:
        return
    import numpy as np
    import oracle as O
    import synth
    O.build()
    threads = host_threads()
    keys = O.keygen(O.DEFAULT, seed=99)
    n = synth.independent_level(threads * (args.warmup + args.steps), seed=1)
    bits = synth.random_bits(2 * n["type"].size, 2)
    ca, cb = O.encrypt_bits(keys, bits[0::2], 3), O.encrypt_bits(keys, bits[1::2], 4)
    per = threads                     # one gate per thread per step: a bounded sample of the workload
    times = []
    for s in range(args.warmup + args.steps):
        sl = slice(s * per, (s + 1) * per)
        t0 = time.perf_counter()
        O.gates(keys, n["type"][sl], ca[sl], cb[sl], nthreads=threads)
        times.append(time.perf_counter() - t0)
    t = sum(times[args.warmup:])
    value = per * args.steps / t
    sample = "%d steps x %d NAND/XOR gates (one per host thread) of the cfg3 workload" % (args.steps, per)
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic (seeded keys and inputs)",
        "config": {"workload": workload_name(args.gates_per_gpu), "oracle": "plain C schoolbook TFHE (oracle/)"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ------------------------------------------------------------------------------------------------ launch
def _free_port():
    import socket
    so = socket.socket()
    so.bind(("127.0.0.1", 0))
    port = so.getsockname()[1]
    so.close()
    return port


def spawn_ranks(args):
    """`python bench.py --gpus N` without torchrun: start N ranks (one per GPU) ourselves, the way the driver
    does (torch.distributed.run, rendezvous on 127.0.0.1).  Fails loudly if the node has fewer GPUs (a run that
    silently timed one GPU would print the wrong n_gpus)."""
    import torch
    if not args.one_gpu_ranks:
        have = torch.cuda.device_count()
        if have < args.gpus:
            print("bench.py: --gpus %d but only %d GPU(s) are visible on this node (use --one-gpu-ranks for a "
                  "functional check of the N > 1 path on one GPU)" % (args.gpus, have), file=sys.stderr)
            sys.exit(2)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(args.gpus),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


# ------------------------------------------------------------------------------------------------ latency roof
# One bootstrap in latency mode runs on one cluster of the latency kernel.  Its
# floor is the pipe work of the 630 CMux steps spread over the cluster's SMs: brl (11) is FP64-bound, per CMux
# step 6 forward + 4 inverse folded 512-point complex transforms (9 radix-2 stages x 256 butterflies, 6 FP64
# lane-ops per CT and 8 per GS butterfly) + the MAC (6 rows x 4 outputs x 512 complex x 4 DFMA):
#   6 x 13,824 + 4 x 18,432 + 49,152 = 205,824 FP64 lane-ops per CMux step, over 4 SMs x 64 FP64 lanes/clk.
# br9 (9) is IMAD-bound: 12 transforms x 5,120 Shoup butterflies x 4 IMAD slots + 36,864 MACs x 2 + 6,144
# reductions x 5 = 350,208 IMAD slots per step over 2 SMs x 64 IMAD lanes/clk.
LATENCY_WORK = {11: ("brl_kernel", 205824, 4, "FP64 lane-ops"), 9: ("br9_kernel", 350208, 2, "IMAD slots")}


def latency_roofline(level_ms, ks_ms, clk_mhz, kernel):
    name, work, sms, unit = LATENCY_WORK[kernel]
    floor_ms = N_LWE * work / (sms * 64 * clk_mhz * 1e6) * 1e3
    br_ms = level_ms - ks_ms
    return {"kernel": name, "cluster_sms": sms, "work_per_cmux": work, "unit": unit,
            "floor_ms_630_steps": floor_ms, "measured_br_ms": br_ms, "frac": floor_ms / br_ms if br_ms > 0 else None,
            "peak_source": "derived: %d SMs x 64 lanes/clk x %.0f MHz (median SM clock in the timed region)"
                           % (sms, clk_mhz)}


# ------------------------------------------------------------------------------------------------ ours
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--gates-per-gpu", type=int, default=65536)
    ap.add_argument("--lanes-per-cta", type=int, default=0, help="0 = auto per launch size")
    ap.add_argument("--br-variant", type=int, default=6, choices=[6, 10, 12, 14, 15])
    ap.add_argument("--ks-tile", type=int, default=8, choices=[8, 16, 32])
    ap.add_argument("--exchange", default="fused", choices=["fused", "allgather"],
                    help="N > 1: per-level exchange of output rows (fused into the key switch over NVLink peer "
                         "memory, or an NCCL all-gather)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-sweep", action="store_true", help="skip the 1 K - 256 K gates-per-level sweep")
    ap.add_argument("--one-gpu-ranks", action="store_true",
                    help="functional check of the N > 1 path on a one-GPU box: every rank on cuda:0, gloo process "
                         "group (the numbers are not a scaling measurement)")
    args = ap.parse_args()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        spawn_ranks(args)
    if world != args.gpus:
        print("bench.py: --gpus %d but WORLD_SIZE=%d" % (args.gpus, world), file=sys.stderr)
        sys.exit(2)
    if args.warmup < 3:
        args.warmup = 3                                  # timing rule: >= 3 warm-up steps
    if world > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")     # keep the communicator / NVLS lines visible (stderr)
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ispass_maxw23_b200 as tb
    import synth

    tb.build()                                        # no-op when the in-tree .so is current
    if args.one_gpu_ranks:
        local = 0
    torch.cuda.set_device(local)
    group = None
    if world > 1:
        if args.one_gpu_ranks:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        group = dist.group.WORLD

    def max_over_ranks(x):
        if group is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=ctx.device)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x):
        if group is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=ctx.device)
        dist.all_reduce(t)
        return float(t.item())

    G = args.gates_per_gpu
    total = G * world
    ctx = tb.Context(local)
    ctx.set_lanes_per_cta(args.lanes_per_cta)
    ctx.set_br_variant(args.br_variant)
    ctx.set_ks_tile(args.ks_tile)
    ctx.load_keys(synth.random_words(tb.BK_WORDS, 11), synth.random_words(tb.KSK_WORDS, 12))
    n = synth.independent_level(total, seed=13)
    net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], outputs=n["outputs"])
    dnet = ctx.upload(net)
    wires = ctx.wire_array(dnet, tb.slack_rows(dnet, world))
    gen = torch.Generator(device=ctx.device)
    gen.manual_seed(14)
    wires[:n["n_inputs"]].random_(-2 ** 31, 2 ** 31 - 1, generator=gen)     # resident inputs (> L2)

    exchange = args.exchange
    coll = "gloo (--one-gpu-ranks functional check)" if args.one_gpu_ranks else "NCCL"
    if group is not None and exchange == "fused":
        try:
            ctx.attach_peers(wires, group)
        except Exception as e:                       # no peer access between the GPUs: NCCL all-gather instead
            print("fused exchange unavailable (%s); using the NCCL all-gather" % e, file=sys.stderr)
            exchange = "allgather"

    def step():
        ctx.run_netlist(dnet, wires, group, exchange=exchange)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    sampler = ClockSampler(gpu_id_for(local))
    sampler.start()
    time.sleep(0.3)
    if group is not None:
        dist.barrier()
    torch.cuda.synchronize()
    ctx.profile(True)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    for _ in range(args.steps):
        step()
    ev1.record()
    torch.cuda.synchronize()
    if group is not None:
        dist.barrier()
    clocks = sampler.stop()
    ms = ev0.elapsed_time(ev1)
    br_ms, br_n, ks_ms, ks_n = ctx.profile_read()
    ctx.profile(False)
    ms = max_over_ranks(ms)
    value = total * args.steps / (ms / 1e3)

    # roofline of the dominant kernel (blind rotation).  Integer variant (br6): the integer-multiply
    # (FMA-heavy) pipe.  Algorithmic work = IMAD issue slots of the method's modular arithmetic (DESIGN.md
    # "Roofline"): per CMux step 61,440 Shoup mulmods x 4 slots (IMAD + IMAD.HI(2) + IMAD) + 36,864 64-bit MACs
    # x 2 (IMAD.WIDE) + 6,144 MAC reductions x 5.  Peak = 148 SMs x 64 IMAD lanes/clk (fma pipe: 16
    # lanes/clk/SMSP, B300_MICROARCH "Pipe rates") x the median SM clock sampled during the timed region.
    # FP64 variant (brf): FP64-pipe lane operations of the implemented structure over 148 SMs x 64 FP64
    # lanes/clk (measured 1.99 warp-instructions/clk/SM by ncu) x the same clock.
    bfly_rate, mac_rate = ctx.microbench()
    g0, g1, _ = tb.parallel.shard(total, world, rank)
    lanes_per_launch = g1 - g0
    br_launch_s = br_ms / max(br_n, 1) / 1e3
    sm_count = torch.cuda.get_device_properties(local).multi_processor_count
    clk_mhz = clocks.get("sm_mhz") or 1965.0
    peak = sm_count * 64 * clk_mhz * 1e6
    throughput_launch = lanes_per_launch > sm_count      # launches of <= SM-count lanes run a latency kernel
    lpc = ctx.br6_lanes_per_cta(lanes_per_launch) if args.br_variant == 6 and throughput_launch else None
    if args.br_variant == 10:
        per_bootstrap = N_LWE * CMUX_FP64_INSTR * 32
        unit, pipe = "G FP64-lane-ops/s", "FP64"
        work_text = "%d FP64 lane-ops = 630 x %d FP64 warp-instructions x 32 lanes" % (per_bootstrap, CMUX_FP64_INSTR)
    else:
        per_bootstrap = N_LWE * (CMUX_BFLY * 4 + CMUX_MAC * 2 + 6 * 1024 * 5)
        unit, pipe = "G IMAD-slots/s", "IMAD"
        work_text = "%d IMAD slots = 630 x (61,440 mulmod x 4 + 36,864 MAC x 2 + 6,144 reductions x 5)" % per_bootstrap
    work = per_bootstrap * lanes_per_launch
    achieved = work / br_launch_s
    bfly_work = N_LWE * (CMUX_BFLY + CMUX_MAC * bfly_rate / mac_rate) * lanes_per_launch
    traffic = None
    prof_path = os.path.join(ROOT, "profiles", "ncu_br_kernel_summary.json")
    if os.path.exists(prof_path):
        try:
            pj = json.load(open(prof_path))
            if (pj.get("lanes") == lanes_per_launch and pj.get("lanes_per_cta") == lpc
                    and pj.get("br_variant", 6) == args.br_variant):
                traffic = pj.get("dram_bytes_per_launch")
        except Exception:
            traffic = None
    roofline = {"bound": "alu", "achieved": achieved / 1e9, "peak": peak / 1e9, "unit": unit,
                "frac": achieved / peak, "traffic": traffic,
                "kernel": "%s (blind rotation + extraction)" % {10: "brf_kernel", 12: "brt_kernel", 14: "br6t_kernel", 15: "brq_kernel"}.get(
                    args.br_variant, "br%d_kernel" % args.br_variant),
                "kernel_ms_per_launch": br_launch_s * 1e3,
                "kernel_share_of_step": br_ms / ms if ms else None,
                "ks_kernel_ms_per_launch": ks_ms / max(ks_n, 1),
                "peak_source": "derived: %d SMs x 64 %s lanes/clk x %.0f MHz (median SM clock in the timed region)"
                               % (sm_count, pipe, clk_mhz),
                "work_per_bootstrap": work_text,
                "bootstraps_per_s_at_peak": peak / per_bootstrap}
    if args.br_variant != 10:
        roofline["microbench_crosscheck"] = {"butterflies_per_s": bfly_rate, "macs_per_s": mac_rate,
                                             "frac_of_microbench": bfly_work / br_launch_s / bfly_rate}
    # NTT-field choice (R1) from measured rates: per-bootstrap ceiling of each field's CMux work
    fr = ctx.microbench_fields()
    cmux30 = CMUX_BFLY / fr["shoup30_bfly_per_s"] + CMUX_MAC / fr["mac64_per_s"]
    gl_mac = 2 * 6 * 1024 / fr["goldilocks_bfly_per_s"]          # 12,288 Goldilocks MAC mulmods ~ butterflies
    cmux_gl = 8 * 5120 / fr["goldilocks_bfly_per_s"] + gl_mac
    cmux_gl4 = 8 * (5120 / fr["goldilocks_shift_bfly_per_s"] + 992 / fr["goldilocks_bfly_per_s"]) + gl_mac
    roofline["field_choice"] = dict(fr, **{
        "bootstraps_per_s_ceiling_30bit_3part": 1 / (N_LWE * cmux30),
        "bootstraps_per_s_ceiling_goldilocks_radix2": 1 / (N_LWE * cmux_gl),
        "bootstraps_per_s_ceiling_goldilocks_fourstep": 1 / (N_LWE * cmux_gl4),
        "goldilocks_over_30bit_cmux_time": min(cmux_gl, cmux_gl4) / cmux30,
        "note": "chip-wide register-resident rates; 30-bit: 12 transforms + 36,864 MACs per CMux; Goldilocks: 8 "
                "transforms (radix-2, or four-step with 5,120 shift butterflies + 992 general twiddles each) + "
                "12,288 MAC mulmods"})

    # narrow-level latency (one gate) and its roofline
    one = ctx.empty(2)
    one.random_(-2 ** 31, 2 ** 31 - 1, generator=gen)
    outl = ctx.empty(1)
    for _ in range(2):
        ctx.gates(tb.NAND, one[:1], one[1:2], out=outl)
    torch.cuda.synchronize()
    ctx.profile(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        ctx.gates(tb.NAND, one[:1], one[1:2], out=outl)
    e1.record()
    torch.cuda.synchronize()
    lat = e0.elapsed_time(e1) / 3
    _, _, lks_ms, lks_n = ctx.profile_read()
    ctx.profile(False)
    lat_roof = latency_roofline(lat, lks_ms / max(lks_n, 1), clk_mhz, 11)

    # throughput sweep of BASELINE configs[2] (1 K - 256 K independent gates per level, this GPU alone): device time
    # of one level per point, median of 2 after a warm-up (the headline `value` is the 65,536-gate point above)
    sweep = None
    if group is None and not args.no_sweep:
        sweep = {}
        for Gs in (1024, 4096, 16384, 262144):
            ns = synth.independent_level(Gs, seed=16)
            snet = ctx.upload(tb.Netlist(ns["n_inputs"], ns["type"], ns["in0"], ns["in1"], ns["in2"]))
            sw = ctx.wire_array(snet)
            sw[:ns["n_inputs"]].random_(-2 ** 31, 2 ** 31 - 1, generator=gen)
            ctx.run_netlist(snet, sw)
            times = []
            for _ in range(2):
                s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s0.record()
                ctx.run_netlist(snet, sw)
                s1.record()
                torch.cuda.synchronize()
                times.append(s0.elapsed_time(s1))
            sweep[str(Gs)] = {"level_ms": statistics.median(times), "gates_per_s": Gs / (statistics.median(times) / 1e3)}
            del sw
            snet.free()
        sweep[str(G)] = {"level_ms": ms / args.steps, "gates_per_s": G * args.steps / (ms / 1e3)}

    # e2e through the public API with host buffers: N = 1 the C ABI's tb_run_netlist_host; N > 1 the sharded
    # level loop (each rank copies in the input rows its gates read, runs its shard with the level exchange,
    # copies back the outputs it produced)
    e2e = None
    if not args.no_e2e:
        if group is None:
            nr = synth.independent_level(G, seed=15)
            rnet = ctx.upload(tb.Netlist(nr["n_inputs"], nr["type"], nr["in0"], nr["in1"], nr["in2"]))
            hin = torch.empty((nr["n_inputs"], tb.CT_WORDS), dtype=torch.int32, pin_memory=True)
            hin.random_(-2 ** 31, 2 ** 31 - 1)
            hout = torch.empty((G, tb.CT_WORDS), dtype=torch.int32, pin_memory=True)
            ow = np.ascontiguousarray(nr["outputs"], np.int64)
            ctx.run_netlist_host_into(rnet, hin, ow, hout)
            t0 = time.perf_counter()
            for _ in range(args.steps):
                ctx.run_netlist_host_into(rnet, hin, ow, hout)
            dt = time.perf_counter() - t0
            h2d, d2h = int(nr["n_inputs"] * tb.CT_WORDS * 4), int(G * tb.CT_WORDS * 4)
            api = "tb_run_netlist_host (pinned host inputs -> device, all levels, outputs -> host)"
            rnet.free()
        else:
            ow = np.ascontiguousarray(n["outputs"], np.int64)
            in_rows, outs = ctx.shard_io(dnet, world, rank, ow)
            r0 = int(in_rows[0]) if in_rows.size else 0
            hin = torch.empty((max(int(in_rows[-1]) + 1 - r0, 1) if in_rows.size else 1, tb.WIRE_STRIDE),
                              dtype=torch.int32, pin_memory=True)
            hin.random_(-2 ** 31, 2 ** 31 - 1)
            p0 = outs[0][0] if outs else 0
            hout = torch.empty((max(outs[-1][0] + 1 - p0, 1) if outs else 1, tb.CT_WORDS), dtype=torch.int32,
                               pin_memory=True)
            run_e2e = lambda: ctx.run_netlist_host_sharded(dnet, hin, ow, hout, wires, group, exchange=exchange,
                                                           inputs_row0=r0, out_pos0=p0)   # noqa: E731
            run_e2e()
            dist.barrier()
            t0 = time.perf_counter()
            for _ in range(args.steps):
                h2d, d2h = run_e2e()
            dt = time.perf_counter() - t0
            h2d, d2h = int(sum_over_ranks(h2d)), int(sum_over_ranks(d2h))
            api = ("Context.run_netlist_host_sharded (per rank: pinned host input rows of its shard -> device, "
                   "sharded level loop with the %s exchange, its output rows -> host)" % exchange)
        dt = max_over_ranks(dt)
        e2e = {"value": total * args.steps / dt, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "api": api}

    # N > 1: the same level without the exchange step (each rank runs its own gate range; no peer stores, no
    # barrier or all-gather inside the loop), to report the exchange's share of the level time
    exch = None
    if group is not None:
        if exchange == "fused":
            ctx.detach_peers()
        dist.barrier()
        torch.cuda.synchronize()
        k2 = min(args.steps, 3)
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record()
        for _ in range(k2):
            for L, (row0, ng, _, _) in enumerate(dnet.levels, start=1):
                a, b, _ = tb.parallel.shard(ng, world, rank)
                if b > a:
                    ctx.run_level(dnet, L, a, b, wires)
        f1.record()
        torch.cuda.synchronize()
        no_ms = max_over_ranks(f0.elapsed_time(f1) / k2)
        exch = {"level_ms_with_exchange": ms / args.steps, "level_ms_without_exchange": no_ms,
                "exchange_share": 1.0 - no_ms / (ms / args.steps)}

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        v, cores, sample = oracle_rate(n["type"])
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample}
    if group is not None:
        dist.barrier()                                    # other ranks wait while rank 0 times the oracle

    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32",
            "data": "synthetic: seeded uniform key material and ciphertexts (evaluation is data-oblivious, P:160)",
            "config": {"workload": workload_name(G), "gates_per_gpu": G, "total_gates": total,
                       "parallelism": "dp%d (level sharded; output rows exchanged %s)" % (
                           world, "by the key-switch kernels' stores into every GPU's wire array (NVLink peer "
                                  "memory) + %s barrier" % coll if exchange == "fused" else "by a %s all-gather" % coll),
                       "exchange": exchange if world > 1 else None,
                       "lanes_per_cta": lpc, "br_variant": args.br_variant,
                       "l2": "inputs larger than L2 (%.0f MB of input ciphertexts per GPU)" % (2 * G * 2524 / 1e6)},
            "roofline": roofline, "latency_roofline": lat_roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
            "gpu_launches": br_n + ks_n,
            "latency_ms": {"level_of_%d_gates" % total: ms / args.steps, "level_of_1_gate": lat},
            "exchange": exch, "sweep": sweep,
        }), flush=True)
    if group is not None:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
