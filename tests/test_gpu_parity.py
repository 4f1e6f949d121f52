"""GPU parity: the sm_100a kernels (through the C ABI) against the CPU oracle, bit for bit (-m gpu).

Inputs are seeded and synthetic; keys come from the oracle's client-side KeyGen.
Every comparison is element-by-element equality of u32 words -- the path is integer-exact, so the tolerance
is zero (BASELINE north_star: "bit-exact gate-bootstrapping ciphertexts versus the CPU oracle").
"""
import numpy as np
import pytest

import oracle as O
import synth
from oracle.plain import simulate

pytestmark = pytest.mark.gpu

M32 = 1 << 32


@pytest.fixture(scope="module")
def tb():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ispass_maxw23_b200 as tb
    tb.build()
    return tb


@pytest.fixture(scope="module")
def keys():
    return O.keygen(O.DEFAULT, seed=20261017)


@pytest.fixture(scope="module")
def ctx(tb, keys):
    c = tb.Context(0)
    c.load_keys(keys.bk, keys.ksk)
    return c


def enc(keys, bits, seed):
    return O.encrypt_bits(keys, np.asarray(bits, np.uint8), seed)


# ------------------------------------------------------------------------------------- NTT product
def test_ntt_product_equals_schoolbook(tb, ctx):
    import torch
    rng = np.random.default_rng(1)
    cases = [(rng.integers(-64, 64, (6, 1024)), rng.integers(0, M32, (6, 1024), dtype=np.uint64)),
             (np.full((6, 1024), -64), np.full((6, 1024), M32 - 1, np.uint64)),      # worst case
             (np.full((6, 1024), 63), np.full((6, 1024), 1 << 31, np.uint64)),
             (np.zeros((6, 1024), int), rng.integers(0, M32, (6, 1024), dtype=np.uint64))]
    for d, b in cases:
        d32 = d.astype(np.int32)
        b32 = b.astype(np.uint32)
        want = np.zeros(1024, np.uint32)
        for r in range(6):
            want = O.negacyclic_muladd(d32[r], b32[r], want)
        got = ctx.ntt_muladd6(torch.from_numpy(d32).cuda(), torch.from_numpy(b32.view(np.int32)).cuda())
        assert (got.cpu().numpy().view(np.uint32) == want).all()


def test_fft_product_equals_schoolbook(tb, ctx):
    """FP64-pipe folded FFT product (16-bit BK halves) rounds to the exact schoolbook result, incl. worst case"""
    import torch
    rng = np.random.default_rng(3)
    cases = [(rng.integers(-64, 64, (6, 1024)), rng.integers(0, M32, (6, 1024), dtype=np.uint64)),
             (np.full((6, 1024), -64), np.full((6, 1024), 0x80008000, np.uint64)),      # |halves| = 2^15
             (np.full((6, 1024), 63), np.full((6, 1024), M32 - 1, np.uint64)),
             (rng.choice([-64, 63], (6, 1024)), rng.choice([0x80008000, 0x7FFF7FFF], (6, 1024)).astype(np.uint64))]
    for d, b in cases:
        d32 = d.astype(np.int32)
        b32 = b.astype(np.uint32)
        want = np.zeros(1024, np.uint32)
        for r in range(6):
            want = O.negacyclic_muladd(d32[r], b32[r], want)
        got = ctx.fft_muladd6(torch.from_numpy(d32).cuda(), torch.from_numpy(b32.view(np.int32)).cuda())
        assert (got.cpu().numpy().view(np.uint32) == want).all()


# ------------------------------------------------------------------------------------- blind rotation
def test_bootstrap_wo_ks_bit_exact(tb, ctx, keys):
    rng = np.random.default_rng(2)
    cts = rng.integers(0, M32, (5, 631), dtype=np.uint64).astype(np.uint32)      # arbitrary inputs
    cts = np.concatenate([cts, enc(keys, [0, 1, 1], 3)])
    ext = ctx.bootstrap_wo_ks(ctx.to_device(cts))
    got = ext[:, :1025].cpu().numpy().view(np.uint32)
    for k in range(cts.shape[0]):
        assert (got[k] == O.bootstrap_wo_ks(keys, cts[k])).all(), k


def oracle_bootstrap_many(keys, cts):
    """O.bootstrap_wo_ks over independent rows on all host cores (ctypes releases the GIL)"""
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(O.max_threads()) as ex:
        return np.stack(list(ex.map(lambda c: O.bootstrap_wo_ks(keys, c), cts)))


@pytest.mark.parametrize("kernel", [0, 9, 11, 13, 16])
def test_narrow_level_latency_mode_bit_exact(tb, ctx, keys, kernel):
    """small launches run the latency kernel (br9: 2-SM cluster per lane, brl: 4-SM cluster per lane on the
    FP64 path, brtl: one SM per lane on the tensor cores, brl2: 2-SM cluster per lane on the FP64 path; 40 lanes =
    160 CTAs is more than one wave of brl, 80 lanes more than one wave of brl2 / br9); 149 lanes fall back to the
    throughput kernel.  Every lane of the 1-, 3- and 40-lane launches is compared with the oracle, three of 80
    (first, one in the second wave, last) and the first and last of 149."""
    rng = np.random.default_rng(39 + kernel)
    ctx.set_narrow_kernel(kernel)
    try:
        for count in (1, 3, 40, 80, 149):
            cts = rng.integers(0, M32, (count, 631), dtype=np.uint64).astype(np.uint32)
            got = ctx.bootstrap_wo_ks(ctx.to_device(cts))[:, :1025].cpu().numpy().view(np.uint32)
            idx = np.arange(count) if count <= 40 else (np.array([0, 77, count - 1]) if count == 80
                                                         else np.array([0, count - 1]))
            assert (got[idx] == oracle_bootstrap_many(keys, cts[idx])).all(), count
    finally:
        ctx.set_narrow_kernel(0)


@pytest.mark.parametrize("variant", [6, 10, 12, 14, 15])
def test_blind_rotation_variants_bit_exact(tb, ctx, keys, variant):
    """every blind-rotation kernel variant (br6 integer NTT / brf FP64 FFT / brt tensor-core NTT) on a ragged
    batch of 9"""
    rng = np.random.default_rng(40 + variant)
    cts = rng.integers(0, M32, (9, 631), dtype=np.uint64).astype(np.uint32)
    ctx.set_br_variant(variant)
    ctx.set_narrow_lanes(0)                  # throughput kernels even for a small batch
    try:
        got = ctx.bootstrap_wo_ks(ctx.to_device(cts))[:, :1025].cpu().numpy().view(np.uint32)
    finally:
        ctx.set_br_variant(6)
        ctx.set_narrow_lanes(148)
    for k in range(9):
        assert (got[k] == O.bootstrap_wo_ks(keys, cts[k])).all(), k


def test_trivial_inputs_closed_form(tb, ctx):
    phis = [0, 1, (1 << 20) - 1, 1 << 20, 1 << 31, M32 - (1 << 20) - 1, M32 - (1 << 20), M32 - 1, 0x9E3779B9]
    cts = np.zeros((len(phis), 631), np.uint32)
    cts[:, 630] = phis
    ext = ctx.bootstrap_wo_ks(ctx.to_device(cts)).cpu().numpy().view(np.uint32)
    for k, phi in enumerate(phis):
        bbar = ((phi + (1 << 20)) % M32) >> 21
        assert ext[k, :1024].tolist() == [0] * 1024
        assert int(ext[k, 1024]) == ((1 << 29) if bbar < 1024 else M32 - (1 << 29))


def test_structured_key_closed_form(tb):
    """zero-noise BK with masks in 2^11 Z: the extracted phase is +-1/8 by the sign rule, exactly."""
    params = O.Params(sigma_bk=0.0, bk_mask_mult=1 << 11)
    k = O.keygen(params, seed=5, with_ksk=False)
    c = tb.Context(0)
    c.load_bk(k.bk)
    rng = np.random.default_rng(4)
    cts = rng.integers(0, M32, (4, 631), dtype=np.uint64).astype(np.uint32)
    ext = c.bootstrap_wo_ks(c.to_device(cts)).cpu().numpy().view(np.uint32)
    ms = lambda v: ((int(v) + (1 << 20)) % M32) >> 21
    for r in range(4):
        phibar = (ms(cts[r, 630]) - sum(ms(cts[r, i]) * int(k.s[i]) for i in range(630))) % 2048
        want = (1 << 29) if phibar < 1024 else M32 - (1 << 29)
        phase = (int(ext[r, 1024]) - sum(int(ext[r, j]) * int(k.S[j]) for j in range(1024))) % M32
        assert phase == want
    c.close()


# ------------------------------------------------------------------------------------- key switch
@pytest.mark.parametrize("narrow,count", [(148, 37), (0, 37), (148, 3), (148, 7), (0, 600)])
def test_keyswitch_bit_exact(tb, ctx, keys, narrow, count):
    """split key switch (narrow levels: 16 CTAs per gate at 37 gates, 64 at 3, 32 at 7) and tiled key switch
    (ragged: 4 tiles of 8 + 5, each sliced 16 ways over the input coefficients; 600 gates = 75 tiles x 8
    slices + reduction)"""
    rng = np.random.default_rng(6 + count)
    ext = rng.integers(0, M32, (count, 1025), dtype=np.uint64).astype(np.uint32)
    ext[0, :] = 0
    ext[1, :1024] = 0xFFFFFFFF
    dev = ctx.to_device(ext, stride=1028)
    ctx.set_narrow_lanes(narrow)
    try:
        got = ctx.to_host(ctx.keyswitch(dev))
    finally:
        ctx.set_narrow_lanes(148)
    for r in range(ext.shape[0]):
        assert (got[r] == O.keyswitch(keys, ext[r])).all(), r


def test_keyswitch_split_scratch_nondefault_threshold(tb, keys):
    """with a non-default narrow-level threshold (10) on a fresh context, a 9-gate split key switch
    writes 9 x 32 partial rows (more than 10 x 16): the scratch is sized from the launch, results bit-exact"""
    c = tb.Context(0)
    try:
        c.load_keys(keys.bk, keys.ksk)
        c.set_narrow_lanes(10)
        rng = np.random.default_rng(61)
        for count in (9, 4, 10):
            ext = rng.integers(0, M32, (count, 1025), dtype=np.uint64).astype(np.uint32)
            got = c.to_host(c.keyswitch(c.to_device(ext, stride=1028)))
            for r in range(count):
                assert (got[r] == O.keyswitch(keys, ext[r])).all(), (count, r)
    finally:
        c.close()


# ------------------------------------------------------------------------------------- gates
def test_nand_truth_table_config1(tb, ctx, keys):
    """BASELINE configs[0]: NAND truth table, 4 bootstraps, bit-exact and decrypting to 1,1,1,0."""
    A, B = [0, 0, 1, 1], [0, 1, 0, 1]
    ca, cb = enc(keys, A, 11), enc(keys, B, 12)
    out = ctx.to_host(ctx.gates(tb.NAND, ctx.to_device(ca), ctx.to_device(cb)))
    want = O.gates(keys, O.NAND, ca, cb)
    assert (out == want).all()
    assert O.decrypt_bits(keys, out).tolist() == [1, 1, 1, 0]


@pytest.mark.parametrize("gate", [O.AND, O.OR, O.NOR, O.XOR, O.XNOR, O.ANDNY, O.ANDYN, O.ORNY, O.ORYN])
def test_every_two_input_gate_bit_exact(tb, ctx, keys, gate):
    A, B = [0, 0, 1, 1, 1], [0, 1, 0, 1, 1]
    ca, cb = enc(keys, A, 100 + gate), enc(keys, B, 200 + gate)
    out = ctx.to_host(ctx.gates(gate, ctx.to_device(ca), ctx.to_device(cb)))
    assert (out == O.gates(keys, gate, ca, cb)).all()
    assert O.decrypt_bits(keys, out).tolist() == [(gate >> (2 * a + b)) & 1 for a, b in zip(A, B)]


def test_mux_and_not(tb, ctx, keys):
    A8 = [(i >> 2) & 1 for i in range(8)]
    B8 = [(i >> 1) & 1 for i in range(8)]
    C8 = [i & 1 for i in range(8)]
    ca, cb, cc = enc(keys, A8, 31), enc(keys, B8, 32), enc(keys, C8, 33)
    out = ctx.to_host(ctx.gates(tb.MUX, ctx.to_device(ca), ctx.to_device(cb), ctx.to_device(cc)))
    assert (out == O.gates(keys, O.MUX, ca, cb, cc)).all()
    assert O.decrypt_bits(keys, out).tolist() == [b if a else c for a, b, c in zip(A8, B8, C8)]
    nt = ctx.to_host(ctx.gates(tb.NOT, ctx.to_device(ca)))
    assert (nt == O.gates(keys, O.NOT, ca)).all()


@pytest.mark.parametrize("lanes", [1, 2, 3, 4])
def test_lanes_per_cta_and_ragged_tail(tb, ctx, keys, lanes):
    """5 gates over CTAs of 1..4 lanes (ragged last CTA); stride 640 rows."""
    ctx.set_lanes_per_cta(lanes)
    ctx.set_narrow_lanes(0)
    try:
        A, B = synth.random_bits(5, 40 + lanes), synth.random_bits(5, 50 + lanes)
        ca, cb = enc(keys, A, 60 + lanes), enc(keys, B, 70 + lanes)
        out = ctx.to_host(ctx.gates(tb.XOR, ctx.to_device(ca, 640), ctx.to_device(cb, 640)))
        assert (out == O.gates(keys, O.XOR, ca, cb)).all()
    finally:
        ctx.set_lanes_per_cta(0)
        ctx.set_narrow_lanes(148)


def test_auto_lanes_per_cta(tb, ctx):
    """Auto lanes per CTA: 2 on full waves of 148 SMs x 4 lanes, 1 where lane-by-lane
    scheduling of the ragged last wave wins (profiles/r01f_lanes_sweep.txt); fixed settings pass through."""
    import torch
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    slot1, slot2 = 296, 279             # the calibration constants of tb_runtime.cu (kBr6SlotG1 / kBr6SlotG2)

    def expect(n):                      # busiest-SM estimate on this device's SM count
        return 1 if slot1 * -(-n // sms) < 2 * slot2 * -(-n // (2 * sms)) else 2
    ctx.set_lanes_per_cta(0)
    sizes = (4 * sms, 1024, 1536, 2048, 65536)
    assert [ctx.br6_lanes_per_cta(n) for n in sizes] == [expect(n) for n in sizes]
    if sms == 148:                      # the measured B200 picks (profiles/r01f_lanes_sweep.txt)
        assert [ctx.br6_lanes_per_cta(n) for n in sizes] == [2, 1, 1, 2, 2]
    ctx.set_lanes_per_cta(3)
    try:
        assert ctx.br6_lanes_per_cta(1024) == 3
    finally:
        ctx.set_lanes_per_cta(0)
    with pytest.raises(tb.TBError):
        ctx.set_lanes_per_cta(5)


@pytest.mark.parametrize("lanes", [1, 2, 3])
def test_fft_variant_lanes_per_cta(tb, ctx, keys, lanes):
    """FP64 variant at 1, 2, 3 lanes per CTA (16, 16, 18 warps): 7 bootstraps, so every CTA size has a ragged tail"""
    rng = np.random.default_rng(80 + lanes)
    cts = rng.integers(0, M32, (7, 631), dtype=np.uint64).astype(np.uint32)
    ctx.set_br_variant(10)
    ctx.set_lanes_per_cta(lanes)
    ctx.set_narrow_lanes(0)
    try:
        got = ctx.bootstrap_wo_ks(ctx.to_device(cts))[:, :1025].cpu().numpy().view(np.uint32)
    finally:
        ctx.set_br_variant(6)
        ctx.set_lanes_per_cta(0)
        ctx.set_narrow_lanes(148)
    for k in range(7):
        assert (got[k] == O.bootstrap_wo_ks(keys, cts[k])).all(), k


def test_edge_cases(tb, ctx, keys):
    import torch
    empty = ctx.empty(0)
    assert ctx.gates(tb.NAND, empty, empty).shape[0] == 0
    one_a, one_b = enc(keys, [1], 80), enc(keys, [1], 81)
    out = ctx.to_host(ctx.gates(tb.AND, ctx.to_device(one_a, 631), ctx.to_device(one_b, 631)))   # packed stride
    assert (out == O.gates(keys, O.AND, one_a, one_b)).all()
    with pytest.raises(tb.TBError):
        ctx.gates(5, ctx.to_device(one_a), ctx.to_device(one_b))          # not a gate code
    with pytest.raises(tb.TBError):
        ctx.gates(tb.NAND, ctx.to_device(one_a))                            # missing cb


def test_peer_exchange_api_errors_and_scope(tb, ctx, keys):
    """fused-exchange plumbing: bad arguments fail loudly (TB_EINVAL), a handle exports, and with a peer array
    registered a run on another wire array (here tb_run_netlist_host) does not
    store into the peer (the mirror is scoped to the registered array)"""
    import ctypes
    import torch
    from paper_conf_ispass_maxw23_b200 import _native
    L = _native.lib()
    h = (ctypes.c_ubyte * 64)()
    off = ctypes.c_int64()
    assert L.tb_ipc_export(None, h, ctypes.byref(off)) == _native.TB_EINVAL
    assert L.tb_set_peer_wires(ctx._h, None, None, -1) == _native.TB_EINVAL
    assert L.tb_set_peer_wires(ctx._h, None, None, 1) == _native.TB_EINVAL
    w = ctx.empty(8)
    assert L.tb_ipc_export(ctypes.c_void_p(w.data_ptr()), h, ctypes.byref(off)) == 0
    assert L.tb_ipc_import(ctx._h, None, 0, None, None) == _native.TB_EINVAL
    # register `mirror` as the "peer" of `own`; a host-buffer run (context-owned wire array) must not touch it
    n = synth.independent_level(4, 2)
    net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], outputs=n["outputs"])
    dnet = ctx.upload(net)
    own, mirror = ctx.wire_array(dnet), ctx.wire_array(dnet)
    mirror.fill_(7)
    arr = (ctypes.c_void_p * 1)(mirror.data_ptr())
    assert L.tb_set_peer_wires(ctx._h, ctypes.c_void_p(own.data_ptr()), arr, 1) == 0
    try:
        cts = enc(keys, synth.random_bits(n["n_inputs"], 3), 4)
        ctx.run_netlist_host(dnet, cts, n["outputs"])
        torch.cuda.synchronize()
        assert bool((mirror == 7).all())
        own[:n["n_inputs"], :631] = ctx.to_device(cts)[:, :631]
        ctx.run_netlist(dnet, own)                  # the registered array: every output row mirrored
        torch.cuda.synchronize()
        rows = slice(n["n_inputs"], dnet.n_rows)
        assert bool((mirror[rows, :631] == own[rows, :631]).all())
    finally:
        assert L.tb_set_peer_wires(ctx._h, None, None, 0) == 0
    dnet.free()


def test_host_buffer_path_matches(tb, ctx, keys):
    A, B = synth.random_bits(9, 90), synth.random_bits(9, 91)
    ca, cb = enc(keys, A, 92), enc(keys, B, 93)
    host = ctx.gates_host(tb.NAND, ca, cb)
    dev = ctx.to_host(ctx.gates(tb.NAND, ctx.to_device(ca, 631), ctx.to_device(cb, 631)))
    assert (host == dev).all() and (host == O.gates(keys, O.NAND, ca, cb)).all()


# ------------------------------------------------------------------------------------- netlists
def run_netlist_gpu(tb, ctx, net_arrays, in_cts):
    net = tb.Netlist(net_arrays["n_inputs"], net_arrays["type"], net_arrays["in0"], net_arrays["in1"],
                     net_arrays["in2"], outputs=net_arrays["outputs"])
    dnet = ctx.upload(net)
    wires = ctx.wire_array(dnet)
    wires[:net.n_inputs, :631] = ctx.to_device(in_cts)[:, :631]
    ctx.run_netlist(dnet, wires)
    allw = ctx.to_host(wires)
    return allw[dnet.row_of_wire]                       # back to original wire ids


def run_netlist_oracle(keys, n, in_cts):
    from oracle.algorithm1 import algorithm1
    w = np.zeros((n["n_inputs"] + len(n["type"]), 631), np.uint32)
    w[:n["n_inputs"]] = in_cts
    for batch in algorithm1(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]):
        b = np.array(batch)
        O.run_level(keys, w, n["type"][b], n["in0"][b], n["in1"][b], n["in2"][b], n["n_inputs"] + b)
    return w


def test_rca_netlist_config2(tb, ctx, keys):
    """BASELINE configs[1]: 8-bit ripple-carry adder, every gate bit-exact, sum decrypts correctly."""
    n = synth.ripple_carry_adder(8)
    a, b = 173, 98
    bits = np.concatenate([synth.pack_bits([a], 8), synth.pack_bits([b], 8)])
    cts = enc(keys, bits, 7)
    gpu = run_netlist_gpu(tb, ctx, n, cts)
    ref = run_netlist_oracle(keys, n, cts)
    assert (gpu == ref).all()
    dec = O.decrypt_bits(keys, gpu[n["outputs"]])
    assert int(synth.unpack_bits(dec, 9)[0]) == a + b


def test_mixed_netlist_with_not_and_mux(tb, ctx, keys):
    """random small DAG with all gate kinds incl. NOT and MUX, gates listed out of order."""
    from test_host import random_dag
    n_in, t, a, b, c = random_dag(11, n_inputs=5, n_gates=24)
    n = dict(n_inputs=n_in, type=t, in0=a, in1=b, in2=c, outputs=np.arange(n_in, n_in + 24))
    bits = synth.random_bits(n_in, 12)
    cts = enc(keys, bits, 13)
    gpu = run_netlist_gpu(tb, ctx, n, cts)
    ref = run_netlist_oracle(keys, n, cts)
    assert (gpu == ref).all()
    plain = simulate(n_in, t, a, b, c, bits)[0]
    assert (O.decrypt_bits(keys, gpu) == plain).all()


@pytest.mark.parametrize("variant", [6, 10, 12, 14, 15])
def test_throughput_level_bench_size_sampled(tb, ctx, keys, variant):
    """BASELINE configs[2] at the bench's per-GPU size (65,536 NAND/XOR gates, one level, the launch
    configuration bench.py times, default br6 and --br-variant 10): all outputs decrypt to the truth; a
    seeded sample of 48 gates is recomputed by the oracle and compared bit for bit."""
    G = 65536
    n = synth.independent_level(G, seed=3)
    bits = synth.random_bits(2 * G, 4)
    cts = enc(keys, bits, 5)
    ctx.set_br_variant(variant)
    try:
        gpu = run_netlist_gpu(tb, ctx, n, cts)
    finally:
        ctx.set_br_variant(6)
    out = gpu[2 * G:]
    truth = ((n["type"].astype(np.int64) >> (2 * bits[0::2].astype(np.int64) + bits[1::2])) & 1).astype(np.uint8)
    assert (O.decrypt_bits(keys, out) == truth).all()
    idx = np.random.default_rng(6).choice(G, 48, replace=False)
    idx = np.concatenate([idx, [0, G - 1]])
    want = O.gates(keys, n["type"][idx], cts[2 * idx], cts[2 * idx + 1])
    assert (out[idx] == want).all()
