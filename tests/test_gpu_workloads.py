"""End-to-end netlists on the GPU (-m gpu): BASELINE configs[3] (VIP-Bench-shaped 32-bit multiplier,
bubble sort) and configs[4] (ChiselTorch-shaped quantised MNIST Linear tile), plus sharded-level invariance.

Parity at these sizes is (a) the decrypted outputs equal the plaintext function and (b) a seeded sample
of gates is recomputed by the oracle from the GPU's own input wires and compared bit for bit (SURVEY 8(d):
"per-gate local bit-exact parity on a seeded sample").  Whole-netlist oracle runs would take minutes.
"""
import numpy as np
import pytest

import oracle as O
import synth
from oracle.plain import simulate

pytestmark = pytest.mark.gpu


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
    return O.keygen(O.DEFAULT, seed=77)


@pytest.fixture(scope="module")
def ctx(tb, keys):
    c = tb.Context(0)
    c.load_keys(keys.bk, keys.ksk)
    return c


def run(tb, ctx, n, cts):
    net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], outputs=n["outputs"])
    dnet = ctx.upload(net)
    wires = ctx.wire_array(dnet)
    wires[:net.n_inputs, :631] = ctx.to_device(cts)[:, :631]
    ctx.run_netlist(dnet, wires)
    return ctx.to_host(wires)[dnet.row_of_wire], dnet


def sampled_gate_parity(keys, n, w, k, seed):
    """recompute k seeded gates with the oracle from the GPU's own input wires"""
    ng = len(n["type"])
    idx = np.random.default_rng(seed).choice(ng, min(k, ng), replace=False)
    ni = n["n_inputs"]
    t = n["type"][idx]
    a = w[n["in0"][idx]]
    b = w[np.maximum(n["in1"][idx], 0)]
    c = w[np.maximum(n["in2"][idx], 0)]
    want = O.gates(keys, t, a, b, c)
    assert (w[ni + idx] == want).all()
    return idx


def test_multiplier_32bit_config4(tb, ctx, keys):
    n = synth.array_multiplier(32, full=True)
    A, B = 0xDEADBEEF, 0x12345679
    bits = np.concatenate([synth.pack_bits([A], 32), synth.pack_bits([B], 32)])
    w, dnet = run(tb, ctx, n, O.encrypt_bits(keys, bits, 1))
    dec = O.decrypt_bits(keys, w[n["outputs"]])
    assert int(synth.unpack_bits(dec, 64)[0]) == A * B
    plain = simulate(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], bits)[0]
    assert (O.decrypt_bits(keys, w) == plain).all()          # every wire decrypts to its plaintext
    sampled_gate_parity(keys, n, w, 48, 2)


def test_bubble_sort_config4(tb, ctx, keys):
    n = synth.bubble_sort(8, 8)                                 # MUX-heavy, deep and narrow
    vals = np.random.default_rng(3).integers(0, 256, 8)
    bits = synth.pack_bits(vals, 8)
    w, dnet = run(tb, ctx, n, O.encrypt_bits(keys, bits, 4))
    dec = O.decrypt_bits(keys, w[n["outputs"]])
    assert synth.unpack_bits(dec, 8).tolist() == sorted(vals.tolist())
    idx = sampled_gate_parity(keys, n, w, 40, 5)
    assert (n["type"] == O.MUX).any()


def test_mnist_tile_config5(tb, ctx, keys):
    n_in, n_out, bits_w = 8, 2, 8
    n = synth.mnist_mlp_tile(n_in, n_out, bits_w)
    rng = np.random.default_rng(6)
    act, W = rng.integers(0, 256, n_in), rng.integers(0, 256, (n_out, n_in))
    bits = np.concatenate([synth.pack_bits(act, 8), synth.pack_bits(W.reshape(-1), 8)])
    w, dnet = run(tb, ctx, n, O.encrypt_bits(keys, bits, 7))
    dec = O.decrypt_bits(keys, w[n["outputs"]])
    width = len(n["outputs"]) // n_out
    assert synth.unpack_bits(dec, width).tolist() == (W @ act).tolist()
    sampled_gate_parity(keys, n, w, 40, 8)


def test_sharded_levels_are_byte_identical(tb, ctx, keys):
    """virtual ranks on one GPU: every level run as R shards [g0, g1) must give the same bytes as R = 1"""
    n = synth.ripple_carry_adder(8)
    n2 = synth.independent_level(37, 9)
    for net_arrays in (n, n2):
        cts = O.encrypt_bits(keys, synth.random_bits(net_arrays["n_inputs"], 10), 11)
        ref, dnet = run(tb, ctx, net_arrays, cts)
        for R in (2, 3, 8):
            wires = ctx.wire_array(dnet)
            wires[:net_arrays["n_inputs"], :631] = ctx.to_device(cts)[:, :631]
            for L, (row0, ng, _, _) in enumerate(dnet.levels, start=1):
                for r in range(R):
                    g0, g1, _ = tb.parallel.shard(ng, R, r)
                    ctx.run_level(dnet, L, g0, g1, wires)
            got = ctx.to_host(wires)[dnet.row_of_wire]
            assert (got == ref).all(), R


def test_run_netlist_host_matches_device(tb, ctx, keys):
    n = synth.ripple_carry_adder(4)
    cts = O.encrypt_bits(keys, synth.random_bits(n["n_inputs"], 12), 13)
    ref, dnet = run(tb, ctx, n, cts)
    out = ctx.run_netlist_host(dnet, cts, n["outputs"])
    assert (out == ref[n["outputs"]]).all()
    rev = n["outputs"][::-1].copy()                              # non-contiguous rows -> device gather path
    assert (ctx.run_netlist_host(dnet, cts, rev) == ref[rev]).all()
    wide = np.zeros((cts.shape[0], 700), np.uint32)              # host input rows with a wider stride
    wide[:, :631] = cts
    assert (ctx.run_netlist_host(dnet, wide, np.array([0, n["n_inputs"]])) == ref[[0, n["n_inputs"]]]).all()


def test_run_netlist_host_overlap_equals_serial(tb, ctx, keys):
    """tb_run_netlist_host with its copies overlapped with the level loop (inputs in first-use order on one
    stream, each level's outputs copied back on another while the next level runs) gives the same
    bytes as the serial path and as the device path: outputs from every level, inputs passed through, reversed
    order, pinned and pageable host buffers"""
    import torch
    n = synth.array_multiplier(8, full=True)
    cts = O.encrypt_bits(keys, synth.random_bits(n["n_inputs"], 15), 16)
    ref, dnet = run(tb, ctx, n, cts)
    ow = np.arange(dnet.n_rows - 1, -1, -3, dtype=np.int64)          # every third wire, reversed, incl. inputs
    hin = torch.from_numpy(np.ascontiguousarray(cts).view(np.int32)).pin_memory()
    outs = []
    for overlap in (True, False):
        ctx.set_host_overlap(overlap)
        hout = torch.zeros((ow.size, 631), dtype=torch.int32).pin_memory()
        ctx.run_netlist_host_into(dnet, hin, ow, hout)
        outs.append(hout.numpy().view(np.uint32).copy())
        outs.append(ctx.run_netlist_host(dnet, cts, ow))                 # pageable numpy buffers
    ctx.set_host_overlap(True)
    for o in outs:
        assert (o == ref[ow]).all()


def test_run_netlist_host_chunked_wide_level(tb, ctx, keys):
    """tb_run_netlist_host runs a level of more than 8 waves of br6 (a wave = 4 x SM-count gates) as three chunks
    (3 waves, the middle, the rest) whose input copies land, and whose outputs leave, while the neighbouring
    chunks run: a 20,000-gate level followed by gates that read across both chunk boundaries gives the same bytes
    as the device path, overlapped and serial, and the second-level results decrypt to the plaintext"""
    import torch
    G1 = 20000
    W = 4 * torch.cuda.get_device_properties(0).multi_processor_count
    b1 = 3 * W
    b2 = b1 + (G1 - 6 * W) // W * W
    lv = synth.independent_level(G1, 17)
    ni = lv["n_inputs"]
    w = lambda g: ni + g                                            # wire of level-1 gate g
    pairs = [(0, G1 - 1), (b1 - 1, b1), (b2 - 1, b2), (100, b2 + 5), (G1 - 2, 5)]
    t2 = np.array([synth.XOR, synth.XOR, synth.AND, synth.AND, synth.OR], np.int32)
    n = dict(n_inputs=ni, type=np.concatenate([lv["type"], t2]),
             in0=np.concatenate([lv["in0"], [w(a) for a, _ in pairs]]).astype(np.int64),
             in1=np.concatenate([lv["in1"], [w(b) for _, b in pairs]]).astype(np.int64),
             in2=np.full(G1 + len(pairs), -1, np.int64))
    n["outputs"] = np.arange(ni + G1, ni + G1 + len(pairs), dtype=np.int64)
    bits = synth.random_bits(ni, 18)
    cts = O.encrypt_bits(keys, bits, 19)
    ref, dnet = run(tb, ctx, n, cts)
    ow = np.concatenate([n["outputs"], np.arange(ni + G1 - 1, 0, -997)]).astype(np.int64)   # + sampled wires
    for overlap in (True, False):
        ctx.set_host_overlap(overlap)
        try:
            got = ctx.run_netlist_host(dnet, cts, ow)
        finally:
            ctx.set_host_overlap(True)
        assert (got == ref[ow]).all(), overlap
    f = {synth.NAND: lambda a, b: 1 - (a & b), synth.XOR: lambda a, b: a ^ b, synth.AND: lambda a, b: a & b,
         synth.OR: lambda a, b: a | b}
    l1 = np.array([f[int(t)](int(bits[2 * g]), int(bits[2 * g + 1])) for g, t in enumerate(lv["type"])])
    want = [f[int(t)](int(l1[a]), int(l1[b])) for t, (a, b) in zip(t2, pairs)]
    assert O.decrypt_bits(keys, got[:len(pairs)]).tolist() == want


def test_same_wire_twice_and_duplicate_consumers(tb, ctx, keys):
    """XOR(a, a) = 0 and AND(a, a) = a; one wire feeding many gates of a level"""
    n = dict(n_inputs=2, type=np.array([6, 8, 7, 7, 14], np.int32), in0=np.array([0, 0, 0, 1, 2]),
             in1=np.array([0, 0, 1, 0, 3]), in2=np.full(5, -1), outputs=np.arange(2, 7))
    bits = np.array([1, 0], np.uint8)
    cts = O.encrypt_bits(keys, bits, 14)
    w, _ = run(tb, ctx, n, cts)
    ref = run_oracle_levels(keys, n, cts)
    assert (w == ref).all()
    assert O.decrypt_bits(keys, w[2:]).tolist() == [0, 1, 1, 1, 1]


def run_oracle_levels(keys, n, cts):
    from oracle.algorithm1 import algorithm1
    w = np.zeros((n["n_inputs"] + len(n["type"]), 631), np.uint32)
    w[:n["n_inputs"]] = cts
    for batch in algorithm1(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]):
        b = np.array(batch)
        O.run_level(keys, w, n["type"][b], n["in0"][b], n["in1"][b], n["in2"][b], n["n_inputs"] + b)
    return w


def test_errors_without_keys_and_bad_arguments(tb):
    import torch
    c = tb.Context(0)
    x = c.empty(2)
    with pytest.raises(tb.TBError) as e:
        c.gates(tb.NAND, x, x)
    assert e.value.code == -3                                     # TB_ENOKEYS
    with pytest.raises(tb.TBError):
        c.set_br_variant(5)
    with pytest.raises(tb.TBError):
        c.set_ks_tile(12)
    with pytest.raises(ValueError):
        c.gates(tb.NAND, x, x[:, :600])                           # shape mismatch caught in the binding
    c.close()


@pytest.mark.parametrize("fmt", ["yosys", "blif"])
def test_imported_netlist_bit_exact(tb, ctx, keys, fmt):
    """a synthesised gate-level netlist (Yosys JSON / BLIF fixture) imported, run on the GPU for
    all 8 input assignments at once (8 copies side by side), every wire equal to the oracle's, outputs decrypt to
    the full adder"""
    import itertools
    import os
    from oracle.algorithm1 import algorithm1
    from paper_conf_ispass_maxw23_b200 import netlist as NL
    gold = os.path.join(os.path.dirname(__file__), "golden")
    net = (NL.read_yosys_json(open(os.path.join(gold, "full_adder_yosys.json")).read()) if fmt == "yosys"
           else NL.read_blif(open(os.path.join(gold, "full_adder.blif")).read()))
    # 8 disjoint copies of the netlist in one program (copy k uses inputs 3k .. 3k+2)
    k8, ni, ng = 8, net.n_inputs, net.n_gates
    remap = lambda w, k: np.where(w < 0, -1, np.where(w < ni, w + k * ni, k8 * ni + k * ng + (w - ni)))
    n = dict(n_inputs=k8 * ni, type=np.tile(net.type, k8),
             in0=np.concatenate([remap(net.in0, k) for k in range(k8)]),
             in1=np.concatenate([remap(net.in1, k) for k in range(k8)]),
             in2=np.concatenate([remap(net.in2, k) for k in range(k8)]),
             outputs=np.concatenate([remap(net.outputs, k) for k in range(k8)]))
    bits = np.array(list(itertools.product((0, 1), repeat=3)), np.uint8).reshape(-1)
    cts = O.encrypt_bits(keys, bits, 31)
    w, _ = run(tb, ctx, n, cts)
    ref = np.zeros_like(w)
    ref[:n["n_inputs"]] = cts
    for batch in algorithm1(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]):
        b = np.array(batch)
        O.run_level(keys, ref, n["type"][b], n["in0"][b], n["in1"][b], n["in2"][b], n["n_inputs"] + b)
    assert (w == ref).all()
    dec = O.decrypt_bits(keys, w[n["outputs"]]).reshape(k8, -1)
    plain = simulate(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], bits)[0][n["outputs"]].reshape(k8, -1)
    assert (dec == plain).all()
    a, b_, c = bits.reshape(k8, 3).T.astype(int)
    assert (dec[:, 0] == (a ^ b_ ^ c)).all() and (dec[:, 1] == ((a & b_) | (c & (a ^ b_)))).all()


def test_attention_f3(tb, ctx, keys):
    """a small Attention layer (seq 2, hidden 4, 3-bit; 5,866 gates incl. 40 MUX) on the GPU:
    outputs decrypt to the plaintext hard self-attention, 64 seeded gates bit-exact vs the oracle"""
    seq, hidden, bits = 2, 4, 3
    n = synth.attention(seq, hidden, bits)
    rng = np.random.default_rng(12)
    x, wq, wk, wv = rng.integers(0, 8, (seq, hidden)), *(rng.integers(0, 8, (hidden, hidden)) for _ in range(3))
    pbits = np.concatenate([synth.pack_bits(a.reshape(-1), bits) for a in (x, wq, wk, wv)])
    cts = O.encrypt_bits(keys, pbits, 13)
    w, _ = run(tb, ctx, n, cts)
    dec = O.decrypt_bits(keys, w[n["outputs"]])
    assert (synth.unpack_bits(dec, bits).reshape(seq, hidden) == synth.attention_reference(x, wq, wk, wv, bits)).all()
    sampled_gate_parity(keys, n, w, 64, 14)
