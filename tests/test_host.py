"""Host-side logic and the C-ABI boundary, without a GPU (-m "not gpu").

  * libtfhe_b200.so loads and exports every function include/tfhe_b200.h declares
  * without a usable sm_100 device the product fails loudly (no CPU fallback)
  * native Algorithm-1 levelisation == the oracle's literal Algorithm 1
  * the PyTFHE binary reader/writer on the paper's Fig. 6 half adder
  * the synthetic workload generators compute what they claim (plaintext simulation)
"""
import os
import re

import numpy as np
import pytest

import synth
from oracle.algorithm1 import algorithm1
from oracle.plain import simulate

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def tb():
    import paper_conf_ispass_maxw23_b200 as tb
    tb.build()
    return tb


def header_functions():
    src = open(os.path.join(ROOT, "include", "tfhe_b200.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(tb_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_header_symbol(tb):
    from paper_conf_ispass_maxw23_b200 import _native
    L = _native.lib()
    names = header_functions()
    assert len(names) >= 20
    for n in names:
        assert hasattr(L, n), n
        assert n in _native.SIGNATURES, "binding misses %s" % n
    assert set(_native.SIGNATURES) == set(names)
    assert b"sm_100a" in L.tb_version()


def test_library_is_sm100a_code(tb):
    so = tb._native.SO_PATH
    out = os.popen("/usr/local/cuda/bin/cuobjdump -lelf %s" % so).read()
    assert "sm_100a" in out


def test_no_device_fails_loudly(tb):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(tb.TBError):
        tb.Context(0)


def test_default_params_and_errors(tb):
    from paper_conf_ispass_maxw23_b200 import _native
    import ctypes
    L = _native.lib()
    p = L.tb_default_params()
    assert (p.n, p.N, p.k, p.l, p.Bgbit, p.ks_t, p.ks_basebit) == (630, 1024, 1, 3, 7, 8, 2)
    p.n = 500
    h = ctypes.c_void_p()
    assert L.tb_ctx_create(ctypes.byref(p), 0, ctypes.byref(h)) == _native.TB_EUNSUPPORTED
    assert b"n=630" in L.tb_last_error()
    assert L.tb_gates(None, 7, None, None, None, None, 1, 631, None) == _native.TB_EINVAL


# ------------------------------------------------------------------------------------- Algorithm 1
def random_dag(seed, n_inputs=6, n_gates=60, shuffle=True):
    rng = np.random.default_rng(seed)
    kinds = np.array([1, 2, 3, 4, 6, 7, 8, 9, 11, 13, 14, 16], np.int32)
    t = rng.choice(kinds, n_gates).astype(np.int32)
    in0, in1, in2 = [], [], []
    for g in range(n_gates):
        hi = n_inputs + g
        in0.append(rng.integers(0, hi))
        in1.append(rng.integers(0, hi) if t[g] != 3 else -1)
        in2.append(rng.integers(0, hi) if t[g] == 16 else -1)
    in0, in1, in2 = (np.array(x, np.int64) for x in (in0, in1, in2))
    if shuffle:         # gates listed out of topological order (C15: order not assumed)
        perm = rng.permutation(n_gates)
        inv = np.argsort(perm)
        remap = lambda w: np.where(w >= n_inputs, n_inputs + inv[np.maximum(w - n_inputs, 0)], w)
        t, in0, in1, in2 = t[perm], remap(in0[perm]), np.where(in1[perm] < 0, -1, remap(in1[perm])), \
            np.where(in2[perm] < 0, -1, remap(in2[perm]))
    return n_inputs, t, in0, in1, in2


@pytest.mark.parametrize("seed", range(8))
def test_native_levelise_matches_algorithm1(tb, seed):
    n_in, t, a, b, c = random_dag(seed)
    net = tb.Netlist(n_in, t, a, b, c)
    lv, nl = net.levels()
    batches = algorithm1(n_in, t, a, b, c)
    assert nl == len(batches)
    for L, batch in enumerate(batches, start=1):
        assert sorted(np.nonzero(lv == L)[0].tolist()) == batch


def test_levelise_workload_shapes(tb):
    n = synth.ripple_carry_adder(8)
    lv, nl = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]).levels()
    assert (len(n["type"]), nl) == (37, 15)           # SURVEY 8(d) cfg 2
    n = synth.independent_level(1000, 1)
    assert tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]).levels()[1] == 1


def test_levelise_rejects_cycles_and_bad_wires(tb):
    net = tb.Netlist(2, [7, 7], [0, 3], [2, 1])       # gate 0 reads gate 1, gate 1 reads gate 0
    with pytest.raises(tb.TBError):
        net.levels()
    with pytest.raises(tb.TBError):
        tb.Netlist(2, [7], [0], [9]).levels()
    with pytest.raises(tb.TBError):
        tb.Netlist(2, [5], [0], [1]).levels()          # 0101 is not one of the 11 gates (C10)


# ------------------------------------------------------------------------------------- binary format
def golden_half_adder():
    rows = [l.split() for l in open(os.path.join(ROOT, "tests", "golden", "half_adder_fig6.txt"))
            if l.strip() and not l.startswith("#")]
    data = b""
    for in0, in1, t, full in rows:
        v = int(full, 16)
        assert v == (int(in0, 16) << 66) | (int(in1, 16) << 4) | int(t, 16)
        data += v.to_bytes(16, "little")
    return data


def test_fig6_half_adder_decodes(tb):
    net = tb.read_pytfhe_binary(golden_half_adder())
    assert net.n_inputs == 2 and net.n_gates == 2
    assert net.type.tolist() == [tb.XOR, tb.AND] and tb.XOR == 0b0110
    assert net.in0.tolist() == [0, 0] and net.in1.tolist() == [1, 1]   # indices 1, 2 -> wires 0, 1
    assert net.outputs.tolist() == [2, 3]                               # gates 3, 4 -> wires 2, 3
    x = np.array([[0, 0], [0, 1], [1, 0], [1, 1]], np.uint8)
    w = simulate(net.n_inputs, net.type, net.in0, net.in1, net.in2, x)
    assert w[:, net.outputs].tolist() == [[0, 0], [1, 0], [1, 0], [0, 1]]  # (sum, carry)


def test_fig6_round_trip(tb):
    data = golden_half_adder()
    assert tb.write_pytfhe_binary(tb.read_pytfhe_binary(data)) == data


def test_binary_round_trip_random(tb):
    n_in, t, a, b, c = random_dag(3, shuffle=True)
    keep = t != 16
    # drop MUX (not encodable) by rebuilding a netlist without them
    net = tb.Netlist(4, [7, 6, 3, 14], [0, 4, 5, 6], [1, 2, -1, 3], outputs=[7, 5])
    back = tb.read_pytfhe_binary(tb.write_pytfhe_binary(net))
    assert back.type.tolist() == net.type.tolist() and back.in0.tolist() == net.in0.tolist()
    assert back.in1.tolist() == net.in1.tolist() and back.outputs.tolist() == net.outputs.tolist()
    with pytest.raises(ValueError):
        tb.write_pytfhe_binary(tb.Netlist(3, [16], [0], [1], [2]))


# ------------------------------------------------------------------------------------- generators
def _eval(n, x):
    return simulate(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], x)[:, n["outputs"]]


def test_rca_adds():
    n = synth.ripple_carry_adder(8)
    rng = np.random.default_rng(1)
    A, B = rng.integers(0, 256, 40), rng.integers(0, 256, 40)
    x = np.concatenate([synth.pack_bits(A, 8).reshape(40, 8), synth.pack_bits(B, 8).reshape(40, 8)], 1)
    assert (synth.unpack_bits(_eval(n, x), 9) == A + B).all()


@pytest.mark.parametrize("bits,full", [(8, True), (8, False), (12, True)])
def test_multiplier_multiplies(bits, full):
    n = synth.array_multiplier(bits, full)
    rng = np.random.default_rng(bits)
    A, B = rng.integers(0, 1 << bits, 30), rng.integers(0, 1 << bits, 30)
    x = np.concatenate([synth.pack_bits(A, bits).reshape(30, bits), synth.pack_bits(B, bits).reshape(30, bits)], 1)
    w = 2 * bits if full else bits
    assert (synth.unpack_bits(_eval(n, x), w) == (A * B) % (1 << w)).all()


def test_bubble_sort_sorts():
    n = synth.bubble_sort(5, 6)
    rng = np.random.default_rng(2)
    v = rng.integers(0, 64, (10, 5))
    x = np.stack([synth.pack_bits(r, 6) for r in v])
    got = synth.unpack_bits(_eval(n, x), 6).reshape(10, 5)
    assert (got == np.sort(v, axis=1)).all()


def test_mnist_tile_dot_products():
    n = synth.mnist_mlp_tile(n_in=3, n_out=2, bits=4)
    rng = np.random.default_rng(3)
    act, W = rng.integers(0, 16, (6, 3)), rng.integers(0, 16, (6, 2, 3))
    x = np.stack([np.concatenate([synth.pack_bits(a, 4), synth.pack_bits(w.reshape(-1), 4)]) for a, w in zip(act, W)])
    out = _eval(n, x)
    width = out.shape[1] // 2
    got = synth.unpack_bits(out, width).reshape(6, 2)
    assert (got == np.einsum("bi,boi->bo", act, W)).all()


def test_mnist_fig4_network_computes_relu_maxpool_linear():
    n = synth.mnist_fig4(side=5, bits=4, n_out=2, pool=3)
    rng = np.random.default_rng(4)
    for _ in range(4):
        act, W = rng.integers(-8, 8, 25), rng.integers(0, 8, (2, 9))
        x = np.concatenate([synth.pack_bits(act & 15, 4), synth.pack_bits(W.reshape(-1), 3)])
        out = _eval(n, x[None])[0]
        r = np.maximum(act, 0).reshape(5, 5)
        f = np.array([r[y:y + 3, c:c + 3].max() for y in range(3) for c in range(3)])
        assert synth.unpack_bits(out, len(out) // 2).tolist() == (W @ f).tolist()


def test_mnist_fig4_full_size_shape(tb):
    """SURVEY 8(d) cfg 5: ~2 M gates, ~130 levels, >90 % of gates in levels >= 8192 wide"""
    n = synth.mnist_fig4()
    lv, nl = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]).levels()
    w = np.bincount(lv)[1:]
    assert 1_500_000 < len(n["type"]) < 3_000_000 and 100 < nl < 160
    assert w[w >= 8192].sum() / w.sum() > 0.9


@pytest.mark.parametrize("seq,hidden,bits", [(3, 4, 3), (2, 8, 2), (4, 2, 3)])
def test_attention_computes_hard_self_attention(seq, hidden, bits):
    """the gate-level Attention layer equals its plaintext integer definition (requantised
    projections, Q K^T, first-maximum argmax, V row select), on random tokens/weights and on tie cases"""
    n = synth.attention(seq, hidden, bits)
    rng = np.random.default_rng(seq * 100 + hidden)
    cases = [tuple(rng.integers(0, 1 << bits, sh) for sh in [(seq, hidden)] + [(hidden, hidden)] * 3) for _ in range(5)]
    z = np.zeros((hidden, hidden), np.int64)
    cases.append((rng.integers(0, 1 << bits, (seq, hidden)), z, z, rng.integers(0, 1 << bits, (hidden, hidden))))
    for x, wq, wk, wv in cases:                       # the last case: all scores 0, so argmax = 0 everywhere
        bitsv = np.concatenate([synth.pack_bits(a.reshape(-1), bits) for a in (x, wq, wk, wv)])
        got = synth.unpack_bits(_eval(n, bitsv[None])[0], bits).reshape(seq, hidden)
        assert (got == synth.attention_reference(x, wq, wk, wv, bits)).all()


def test_attention_paper_sizes(tb):
    """Attention_S / Attention_L shapes (hidden 32 / 64) at seq 4, 4-bit: ~1.3 M / ~5.3 M gates"""
    for hidden, lo, hi in ((32, 1_000_000, 2_000_000), (64, 4_000_000, 7_000_000)):
        n = synth.attention(4, hidden, 4)
        assert lo < len(n["type"]) < hi
        assert len(n["outputs"]) == 4 * hidden * 4


def test_independent_level_shape():
    n = synth.independent_level(64, 5)
    assert n["n_inputs"] == 128 and set(np.unique(n["type"]).tolist()) <= {6, 7}
    assert len(set(n["in0"].tolist()) | set(n["in1"].tolist())) == 128


# ------------------------------------------------------------------- f1: capacity-aware level schedule
def _sched(net, cap):
    levels, rows = net.plan(cap)
    lv = np.zeros(net.n_gates, np.int64)
    for L, (row0, cnt) in enumerate(levels, 1):
        g = np.where((rows[net.n_inputs:] >= row0) & (rows[net.n_inputs:] < row0 + cnt))[0]
        lv[g] = L
    return levels, rows, lv


@pytest.mark.parametrize("shape", ["mul", "sort", "rca", "random"])
def test_capacity_schedule_is_valid_and_keeps_depth(tb, shape):
    """same number of levels as Algorithm 1, every gate after all its inputs, and a level that
    exceeds the capacity holds only gates at their deadline (latest level that keeps the depth)"""
    if shape == "random":
        r = np.random.default_rng(9)
        n_in, ng = 20, 600
        t = r.choice([1, 3, 6, 7, 8, 16], ng).astype(np.int32)
        a = np.array([r.integers(0, n_in + g) for g in range(ng)])
        b = np.array([r.integers(0, n_in + g) for g in range(ng)])
        c = np.where(t == 16, [r.integers(0, n_in + g) for g in range(ng)], -1)
        n = dict(n_inputs=n_in, type=t, in0=a, in1=np.where(t == 3, -1, b), in2=c, outputs=np.arange(ng) + n_in)
    else:
        n = {"mul": lambda: synth.array_multiplier(12), "sort": lambda: synth.bubble_sort(8, 6),
             "rca": lambda: synth.ripple_carry_adder(8)}[shape]()
    net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], outputs=n["outputs"])
    asap, depth = net.levels()
    cap = 8
    levels, rows, lv = _sched(net, cap)
    assert len(levels) == depth
    ni = net.n_inputs
    lvl_of = lambda w: 0 if w < ni else lv[w - ni]
    for g in range(net.n_gates):
        ins = [net.in0[g]] + ([net.in1[g]] if net.type[g] != 3 else []) + ([net.in2[g]] if net.type[g] == 16 else [])
        assert all(lvl_of(w) < lv[g] for w in ins), g
    assert (lv >= asap).all()
    # deadlines: ALAP by a reverse sweep
    alap = np.full(net.n_gates, depth)
    for g in np.argsort(-asap, kind="stable"):
        for w in [net.in0[g], net.in1[g], net.in2[g]]:
            if w >= ni and (w != net.in1[g] or net.type[g] != 3) and (w != net.in2[g] or net.type[g] == 16):
                alap[w - ni] = min(alap[w - ni], alap[g] - 1)
    assert (lv <= alap).all()
    lanes = np.where(net.type == 16, 2, np.where(net.type == 3, 0, 1))
    for L in range(1, depth + 1):
        m = lv == L
        if lanes[m].sum() > cap:
            assert (alap[m] == L).all(), L
    # the schedule is only an order: the plaintext function is unchanged
    bits = np.random.default_rng(1).integers(0, 2, (3, ni)).astype(np.uint8)
    want = simulate(ni, net.type, net.in0, net.in1, net.in2, bits)
    order = np.argsort(lv, kind="stable")
    inv = np.empty_like(order)
    inv[order] = np.arange(order.size)
    remap = lambda w: np.where(w < ni, w, ni + inv[np.maximum(w - ni, 0)])
    got = simulate(ni, net.type[order], remap(net.in0[order]), np.where(net.in1[order] < 0, -1, remap(net.in1[order])),
                   np.where(net.in2[order] < 0, -1, remap(net.in2[order])), bits)
    assert (got[:, ni:][:, inv] == want[:, ni:]).all()


def test_capacity_schedule_narrows_vip_levels(tb):
    """on the VIP-shaped bubble sort, fewer levels exceed one latency-kernel wave (32 bootstraps)"""
    n = synth.bubble_sort(16, 16)
    net = tb.Netlist(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"], outputs=n["outputs"])
    lanes = np.where(net.type == 16, 2, np.where(net.type == 3, 0, 1))
    over = []
    for cap in (0, 32):
        _, _, lv = _sched(net, cap)
        per = np.bincount(lv, weights=lanes)[1:]
        over.append(int((per > 32).sum()))
    assert over[1] < over[0] // 2, over
