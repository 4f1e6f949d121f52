"""Seeded synthetic inputs shared by tests/, bench.py and the oracle calls in them.

This module holds NONE of the method's arithmetic: no torus arithmetic, no encryption, no gate evaluation.
It produces (a) plaintext bits, (b) uniform random words standing in for key material when only timing is
measured (TFHE evaluation is data-oblivious, so timing does not depend on key or ciphertext values),
and (c) gate netlists with the shapes of the paper's workloads:
  cfg 1  NAND truth table           (BASELINE configs[0])
  cfg 2  8-bit ripple-carry adder   (configs[1]; 37 gates, 15 levels)
  cfg 3  one level of G independent NAND/XOR gates (configs[2], the throughput sweep)
  cfg 4  VIP-Bench-shaped 32x32 multiplier / bubble sort of 16 x 16-bit (configs[3])
  cfg 5  ChiselTorch-shaped 8-bit MNIST MLP tile (configs[4])
  f3     self-attention layer shaped like Attention_S / Attention_L
Netlists are returned as plain arrays: (n_inputs, type int32, in0/in1/in2 int64, outputs int64); wire ids
[0, n_inputs) are inputs and n_inputs + g is gate g's output.  Gate codes follow reading C15.
"""
from __future__ import annotations

import numpy as np

NOR, ANDNY, NOT, ANDYN, XOR, NAND, AND, XNOR, ORNY, ORYN, OR, MUX = 1, 2, 3, 4, 6, 7, 8, 9, 11, 13, 14, 16


def rng(seed: int) -> np.random.Generator:
    return np.random.default_rng(np.random.SeedSequence(seed))


def random_bits(n: int, seed: int) -> np.ndarray:
    return rng(seed).integers(0, 2, n, dtype=np.uint8)


def random_words(n: int, seed: int) -> np.ndarray:
    """n uniform u32 words (timing-only stand-in for key material / ciphertext masks)."""
    return rng(seed).integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)


class Builder:
    """Append-only gate-list builder (wire ids as above)."""

    def __init__(self, n_inputs: int):
        self.n_inputs = n_inputs
        self.t, self.a, self.b, self.c = [], [], [], []

    def gate(self, t: int, a: int, b: int = -1, c: int = -1) -> int:
        self.t.append(t)
        self.a.append(a)
        self.b.append(b)
        self.c.append(c)
        return self.n_inputs + len(self.t) - 1

    def arrays(self, outputs):
        return dict(n_inputs=self.n_inputs, type=np.array(self.t, np.int32), in0=np.array(self.a, np.int64),
                    in1=np.array(self.b, np.int64), in2=np.array(self.c, np.int64),
                    outputs=np.array(outputs, np.int64))


def full_adder(B: Builder, a: int, b: int, cin: int):
    x = B.gate(XOR, a, b)
    s = B.gate(XOR, x, cin)
    c1 = B.gate(AND, a, b)
    c2 = B.gate(AND, x, cin)
    return s, B.gate(OR, c1, c2)


def ripple_carry_adder(bits: int = 8):
    """cfg 2: a + b, inputs a[0..bits) then b[0..bits) (LSB first); outputs sum bits then carry.
    Half adder + (bits-1) full adders: 2 + 5 (bits-1) gates (37 for 8 bits)."""
    B = Builder(2 * bits)
    a = list(range(bits))
    b = list(range(bits, 2 * bits))
    s0 = B.gate(XOR, a[0], b[0])
    c = B.gate(AND, a[0], b[0])
    sums = [s0]
    for i in range(1, bits):
        s, c = full_adder(B, a[i], b[i], c)
        sums.append(s)
    return B.arrays(sums + [c])


def independent_level(G: int, seed: int, kinds=(NAND, XOR)):
    """cfg 3: one level of G independent gates, each on two fresh inputs (2G inputs); types drawn
    uniformly from `kinds` (all-NAND, all-XOR or a seeded 50/50 mix)."""
    t = rng(seed).choice(np.array(kinds, np.int32), G)
    return dict(n_inputs=2 * G, type=t.astype(np.int32), in0=np.arange(0, 2 * G, 2, dtype=np.int64),
                in1=np.arange(1, 2 * G, 2, dtype=np.int64), in2=np.full(G, -1, np.int64),
                outputs=np.arange(2 * G, 3 * G, dtype=np.int64))


def array_multiplier(bits: int = 32, full: bool = True):
    """cfg 4a: bits x bits -> 2 bits (full) unsigned array multiplier: AND partial products reduced row by
    row with ripple-carry adders.  Inputs a[0..bits), b[0..bits) LSB first; outputs the product bits."""
    B = Builder(2 * bits)
    a = list(range(bits))
    b = list(range(bits, 2 * bits))
    width = 2 * bits if full else bits
    pp = lambda i, j: B.gate(AND, a[j], b[i])
    acc = [pp(0, j) for j in range(min(bits, width))]          # row 0: bits [0, bits)
    out = [acc[0]]
    acc = acc[1:]
    for i in range(1, bits):
        row = [pp(i, j) for j in range(bits) if i + j < width]   # bits [i, i + bits)
        nxt, carry = [], None
        for k, p in enumerate(row):
            if k < len(acc):
                if carry is None:
                    s = B.gate(XOR, acc[k], p)
                    carry = B.gate(AND, acc[k], p)
                else:
                    s, carry = full_adder(B, acc[k], p, carry)
                    if i + k + 1 >= width:
                        carry = None
                nxt.append(s)
            else:
                if carry is not None:
                    s = B.gate(XOR, p, carry)
                    carry = B.gate(AND, p, carry) if i + k + 1 < width else None
                    nxt.append(s)
                else:
                    nxt.append(p)
        if carry is not None and i + len(row) < width:
            nxt.append(carry)
        out.append(nxt[0])
        acc = nxt[1:]
    out += acc
    return B.arrays(out[:width])


def _less_than(B: Builder, x, y):
    """x < y for unsigned LSB-first bit lists: ripple comparator (ANDNY / XNOR / OR chain)."""
    lt = None
    for i in range(len(x)):
        lt_i = B.gate(ANDNY, x[i], y[i])          # !x & y
        if lt is None:
            lt = lt_i
        else:
            eq = B.gate(XNOR, x[i], y[i])
            lt = B.gate(OR, lt_i, B.gate(AND, eq, lt))
    return lt


def bubble_sort(n: int = 16, bits: int = 16):
    """cfg 4b: bubble sort of n unsigned `bits`-bit words (n(n-1)/2 compare-exchanges, each a ripple
    less-than plus 2*bits MUXes).  Inputs word-major, LSB first; outputs the sorted words ascending."""
    B = Builder(n * bits)
    words = [list(range(w * bits, (w + 1) * bits)) for w in range(n)]
    for i in range(n - 1):
        for j in range(n - 1 - i):
            x, y = words[j], words[j + 1]
            swap = _less_than(B, y, x)                               # y < x -> swap
            lo = [B.gate(MUX, swap, y[k], x[k]) for k in range(bits)]
            hi = [B.gate(MUX, swap, x[k], y[k]) for k in range(bits)]
            words[j], words[j + 1] = lo, hi
    return B.arrays([w for word in words for w in word])


def _add(B: Builder, x, y):
    """ripple add of LSB-first lists, result len max+1"""
    n = max(len(x), len(y))
    out, c = [], None
    for i in range(n):
        xi = x[i] if i < len(x) else None
        yi = y[i] if i < len(y) else None
        if xi is None or yi is None:
            v = xi if yi is None else yi
            if c is None:
                out.append(v)
            else:
                out.append(B.gate(XOR, v, c))
                c = B.gate(AND, v, c)
            continue
        if c is None:
            out.append(B.gate(XOR, xi, yi))
            c = B.gate(AND, xi, yi)
        else:
            s, c = full_adder(B, xi, yi, c)
            out.append(s)
    if c is not None:
        out.append(c)
    return out


def mnist_mlp_tile(n_in: int = 16, n_out: int = 2, bits: int = 8):
    """cfg 5 tile: ChiselTorch-shaped quantised Linear (Fig. 4 P:120-127, 8-bit): n_out dot products of
    n_in encrypted 8-bit unsigned activations with encrypted 8-bit weights (array multipliers + an adder
    tree), then ReLU-free argmax-free logits.  Inputs: activations then weights (n_out x n_in), LSB first.
    The full network of SURVEY 8(d) cfg 5 is this tile scaled up (n_in = 576, n_out = 10)."""
    B = Builder(n_in * bits + n_out * n_in * bits)
    act = [list(range(i * bits, (i + 1) * bits)) for i in range(n_in)]
    base = n_in * bits
    outs = []
    for o in range(n_out):
        prods = []
        for i in range(n_in):
            w = list(range(base + (o * n_in + i) * bits, base + (o * n_in + i + 1) * bits))
            rows = [[B.gate(AND, act[i][k], w[j]) for k in range(bits)] for j in range(bits)]
            acc = rows[0]
            for j in range(1, bits):
                shifted = rows[j]
                low, high = acc[:j], acc[j:]
                acc = low + _add(B, high, shifted)
            prods.append(acc)
        while len(prods) > 1:                      # adder tree
            nxt = [_add(B, prods[k], prods[k + 1]) for k in range(0, len(prods) - 1, 2)]
            if len(prods) % 2:
                nxt.append(prods[-1])
            prods = nxt
        outs += prods[0]
    return B.arrays(outs)


def _relu(B: Builder, x):
    """signed two's-complement x (LSB first, MSB = sign) -> max(x, 0) as unsigned bits[:-1]"""
    s = x[-1]
    return [B.gate(ANDNY, s, xi) for xi in x[:-1]]      # !sign & bit


def _max(B: Builder, x, y):
    lt = _less_than(B, x, y)
    return [B.gate(MUX, lt, y[k], x[k]) for k in range(len(x))]


def mnist_fig4(side: int = 26, bits: int = 8, n_out: int = 10, pool: int = 3):
    """cfg 5: the ChiselTorch MNIST model of Fig. 4 on `side` x `side` encrypted signed `bits`-bit
    activations: ReLU -> MaxPool2d(pool, 1) -> Flatten -> Linear(((side-pool+1)^2), n_out) with encrypted
    unsigned `bits`-bit weights (array multipliers + adder tree).  Fig. 4 declares Float(8,8); BASELINE asks
    for an 8-bit quantised network, so integers are used (SURVEY 8(d) cfg 5).  Inputs: activations (row-major,
    LSB first), then weights [n_out][features].  The default size has ~2.2 M gates."""
    n_act = side * side
    feat_side = side - pool + 1
    n_feat = feat_side * feat_side
    B = Builder(n_act * bits + n_out * n_feat * (bits - 1))
    act = [list(range(i * bits, (i + 1) * bits)) for i in range(n_act)]
    r = [_relu(B, a) for a in act]                                   # bits-1 unsigned bits each
    feats = []
    for y in range(feat_side):
        for x in range(feat_side):
            win = [r[(y + dy) * side + (x + dx)] for dy in range(pool) for dx in range(pool)]
            while len(win) > 1:                                      # max tree
                nxt = [_max(B, win[k], win[k + 1]) for k in range(0, len(win) - 1, 2)]
                if len(win) % 2:
                    nxt.append(win[-1])
                win = nxt
            feats.append(win[0])
    wb = bits - 1
    base = n_act * bits
    outs = []
    for o in range(n_out):
        prods = []
        for i in range(n_feat):
            w = list(range(base + (o * n_feat + i) * wb, base + (o * n_feat + i + 1) * wb))
            rows = [[B.gate(AND, feats[i][k], w[j]) for k in range(len(feats[i]))] for j in range(wb)]
            acc = rows[0]
            for j in range(1, wb):
                acc = acc[:j] + _add(B, acc[j:], rows[j])
            prods.append(acc)
        while len(prods) > 1:
            nxt = [_add(B, prods[k], prods[k + 1]) for k in range(0, len(prods) - 1, 2)]
            if len(prods) % 2:
                nxt.append(prods[-1])
            prods = nxt
        outs += prods[0]
    return B.arrays(outs)


def _mul(B: Builder, x, y):
    """unsigned array multiply of LSB-first lists (AND partial products, ripple rows)"""
    rows = [[B.gate(AND, x[k], y[j]) for k in range(len(x))] for j in range(len(y))]
    acc = rows[0]
    for j in range(1, len(y)):
        acc = acc[:j] + _add(B, acc[j:], rows[j])
    return acc


def _dot(B: Builder, xs, ys):
    """sum_i xs[i] * ys[i] (array multipliers + adder tree)"""
    prods = [_mul(B, x, y) for x, y in zip(xs, ys)]
    while len(prods) > 1:
        nxt = [_add(B, prods[k], prods[k + 1]) for k in range(0, len(prods) - 1, 2)]
        if len(prods) % 2:
            nxt.append(prods[-1])
        prods = nxt
    return prods[0]


def attention(seq: int = 4, hidden: int = 32, bits: int = 4):
    """f3: a self-attention layer shaped like the paper's Attention_S / Attention_L (hidden 32 /
    64), built from Table I primitives (matmul, argmax, +, *) on encrypted `bits`-bit unsigned
    tokens X [seq][hidden] and encrypted weights Wq, Wk, Wv [hidden][hidden]:
        Q, K, V = requant(X Wq), requant(X Wk), requant(X Wv)      requant(z) = top `bits` bits of the
                                                                   (2 bits + ceil(log2 hidden))-bit dot product
        S = Q K^T;  out[i] = V[argmax_j S[i][j]]                   (hard attention: argmax in place of softmax,
                                                                   the first maximum wins)
    The paper gives neither the sequence length nor the number format, so both are parameters.  Inputs: X, then
    Wq, Wk, Wv (row-major, LSB first); outputs out [seq][hidden] (LSB first).  attention_reference() is the same
    function on plaintext integers."""
    w_full = 2 * bits + max(1, (hidden - 1).bit_length())
    n_in = seq * hidden * bits + 3 * hidden * hidden * bits
    B = Builder(n_in)
    word = lambda base, i: list(range(base + i * bits, base + (i + 1) * bits))
    X = [[word(0, t * hidden + h) for h in range(hidden)] for t in range(seq)]
    W = []
    for m in range(3):
        base = seq * hidden * bits + m * hidden * hidden * bits
        W.append([[word(base, r * hidden + c) for c in range(hidden)] for r in range(hidden)])

    def requant(z):
        if len(z) != w_full:
            raise ValueError("dot-product width %d, expected %d (hidden must be a power of two)" % (len(z), w_full))
        return z[w_full - bits:]

    proj = [[[requant(_dot(B, X[t], [W[m][r][c] for r in range(hidden)])) for c in range(hidden)]
             for t in range(seq)] for m in range(3)]
    Q, K, V = proj
    outs = []
    for i in range(seq):
        cands = [(_dot(B, Q[i], K[j]), V[j]) for j in range(seq)]
        while len(cands) > 1:                          # argmax tournament, earlier index wins ties
            nxt = []
            for k in range(0, len(cands) - 1, 2):
                (s1, v1), (s2, v2) = cands[k], cands[k + 1]
                take2 = _less_than(B, s1, s2)                   # all scores have the same width
                s = [B.gate(MUX, take2, s2[b], s1[b]) for b in range(len(s1))]
                v = [[B.gate(MUX, take2, v2[h][b], v1[h][b]) for b in range(bits)] for h in range(hidden)]
                nxt.append((s, v))
            if len(cands) % 2:
                nxt.append(cands[-1])
            cands = nxt
        outs += [b for h in cands[0][1] for b in h]
    return B.arrays(outs)


def attention_reference(x, wq, wk, wv, bits: int):
    """plaintext integers of attention(): x [seq][hidden], w* [hidden][hidden] -> out [seq][hidden]"""
    x, wq, wk, wv = (np.asarray(a, np.int64) for a in (x, wq, wk, wv))
    hidden = x.shape[1]
    w_full = 2 * bits + max(1, (hidden - 1).bit_length())
    rq = lambda z: (z >> (w_full - bits)) & ((1 << bits) - 1)
    q, k, v = rq(x @ wq), rq(x @ wk), rq(x @ wv)
    s = q @ k.T
    return v[np.argmax(s, axis=1)]


def pack_bits(values, bits: int) -> np.ndarray:
    """unsigned ints -> LSB-first bit array"""
    v = np.asarray(values, np.uint64)
    return ((v[:, None] >> np.arange(bits, dtype=np.uint64)) & 1).astype(np.uint8).reshape(-1)


def unpack_bits(b, bits: int) -> np.ndarray:
    b = np.asarray(b, np.uint64).reshape(-1, bits)
    return (b << np.arange(bits, dtype=np.uint64)).sum(axis=1)
