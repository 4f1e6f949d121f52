"""Pins for the CPU oracle (oracle/), checked against what the mathematics and the paper fix -- never
against the oracle itself and never against the CUDA path.

Each pin is chosen so a plausible mistake (dropped term, wrong sign, wrong index, transposed operand,
wrong rounding) in the step it covers fails it:
  * negacyclic product      -- brute-force full product reduced mod X^N + 1 (Python ints)
  * X^a rotation            -- the negacyclic product with a monomial
  * mod switch (a2, C5)     -- tfhe-lib's 64-bit interval formula, exact rationals
  * decomposition (a4.1,C4) -- uniqueness: digits in [-64,63] and x - Recon(x) in [0, 2^11)
  * external product (a4)   -- zero-noise closed form phase(C [x] TGSW(mu)) = mu * phase(Recon(C))
  * key switch (a6, C9)     -- zero-noise closed form phase(KS(c)) = b - sum s'_i round16(a_i)
  * bootstrap (a2-a6, C6)   -- trivial input (0, phi) -> (0, +-mu) exactly, at the real parameters
  * blind rotation (a2-a5)  -- structured zero-noise key: phase = +-mu by the sign rule, exactly
  * gates (a1, a7)          -- truth tables after decryption, toy and real parameters
  * decryption (C11)        -- exact phase-0 / int32 sign-edge ciphertexts built from the secret
  * level executor          -- ripple-carry adder through or_level_batch: decrypted sum == a + b
  * noise                   -- [7]'s variance bounds for BR (256 bootstraps) and KS at the real parameters
Phases in these tests are computed in plain Python (brute force) so the check does not route through
the oracle's own phase function.
"""
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle as O
import synth

M32 = 1 << 32
MU = 1 << 29


# ---------------------------------------------------------------- independent Python helpers
def py_negacyclic(d, b):
    """full product then reduction by X^N = -1, mod 2^32 (the definition)."""
    N = len(b)
    full = [0] * (2 * N)
    for i in range(N):
        for j in range(N):
            full[i + j] += int(d[i]) * int(b[j])
    return [(full[c] - full[c + N]) % M32 for c in range(N)]


def py_trlwe_phase(S, trlwe):
    N = len(S)
    a, b = [int(x) for x in trlwe[:N]], [int(x) for x in trlwe[N:]]
    aS = py_negacyclic(S, a)
    return [(b[c] - aS[c]) % M32 for c in range(N)]


def py_lwe_phase(s, ct):
    n = len(s)
    return (int(ct[n]) - sum(int(ct[i]) * int(s[i]) for i in range(n))) % M32


def signed(x):
    x %= M32
    return x - M32 if x >= 1 << 31 else x


def py_recon(x, Bgbit=7, l=3):
    """the unique value in (2^(32-l*Bgbit)) Z that the l signed digits in [-Bg/2, Bg/2) reconstruct:
    x rounded down to a multiple of 2^(32 - l Bgbit) (truncating reading C4)."""
    q = 1 << (32 - l * Bgbit)
    return (x - x % q) % M32


# ---------------------------------------------------------------- negacyclic product
@pytest.mark.parametrize("N", [4, 8, 16])
def test_negacyclic_matches_bruteforce(N):
    rng = random.Random(N)
    for _ in range(20):
        d = [rng.randint(-64, 63) for _ in range(N)]
        b = [rng.getrandbits(32) for _ in range(N)]
        acc0 = [rng.getrandbits(32) for _ in range(N)]
        got = O.negacyclic_muladd(np.array(d, np.int32), np.array(b, np.uint32), np.array(acc0, np.uint32))
        want = [(x + y) % M32 for x, y in zip(acc0, py_negacyclic(d, b))]
        assert got.tolist() == want


def test_negacyclic_worst_case_and_identity():
    N = 16
    b = np.full(N, 0xFFFFFFFF, np.uint32)
    d = np.full(N, -64, np.int32)
    assert O.negacyclic_muladd(d, b).tolist() == py_negacyclic(d.tolist(), b.tolist())
    one = np.zeros(N, np.int32)
    one[0] = 1
    r = np.arange(N, dtype=np.uint32) * 977
    assert O.negacyclic_muladd(one, r).tolist() == r.tolist()


@pytest.mark.parametrize("N", [8, 64])
def test_mul_xai_is_product_with_monomial(N):
    rng = random.Random(7)
    src = [rng.getrandbits(32) for _ in range(N)]
    for a in range(2 * N):
        mono = [0] * N
        if a < N:
            mono[a] = 1
        else:
            mono[a - N] = -1            # X^a = -X^(a-N)
        assert O.poly_mul_xai(a, np.array(src, np.uint32)).tolist() == py_negacyclic(mono, src)


# ---------------------------------------------------------------- mod switch (a2, C5)
def tfhelib_modswitch(phase, Msize):
    """tfhe-lib modSwitchFromTorus32 (EXT[10]) with 64-bit unsigned wrap, in exact integers."""
    interv = ((1 << 63) // Msize) * 2
    half = interv // 2
    phase64 = ((phase << 32) + half) % (1 << 64)
    return phase64 // interv


def test_mod_switch_matches_interval_formula():
    rng = random.Random(3)
    two_N = 2048
    vals = [0, 1, (1 << 20) - 1, 1 << 20, (1 << 20) + 1, (1 << 21) - 1, 1 << 21, (1 << 31) - 1, 1 << 31,
            M32 - (1 << 20) - 1, M32 - (1 << 20), M32 - 1] + [rng.getrandbits(32) for _ in range(100000)]
    for v in vals:
        assert O.mod_switch(v, two_N) == tfhelib_modswitch(v, two_N) % two_N, v


def test_mod_switch_is_round_half_up():
    # round(a * 2N / 2^32) mod 2N with ties up, in exact rationals (C5)
    for v in [0, (1 << 20) - 1, 1 << 20, 3 << 20, 5 << 20, M32 - 1, 123456789]:
        x = Fraction(v * 2048, M32)
        want = int(x + Fraction(1, 2)) % 2048
        assert O.mod_switch(v, 2048) == want
    assert O.mod_switch(1 << 20, 2048) == 1 and O.mod_switch((1 << 20) - 1, 2048) == 0


# ---------------------------------------------------------------- decomposition (a4.1, C4)
def test_decomposition_is_the_unique_balanced_truncation():
    P = O.DEFAULT
    rng = random.Random(11)
    edge = [0, 1, 2047, 2048, (1 << 31) - 1, 1 << 31, M32 - 1, 0x81020000, 0x7EFE0000, 0x7EFDFFFF]
    xs = edge + [rng.getrandbits(32) for _ in range(1024 - len(edge))]
    dig = O.decompose(P, np.array(xs, np.uint32))
    assert dig.min() >= -64 and dig.max() <= 63
    h = [1 << 25, 1 << 18, 1 << 11]
    for c, x in enumerate(xs):
        rec = sum(int(dig[j, c]) * h[j] for j in range(3)) % M32
        assert rec == py_recon(x), x
        assert (x - rec) % M32 < 2048
    assert O.decompose(P, np.zeros(1024, np.uint32)).tolist() == np.zeros((3, 1024), int).tolist()


# ---------------------------------------------------------------- TRLWE / TGSW (keygen pins)
def test_trlwe_encrypt_phase_is_message_plus_small_noise():
    N = 64
    rng = np.random.default_rng(1)
    S = rng.integers(0, 2, N).astype(np.int32)
    mu = rng.integers(0, M32, N, dtype=np.uint64).astype(np.uint32)
    ct = O.trlwe_encrypt(S, seed=9, sigma=0.0, mu=mu)
    assert py_trlwe_phase(S.tolist(), ct.tolist()) == mu.tolist()          # exact at sigma = 0
    ct = O.trlwe_encrypt(S, seed=9, sigma=2.0 ** -25, mu=mu)
    err = [signed(p - int(m)) for p, m in zip(py_trlwe_phase(S.tolist(), ct.tolist()), mu)]
    assert max(abs(e) for e in err) < 6 * 2 ** 7                              # 6 sigma at 2^-25


def tgsw_rows(params, s_i, S, seed):
    p1 = O.Params(**{**params.__dict__, "n": 1})
    bk = np.zeros(p1.bk_words, np.uint32)
    O.lib().or_make_bk(__import__("ctypes").byref(p1.c()), seed, np.array([s_i], np.int32), S, bk)
    return bk.reshape(2 * params.l, 2, params.N)


def test_tgsw_rows_carry_mu_times_gadget():
    params = O.Params(n=1, N=32, sigma_bk=0.0)
    S = np.random.default_rng(2).integers(0, 2, 32).astype(np.int32)
    rows = tgsw_rows(params, 1, S, seed=4)
    h = [1 << 25, 1 << 18, 1 << 11]
    for bloc in range(2):
        for j in range(3):
            ph = py_trlwe_phase(S.tolist(), rows[bloc * 3 + j].reshape(-1).tolist())
            if bloc == 1:   # message on b: phase = mu h_j (constant poly)
                want = [h[j]] + [0] * 31
            else:           # message on a: phase = -mu h_j S
                want = [(-h[j] * int(S[c])) % M32 for c in range(32)]
            assert ph == want


@pytest.mark.parametrize("mu_bit", [0, 1])
def test_external_product_zero_noise_closed_form(mu_bit):
    params = O.Params(n=1, N=32, sigma_bk=0.0)
    rng = np.random.default_rng(5 + mu_bit)
    S = rng.integers(0, 2, 32).astype(np.int32)
    tg = tgsw_rows(params, mu_bit, S, seed=6)
    for _ in range(5):
        C = rng.integers(0, M32, 64, dtype=np.uint64).astype(np.uint32)
        out = O.external_product(params, tg, C)
        recon = [py_recon(int(x)) for x in C]
        want = [(mu_bit * p) % M32 for p in py_trlwe_phase(S.tolist(), recon)]
        assert py_trlwe_phase(S.tolist(), out.tolist()) == want


def test_cmux_with_abar_zero_is_identity():
    params = O.Params(n=1, N=32)
    rng = np.random.default_rng(8)
    S = rng.integers(0, 2, 32).astype(np.int32)
    tg = tgsw_rows(params, 1, S, seed=3)
    acc = rng.integers(0, M32, 64, dtype=np.uint64).astype(np.uint32)
    assert O.cmux_step(params, tg, 0, acc).tolist() == acc.tolist()        # C7: skipping is exact


# ---------------------------------------------------------------- key switch (a6, C9)
def test_keyswitch_zero_noise_closed_form():
    params = O.Params(n=16, N=64, sigma_ks=0.0)
    keys = O.keygen(params, seed=12, with_bk=False)
    rng = random.Random(4)
    for _ in range(20):
        ext = np.array([rng.getrandbits(32) for _ in range(65)], np.uint32)
        out = O.keyswitch(keys, ext)
        r16 = [((int(a) + (1 << 15)) % M32) & ~0xFFFF for a in ext[:64]]
        want = (int(ext[64]) - sum(r * int(keys.S[i]) for i, r in enumerate(r16))) % M32
        assert py_lwe_phase(keys.s.tolist(), out.tolist()) == want


def test_sample_extract_phase_equals_coefficient_zero():
    params = O.Params(n=1, N=32)
    rng = np.random.default_rng(13)
    S = rng.integers(0, 2, 32).astype(np.int32)
    acc = rng.integers(0, M32, 64, dtype=np.uint64).astype(np.uint32)
    ext = O.sample_extract(params, acc)
    assert py_lwe_phase(S.tolist(), ext.tolist()) == py_trlwe_phase(S.tolist(), acc.tolist())[0]


# ---------------------------------------------------------------- bootstrapping closed forms
@pytest.fixture(scope="module")
def real_keys():
    return O.keygen(O.DEFAULT, seed=2024)


def test_trivial_input_bootstrap_exact_real_params(real_keys):
    n = O.DEFAULT.n
    for phi in [0, 1, (1 << 20) - 1, 1 << 20, (1 << 29), (1 << 31) - (1 << 20) - 1, (1 << 31) - (1 << 20),
                1 << 31, M32 - (1 << 20) - 1, M32 - (1 << 20), M32 - 1, 0x9E3779B9]:
        ct = np.zeros(n + 1, np.uint32)
        ct[n] = phi
        ext = O.bootstrap_wo_ks(real_keys, ct)
        bbar = ((phi + (1 << 20)) % M32) >> 21
        want_b = MU if bbar < 1024 else M32 - MU
        assert ext[:1024].tolist() == [0] * 1024 and int(ext[1024]) == want_b, hex(phi)
        out = O.keyswitch(real_keys, ext)
        assert out[:n].tolist() == [0] * n and int(out[n]) == want_b


def sign_rule(params, s, ct):
    """C6: +mu iff phibar = (bbar - sum abar_i s_i) mod 2N lies in [0, N)."""
    two_N = 2 * params.N
    ms = lambda v: O.mod_switch(int(v), two_N)
    phibar = (ms(ct[params.n]) - sum(ms(ct[i]) * int(s[i]) for i in range(params.n))) % two_N
    return MU if phibar < params.N else M32 - MU


def test_structured_key_blind_rotation_exact_toy():
    params = O.Params(n=12, N=64, sigma_bk=0.0, bk_mask_mult=1 << 11)
    keys = O.keygen(params, seed=77, with_ksk=False)
    rng = random.Random(1)
    for _ in range(40):
        ct = np.array([rng.getrandbits(32) for _ in range(13)], np.uint32)
        ext = O.bootstrap_wo_ks(keys, ct)
        assert py_lwe_phase(keys.S.tolist(), ext.tolist()) == sign_rule(params, keys.s, ct)


@pytest.mark.slow
def test_structured_key_blind_rotation_exact_real_params():
    params = O.Params(sigma_bk=0.0, bk_mask_mult=1 << 11)
    keys = O.keygen(params, seed=78, with_ksk=False)
    rng = random.Random(2)
    for _ in range(2):
        ct = np.array([rng.getrandbits(32) for _ in range(631)], np.uint32)
        ext = O.bootstrap_wo_ks(keys, ct)
        assert py_lwe_phase(keys.S.tolist(), ext.tolist()) == sign_rule(params, keys.s, ct)


# ---------------------------------------------------------------- gates (P:46 correctness)
def truth(g, a, b):
    return (g >> (2 * a + b)) & 1


def test_all_gate_truth_tables_toy():
    keys = O.keygen(O.TOY, seed=31)
    A = np.array([0, 0, 1, 1] * 3, np.uint8)
    B = np.array([0, 1, 0, 1] * 3, np.uint8)
    ca, cb = O.encrypt_bits(keys, A, 1), O.encrypt_bits(keys, B, 2)
    for g in O.TWO_INPUT:
        got = O.decrypt_bits(keys, O.gates(keys, g, ca, cb))
        assert got.tolist() == [truth(g, a, b) for a, b in zip(A, B)], O.GATE_NAMES[g]
    assert O.decrypt_bits(keys, O.gates(keys, O.NOT, ca)).tolist() == [1 - a for a in A]
    A8 = np.array([(i >> 2) & 1 for i in range(8)], np.uint8)
    B8 = np.array([(i >> 1) & 1 for i in range(8)], np.uint8)
    C8 = np.array([i & 1 for i in range(8)], np.uint8)
    out = O.gates(keys, O.MUX, O.encrypt_bits(keys, A8, 3), O.encrypt_bits(keys, B8, 4), O.encrypt_bits(keys, C8, 5))
    assert O.decrypt_bits(keys, out).tolist() == [b if a else c for a, b, c in zip(A8, B8, C8)]


def test_nand_truth_table_real_params(real_keys):
    A, B = np.array([0, 0, 1, 1], np.uint8), np.array([0, 1, 0, 1], np.uint8)
    out = O.gates(real_keys, O.NAND, O.encrypt_bits(real_keys, A, 1), O.encrypt_bits(real_keys, B, 2))
    assert O.decrypt_bits(real_keys, out).tolist() == [1, 1, 1, 0]


def test_not_is_negation():
    keys = O.keygen(O.TOY, seed=3, with_bk=False, with_ksk=False)
    c = O.encrypt_bits(keys, [1, 0], 5)
    out = O.gates(keys, O.NOT, c)
    assert ((out.astype(np.uint64) + c) % M32 == 0).all()


# ---------------------------------------------------------------- decryption tie (C11) and netlists
def test_decrypt_phase_zero_is_zero_and_sign_edges():
    """C11: Decrypt = [(int32) phase > 0]; an exact phase-0 ciphertext decrypts to 0 (a `>= 0` slip fails here),
    and the int32 sign edges: phase 1 -> 1, 2^31 - 1 -> 1, 2^31 (= -2^31) -> 0, 2^32 - 1 (= -1) -> 0"""
    keys = O.keygen(O.TOY, seed=21, with_bk=False, with_ksk=False)
    rng = np.random.default_rng(22)
    phases = [0, 1, (1 << 31) - 1, 1 << 31, M32 - 1, MU, M32 - MU]
    cts = np.zeros((len(phases), O.TOY.n + 1), np.uint32)
    for k, ph in enumerate(phases):
        a = rng.integers(0, M32, O.TOY.n, dtype=np.uint64)
        cts[k, :O.TOY.n] = a
        cts[k, O.TOY.n] = (ph + int((a * keys.s.astype(np.uint64)).sum())) % M32   # b = <a,s> + phase exactly
    assert [py_lwe_phase(keys.s.tolist(), c.tolist()) for c in cts] == phases
    assert O.decrypt_bits(keys, cts).tolist() == [0, 1, 1, 0, 0, 1, 0]


def _rca_oracle(keys, bits_n, A, B, seed):
    """Algorithm 1 levels of the ripple-carry adder, each evaluated by O.run_level (or_level_batch)"""
    from oracle.algorithm1 import algorithm1
    n = synth.ripple_carry_adder(bits_n)
    x = np.concatenate([synth.pack_bits([A], bits_n), synth.pack_bits([B], bits_n)])
    w = np.zeros((n["n_inputs"] + len(n["type"]), keys.params.n + 1), np.uint32)
    w[:n["n_inputs"]] = O.encrypt_bits(keys, x, seed)
    for batch in algorithm1(n["n_inputs"], n["type"], n["in0"], n["in1"], n["in2"]):
        b = np.array(batch)
        O.run_level(keys, w, n["type"][b], n["in0"][b], n["in1"][b], n["in2"][b], n["n_inputs"] + b)
    return int(synth.unpack_bits(O.decrypt_bits(keys, w[n["outputs"]]), bits_n + 1)[0])


def test_level_batch_ripple_carry_adder_toy():
    """or_level_batch (the oracle's level executor, used by the GPU parity tests) end to end on the 8-bit RCA of
    cfg 2: the decrypted sum equals a + b for seeded pairs, edge pairs included"""
    keys = O.keygen(O.TOY, seed=23)
    rng = np.random.default_rng(24)
    pairs = [(0, 0), (255, 255), (255, 1), (128, 128)] + [tuple(rng.integers(0, 256, 2)) for _ in range(4)]
    for k, (A, B) in enumerate(pairs):
        assert _rca_oracle(keys, 8, int(A), int(B), 30 + k) == int(A) + int(B), (A, B)


@pytest.mark.slow
def test_level_batch_ripple_carry_adder_real_params(real_keys):
    """the same at the real parameters on a 2-bit adder (7 gates, 4 levels)"""
    assert _rca_oracle(real_keys, 2, 3, 3, 40) == 6
    assert _rca_oracle(real_keys, 2, 2, 1, 41) == 3


# ---------------------------------------------------------------- noise bounds ([7]; SURVEY 8(c) noise row)
def np_trlwe_phase_binary(S, acc, N):
    """phase(b - a * S) of a TRLWE sample for a binary S in numpy: a * S = sum_{j: S_j = 1} X^j a (negacyclic
    shifts), independent of the oracle's C code"""
    a, b = acc[:N].astype(np.int64), acc[N:].astype(np.int64)
    prod = np.zeros(N, np.int64)
    for j in np.nonzero(S)[0]:
        rot = np.concatenate([-a[N - j:], a[:N - j]])        # X^j a mod X^N + 1
        prod = (prod + rot) % M32
    return (b - prod) % M32


@pytest.mark.slow
def test_blind_rotation_noise_within_bound(real_keys):
    """MSE of phase(ACC) - X^{-phibar} v over all N coefficients of 256 blind rotations <= V_BR bound
    1.408e-5 + 3.7e-8 (the mean-square error, bias included, over >= 256 bootstraps)."""
    from concurrent.futures import ThreadPoolExecutor
    P = O.DEFAULT
    K = 256
    cts = O.encrypt_bits(real_keys, np.arange(K) & 1, 100)
    with ThreadPoolExecutor(O.max_threads()) as ex:           # ctypes releases the GIL
        accs = list(ex.map(lambda c: O.blind_rotate(real_keys, c), cts))
    two_N = 2 * P.N
    # tfhe-lib mod switch (pinned above): round(v 2N / 2^32) = ((v + 2^20) mod 2^32) >> 21
    ms = lambda v: ((np.asarray(v, np.uint64) + (1 << 20)) % M32) >> 21
    s = real_keys.s.astype(np.uint64)
    errs = []
    for ct, acc in zip(cts, accs):
        ph = np_trlwe_phase_binary(real_keys.S, acc, P.N)
        phibar = (int(ms(ct[P.n])) - int((ms(ct[:P.n]) * s).sum())) % two_N
        # expected message: X^{-phibar} (mu,...,mu): coefficient c = +mu if c + phibar mod 2N < N else -mu
        e = (np.arange(P.N) + phibar) % two_N
        want = np.where(e < P.N, MU, M32 - MU)
        d = (ph - want) % M32
        errs.append(np.where(d >= 1 << 31, d - M32, d) / M32)
    mse = float(np.mean(np.square(np.concatenate(errs))))
    assert mse < 1.408e-5 + 3.7e-8, mse
    assert mse > 1e-7            # the noise is really there (keys are not noiseless)


def test_keyswitch_noise_within_bound(real_keys):
    """MSE of KS(noiseless LWE_S(m)) - m <= V_KS bound kN t sigma_ks^2 + kN 2^-2(t basebit + 1)."""
    P = O.DEFAULT
    rng = np.random.default_rng(17)
    errs = []
    for k in range(300):
        m = int(rng.integers(0, M32))
        a = rng.integers(0, M32, P.N, dtype=np.uint64).astype(np.uint32)
        b = (m + int((a.astype(np.int64) * real_keys.S).sum())) % M32
        out = O.keyswitch(real_keys, np.concatenate([a, np.array([b], np.uint32)]))
        errs.append(signed(py_lwe_phase(real_keys.s.tolist(), out.tolist()) - m) / M32)
    mse = float(np.mean(np.square(errs)))
    bound = 1024 * 8 * (2.0 ** -15) ** 2 + 1024 * 2.0 ** (-2 * 17)
    assert mse < bound, (mse, bound)
