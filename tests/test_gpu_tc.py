"""Tensor-core (tcgen05.mma kind::i8) building blocks against plain integer arithmetic (-m gpu).

The tensor-core NTT of the blind rotation multiplies byte limbs on the tensor
cores; these tests pin the descriptor encodings, operand layouts (K-major core matrices, padded strides), the
s8 / u8 signedness and the TMEM read-back against numpy's exact int64 matrix product.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ispass_maxw23_b200 as tb
    tb.build()
    c = tb.Context(0)
    yield c
    c.close()


@pytest.mark.parametrize("K,N,a_signed,lbo", [(32, 16, False, 128), (32, 128, True, 144), (128, 128, False, 144),
                                              (128, 128, True, 128), (256, 256, False, 144)])
def test_mma_i8_equals_integer_matmul(ctx, K, N, a_signed, lbo):
    rng = np.random.default_rng(K + N + lbo)
    A = rng.integers(-128 if a_signed else 0, 128 if a_signed else 256, (128, K)).astype(np.int8 if a_signed else np.uint8)
    B = rng.integers(0, 256, (N, K)).astype(np.uint8)
    D = ctx.tc_mma_test(A, B, a_signed=a_signed, b_signed=False, lbo=lbo)
    want = A.astype(np.int64) @ B.astype(np.int64).T
    assert (D.astype(np.int64) == want).all()


def test_mma_i8_extremes(ctx):
    """all-255 x all-255 at K = 256: 256 * 255^2 = 16,646,400 per entry, the largest the NTT accumulates"""
    A = np.full((128, 256), 255, np.uint8)
    B = np.full((256, 256), 255, np.uint8)
    D = ctx.tc_mma_test(A, B, lbo=144)
    assert (D == 256 * 255 * 255).all()


def test_tc_muladd_equals_schoolbook(ctx):
    """one CMux step's exact external-product core on the tensor cores (four-step NTT, MAC against the NTT-domain
    BK, inverse, centred lift) == the schoolbook negacyclic sums mod 2^32, random and worst-case inputs"""
    import torch
    import oracle as O
    rng = np.random.default_rng(5)
    M32 = 1 << 32
    cases = [(rng.integers(-64, 64, (4, 6, 1024)), rng.integers(0, M32, (6, 2, 1024), dtype=np.uint64)),
             (np.full((4, 6, 1024), -64), np.full((6, 2, 1024), M32 - 1, np.uint64)),
             (np.stack([np.full((6, 1024), 63), np.full((6, 1024), -64)] * 2), np.full((6, 2, 1024), 1 << 31, np.uint64)),
             (np.zeros((4, 6, 1024), int), rng.integers(0, M32, (6, 2, 1024), dtype=np.uint64))]
    for d, b in cases:
        d32 = d.astype(np.int32)
        b32 = b.astype(np.uint32)
        got = ctx.tc_muladd(torch.from_numpy(d32).cuda(), torch.from_numpy(b32.view(np.int32)).cuda())
        got = got.cpu().numpy().view(np.uint32)
        for g in range(4):
            for q in range(2):
                want = np.zeros(1024, np.uint32)
                for r in range(6):
                    want = O.negacyclic_muladd(d32[g, r], b32[r, q], want)
                assert (got[g, q] == want).all(), (g, q)


def test_bk_domains_built_on_demand():
    """only the BK domains the selected kernels read are resident: the tensor-core domain
    appears when variant 12 is selected after the load, and its kernel is then bit-exact"""
    import torch
    import oracle as O
    import paper_conf_ispass_maxw23_b200 as tb
    keys = O.keygen(O.DEFAULT, seed=31)
    c = tb.Context(0)
    try:
        c.set_narrow_kernel(11)                     # brl only in latency mode: no four-step domain needed yet
        c.load_keys(keys.bk, keys.ksk)
        before = c.key_bytes()
        c.set_br_variant(12)
        after = c.key_bytes()
        assert after - before == 630 * 1024 * 36 * 4                    # the four-step domain, 92.9 MB
        c.set_narrow_lanes(0)
        cts = O.encrypt_bits(keys, [1, 0, 1], 32)
        got = c.bootstrap_wo_ks(c.to_device(cts))[:, :1025].cpu().numpy().view(np.uint32)
        for k in range(3):
            assert (got[k] == O.bootstrap_wo_ks(keys, cts[k])).all()
    finally:
        c.close()
