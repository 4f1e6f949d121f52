"""Plain CPU oracle for TFHE gate bootstrapping -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package.  The product package ``paper_conf_ispass_maxw23_b200`` never imports it and
the two share no code.

The arithmetic lives in ``tfhe_oracle.c`` (plain C, schoolbook products, OpenMP only across independent
gates); this module is ctypes marshalling plus the plain-Python pieces of the method that are host logic:
Algorithm 1 levelisation (``algorithm1.py``) and the plaintext gate semantics (``plain.py``).

Citations: P:N = /root/reference/PAPER.md line N; Cn = reading Cn in DESIGN.md / SURVEY.md Sec. 8(c).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tfhe_oracle.c")


def _cpu_tag() -> str:
    """short hash of this host's CPU flags: the library is compiled with -march=native, so each host (this
    container, the GPU box's host) gets its own build, compiled on first use"""
    import hashlib
    try:
        flags = next(l for l in open("/proc/cpuinfo") if l.startswith("flags"))
    except Exception:
        flags = "unknown"
    return hashlib.sha1(flags.encode()).hexdigest()[:10]


_SO = os.path.join(_HERE, "liboracle-%s.so" % _cpu_tag())

# gate codes: truth table f(a,b) at bit (2a+b) (C15); MUX = 3-input extension
NOR, ANDNY, NOT, ANDYN, XOR, NAND, AND, XNOR, ORNY, ORYN, OR, MUX = 1, 2, 3, 4, 6, 7, 8, 9, 11, 13, 14, 16
TWO_INPUT = (NAND, AND, OR, NOR, XOR, XNOR, ANDNY, ANDYN, ORNY, ORYN)
GATE_NAMES = {NOR: "NOR", ANDNY: "ANDNY", NOT: "NOT", ANDYN: "ANDYN", XOR: "XOR", NAND: "NAND", AND: "AND",
              XNOR: "XNOR", ORNY: "ORNY", ORYN: "ORYN", OR: "OR", MUX: "MUX"}


def build(force: bool = False) -> str:
    """Compile liboracle-<cpu>.so with gcc (plain C + OpenMP) at -O3 -march=native: one build per
    host CPU type, so the cpu_baseline is not understated on a host with wider vector units."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "tfhe_oracle.h"))):
        tmp = _SO + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O3", "-march=native", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


class _Params(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int32), ("N", ctypes.c_int32), ("l", ctypes.c_int32), ("Bgbit", ctypes.c_int32),
                ("ks_t", ctypes.c_int32), ("ks_basebit", ctypes.c_int32), ("sigma_lwe", ctypes.c_double),
                ("sigma_bk", ctypes.c_double), ("sigma_ks", ctypes.c_double), ("bk_mask_mult", ctypes.c_uint32)]


@dataclass(frozen=True)
class Params:
    """TFHE parameters.  Default = tfhe-lib's 128-bit gate-bootstrapping set ("default parameter set of
    Sec. VIII of [7]"; C2): n=630, N=1024, l=3, Bgbit=7, KS t=8, basebit=2, sigma 2^-15 / 2^-25 / 2^-15."""
    n: int = 630
    N: int = 1024
    l: int = 3
    Bgbit: int = 7
    ks_t: int = 8
    ks_basebit: int = 2
    sigma_lwe: float = 2.0 ** -15
    sigma_bk: float = 2.0 ** -25
    sigma_ks: float = 2.0 ** -15
    bk_mask_mult: int = 1

    def c(self) -> _Params:
        return _Params(self.n, self.N, self.l, self.Bgbit, self.ks_t, self.ks_basebit, self.sigma_lwe,
                       self.sigma_bk, self.sigma_ks, self.bk_mask_mult)

    @property
    def bk_words(self) -> int:
        return self.n * 2 * self.l * 2 * self.N

    @property
    def ksk_words(self) -> int:
        return self.N * self.ks_t * (1 << self.ks_basebit) * (self.n + 1)


DEFAULT = Params()
TOY = Params(n=16, N=64)           # real l/Bg/t/base/sigma, tiny n and N (SURVEY App. A "toy TFHE")

_lib = None
_u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")
_i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
_u8p = np.ctypeslib.ndpointer(np.uint8, flags="C_CONTIGUOUS")


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P = ctypes.POINTER(_Params)
        sig = {
            "or_keygen": (None, [P, ctypes.c_uint64, _i32p, _i32p, ctypes.c_void_p, ctypes.c_void_p]),
            "or_make_bk": (None, [P, ctypes.c_uint64, _i32p, _i32p, _u32p]),
            "or_make_ksk": (None, [P, ctypes.c_uint64, _i32p, _i32p, _u32p]),
            "or_lwe_encrypt": (None, [P, _i32p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_double, _u32p]),
            "or_lwe_phase": (ctypes.c_uint32, [ctypes.c_int32, _i32p, _u32p]),
            "or_encrypt_bits": (None, [P, _i32p, ctypes.c_uint64, ctypes.c_int64, _u8p, _u32p, ctypes.c_int64]),
            "or_decrypt_bits": (None, [ctypes.c_int32, _i32p, ctypes.c_int64, _u32p, ctypes.c_int64, _u8p]),
            "or_negacyclic_muladd": (None, [ctypes.c_int32, _i32p, _u32p, _u32p]),
            "or_poly_mul_xai": (None, [ctypes.c_int32, ctypes.c_int32, _u32p, _u32p]),
            "or_trlwe_phase": (None, [ctypes.c_int32, _i32p, _u32p, _u32p]),
            "or_trlwe_encrypt": (None, [ctypes.c_int32, _i32p, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p,
                                        _u32p]),
            "or_mod_switch": (ctypes.c_uint32, [ctypes.c_uint32, ctypes.c_int32]),
            "or_decompose": (None, [P, _u32p, _i32p]),
            "or_external_product": (None, [P, _u32p, _u32p, _u32p]),
            "or_cmux_step": (None, [P, _u32p, ctypes.c_int32, _u32p]),
            "or_blind_rotate": (None, [P, _u32p, _u32p, ctypes.c_uint32, _u32p]),
            "or_sample_extract": (None, [P, _u32p, _u32p]),
            "or_keyswitch": (None, [P, _u32p, _u32p, _u32p]),
            "or_bootstrap_wo_ks": (None, [P, _u32p, ctypes.c_uint32, _u32p, _u32p]),
            "or_gate_linear": (ctypes.c_int, [P, ctypes.c_int, _u32p, _u32p, _u32p]),
            "or_gate_batch": (ctypes.c_int, [P, _u32p, _u32p, ctypes.c_int64, _i32p, _u32p, ctypes.c_void_p,
                                             ctypes.c_void_p, _u32p, ctypes.c_int64, ctypes.c_int]),
            "or_level_batch": (ctypes.c_int, [P, _u32p, _u32p, ctypes.c_int64, _i32p, _i64p, _i64p, _i64p, _i64p,
                                              _u32p, ctypes.c_int64, ctypes.c_int]),
            "or_max_threads": (ctypes.c_int, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _vp(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


@dataclass
class Keys:
    params: Params
    s: np.ndarray          # LWE secret, n bits (int32)
    S: np.ndarray          # TRLWE secret, N bits (int32)
    bk: np.ndarray         # [n][2l][2][N] u32
    ksk: np.ndarray        # [N][t][base][n+1] u32


def keygen(params: Params = DEFAULT, seed: int = 1, with_ksk: bool = True, with_bk: bool = True) -> Keys:
    """Seeded KeyGen (EXT[10]; C12).  Client side: the GPU library never sees s or S."""
    p = params.c()
    s = np.zeros(params.n, np.int32)
    S = np.zeros(params.N, np.int32)
    bk = np.zeros(params.bk_words if with_bk else 1, np.uint32)
    ksk = np.zeros(params.ksk_words if with_ksk else 1, np.uint32)
    lib().or_keygen(ctypes.byref(p), seed, s, S, _vp(bk) if with_bk else None, _vp(ksk) if with_ksk else None)
    return Keys(params, s, S, bk, ksk)


def encrypt_bits(keys: Keys, bits, seed: int, stride: int | None = None) -> np.ndarray:
    """Encrypt(bit) = (a, <a,s> + (bit ? +1/8 : -1/8) + e)  (C6)."""
    bits = np.ascontiguousarray(np.asarray(bits, np.uint8).reshape(-1))
    stride = stride or keys.params.n + 1
    out = np.zeros((bits.size, stride), np.uint32)
    lib().or_encrypt_bits(ctypes.byref(keys.params.c()), keys.s, seed, bits.size, bits, out.reshape(-1), stride)
    return out


def decrypt_bits(keys: Keys, cts: np.ndarray) -> np.ndarray:
    cts = np.ascontiguousarray(cts, np.uint32)
    out = np.zeros(cts.shape[0], np.uint8)
    lib().or_decrypt_bits(keys.params.n, keys.s, cts.shape[0], cts.reshape(-1), cts.shape[1], out)
    return out


def lwe_phase(keys_or_s, ct: np.ndarray) -> int:
    s = keys_or_s.s if isinstance(keys_or_s, Keys) else np.ascontiguousarray(keys_or_s, np.int32)
    return int(lib().or_lwe_phase(s.size, s, np.ascontiguousarray(ct, np.uint32)))


def lwe_encrypt(params: Params, s, mu: int, seed: int, sigma: float | None = None) -> np.ndarray:
    ct = np.zeros(params.n + 1, np.uint32)
    lib().or_lwe_encrypt(ctypes.byref(params.c()), np.ascontiguousarray(s, np.int32), seed, mu & 0xFFFFFFFF,
                         params.sigma_lwe if sigma is None else sigma, ct)
    return ct


def negacyclic_muladd(d, b, res=None) -> np.ndarray:
    d = np.ascontiguousarray(d, np.int32)
    b = np.ascontiguousarray(b, np.uint32)
    res = np.zeros(b.size, np.uint32) if res is None else np.ascontiguousarray(res, np.uint32).copy()
    lib().or_negacyclic_muladd(b.size, d, b, res)
    return res


def poly_mul_xai(a: int, src) -> np.ndarray:
    src = np.ascontiguousarray(src, np.uint32)
    out = np.zeros_like(src)
    lib().or_poly_mul_xai(src.size, a, src, out)
    return out


def trlwe_phase(S, trlwe) -> np.ndarray:
    S = np.ascontiguousarray(S, np.int32)
    out = np.zeros(S.size, np.uint32)
    lib().or_trlwe_phase(S.size, S, np.ascontiguousarray(trlwe, np.uint32).reshape(-1), out)
    return out


def trlwe_encrypt(S, seed: int, sigma: float, mu=None) -> np.ndarray:
    S = np.ascontiguousarray(S, np.int32)
    out = np.zeros(2 * S.size, np.uint32)
    m = None if mu is None else np.ascontiguousarray(mu, np.uint32)
    lib().or_trlwe_encrypt(S.size, S, seed, sigma, _vp(m), out)
    return out


def mod_switch(a: int, two_N: int) -> int:
    return int(lib().or_mod_switch(a & 0xFFFFFFFF, two_N))


def decompose(params: Params, poly) -> np.ndarray:
    out = np.zeros((params.l, params.N), np.int32)
    lib().or_decompose(ctypes.byref(params.c()), np.ascontiguousarray(poly, np.uint32), out.reshape(-1))
    return out


def external_product(params: Params, tgsw, acc) -> np.ndarray:
    out = np.zeros(2 * params.N, np.uint32)
    lib().or_external_product(ctypes.byref(params.c()), np.ascontiguousarray(tgsw, np.uint32).reshape(-1),
                              np.ascontiguousarray(acc, np.uint32).reshape(-1), out)
    return out


def cmux_step(params: Params, tgsw, abar: int, acc) -> np.ndarray:
    acc = np.ascontiguousarray(acc, np.uint32).reshape(-1).copy()
    lib().or_cmux_step(ctypes.byref(params.c()), np.ascontiguousarray(tgsw, np.uint32).reshape(-1), abar, acc)
    return acc


def blind_rotate(keys: Keys, ct, mu: int = 1 << 29) -> np.ndarray:
    acc = np.zeros(2 * keys.params.N, np.uint32)
    lib().or_blind_rotate(ctypes.byref(keys.params.c()), keys.bk, np.ascontiguousarray(ct, np.uint32), mu, acc)
    return acc


def sample_extract(params: Params, acc) -> np.ndarray:
    out = np.zeros(params.N + 1, np.uint32)
    lib().or_sample_extract(ctypes.byref(params.c()), np.ascontiguousarray(acc, np.uint32), out)
    return out


def keyswitch(keys: Keys, ext) -> np.ndarray:
    out = np.zeros(keys.params.n + 1, np.uint32)
    lib().or_keyswitch(ctypes.byref(keys.params.c()), keys.ksk, np.ascontiguousarray(ext, np.uint32), out)
    return out


def bootstrap_wo_ks(keys: Keys, ct, mu: int = 1 << 29) -> np.ndarray:
    out = np.zeros(keys.params.N + 1, np.uint32)
    lib().or_bootstrap_wo_ks(ctypes.byref(keys.params.c()), keys.bk, mu, np.ascontiguousarray(ct, np.uint32), out)
    return out


def gate_linear(params: Params, gate: int, ca, cb) -> np.ndarray:
    out = np.zeros(params.n + 1, np.uint32)
    rc = lib().or_gate_linear(ctypes.byref(params.c()), gate, np.ascontiguousarray(ca, np.uint32),
                              np.ascontiguousarray(cb, np.uint32), out)
    if rc:
        raise ValueError("not a two-input gate: %r" % gate)
    return out


def gates(keys: Keys, gate, ca, cb=None, cc=None, nthreads: int = 0) -> np.ndarray:
    """Bootstrapped gates, row i = gate[i](ca[i], cb[i][, cc[i]])  (P:54 bootstrapped-Gate; EXT[10])."""
    ca = np.ascontiguousarray(ca, np.uint32)
    count, stride = ca.shape
    g = np.ascontiguousarray(np.broadcast_to(np.asarray(gate, np.int32), (count,)), np.int32)
    cb_ = None if cb is None else np.ascontiguousarray(cb, np.uint32)
    cc_ = None if cc is None else np.ascontiguousarray(cc, np.uint32)
    if (g == MUX).any() and cc_ is None:
        raise ValueError("MUX needs cc")
    if np.isin(g, TWO_INPUT + (MUX,)).any() and cb_ is None:
        raise ValueError("two-input gates need cb")
    out = np.zeros_like(ca)
    rc = lib().or_gate_batch(ctypes.byref(keys.params.c()), keys.bk, keys.ksk, count, g, ca, _vp(cb_), _vp(cc_),
                             out, stride, nthreads)
    if rc:
        raise ValueError("bad gate code")
    return out


def run_level(keys: Keys, wires: np.ndarray, gate, in0, in1, in2, out, nthreads: int = 0) -> None:
    """One Algorithm-1 level: wires[out[i]] = gate[i](wires[in0[i]], wires[in1[i]], wires[in2[i]])."""
    a = lambda x: np.ascontiguousarray(x, np.int64)
    rc = lib().or_level_batch(ctypes.byref(keys.params.c()), keys.bk, keys.ksk, len(gate),
                              np.ascontiguousarray(gate, np.int32), a(in0), a(in1), a(in2), a(out),
                              wires.reshape(-1), wires.shape[1], nthreads)
    if rc:
        raise ValueError("bad gate code")


def max_threads() -> int:
    return int(lib().or_max_threads())
