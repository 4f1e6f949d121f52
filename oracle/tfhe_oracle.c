/*
 * tfhe_oracle.c -- plain CPU oracle for TFHE gate bootstrapping.  TEST INFRASTRUCTURE ONLY (see
 * tfhe_oracle.h): never linked or executed by the product path.
 *
 * Citations: "P:N" = /root/reference/PAPER.md line N.  PAPER.md names the blocks of a bootstrapped
 * gate but delegates their definition to the TFHE paper [7] and the
 * TFHE library [10]; "Cn" = the reading recorded in DESIGN.md / SURVEY.md Sec. 8(c) row Cn.
 * Each step is the textbook definition, in the order the algorithm states it, with plain loops:
 * schoolbook negacyclic products, no transforms, no blocking, no reordering.
 */
#include "tfhe_oracle.h"
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

size_t or_bk_words(const or_params* P) { return (size_t)P->n * (2 * P->l) * 2 * P->N; }
size_t or_ksk_words(const or_params* P) {
    return (size_t)P->N * P->ks_t * ((size_t)1 << P->ks_basebit) * (P->n + 1);
}

/* ---------------------------------------------------------------- randomness (C12) */
uint64_t or_rng_u64(uint64_t* st) {           /* splitmix64 */
    uint64_t z = (*st += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
uint32_t or_rng_u32(uint64_t* st) { return (uint32_t)(or_rng_u64(st) >> 32); }
double or_rng_normal(uint64_t* st) {          /* Box-Muller, u1 in (0,1] */
    double u1 = ((double)(or_rng_u64(st) >> 11) + 1.0) * (1.0 / 9007199254740992.0);
    double u2 = (double)(or_rng_u64(st) >> 11) * (1.0 / 9007199254740992.0);
    return sqrt(-2.0 * log(u1)) * cos(6.283185307179586476925286766559 * u2);
}
uint32_t or_rng_gauss_torus(uint64_t* st, double sigma) {
    if (sigma == 0.0) return 0u;
    double e = sigma * or_rng_normal(st) * 4294967296.0;     /* torus units -> 2^32 scale */
    return (uint32_t)(int64_t)llround(e);
}
static uint64_t stream(uint64_t seed, uint64_t purpose, uint64_t index) {
    uint64_t st = seed ^ (purpose * 0xD1B54A32D192ED03ull) ^ (index * 0x8CB92BA72F3D8DD7ull);
    or_rng_u64(&st);
    return st;
}

/* ---------------------------------------------------------------- polynomials */
/* res += d (x) b  mod (X^N + 1, 2^32), by the definition of the negacyclic product:
 * X^i * X^j = X^(i+j) if i+j < N, else -X^(i+j-N). */
void or_negacyclic_muladd(int32_t N, const int32_t* d, const uint32_t* b, uint32_t* res) {
    for (int32_t i = 0; i < N; i++) {
        uint32_t di = (uint32_t)d[i];
        if (di == 0) continue;
        for (int32_t j = 0; j < N - i; j++) res[i + j] += di * b[j];          /* i + j <  N */
        for (int32_t j = N - i; j < N; j++) res[i + j - N] -= di * b[j];      /* i + j >= N: X^N = -1 */
    }
}

/* res = X^a * src for 0 <= a < 2N (X^N = -1) */
void or_poly_mul_xai(int32_t N, int32_t a, const uint32_t* src, uint32_t* res) {
    for (int32_t i = 0; i < N; i++) {
        /* coefficient i of X^a * src comes from src[i - a (mod 2N)] with sign (-1)^wraps */
        int32_t src_idx = i - a;
        uint32_t sign_neg = 0;
        while (src_idx < 0) { src_idx += N; sign_neg ^= 1u; }
        res[i] = sign_neg ? (uint32_t)(0u - src[src_idx]) : src[src_idx];
    }
}

void or_trlwe_phase(int32_t N, const int32_t* S, const uint32_t* trlwe, uint32_t* out) {
    uint32_t* aS = (uint32_t*)calloc((size_t)N, 4);
    or_negacyclic_muladd(N, S, trlwe, aS);                  /* a (x) S */
    for (int32_t c = 0; c < N; c++) out[c] = trlwe[N + c] - aS[c];
    free(aS);
}

void or_trlwe_encrypt(int32_t N, const int32_t* S, uint64_t seed, double sigma, const uint32_t* mu,
                      uint32_t* trlwe) {
    uint64_t st = stream(seed, 11, 0);
    uint32_t* a = trlwe;
    uint32_t* b = trlwe + N;
    for (int32_t c = 0; c < N; c++) a[c] = or_rng_u32(&st);
    for (int32_t c = 0; c < N; c++) b[c] = or_rng_gauss_torus(&st, sigma) + (mu ? mu[c] : 0u);
    or_negacyclic_muladd(N, S, a, b);                        /* b = a (x) S + e + mu */
}

/* ---------------------------------------------------------------- LWE */
uint32_t or_lwe_phase(int32_t n, const int32_t* s, const uint32_t* ct) {
    uint32_t acc = ct[n];
    for (int32_t i = 0; i < n; i++) acc -= ct[i] * (uint32_t)s[i];
    return acc;
}
int or_bit_decrypt(int32_t n, const int32_t* s, const uint32_t* ct) {
    return (int32_t)or_lwe_phase(n, s, ct) > 0 ? 1 : 0;     /* C11: phase exactly 0 -> 0 */
}
static void lwe_encrypt_state(int32_t n, const int32_t* s, uint64_t* st, uint32_t mu, double sigma,
                              uint32_t* ct) {
    uint32_t b = mu + or_rng_gauss_torus(st, sigma);
    for (int32_t i = 0; i < n; i++) {
        ct[i] = or_rng_u32(st);
        b += ct[i] * (uint32_t)s[i];
    }
    ct[n] = b;                                              /* b = <a,s> + mu + e */
}
void or_lwe_encrypt(const or_params* P, const int32_t* s, uint64_t seed, uint32_t mu, double sigma,
                    uint32_t* ct) {
    uint64_t st = stream(seed, 21, 0);
    lwe_encrypt_state(P->n, s, &st, mu, sigma, ct);
}
void or_encrypt_bits(const or_params* P, const int32_t* s, uint64_t seed, int64_t count, const uint8_t* bits,
                     uint32_t* cts, int64_t stride) {
    const uint32_t mu = 1u << 29;                            /* 1/8 on the torus */
    for (int64_t g = 0; g < count; g++) {
        uint64_t st = stream(seed, 22, (uint64_t)g);
        lwe_encrypt_state(P->n, s, &st, bits[g] ? mu : (uint32_t)(0u - mu), P->sigma_lwe, cts + g * stride);
    }
}
void or_decrypt_bits(int32_t n, const int32_t* s, int64_t count, const uint32_t* cts, int64_t stride,
                     uint8_t* bits) {
    for (int64_t g = 0; g < count; g++) bits[g] = (uint8_t)or_bit_decrypt(n, s, cts + g * stride);
}

/* ---------------------------------------------------------------- keys */
/* BK_i = TGSW_S(s_i): row r = bloc*l + j is a TRLWE encryption of 0 under S, then coefficient 0 of its
 * poly `bloc` gets + s_i * h_j with h_j = 2^(32 - Bgbit (j+1))  (EXT[10]; SURVEY 8(c) KeyGen). */
void or_make_bk(const or_params* P, uint64_t seed, const int32_t* s, const int32_t* S, uint32_t* bk) {
    const int32_t N = P->N, l = P->l;
    for (int32_t i = 0; i < P->n; i++) {
        for (int32_t bloc = 0; bloc < 2; bloc++) {
            for (int32_t j = 0; j < l; j++) {
                int32_t r = bloc * l + j;
                uint32_t* row = bk + (((size_t)i * 2 * l + r) * 2) * N;
                uint32_t* a = row;
                uint32_t* b = row + N;
                uint64_t st = stream(seed, 31, (uint64_t)i * 64 + r);
                for (int32_t c = 0; c < N; c++) {
                    uint32_t m = P->bk_mask_mult ? P->bk_mask_mult : 1u;
                    a[c] = or_rng_u32(&st);
                    a[c] -= a[c] % m;                        /* structured test key: masks in m*Z */
                }
                for (int32_t c = 0; c < N; c++) b[c] = or_rng_gauss_torus(&st, P->sigma_bk);
                or_negacyclic_muladd(N, S, a, b);            /* b = a (x) S + e */
                uint32_t h = 1u << (32 - P->Bgbit * (j + 1));
                row[bloc * N + 0] += (uint32_t)s[i] * h;     /* + s_i * h_j on poly `bloc` */
            }
        }
    }
}
/* KSK[i][j][d] = LWE_s(s'_i * d * 2^(32 - basebit (j+1))), d = 0 trivial zero (EXT[10]; C9). */
void or_make_ksk(const or_params* P, uint64_t seed, const int32_t* s, const int32_t* S, uint32_t* ksk) {
    const int32_t n = P->n, t = P->ks_t, base = 1 << P->ks_basebit;
    for (int32_t i = 0; i < P->N; i++) {
        for (int32_t j = 0; j < t; j++) {
            for (int32_t d = 0; d < base; d++) {
                uint32_t* row = ksk + (((size_t)i * t + j) * base + d) * (n + 1);
                if (d == 0) { memset(row, 0, (size_t)(n + 1) * 4); continue; }
                uint32_t msg = (uint32_t)S[i] * (uint32_t)d * (1u << (32 - P->ks_basebit * (j + 1)));
                uint64_t st = stream(seed, 41, ((uint64_t)i * t + j) * base + d);
                lwe_encrypt_state(n, s, &st, msg, P->sigma_ks, row);
            }
        }
    }
}
void or_keygen(const or_params* P, uint64_t seed, int32_t* s, int32_t* S, uint32_t* bk, uint32_t* ksk) {
    uint64_t st = stream(seed, 1, 0);
    for (int32_t i = 0; i < P->n; i++) s[i] = (int32_t)(or_rng_u64(&st) >> 63);      /* s in {0,1}^n */
    for (int32_t i = 0; i < P->N; i++) S[i] = (int32_t)(or_rng_u64(&st) >> 63);      /* S in {0,1}^N */
    if (bk) or_make_bk(P, seed, s, S, bk);
    if (ksk) or_make_ksk(P, seed, s, S, ksk);
}

/* ---------------------------------------------------------------- bootstrapping steps */
/* a2 / C5: round(a * 2N / 2^32) mod 2N, half up == ((a + 2^(31 - log2 2N)) mod 2^32) >> (32 - log2 2N) */
uint32_t or_mod_switch(uint32_t a, int32_t two_N) {
    int32_t logm = 0;
    while ((1 << logm) < two_N) logm++;
    uint32_t half = 1u << (31 - logm);
    return (uint32_t)(a + half) >> (32 - logm);
}

/* a4.1 / C4: signed gadget digits, tfhe-lib's truncating offset = sum_j (Bg/2) h_j */
void or_decompose(const or_params* P, const uint32_t* poly, int32_t* digits) {
    const int32_t N = P->N, l = P->l, Bgbit = P->Bgbit;
    const uint32_t Bg = 1u << Bgbit, halfBg = Bg / 2, mask = Bg - 1;
    uint32_t offset = 0;
    for (int32_t j = 0; j < l; j++) offset += halfBg * (1u << (32 - Bgbit * (j + 1)));
    for (int32_t j = 0; j < l; j++) {
        int32_t shift = 32 - Bgbit * (j + 1);
        for (int32_t c = 0; c < N; c++) {
            uint32_t buf = poly[c] + offset;
            digits[j * N + c] = (int32_t)((buf >> shift) & mask) - (int32_t)halfBg;
        }
    }
}

/* a4: out = sum_{r = bloc*l + j} Decomp(acc[bloc])_j (x) tgsw[r]   (both polys of each row) */
void or_external_product(const or_params* P, const uint32_t* tgsw, const uint32_t* acc, uint32_t* out) {
    const int32_t N = P->N, l = P->l;
    int32_t* dig = (int32_t*)malloc((size_t)2 * l * N * 4);
    or_decompose(P, acc, dig);                  /* rows 0..l-1   : digits of poly a */
    or_decompose(P, acc + N, dig + (size_t)l * N); /* rows l..2l-1 : digits of poly b */
    memset(out, 0, (size_t)2 * N * 4);
    for (int32_t r = 0; r < 2 * l; r++) {
        const uint32_t* row = tgsw + (size_t)r * 2 * N;
        or_negacyclic_muladd(N, dig + (size_t)r * N, row, out);          /* a part */
        or_negacyclic_muladd(N, dig + (size_t)r * N, row + N, out + N);  /* b part */
    }
    free(dig);
}

/* a4: acc <- acc + ExtProd(BK_i, (X^abar - 1) acc)  -- the CMux of the blind rotation */
void or_cmux_step(const or_params* P, const uint32_t* tgsw, int32_t abar, uint32_t* acc) {
    const int32_t N = P->N;
    uint32_t* rot = (uint32_t*)malloc((size_t)2 * N * 4);
    uint32_t* prod = (uint32_t*)malloc((size_t)2 * N * 4);
    for (int32_t p = 0; p < 2; p++) {
        or_poly_mul_xai(N, abar, acc + p * N, rot + p * N);
        for (int32_t c = 0; c < N; c++) rot[p * N + c] -= acc[p * N + c];   /* (X^abar - 1) acc */
    }
    or_external_product(P, tgsw, rot, prod);
    for (int32_t c = 0; c < 2 * N; c++) acc[c] += prod[c];
    free(rot);
    free(prod);
}

/* a2-a4: ACC = (0, X^{-bbar} v), v = (mu, ..., mu) (C6); then for each i with abar_i != 0 a CMux with
 * BK_i (tfhe-lib skips abar_i = 0; C7 shows the skip is exact). */
void or_blind_rotate(const or_params* P, const uint32_t* bk, const uint32_t* in_lwe, uint32_t mu,
                     uint32_t* acc) {
    const int32_t N = P->N, n = P->n, two_N = 2 * N;
    const size_t tgsw_words = (size_t)2 * P->l * 2 * N;
    uint32_t* v = (uint32_t*)malloc((size_t)N * 4);
    for (int32_t c = 0; c < N; c++) v[c] = mu;
    int32_t bbar = (int32_t)or_mod_switch(in_lwe[n], two_N);
    memset(acc, 0, (size_t)N * 4);                                       /* ACC.a = 0 */
    or_poly_mul_xai(N, (two_N - bbar) % two_N, v, acc + N);              /* ACC.b = X^{2N-bbar} v */
    for (int32_t i = 0; i < n; i++) {
        int32_t abar = (int32_t)or_mod_switch(in_lwe[i], two_N);
        if (abar == 0) continue;
        or_cmux_step(P, bk + (size_t)i * tgsw_words, abar, acc);
    }
    free(v);
}

/* a5 / C8: index-0 extraction: a'_0 = a_0, a'_j = -a_{N-j}, b' = b_0 */
void or_sample_extract(const or_params* P, const uint32_t* acc, uint32_t* out) {
    const int32_t N = P->N;
    out[0] = acc[0];
    for (int32_t j = 1; j < N; j++) out[j] = 0u - acc[N - j];
    out[N] = acc[N + 0];
}

/* a6 / C9: out = (0, b) - sum_{i,j: d_ij != 0} KSK[i][j][d_ij], d_ij = base-2^basebit digits of
 * a_i + 2^(32 - (1 + basebit t)) */
void or_keyswitch(const or_params* P, const uint32_t* ksk, const uint32_t* in, uint32_t* out) {
    const int32_t n = P->n, t = P->ks_t, bb = P->ks_basebit, base = 1 << bb, Nin = P->N;
    const uint32_t prec_offset = 1u << (32 - (1 + bb * t));
    const uint32_t mask = (uint32_t)base - 1;
    memset(out, 0, (size_t)n * 4);
    out[n] = in[Nin];
    for (int32_t i = 0; i < Nin; i++) {
        uint32_t abar = in[i] + prec_offset;
        for (int32_t j = 0; j < t; j++) {
            uint32_t d = (abar >> (32 - (j + 1) * bb)) & mask;
            if (d == 0) continue;
            const uint32_t* row = ksk + (((size_t)i * t + j) * base + d) * (n + 1);
            for (int32_t c = 0; c <= n; c++) out[c] -= row[c];
        }
    }
}

void or_bootstrap_wo_ks(const or_params* P, const uint32_t* bk, uint32_t mu, const uint32_t* in,
                        uint32_t* out) {
    uint32_t* acc = (uint32_t*)malloc((size_t)2 * P->N * 4);
    or_blind_rotate(P, bk, in, mu, acc);
    or_sample_extract(P, acc, out);
    free(acc);
}

/* ---------------------------------------------------------------- gates (a1, a7) */
/* (C_g, w_a, w_b) per gate type (EXT[10] boot gates; SURVEY 8(c) gate table) */
static int gate_coeffs(int gate, uint32_t* C, int32_t* wa, int32_t* wb) {
    const uint32_t e8 = 1u << 29, e4 = 1u << 30;
    switch (gate) {
        case OR_NAND:  *C = e8;       *wa = -1; *wb = -1; return 0;
        case OR_AND:   *C = 0u - e8;  *wa = 1;  *wb = 1;  return 0;
        case OR_OR:    *C = e8;       *wa = 1;  *wb = 1;  return 0;
        case OR_NOR:   *C = 0u - e8;  *wa = -1; *wb = -1; return 0;
        case OR_XOR:   *C = e4;       *wa = 2;  *wb = 2;  return 0;
        case OR_XNOR:  *C = 0u - e4;  *wa = -2; *wb = -2; return 0;
        case OR_ANDNY: *C = 0u - e8;  *wa = -1; *wb = 1;  return 0;
        case OR_ANDYN: *C = 0u - e8;  *wa = 1;  *wb = -1; return 0;
        case OR_ORNY:  *C = e8;       *wa = -1; *wb = 1;  return 0;
        case OR_ORYN:  *C = e8;       *wa = 1;  *wb = -1; return 0;
        default: return -1;
    }
}
int or_gate_linear(const or_params* P, int gate, const uint32_t* ca, const uint32_t* cb, uint32_t* out) {
    uint32_t C; int32_t wa, wb;
    if (gate_coeffs(gate, &C, &wa, &wb)) return -1;
    for (int32_t c = 0; c <= P->n; c++)
        out[c] = (uint32_t)wa * ca[c] + (uint32_t)wb * cb[c] + (c == P->n ? C : 0u);
    return 0;
}

int or_gate(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int gate, const uint32_t* ca,
            const uint32_t* cb, const uint32_t* cc, uint32_t* out) {
    const int32_t n = P->n, N = P->N;
    const uint32_t mu = 1u << 29;
    if (gate == OR_NOT) {                                   /* NOT = -c, no bootstrap (C10) */
        for (int32_t c = 0; c <= n; c++) out[c] = 0u - ca[c];
        return 0;
    }
    uint32_t* lin = (uint32_t*)malloc((size_t)(n + 1) * 4);
    uint32_t* ext = (uint32_t*)malloc((size_t)(N + 1) * 4);
    int rc = 0;
    if (gate == OR_MUX) {                                   /* a7: KS((0,1/8) + BR(AND(a,b)) + BR(ANDNY(a,c))) */
        uint32_t* ext2 = (uint32_t*)malloc((size_t)(N + 1) * 4);
        or_gate_linear(P, OR_AND, ca, cb, lin);
        or_bootstrap_wo_ks(P, bk, mu, lin, ext);
        or_gate_linear(P, OR_ANDNY, ca, cc, lin);
        or_bootstrap_wo_ks(P, bk, mu, lin, ext2);
        for (int32_t c = 0; c <= N; c++) ext[c] += ext2[c];
        ext[N] += mu;
        free(ext2);
        or_keyswitch(P, ksk, ext, out);
    } else if (or_gate_linear(P, gate, ca, cb, lin) == 0) {
        or_bootstrap_wo_ks(P, bk, mu, lin, ext);
        or_keyswitch(P, ksk, ext, out);
    } else {
        rc = -1;
    }
    free(lin);
    free(ext);
    return rc;
}

int or_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

int or_gate_batch(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int64_t count,
                  const int32_t* gates, const uint32_t* ca, const uint32_t* cb, const uint32_t* cc,
                  uint32_t* out, int64_t stride, int nthreads) {
    int bad = 0;
    if (nthreads <= 0) nthreads = or_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads) reduction(| : bad)
    for (int64_t g = 0; g < count; g++) {
        const uint32_t* c3 = cc ? cc + g * stride : NULL;
        if (or_gate(P, bk, ksk, gates[g], ca + g * stride, cb ? cb + g * stride : NULL, c3, out + g * stride))
            bad |= 1;
    }
    return bad ? -1 : 0;
}

int or_level_batch(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int64_t count,
                   const int32_t* gates, const int64_t* in0, const int64_t* in1, const int64_t* in2,
                   const int64_t* outw, uint32_t* wires, int64_t stride, int nthreads) {
    int bad = 0;
    if (nthreads <= 0) nthreads = or_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads) reduction(| : bad)
    for (int64_t g = 0; g < count; g++) {
        const uint32_t* a = wires + in0[g] * stride;
        const uint32_t* b = in1[g] >= 0 ? wires + in1[g] * stride : NULL;
        const uint32_t* c = in2[g] >= 0 ? wires + in2[g] * stride : NULL;
        if (or_gate(P, bk, ksk, gates[g], a, b, c, wires + outw[g] * stride)) bad |= 1;
    }
    return bad ? -1 : 0;
}
