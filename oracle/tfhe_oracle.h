/*
 * tfhe_oracle.h -- plain, slow, obviously-correct CPU oracle for TFHE gate bootstrapping.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product (paper_conf_ispass_maxw23_b200/) never
 * links, imports or executes anything under oracle/, and this file shares no code, header, table or
 * constant with the CUDA path.
 *
 * What it computes (PAPER.md, "P:N" = /root/reference/PAPER.md line N):
 *   - the FHE API KeyGen / Encrypt / Decrypt / Evaluate (Sec. II-A) for the TFHE scheme (P:54,
 *     Sec. II-B) at "the default parameter set of Section VIII of the TFHE paper" (Sec. II-D);
 *   - the bootstrapped gate = linear gate combination -> blind rotation (Fig. 7) ->
 *     sample extraction -> key switching (Fig. 7; Sec. IV-E).
 * PAPER.md gives no formula for any of these; it delegates to the TFHE library [10].  Every
 * step below is the reading recorded in DESIGN.md ("Readings") / SURVEY.md Sec. 8(c) rows C1-C17,
 * written out as the textbook definition with schoolbook negacyclic products mod 2^32 (no NTT/FFT).
 *
 * All torus arithmetic is uint32_t (wraps mod 2^32).  Layouts (SURVEY 8 preamble):
 *   LWE ciphertext      : a[0..n-1], b            (n+1 words, packed at `stride` >= n+1)
 *   TRLWE               : poly a[N], poly b[N]    (k = 1)
 *   bootstrapping key   : [i < n][row r = bloc*l + j < 2l][poly < 2][N]
 *   key-switching key   : [i < N][j < t][d < 2^basebit][n+1]
 *
 * Every function is single-threaded except the *_batch entry points, which spread independent gates
 * over `nthreads` OpenMP threads (the gates are independent, so this is plain data parallelism).
 */
#ifndef TFHE_ORACLE_H
#define TFHE_ORACLE_H
#include <stdint.h>
#include <stddef.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
    int32_t n;            /* LWE dimension                          (630)   */
    int32_t N;            /* ring degree, power of two             (1024)  */
    int32_t l;            /* gadget length                         (3)     */
    int32_t Bgbit;        /* log2 gadget base                      (7)     */
    int32_t ks_t;         /* key-switch length                     (8)     */
    int32_t ks_basebit;   /* log2 key-switch base                  (2)     */
    double sigma_lwe;     /* stdev of fresh LWE noise, torus units (2^-15) */
    double sigma_bk;      /* stdev of bootstrapping-key noise      (2^-25) */
    double sigma_ks;      /* stdev of key-switching-key noise      (2^-15) */
    uint32_t bk_mask_mult;/* 1 normally; 2^11 = "structured test key" (masks multiples of it) */
} or_params;

/* gate codes: truth table f(a,b) at bit (2a+b) (reading C15); MUX is the 3-input extension */
enum { OR_NOR = 1, OR_ANDNY = 2, OR_NOT = 3, OR_ANDYN = 4, OR_XOR = 6, OR_NAND = 7, OR_AND = 8,
       OR_XNOR = 9, OR_ORNY = 11, OR_ORYN = 13, OR_OR = 14, OR_MUX = 16 };

size_t or_bk_words(const or_params* P);
size_t or_ksk_words(const or_params* P);

/* ---- randomness (oracle-owned, seeded; reading C12) ---- */
uint64_t or_rng_u64(uint64_t* state);       /* splitmix64 step */
uint32_t or_rng_u32(uint64_t* state);
double   or_rng_normal(uint64_t* state);     /* Box-Muller */
uint32_t or_rng_gauss_torus(uint64_t* state, double sigma); /* round(sigma*z*2^32) mod 2^32 */

/* ---- key generation (client side) ---- */
/* s: n bits; S: N bits (TRLWE key, k = 1); bk, ksk as laid out above. */
void or_keygen(const or_params* P, uint64_t seed, int32_t* s, int32_t* S, uint32_t* bk, uint32_t* ksk);
/* the two halves separately (for tests that need a BK built from a given TRLWE key) */
void or_make_bk(const or_params* P, uint64_t seed, const int32_t* s, const int32_t* S, uint32_t* bk);
void or_make_ksk(const or_params* P, uint64_t seed, const int32_t* s, const int32_t* S, uint32_t* ksk);

/* ---- LWE ---- */
void     or_lwe_encrypt(const or_params* P, const int32_t* s, uint64_t seed, uint32_t mu, double sigma,
                        uint32_t* ct);
uint32_t or_lwe_phase(int32_t n, const int32_t* s, const uint32_t* ct);
int      or_bit_decrypt(int32_t n, const int32_t* s, const uint32_t* ct);   /* (int32)phase > 0 */
void     or_encrypt_bits(const or_params* P, const int32_t* s, uint64_t seed, int64_t count,
                         const uint8_t* bits, uint32_t* cts, int64_t stride);
void     or_decrypt_bits(int32_t n, const int32_t* s, int64_t count, const uint32_t* cts, int64_t stride,
                         uint8_t* bits);

/* ---- polynomial / TRLWE primitives ---- */
/* res += d (x) b  in Z_{2^32}[X]/(X^N + 1), d integer poly, b torus poly; schoolbook */
void or_negacyclic_muladd(int32_t N, const int32_t* d, const uint32_t* b, uint32_t* res);
/* res = X^a * src, 0 <= a < 2N */
void or_poly_mul_xai(int32_t N, int32_t a, const uint32_t* src, uint32_t* res);
/* TRLWE phase: out = b - a (x) S */
void or_trlwe_phase(int32_t N, const int32_t* S, const uint32_t* trlwe, uint32_t* out);
/* TRLWE encryption of the torus polynomial `mu` (may be NULL = 0) under S */
void or_trlwe_encrypt(int32_t N, const int32_t* S, uint64_t seed, double sigma, const uint32_t* mu,
                      uint32_t* trlwe);

/* ---- bootstrapping steps ---- */
uint32_t or_mod_switch(uint32_t a, int32_t two_N);                    /* a2 */
void     or_decompose(const or_params* P, const uint32_t* poly, int32_t* digits /* [l][N] */); /* a4.1 */
/* out = ExtProd(tgsw, acc) = sum_r Decomp(acc)_r (x) tgsw_row_r  (a4) ; tgsw = [2l][2][N] */
void     or_external_product(const or_params* P, const uint32_t* tgsw, const uint32_t* acc, uint32_t* out);
/* acc <- acc + ExtProd(tgsw, (X^abar - 1) acc)  (one CMux step, a4) */
void     or_cmux_step(const or_params* P, const uint32_t* tgsw, int32_t abar, uint32_t* acc);
/* ACC <- BlindRotate(ACC = (0, X^{-bbar} v), bara); v = (mu,...,mu)  (a3, a4) */
void     or_blind_rotate(const or_params* P, const uint32_t* bk, const uint32_t* in_lwe, uint32_t mu,
                         uint32_t* acc /* [2][N] */);
void     or_sample_extract(const or_params* P, const uint32_t* acc, uint32_t* out /* N+1 */); /* a5 */
void     or_keyswitch(const or_params* P, const uint32_t* ksk, const uint32_t* in /* N+1 */,
                      uint32_t* out /* n+1 */);                                               /* a6 */
/* out(N+1) = Extract(BlindRotate(ModSwitch(in))) */
void     or_bootstrap_wo_ks(const or_params* P, const uint32_t* bk, uint32_t mu, const uint32_t* in,
                            uint32_t* out);

/* ---- gates (a1 + a7) ---- */
/* linear combination (0, C_g) + w_a ca + w_b cb; returns 0 on success, -1 for a non-2-input code */
int  or_gate_linear(const or_params* P, int gate, const uint32_t* ca, const uint32_t* cb, uint32_t* out);
/* out = bootstrapped gate (or NOT / MUX); cc only for MUX */
int  or_gate(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int gate, const uint32_t* ca,
             const uint32_t* cb, const uint32_t* cc, uint32_t* out);
/* gate[i] applied to rows i of ca/cb/cc (stride words apart) -> out row i; OpenMP over i */
int  or_gate_batch(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int64_t count,
                   const int32_t* gates, const uint32_t* ca, const uint32_t* cb, const uint32_t* cc,
                   uint32_t* out, int64_t stride, int nthreads);
/* netlist gather form: wires[out[i]] = gate[i](wires[in0[i]], wires[in1[i]], wires[in2[i]]) for one
 * level (all gates independent); OpenMP over i */
int  or_level_batch(const or_params* P, const uint32_t* bk, const uint32_t* ksk, int64_t count,
                    const int32_t* gates, const int64_t* in0, const int64_t* in1, const int64_t* in2,
                    const int64_t* outw, uint32_t* wires, int64_t stride, int nthreads);
int  or_max_threads(void);

#ifdef __cplusplus
}
#endif
#endif
