// tb_fft.cuh -- warp-level negacyclic transform of length 1024 in double precision, on the FP64 pipe (sm_100a).
//
// Alternative engine for the exact products of the CMux: a real polynomial
// a mod X^1024 + 1 is folded to z = a mod (X^512 - i), z_k = a_k + i a_{k+512}, and transformed by stages 1..9
// of the merged-twist Cooley-Tukey tree of X^1024 + 1 (zeta_{s,b} = psi^brv10(2^s + b), psi = e^{i pi/1024}),
// i.e. evaluated at the 512 roots of X^512 = i.  Pointwise products + the Gentleman-Sande inverse + unfold give
// the negacyclic product.  With 16-bit signed BK halves every product coefficient is an integer of magnitude
// <= 6 * 1024 * 64 * 2^15 = 2^33.6 and the rounding error of the whole pipeline is < 1e-3, so rounding to the
// nearest integer recovers it exactly.
//
// One warp owns one transform, 16 complex values per lane, three register layouts (k = transform index):
//   A: k = t + 32 j                  stages 1-4 in-thread, warp-uniform twiddles (constant bank)
//   B: k = 32 (t>>1) + 2 j + (t&1)   stages 5-8 in-thread, per-lane twiddles (one shared base per stage)
//   D: k = 16 t + 2 (j&7) + (j>>3)   stage 9 pairs lanes t, t^1: each lane sends 8 values with one shuffle
//                                    each and computes 8 butterflies (per-lane twiddles from one base)
// D is the frequency-domain layout every caller (BK, MAC) uses.  The A <-> B transpose goes through a 512 x 16-B
// shared buffer whose 16-B granules are XOR-swizzled so that every access pattern is bank-conflict free.
#pragma once
#include "tb_common.cuh"

namespace tb {

// stages 1-4 twiddles: index (2^(s-1) - 1) + b for s = 1..4 (15 entries), as (re, im)
__constant__ double2 c_zeta[16];
// Per-lane twiddles of stages 5-9 from one base per stage.  In layout B the in-thread block bj of stage s
// (5 <= s <= 8) has zeta = psi^brv10(2^s + u 2^(s-5) + bj), u = lane >> 1; the bits of bj land on exponent
// bits 9, 8, 7, so zeta = base_s(u) * e^{i pi brv(bj) / 2^(s-5)} with base_s(u) = psi^brv10(2^s + u 2^(s-5)).
// Stage 9 (lane t, butterfly m) likewise: zeta = psi^brv10(512 + 8t + m) = base_9(t) * e^{i pi brv3(m) / 8}.
// The factors are 1, i (free) and e^{i pi/4}, e^{i pi/8}, e^{i 3pi/8} (one constant complex product each), so
// a transform reads 5 bases instead of 23 twiddles.  Tables: twB = [4][16] (stage 5..8, lane pair),
// twC = [32] (stage 9, lane).
constexpr int kTwB = 4 * 16;
constexpr int kTwC = 32;

struct dcplx {
    double re, im;
};

__device__ __forceinline__ dcplx mul_i(dcplx a) { return dcplx{-a.im, a.re}; }
__device__ __forceinline__ dcplx mul_k(dcplx a, double cr, double ci) {   // a * (cr + i ci)
    return dcplx{fma(a.re, cr, -a.im * ci), fma(a.re, ci, a.im * cr)};
}
// base * e^{i pi brv(bj) / NB} for the NB in-thread blocks of a stage (bj a compile-time constant after unrolling)
template <int NB>
__device__ __forceinline__ dcplx tw_factor(dcplx b, int bj) {
    constexpr double c4 = 0.70710678118654752440, c8 = 0.92387953251128675613, s8 = 0.38268343236508977173;
    const int m = bj >> 1;                 // the odd blocks are i times the even ones (brv puts bit 0 on top)
    dcplx w = b;
    if (NB >= 4 && (m & 1)) w = mul_k(b, c4, c4);                                  // e^{i pi/4}
    if (NB == 8 && m == 2) w = mul_k(b, c8, s8);                                   // e^{i pi/8}
    if (NB == 8 && m == 3) w = mul_k(b, s8, c8);                                   // e^{i 3pi/8}
    return (NB >= 2 && (bj & 1)) ? mul_i(w) : w;
}

__device__ __forceinline__ int fswz(int k) {   // swizzled 16-B slot of transform index k
    return (k & ~7) | ((k ^ ((k >> 4) & 1) ^ (((k >> 5) & 3) << 1)) & 7);
}
__device__ __forceinline__ int lay_a(int t, int j) { return t + 32 * j; }
__device__ __forceinline__ int lay_b(int t, int j) { return ((t >> 1) << 5) | (j << 1) | (t & 1); }
__device__ __forceinline__ int lay_c(int t, int j) { return (t << 4) | j; }
__device__ __forceinline__ int lay_d(int t, int j) { return (t << 4) | ((j & 7) << 1) | (j >> 3); }

__device__ __forceinline__ dcplx cmul(dcplx w, dcplx y) {
    dcplx r;
    r.re = fma(w.re, y.re, -w.im * y.im);
    r.im = fma(w.re, y.im, w.im * y.re);
    return r;
}
__device__ __forceinline__ dcplx cmulc(dcplx w, dcplx y) {   // conj(w) * y
    dcplx r;
    r.re = fma(w.re, y.re, w.im * y.im);
    r.im = fma(w.re, y.im, -w.im * y.re);
    return r;
}
// (x, y) <- (x + w y, x - w y) in 6 DFMA: x' = x + w y by two chained FMAs per component, y' = 2x - x'
__device__ __forceinline__ void ct_c(dcplx& x, dcplx& y, dcplx w) {
    const double xr = fma(w.re, y.re, fma(-w.im, y.im, x.re));
    const double xi = fma(w.re, y.im, fma(w.im, y.re, x.im));
    y.re = fma(2.0, x.re, -xr);
    y.im = fma(2.0, x.im, -xi);
    x.re = xr;
    x.im = xi;
}
__device__ __forceinline__ void gs_c(dcplx& x, dcplx& y, dcplx w) {
    const dcplx d = {x.re - y.re, x.im - y.im};
    x.re += y.re;
    x.im += y.im;
    y = cmulc(w, d);
}
__device__ __forceinline__ dcplx ld_tw(const double2* t, int idx) {
    const double2 v = t[idx];
    return dcplx{v.x, v.y};
}

// One stage on 16 in-thread values: blocks of 2*LJ, NB blocks, twiddle of block bj from (a) the constant bank
// (layout A: index CB + bj) or (b) a per-lane-pair shared table (index (TB + bj) * 16 + (lane >> 1)).  Explicit template
// instantiation keeps every register index a compile-time constant.
template <int LJ, int NB, int CB>
__device__ __forceinline__ void ct_stage_const(dcplx (&x)[16]) {
#pragma unroll
    for (int bj = 0; bj < NB; bj++) {
        const double2 z = c_zeta[CB + bj];
        const dcplx w = {z.x, z.y};
#pragma unroll
        for (int u = 0; u < LJ; u++) ct_c(x[bj * 2 * LJ + u], x[bj * 2 * LJ + u + LJ], w);
    }
}
template <int LJ, int NB, int CB>
__device__ __forceinline__ void gs_stage_const(dcplx (&x)[16]) {
#pragma unroll
    for (int bj = 0; bj < NB; bj++) {
        const double2 z = c_zeta[CB + bj];
        const dcplx w = {z.x, z.y};
#pragma unroll
        for (int u = 0; u < LJ; u++) gs_c(x[bj * 2 * LJ + u], x[bj * 2 * LJ + u + LJ], w);
    }
}
template <int LJ, int NB, int TB>
__device__ __forceinline__ void ct_stage_tab(dcplx (&x)[16], const double2* tw, int lane) {
    const dcplx base = ld_tw(tw, TB * 16 + (lane >> 1));
#pragma unroll
    for (int bj = 0; bj < NB; bj++) {
        const dcplx w = tw_factor<NB>(base, bj);
#pragma unroll
        for (int u = 0; u < LJ; u++) ct_c(x[bj * 2 * LJ + u], x[bj * 2 * LJ + u + LJ], w);
    }
}
template <int LJ, int NB, int TB>
__device__ __forceinline__ void gs_stage_tab(dcplx (&x)[16], const double2* tw, int lane) {
    const dcplx base = ld_tw(tw, TB * 16 + (lane >> 1));
#pragma unroll
    for (int bj = 0; bj < NB; bj++) {
        const dcplx w = tw_factor<NB>(base, bj);
#pragma unroll
        for (int u = 0; u < LJ; u++) gs_c(x[bj * 2 * LJ + u], x[bj * 2 * LJ + u + LJ], w);
    }
}

// 16 values through the transpose buffer: write at layout FROM, read at layout TO (0 = A, 1 = B, 2 = C)
template <int FROM, int TO>
__device__ __forceinline__ void fft_transpose(dcplx (&x)[16], double2* buf, int lane) {
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 16; j++) {
        const int k = FROM == 0 ? lay_a(lane, j) : (FROM == 1 ? lay_b(lane, j) : lay_c(lane, j));
        buf[fswz(k)] = make_double2(x[j].re, x[j].im);
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 16; j++) {
        const int k = TO == 0 ? lay_a(lane, j) : (TO == 1 ? lay_b(lane, j) : lay_c(lane, j));
        const double2 v = buf[fswz(k)];
        x[j] = dcplx{v.x, v.y};
    }
}

__device__ __forceinline__ dcplx sel(bool p, dcplx a, dcplx b) { return p ? a : b; }
__device__ __forceinline__ dcplx shfl_x1(dcplx v) {
    return dcplx{__shfl_xor_sync(0xffffffffu, v.re, 1), __shfl_xor_sync(0xffffffffu, v.im, 1)};
}

// stage 9 forward: B -> D.  Lane pair (t even, t odd) holds positions 2b, 2b+1 of block b = 16 (t>>1) + j in
// x[j]; the even lane computes the butterflies j < 8, the odd lane j >= 8 (block b = 8 t + m, m < 8).
__device__ __forceinline__ void stage9_fwd(dcplx (&x)[16], const double2* twC, int lane) {
    const bool p = lane & 1;
    const dcplx base = ld_tw(twC, lane);
#pragma unroll
    for (int m = 0; m < 8; m++) {
        const dcplx r = shfl_x1(sel(p, x[m], x[m + 8]));
        dcplx e = sel(p, r, x[m]), o = sel(p, x[m + 8], r);
        ct_c(e, o, tw_factor<8>(base, m));
        x[m] = e;
        x[m + 8] = o;
    }
}
// stage 9 inverse: D -> B
__device__ __forceinline__ void stage9_inv(dcplx (&x)[16], const double2* twC, int lane) {
    const bool p = lane & 1;
    const dcplx base = ld_tw(twC, lane);
#pragma unroll
    for (int m = 0; m < 8; m++) {
        gs_c(x[m], x[m + 8], tw_factor<8>(base, m));
        const dcplx r = shfl_x1(sel(p, x[m], x[m + 8]));
        if (p) x[m] = r;
        else x[m + 8] = r;
    }
}

// buf: 512 x double2 (8 KB) warp-private; twB: [4][16] stage 5-8 bases per lane pair; twC: [32] stage 9 bases
// In: x[j] = z[lay_a(lane, j)].  Out: x[j] = Z[lay_d(lane, j)] (bit-reversed-order transform positions).
__device__ __forceinline__ void fft_fwd(dcplx (&x)[16], double2* buf, const double2* twB, const double2* twC,
                                        int lane) {
    ct_stage_const<8, 1, 0>(x);       // stage 1 (pairs k bit 8)
    ct_stage_const<4, 2, 1>(x);       // stage 2
    ct_stage_const<2, 4, 3>(x);       // stage 3
    ct_stage_const<1, 8, 7>(x);       // stage 4
    fft_transpose<0, 1>(x, buf, lane);
    ct_stage_tab<8, 1, 0>(x, twB, lane);    // stage 5 (pairs k bit 4)
    ct_stage_tab<4, 2, 1>(x, twB, lane);    // stage 6
    ct_stage_tab<2, 4, 2>(x, twB, lane);    // stage 7
    ct_stage_tab<1, 8, 3>(x, twB, lane);    // stage 8
    stage9_fwd(x, twC, lane);               // stage 9 (pairs k bit 0)
}

// In: x[j] = Z[lay_d(lane, j)].  Out: x[j] = 512 z[lay_a(lane, j)] (the 1/512 is folded into the stored BK).
__device__ __forceinline__ void fft_inv(dcplx (&x)[16], double2* buf, const double2* twB, const double2* twC,
                                        int lane) {
    stage9_inv(x, twC, lane);               // stage 9
    gs_stage_tab<1, 8, 3>(x, twB, lane);    // stage 8
    gs_stage_tab<2, 4, 2>(x, twB, lane);    // stage 7
    gs_stage_tab<4, 2, 1>(x, twB, lane);    // stage 6
    gs_stage_tab<8, 1, 0>(x, twB, lane);    // stage 5
    fft_transpose<1, 0>(x, buf, lane);
    gs_stage_const<1, 8, 7>(x);       // stage 4
    gs_stage_const<2, 4, 3>(x);       // stage 3
    gs_stage_const<4, 2, 1>(x);       // stage 2
    gs_stage_const<8, 1, 0>(x);       // stage 1
}

__device__ __forceinline__ double small_to_double(uint32_t v, double bias) {   // v < 2^31 exactly, minus bias
    return __hiloint2double(0x43300000, (int)v) - (4503599627370496.0 + bias);
}

// exact integer value (|v| < 2^51) of a double that is within 0.5 of it, reduced mod 2^32
__device__ __forceinline__ uint32_t round_mod32(double v) {
    return (uint32_t)__double2loint(v + 6755399441055744.0);   // 1.5 * 2^52: mantissa holds v + 2^51
}

}  // namespace tb
