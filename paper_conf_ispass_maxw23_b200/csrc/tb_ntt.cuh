// tb_ntt.cuh -- warp-level exact negacyclic NTT of length 1024 over Z_p, p = 0x3FFF7801 (sm_100a).
//
// Role on the hot path: the "NTT" that PAPER.md names as the vectorisable part of a bootstrapped gate
// (Sec. IV-E) -- here the engine of the exact negacyclic products of the CMux.
//
// Formulation: merged-twist Cooley-Tukey forward transform with zeta_k = psi^brv10(k)
// (psi a primitive 2048-th root of unity mod p), natural-order input -> bit-reversed output; the inverse is
// the matching Gentleman-Sande transform with psi^-brv10(k); the 1/N scale is folded into the stored BK.
// One warp owns one transform: lane t holds a[t + 32 j] (j < 32) for stages 0-4 (strides 512..32: the
// butterfly partner is in the same lane and the twiddle is warp-uniform -> constant bank operands), one
// transpose through a padded 32x33 shared buffer, then a[32 t + j] for stages 5-9 (per-lane twiddles from a
// shared table).  Harvey lazy reduction with Shoup multiplication: values stay < 4p < 2^32.
#pragma once
#include "tb_common.cuh"

namespace tb {

// warp-uniform twiddles of stages 0-4 (k = 1..31) and their Shoup companions floor(w 2^32 / p).
// (The library is one translation unit, tb_lib.cu, so these are defined here.)
__constant__ uint32_t c_fw[32], c_fwp[32], c_iw[32], c_iwp[32];
// misc constants: [0] = 2^32 mod p, [1] = Shoup(2^32 mod p), [2] = 2p (as a constant-bank operand, below),
// [3] = the gadget decomposition offset
__constant__ uint32_t c_misc[4];
// Always 0.  Butterfly sums are written as x + y + c_zero: a three-input add can only be an ALU IADD3, while
// a plain x + y is often emitted as IMAD.IADD on the FMA pipe -- the pipe the Shoup products saturate
// (measured: ~150 of the ~640 butterfly adds per thread and transform pair went to IMAD.IADD, 12 % more
// FMA-pipe cycles).
__constant__ uint32_t c_zero;
__device__ __forceinline__ uint32_t add_alu(uint32_t a, uint32_t b) { return a + b + c_zero; }
// a - b + 2p with 2p from the constant bank: one IADD3 (with the immediate, ptxas splits off a - b as IMAD.IADD)
__device__ __forceinline__ uint32_t sub_alu(uint32_t a, uint32_t b) { return a - b + c_misc[2]; }

__device__ __forceinline__ uint32_t shoup_mul(uint32_t y, uint32_t w, uint32_t wp) {
    // y * w mod p in [0, 2p) for any y < 2^32 (Shoup)
    const uint32_t q = __umulhi(y, wp);
    return y * w - q * kP;
}
__device__ __forceinline__ uint32_t red_2p(uint32_t x) { return min(x, x - kTwoP); }  // [0,4p) -> [0,2p)
__device__ __forceinline__ uint32_t red_p(uint32_t x) { return min(x, x - kP); }      // [0,2p) -> [0,p)

// element (row, col) of a 32x32 transpose buffer: padded rows of 33 words, or 32-word rows with the column
// XOR-swizzled by the row (both conflict-free for row-wise and column-wise warp access)
template <bool SWZ>
__device__ __forceinline__ int sidx(int row, int col) {
    return SWZ ? ((row << 5) | (col ^ row)) : row * kPadRow + col;
}

// CT butterfly, inputs and outputs in [0, 4p)
__device__ __forceinline__ void ct_bfly(uint32_t& x, uint32_t& y, uint32_t w, uint32_t wp) {
    const uint32_t X = red_2p(x);
    const uint32_t T = shoup_mul(y, w, wp);
    x = add_alu(X, T);
    y = sub_alu(X, T);
}
// GS butterfly, inputs and outputs in [0, 2p)
__device__ __forceinline__ void gs_bfly(uint32_t& x, uint32_t& y, uint32_t w, uint32_t wp) {
    const uint32_t S = red_2p(add_alu(x, y));
    const uint32_t D = sub_alu(x, y);
    x = S;
    y = shoup_mul(D, w, wp);
}

// Forward NTT.  In: x[j] = a[lane + 32 j] (< 4p).  Out: x[j] = A[32 lane + j] (< 4p).
// buf: warp-private 32x33 shared buffer.  twT: shared per-lane twiddle table [31][32] (w, w').
template <bool SWZ = false>
__device__ __forceinline__ void ntt_fwd(uint32_t (&x)[32], uint32_t* buf, const uint2* twT, int lane) {
#pragma unroll
    for (int s = 0; s < 5; s++) {
        const int len = 16 >> s;
#pragma unroll
        for (int bj = 0; bj < (1 << s); bj++) {
            const uint32_t w = c_fw[(1 << s) + bj], wp = c_fwp[(1 << s) + bj];
#pragma unroll
            for (int u = 0; u < len; u++) ct_bfly(x[bj * 2 * len + u], x[bj * 2 * len + u + len], w, wp);
        }
    }
#pragma unroll
    for (int j = 0; j < 32; j++) buf[sidx<SWZ>(j, lane)] = x[j];
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 32; j++) x[j] = buf[sidx<SWZ>(lane, j)];
#pragma unroll
    for (int s = 5; s < 10; s++) {
        const int len = 16 >> (s - 5);
#pragma unroll
        for (int bj = 0; bj < 16 / len; bj++) {
            const uint2 tw = twT[((1 << (s - 5)) - 1 + bj) * 32 + lane];
#pragma unroll
            for (int u = 0; u < len; u++) ct_bfly(x[bj * 2 * len + u], x[bj * 2 * len + u + len], tw.x, tw.y);
        }
    }
}

// Inverse NTT (without the 1/N factor).  In: x[j] = A[32 lane + j] (< 2p).  Out: x[j] = N a[lane + 32 j] (< 2p).
template <bool SWZ = false>
__device__ __forceinline__ void ntt_inv(uint32_t (&x)[32], uint32_t* buf, const uint2* twTi, int lane) {
#pragma unroll
    for (int s = 9; s >= 5; s--) {
        const int len = 16 >> (s - 5);
#pragma unroll
        for (int bj = 0; bj < 16 / len; bj++) {
            const uint2 tw = twTi[((1 << (s - 5)) - 1 + bj) * 32 + lane];
#pragma unroll
            for (int u = 0; u < len; u++) gs_bfly(x[bj * 2 * len + u], x[bj * 2 * len + u + len], tw.x, tw.y);
        }
    }
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 32; j++) buf[sidx<SWZ>(lane, j)] = x[j];
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 32; j++) x[j] = buf[sidx<SWZ>(j, lane)];
#pragma unroll
    for (int s = 4; s >= 0; s--) {
        const int len = 16 >> s;
#pragma unroll
        for (int bj = 0; bj < (1 << s); bj++) {
            const uint32_t w = c_iw[(1 << s) + bj], wp = c_iwp[(1 << s) + bj];
#pragma unroll
            for (int u = 0; u < len; u++) gs_bfly(x[bj * 2 * len + u], x[bj * 2 * len + u + len], w, wp);
        }
    }
}

// centred lift of v in [0, 2p) (an exact integer |z| < p/2 mod p) to z mod 2^32
__device__ __forceinline__ uint32_t lift_centred(uint32_t v) {
    v = red_p(v);
    return v > kHalfP ? v - kP : v;
}

}  // namespace tb
