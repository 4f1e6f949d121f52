// tb_brtl.cu -- latency-mode blind rotation on the tensor cores: one bootstrap per SM (SURVEY 8(f) f4,
// single-gate latency; P:299 / P:303 -- narrow, serial levels are bound by the 630-step chain of one gate).
//
// Same arithmetic as brt_kernel (tb_brt.cu): the four-step NTTs of the CMux as
// tcgen05.mma.kind::i8 byte-limb GEMMs, the MAC against the four-step BK records, centred lift -- bit-identical to
// every other variant.  What changes is the shape: one lane (6 + 6 polynomials = 2 M-tiles per stage) on a whole SM,
// 16 warps, every stage synchronous (thread 0 issues, everyone waits on the commit): a CMux step costs 4 small GEMMs
// + 4 short epilogues (16 values per thread) + a MAC over 2 coefficients per thread.  A level of <= 148 bootstraps
// runs in one wave (one CTA per SM): 4.6-4.7 ms for 1-148 bootstraps on B200, which beats br9 from ~75 bootstraps
// on; a single gate stays faster on brl (1.9 ms), whose 4 SMs share the step's BK stream (one SM must ingest the
// whole 147 KB of BK records per step here; requesting them at the top of the step was measured slower, 5.3 ms:
// the 18 16-byte loads per thread throttle the load queue and the registers they hold spill).
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"
#include "tb_tc.cuh"

namespace tb {

constexpr int kTlWarps = 16;
constexpr int kTlThreads = 32 * kTlWarps;
constexpr int kTlTiles = 2;
#ifndef TB_BRTL_BK
#define TB_BRTL_BK 0                          // BK records: 0 = all at the top of the step, 1 = split, 2 = in the MAC
#endif                   // polys 0-3 and 4-5 (rows 64-127 of tile 1 are padding)

struct BrtlSmem {
    unsigned char B[kTcBTotal];               // constant B operands (the same as brt_kernel's)
    unsigned char op[kTlTiles * kOpTile];     // per tile: A1 | A2 | MAC in / out = A3 | A4
    uint2 twF[32 * 32];
    uint2 twI[32 * 32];
    uint32_t acc[2][kN];
    uint16_t bar[kn + 2];
    uint64_t mbar;
    uint32_t tmem;
};

// one synchronous GEMM stage: stage 0 = A1 x B1 (K = 32, s8 digits), 1..3 = op x B2 / B3 / B4 (K = 128)
__device__ __forceinline__ void brtl_gemm(BrtlSmem& S, int stage, uint32_t& phase) {
    fence_async_smem();
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x == 0) {
        tc_fence_after();
        const uint32_t sB = smem_u32(S.B), sOp = smem_u32(S.op);
        constexpr uint32_t id_s = tc_idesc_i8(128, 128, true, false), id_u = tc_idesc_i8(128, 128, false, false);
        for (int t = 0; t < kTlTiles; t++) {
            const uint32_t d = S.tmem + 128 * t, a = sOp + t * kOpTile;
            if (stage == 0) {
                tc_mma_i8(d, tc_sdesc(a, kA1Lbo, kA1Sbo), tc_sdesc(sB, 128, 256), id_s, 0);
            } else {
                const uint32_t bb = sB + kB1Bytes + (stage - 1) * kBBytes;
#pragma unroll
                for (int q = 0; q < 4; q++)
                    tc_mma_i8(d, tc_sdesc(a + 2 * q * kOpLbo, kOpLbo, kOpSbo), tc_sdesc(bb + 2 * q * 128, 128, 1024),
                              id_u, q > 0);
            }
        }
        tc_commit(smem_u32(&S.mbar));
    }
    mbar_wait(&S.mbar, phase);
    phase ^= 1;
    tc_fence_after();
}

__global__ void __launch_bounds__(kTlThreads, 1) brtl_kernel(BrArgs A, const uint32_t* __restrict__ bk4,
                                                              const unsigned char* __restrict__ tcB,
                                                              const uint2* __restrict__ tcTw) {
    extern __shared__ __align__(1024) unsigned char brtl_smem[];
    BrtlSmem& S = *reinterpret_cast<BrtlSmem*>(brtl_smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int gl = blockIdx.x;                               // one lane (bootstrap) per CTA
    for (int e = tid; e < (int)(kTcBTotal / 16); e += kTlThreads)
        reinterpret_cast<uint4*>(S.B)[e] = __ldg(reinterpret_cast<const uint4*>(tcB) + e);
    for (int e = tid; e < 32 * 32; e += kTlThreads) {
        S.twF[e] = tcTw[e];
        S.twI[e] = tcTw[1024 + e];
    }
    for (int e = tid; e < kTlTiles * (int)kOpTile / 16; e += kTlThreads)   // padding rows: defined values
        reinterpret_cast<uint4*>(S.op)[e] = make_uint4(0u, 0u, 0u, 0u);
    if (warp == 0) tc_alloc<256>(&S.tmem);
    if (tid == 0) {
        mbar_init(&S.mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    {   // a1, a2: linear combination and mod switch
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t sa = d.sel & 3u, sb = (d.sel >> 2) & 3u;
        const uint32_t* s0 = sa == 0 ? A.src0 : (sa == 1 ? A.src1 : A.src2);
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = tid; w <= kn; w += kTlThreads) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[w] = (uint16_t)((v + (1u << 20)) >> 21);      // round(v 2N / 2^32) mod 2N (C5)
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    for (int c = tid; c < kN; c += kTlThreads) {                  // a3: ACC = (0, X^{-bbar} (mu, ..., mu))  (C6)
        S.acc[0][c] = 0u;
        S.acc[1][c] = ((c + S.bar[kn]) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    // epilogue roles: warps 0-7 read tile 0 (quadrant = warp % 4, column half = warp / 4); warps 8-15 tile 1, of
    // which only quadrants 0, 1 (polys 4, 5) carry data
    const int et = warp >> 3, hq = (warp >> 2) & 1, qd = warp & 3;
    const bool ework = et == 0 || qd < 2;
    const uint32_t tq = S.tmem + ((uint32_t)(32 * qd) << 16) + 128 * et + 64 * hq;
    const int P = 4 * et + qd;                                    // polynomial of this warp's TMEM quadrant
    // digits role: lanes = k2 (consecutive coefficients: conflict-free ACC reads), warp = (bloc, u4)
    const int dbloc = warp >> 3, du4 = warp & 7;
    uint32_t phase = 0;
    for (int i = 0; i < kn; i++) {
        // ---- BK records of this step's MAC (positions tid, tid + 512), in flight during the forward half
        const uint4* rec = reinterpret_cast<const uint4*>(bk4 + ((size_t)i * kN + tid) * kBk4Rec);
        // ---- a4.1 digits of (X^abar - 1) ACC[bloc]: coefficients c = 32 (4 du4 + u) + lane, u < 4
        {
            const uint32_t ab = S.bar[i];
            const uint32_t* acc = S.acc[dbloc];
            uint32_t dw[3] = {0u, 0u, 0u};
#pragma unroll
            for (int u = 0; u < 4; u++) {
                const uint32_t c = 32u * (4 * du4 + u) + lane;
                const uint32_t mm = (c - ab) & (kTwoN - 1);
                const uint32_t src = acc[mm & (kN - 1)];
                const uint32_t rot = mm < (uint32_t)kN ? src : 0u - src;
                const uint32_t x = rot - acc[c] + c_misc[3];
#pragma unroll
                for (int jd = 0; jd < 3; jd++)
                    dw[jd] |= ((((x >> (32 - kBgbit * (jd + 1))) & 127u) - 64u) & 0xFFu) << (8 * u);
            }
#pragma unroll
            for (int jd = 0; jd < 3; jd++) {
                const int PP = dbloc * 3 + jd;
                *reinterpret_cast<uint32_t*>(S.op + (PP >> 2) * kOpTile +
                                             tc_off((PP & 3) * 32 + lane, 4 * du4, kA1Lbo, kA1Sbo)) = dw[jd];
            }
        }
        brtl_gemm(S, 0, phase);
        // ---- ep1: thread (P, k2 = lane), j1 in its half: C[j1][k2] -> A2 row (P, j1), word k2
        if (ework) {
            unsigned char* base = S.op + et * kOpTile + opw(qd * 32 + 16 * hq, lane);
            const uint2* tw = S.twF + 32 * 16 * hq + lane;
#pragma unroll
            for (int jc = 0; jc < 4; jc += 2) {
                uint32_t v[2][16];
                tc_ld16(tq + 16 * jc, v[0]);
                tc_ld16(tq + 16 * jc + 16, v[1]);
                tc_wait_ld();
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int j = 4 * jc + u;
                    const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                    const uint2 w = tw[32 * j];
                    *reinterpret_cast<uint32_t*>(base + (j >> 3) * kOpSbo + (j & 7) * 16) =
                        shoup_mul(limbs_s(y[0], y[1], y[2], y[3]), w.x, w.y);
                }
            }
        }
        brtl_gemm(S, 1, phase);
        // ---- ep2: thread (P, j1 = lane), j2 in its half: A[j1 + 32 j2] in [0, 2p) -> row (P, j1), words j2
        if (ework) {
            unsigned char* base = S.op + et * kOpTile + opw(qd * 32 + lane, 16 * hq);
#pragma unroll
            for (int c = 0; c < 4; c += 2) {
                uint32_t v[2][16];
                tc_ld16(tq + 16 * c, v[0]);
                tc_ld16(tq + 16 * c + 16, v[1]);
                tc_wait_ld();
#pragma unroll
                for (int h = 0; h < 2; h++) {
                    uint4 o;
                    o.x = red_2p(limbs_u(v[h][0], v[h][1], v[h][2], v[h][3]));
                    o.y = red_2p(limbs_u(v[h][4], v[h][5], v[h][6], v[h][7]));
                    o.z = red_2p(limbs_u(v[h][8], v[h][9], v[h][10], v[h][11]));
                    o.w = red_2p(limbs_u(v[h][12], v[h][13], v[h][14], v[h][15]));
                    *reinterpret_cast<uint4*>(base + (c + h) * kOpLbo) = o;
                }
            }
        }
        tc_fence_before();
        __syncthreads();
        // ---- a4.3 MAC at positions tid and tid + 512 (j1 = pos / 32, j2 = pos % 32), in place
        {
            const uint32_t R = c_misc[0], Rp = c_misc[1];
#pragma unroll
            for (int h = 0; h < 2; h++) {
                const int pos = tid + 512 * h, j1 = pos >> 5, j2 = pos & 31;
                const uint32_t rowoff = (j1 >> 3) * kOpSbo + (j1 & 7) * 16 + (j2 >> 2) * kOpLbo + (j2 & 3) * 4;
                uint32_t* w[6];
                uint32_t D[6];
#pragma unroll
                for (int r = 0; r < 6; r++) {
                    w[r] = reinterpret_cast<uint32_t*>(S.op + (r >> 2) * kOpTile + (r & 3) * 4 * kOpSbo + rowoff);
                    D[r] = *w[r];
                }
                uint32_t B[kBk4Rec];
#pragma unroll
                for (int q = 0; q < kBk4Rec / 4; q++) {
                    const uint4 b4 = __ldg(rec + h * 512 * (kBk4Rec / 4) + q);
                    B[4 * q] = b4.x; B[4 * q + 1] = b4.y; B[4 * q + 2] = b4.z; B[4 * q + 3] = b4.w;
                }
#pragma unroll
                for (int o = 0; o < 6; o++) {
                    uint64_t s = 0;
#pragma unroll
                    for (int r = 0; r < 6; r++) s += (uint64_t)D[r] * B[r * 6 + o];
                    const uint32_t hi = (uint32_t)(s >> 32), lo = (uint32_t)s;
                    *w[o] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                }
            }
        }
        brtl_gemm(S, 2, phase);
        // ---- ep3: thread (O = P, j1 = lane), k2 in its half: E = D . psi^(-(2 j1 + 1) k2) -> A4 row of (m, q, k2)
        // (A4: tile 0 rows m * 64 + q * 32 + k2 for m = 0, 1; tile 1 rows q * 32 + k2 for m = 2)
        if (ework) {                                                // GEMM3 has consumed op (A3): rewrite as A4
            const int o = P, q = o / 3, m = o % 3;
            unsigned char* base = S.op + (m == 2 ? kOpTile : 0) + opw((m & 1) * 64 + q * 32 + 16 * hq, lane);
            const uint2* tw = S.twI + 32 * 16 * hq + lane;
#pragma unroll
            for (int c = 0; c < 4; c += 2) {
                uint32_t v[2][16];
                tc_ld16(tq + 16 * c, v[0]);
                tc_ld16(tq + 16 * c + 16, v[1]);
                tc_wait_ld();
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int j = 4 * c + u;
                    const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                    const uint2 w = tw[32 * j];
                    *reinterpret_cast<uint32_t*>(base + (j >> 3) * kOpSbo + (j & 7) * 16) =
                        shoup_mul(limbs_u(y[0], y[1], y[2], y[3]), w.x, w.y);
                }
            }
        }
        brtl_gemm(S, 3, phase);
        // ---- ep4: tile 0 quadrant qd = (m, q) for m = qd / 2; tile 1 quadrant qd = q (m = 2); k1 in its half:
        // centred lift, << 11 m, added into ACC[q] (the three parts of a coefficient add atomically)
        if (ework) {
            const int m = et == 0 ? (qd >> 1) : 2, q = et == 0 ? (qd & 1) : qd;
            uint32_t* acc = &S.acc[q][32 * 16 * hq + lane];
#pragma unroll
            for (int c = 0; c < 4; c += 2) {
                uint32_t v[2][16];
                tc_ld16(tq + 16 * c, v[0]);
                tc_ld16(tq + 16 * c + 16, v[1]);
                tc_wait_ld();
#pragma unroll
                for (int u = 0; u < 8; u++) {
                    const int j = 4 * c + u;
                    const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                    const uint32_t a = lift_centred(red_2p(limbs_u(y[0], y[1], y[2], y[3])));
                    atomicAdd(acc + 32 * j, a << (11 * m));
                }
            }
        }
        tc_fence_before();
        __syncthreads();
    }
    // a5: sample extraction, index 0 (C8)
    if (gl < A.nlanes) {
        uint32_t* out = A.out + (int64_t)gl * A.out_stride;
        for (int j = tid; j <= kN; j += kTlThreads) {
            uint32_t v;
            if (j == 0) v = S.acc[0][0];
            else if (j < kN) v = 0u - S.acc[0][kN - j];
            else v = S.acc[1][0];
            out[j] = v;
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tc_dealloc<256>(S.tmem);
}

int launch_brtl(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st) {
    static_assert(sizeof(BrtlSmem) <= 232448, "brtl shared memory");
    if (ensure_smem_attr<brtl_kernel>(sizeof(BrtlSmem))) return -1;
    if (A.nlanes <= 0) return 0;
    brtl_kernel<<<A.nlanes, kTlThreads, sizeof(BrtlSmem), st>>>(A, bk4, tcB, tcTw);
    return 0;
}

}  // namespace tb
