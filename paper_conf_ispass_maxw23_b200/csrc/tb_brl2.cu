// tb_brl2.cu -- latency-mode blind rotation on the FP64 pipe: one bootstrap per thread-block cluster of TWO SMs
// (SURVEY 8(f) f4 "single-gate latency path ... split across a thread-block cluster").
//
// brl's arithmetic, transforms and hand-over protocol (tb_brl.cu, same exact FFT-domain products, bit-identical
// output) with the cluster halved: CTA q (rank q) owns output polynomial q and BOTH 16-bit BK halves h, so
//   * it computes the 3 digit rows of ACC[q] (3 forward transforms on warp pairs 0-2),
//   * its MAC is split by bloc like brl's: the own rows times BK_i for the partner's two outputs 2(1-q) + h go to
//     CTA 1-q per thread with st.async (16 KB; round 1 pushed the three rows, 24 KB, with bulk copies), then the
//     own rows for the own outputs o = 2q + h, plus the partner's partials of those (1.92 -> 1.82 ms for one gate),
//   * warp pairs 0 and 1 run the two inverse transforms side by side (h = 0, 1), and the halves meet locally:
//     ACC[q] += lo + 2^16 hi with no second hand-over.
// Per CMux step that is brl's forward phase, twice its MAC, the same inverse latency (two transforms in parallel
// instead of one) and one DSMEM hand-over instead of two, on half the SMs: 74 bootstraps fit one wave on B200 (brl:
// 32), which is what levels of 33-148 bootstraps need (br9 and brtl were 3.5-4.7 ms there).
// Shared memory: BK_i for both halves is 96 KB, so it is single-buffered -- step i + 1's BK is requested as soon as
// step i's MAC has read it, and lands during the inverse, the ACC update and the next forward phase.
#include "tb_fft.cuh"
#include "tb_kernels.cuh"

namespace tb {

struct __align__(128) Brl2Smem {
    double2 bk[2][kRows][512];                 // BK_i (issue_bk_l2), h = 0, 1 (96 KB)
    double2 dslot[kL][512];                    // own forward rows (bloc q), swizzled positions
    double2 precv[2][2][512];                  // the partner's partial MACs of this CTA's outputs, by step parity
    double2 oslot[2][512];                     // MAC outputs (h = 0, 1), then the inverses' exchange buffers
    uint32_t res[2][kN];                       // rounded halves, h = 0 (lo) and 1 (hi, << 16)
    uint32_t acc[3 * kN];                      // ACC[q] as (acc, -acc, acc)
    uint16_t bar[kn + 2];
    unsigned long long mbar_bk, mbar_part[2];
};

// BK_i -> bk (one thread): slot (h, r) = the own bloc's row 3q + (r mod 3) of output 2q + h (r < 3) and of the
// partner's output 2(1-q) + h (r >= 3)
__device__ __forceinline__ void issue_bk_l2(Brl2Smem& S, const double2* bkf, int i, int q) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mb_expect(&S.mbar_bk, 2 * kRows * 512 * 16);
#pragma unroll
    for (int h = 0; h < 2; h++)
#pragma unroll
        for (int r = 0; r < kRows; r++) {
            const size_t row = (size_t)(i * kRows + kL * q + r % kL) * 4 + (r < kL ? 2 * q + h : 2 * (1 - q) + h);
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    sm32(S.bk[h][r])),
                "l"(bkf + row * 512), "r"(512 * 16), "r"(sm32(&S.mbar_bk))
                : "memory");
        }
}

constexpr int kBk2Issuer = 128;   // issues the per-step BK TMA: warp 4 has no inverse to run

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kLThreads, 1)
    brl2_kernel(BrArgs A, const double2* __restrict__ bkf, const double2* __restrict__ twL) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Brl2Smem& S = *reinterpret_cast<Brl2Smem*>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t rank = cl_rank();
    const int q = (int)rank;
    const int gl = blockIdx.x >> 1;                      // one lane (bootstrap) per cluster

    if (tid == 0) {
        mb_init(&S.mbar_bk);
        for (int b = 0; b < 2; b++) mb_init(&S.mbar_part[b]);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int b = 0; b < 2; b++) mb_expect(&S.mbar_part[b], 2 * 512 * 16);   // partials of steps 0 and 1
    }
    __syncthreads();
    if (tid == 0) issue_bk_l2(S, bkf, 0, q);
    {   // a1, a2 (both CTAs of the cluster)
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t sa = d.sel & 3u, sb = (d.sel >> 2) & 3u;
        const uint32_t* s0 = sa == 0 ? A.src0 : (sa == 1 ? A.src1 : A.src2);
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = tid; w <= kn; w += kLThreads) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[w] = (uint16_t)((v + (1u << 20)) >> 21);
        }
    }
    __syncthreads();
    for (int k = tid; k < kN; k += kLThreads) {           // a3: ACC[0] = 0, ACC[1] = X^{-bbar} (mu, ..., mu)
        const uint32_t bbar = S.bar[kn];
        const uint32_t v = q == 0 ? 0u : (((k + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu));
        S.acc[k] = S.acc[k + 2 * kN] = v;
        S.acc[k + kN] = 0u - v;
    }
    cl_sync();                                            // every mbarrier of the cluster is initialised and armed

    const int tt = (warp & 1) * 32 + lane;               // thread index within its warp pair
    const int jd = warp >> 1;                             // forward role: digit jd of bloc q (warp pairs 0-2);
                                                          // inverse role: half h = jd (warp pairs 0-1)
    const int shift = 32 - kBgbit * (jd < kL ? jd + 1 : 1);
    PassTw t1, t2, t3;
    t1.a = dcplx{c_zeta[0].x, c_zeta[0].y};
    t1.b = dcplx{c_zeta[1].x, c_zeta[1].y};
    t1.c = dcplx{c_zeta[3].x, c_zeta[3].y};
    t2.a = ldc(twL + tt * 6 + 0);
    t2.b = ldc(twL + tt * 6 + 1);
    t2.c = ldc(twL + tt * 6 + 2);
    t3.a = ldc(twL + tt * 6 + 3);
    t3.b = ldc(twL + tt * 6 + 4);
    t3.c = ldc(twL + tt * 6 + 5);
    const uint32_t part_dst = cl_map(sm32(&S.precv[0][0][0]), rank ^ 1u);
    const uint32_t part_mb = cl_map(sm32(&S.mbar_part[0]), rank ^ 1u);

    for (int i = 0; i < kn; i++) {
        const int buf = i & 1;
        const uint32_t par = (uint32_t)((i >> 1) & 1);
        if (jd < kL) {   // ---- A: digit jd of (X^abar - 1) ACC[q], folded, forward transform (warp pair jd) ----
            const uint32_t ab = S.bar[i];
            const uint32_t* win = S.acc + ((tt - (int)ab) & (kTwoN - 1));
            dcplx x[8];
#pragma unroll
            for (int v = 0; v < 8; v++) {
                const int c = gp1(tt, v);
                const uint32_t u0 = win[64 * v] - S.acc[c] + kDecompOffset;
                const uint32_t u1 = win[64 * v + 512] - S.acc[c + 512] + kDecompOffset;
                x[v] = dcplx{small_to_double((u0 >> shift) & 127u, 64.0), small_to_double((u1 >> shift) & 127u, 64.0)};
            }
            fwd2w(x, S.dslot[jd], t1, t2, t3, tt, 1 + jd);
        }
        __syncthreads();
        mb_wait(&S.mbar_bk, (uint32_t)(i & 1));
        // ---- B: the MAC split by bloc (brl's partial exchange): own rows x BK_i for the own outputs 2q + h and for
        // the partner's outputs 2(1-q) + h; the partner's partials go out per thread with st.async (16 KB) ----
        dcplx m3[kLMacIt][2];
#pragma unroll
        for (int e = 0; e < kLMacIt; e++) {
            const int k = tid + kLThreads * e;
            dcplx s0 = {0.0, 0.0}, s1 = {0.0, 0.0}, p0 = {0.0, 0.0}, p1 = {0.0, 0.0};
            if (k < 512) {
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const dcplx d = ldc(&S.dslot[r][lsw(k)]);
                    const dcplx c0 = ldc(&S.bk[0][kL + r][k]), c1 = ldc(&S.bk[1][kL + r][k]);
                    p0.re = fma(d.re, c0.re, fma(-d.im, c0.im, p0.re));
                    p0.im = fma(d.re, c0.im, fma(d.im, c0.re, p0.im));
                    p1.re = fma(d.re, c1.re, fma(-d.im, c1.im, p1.re));
                    p1.im = fma(d.re, c1.im, fma(d.im, c1.re, p1.im));
                }
                asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.f64 [%0], {%1, %2}, [%3];" ::"r"(
                                 part_dst + (uint32_t)(((buf * 2 + 0) * 512 + k) * 16)),
                             "d"(p0.re), "d"(p0.im), "r"(part_mb + (uint32_t)(buf * 8))
                             : "memory");
                asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.f64 [%0], {%1, %2}, [%3];" ::"r"(
                                 part_dst + (uint32_t)(((buf * 2 + 1) * 512 + k) * 16)),
                             "d"(p1.re), "d"(p1.im), "r"(part_mb + (uint32_t)(buf * 8))
                             : "memory");
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const dcplx d = ldc(&S.dslot[r][lsw(k)]);
                    const dcplx b0 = ldc(&S.bk[0][r][k]), b1 = ldc(&S.bk[1][r][k]);
                    s0.re = fma(d.re, b0.re, fma(-d.im, b0.im, s0.re));
                    s0.im = fma(d.re, b0.im, fma(d.im, b0.re, s0.im));
                    s1.re = fma(d.re, b1.re, fma(-d.im, b1.im, s1.re));
                    s1.im = fma(d.re, b1.im, fma(d.im, b1.re, s1.im));
                }
            }
            m3[e][0] = s0;
            m3[e][1] = s1;
        }
        mb_wait(&S.mbar_part[buf], par);
#pragma unroll
        for (int e = 0; e < kLMacIt; e++) {
            const int k = tid + kLThreads * e;
            if (k < 512) {
                const dcplx r0 = ldc(&S.precv[buf][0][k]), r1 = ldc(&S.precv[buf][1][k]);
                stc(&S.oslot[0][lsw(k)], dcplx{m3[e][0].re + r0.re, m3[e][0].im + r0.im});
                stc(&S.oslot[1][lsw(k)], dcplx{m3[e][1].re + r1.re, m3[e][1].im + r1.im});
            }
        }
        __syncthreads();                                  // bk, precv[buf] consumed; oslot complete
        if (tid == kBk2Issuer) {   // a thread of warp 4, idle during the two inverses (warp pairs 0 and 1)
            if (i + 2 < kn) mb_expect(&S.mbar_part[buf], 2 * 512 * 16);    // partials of step i + 2
            if (i + 1 < kn) issue_bk_l2(S, bkf, i + 1, q);                  // lands during C and the next A
        }
        if (jd < 2) {   // ---- C: inverse of half h = jd (warp pair jd), round, << 16 h ----
            dcplx x[8];
            inv2w(x, S.oslot[jd], t1, t2, t3, tt, 4 + jd);
#pragma unroll
            for (int v = 0; v < 8; v++) {
                const int c = gp1(tt, v);
                S.res[jd][c] = round_mod32(x[v].re) << (16 * jd);
                S.res[jd][c + 512] = round_mod32(x[v].im) << (16 * jd);
            }
        }
        __syncthreads();
        for (int c = tid; c < kN; c += kLThreads) {       // ACC[q] += lo + 2^16 hi
            const uint32_t nv = S.acc[c] + S.res[0][c] + S.res[1][c];
            S.acc[c] = nv;
            S.acc[c + kN] = 0u - nv;
            S.acc[c + 2 * kN] = nv;
        }
        __syncthreads();
    }
    cl_sync();
    if (gl < A.nlanes) {   // a5: CTA 0 holds ACC.a, CTA 1 holds ACC.b
        uint32_t* out = A.out + (int64_t)gl * A.out_stride;
        if (q == 0) {
            for (int j = tid; j < kN; j += kLThreads) out[j] = j == 0 ? S.acc[0] : 0u - S.acc[kN - j];
        } else if (tid == 0) {
            out[kN] = S.acc[0];
        }
    }
}

static int brl2_attr() {
    if (ensure_smem_attr<brl2_kernel>(sizeof(Brl2Smem))) return -1;
    return 0;
}

// clusters of brl2 that are co-resident on the device (one wave of bootstraps), or <= 0 on error
int brl2_wave_lanes() {
    if (brl2_attr()) return -1;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3(2 * 256);
    cfg.blockDim = dim3(kLThreads);
    cfg.dynamicSmemBytes = sizeof(Brl2Smem);
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, brl2_kernel, &cfg) != cudaSuccess) return -1;
    return n;
}

int launch_brl2(const BrArgs& A, const double2* bkf, const double2* twL, cudaStream_t st) {
    const size_t smem = sizeof(Brl2Smem);
    static_assert(sizeof(Brl2Smem) <= 232448, "brl2 shared memory");
    if (brl2_attr()) return -1;
    if (A.nlanes <= 0) return 0;
    brl2_kernel<<<2 * A.nlanes, kLThreads, smem, st>>>(A, bkf, twL);
    return 0;
}

}  // namespace tb
