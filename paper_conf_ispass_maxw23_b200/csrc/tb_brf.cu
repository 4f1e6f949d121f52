// tb_brf.cu -- blind rotation on the FP64 pipe.
//
// Same CMux as br6 (bit-identical output), with the exact negacyclic products computed by the folded
// 512-point complex transform of tb_fft.cuh instead of the integer NTT: the integer kernels are bound by the
// IMAD pipe, and B200 executes DFMA at the IMAD rate on a separate pipe.  Each torus BK coefficient is split
// into two signed 16-bit halves (x = lo + 2^16 hi mod 2^32); per output polynomial q the two half products
// are exact integers of magnitude < 2^33.6, recovered by rounding, and recombined mod 2^32.
// Per CMux step, G lanes per CTA, 8 warps per lane:
//   A  warp r = bloc*3 + jd < 6: digit jd of (X^abar - 1) ACC[bloc], folded, forward transform -> slot r
//   B  thread item = position k for all G lanes: out[g][o][k] = sum_r D_{g,r}[k] * BKf_i[r][o][k] for the 4
//      outputs o = (q, half), complex FMA, written back in place (slots 0..3); each BK word is loaded once
//      per CTA and used G times
//   C  warp o < 4: inverse transform, unfold, round, (<< 16 for the high half); the two half warps of q meet
//      at a named barrier and the low-half warp adds both into ACC[q]
#include "tb_fft.cuh"
#include "tb_kernels.cuh"

namespace tb {

constexpr int kFOuts = 4;                       // (q, half)
constexpr int kFStepD2 = kRows * kFOuts * 512;  // double2 per CMux step = 196,608 B

template <int G>
struct BrfSmem {
    double2 twB[kTwB];
    double2 twC[kTwC];
    double2 slot[G][kRows][512];
    uint32_t acc[G][2][3 * kN];   // ACC polys, each stored as (acc, -acc, acc): X^{-a} ACC is a window read
    uint16_t bar[G][kn + 2];
};


// Warps per lane: W = 8 for G <= 2 (6 forward transforms, 4 inverse; 16 warps, 126 registers), W = 6 for G = 3
// (18 warps: more transforms in flight per SM; the register file is split over the 4 sub-partitions, so 5 warps
// on one of them cap the kernel at 96 registers).
template <int G>
struct BrfCfg {
    static constexpr int W = G == 3 ? 6 : 8;
    static constexpr int NT = 32 * W * G;
};

// The G lanes of the CTA move in lockstep and share every BK load in the MAC (measured: letting the lanes
// drift apart with per-lane named barriers and per-lane BK loads is 6 % slower).
template <int G>
__device__ __forceinline__ void brf_body(BrArgs A, const double2* __restrict__ bkf, const double2* __restrict__ twB,
                                         const double2* __restrict__ twC) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    BrfSmem<G>& S = *reinterpret_cast<BrfSmem<G>*>(smem_raw);
    constexpr int kFWarps = BrfCfg<G>::W, NT = BrfCfg<G>::NT, NL = 32 * kFWarps;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = warp / kFWarps, w8 = warp % kFWarps;
    const int lane0 = blockIdx.x * G;

    for (int k = tid; k < kTwB; k += NT) S.twB[k] = twB[k];
    for (int k = tid; k < kTwC; k += NT) S.twC[k] = twC[k];
    {   // a1, a2
        const int gl = lane0 + g;
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t sa = d.sel & 3u, sb = (d.sel >> 2) & 3u;
        const uint32_t* s0 = sa == 0 ? A.src0 : (sa == 1 ? A.src1 : A.src2);
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = w8 * 32 + lane; w <= kn; w += NL) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[g][w] = (uint16_t)((v + (1u << 20)) >> 21);
        }
    }
    __syncthreads();
    for (int k = tid; k < G * kN; k += NT) {                  // a3
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        const uint32_t tv = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
        S.acc[gg][0][c] = S.acc[gg][0][c + kN] = S.acc[gg][0][c + 2 * kN] = 0u;
        S.acc[gg][1][c] = S.acc[gg][1][c + 2 * kN] = tv;
        S.acc[gg][1][c + kN] = 0u - tv;
    }
    __syncthreads();

    // phase A role ra < 6: with 8 warps per lane, rotating the two idle roles by 2 per lane spreads the 6G
    // busy warps evenly over the 4 SM sub-partitions (warp w runs on sub-partition w % 4)
    const int ra = kFWarps == 8 ? (w8 + 2 * g) % kFWarps : w8;
    const int bloc = ra / kL, jd = ra % kL;
    const int q = w8 >> 1, h = w8 & 1;                        // phase C role (w8 < 4)
    const int shift = 32 - kBgbit * (jd + 1);
    for (int i = 0; i < kn; i++) {
        if (ra < kRows) {   // ---- A ----
            const uint32_t ab = S.bar[g][i];
            const uint32_t* acc = S.acc[g][bloc];
            // coefficient c of X^{-ab} ACC is ext[(c - ab) mod 2N]; with c = lane + 32 j + 512 half the index is
            // ((lane - ab) mod 2N) + 32 j + 512 half < 3N: one window base per lane, immediate offsets after it
            const uint32_t* win = acc + ((lane - ab) & (kTwoN - 1));
            dcplx x[16];
#pragma unroll
            for (int j = 0; j < 16; j++) {
                double v2[2];
#pragma unroll
                for (int half = 0; half < 2; half++) {
                    const uint32_t c = lane + 32 * j + 512 * half;
                    const uint32_t u = win[32 * j + 512 * half] - acc[c] + kDecompOffset;
                    v2[half] = small_to_double((u >> shift) & 127u, 64.0);   // digit in [-64, 63]
                }
                x[j] = dcplx{v2[0], v2[1]};                                    // fold: a_k + i a_{k+512}
            }
            double2* slot = S.slot[g][ra];
            fft_fwd(x, slot, S.twB, S.twC, lane);
            __syncwarp();
#pragma unroll
            for (int j = 0; j < 16; j++) slot[fswz(lay_d(lane, j))] = make_double2(x[j].re, x[j].im);
        }
        __syncthreads();
        {   // ---- B: one BK load serves the G lanes of the CTA ----
            const double2* bki = bkf + (size_t)i * kFStepD2;
#pragma unroll 1
            for (int k = tid; k < 512; k += NT) {
                const int sk = fswz(k);
                if constexpr (G <= 2) {
                    // all 6G digit values first, then per output the 6 BK words (ptxas hoists ~15 of the 24 BK
                    // loads above the phase barrier: the L2 latency overlaps the tail of phase A)
                    dcplx D[G][kRows];
#pragma unroll
                    for (int gm = 0; gm < G; gm++)
#pragma unroll
                        for (int r = 0; r < kRows; r++) {
                            const double2 v = S.slot[gm][r][sk];
                            D[gm][r] = dcplx{v.x, v.y};
                        }
#pragma unroll
                    for (int o = 0; o < kFOuts; o++) {
                        double2 b[kRows];
#pragma unroll
                        for (int r = 0; r < kRows; r++) b[r] = __ldg(bki + (r * kFOuts + o) * 512 + k);
#pragma unroll
                        for (int gm = 0; gm < G; gm++) {
                            double re = 0.0, im = 0.0;
#pragma unroll
                            for (int r = 0; r < kRows; r++) {
                                re = fma(D[gm][r].re, b[r].x, fma(-D[gm][r].im, b[r].y, re));
                                im = fma(D[gm][r].re, b[r].y, fma(D[gm][r].im, b[r].x, im));
                            }
                            S.slot[gm][o][sk] = make_double2(re, im);
                        }
                    }
                } else {
                    // row-outer order for G = 3 (96 registers): per row r the G digit values and the 4 BK words
                    // of position k, accumulated into 4G complex registers
                    double re[G][kFOuts], im[G][kFOuts];
#pragma unroll
                    for (int gm = 0; gm < G; gm++)
#pragma unroll
                        for (int o = 0; o < kFOuts; o++) re[gm][o] = im[gm][o] = 0.0;
#pragma unroll
                    for (int r = 0; r < kRows; r++) {
                        double2 b[kFOuts], d[G];
#pragma unroll
                        for (int o = 0; o < kFOuts; o++) b[o] = __ldg(bki + (r * kFOuts + o) * 512 + k);
#pragma unroll
                        for (int gm = 0; gm < G; gm++) d[gm] = S.slot[gm][r][sk];
#pragma unroll
                        for (int gm = 0; gm < G; gm++)
#pragma unroll
                            for (int o = 0; o < kFOuts; o++) {
                                re[gm][o] = fma(d[gm].x, b[o].x, fma(-d[gm].y, b[o].y, re[gm][o]));
                                im[gm][o] = fma(d[gm].x, b[o].y, fma(d[gm].y, b[o].x, im[gm][o]));
                            }
                    }
#pragma unroll
                    for (int gm = 0; gm < G; gm++)
#pragma unroll
                        for (int o = 0; o < kFOuts; o++) S.slot[gm][o][sk] = make_double2(re[gm][o], im[gm][o]);
                }
            }
        }
        __syncthreads();
        if (w8 < kFOuts) {   // ---- C ----
            double2* slot = S.slot[g][w8];
            dcplx x[16];
#pragma unroll
            for (int j = 0; j < 16; j++) {
                const double2 v = slot[fswz(lay_d(lane, j))];
                x[j] = dcplx{v.x, v.y};
            }
            fft_inv(x, slot, S.twB, S.twC, lane);
            uint32_t v[32];
#pragma unroll
            for (int j = 0; j < 16; j++) {
                v[j] = round_mod32(x[j].re) << (16 * h);                  // coefficient lane + 32 j
                v[j + 16] = round_mod32(x[j].im) << (16 * h);             // coefficient lane + 32 j + 512
            }
            uint32_t* scratch = reinterpret_cast<uint32_t*>(slot);
            __syncwarp();
            if (h == 1) {
#pragma unroll
                for (int j = 0; j < 32; j++) scratch[lane + 32 * j] = v[j];
            }
            asm volatile("bar.sync %0, 64;" ::"r"(1 + g * 2 + q) : "memory");
            if (h == 0) {
                const uint32_t* other = reinterpret_cast<const uint32_t*>(S.slot[g][w8 + 1]);
                uint32_t* accq = S.acc[g][q];
#pragma unroll
                for (int j = 0; j < 32; j++) {
                    const uint32_t nv = accq[lane + 32 * j] + v[j] + other[lane + 32 * j];
                    accq[lane + 32 * j] = nv;
                    accq[lane + 32 * j + kN] = 0u - nv;
                    accq[lane + 32 * j + 2 * kN] = nv;
                }
            }
        }
        __syncthreads();
    }
    {   // a5
        const int gl = lane0 + g;
        if (gl < A.nlanes) {
            uint32_t* o = A.out + (int64_t)gl * A.out_stride;
            for (int j = w8 * 32 + lane; j <= kN; j += NL) {
                uint32_t v;
                if (j == 0) v = S.acc[g][0][0];
                else if (j < kN) v = 0u - S.acc[g][0][kN - j];
                else v = S.acc[g][1][0];
                o[j] = v;
            }
        }
    }
}

template <int G>
__global__ void __launch_bounds__(BrfCfg<G>::NT, G == 1 ? 2 : 1) brf_kernel(BrArgs A, const double2* __restrict__ bkf,
                                                                            const double2* __restrict__ twB,
                                                                            const double2* __restrict__ twC) {
    brf_body<G>(A, bkf, twB, twC);
}
// BK (torus) -> FFT domain: one warp per (i, r, q, half); stored [i][r][o = q*2 + half][k], scaled by 1/512
__global__ void __launch_bounds__(128) bk_to_fft_kernel(const uint32_t* __restrict__ bk, double2* __restrict__ bkf,
                                                        const double2* twB, const double2* twC) {
    __shared__ double2 buf[4][512];
    __shared__ double2 tB[kTwB], tC[kTwC];
    for (int k = threadIdx.x; k < kTwB; k += blockDim.x) tB[k] = twB[k];
    for (int k = threadIdx.x; k < kTwC; k += blockDim.x) tC[k] = twC[k];
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int task = blockIdx.x * 4 + warp;
    if (task >= kn * kRows * 2 * 2) return;
    const int half = task & 1, q = (task >> 1) & 1, r = (task >> 2) % kRows, i = (task >> 2) / kRows;
    const uint32_t* src = bk + (((size_t)i * kRows + r) * 2 + q) * kN;
    dcplx x[16];
#pragma unroll
    for (int j = 0; j < 16; j++) {
        double v[2];
#pragma unroll
        for (int f = 0; f < 2; f++) {
            const uint32_t w = src[lane + 32 * j + 512 * f];
            const int32_t lo = (int32_t)(int16_t)(w & 0xFFFFu);
            const int32_t hi = (int32_t)(int16_t)((w - (uint32_t)lo) >> 16);
            v[f] = (double)(half == 0 ? lo : hi);
        }
        x[j] = dcplx{v[0], v[1]};
    }
    fft_fwd(x, buf[warp], tB, tC, lane);
    double2* dst = bkf + ((size_t)i * kRows + r) * kFOuts * 512 + (q * 2 + half) * 512;
#pragma unroll
    for (int j = 0; j < 16; j++) dst[lay_d(lane, j)] = make_double2(x[j].re * (1.0 / 512), x[j].im * (1.0 / 512));
}

template <int G>
static int launch_brf_g(const BrArgs& A, const double2* bkf, const double2* twB, const double2* twC, cudaStream_t st) {
    const size_t smem = sizeof(BrfSmem<G>);
    static_assert(sizeof(BrfSmem<G>) <= 232448, "brf shared memory");
    auto* kern = brf_kernel<G>;
    if (ensure_smem_attr<brf_kernel<G>>(smem)) return -1;
    const int blocks = (A.nlanes + G - 1) / G;
    if (blocks == 0) return 0;
    kern<<<blocks, BrfCfg<G>::NT, smem, st>>>(A, bkf, twB, twC);
    return 0;
}

int launch_brf(const BrArgs& A, int G, const double2* bkf, const double2* twB, const double2* twC, cudaStream_t st) {
    switch (G) {
        case 1: return launch_brf_g<1>(A, bkf, twB, twC, st);
        case 2: return launch_brf_g<2>(A, bkf, twB, twC, st);
        default: return launch_brf_g<3>(A, bkf, twB, twC, st);
    }
}

void launch_bk_to_fft(const uint32_t* bk, double2* bkf, const double2* twB, const double2* twC, cudaStream_t st) {
    const int tasks = kn * kRows * 2 * 2;
    bk_to_fft_kernel<<<(tasks + 3) / 4, 128, 0, st>>>(bk, bkf, twB, twC);
}
size_t bkf_bytes() { return (size_t)kn * kFStepD2 * sizeof(double2); }

}  // namespace tb
