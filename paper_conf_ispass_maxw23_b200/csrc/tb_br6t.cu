// tb_br6t.cu -- br6 with its forward NTT on the tensor cores.
//
// PAPER.md: bootstrapping "dominates the execution time", blind rotation is the largest slice of a gate
// (Fig. 7) and its NTT work is "highly vectorizable".  br6 spends a third of its time in the
// forward transforms of the 6 gadget digits (phase A: 50 Shoup butterflies per coefficient on the FMA pipe).
// This kernel keeps br6's CTA shape (2 lanes = 2 independent bootstraps per CTA, 12 warps, 2 CTAs per SM),
// its MAC (phase B) and its inverse NTT (phase C) unchanged, and computes phase A as the four-step forward NTT
// of tb_brt.cu: digits -> GEMM1 (32 x 32 DFT over k1, s8 x u8) -> limbs + twiddle -> GEMM2 (32 x 32 DFT over
// k2, byte limbs u8 x u8) -> limbs, i.e. A[j] = a(psi^(2 j + 1)) in natural order j = j1 + 32 j2.  br6's
// transform leaves a(psi^(2 brv10(a) + 1)) at position a, so A[j] is stored at position brv10(j) and the MAC
// and the inverse read exactly what they read in br6 (same NTT-domain BK, bit-identical results).
//
// Resources per CTA (2 per SM): TMEM 256 columns -- a GEMM stage is done as two N = 64 halves (3 tiles x 64
// columns), the first half's results held in registers until the second half has consumed the operands;
// shared memory ~108 KB -- the 3 operand tiles (digits A1, then GEMM2's A2) alias br6's 12 transform slots,
// which are written only once GEMM2 is complete.  One thread issues the MMAs of a half; all 12 warps run the
// epilogues (warp w: tile w / 4 = polynomials 4 (w / 4) .. + 3, TMEM lane quadrant w % 4); the other CTA on the
// SM fills the MMA waits.
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"
#include "tb_tc.cuh"

namespace tb {

constexpr int kHyG = 2;                        // lanes per CTA
constexpr int kHyThreads = 192 * kHyG;         // 12 warps
constexpr uint32_t kHyB = kB1Bytes + kBBytes;  // B1 (W1 bytes), B2 (W2' bytes) of tb_brt.cu

constexpr uint32_t kHySlotBytes = 4u * kSlotWords;    // br6 transform slot (32 x 33 words)
struct HySmem {
    unsigned char B[kHyB];
    unsigned char op[3 * kOpTile];   // tile t: A1 (digits) -> A2 (GEMM2 operand) -> the slots of polys 4t .. 4t+3
    uint2 twF[32 * 32];              // four-step forward twiddles [j1][k2]
    uint2 twI[31 * 32];              // br6 inverse NTT twiddles
    uint32_t acc[kHyG][2][kN];
    uint16_t bar[kHyG][kn + 2];
    uint64_t mbar[3];
    uint32_t tmem;
};
static_assert(4 * kHySlotBytes <= kOpTile, "the slots of a tile's 4 polynomials must fit its operand region");
// br6 slot of polynomial P = g*6 + r (lane g, row / output r): inside the operand region of tile P / 4, so a quad
// writes its slots while the other quads' GEMMs still read their own tiles
__device__ __forceinline__ uint32_t* hy_slot(HySmem& S, int P) {
    return reinterpret_cast<uint32_t*>(S.op + (P >> 2) * kOpTile + (P & 3) * kHySlotBytes);
}

// Forward NTT pipeline of one quad (4 warps, tile t = polynomials 4t .. 4t+3, 128 threads, named barrier 5 + t):
// the quad's leader issues the tile's MMAs and waits for the commit, the quad meets at its barrier.  The three
// quads (and the other CTA on the SM) overlap one another's MMA waits.
__device__ __forceinline__ void quad_sync(int t) {
    asm volatile("bar.sync %0, %1;" ::"r"(5 + t), "n"(128) : "memory");
}
// one N = 64 half of GEMM stage s (0: digits x W1, 1: A2 x W2') for tile t: MMA, commit, wait (leader only)
__device__ __forceinline__ void hy_gemm(HySmem& S, int t, int s, int h, bool leader, uint32_t& ph) {
    tc_fence_before();
    quad_sync(t);
    if (leader) {
        tc_fence_after();
        const uint32_t sB = smem_u32(S.B), a = smem_u32(S.op) + t * kOpTile, d = S.tmem + 64 * t;
        constexpr uint32_t id_s = tc_idesc_i8(128, 64, true, false), id_u = tc_idesc_i8(128, 64, false, false);
        if (s == 0) {
            tc_mma_i8(d, tc_sdesc(a, kA1Lbo, kA1Sbo), tc_sdesc(sB + 2048 * h, 128, 256), id_s, 0);
        } else {
            const uint32_t bb = sB + kB1Bytes + 8192 * h;
#pragma unroll
            for (int q = 0; q < 4; q++)
                tc_mma_i8(d, tc_sdesc(a + 2 * q * kOpLbo, kOpLbo, kOpSbo), tc_sdesc(bb + 2 * q * 128, 128, 1024),
                          id_u, q > 0);
        }
        tc_commit(smem_u32(&S.mbar[t]));
        mbar_wait(&S.mbar[t], ph);
    }
    ph ^= 1;
    quad_sync(t);
    tc_fence_after();
}

__global__ void __launch_bounds__(kHyThreads, 2) br6t_kernel(BrArgs A, const unsigned char* __restrict__ tcB,
                                                              const uint2* __restrict__ tcTw) {
    extern __shared__ __align__(1024) unsigned char hy_smem[];
    HySmem& S = *reinterpret_cast<HySmem*>(hy_smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = warp / 6, w6 = warp % 6;
    const int lane0 = blockIdx.x * kHyG;

    for (int e = tid; e < (int)(kHyB / 16); e += kHyThreads)
        reinterpret_cast<uint4*>(S.B)[e] = __ldg(reinterpret_cast<const uint4*>(tcB) + e);
    for (int e = tid; e < 32 * 32; e += kHyThreads) S.twF[e] = tcTw[e];
    for (int e = tid; e < 31 * 32; e += kHyThreads) S.twI[e] = A.twI[e];
    if (warp == 0) tc_alloc<256>(&S.tmem);
    if (tid == 0) {
        for (int t = 0; t < 3; t++) mbar_init(&S.mbar[t], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // ---- prologue (a1, a2): linear gate combination + mod switch to 2N (6 warps per lane) ----
    {
        const int gl = lane0 + g;
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t* s0 = (d.sel & 3u) == 0 ? A.src0 : ((d.sel & 3u) == 1 ? A.src1 : A.src2);
        const uint32_t sb = (d.sel >> 2) & 3u;
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = w6 * 32 + lane; w <= kn; w += 192) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[g][w] = (uint16_t)((v + (1u << 20)) >> 21);      // round(v 2N / 2^32) mod 2N (C5)
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    // ---- ACC = (0, X^{-bbar} (mu, ..., mu))  (a3, C6) ----
    for (int k = tid; k < kHyG * kN; k += kHyThreads) {
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        S.acc[gg][0][c] = 0u;
        S.acc[gg][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int q = w6 / kParts, m = w6 % kParts;           // phase C role (br6)
    const int et = warp >> 2, qd = warp & 3;              // epilogue role: tile, TMEM lane quadrant
    const uint32_t tq = S.tmem + ((uint32_t)(32 * qd) << 16) + 64 * et;
    const bool leader = qd == 0 && lane == 0;
    uint32_t ph = 0;
    for (int i = 0; i < kn; i++) {
        // ---- a4.1: digits of (X^abar - 1) ACC -> A1 of the quad's tile.  Polynomial P = gd*6 + bloc*3 + jd is
        // digit jd of source pair P / 3 = (gd, bloc); tile t needs pairs 4t / 3 and (4t + 3) / 3.  Thread
        // (qd, k2): coefficients c = 32 (8 qd + u) + k2, u < 8 -> rows (P % 4)*32 + k2, K bytes 8 qd .. 8 qd + 7
        {
            const int pr0 = (4 * et) / 3, pr1 = (4 * et + 3) / 3;
            const uint32_t ab0 = S.bar[pr0 >> 1][i], ab1 = S.bar[pr1 >> 1][i];
            const uint32_t* acc0 = S.acc[pr0 >> 1][pr0 & 1];
            const uint32_t* acc1 = S.acc[pr1 >> 1][pr1 & 1];
            uint32_t d[4][2] = {};
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const uint32_t c = 32u * (8 * qd + u) + lane;
                uint32_t x[2];
#pragma unroll
                for (int s2 = 0; s2 < 2; s2++) {
                    const uint32_t ab = s2 ? ab1 : ab0;
                    const uint32_t* acc = s2 ? acc1 : acc0;
                    const uint32_t mm = (c - ab) & (kTwoN - 1);
                    const uint32_t src = acc[mm & (kN - 1)];
                    const uint32_t rot = mm < (uint32_t)kN ? src : 0u - src;
                    x[s2] = rot - acc[c] + c_misc[3];                 // (X^abar - 1) ACC + decomposition offset
                }
#pragma unroll
                for (int pp = 0; pp < 4; pp++) {
                    const int P = 4 * et + pp, jd = P % 3;
                    const uint32_t xx = (P / 3 == pr0) ? x[0] : x[1];
                    const uint32_t dig = ((xx >> (32 - kBgbit * (jd + 1))) & 127u) - 64u;   // in [-64, 63]
                    d[pp][u >> 2] |= (dig & 0xFFu) << (8 * (u & 3));
                }
            }
            unsigned char* tile = S.op + et * kOpTile;
#pragma unroll
            for (int pp = 0; pp < 4; pp++)
                *reinterpret_cast<uint2*>(tile + tc_off(pp * 32 + lane, 8 * qd, kA1Lbo, kA1Sbo)) =
                    make_uint2(d[pp][0], d[pp][1]);
            fence_async_smem();
        }
        // ---- a4.2 forward NTT, stage 1: B[j1][k2] = sum_k1 W1[j1][k1] digit[32 k1 + k2], C = B psi^((2j1+1)k2)
        // thread (P = 4 et + qd, k2 = lane), j1 = 16 h + u
        uint32_t e[32];
#pragma unroll
        for (int h = 0; h < 2; h++) {
            hy_gemm(S, et, 0, h, leader, ph);
#pragma unroll
            for (int c = 0; c < 4; c++) {
                uint32_t v[16];
                tc_ld16(tq + 16 * c, v);
                tc_wait_ld();
#pragma unroll
                for (int u4 = 0; u4 < 4; u4++) {
                    const int j1 = 16 * h + 4 * c + u4;
                    const uint2 w = S.twF[32 * j1 + lane];
                    e[j1] = shoup_mul(limbs_s(v[4 * u4], v[4 * u4 + 1], v[4 * u4 + 2], v[4 * u4 + 3]), w.x, w.y);
                }
            }
        }
        {   // A2 tile et, row (qd, j1), word k2 (A1 is consumed: both halves of GEMM1 are complete)
            unsigned char* base = S.op + et * kOpTile + opw(qd * 32, lane);
#pragma unroll
            for (int j1 = 0; j1 < 32; j1++)
                *reinterpret_cast<uint32_t*>(base + (j1 >> 3) * kOpSbo + (j1 & 7) * 16) = e[j1];
            fence_async_smem();
        }
        // ---- stage 2: A[j1 + 32 j2] = sum_k2 W2[j2][k2] C[j1][k2]; thread (P, j1 = lane), j2 = 16 h + u
#pragma unroll
        for (int h = 0; h < 2; h++) {
            hy_gemm(S, et, 1, h, leader, ph);
#pragma unroll
            for (int c = 0; c < 4; c++) {
                uint32_t v[16];
                tc_ld16(tq + 16 * c, v);
                tc_wait_ld();
#pragma unroll
                for (int u4 = 0; u4 < 4; u4++)
                    e[16 * h + 4 * c + u4] = red_2p(limbs_u(v[4 * u4], v[4 * u4 + 1], v[4 * u4 + 2], v[4 * u4 + 3]));
            }
        }
        {   // slot of polynomial P, position brv10(j1 + 32 j2) = 32 brv5(j1) + brv5(j2) (padded rows); the
            // quad's tile is no longer read by the tensor core (GEMM2 complete)
            uint32_t* sl = hy_slot(S, 4 * et + qd) + kPadRow * (int)(__brev((uint32_t)lane) >> 27);
#pragma unroll
            for (int j2 = 0; j2 < 32; j2++) sl[(int)(__brev((uint32_t)j2) >> 27)] = e[j2];
        }
        __syncthreads();
        // ---- phase B: pointwise MAC against BKhat_i, shared by the CTA's lanes (a4.3; br6) ----
        {
            const uint32_t* bki = A.bkhat + (size_t)i * (kRows * kOuts * kN);
            for (int a = tid; a < kN; a += kHyThreads) {
                const int pa = a + (a >> 5);
                uint32_t B[kRows][kOuts];
#pragma unroll
                for (int r = 0; r < kRows; r++)
#pragma unroll
                    for (int o = 0; o < kOuts; o++) B[r][o] = __ldg(bki + (r * kOuts + o) * kN + a);
#pragma unroll
                for (int gg = 0; gg < kHyG; gg++) {
                    uint32_t D[kRows];
#pragma unroll
                    for (int r = 0; r < kRows; r++) D[r] = hy_slot(S, gg * 6 + r)[pa];
#pragma unroll
                    for (int o = 0; o < kOuts; o++) {
                        uint64_t s = 0;
#pragma unroll
                        for (int r = 0; r < kRows; r++) s += (uint64_t)D[r] * B[r][o];
                        const uint32_t hi = (uint32_t)(s >> 32), lo = (uint32_t)s;
                        hy_slot(S, gg * 6 + o)[pa] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                    }
                }
            }
        }
        __syncthreads();
        // ---- phase C: inverse NTT, centred lift, part recombination, ACC += (a4.4; br6) ----
        {
            uint32_t* slot = hy_slot(S, g * 6 + w6);
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = slot[kPadRow * lane + j];
            ntt_inv(x, slot, S.twI, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = lift_centred(x[j]) << (11 * m);
            if (m != 0) {
#pragma unroll
                for (int j = 0; j < 32; j++) slot[kPadRow * j + lane] = x[j];
            }
            named_bar(1 + g * 2 + q, 96);
            if (m == 0) {
                const uint32_t* p1 = hy_slot(S, g * 6 + q * kParts + 1);
                const uint32_t* p2 = hy_slot(S, g * 6 + q * kParts + 2);
                uint32_t* acc = S.acc[g][q];
#pragma unroll
                for (int j = 0; j < 32; j++)
                    acc[lane + 32 * j] = add_alu(acc[lane + 32 * j] + x[j] + p1[kPadRow * j + lane], p2[kPadRow * j + lane]);
            }
        }
        __syncthreads();
    }
    // ---- sample extraction, index 0 (a5, C8) ----
    {
        const int gl = lane0 + g;
        if (gl < A.nlanes) {
            uint32_t* o = A.out + (int64_t)gl * A.out_stride;
            for (int j = w6 * 32 + lane; j <= kN; j += 192) {
                uint32_t v;
                if (j == 0) v = S.acc[g][0][0];
                else if (j < kN) v = 0u - S.acc[g][0][kN - j];
                else v = S.acc[g][1][0];
                o[j] = v;
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tc_dealloc<256>(S.tmem);
}

int launch_br6t(const BrArgs& A, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st) {
    const size_t smem = sizeof(HySmem);
    if (ensure_smem_attr<br6t_kernel>(smem)) return -1;
    const int blocks = (A.nlanes + kHyG - 1) / kHyG;
    if (blocks == 0) return 0;
    br6t_kernel<<<blocks, kHyThreads, smem, st>>>(A, tcB, tcTw);
    return 0;
}

}  // namespace tb
