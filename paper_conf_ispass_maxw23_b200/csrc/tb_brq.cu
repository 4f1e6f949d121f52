// tb_brq.cu -- blind rotation with both NTT directions on the tensor cores in br6's occupancy shape
// (variant 15).
//
// PAPER.md: bootstrapping "dominates the execution time", blind rotation is the largest slice of a gate
// (Fig. 7) and its NTT work is "highly vectorizable".  The arithmetic is brt's (tb_brt.cu): the
// four-step transforms as byte-limb tcgen05 GEMMs, the MAC against the natural-order NTT-domain BK (bk4) on the
// CUDA cores, exact and bit-identical to br6.  The execution shape is br6t's (tb_br6t.cu): 2 lanes (independent
// bootstraps) per CTA, 12 warps, 2 CTAs per SM, and the transform work of a CMux step split into three
// independent quad pipelines -- quad t (warps 4t .. 4t+3, TMEM lane quadrant = warp % 4, TMEM columns
// 64t .. 64t+63) owns operand tile t (4 polynomials) for all four GEMM stages, its leader thread issues the tile's
// MMAs (N = 64 halves) and waits for the commit, the quad meets at named barrier 5 + t.  Per CMux step:
//
//   quad t:  digits -> A1 | GEMM1, ep1 (limbs, twiddle) -> A2 | GEMM2, ep2 (limbs) -> A3 (natural order)
//   CTA:     MAC (in place in A3: output o of lane g -> tile o % 3, quadrant g*2 + o/3; each BK record is read
//            once for the 2 lanes)
//   quad t:  GEMM3, ep3 (limbs, twiddle) -> A4 | GEMM4, ep4 (limbs, centred lift, << 11 t, ACC += part t)
//
// Shared memory per CTA ~110 KB (two CTAs per SM): GEMM3 needs no constant matrix of its own -- V2[k2][j2] =
// psi^(-64 j2 k2) is W2's row -k2 mod 32, so GEMM3 multiplies by B2 and its TMEM column k2' holds D[-k2'] (ep3
// reads the columns in that order) -- and the twiddle tables are read through L1 (__ldg) instead of shared memory.
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"
#include "tb_tc.cuh"

namespace tb {

constexpr int kBqG = 2;                             // lanes per CTA
constexpr int kBqThreads = 192 * kBqG;              // 12 warps = 3 quads
constexpr uint32_t kBqB = kB1Bytes + 2 * kBBytes;   // B1 (W1 bytes), B2 (W2' = V2' up to the row order), B4 (V1')

struct BqSmem {
    unsigned char B[kBqB];
    unsigned char op[3 * kOpTile];      // tile t: A1 -> A2 -> A3 (MAC in / out) -> A4
    uint32_t acc[kBqG][2][kN];
    uint16_t bar[kBqG][kn + 2];
    uint64_t mbar[3];
    uint32_t tmem;
};

// one N = 64 half of GEMM stage s for tile t (0: digits x W1, 1: A2 x W2', 2: A3 x W2' (= V2' with the output
// columns in the order -k2), 3: A4 x V1'): leader issues + waits, the quad meets before and after
__device__ __forceinline__ void bq_gemm(BqSmem& S, int t, int s, int h, bool leader, uint32_t& ph) {
    tc_fence_before();
    quad_sync(t);
    if (leader) {
        tc_fence_after();
        const uint32_t sB = smem_u32(S.B), a = smem_u32(S.op) + t * kOpTile, d = S.tmem + 64 * t;
        constexpr uint32_t id_s = tc_idesc_i8(128, 64, true, false), id_u = tc_idesc_i8(128, 64, false, false);
        if (s == 0) {
            tc_mma_i8(d, tc_sdesc(a, kA1Lbo, kA1Sbo), tc_sdesc(sB + 2048 * h, 128, 256), id_s, 0);
        } else {
            const uint32_t bb = sB + kB1Bytes + (s == 3 ? kBBytes : 0) + 8192 * h;
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

__global__ void __launch_bounds__(kBqThreads, 2) brq_kernel(BrArgs A, const uint32_t* __restrict__ bk4,
                                                             const unsigned char* __restrict__ tcB,
                                                             const uint2* __restrict__ tcTw) {
    extern __shared__ __align__(1024) unsigned char bq_smem[];
    BqSmem& S = *reinterpret_cast<BqSmem*>(bq_smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int lane0 = blockIdx.x * kBqG;

    for (int e = tid; e < (int)((kB1Bytes + kBBytes) / 16); e += kBqThreads)          // B1, B2
        reinterpret_cast<uint4*>(S.B)[e] = __ldg(reinterpret_cast<const uint4*>(tcB) + e);
    for (int e = tid; e < (int)(kBBytes / 16); e += kBqThreads)                        // B4 (after B3 in tcB)
        reinterpret_cast<uint4*>(S.B + kB1Bytes + kBBytes)[e] =
            __ldg(reinterpret_cast<const uint4*>(tcB + kB1Bytes + 2 * kBBytes) + e);
    if (warp == 0) tc_alloc<256>(&S.tmem);
    if (tid == 0) {
        for (int t = 0; t < 3; t++) mbar_init(&S.mbar[t], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    // ---- prologue (a1, a2): linear gate combination + mod switch to 2N (6 warps per lane) ----
    {
        const int g = warp / 6, w6 = warp % 6;
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
    for (int k = tid; k < kBqG * kN; k += kBqThreads) {
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        S.acc[gg][0][c] = 0u;
        S.acc[gg][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int et = warp >> 2, qd = warp & 3;              // quad = tile, TMEM lane quadrant
    const uint32_t tq = S.tmem + ((uint32_t)(32 * qd) << 16) + 64 * et;
    const bool leader = qd == 0 && lane == 0;
    unsigned char* tile = S.op + et * kOpTile;
    const uint2* twF = tcTw;                              // [j1][k2]
    const uint2* twI = tcTw + 1024;                       // [k2][j1]
    uint32_t ph = 0;
    for (int i = 0; i < kn; i++) {
        // ---- a4.1: digits of (X^abar - 1) ACC -> A1 of the quad's tile (as tb_br6t.cu): polynomial
        // P = gd*6 + bloc*3 + jd is digit jd of source pair P / 3 = (gd, bloc); thread (qd, k2): coefficients
        // c = 32 (8 qd + u) + k2 -> rows (P % 4)*32 + k2, K bytes 8 qd .. 8 qd + 7
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
#pragma unroll
            for (int pp = 0; pp < 4; pp++)
                *reinterpret_cast<uint2*>(tile + tc_off(pp * 32 + lane, 8 * qd, kA1Lbo, kA1Sbo)) =
                    make_uint2(d[pp][0], d[pp][1]);
            fence_async_smem();
        }
        uint32_t e[32];
        // ---- a4.2 GEMM1 + ep1: thread (P = 4 et + qd, k2 = lane), j1 = 16 h + u: C[j1][k2] -> A2 row (qd, j1)
#pragma unroll
        for (int h = 0; h < 2; h++) {
            bq_gemm(S, et, 0, h, leader, ph);
#pragma unroll
            for (int c = 0; c < 4; c++) {
                uint32_t v[16];
                tc_ld16(tq + 16 * c, v);
                tc_wait_ld();
#pragma unroll
                for (int u4 = 0; u4 < 4; u4++) {
                    const int j1 = 16 * h + 4 * c + u4;
                    const uint2 w = __ldg(twF + 32 * j1 + lane);
                    e[j1] = shoup_mul(limbs_s(v[4 * u4], v[4 * u4 + 1], v[4 * u4 + 2], v[4 * u4 + 3]), w.x, w.y);
                }
            }
        }
        {
            unsigned char* base = tile + opw(qd * 32, lane);
#pragma unroll
            for (int j1 = 0; j1 < 32; j1++)
                *reinterpret_cast<uint32_t*>(base + (j1 >> 3) * kOpSbo + (j1 & 7) * 16) = e[j1];
            fence_async_smem();
        }
        // ---- GEMM2 + ep2: thread (P, j1 = lane), j2 = 16 h + u: A[j1 + 32 j2] in [0, 2p) -> A3 row (qd, j1)
#pragma unroll
        for (int h = 0; h < 2; h++) {
            bq_gemm(S, et, 1, h, leader, ph);
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
        {
            unsigned char* base = tile + opw(qd * 32 + lane, 0);
#pragma unroll
            for (int c = 0; c < 8; c++)
                *reinterpret_cast<uint4*>(base + c * kOpLbo) = make_uint4(e[4 * c], e[4 * c + 1], e[4 * c + 2], e[4 * c + 3]);
        }
        // ---- a4.3 MAC: position (j1, j2 = lane), j1 = warp + 12 k; M_o = sum_r A_r BK4[r][o] for both lanes, in
        // place (output o of lane g -> tile o % 3, quadrant g*2 + o/3).  The first BK record is requested before
        // the CTA barrier, so its L2 latency overlaps the wait.
        {
            const uint32_t* bki = bk4 + (size_t)i * kN * kBk4Rec;
            uint4 Bn[kBk4Rec / 4];
            {
                const uint4* rec = reinterpret_cast<const uint4*>(bki + (size_t)(warp * 32 + lane) * kBk4Rec);
#pragma unroll
                for (int q = 0; q < kBk4Rec / 4; q++) Bn[q] = __ldg(rec + q);
            }
            __syncthreads();                              // every quad's A3 written
            for (int j1 = warp; j1 < 32; j1 += 12) {
                if (j1 != warp) {
                    const uint4* rec = reinterpret_cast<const uint4*>(bki + (size_t)(j1 * 32 + lane) * kBk4Rec);
#pragma unroll
                    for (int q = 0; q < kBk4Rec / 4; q++) Bn[q] = __ldg(rec + q);
                }
                uint32_t B[kBk4Rec];
#pragma unroll
                for (int q = 0; q < kBk4Rec / 4; q++) {
                    B[4 * q] = Bn[q].x; B[4 * q + 1] = Bn[q].y; B[4 * q + 2] = Bn[q].z; B[4 * q + 3] = Bn[q].w;
                }
                const uint32_t off = opw(j1, lane);
                uint32_t D[kBqG][6];                      // both lanes' inputs first: the outputs overwrite them
#pragma unroll
                for (int g = 0; g < kBqG; g++)
#pragma unroll
                    for (int r = 0; r < 6; r++) {
                        const int P = g * 6 + r;
                        D[g][r] = *reinterpret_cast<const uint32_t*>(S.op + (P >> 2) * kOpTile + (P & 3) * 4 * kOpSbo + off);
                    }
#pragma unroll
                for (int g = 0; g < kBqG; g++) {
#pragma unroll
                    for (int o = 0; o < 6; o++) {
                        uint64_t s = 0;
#pragma unroll
                        for (int r = 0; r < 6; r++) s += (uint64_t)D[g][r] * B[r * 6 + o];
                        const uint32_t hi = (uint32_t)(s >> 32), lo = (uint32_t)s;
                        *reinterpret_cast<uint32_t*>(S.op + (o % 3) * kOpTile + (g * 2 + o / 3) * 4 * kOpSbo + off) =
                            red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                    }
                }
            }
            fence_async_smem();
            __syncthreads();                              // every MAC output written
        }
        // ---- a4.4 GEMM3 (B2: column k2' holds D[j1][-k2']) + ep3: thread (quadrant qd, j1 = lane):
        // E[j1][k2] = D[j1][k2] psi^(-(2 j1 + 1) k2) -> A4 row (qd, k2), word j1
#pragma unroll
        for (int h = 0; h < 2; h++) {
            bq_gemm(S, et, 2, h, leader, ph);
#pragma unroll
            for (int c = 0; c < 4; c++) {
                uint32_t v[16];
                tc_ld16(tq + 16 * c, v);
                tc_wait_ld();
#pragma unroll
                for (int u4 = 0; u4 < 4; u4++) {
                    const int k2 = (32 - (16 * h + 4 * c + u4)) & 31;
                    const uint2 w = __ldg(twI + 32 * k2 + lane);
                    e[16 * h + 4 * c + u4] = shoup_mul(limbs_u(v[4 * u4], v[4 * u4 + 1], v[4 * u4 + 2], v[4 * u4 + 3]), w.x, w.y);
                }
            }
        }
        {
            unsigned char* base = tile + opw(qd * 32, lane);
#pragma unroll
            for (int kk = 0; kk < 32; kk++) {
                const int k2 = (32 - kk) & 31;
                *reinterpret_cast<uint32_t*>(base + (k2 >> 3) * kOpSbo + (k2 & 7) * 16) = e[kk];
            }
            fence_async_smem();
        }
        // ---- GEMM4 + ep4: thread (g = qd / 2, q = qd % 2, k2 = lane), k1 = 16 h + u: part t of N a[32 k1 + k2]
        // -> centred lift, << 11 t, added into ACC[g][q] (the three quads add their parts concurrently: atomics)
        {
            uint32_t* acc = &S.acc[qd >> 1][qd & 1][lane];
#pragma unroll
            for (int h = 0; h < 2; h++) {
                bq_gemm(S, et, 3, h, leader, ph);
#pragma unroll
                for (int c = 0; c < 4; c++) {
                    uint32_t v[16];
                    tc_ld16(tq + 16 * c, v);
                    tc_wait_ld();
#pragma unroll
                    for (int u4 = 0; u4 < 4; u4++) {
                        const int k1 = 16 * h + 4 * c + u4;
                        const uint32_t a = lift_centred(red_2p(limbs_u(v[4 * u4], v[4 * u4 + 1], v[4 * u4 + 2], v[4 * u4 + 3])));
                        atomicAdd(acc + 32 * k1, a << (11 * et));
                    }
                }
            }
        }
        __syncthreads();                                  // ACC complete before the next step's digits
    }
    // ---- sample extraction, index 0 (a5, C8) ----
    for (int e = tid; e < kBqG * (kN + 1); e += kBqThreads) {
        const int g = e / (kN + 1), j = e % (kN + 1);
        const int gl = lane0 + g;
        if (gl >= A.nlanes) continue;
        uint32_t v;
        if (j == 0) v = S.acc[g][0][0];
        else if (j < kN) v = 0u - S.acc[g][0][kN - j];
        else v = S.acc[g][1][0];
        A.out[(int64_t)gl * A.out_stride + j] = v;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tc_dealloc<256>(S.tmem);
}

int launch_brq(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st) {
    const size_t smem = sizeof(BqSmem);
    if (ensure_smem_attr<brq_kernel>(smem)) return -1;
    const int blocks = (A.nlanes + kBqG - 1) / kBqG;
    if (blocks == 0) return 0;
    brq_kernel<<<blocks, kBqThreads, smem, st>>>(A, bk4, tcB, tcTw);
    return 0;
}

}  // namespace tb
