// tb_brt.cu -- blind rotation on the 5th-generation tensor cores (DESIGN.md
// "Tensor-core NTT").
//
// PAPER.md: bootstrapping "dominates the execution time", blind rotation is the largest slice of a gate
// (Fig. 7) and its NTT work is "highly vectorizable".  The arithmetic is the same exact integer
// external product as br6 (field p = 0x3FFF7801, BK split in 3 signed 11-bit parts, centred lift; DESIGN.md
// "Exactness"), but each length-1024 negacyclic NTT is evaluated in four steps whose two 32-point DFTs are
// integer matrix products on the tensor cores (tcgen05.mma kind::i8, byte limbs, s32 accumulators in TMEM):
//
//   forward   a[32 k1 + k2] -> B[j1][k2] = sum_k1 W1[j1][k1] a[32 k1 + k2]          W1 = psi^(32 (2 j1 + 1) k1)
//             C[j1][k2] = B[j1][k2] psi^((2 j1 + 1) k2)                              (twiddle, CUDA cores)
//             A[j1 + 32 j2] = sum_k2 W2[j2][k2] C[j1][k2]                            W2 = psi^(64 j2 k2)
//   i.e. A[j] = a(psi^(2 j + 1)), the evaluation at the roots of X^1024 + 1 in natural order;
//   inverse   D[j1][k2] = sum_j2 V2[k2][j2] M[j1 + 32 j2]                            V2 = psi^(-64 j2 k2)
//             E[j1][k2] = D[j1][k2] psi^(-(2 j1 + 1) k2)
//             N a[32 k1 + k2] = sum_j1 V1[k1][j1] E[j1][k2]                          V1 = psi^(-32 (2 j1 + 1) k1)
//
// A product with a 30-bit constant matrix is exact as sum_b 2^(8 b) (X . bytes_b(W)); a 30-bit data operand
// enters as its 4 bytes along K, against bytes_b(2^(8 c) W mod p) (precomputed), so every GEMM is
// u8 x u8 (digits: s8 x u8) with K = 32 (digits) or 128 and N = 128 (4 limbs x 32), and the CUDA cores only
// recombine the 4 limbs (one Shoup product by 2^16) and apply the twiddles.
//
// Structure: one CTA per SM holds two independent groups of G = 2 lanes (bootstraps); each group's accumulators
// stay in shared memory for all n = 630 CMux steps.  A group's CMux step is 4 GEMM stages x 3 tile jobs (a tile
// = 4 polynomials = 128 rows of the M = 128 MMA):
//   digits -> GEMM1 -> ep1 (limbs, twiddle) -> GEMM2 -> ep2 (limbs) -> MAC (each NTT-domain BK word read once
//   for the group's 2 lanes) -> GEMM3 -> ep3 (limbs, twiddle) -> GEMM4 -> ep4 (limbs, lift, ACC +=).
// Per group: one MMA warp (one thread issues) fills a ring of 2 TMEM slots (128 columns each) and runs ahead of
// 8 compute warps (2 quads; a warp reads its TMEM lane quadrant, the two quads split a slot's columns).  The two
// groups drift apart, so one group's MAC and digit phases (CUDA cores and L2 only) overlap the other group's
// GEMMs and epilogues.  mbarriers per group: full[slot] (MMA commit -> epilogue), empty[slot] (8 epilogue warps
// -> MMA), a2[tile] (ep1 wrote GEMM2's operand tile), gate (all 8 compute warps done with digits / MAC / ep3).
#include <cstring>

#include "tb_kernels.cuh"
#include "tb_ntt.cuh"
#include "tb_tc.cuh"

namespace tb {

constexpr int kTcG = 2;                       // lanes per group
constexpr int kTcGroups = 2;                  // groups per CTA
constexpr int kTcLanes = kTcG * kTcGroups;    // lanes per CTA
constexpr int kTcPolys = 6 * kTcG;            // polynomials per transform stage of a group (12 = 3 tiles of 4)
constexpr int kTcTiles = kTcPolys / 4;
constexpr int kTcGWarps = 8;                  // compute warps per group
constexpr int kTcGThreads = 32 * kTcGWarps;
constexpr int kTcCompWarps = kTcGWarps * kTcGroups;
constexpr int kTcThreads = 32 * (kTcCompWarps + kTcGroups);   // + one MMA warp per group
constexpr int kTcSlots = 2;                              // TMEM ring per group: 2 x 128 columns
// shared-memory operand layouts (K-major core matrices, tb_tc.cuh)
constexpr uint32_t kA1Lbo = 128, kA1Sbo = 256;          // digits: 128 rows x 32 B per tile (at the tile's start)
constexpr uint32_t kOpLbo = 144, kOpSbo = 8 * 144;      // 30-bit operands: 128 rows x 128 B per tile (padded)
constexpr uint32_t kOpTile = 16 * kOpSbo;               // 18,432 B
constexpr uint32_t kB1Bytes = 128 * 32, kBBytes = 128 * 128;
constexpr uint32_t kTcBTotal = kB1Bytes + 3 * kBBytes;  // B1 (W1 bytes), B2 (W2'), B3 (V2'), B4 (V1')
constexpr int kBk4Rec = 36;                              // NTT-domain BK record per coefficient: [r][o]

struct BrtGroup {
    unsigned char op[kTcTiles * kOpTile];        // per tile: A1 | A2 | MAC in / out = A3 | A4 (stage-aliased)
    uint32_t acc[kTcG][2][kN];
    uint16_t bar[kTcG][kn + 2];
    uint64_t full[kTcSlots], empty[kTcSlots], a2[kTcTiles], gate;
};
struct BrtSmem {
    unsigned char B[kTcBTotal];                  // constant B operands (dense: LBO 128)
    uint2 twF[32 * 32];                          // [j1][k2] (psi^((2 j1 + 1) k2), Shoup)
    uint2 twI[32 * 32];                          // [k2][j1] (psi^(-(2 j1 + 1) k2), Shoup)
    BrtGroup grp[kTcGroups];
    uint32_t tmem;
};

// ---- limb recombination: sum_b 2^(8 b) Y_b mod p ----------------------------------------------------------
constexpr uint32_t kW16p = (uint32_t)((((uint64_t)1 << 48)) / kP);    // Shoup companion of 2^16
// operands < 2p (top byte <= 127): Y0 + 2^8 Y1 <= 32 (3*255 + 127) 255 * 257 < 1.9e9, hi 2^16 mod p < 2p,
// so the sum stays below 4.1e9 < 4p: no reduction of the low half is needed
// The shift-adds are written as funnel shifts (SHF) and three-input adds (IADD3) so that ptxas keeps them on the
// ALU pipe: plain `y0 + (y1 << 8)` becomes an IMAD on the FMA-heavy pipe, which the Shoup products and the MAC
// already load (measured: IMAD was 28 % of the kernel's executed instructions).
__device__ __forceinline__ uint32_t shl_alu(uint32_t x, int s) { return __funnelshift_l(0u, x, s); }
__device__ __forceinline__ uint32_t limbs_u(uint32_t y0, uint32_t y1, uint32_t y2, uint32_t y3) {
    const uint32_t hi = y2 + shl_alu(y3, 8) + c_zero;
    const uint32_t q = __umulhi(hi, kW16p);
    const uint32_t r = shl_alu(hi, 16) - q * kP;                   // hi 2^16 mod p in [0, 2p)
    return y0 + shl_alu(y1, 8) + r;
}
// signed limbs (s8 digits x u8, |Y_b| < 2^19): lo + p, hi + p are in (0, 2p); result < 4p
__device__ __forceinline__ uint32_t limbs_s(uint32_t y0, uint32_t y1, uint32_t y2, uint32_t y3) {
    const uint32_t hi = y2 + shl_alu(y3, 8) + kP;
    const uint32_t q = __umulhi(hi, kW16p);
    const uint32_t r = shl_alu(hi, 16) - q * kP;
    return y0 + shl_alu(y1, 8) + (r + kP + c_zero);
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// named barrier of a group's compute warps (ids 1, 2)
__device__ __forceinline__ void grp_sync(int grp) {
    asm volatile("bar.sync %0, %1;" ::"r"(1 + grp), "n"(kTcGThreads) : "memory");
}

// byte offset of (row, 32-bit word) of an operand tile
__host__ __device__ constexpr uint32_t opw(uint32_t row, uint32_t word) { return tc_off(row, 4 * word, kOpLbo, kOpSbo); }

// ---- MMA warp of a group: the static job sequence of one CMux step (stage s, tile t); k counts jobs ---------
__device__ __forceinline__ void brt_mma_step(BrtSmem& S, BrtGroup& G, uint32_t tmem, uint32_t& k, uint32_t& gate_ph,
                                             uint32_t& a2_ph) {
    const uint32_t sB = smem_u32(S.B), sOp = smem_u32(G.op);
    constexpr uint32_t id_s = tc_idesc_i8(128, 128, true, false), id_u = tc_idesc_i8(128, 128, false, false);
    for (int s = 0; s < 4; s++) {
        if (s != 1) {                                   // digits / MAC / ep3 of every compute warp done
            mbar_wait(&G.gate, gate_ph);
            gate_ph ^= 1;
        }
        for (int t = 0; t < kTcTiles; t++, k++) {
            const uint32_t slot = k % kTcSlots;
            if (s == 1) mbar_wait(&G.a2[t], a2_ph);     // ep1 wrote this tile's GEMM2 operand
            if (k >= kTcSlots) mbar_wait(&G.empty[slot], ((k / kTcSlots) - 1) & 1);
            tc_fence_after();
            const uint32_t d = tmem + 128 * slot;
            const uint32_t a = sOp + t * kOpTile;
            if (s == 0) {
                tc_mma_i8(d, tc_sdesc(a, kA1Lbo, kA1Sbo), tc_sdesc(sB, 128, 256), id_s, 0);
            } else {
                const uint32_t bb = sB + kB1Bytes + (s - 1) * kBBytes;
#pragma unroll
                for (int q = 0; q < 4; q++)
                    tc_mma_i8(d, tc_sdesc(a + 2 * q * kOpLbo, kOpLbo, kOpSbo), tc_sdesc(bb + 2 * q * 128, 128, 1024),
                              id_u, q > 0);
            }
            tc_commit(smem_u32(&G.full[slot]));
        }
        if (s == 1) a2_ph ^= 1;
    }
}

// ---- compute warps of a group ----------------------------------------------------------------------------
// digits of (X^abar - 1) ACC for the group's 2 lanes -> A1 (a4.1).  Thread (g, bloc, h, k2): coefficients
// c = 32 (16 h + u) + k2, u < 16; digit jd of polynomial P = g*6 + bloc*3 + jd goes to tile P / 4, row
// (P % 4)*32 + k2, K bytes 16 h .. 16 h + 15 (one 16-byte store)
__device__ __forceinline__ void brt_digits(BrtGroup& G, int i, int gt) {
    const int k2 = gt & 31, h = (gt >> 5) & 1, bloc = (gt >> 6) & 1, g = gt >> 7;
    const uint32_t ab = G.bar[g][i];
    const uint32_t* acc = G.acc[g][bloc];
    uint32_t d[3][4] = {};
#pragma unroll
    for (int u = 0; u < 16; u++) {
        const uint32_t c = 32u * (16 * h + u) + k2;
        const uint32_t mm = (c - ab) & (kTwoN - 1);
        const uint32_t src = acc[mm & (kN - 1)];
        const uint32_t rot = mm < (uint32_t)kN ? src : 0u - src;
        const uint32_t x = rot - acc[c] + c_misc[3];             // (X^abar - 1) ACC + decomposition offset
#pragma unroll
        for (int jd = 0; jd < 3; jd++) {
            const uint32_t dig = ((x >> (32 - kBgbit * (jd + 1))) & 127u) - 64u;   // digit in [-64, 63]
            d[jd][u >> 2] |= (dig & 0xFFu) << (8 * (u & 3));
        }
    }
#pragma unroll
    for (int jd = 0; jd < 3; jd++) {
        const int P = g * 6 + bloc * 3 + jd;
        *reinterpret_cast<uint4*>(G.op + (P >> 2) * kOpTile + tc_off((P & 3) * 32 + k2, 16 * h, kA1Lbo, kA1Sbo)) =
            make_uint4(d[jd][0], d[jd][1], d[jd][2], d[jd][3]);
    }
}

// Where the MAC writes output o of lane g (and so where GEMM3 / ep3 / GEMM4 / ep4 find it): tile m = o % 3,
// quadrant g * 2 + q (q = o / 3).  GEMM3's tile m then holds exactly the polynomials whose ep3 output fills A4
// tile m (rows (g, q, k2)): ep3 rewrites only the tile it has just consumed, and ep4 of tile m adds part m.

// One CMux step of a group's compute warps (the digits are in A1); k = job counter (same as the MMA warp's)
__device__ __forceinline__ void brt_comp_step(BrtSmem& S, BrtGroup& G, uint32_t tmem, int grp, int gw,
                                              const uint32_t* __restrict__ bk4, uint32_t& k) {
    const int lane = threadIdx.x & 31;
    const int hq = gw >> 2, qd = gw & 3;                 // column half (quad) and TMEM lane quadrant
    const uint32_t tq = tmem + ((uint32_t)(32 * qd) << 16) + 64 * hq;
    fence_async_smem();                                  // publish the digits to the MMA warp
    __syncwarp();
    if (lane == 0) mbar_arrive(&G.gate);
    // ---- ep1: tile t, thread (P = 4t + qd, k2 = lane), j1 in this quad's half: C[j1][k2] -> A2 row (qd, j1)
    uint2 twr[16];                                       // this thread's 16 forward twiddles (all tiles)
#pragma unroll
    for (int j = 0; j < 16; j++) twr[j] = S.twF[32 * (16 * hq + j) + lane];
    for (int t = 0; t < kTcTiles; t++) {
        const uint32_t kk = k + t, slot = kk % kTcSlots;
        mbar_wait(&G.full[slot], (kk / kTcSlots) & 1);
        tc_fence_after();
        unsigned char* base = G.op + t * kOpTile + opw(qd * 32 + 16 * hq, lane);
#pragma unroll
        for (int jc = 0; jc < 4; jc += 2) {
            uint32_t v[2][16];
            tc_ld16(tq + 128 * slot + 16 * jc, v[0]);
            tc_ld16(tq + 128 * slot + 16 * jc + 16, v[1]);
            tc_wait_ld();
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int j = 4 * jc + u;                  // j1 = 16 hq + j
                const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                const uint32_t x = limbs_s(y[0], y[1], y[2], y[3]);
                *reinterpret_cast<uint32_t*>(base + (j >> 3) * kOpSbo + (j & 7) * 16) = shoup_mul(x, twr[j].x, twr[j].y);
            }
        }
        fence_async_smem();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
            mbar_arrive(&G.empty[slot]);
            mbar_arrive(&G.a2[t]);
        }
    }
    k += kTcTiles;
    // ---- ep2: tile t, thread (P = 4t + qd, j1 = lane), j2 in this quad's half: A[j1 + 32 j2] in [0, 2p)
    for (int t = 0; t < kTcTiles; t++) {
        const uint32_t kk = k + t, slot = kk % kTcSlots;
        mbar_wait(&G.full[slot], (kk / kTcSlots) & 1);
        tc_fence_after();
        unsigned char* base = G.op + t * kOpTile + opw(qd * 32 + lane, 16 * hq);
#pragma unroll
        for (int c = 0; c < 4; c += 2) {
            uint32_t v[2][16];
            tc_ld16(tq + 128 * slot + 16 * c, v[0]);
            tc_ld16(tq + 128 * slot + 16 * c + 16, v[1]);
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
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&G.empty[slot]);
    }
    k += kTcTiles;
    // ---- MAC: coefficient (j1, j2 = lane) of the 2 lanes, M_o = sum_r A_r BK4[r][o] (a4.3), in place per thread.
    // The first row's BK record is requested before the group barrier (its L2 latency overlaps the wait).
    {
        const uint32_t R = c_misc[0], Rp = c_misc[1];
        const uint32_t lanew = (lane >> 2) * kOpLbo + (lane & 3) * 4;
        uint4 Bn[kBk4Rec / 4];
        const uint4* rec0 = reinterpret_cast<const uint4*>(bk4 + (size_t)(gw * 32 + lane) * kBk4Rec);
#pragma unroll
        for (int q = 0; q < kBk4Rec / 4; q++) Bn[q] = __ldg(rec0 + q);
        grp_sync(grp);                                   // every ep2 tile of the group written
        for (int j1 = gw; j1 < 32; j1 += kTcGWarps) {
            uint32_t B[kBk4Rec];
            if (j1 != gw) {
                const uint4* rec = reinterpret_cast<const uint4*>(bk4 + (size_t)(j1 * 32 + lane) * kBk4Rec);
#pragma unroll
                for (int q = 0; q < kBk4Rec / 4; q++) Bn[q] = __ldg(rec + q);
            }
#pragma unroll
            for (int q = 0; q < kBk4Rec / 4; q++) {
                B[4 * q] = Bn[q].x; B[4 * q + 1] = Bn[q].y; B[4 * q + 2] = Bn[q].z; B[4 * q + 3] = Bn[q].w;
            }
            const uint32_t rowoff = (j1 >> 3) * kOpSbo + (j1 & 7) * 16 + lanew;
            uint32_t D[kTcG][6];
#pragma unroll
            for (int g = 0; g < kTcG; g++)
#pragma unroll
                for (int r = 0; r < 6; r++) {
                    const int P = g * 6 + r;
                    D[g][r] = *reinterpret_cast<const uint32_t*>(G.op + (P >> 2) * kOpTile + (P & 3) * 4 * kOpSbo + rowoff);
                }
#pragma unroll
            for (int g = 0; g < kTcG; g++)
#pragma unroll
                for (int o = 0; o < 6; o++) {
                    uint64_t s = 0;
#pragma unroll
                    for (int r = 0; r < 6; r++) s += (uint64_t)D[g][r] * B[r * 6 + o];
                    const uint32_t hi = (uint32_t)(s >> 32), lo = (uint32_t)s;
                    *reinterpret_cast<uint32_t*>(G.op + (o % 3) * kOpTile + (g * 2 + o / 3) * 4 * kOpSbo + rowoff) =
                        red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                }
        }
    }
    fence_async_smem();
    __syncwarp();
    if (lane == 0) mbar_arrive(&G.gate);
    // ---- ep3: tile m, thread (quadrant qd = g*2 + q, j1 = lane), k2 in this quad's half: D[j1][k2] -> E -> A4
    // tile m row (qd, k2) word j1 (the tile GEMM3 just consumed)
#pragma unroll
    for (int j = 0; j < 16; j++) twr[j] = S.twI[32 * (16 * hq + j) + lane];
    for (int t = 0; t < kTcTiles; t++) {
        const uint32_t kk = k + t, slot = kk % kTcSlots;
        mbar_wait(&G.full[slot], (kk / kTcSlots) & 1);
        tc_fence_after();
        unsigned char* base = G.op + t * kOpTile + opw(qd * 32 + 16 * hq, lane);
#pragma unroll
        for (int c = 0; c < 4; c += 2) {
            uint32_t v[2][16];
            tc_ld16(tq + 128 * slot + 16 * c, v[0]);
            tc_ld16(tq + 128 * slot + 16 * c + 16, v[1]);
            tc_wait_ld();
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int j = 4 * c + u;                  // k2 = 16 hq + j
                const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                const uint32_t x = limbs_u(y[0], y[1], y[2], y[3]);
                *reinterpret_cast<uint32_t*>(base + (j >> 3) * kOpSbo + (j & 7) * 16) = shoup_mul(x, twr[j].x, twr[j].y);
            }
        }
        fence_async_smem();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&G.empty[slot]);
    }
    k += kTcTiles;
    __syncwarp();
    if (lane == 0) mbar_arrive(&G.gate);                 // GEMM4 needs every A4 tile
    // ---- ep4: tile m, thread (g = qd / 2, q = qd % 2, k2 = lane), k1 in this quad's half: part m of
    // N a[32 k1 + k2] -> centred lift, << 11 m, added into ACC[g][q] (a4.4; the parts are added one tile after
    // the other, the quads own disjoint k1)
    for (int t = 0; t < kTcTiles; t++) {
        const uint32_t kk = k + t, slot = kk % kTcSlots;
        mbar_wait(&G.full[slot], (kk / kTcSlots) & 1);
        tc_fence_after();
        uint32_t* acc = &G.acc[qd >> 1][qd & 1][32 * 16 * hq + lane];
#pragma unroll
        for (int c = 0; c < 4; c += 2) {
            uint32_t v[2][16];
            tc_ld16(tq + 128 * slot + 16 * c, v[0]);
            tc_ld16(tq + 128 * slot + 16 * c + 16, v[1]);
            tc_wait_ld();
#pragma unroll
            for (int u = 0; u < 8; u++) {
                const int j = 4 * c + u;                  // k1 = 16 hq + j
                const uint32_t* y = &v[u >> 2][4 * (u & 3)];
                const uint32_t a = lift_centred(red_2p(limbs_u(y[0], y[1], y[2], y[3])));
                acc[32 * j] += a << (11 * t);
            }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&G.empty[slot]);
    }
    k += kTcTiles;
    grp_sync(grp);                                       // ACC complete before the next step's digits
}

__device__ __forceinline__ void brt_setup(BrtSmem& S, const unsigned char* tcB, const uint2* tcTw) {
    const int tid = threadIdx.x;
    for (int e = tid; e < (int)(kTcBTotal / 16); e += kTcThreads)
        reinterpret_cast<uint4*>(S.B)[e] = __ldg(reinterpret_cast<const uint4*>(tcB) + e);
    for (int e = tid; e < 32 * 32; e += kTcThreads) {
        S.twF[e] = tcTw[e];
        S.twI[e] = tcTw[1024 + e];
    }
    if (tid >> 5 == kTcCompWarps) tc_alloc<512>(&S.tmem);
    if (tid == 0) {
        for (int gi = 0; gi < kTcGroups; gi++) {
            BrtGroup& G = S.grp[gi];
            for (int s = 0; s < kTcSlots; s++) {
                mbar_init(&G.full[s], 1);
                mbar_init(&G.empty[s], kTcGWarps);
            }
            for (int t = 0; t < kTcTiles; t++) mbar_init(&G.a2[t], kTcGWarps);
            mbar_init(&G.gate, kTcGWarps);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
}
__device__ __forceinline__ void brt_teardown(BrtSmem& S) {
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x >> 5 == kTcCompWarps) tc_dealloc<512>(S.tmem);
}

// the 630 CMux steps of the CTA: warps [8 grp, 8 grp + 8) compute for group grp, warp 16 + grp issues its MMAs
template <bool kDiag>
__device__ __forceinline__ void brt_main(BrtSmem& S, const uint32_t* __restrict__ bk4, int nsteps) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t k = 0;
    if (warp >= kTcCompWarps) {
        const int grp = warp - kTcCompWarps;
        if (lane == 0) {
            uint32_t gph = 0, aph = 0;
            for (int i = 0; i < nsteps; i++) brt_mma_step(S, S.grp[grp], S.tmem + 256 * grp, k, gph, aph);
        }
        __syncwarp();
    } else {
        const int grp = warp / kTcGWarps, gw = warp % kTcGWarps;
        BrtGroup& G = S.grp[grp];
        for (int i = 0; i < nsteps; i++) {
            if (!kDiag) brt_digits(G, i, threadIdx.x % kTcGThreads);
            brt_comp_step(S, G, S.tmem + 256 * grp, grp, gw, bk4 + (size_t)i * kN * kBk4Rec, k);
        }
    }
}

// ---- the blind-rotation kernel: a1 linear combination, a2 mod switch, a3 ACC init, a4 630 CMux, a5 extract ---
__global__ void __launch_bounds__(kTcThreads, 1) brt_kernel(BrArgs A, const uint32_t* __restrict__ bk4,
                                                             const unsigned char* __restrict__ tcB,
                                                             const uint2* __restrict__ tcTw) {
    extern __shared__ __align__(1024) unsigned char brt_smem[];
    BrtSmem& S = *reinterpret_cast<BrtSmem*>(brt_smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int lane0 = blockIdx.x * kTcLanes;
    brt_setup(S, tcB, tcTw);
    // a1 + a2: 4 compute warps per lane (lane L = grp * 2 + g)
    if (warp < kTcCompWarps) {
        const int L = warp / 4, w4 = warp % 4;
        const int gl = lane0 + L;
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t* s0 = (d.sel & 3u) == 0 ? A.src0 : ((d.sel & 3u) == 1 ? A.src1 : A.src2);
        const uint32_t sb = (d.sel >> 2) & 3u;
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        uint16_t* bar = S.grp[L / kTcG].bar[L % kTcG];
        for (int w = w4 * 32 + lane; w <= kn; w += 128) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            bar[w] = (uint16_t)((v + (1u << 20)) >> 21);      // round(v 2N / 2^32) mod 2N (C5)
        }
    }
    __syncthreads();
    // a3: ACC = (0, X^{-bbar} (mu, ..., mu))  (C6)
    for (int e = tid; e < kTcLanes * kN; e += kTcThreads) {
        const int L = e / kN, c = e % kN;
        BrtGroup& G = S.grp[L / kTcG];
        const uint32_t bbar = G.bar[L % kTcG][kn];
        G.acc[L % kTcG][0][c] = 0u;
        G.acc[L % kTcG][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();
    brt_main<false>(S, bk4, kn);
    __syncthreads();
    // a5: sample extraction, index 0 (C8)
    for (int e = tid; e < kTcLanes * (kN + 1); e += kTcThreads) {
        const int L = e / (kN + 1), j = e % (kN + 1);
        const int gl = lane0 + L;
        if (gl >= A.nlanes) continue;
        const uint32_t(*acc)[kN] = S.grp[L / kTcG].acc[L % kTcG];
        uint32_t v;
        if (j == 0) v = acc[0][0];
        else if (j < kN) v = 0u - acc[0][kN - j];
        else v = acc[1][0];
        A.out[(int64_t)gl * A.out_stride + j] = v;
    }
    brt_teardown(S);
}

// ---- diagnostic: res[L][q] = sum_r d[L][r] (x) polys[r][q] mod 2^32 through one CMux step (acc starts at 0) --
__global__ void __launch_bounds__(kTcThreads, 1) brt_muladd_kernel(const int32_t* __restrict__ digits,
                                                                    const uint32_t* __restrict__ bk4,
                                                                    const unsigned char* __restrict__ tcB,
                                                                    const uint2* __restrict__ tcTw,
                                                                    uint32_t* __restrict__ res) {
    extern __shared__ __align__(1024) unsigned char brt_smem[];
    BrtSmem& S = *reinterpret_cast<BrtSmem*>(brt_smem);
    const int tid = threadIdx.x;
    brt_setup(S, tcB, tcTw);
    for (int e = tid; e < kTcLanes * 2 * kN; e += kTcThreads) {
        const int L = e / (2 * kN);
        (&S.grp[L / kTcG].acc[L % kTcG][0][0])[e % (2 * kN)] = 0u;
    }
    // digits [L][r][1024] -> group L / 2, tile P / 4 (P = (L % 2)*6 + r), row (P % 4)*32 + k2, K byte k1
    for (int e = tid; e < kTcLanes * 6 * kN; e += kTcThreads) {
        const int L = e / (6 * kN), r = (e / kN) % 6, c = e % kN, k1 = c >> 5, k2 = c & 31;
        const int P = (L % kTcG) * 6 + r;
        S.grp[L / kTcG].op[(P >> 2) * kOpTile + tc_off((P & 3) * 32 + k2, k1, kA1Lbo, kA1Sbo)] =
            (unsigned char)(digits[e] & 0xFF);
    }
    fence_async_smem();
    __syncthreads();
    brt_main<true>(S, bk4, 1);
    __syncthreads();
    for (int e = tid; e < kTcLanes * 2 * kN; e += kTcThreads) {
        const int L = e / (2 * kN);
        res[e] = (&S.grp[L / kTcG].acc[L % kTcG][0][0])[e % (2 * kN)];
    }
    brt_teardown(S);
}

// ---- load time: BK (torus, [n][6][2][N]) -> bk4[i][32 j1 + j2][r*6 + o], o = q*3 + m: the evaluation of part m
// of BK_i[r][q] at psi^(2 j + 1), j = j1 + 32 j2, times N^-1 (Horner's rule; plain and exact, ~24 G mulmods)
__global__ void __launch_bounds__(256) bk_to_bk4_kernel(const uint32_t* __restrict__ bk, uint32_t* __restrict__ bk4,
                                                         const uint2* __restrict__ pts, uint32_t ninv,
                                                         uint32_t ninvp, int npolys) {
    __shared__ uint32_t x[kN];
    const int task = blockIdx.x;                        // (i, r, q, m)
    if (task >= npolys) return;
    const int m = task % kParts, q = (task / kParts) % 2, r = (task / (2 * kParts)) % kRows, i = task / (2 * kParts * kRows);
    const uint32_t* src = bk + (((size_t)i * kRows + r) * 2 + q) * kN;
    for (int k = threadIdx.x; k < kN; k += blockDim.x) {
        uint32_t v = src[k];
        const int32_t p0 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
        v = (v - (uint32_t)p0) >> 11;
        const int32_t p1 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
        v = (v - (uint32_t)p1) >> 11;
        const int32_t p2 = ((int32_t)((v & 0x3FFu) << 22)) >> 22;
        const int32_t pm = m == 0 ? p0 : (m == 1 ? p1 : p2);
        x[k] = pm < 0 ? (uint32_t)(pm + (int32_t)kP) : (uint32_t)pm;
    }
    __syncthreads();
    for (int j = threadIdx.x; j < kN; j += blockDim.x) {
        const uint2 w = pts[j];                         // psi^(2 j + 1) and its Shoup companion
        uint32_t acc = 0;
        for (int k = kN - 1; k >= 0; k--) acc = red_2p(add_alu(shoup_mul(acc, w.x, w.y), x[k]));
        acc = red_p(shoup_mul(acc, ninv, ninvp));
        const int j1 = j & 31, j2 = j >> 5;
        bk4[((size_t)i * kN + (j1 * 32 + j2)) * kBk4Rec + r * 6 + q * kParts + m] = acc;
    }
}

static size_t brt_smem_bytes() { return sizeof(BrtSmem); }

int launch_brt(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st) {
    static_assert(sizeof(BrtSmem) <= 232448, "brt shared memory");
    if (ensure_smem_attr<brt_kernel>(brt_smem_bytes())) return -1;
    const int blocks = (A.nlanes + kTcLanes - 1) / kTcLanes;
    if (blocks == 0) return 0;
    brt_kernel<<<blocks, kTcThreads, brt_smem_bytes(), st>>>(A, bk4, tcB, tcTw);
    return 0;
}

int launch_brt_muladd(const int32_t* digits, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw,
                      uint32_t* res, cudaStream_t st) {
    if (ensure_smem_attr<brt_muladd_kernel>(brt_smem_bytes())) return -1;
    brt_muladd_kernel<<<1, kTcThreads, brt_smem_bytes(), st>>>(digits, bk4, tcB, tcTw, res);
    return 0;
}

void launch_bk_to_bk4(const uint32_t* bk, uint32_t* bk4, const uint2* pts, uint32_t ninv, uint32_t ninvp, int n_i,
                      cudaStream_t st) {
    const int npolys = n_i * kRows * 2 * kParts;
    bk_to_bk4_kernel<<<npolys, 256, 0, st>>>(bk, bk4, pts, ninv, ninvp, npolys);
}

size_t bk4_bytes() { return (size_t)kn * kN * kBk4Rec * 4; }

// host: constant B operands and twiddle tables of the four-step transform for the root psi
void brt_tables(uint32_t psi, unsigned char* B, uint2* tw, uint2* pts) {
    auto powm = [](uint64_t b, uint64_t e) {
        uint64_t r = 1;
        b %= kP;
        while (e) {
            if (e & 1) r = r * b % kP;
            b = b * b % kP;
            e >>= 1;
        }
        return (uint32_t)r;
    };
    auto pw = [&](int64_t e) { return powm(psi, (uint64_t)(((e % 2048) + 2048) % 2048)); };
    auto shoup = [](uint32_t w) { return (uint32_t)(((uint64_t)w << 32) / kP); };
    auto byte = [](uint32_t v, int b) { return (unsigned char)((v >> (8 * b)) & 0xFFu); };
    auto dense = [](uint32_t n, uint32_t k, uint32_t K) { return tc_off(n, k, 128, (K / 16) * 128); };
    memset(B, 0, kTcBTotal);
    for (int j1 = 0; j1 < 32; j1++)                       // B1[(j1, b)][k1] = byte_b(W1[j1][k1])
        for (int k1 = 0; k1 < 32; k1++)
            for (int b = 0; b < 4; b++) B[dense(4 * j1 + b, k1, 32)] = byte(pw(32 * (2 * j1 + 1) * k1), b);
    unsigned char* B2 = B + kB1Bytes;
    unsigned char* B3 = B2 + kBBytes;
    unsigned char* B4 = B3 + kBBytes;
    for (int x = 0; x < 32; x++)
        for (int y = 0; y < 32; y++)
            for (int c = 0; c < 4; c++) {
                const uint64_t s = ((uint64_t)1 << (8 * c)) % kP;
                // B2[(j2 = x, b)][(k2 = y, c)] = byte_b(2^(8c) W2[j2][k2]), W2 = psi^(64 j2 k2)
                const uint32_t w2 = (uint32_t)(s * pw(64 * x * y) % kP);
                // B3[(k2 = x, b)][(j2 = y, c)] = byte_b(2^(8c) V2[k2][j2]), V2 = psi^(-64 j2 k2)
                const uint32_t v2 = (uint32_t)(s * pw(-64 * x * y) % kP);
                // B4[(k1 = x, b)][(j1 = y, c)] = byte_b(2^(8c) V1[k1][j1]), V1 = psi^(-32 (2 j1 + 1) k1)
                const uint32_t v1 = (uint32_t)(s * pw(-32 * (2 * y + 1) * x) % kP);
                for (int b = 0; b < 4; b++) {
                    B2[dense(4 * x + b, 4 * y + c, 128)] = byte(w2, b);
                    B3[dense(4 * x + b, 4 * y + c, 128)] = byte(v2, b);
                    B4[dense(4 * x + b, 4 * y + c, 128)] = byte(v1, b);
                }
            }
    for (int j1 = 0; j1 < 32; j1++)
        for (int k2 = 0; k2 < 32; k2++) {
            const uint32_t f = pw((2 * j1 + 1) * k2), iv = pw(-(2 * j1 + 1) * k2);
            tw[j1 * 32 + k2] = make_uint2(f, shoup(f));            // twF[j1][k2]
            tw[1024 + k2 * 32 + j1] = make_uint2(iv, shoup(iv));    // twI[k2][j1]
        }
    for (int j = 0; j < kN; j++) {
        const uint32_t w = pw(2 * j + 1);
        pts[j] = make_uint2(w, shoup(w));
    }
}
size_t brt_table_bytes() { return kTcBTotal; }

}  // namespace tb
