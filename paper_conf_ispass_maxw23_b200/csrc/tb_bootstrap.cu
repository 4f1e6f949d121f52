// tb_bootstrap.cu -- the blind-rotation kernel and the BK -> NTT-domain kernel.
//
// PAPER.md: bootstrapping "dominates the execution time"; in a gate, blind rotation is the largest
// slice (Fig. 7); its NTT work is "highly vectorizable" and independent gates "can be executed in
// parallel".  This kernel therefore batches G independent bootstraps ("lanes") per CTA so that each
// NTT-domain BK tile fetched for CMux step i feeds G accumulators, and runs all n = 630 CMux steps of those
// lanes with the accumulators resident in shared memory (no HBM traffic for ACC).
//
// Per CTA: 2G warps.  Per CMux step i (for every lane g):
//   phase A (warp (g, bloc)): T = (X^abar_i - 1) ACC[bloc]; 3 gadget digits of T (a4.1) -> 3 forward NTTs
//   phase B (all threads)   : per NTT slot a: out[g][o][a] = sum_r D[g][r][a] * BKhat_i[r][o][a]  (a4.3)
//   phase C (warp (g, q))   : 3 inverse NTTs (one per BK part), centred lift, recombine the parts,
//                             ACC[q] += result (a4.4)
// Exactness: DESIGN.md "Exactness" -- the integer result equals the schoolbook product mod 2^32 bit for bit.
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {


template <int G>
struct BrSmem {
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t acc[G][2][kN];
    uint32_t slot[G][kOuts][kSlotWords];
    uint16_t bar[G][kn + 2];
};

__device__ __forceinline__ const uint32_t* src_ptr(const BrArgs& A, uint32_t sel) {
    return sel == 0 ? A.src0 : (sel == 1 ? A.src1 : A.src2);
}

template <int G>
__global__ void __launch_bounds__(64 * G) br_kernel(BrArgs A) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    BrSmem<G>& S = *reinterpret_cast<BrSmem<G>*>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int lane0 = blockIdx.x * G;

    for (int k = tid; k < 31 * 32; k += blockDim.x) {
        S.twF[k] = A.twF[k];
        S.twI[k] = A.twI[k];
    }
    // ---- prologue (a1, a2): linear gate combination + mod switch to 2N, one warp pair per lane ----
    {
        const int g = warp >> 1;
        const int gl = lane0 + g;
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t* pa = src_ptr(A, d.sel & 3u) + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? src_ptr(A, (d.sel >> 2) & 3u) + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = (warp & 1) * 32 + lane; w <= kn; w += 64) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[g][w] = (uint16_t)((v + (1u << 20)) >> 21);      // round(v 2N / 2^32) mod 2N (C5)
        }
    }
    __syncthreads();
    // ---- ACC = (0, X^{-bbar} (mu, ..., mu))  (a3, C6) ----
    for (int k = tid; k < G * kN; k += blockDim.x) {
        const int g = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[g][kn];
        S.acc[g][0][c] = 0u;
        S.acc[g][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    for (int i = 0; i < kn; i++) {
        // ---- phase A: rotate, decompose, forward NTT (a4.1, a4.2) ----
        {
            const int g = warp >> 1, bloc = warp & 1;
            const uint32_t ab = S.bar[g][i];
            const uint32_t* acc = S.acc[g][bloc];
            uint32_t U[32];
#pragma unroll
            for (int j = 0; j < 32; j++) {
                const uint32_t c = lane + 32 * j;
                const uint32_t m = (c - ab) & (kTwoN - 1);            // X^ab ACC: coefficient c
                const uint32_t src = acc[m & (kN - 1)];
                const uint32_t rot = m < (uint32_t)kN ? src : 0u - src;
                U[j] = rot - acc[c] + kDecompOffset;                    // (X^ab - 1) ACC + offset
            }
#pragma unroll
            for (int jd = 0; jd < kL; jd++) {
                uint32_t x[32];
#pragma unroll
                for (int j = 0; j < 32; j++)                             // digit in [-64, 63], as mod p
                    x[j] = ((U[j] >> (32 - kBgbit * (jd + 1))) & 127u) + (kP - 64u);
                uint32_t* slot = S.slot[g][bloc * kL + jd];
                ntt_fwd(x, slot, S.twF, lane);
#pragma unroll
                for (int j = 0; j < 32; j++) slot[kPadRow * lane + j] = red_2p(x[j]);
            }
        }
        __syncthreads();
        // ---- phase B: pointwise MAC against the NTT-domain BK_i, shared by the CTA's G lanes (a4.3) ----
        {
            const uint32_t* bki = A.bkhat + (size_t)i * (kRows * kOuts * kN);
            for (int a = tid; a < kN; a += 64 * G) {
                const int pa = a + (a >> 5);
                uint64_t acc[G][kOuts];
#pragma unroll
                for (int g = 0; g < G; g++)
#pragma unroll
                    for (int o = 0; o < kOuts; o++) acc[g][o] = 0ull;
#pragma unroll
                for (int r = 0; r < kRows; r++) {
                    uint32_t B[kOuts];
#pragma unroll
                    for (int o = 0; o < kOuts; o++) B[o] = __ldg(bki + (r * kOuts + o) * kN + a);
#pragma unroll
                    for (int g = 0; g < G; g++) {
                        const uint32_t dv = S.slot[g][r][pa];
#pragma unroll
                        for (int o = 0; o < kOuts; o++) acc[g][o] += (uint64_t)dv * B[o];
                    }
                }
#pragma unroll
                for (int g = 0; g < G; g++)
#pragma unroll
                    for (int o = 0; o < kOuts; o++) {
                        const uint32_t hi = (uint32_t)(acc[g][o] >> 32), lo = (uint32_t)acc[g][o];
                        const uint32_t v = shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP);   // < 4p
                        S.slot[g][o][pa] = red_2p(v);
                    }
            }
        }
        __syncthreads();
        // ---- phase C: inverse NTTs, centred lift, part recombination, ACC += (a4.4) ----
        {
            const int g = warp >> 1, q = warp & 1;
            uint32_t sum[32];
#pragma unroll
            for (int j = 0; j < 32; j++) sum[j] = 0u;
#pragma unroll
            for (int m = 0; m < kParts; m++) {
                uint32_t* slot = S.slot[g][q * kParts + m];
                uint32_t x[32];
#pragma unroll
                for (int j = 0; j < 32; j++) x[j] = slot[kPadRow * lane + j];
                ntt_inv(x, slot, S.twI, lane);
#pragma unroll
                for (int j = 0; j < 32; j++) sum[j] += lift_centred(x[j]) << (11 * m);
            }
            uint32_t* acc = S.acc[g][q];
#pragma unroll
            for (int j = 0; j < 32; j++) acc[lane + 32 * j] += sum[j];
        }
        __syncthreads();
    }
    // ---- sample extraction, index 0 (a5, C8) ----
    {
        const int g = warp >> 1;
        const int gl = lane0 + g;
        if (gl < A.nlanes) {
            uint32_t* o = A.out + (int64_t)gl * A.out_stride;
            for (int j = (warp & 1) * 32 + lane; j <= kN; j += 64) {
                uint32_t v;
                if (j == 0) v = S.acc[g][0][0];
                else if (j < kN) v = 0u - S.acc[g][0][kN - j];
                else v = S.acc[g][1][0];
                o[j] = v;
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------------
// BK (torus, [n][6][2][N] u32) -> NTT domain [n][6][6][N]: each coefficient split into 3 signed parts
// x = x0 + 2^11 x1 + 2^22 x2 (mod 2^32), |x_m| <= 2^10; each part transformed and scaled by N^-1 mod p.
// One warp per (i, r, q, m).  Load time only (tb_load_bk), not on the timed path.
__global__ void __launch_bounds__(256) bk_to_ntt_kernel(const uint32_t* __restrict__ bk, uint32_t* __restrict__ bkhat,
                                                        const uint2* twF, uint32_t ninv, uint32_t ninvp) {
    __shared__ uint32_t buf[8][kSlotWords];
    __shared__ uint2 tw[31 * 32];
    for (int k = threadIdx.x; k < 31 * 32; k += blockDim.x) tw[k] = twF[k];
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int task = blockIdx.x * 8 + warp;
    if (task >= kn * kRows * 2 * kParts) return;
    const int m = task % kParts;
    const int q = (task / kParts) % 2;
    const int r = (task / (2 * kParts)) % kRows;
    const int i = task / (2 * kParts * kRows);
    const uint32_t* src = bk + (((size_t)i * kRows + r) * 2 + q) * kN;
    uint32_t x[32];
#pragma unroll
    for (int j = 0; j < 32; j++) {
        uint32_t v = src[lane + 32 * j];
        const int32_t p0 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
        v = (v - (uint32_t)p0) >> 11;
        const int32_t p1 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
        v = (v - (uint32_t)p1) >> 11;
        const int32_t p2 = ((int32_t)((v & 0x3FFu) << 22)) >> 22;
        const int32_t pm = m == 0 ? p0 : (m == 1 ? p1 : p2);
        x[j] = pm < 0 ? (uint32_t)(pm + (int32_t)kP) : (uint32_t)pm;
    }
    ntt_fwd(x, buf[warp], tw, lane);
    uint32_t* dst = bkhat + (((size_t)i * kRows + r) * kOuts + q * kParts + m) * kN;
#pragma unroll
    for (int j = 0; j < 32; j++) dst[32 * lane + j] = red_p(shoup_mul(x[j], ninv, ninvp));
}

// ---------------------------------------------------------------------------------------------------
// Descriptor builder for tb_gates: count gates of one type over arrays (src0 = ca, src1 = cb, src2 = cc).
__global__ void build_gate_desc_kernel(int gate_kind, int32_t wa, int32_t wb, uint32_t cst, int64_t count,
                                       LaneDesc* lanes, GateDesc* gates) {
    const int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (g >= count) return;
    GateDesc gd;
    gd.out_row = (int32_t)g;
    gd.kind = gate_kind;
    if (gate_kind == kGateNot) {
        gd.lane0 = (int32_t)g;
        gd.lane1 = -1;
    } else if (gate_kind == kGateMux) {
        // MUX(a,b,c) = KS((0,1/8) + BR(AND(a,b)) + BR(ANDNY(a,c)))
        LaneDesc l0 = {(int32_t)g, (int32_t)g, 1, 1, (uint32_t)(0u - kMu), 0u | (1u << 2), 0u, 0u};
        LaneDesc l1 = {(int32_t)g, (int32_t)g, -1, 1, (uint32_t)(0u - kMu), 0u | (2u << 2), 0u, 0u};
        lanes[2 * g] = l0;
        lanes[2 * g + 1] = l1;
        gd.lane0 = (int32_t)(2 * g);
        gd.lane1 = (int32_t)(2 * g + 1);
    } else {
        LaneDesc l0 = {(int32_t)g, wb ? (int32_t)g : -1, wa, wb, cst, 0u | (1u << 2), 0u, 0u};
        lanes[g] = l0;
        gd.lane0 = (int32_t)g;
        gd.lane1 = -1;
    }
    gates[g] = gd;
}

// ---------------------------------------------------------------------------------------------------
// host-side launchers (C++ linkage, used by tb_runtime.cu)
template <int G>
static int launch_br_g(const BrArgs& A, cudaStream_t st) {
    const size_t smem = sizeof(BrSmem<G>);
    static bool attr = false;
    if (!attr) {
        if (cudaFuncSetAttribute(br_kernel<G>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
            return -1;
        attr = true;
    }
    const int blocks = (A.nlanes + G - 1) / G;
    if (blocks == 0) return 0;
    br_kernel<G><<<blocks, 64 * G, smem, st>>>(A);
    return 0;
}

int launch_br(const BrArgs& A, int G, cudaStream_t st) {
    switch (G) {
        case 1: return launch_br_g<1>(A, st);
        case 2: return launch_br_g<2>(A, st);
        case 3: return launch_br_g<3>(A, st);
        case 4: return launch_br_g<4>(A, st);
        default: return -2;
    }
}

size_t br_smem_bytes(int G) {
    switch (G) {
        case 1: return sizeof(BrSmem<1>);
        case 2: return sizeof(BrSmem<2>);
        case 3: return sizeof(BrSmem<3>);
        case 4: return sizeof(BrSmem<4>);
        default: return 0;
    }
}

void launch_bk_to_ntt(const uint32_t* bk, uint32_t* bkhat, const uint2* twF, uint32_t ninv, uint32_t ninvp,
                      cudaStream_t st) {
    const int tasks = kn * kRows * 2 * kParts;
    bk_to_ntt_kernel<<<(tasks + 7) / 8, 256, 0, st>>>(bk, bkhat, twF, ninv, ninvp);
}

void launch_build_gate_desc(int kind, int32_t wa, int32_t wb, uint32_t cst, int64_t count, LaneDesc* lanes,
                            GateDesc* gates, cudaStream_t st) {
    if (count <= 0) return;
    build_gate_desc_kernel<<<(unsigned)((count + 255) / 256), 256, 0, st>>>(kind, wa, wb, cst, count, lanes, gates);
}

}  // namespace tb
