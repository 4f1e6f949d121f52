// tb_bootstrap.cu -- load-time BK -> NTT-domain conversion and the tb_gates descriptor builder.
// (The blind-rotation kernels themselves are in tb_br6.cu, tb_br9.cu, tb_brf.cu, tb_brl.cu.)
//
// The BK split used by every blind-rotation kernel: each torus coefficient
// x = x0 + 2^11 x1 + 2^22 x2 (mod 2^32) with |x_m| <= 2^10, each part NTT-transformed mod p and pre-scaled by
// N^-1, stored [i][r][o = q*3 + m][a].
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {


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
