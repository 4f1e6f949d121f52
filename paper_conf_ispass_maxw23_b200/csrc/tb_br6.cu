// tb_br6.cu -- the blind-rotation kernel, six warps per lane.
//
// PAPER.md: bootstrapping "dominates the execution time"; in a gate, blind rotation is the largest
// slice (Fig. 7); its NTT work is "highly vectorizable" and independent gates "can be executed in
// parallel".  A CTA therefore batches G independent bootstraps ("lanes") so that each NTT-domain BK
// word fetched for CMux step i feeds G accumulators, and runs all n = 630 CMux steps of those lanes with the
// accumulators resident in shared memory.  The work of one CMux step is spread over 6 warps per lane (one
// transform per warp) so that an SM holds 24 warps (2 CTAs x 2 lanes x 6):
//   phase A (warp (g, r), r = bloc*l + jd): digit jd of (X^abar - 1) ACC[bloc] -> forward NTT -> slot r
//   phase B (all threads, one coefficient a per item): the 36 BK_i words of a are loaded at once (MLP for
//           the L2 latency), out[g][o][a] = sum_r D[g][r][a] BKhat_i[r][o][a], written back in place
//   phase C (warp (g, o), o = q*3 + m): inverse NTT of slot o, centred lift, << 11m; the three part warps of
//           output q meet at a named barrier and warp m = 0 adds the parts into ACC[q].
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {

template <int G>
struct Br6Smem {
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t acc[G][2][kN];
    uint32_t slot[G][kOuts][kSlotWords];
    uint16_t bar[G][kn + 2];
};

__device__ __forceinline__ void named_bar(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

template <int G>
__global__ void __launch_bounds__(192 * G, (G <= 2 ? 2 : 1)) br6_kernel(BrArgs A) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Br6Smem<G>& S = *reinterpret_cast<Br6Smem<G>*>(smem_raw);
    constexpr int NT = 192 * G;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = warp / 6, w6 = warp % 6;
    const int lane0 = blockIdx.x * G;

    for (int k = tid; k < 31 * 32; k += NT) {
        S.twF[k] = A.twF[k];
        S.twI[k] = A.twI[k];
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
    __syncthreads();
    // ---- ACC = (0, X^{-bbar} (mu, ..., mu))  (a3, C6) ----
    for (int k = tid; k < G * kN; k += NT) {
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        S.acc[gg][0][c] = 0u;
        S.acc[gg][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int bloc = w6 / kL, jd = w6 % kL;      // phase A role
    const int q = w6 / kParts, m = w6 % kParts;  // phase C role
    const int shift = 32 - kBgbit * (jd + 1);
    for (int i = 0; i < kn; i++) {
        // ---- phase A: rotate, one gadget digit, forward NTT (a4.1, a4.2) ----
        {
            const uint32_t ab = S.bar[g][i];
            const uint32_t* acc = S.acc[g][bloc];
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) {
                const uint32_t c = lane + 32 * j;
                const uint32_t mm = (c - ab) & (kTwoN - 1);           // X^ab ACC: coefficient c
                const uint32_t src = acc[mm & (kN - 1)];
                const uint32_t rot = mm < (uint32_t)kN ? src : 0u - src;
                const uint32_t u = rot - acc[c] + c_misc[3];          // (X^ab - 1) ACC + offset (misc[3])
                x[j] = ((u >> shift) & 127u) + (kP - 64u);             // digit in [-64, 63], as mod p
            }
            uint32_t* slot = S.slot[g][w6];
            ntt_fwd(x, slot, S.twF, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) slot[kPadRow * lane + j] = red_2p(x[j]);
        }
        __syncthreads();
        // ---- phase B: pointwise MAC against BKhat_i, shared by the CTA's lanes (a4.3) ----
        {
            const uint32_t* bki = A.bkhat + (size_t)i * (kRows * kOuts * kN);
            for (int a = tid; a < kN; a += NT) {
                const int pa = a + (a >> 5);
                uint32_t B[kRows][kOuts];
#pragma unroll
                for (int r = 0; r < kRows; r++)
#pragma unroll
                    for (int o = 0; o < kOuts; o++) B[r][o] = __ldg(bki + (r * kOuts + o) * kN + a);
#pragma unroll
                for (int gg = 0; gg < G; gg++) {
                    uint32_t D[kRows];
#pragma unroll
                    for (int r = 0; r < kRows; r++) D[r] = S.slot[gg][r][pa];
#pragma unroll
                    for (int o = 0; o < kOuts; o++) {
                        uint64_t s = 0;
#pragma unroll
                        for (int r = 0; r < kRows; r++) s += (uint64_t)D[r] * B[r][o];
                        const uint32_t hi = (uint32_t)(s >> 32), lo = (uint32_t)s;
                        S.slot[gg][o][pa] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                    }
                }
            }
        }
        __syncthreads();
        // ---- phase C: inverse NTT, centred lift, part recombination, ACC += (a4.4) ----
        {
            uint32_t* slot = S.slot[g][w6];
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = slot[kPadRow * lane + j];
            ntt_inv(x, slot, S.twI, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = lift_centred(x[j]) << (11 * m);
            if (m != 0) {
#pragma unroll
                for (int j = 0; j < 32; j++) slot[kPadRow * j + lane] = x[j];   // natural order c = lane + 32 j
            }
            named_bar(1 + g * 2 + q, 96);
            if (m == 0) {
                const uint32_t* p1 = S.slot[g][q * kParts + 1];
                const uint32_t* p2 = S.slot[g][q * kParts + 2];
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
}

template <int G>
static int launch_br6_g(const BrArgs& A, cudaStream_t st) {
    const size_t smem = sizeof(Br6Smem<G>);
    if (ensure_smem_attr<br6_kernel<G>>(smem)) return -1;
    const int blocks = (A.nlanes + G - 1) / G;
    if (blocks == 0) return 0;
    br6_kernel<G><<<blocks, 192 * G, smem, st>>>(A);
    return 0;
}

int launch_br6(const BrArgs& A, int G, cudaStream_t st) {
    switch (G) {
        case 1: return launch_br6_g<1>(A, st);
        case 2: return launch_br6_g<2>(A, st);
        case 3: return launch_br6_g<3>(A, st);
        case 4: return launch_br6_g<4>(A, st);
        default: return -2;
    }
}

}  // namespace tb
