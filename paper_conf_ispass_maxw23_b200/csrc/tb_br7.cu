// tb_br7.cu -- blind rotation with the NTT-domain bootstrapping key streamed into shared memory by TMA bulk
// copies (the north star's "TMA-staged BK streaming amortised across a batch of gates").
//
// Same arithmetic and work split as br6_kernel (6 warps per lane, one transform per warp; bit-identical
// output).  Difference: one CTA per SM holds two lanes and the whole 144 KB NTT-domain tile BK_i of the current
// CMux step in shared memory.  One elected thread issues cp.async.bulk copies of BK_{i+1} as soon as the MAC of
// step i has consumed BK_i; they land during phases C(i) and A(i+1), so the MAC reads the key from shared memory
// instead of waiting on L2.  The transpose slots use an XOR swizzle instead of padding to make the tile fit:
// 147,456 (BK) + 49,152 (slots) + 16,384 (ACC) + 15,872 (twiddles) + 2,528 (mod-switched a) < 227 KB.
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {

constexpr int kBkStepWords = kRows * kOuts * kN;          // 36,864 words = 147,456 B per CMux step

template <int G>
struct __align__(128) Br7Smem {
    uint32_t bk[kBkStepWords];
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t acc[G][2][kN];
    uint32_t slot[G][kOuts][32 * 32];
    uint16_t bar[G][kn + 2];
    unsigned long long mbar;
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long* bar, int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}\n" ::"r"(
            smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
// one thread: request BK_i (6 bulk copies of 24 KB) on the CTA's mbarrier
template <int G>
__device__ __forceinline__ void issue_bk(Br7Smem<G>& S, const uint32_t* bkhat, int i) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // prior generic reads of S.bk are done
    mbar_expect_tx(&S.mbar, kBkStepWords * 4);
    const uint32_t* src = bkhat + (size_t)i * kBkStepWords;
#pragma unroll
    for (int r = 0; r < kRows; r++)
        bulk_g2s(S.bk + r * kOuts * kN, src + r * kOuts * kN, kOuts * kN * 4, &S.mbar);
}

__device__ __forceinline__ void named_bar7(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

template <int G>
__global__ void __launch_bounds__(192 * G, 1) br7_kernel(BrArgs A) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Br7Smem<G>& S = *reinterpret_cast<Br7Smem<G>*>(smem_raw);
    constexpr int NT = 192 * G;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = warp / 6, w6 = warp % 6;
    const int lane0 = blockIdx.x * G;

    if (tid == 0) {
        mbar_init(&S.mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (tid == 0) issue_bk(S, A.bkhat, 0);
    for (int k = tid; k < 31 * 32; k += NT) {
        S.twF[k] = A.twF[k];
        S.twI[k] = A.twI[k];
    }
    // ---- prologue (a1, a2): linear gate combination + mod switch to 2N ----
    {
        const int gl = lane0 + g;
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t sa = d.sel & 3u, sb = (d.sel >> 2) & 3u;
        const uint32_t* s0 = sa == 0 ? A.src0 : (sa == 1 ? A.src1 : A.src2);
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
    for (int k = tid; k < G * kN; k += NT) {                      // ACC = (0, X^{-bbar} (mu, ..., mu))
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        S.acc[gg][0][c] = 0u;
        S.acc[gg][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int bloc = w6 / kL, jd = w6 % kL;
    const int q = w6 / kParts, m = w6 % kParts;
    const int shift = 32 - kBgbit * (jd + 1);
    for (int i = 0; i < kn; i++) {
        // ---- phase A: rotate, one gadget digit, forward NTT ----
        {
            const uint32_t ab = S.bar[g][i];
            const uint32_t* acc = S.acc[g][bloc];
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) {
                const uint32_t c = lane + 32 * j;
                const uint32_t mm = (c - ab) & (kTwoN - 1);
                const uint32_t src = acc[mm & (kN - 1)];
                const uint32_t rot = mm < (uint32_t)kN ? src : 0u - src;
                const uint32_t u = rot - acc[c] + kDecompOffset;
                x[j] = ((u >> shift) & 127u) + (kP - 64u);
            }
            uint32_t* slot = S.slot[g][w6];
            ntt_fwd<true>(x, slot, S.twF, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) slot[sidx<true>(lane, j)] = red_2p(x[j]);
        }
        __syncthreads();
        mbar_wait(&S.mbar, (uint32_t)(i & 1));                      // BK_i has landed in shared memory
        // ---- phase B: pointwise MAC against BK_i (shared memory), both lanes ----
        for (int a = tid; a < kN; a += NT) {
            const int sa = sidx<true>(a >> 5, a & 31);
            uint32_t D[G][kRows];
#pragma unroll
            for (int gg = 0; gg < G; gg++)
#pragma unroll
                for (int r = 0; r < kRows; r++) D[gg][r] = S.slot[gg][r][sa];
#pragma unroll
            for (int o = 0; o < kOuts; o++) {
                uint64_t s[G];
#pragma unroll
                for (int gg = 0; gg < G; gg++) s[gg] = 0;
#pragma unroll
                for (int r = 0; r < kRows; r++) {
                    const uint32_t b = S.bk[(r * kOuts + o) * kN + a];
#pragma unroll
                    for (int gg = 0; gg < G; gg++) s[gg] += (uint64_t)D[gg][r] * b;
                }
#pragma unroll
                for (int gg = 0; gg < G; gg++) {
                    const uint32_t hi = (uint32_t)(s[gg] >> 32), lo = (uint32_t)s[gg];
                    S.slot[gg][o][sa] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                }
            }
        }
        __syncthreads();
        if (tid == 0 && i + 1 < kn) issue_bk(S, A.bkhat, i + 1);   // overlaps phases C(i), A(i+1)
        // ---- phase C: inverse NTT, centred lift, part recombination, ACC += ----
        {
            uint32_t* slot = S.slot[g][w6];
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = slot[sidx<true>(lane, j)];
            ntt_inv<true>(x, slot, S.twI, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = lift_centred(x[j]) << (11 * m);
            if (m != 0) {
#pragma unroll
                for (int j = 0; j < 32; j++) slot[sidx<true>(j, lane)] = x[j];
            }
            named_bar7(1 + g * 2 + q, 96);
            if (m == 0) {
                const uint32_t* p1 = S.slot[g][q * kParts + 1];
                const uint32_t* p2 = S.slot[g][q * kParts + 2];
                uint32_t* acc = S.acc[g][q];
#pragma unroll
                for (int j = 0; j < 32; j++)
                    acc[lane + 32 * j] += x[j] + p1[sidx<true>(j, lane)] + p2[sidx<true>(j, lane)];
            }
        }
        __syncthreads();
    }
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
static int launch_br7_g(const BrArgs& A, cudaStream_t st) {
    const size_t smem = sizeof(Br7Smem<G>);
    static bool attr = false;
    if (!attr) {
        if (cudaFuncSetAttribute(br7_kernel<G>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
            cudaSuccess)
            return -1;
        attr = true;
    }
    const int blocks = (A.nlanes + G - 1) / G;
    if (blocks == 0) return 0;
    br7_kernel<G><<<blocks, 192 * G, smem, st>>>(A);
    return 0;
}

// G = 2: throughput variant; G = 1: latency mode for narrow levels (one lane per SM, BK staged per step)
int launch_br7(const BrArgs& A, int G, cudaStream_t st) {
    return G == 1 ? launch_br7_g<1>(A, st) : launch_br7_g<2>(A, st);
}

}  // namespace tb
