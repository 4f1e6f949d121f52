// tb_br9.cu -- latency-mode blind rotation: one bootstrap per thread-block cluster of two SMs (SURVEY 8(a)
// rows a1-a5; SURVEY 8(f) f4 "split one gate's CMux across a thread-block cluster").
//
// Same arithmetic as br6 (bit-identical).  CTA c of the cluster owns accumulator polynomial c (c = 0: a,
// c = 1: b).  Per CMux step i:
//   A  warps 0-2: digit jd of (X^abar - 1) ACC[c] -> forward NTT -> local rows (global rows r = 3c + jd); one
//      thread pushes the 3 rows (12 KB) into the peer's receive buffer with a shared::cta -> shared::cluster
//      bulk copy that completes on the peer's mbarrier (double-buffered by step parity)
//   B  all 8 warps: for output polynomial q = c (3 BK parts): MAC over the 3 local rows, wait for the peer's
//      rows, MAC over them (both from local shared memory), reduce
//   C  warps 0-2: inverse NTT of part m, lift, << 11m; CTA barrier; all 8 warps add the parts into ACC[c]
// The output of step i on CTA c is ACC[c] of step i+1, so accumulators never cross the cluster.  Each CTA
// stages the half of BK_i it needs (72 KB) by cp.async.bulk two steps ahead (double buffer).  There is no
// cluster-wide barrier inside the loop: the two CTAs are coupled only by the row hand-over, which also makes
// the double buffers safe (a CTA can only send rows for step i+1 after it received the peer's rows for step i,
// which the peer sent after finishing its MAC of step i-1, the last reader of that buffer).
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {

constexpr int kB9HalfWords = kRows * kParts * kN;          // 18,432 words = 72 KB per CTA per step
constexpr int kB9RowWords = kL * 32 * 32;                   // 3 rows = 12 KB
constexpr int kB9Threads = 256;                             // 8 warps: 0-2 transform, all 8 MAC (4 coefficients each)

struct __align__(128) Br9Smem {
    uint32_t bk[2][kB9HalfWords];       // [step & 1][r][m][a] for this CTA's output q = c
    uint32_t dslot[kL][32 * 32];        // own forward NTT rows (swizzled 32x32)
    uint32_t rrows[2][kL][32 * 32];     // the peer's rows, by step parity
    uint32_t oslot[kParts][32 * 32];    // MAC outputs (q = c, part m)
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t acc[kN];                   // ACC[c]
    uint16_t bar[kn + 2];
    unsigned long long mbar_bk[2];
    unsigned long long mbar_rows[2];
};

__device__ __forceinline__ uint32_t smem_u32_9(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void cluster_sync9() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t map_peer(uint32_t local_shared_addr, uint32_t rank) {
    uint32_t out;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(out) : "r"(local_shared_addr), "r"(rank));
    return out;
}
__device__ __forceinline__ void mbar_init9(unsigned long long* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32_9(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect9(unsigned long long* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32_9(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait9(unsigned long long* bar, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n W9_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra W9_%=;\n}\n" ::"r"(smem_u32_9(bar)),
        "r"(parity)
        : "memory");
}
// one thread: BK_i (this CTA's outputs 3c..3c+2 for all 6 rows) -> bk[buf]
__device__ __forceinline__ void issue_bk9(Br9Smem& S, const uint32_t* bkhat, int i, int c, int buf) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mbar_expect9(&S.mbar_bk[buf], kB9HalfWords * 4);
    const uint32_t* src = bkhat + (size_t)i * (kRows * kOuts * kN) + c * kParts * kN;
#pragma unroll
    for (int r = 0; r < kRows; r++)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32_9(S.bk[buf] + r * kParts * kN)),
            "l"(src + r * kOuts * kN), "r"(kParts * kN * 4), "r"(smem_u32_9(&S.mbar_bk[buf]))
            : "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kB9Threads, 1) br9_kernel(BrArgs A) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Br9Smem& S = *reinterpret_cast<Br9Smem*>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t c = cluster_rank(), peer = c ^ 1u;
    const int gl = blockIdx.x >> 1;                        // one lane (bootstrap) per cluster

    if (tid == 0) {
        for (int b = 0; b < 2; b++) {
            mbar_init9(&S.mbar_bk[b]);
            mbar_init9(&S.mbar_rows[b]);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        mbar_expect9(&S.mbar_rows[0], kB9RowWords * 4);    // rows of steps 0 and 1 may arrive any time now
        mbar_expect9(&S.mbar_rows[1], kB9RowWords * 4);
    }
    __syncthreads();
    if (tid == 0) {
        issue_bk9(S, A.bkhat, 0, (int)c, 0);
        issue_bk9(S, A.bkhat, 1, (int)c, 1);
    }
    for (int k = tid; k < 31 * 32; k += kB9Threads) {
        S.twF[k] = A.twF[k];
        S.twI[k] = A.twI[k];
    }
    {   // a1, a2: both CTAs mod-switch the lane's linear combination
        LaneDesc d = {0, -1, 0, 0, 0u, 0u, 0u, 0u};
        if (gl < A.nlanes) d = A.lanes[gl];
        const uint32_t sa = d.sel & 3u, sb = (d.sel >> 2) & 3u;
        const uint32_t* s0 = sa == 0 ? A.src0 : (sa == 1 ? A.src1 : A.src2);
        const uint32_t* s1 = sb == 0 ? A.src0 : (sb == 1 ? A.src1 : A.src2);
        const uint32_t* pa = s0 + (int64_t)d.ia * A.src_stride;
        const uint32_t* pb = d.ib >= 0 ? s1 + (int64_t)d.ib * A.src_stride : nullptr;
        for (int w = tid; w <= kn; w += kB9Threads) {
            uint32_t v = (gl < A.nlanes) ? (uint32_t)d.wa * __ldg(pa + w) : 0u;
            if (pb) v += (uint32_t)d.wb * __ldg(pb + w);
            if (w == kn) v += d.cst;
            S.bar[w] = (uint16_t)((v + (1u << 20)) >> 21);
        }
    }
    __syncthreads();
    for (int k = tid; k < kN; k += kB9Threads) {                  // a3: ACC[0] = 0, ACC[1] = X^{-bbar} (mu, ..., mu)
        const uint32_t bbar = S.bar[kn];
        S.acc[k] = c == 0 ? 0u : (((k + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu));
    }
    cluster_sync9();                                        // both CTAs' mbarriers are initialised and armed

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int jd = warp;                                    // warps 0-2: digit jd / part m = warp
    const int shift = 32 - kBgbit * (jd + 1);
    const uint32_t peer_rrows = map_peer(smem_u32_9(&S.rrows[0][0][0]), peer);
    const uint32_t peer_mbar = map_peer(smem_u32_9(&S.mbar_rows[0]), peer);

    for (int i = 0; i < kn; i++) {
        const int buf = i & 1;
        {   // ---- A0: (X^abar - 1) ACC[c] + decomposition offset, all 8 warps, into oslot[0] (free until the MAC)
            const uint32_t ab = S.bar[i];
            for (int k = tid; k < kN; k += kB9Threads) {
                const uint32_t mm = ((uint32_t)k - ab) & (kTwoN - 1);
                const uint32_t src = S.acc[mm & (kN - 1)];
                S.oslot[0][k] = (mm < (uint32_t)kN ? src : 0u - src) - S.acc[k] + kDecompOffset;
            }
        }
        __syncthreads();
        if (warp < kL) {   // ---- A ----
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = ((S.oslot[0][lane + 32 * j] >> shift) & 127u) + (kP - 64u);
            ntt_fwd<true>(x, S.dslot[jd], S.twF, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) S.dslot[jd][sidx<true>(lane, j)] = red_2p(x[j]);
        }
        __syncthreads();
        if (tid == 0) {   // hand our rows to the peer (lands in its rrows[buf], completes its mbar_rows[buf])
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile(
                "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    peer_rrows + (uint32_t)(buf * kB9RowWords * 4)),
                "r"(smem_u32_9(&S.dslot[0][0])), "r"(kB9RowWords * 4), "r"(peer_mbar + (uint32_t)(buf * 8))
                : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
        mbar_wait9(&S.mbar_bk[buf], (uint32_t)((i >> 1) & 1));             // BK_i has landed
        // ---- B: out[m][a] = sum_{r<6} D_r[a] BK_i[r][3c + m][a]; own rows first, then the peer's ----
        constexpr int KMAX = (kN + kB9Threads - 1) / kB9Threads;
        uint64_t acc[KMAX][kParts];
        const uint32_t* bk = S.bk[buf];
#pragma unroll
        for (int k = 0; k < KMAX; k++) {
            const int a = tid + kB9Threads * k;
#pragma unroll
            for (int m = 0; m < kParts; m++) acc[k][m] = 0ull;
            if (a < kN) {
                const int sa = sidx<true>(a >> 5, a & 31);
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const uint32_t dv = S.dslot[r][sa];
                    const int rg = (int)c * kL + r;
#pragma unroll
                    for (int m = 0; m < kParts; m++) acc[k][m] += (uint64_t)dv * bk[(rg * kParts + m) * kN + a];
                }
            }
        }
        mbar_wait9(&S.mbar_rows[buf], (uint32_t)((i >> 1) & 1));           // the peer's rows have landed
#pragma unroll
        for (int k = 0; k < KMAX; k++) {
            const int a = tid + kB9Threads * k;
            if (a < kN) {
                const int sa = sidx<true>(a >> 5, a & 31);
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const uint32_t dv = S.rrows[buf][r][sa];
                    const int rg = (int)peer * kL + r;
#pragma unroll
                    for (int m = 0; m < kParts; m++) acc[k][m] += (uint64_t)dv * bk[(rg * kParts + m) * kN + a];
                }
#pragma unroll
                for (int m = 0; m < kParts; m++) {
                    const uint32_t hi = (uint32_t)(acc[k][m] >> 32), lo = (uint32_t)acc[k][m];
                    S.oslot[m][sa] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
                }
            }
        }
        __syncthreads();                                   // bk[buf], rrows[buf] consumed; oslot complete
        if (tid == 0) {
            if (i + 2 < kn) {
                mbar_expect9(&S.mbar_rows[buf], kB9RowWords * 4);            // rows of step i + 2
                issue_bk9(S, A.bkhat, i + 2, (int)c, buf);
            }
        }
        if (warp < kParts) {   // ---- C ----
            const int m = warp;
            uint32_t* slot = S.oslot[m];
            uint32_t x[32];
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = slot[sidx<true>(lane, j)];
            ntt_inv<true>(x, slot, S.twI, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) slot[sidx<true>(j, lane)] = lift_centred(x[j]) << (11 * m);
        }
        __syncthreads();
        for (int k = tid; k < kN; k += kB9Threads) {       // ACC[c] += the three parts, over all 8 warps
            const int sk = sidx<true>(k >> 5, k & 31);
            S.acc[k] += S.oslot[0][sk] + S.oslot[1][sk] + S.oslot[2][sk];
        }
        if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");   // dslot free again
        __syncthreads();
    }
    cluster_sync9();
    if (gl < A.nlanes) {   // a5: CTA 0 holds ACC.a, CTA 1 holds ACC.b
        uint32_t* o = A.out + (int64_t)gl * A.out_stride;
        if (c == 0) {
            for (int j = tid; j < kN; j += kB9Threads) o[j] = j == 0 ? S.acc[0] : 0u - S.acc[kN - j];
        } else if (tid == 0) {
            o[kN] = S.acc[0];
        }
    }
}

int launch_br9(const BrArgs& A, cudaStream_t st) {
    const size_t smem = sizeof(Br9Smem);
    if (ensure_smem_attr<br9_kernel>(smem)) return -1;
    if (A.nlanes <= 0) return 0;
    br9_kernel<<<2 * A.nlanes, kB9Threads, smem, st>>>(A);
    return 0;
}

}  // namespace tb
