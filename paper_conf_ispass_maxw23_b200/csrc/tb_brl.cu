// tb_brl.cu -- latency-mode blind rotation on the FP64 pipe: one bootstrap per thread-block cluster of four SMs
// (SURVEY 8(f) f4 "single-gate latency path ... split across a thread-block cluster").
//
// Same CMux and the same exact FFT-domain products as brf (tb_fft.cuh),
// so the output is bit-identical to every other variant.  What changes is how one CMux step is spread out, to
// shorten the serial chain of 630 steps that bounds a narrow netlist level:
//   * CTA (q, h) of the cluster (rank 2q + h) owns output polynomial q and BK half h: it computes the 3 digit
//     rows of ACC[q] (the two CTAs of a q compute them redundantly) and splits the MAC by bloc (it is linear):
//     its own rows times BK_i for its output o = 2q + h and, for half of the positions ([256 h, 256 h + 256)),
//     for both outputs of the other bloc; it sends each of those two partials (4 KB) to the CTA that owns the
//     output, receives its own output's other-bloc partial from both CTAs of bloc 1-q (8 KB; round 1 sent the
//     three rows, 24 KB, and multiplied the received rows itself), and runs one inverse transform; the two CTAs
//     of a q swap their rounded halves
//     and both add lo + 2^16 hi into their copy of ACC[q].  The summation order differs from the other
//     variants; the FP64 error bound does not depend on it, so the rounded products are identical.
//   * both hand-overs are per-thread st.async stores straight from registers into the peer's shared memory,
//     completing on its mbarrier (no staging buffer, no barrier and proxy fence before a bulk copy: one-gate
//     level 1.79 -> 1.58 ms), double-buffered by step parity (safe for the same reason as br9's
//     hand-over: a CTA can only send for step i+2 after it has received the receiver's data of step i+1 -- both
//     CTAs of the other bloc send to both of this bloc -- which the receiver produced after consuming step i).
//   * every transform is split over 2 warps (64 threads x 8 values) and done as three radix-8 passes (stages
//     1-3, 4-6, 7-9 of the merged-twist tree), with one shared-memory exchange between passes; the pass-2/3
//     twiddles of a thread stay in registers for the whole kernel.
//   * BK_i's 48 KB (own rows x output o, and x the other bloc's outputs on half the positions) are TMA-staged
//     two steps ahead.
#include "tb_fft.cuh"
#include "tb_kernels.cuh"

namespace tb {

constexpr int kLThreads = 256;                 // 8 warps: 3 forward transforms x 2 warps (0-5); warps 0-1 invert; all MAC
constexpr int kLMacIt = (512 + kLThreads - 1) / kLThreads;
#ifndef TB_BRL_BK_ISSUER
#define TB_BRL_BK_ISSUER 64
#endif
constexpr int kBkIssuer = TB_BRL_BK_ISSUER;   // thread that issues the per-step BK TMA (outside warps 0-1)
constexpr uint32_t kPartBytes = 512 * 16;   // the other bloc's partial MAC of this CTA's output (512 complex)

#ifdef TB_BRL_TRACE   // scratch instrumentation (tools/buildvar.sh WORK name -DTB_BRL_TRACE): clock64 per phase
__device__ long long g_brl_trace[4][8][16];
#define BRL_T(p)                                                                                              \
    if (gl == 0 && tid == 0 && i >= 100 && i < 116) g_brl_trace[rank][p][i - 100] = clock64();
#else
#define BRL_T(p)
#endif

struct __align__(128) BrlSmem {
    double2 bk[2][kRows][512];                 // BK_i (issue_bk_l), by step parity (96 KB)
    double2 dslot[kL][512];                    // own forward rows (bloc q), swizzled positions
    double2 precv[2][512];                     // the partner's partial MAC of this CTA's output, by step parity
    double2 oslot[512];                        // MAC output, then the inverse's exchange buffer
    uint32_t res[kN];                          // own rounded half of the product (sent to the sibling)
    uint32_t rres[2][kN];                      // the sibling's half, by step parity
    uint32_t acc[3 * kN];                      // ACC[q] as (acc, -acc, acc)
    uint16_t bar[kn + 2];
    unsigned long long mbar_bk[2], mbar_part[2], mbar_res[2];
};

// swizzled slot of transform position k: each of the three pass groupings below touches 8 distinct 16-byte
// bank groups per 8 consecutive threads (conflict-free)
__device__ __forceinline__ int lsw(int k) { return k ^ ((k >> 3) & 7); }
// position of element v of thread tt in the groupings of pass 1 (bits 8-6 in-thread), 2 (bits 5-3), 3 (bits 2-0)
__device__ __forceinline__ int gp1(int tt, int v) { return (v << 6) | tt; }
__device__ __forceinline__ int gp2(int tt, int v) { return ((tt >> 3) << 6) | (v << 3) | (tt & 7); }
__device__ __forceinline__ int gp3(int tt, int v) { return (tt << 3) | v; }

struct PassTw {
    dcplx a, b, c;    // zeta_{s, b0}, zeta_{s+1, 2 b0}, zeta_{s+2, 4 b0} for the pass's stages s, s+1, s+2
};
// twiddle of the third stage of a pass, block 4 b0 + f: the bits of f land on exponent bits 9, 8 of brv10
__device__ __forceinline__ dcplx tw_third(dcplx c, int f) {
    constexpr double c4 = 0.70710678118654752440;
    const dcplx w = (f >> 1) ? mul_k(c, c4, c4) : c;
    return (f & 1) ? mul_i(w) : w;
}
// element v = (v2 v1 v0): first stage pairs v2, second v1 (block 2 b0 + v2), third v0 (block 4 b0 + 2 v2 + v1)
__device__ __forceinline__ void pass_fwd(dcplx (&x)[8], const PassTw& t) {
#pragma unroll
    for (int u = 0; u < 4; u++) ct_c(x[u], x[u + 4], t.a);
#pragma unroll
    for (int e = 0; e < 2; e++) {
        const dcplx w = e ? mul_i(t.b) : t.b;
#pragma unroll
        for (int u = 0; u < 2; u++) ct_c(x[4 * e + u], x[4 * e + u + 2], w);
    }
#pragma unroll
    for (int f = 0; f < 4; f++) ct_c(x[2 * f], x[2 * f + 1], tw_third(t.c, f));
}
__device__ __forceinline__ void pass_inv(dcplx (&x)[8], const PassTw& t) {
#pragma unroll
    for (int f = 0; f < 4; f++) gs_c(x[2 * f], x[2 * f + 1], tw_third(t.c, f));
#pragma unroll
    for (int e = 0; e < 2; e++) {
        const dcplx w = e ? mul_i(t.b) : t.b;
#pragma unroll
        for (int u = 0; u < 2; u++) gs_c(x[4 * e + u], x[4 * e + u + 2], w);
    }
#pragma unroll
    for (int u = 0; u < 4; u++) gs_c(x[u], x[u + 4], t.a);
}
__device__ __forceinline__ void bar_pair(int id) { asm volatile("bar.sync %0, 64;" ::"r"(id) : "memory"); }
__device__ __forceinline__ dcplx ldc(const double2* p) {
    const double2 v = *p;
    return dcplx{v.x, v.y};
}
__device__ __forceinline__ void stc(double2* p, dcplx v) { *p = make_double2(v.re, v.im); }

// forward transform by a warp pair.  In: x[v] = z[gp1(tt, v)].  Out: Z[k] at buf[lsw(k)] (written by this pair;
// each thread writes back exactly the positions it read, so one barrier per exchange suffices).
__device__ __forceinline__ void fwd2w(dcplx (&x)[8], double2* buf, const PassTw& t1, const PassTw& t2,
                                      const PassTw& t3, int tt, int id) {
    pass_fwd(x, t1);
#pragma unroll
    for (int v = 0; v < 8; v++) stc(buf + lsw(gp1(tt, v)), x[v]);
    bar_pair(id);
#pragma unroll
    for (int v = 0; v < 8; v++) x[v] = ldc(buf + lsw(gp2(tt, v)));
    pass_fwd(x, t2);
#pragma unroll
    for (int v = 0; v < 8; v++) stc(buf + lsw(gp2(tt, v)), x[v]);
    bar_pair(id);
#pragma unroll
    for (int v = 0; v < 8; v++) x[v] = ldc(buf + lsw(gp3(tt, v)));
    pass_fwd(x, t3);
#pragma unroll
    for (int v = 0; v < 8; v++) stc(buf + lsw(gp3(tt, v)), x[v]);
}
// inverse by a warp pair.  In: Z[k] at buf[lsw(k)] (complete).  Out: x[v] = 512 z[gp1(tt, v)].
__device__ __forceinline__ void inv2w(dcplx (&x)[8], double2* buf, const PassTw& t1, const PassTw& t2,
                                      const PassTw& t3, int tt, int id) {
#pragma unroll
    for (int v = 0; v < 8; v++) x[v] = ldc(buf + lsw(gp3(tt, v)));
    pass_inv(x, t3);
#pragma unroll
    for (int v = 0; v < 8; v++) stc(buf + lsw(gp3(tt, v)), x[v]);
    bar_pair(id);
#pragma unroll
    for (int v = 0; v < 8; v++) x[v] = ldc(buf + lsw(gp2(tt, v)));
    pass_inv(x, t2);
#pragma unroll
    for (int v = 0; v < 8; v++) stc(buf + lsw(gp2(tt, v)), x[v]);
    bar_pair(id);
#pragma unroll
    for (int v = 0; v < 8; v++) x[v] = ldc(buf + lsw(gp1(tt, v)));
    pass_inv(x, t1);
}

__device__ __forceinline__ uint32_t sm32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t cl_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cl_map(uint32_t a, uint32_t rank) {
    uint32_t out;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(out) : "r"(a), "r"(rank));
    return out;
}
__device__ __forceinline__ void cl_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void mb_init(unsigned long long* b) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sm32(b)) : "memory");
}
__device__ __forceinline__ void mb_expect(unsigned long long* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sm32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mb_wait(unsigned long long* b, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred p;\n WL_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra WL_%=;\n}\n" ::"r"(sm32(b)),
        "r"(parity)
        : "memory");
}
// local shared -> peer shared bulk copy completing on the peer's mbarrier
__device__ __forceinline__ void push_peer(uint32_t dst, const void* src, uint32_t bytes, uint32_t mbar) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
        "r"(sm32(src)), "r"(bytes), "r"(mbar)
        : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
// BK_i -> bk[buf] (one thread): the own bloc's rows 3q..3q+2 of output o (slots 0-2) and, for positions
// [256 h, 256 h + 256), of the other bloc's two outputs 2(1-q) + 0 and + 1 (slots 3-5, one half each).
__device__ __forceinline__ void issue_bk_l(BrlSmem& S, const double2* bkf, int i, int o, int q, int h,
                                           int buf) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mb_expect(&S.mbar_bk[buf], kRows * 512 * 16);
#pragma unroll
    for (int r = 0; r < kRows; r++) {
        if (r >= kL) {
            // slot r: the partner bloc's outputs 2(1-q) + 0 and + 1, positions [256 h, 256 h + 256) of each
#pragma unroll
            for (int hh = 0; hh < 2; hh++)
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                        sm32(&S.bk[buf][r][256 * hh])),
                    "l"(bkf + ((size_t)(i * kRows + kL * q + r % kL) * 4 + 2 * (1 - q) + hh) * 512 + 256 * h),
                    "r"(256 * 16), "r"(sm32(&S.mbar_bk[buf]))
                    : "memory");
            continue;
        }
        const size_t row = (size_t)(i * kRows + kL * q + r) * 4 + o;
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                sm32(S.bk[buf][r])),
            "l"(bkf + row * 512), "r"(512 * 16), "r"(sm32(&S.mbar_bk[buf]))
            : "memory");
    }
}

// twL: [64][6] per-thread pass bases: (pass 2: zeta_{4,t>>3}, zeta_{5,2(t>>3)}, zeta_{6,4(t>>3)},
//       pass 3: zeta_{7,t}, zeta_{8,2t}, zeta_{9,4t}); pass 1 bases come from the constant bank
__global__ void __cluster_dims__(4, 1, 1) __launch_bounds__(kLThreads, 1)
    brl_kernel(BrArgs A, const double2* __restrict__ bkf, const double2* __restrict__ twL) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    BrlSmem& S = *reinterpret_cast<BrlSmem*>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t rank = cl_rank();
    const int q = (int)(rank >> 1), h = (int)(rank & 1), o = 2 * q + h;
    const int gl = blockIdx.x >> 2;                      // one lane (bootstrap) per cluster

    if (tid == 0) {
        for (int b = 0; b < 2; b++) {
            mb_init(&S.mbar_bk[b]);
            mb_init(&S.mbar_part[b]);
            mb_init(&S.mbar_res[b]);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int b = 0; b < 2; b++) {                    // partials and halves of steps 0 and 1 may arrive any time
            mb_expect(&S.mbar_part[b], kPartBytes);
            mb_expect(&S.mbar_res[b], kN * 4);
        }
    }
    __syncthreads();
    if (tid == 0) {
        issue_bk_l(S, bkf, 0, o, q, h, 0);
        issue_bk_l(S, bkf, 1, o, q, h, 1);
    }
    {   // a1, a2 (every CTA of the cluster)
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
    const int jd = warp >> 1;                             // forward role: digit jd of bloc q (warps 0-5)
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
    const uint32_t part_dst = cl_map(sm32(&S.precv[0][0]), rank ^ 2u);
    const uint32_t part_mb = cl_map(sm32(&S.mbar_part[0]), rank ^ 2u);
    const uint32_t part_dst_x = cl_map(sm32(&S.precv[0][0]), rank ^ 3u);   // CTA (1-q, 1-h)
    const uint32_t part_mb_x = cl_map(sm32(&S.mbar_part[0]), rank ^ 3u);
    const uint32_t res_dst = cl_map(sm32(&S.rres[0][0]), rank ^ 1u);
    const uint32_t res_mb = cl_map(sm32(&S.mbar_res[0]), rank ^ 1u);

    for (int i = 0; i < kn; i++) {
        const int buf = i & 1;
        const uint32_t par = (uint32_t)((i >> 1) & 1);
        BRL_T(0)
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
        BRL_T(1)
        mb_wait(&S.mbar_bk[buf], par);
        BRL_T(2)
        // ---- B: the MAC split by bloc (it is linear): this CTA multiplies its own rows (bloc q) by BK_i for its
        // output o on all positions and for the other bloc's two outputs on positions [256 h, 256 h + 256), sends
        // those two partials (4 KB each) to their owners, and adds the other bloc's partial of o, received half
        // from each CTA of bloc 1-q.  Round-off: the FP64 error bound of 5b holds for any summation order. ----
        // the partners' partials first: positions [256 h, 256 h + 256) of both outputs of bloc 1-q, one to each of
        // CTA (1-q, h) and (1-q, 1-h); each receives its 8 KB half from two senders at once
        dcplx dr[kLMacIt][kL];
#pragma unroll
        for (int e = 0; e < kLMacIt; e++) {
            const int k = tid + kLThreads * e;
#pragma unroll
            for (int r = 0; r < kL; r++) dr[e][r] = ldc(&S.dslot[r][lsw(k)]);
        }
        {
            const int k = tid + kLThreads * h;
            const dcplx d0 = h ? dr[1][0] : dr[0][0], d1 = h ? dr[1][1] : dr[0][1], d2 = h ? dr[1][2] : dr[0][2];
#pragma unroll
            for (int hh = 0; hh < 2; hh++) {
                dcplx s2 = {0.0, 0.0};
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const dcplx d = r == 0 ? d0 : (r == 1 ? d1 : d2), b2 = ldc(&S.bk[buf][kL + r][256 * hh + tid]);
                    s2.re = fma(d.re, b2.re, fma(-d.im, b2.im, s2.re));
                    s2.im = fma(d.re, b2.im, fma(d.im, b2.re, s2.im));
                }
                const bool same = hh == h;
                asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.f64 [%0], {%1, %2}, [%3];" ::"r"(
                                 (same ? part_dst : part_dst_x) + (uint32_t)((buf * 512 + k) * 16)),
                             "d"(s2.re), "d"(s2.im), "r"((same ? part_mb : part_mb_x) + (uint32_t)(buf * 8))
                             : "memory");
            }
        }
        dcplx m3[kLMacIt];
#pragma unroll
        for (int e = 0; e < kLMacIt; e++) {
            const int k = tid + kLThreads * e;
            dcplx s = {0.0, 0.0};
            if (k < 512) {
#pragma unroll
                for (int r = 0; r < kL; r++) {
                    const dcplx d = dr[e][r], b = ldc(&S.bk[buf][r][k]);
                    s.re = fma(d.re, b.re, fma(-d.im, b.im, s.re));
                    s.im = fma(d.re, b.im, fma(d.im, b.re, s.im));
                }
            }
            m3[e] = s;
        }
        mb_wait(&S.mbar_part[buf], par);
        BRL_T(3)
#pragma unroll
        for (int e = 0; e < kLMacIt; e++) {
            const int k = tid + kLThreads * e;
            if (k < 512) {
                const dcplx pr = ldc(&S.precv[buf][k]);
                stc(&S.oslot[lsw(k)], dcplx{m3[e].re + pr.re, m3[e].im + pr.im});
            }
        }
        __syncthreads();                                  // bk[buf], precv[buf] consumed; oslot complete
        BRL_T(4)
        // step i + 2's BK and the expectation of its rows: issued by a thread of warp 2, idle during the inverse
        // (from warp 0, the fence.proxy.async + six bulk copies delayed the inverse's warp pair and the half
        // swap behind it: one-gate level 1.92 -> 1.83 ms)
        if (tid == kBkIssuer) {
            if (i + 2 < kn) {
                mb_expect(&S.mbar_part[buf], kPartBytes);                     // partials of step i + 2
                issue_bk_l(S, bkf, i + 2, o, q, h, buf);
            }
        }
        if (warp < 2) {   // ---- C: inverse (warp pair 0), round, << 16 h ----
            dcplx x[8];
            inv2w(x, S.oslot, t1, t2, t3, tt, 4);
#pragma unroll
            for (int v = 0; v < 8; v++) {
                const int c = gp1(tt, v);
                const uint32_t lo = round_mod32(x[v].re) << (16 * h), hi = round_mod32(x[v].im) << (16 * h);
                S.res[c] = lo;
                S.res[c + 512] = hi;
                // and straight into the sibling's rres[buf] (4 KB per step, completing on its mbarrier)
                asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(
                                 res_dst + (uint32_t)((buf * kN + c) * 4)),
                             "r"(lo), "r"(res_mb + (uint32_t)(buf * 8))
                             : "memory");
                asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(
                                 res_dst + (uint32_t)((buf * kN + c + 512) * 4)),
                             "r"(hi), "r"(res_mb + (uint32_t)(buf * 8))
                             : "memory");
            }
        }
        __syncthreads();
        BRL_T(5)
        mb_wait(&S.mbar_res[buf], par);
        BRL_T(6)
        for (int c = tid; c < kN; c += kLThreads) {       // ACC[q] += lo + 2^16 hi (own half + the sibling's)
            const uint32_t nv = S.acc[c] + S.res[c] + S.rres[buf][c];
            S.acc[c] = nv;
            S.acc[c + kN] = 0u - nv;
            S.acc[c + 2 * kN] = nv;
        }
        __syncthreads();                                  // rres[buf] consumed
        BRL_T(7)
        if (tid == 0) {   // (no barrier after this: warps 0-1 rewrite res only after the next phase-A barrier,
                          // which tid 0 reaches after the wait; the expect precedes tid 0's own next push)
            if (i + 2 < kn) mb_expect(&S.mbar_res[buf], kN * 4);            // the sibling's half of step i + 2
        }
    }
    cl_sync();
    if (gl < A.nlanes && h == 0) {   // a5: CTA (0, 0) holds ACC.a, CTA (1, 0) holds ACC.b
        uint32_t* out = A.out + (int64_t)gl * A.out_stride;
        if (q == 0) {
            for (int j = tid; j < kN; j += kLThreads) out[j] = j == 0 ? S.acc[0] : 0u - S.acc[kN - j];
        } else if (tid == 0) {
            out[kN] = S.acc[0];
        }
    }
}

static int brl_attr() {
    if (ensure_smem_attr<brl_kernel>(sizeof(BrlSmem))) return -1;
    return 0;
}

// clusters of brl that are co-resident on the device (one wave of bootstraps; 32 measured on B200: the 4-SM
// clusters must fit inside a GPC), or <= 0 on error
int brl_wave_lanes() {
    if (brl_attr()) return -1;
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 4;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3(4 * 256);
    cfg.blockDim = dim3(kLThreads);
    cfg.dynamicSmemBytes = sizeof(BrlSmem);
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, brl_kernel, &cfg) != cudaSuccess) return -1;
    return n;
}

#ifdef TB_BRL_TRACE
extern "C" int tb_debug_brl_trace(long long* host) {
    return cudaMemcpyFromSymbol(host, g_brl_trace, sizeof(g_brl_trace)) == cudaSuccess ? 0 : -1;
}
#endif

int launch_brl(const BrArgs& A, const double2* bkf, const double2* twL, cudaStream_t st) {
    const size_t smem = sizeof(BrlSmem);
    static_assert(sizeof(BrlSmem) <= 232448, "brl shared memory");
    if (brl_attr()) return -1;
    if (A.nlanes <= 0) return 0;
    brl_kernel<<<4 * A.nlanes, kLThreads, smem, st>>>(A, bkf, twL);
    return 0;
}

}  // namespace tb
