// tb_br8.cu -- blind rotation with two ping-ponged lane groups per CTA.
//
// Same arithmetic and per-lane work split as br6_kernel (bit-identical output).  One CTA (24 warps, 1 per SM)
// holds two groups of two lanes.  Each group synchronises only with itself (named barriers), and the two groups
// take turns on the MAC phase B, whose latency is dominated by L2 reads of BK_i: group X may enter B only after
// group Y has left B and vice versa, so one group's MAC overlaps the other group's NTT phases (A, C), which are
// bound by the integer-multiply pipe.  (The schedule is the "ping-pong" of two consumer warpgroups.)
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {

constexpr int kB8Lanes = 4;                 // lanes per CTA (2 groups x 2)
constexpr int kB8Threads = 6 * 32 * kB8Lanes;
constexpr int kB8Group = kB8Threads / 2;    // 384 threads per group

struct Br8Smem {
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t acc[kB8Lanes][2][kN];
    uint32_t slot[kB8Lanes][kOuts][kSlotWords];
    uint16_t bar[kB8Lanes][kn + 2];
};

__device__ __forceinline__ void nb_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void nb_arrive(int id, int n) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}

// barrier ids: 1, 2 = group-local; 3, 4 = "group x may enter B"; 5..12 = part combine of (lane, q)
__global__ void __launch_bounds__(kB8Threads, 1) br8_kernel(BrArgs A) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Br8Smem& S = *reinterpret_cast<Br8Smem*>(smem_raw);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = warp / 6, w6 = warp % 6;
    const int grp = g >> 1;                          // lanes {0,1} -> group 0, {2,3} -> group 1
    const int gtid = tid - grp * kB8Group;           // thread index inside the group
    const int lane0 = blockIdx.x * kB8Lanes;
    const int bar_grp = 1 + grp, bar_mine = 3 + grp, bar_other = 3 + (grp ^ 1);

    for (int k = tid; k < 31 * 32; k += kB8Threads) {
        S.twF[k] = A.twF[k];
        S.twI[k] = A.twI[k];
    }
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
            S.bar[g][w] = (uint16_t)((v + (1u << 20)) >> 21);      // a1, a2 (C5)
        }
    }
    __syncthreads();
    for (int k = tid; k < kB8Lanes * kN; k += kB8Threads) {       // a3 (C6)
        const int gg = k / kN, c = k % kN;
        const uint32_t bbar = S.bar[gg][kn];
        S.acc[gg][0][c] = 0u;
        S.acc[gg][1][c] = ((c + bbar) & (kTwoN - 1)) < (uint32_t)kN ? kMu : (uint32_t)(0u - kMu);
    }
    __syncthreads();
    if (grp == 1) nb_arrive(3, kB8Threads);          // group 0 may take the first MAC turn

    const uint32_t R = c_misc[0], Rp = c_misc[1];
    const int bloc = w6 / kL, jd = w6 % kL;
    const int q = w6 / kParts, m = w6 % kParts;
    const int shift = 32 - kBgbit * (jd + 1);
    for (int i = 0; i < kn; i++) {
        {   // phase A
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
            ntt_fwd(x, slot, S.twF, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) slot[kPadRow * lane + j] = red_2p(x[j]);
        }
        nb_sync(bar_grp, kB8Group);
        nb_sync(bar_mine, kB8Threads);               // our MAC turn (the other group has left B)
        {   // phase B: this group's two lanes
            const uint32_t* bki = A.bkhat + (size_t)i * (kRows * kOuts * kN);
            const int g0 = grp * 2;
            for (int a = gtid; a < kN; a += kB8Group) {
                const int pa = a + (a >> 5);
                uint32_t B[kRows][kOuts];
#pragma unroll
                for (int r = 0; r < kRows; r++)
#pragma unroll
                    for (int o = 0; o < kOuts; o++) B[r][o] = __ldg(bki + (r * kOuts + o) * kN + a);
#pragma unroll
                for (int gg = g0; gg < g0 + 2; gg++) {
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
        nb_arrive(bar_other, kB8Threads);            // hand the MAC turn to the other group
        nb_sync(bar_grp, kB8Group);
        {   // phase C
            uint32_t* slot = S.slot[g][w6];
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
            nb_sync(5 + g * 2 + q, 96);
            if (m == 0) {
                const uint32_t* p1 = S.slot[g][q * kParts + 1];
                const uint32_t* p2 = S.slot[g][q * kParts + 2];
                uint32_t* acc = S.acc[g][q];
#pragma unroll
                for (int j = 0; j < 32; j++)
                    acc[lane + 32 * j] += x[j] + p1[kPadRow * j + lane] + p2[kPadRow * j + lane];
            }
        }
        nb_sync(bar_grp, kB8Group);
    }
    if (grp == 0) nb_sync(3, kB8Threads);            // consume group 1's last hand-over
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

int launch_br8(const BrArgs& A, cudaStream_t st) {
    const size_t smem = sizeof(Br8Smem);
    static bool attr = false;
    if (!attr) {
        if (cudaFuncSetAttribute(br8_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
            return -1;
        attr = true;
    }
    const int blocks = (A.nlanes + kB8Lanes - 1) / kB8Lanes;
    if (blocks == 0) return 0;
    br8_kernel<<<blocks, kB8Threads, smem, st>>>(A);
    return 0;
}

}  // namespace tb
