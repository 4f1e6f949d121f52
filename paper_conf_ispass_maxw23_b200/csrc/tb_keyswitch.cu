// tb_keyswitch.cu -- batched LWE key switching N -> n ("key switching", the second slice
// of a gate's profile, Fig. 7, named as vectorisable at P:247), plus the MUX lane combine and
// NOT (negation, no bootstrap) of a level.
//
// out = (0, b) - sum_{i < N, j < t, d_ij != 0} KSK[i][j][d_ij], d_ij = base-4 digits of a_i + 2^15 (C9).
// A CTA owns a tile of T gates; its threads own 4 consecutive output words each (16-B vector loads of the
// 632-word device KSK rows).  For every (i, j) the digits of the T gates select rows of the 3-row group
// KSK[i][j][1..3]; the group is read from L2 once per tile and re-read from L1 by the other gates, so HBM/L2
// traffic per gate is (62 MB KSK) / T instead of 15.5 MB of data-dependent row gathers.
#include "tb_kernels.cuh"

namespace tb {

constexpr int kKsThreads = 160;                  // 158 threads x 4 words = 632 words

// words k0..k0+3 (<= n) of an output row: one 16-byte store when aligned (whole-line NVLink writes for the
// peer copies), else scalar
__device__ __forceinline__ void store_row4(uint32_t* d, const uint32_t (&v)[4], int k0) {
    if (k0 + 3 <= kn && (reinterpret_cast<uintptr_t>(d) & 15) == 0) {
        *reinterpret_cast<uint4*>(d) = make_uint4(v[0], v[1], v[2], v[3]);
    } else {
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (k0 + q <= kn) d[q] = v[q];
    }
}

// partial != nullptr: CTA (tile, s) covers input coefficients i in slice s of S (blockIdx.y) and writes its
// partial sums to partial[gate][s][kKsRow] for ks_reduce_kernel (mid-size levels: more CTAs than tiles)
template <int T>
__global__ void __launch_bounds__(kKsThreads) ks_kernel(KsArgs A, uint32_t* __restrict__ partial, int S) {
    extern __shared__ __align__(128) unsigned char ks_smem[];
    const int s = blockIdx.y, I = kN / S, i0 = s * I;
    uint16_t (*sW)[T] = reinterpret_cast<uint16_t (*)[T]>(ks_smem);   // [kN][T]: (a_i + 2^15) >> 16 = 8 digits
    uint32_t* sB = reinterpret_cast<uint32_t*>(ks_smem + (size_t)kN * T * 2);
    const int tid = threadIdx.x;
    const int g0 = blockIdx.x * T;

    // prologue: combine lanes (MUX: u1 + u2 + (0, mu)), take digit words
    for (int g = 0; g < T; g++) {
        const int gi = g0 + g;
        GateDesc gd = {0, 0, -1, kGateNot};
        bool valid = gi < A.ngates;
        if (valid) gd = A.gates[gi];
        const bool boot = valid && gd.kind != kGateNot;
        const uint32_t* l0 = A.lanes + (int64_t)(gd.lane0 - A.lane_base) * A.lane_stride;
        const uint32_t* l1 = gd.lane1 >= 0 ? A.lanes + (int64_t)(gd.lane1 - A.lane_base) * A.lane_stride : nullptr;
        for (int i = tid; i <= kN; i += kKsThreads) {
            uint32_t e = 0u;
            if (boot) {
                e = __ldg(l0 + i);
                if (l1) e += __ldg(l1 + i);
            }
            if (i < kN) sW[i][g] = boot ? (uint16_t)((e + (1u << 15)) >> 16) : (uint16_t)0;
            else sB[g] = l1 ? e + kMu : e;
        }
    }
    __syncthreads();

    const int k0 = 4 * tid;                         // output words k0..k0+3
    const bool active = tid < kKsRow / 4;
    uint32_t acc[T][4];
#pragma unroll
    for (int g = 0; g < T; g++) {
        const int gi = g0 + g;
        const bool isnot = gi < A.ngates && A.gates[gi].kind == kGateNot;
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const int k = k0 + q;
            uint32_t v = (k == kn) ? sB[g] : 0u;
            if (isnot && active && k <= kn) v = 0u - __ldg(A.not_src + (int64_t)A.gates[gi].lane0 * A.not_stride + k);
            acc[g][q] = s == 0 ? v : 0u;
        }
    }
    if (active) {
        for (int i = i0; i < i0 + I; i++) {
            uint16_t w[T];
#pragma unroll
            for (int g = 0; g < T; g += 8) {
                const uint4 v = *reinterpret_cast<const uint4*>(&sW[i][g]);
                w[g + 0] = (uint16_t)(v.x & 0xFFFF); w[g + 1] = (uint16_t)(v.x >> 16);
                w[g + 2] = (uint16_t)(v.y & 0xFFFF); w[g + 3] = (uint16_t)(v.y >> 16);
                w[g + 4] = (uint16_t)(v.z & 0xFFFF); w[g + 5] = (uint16_t)(v.z >> 16);
                w[g + 6] = (uint16_t)(v.w & 0xFFFF); w[g + 7] = (uint16_t)(v.w >> 16);
            }
            const uint32_t* rowi = A.ksk + (size_t)i * kKsT * (kKsBase - 1) * kKsRow + k0;
#pragma unroll
            for (int j = 0; j < kKsT; j++) {
#pragma unroll
                for (int g = 0; g < T; g++) {
                    const uint32_t d = (w[g] >> (14 - 2 * j)) & 3u;
                    if (d) {
                        const uint4 v = __ldg(reinterpret_cast<const uint4*>(rowi + (j * (kKsBase - 1) + d - 1) * kKsRow));
                        acc[g][0] -= v.x; acc[g][1] -= v.y; acc[g][2] -= v.z; acc[g][3] -= v.w;
                    }
                }
            }
        }
#pragma unroll
        for (int g = 0; g < T; g++) {
            const int gi = g0 + g;
            if (gi < A.ngates && partial) {
                *reinterpret_cast<uint4*>(partial + ((size_t)gi * S + s) * kKsRow + k0) =
                    make_uint4(acc[g][0], acc[g][1], acc[g][2], acc[g][3]);
            } else if (gi < A.ngates) {
                const int64_t off = (int64_t)A.gates[gi].out_row * A.out_stride;
                store_row4(A.out + off + k0, acc[g], k0);
                for (int p = 0; p < A.npeers; p++)     // fused all-gather: the same row into every peer's array
                    store_row4(A.peers[p] + off + k0, acc[g], k0);
            }
        }
        if (A.npeers) __threadfence_system();
    }
}

// ---- narrow levels: one gate's key switch split over S CTAs ---------------------------------------
// A level with few gates leaves the tiled kernel with a handful of CTAs that each walk all 8,192 (i, j) digit
// groups one after another.  Here CTA (g, s) owns input coefficients i in slice s of [0, N) for gate g and writes
// its partial sum (words mod 2^32) to scratch; ks_reduce_kernel adds the S partials (integer sums mod 2^32 are
// order-independent, so the result is bit-identical to the tiled kernel).
constexpr int kKsSplitMin = 16;                  // slices per gate: 16, or 32 / 64 for levels of <= 9 / 4 gates
__host__ __device__ constexpr int ks_split_count(int64_t ngates) { return ngates <= 4 ? 64 : ngates <= 9 ? 32 : 16; }

__global__ void __launch_bounds__(kKsThreads) ks_split_kernel(KsArgs A, uint32_t* __restrict__ partial, int S) {
    const int I = kN / S;
    __shared__ uint16_t sW[kN / kKsSplitMin];
    __shared__ uint32_t sB;
    const int tid = threadIdx.x, gi = blockIdx.x, s = blockIdx.y;
    const GateDesc gd = A.gates[gi];
    const bool boot = gd.kind != kGateNot;
    const uint32_t* l0 = A.lanes + (int64_t)(gd.lane0 - A.lane_base) * A.lane_stride;
    const uint32_t* l1 = gd.lane1 >= 0 ? A.lanes + (int64_t)(gd.lane1 - A.lane_base) * A.lane_stride : nullptr;
    for (int ii = tid; ii < I; ii += kKsThreads) {
        uint32_t e = 0u;
        if (boot) {
            e = __ldg(l0 + s * I + ii);
            if (l1) e += __ldg(l1 + s * I + ii);
        }
        sW[ii] = boot ? (uint16_t)((e + (1u << 15)) >> 16) : (uint16_t)0;
    }
    if (tid == 0) {
        uint32_t b = 0u;
        if (boot) {
            b = __ldg(l0 + kN);
            if (l1) b += __ldg(l1 + kN) + kMu;
        }
        sB = b;
    }
    __syncthreads();
    const int k0 = 4 * tid;
    if (k0 >= kKsRow) return;
    uint32_t acc[4];
#pragma unroll
    for (int q = 0; q < 4; q++) {
        const int k = k0 + q;
        uint32_t v = 0u;
        if (s == 0) {
            if (!boot && k <= kn) v = 0u - __ldg(A.not_src + (int64_t)gd.lane0 * A.not_stride + k);
            else if (k == kn) v = sB;
        }
        acc[q] = v;
    }
    for (int ii = 0; ii < I; ii++) {
        const uint32_t w = sW[ii];
        const uint32_t* rowi = A.ksk + (size_t)(s * I + ii) * kKsT * (kKsBase - 1) * kKsRow + k0;
#pragma unroll
        for (int j = 0; j < kKsT; j++) {
            const uint32_t d = (w >> (14 - 2 * j)) & 3u;
            if (d) {
                const uint4 v = __ldg(reinterpret_cast<const uint4*>(rowi + (j * (kKsBase - 1) + d - 1) * kKsRow));
                acc[0] -= v.x; acc[1] -= v.y; acc[2] -= v.z; acc[3] -= v.w;
            }
        }
    }
    *reinterpret_cast<uint4*>(partial + ((size_t)gi * S + s) * kKsRow + k0) = make_uint4(acc[0], acc[1], acc[2], acc[3]);
}

__global__ void __launch_bounds__(kKsThreads) ks_reduce_kernel(KsArgs A, const uint32_t* __restrict__ partial, int S) {
    const int gi = blockIdx.x;
    const int64_t off = (int64_t)A.gates[gi].out_row * A.out_stride;
    uint32_t* o = A.out + off;
    for (int k = threadIdx.x; k <= kn; k += kKsThreads) {
        uint32_t v = 0u;
#pragma unroll
        for (int s = 0; s < S; s++) v += partial[((size_t)gi * S + s) * kKsRow + k];
        o[k] = v;
        for (int p = 0; p < A.npeers; p++) A.peers[p][off + k] = v;   // fused all-gather
    }
    if (A.npeers) __threadfence_system();
}

int launch_ks_split(const KsArgs& A, uint32_t* partial, cudaStream_t st) {
    if (A.ngates <= 0) return 0;
    const int S = ks_split_count(A.ngates);
    ks_split_kernel<<<dim3(A.ngates, S), kKsThreads, 0, st>>>(A, partial, S);
    ks_reduce_kernel<<<A.ngates, kKsThreads, 0, st>>>(A, partial, S);
    return 0;
}
size_t ks_split_scratch_words(int64_t ngates) { return (size_t)ngates * ks_split_count(ngates) * kKsRow; }

// digit-0 rows dropped, rows padded to 632 words: [i][j][d][631] (host layout) -> [i][j][d-1][632]
__global__ void ksk_relayout_kernel(const uint32_t* __restrict__ src, uint32_t* __restrict__ dst) {
    const size_t row = blockIdx.x;                   // (i, j, d-1)
    const size_t dm1 = row % (kKsBase - 1), ij = row / (kKsBase - 1);
    const uint32_t* s = src + (ij * kKsBase + dm1 + 1) * (kn + 1);
    uint32_t* d = dst + row * kKsRow;
    for (int k = threadIdx.x; k < kKsRow; k += blockDim.x) d[k] = k <= kn ? s[k] : 0u;
}

template <int T>
static int launch_ks_t(const KsArgs& A, uint32_t* partial, int S, cudaStream_t st) {
    const size_t smem = (size_t)kN * T * 2 + T * 4;
    if (ensure_smem_attr<ks_kernel<T>>(smem)) return -1;
    const int blocks = (A.ngates + T - 1) / T;
    ks_kernel<T><<<dim3(blocks, S), kKsThreads, smem, st>>>(A, S > 1 ? partial : nullptr, S);
    if (S > 1) ks_reduce_kernel<<<A.ngates, kKsThreads, 0, st>>>(A, partial, S);
    return 0;
}

// slices per tile so that a mid-size level still fills the GPU: ~4 CTAs per SM (592 on B200) at least
int ks_tile_slices(int64_t ngates, int tile) {
    const int64_t tiles = (ngates + tile - 1) / tile;
    int S = 1;
    while (S < 16 && tiles * S < 592) S *= 2;
    return S;
}

int launch_ks(const KsArgs& A, int tile, uint32_t* partial, int S, cudaStream_t st) {
    if (A.ngates <= 0) return 0;
    switch (tile) {
        case 8: return launch_ks_t<8>(A, partial, S, st);
        case 16: return launch_ks_t<16>(A, partial, S, st);
        case 32: return launch_ks_t<32>(A, partial, S, st);
        default: return -2;
    }
}

void launch_ksk_relayout(const uint32_t* src, uint32_t* dst, cudaStream_t st) {
    ksk_relayout_kernel<<<kN * kKsT * (kKsBase - 1), 128, 0, st>>>(src, dst);
}

}  // namespace tb
