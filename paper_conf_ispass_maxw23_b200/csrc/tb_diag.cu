// tb_diag.cu -- constant upload, the NTT-product diagnostic used by the unit parity test, and the
// integer-pipe microbenchmark that gives the "alu" roofline denominator.
#include "tb_kernels.cuh"
#include "tb_ntt.cuh"

namespace tb {

int set_ntt_constants(const uint32_t* fw, const uint32_t* fwp, const uint32_t* iw, const uint32_t* iwp,
                      const uint32_t* misc) {
    if (cudaMemcpyToSymbol(c_fw, fw, 32 * 4) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(c_fwp, fwp, 32 * 4) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(c_iw, iw, 32 * 4) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(c_iwp, iwp, 32 * 4) != cudaSuccess) return -1;
    if (cudaMemcpyToSymbol(c_misc, misc, 4 * 4) != cudaSuccess) return -1;
    return 0;
}

// res = sum_{r<6} digits[r] (x) polys[r] mod 2^32 through the same field, split, transforms, MAC reduction
// and lift that the blind-rotation kernel uses (one CTA, 6 warps).
struct DiagSmem {
    uint2 twF[31 * 32];
    uint2 twI[31 * 32];
    uint32_t d[kRows][kSlotWords];
    uint32_t b[kRows][kParts][kSlotWords];
    uint32_t o[kParts][kSlotWords];
};

__global__ void __launch_bounds__(192) ntt_muladd6_kernel(const int32_t* digits, const uint32_t* polys,
                                                          uint32_t* res, const uint2* twF, const uint2* twI,
                                                          uint32_t ninv, uint32_t ninvp) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    DiagSmem& S = *reinterpret_cast<DiagSmem*>(smem_raw);
    const int lane = threadIdx.x & 31, r = threadIdx.x >> 5;
    for (int k = threadIdx.x; k < 31 * 32; k += blockDim.x) {
        S.twF[k] = twF[k];
        S.twI[k] = twI[k];
    }
    __syncthreads();
    uint32_t x[32];
#pragma unroll
    for (int j = 0; j < 32; j++) {
        const int32_t dv = digits[r * kN + lane + 32 * j];
        x[j] = dv < 0 ? (uint32_t)(dv + (int32_t)kP) : (uint32_t)dv;
    }
    ntt_fwd(x, S.d[r], S.twF, lane);
#pragma unroll
    for (int j = 0; j < 32; j++) S.d[r][kPadRow * lane + j] = red_2p(x[j]);
    for (int m = 0; m < kParts; m++) {
#pragma unroll
        for (int j = 0; j < 32; j++) {
            uint32_t v = polys[r * kN + lane + 32 * j];
            const int32_t p0 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
            v = (v - (uint32_t)p0) >> 11;
            const int32_t p1 = ((int32_t)((v & 0x7FFu) << 21)) >> 21;
            v = (v - (uint32_t)p1) >> 11;
            const int32_t p2 = ((int32_t)((v & 0x3FFu) << 22)) >> 22;
            const int32_t pm = m == 0 ? p0 : (m == 1 ? p1 : p2);
            x[j] = pm < 0 ? (uint32_t)(pm + (int32_t)kP) : (uint32_t)pm;
        }
        ntt_fwd(x, S.b[r][m], S.twF, lane);
#pragma unroll
        for (int j = 0; j < 32; j++) S.b[r][m][kPadRow * lane + j] = red_p(shoup_mul(x[j], ninv, ninvp));
    }
    __syncthreads();
    const uint32_t R = c_misc[0], Rp = c_misc[1];
    for (int a = threadIdx.x; a < kN; a += blockDim.x) {
        const int pa = a + (a >> 5);
        for (int m = 0; m < kParts; m++) {
            uint64_t acc = 0;
            for (int rr = 0; rr < kRows; rr++) acc += (uint64_t)S.d[rr][pa] * S.b[rr][m][pa];
            const uint32_t hi = (uint32_t)(acc >> 32), lo = (uint32_t)acc;
            S.o[m][pa] = red_2p(shoup_mul(hi, R, Rp) + (lo - (lo >> 30) * kP));
        }
    }
    __syncthreads();
    if (r == 0) {
        uint32_t sum[32];
#pragma unroll
        for (int j = 0; j < 32; j++) sum[j] = 0u;
        for (int m = 0; m < kParts; m++) {
#pragma unroll
            for (int j = 0; j < 32; j++) x[j] = S.o[m][kPadRow * lane + j];
            ntt_inv(x, S.o[m], S.twI, lane);
#pragma unroll
            for (int j = 0; j < 32; j++) sum[j] += lift_centred(x[j]) << (11 * m);
        }
#pragma unroll
        for (int j = 0; j < 32; j++) res[lane + 32 * j] = sum[j];
    }
}

int launch_ntt_muladd6(const int32_t* digits, const uint32_t* polys, uint32_t* res, const uint2* twF,
                       const uint2* twI, uint32_t ninv, uint32_t ninvp, cudaStream_t st) {
    const size_t smem = sizeof(DiagSmem);
    if (cudaFuncSetAttribute(ntt_muladd6_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess)
        return -1;
    ntt_muladd6_kernel<<<1, 192, smem, st>>>(digits, polys, res, twF, twI, ninv, ninvp);
    return 0;
}

// ---- microbenchmark: the kernels' own lazy CT butterfly and 64-bit MAC, register resident ----------
template <int NV>
__global__ void __launch_bounds__(256) mb_bfly_kernel(uint32_t* sink, int iters, uint32_t w, uint32_t wp) {
    uint32_t x[NV], y[NV];
#pragma unroll
    for (int i = 0; i < NV; i++) {
        x[i] = threadIdx.x * 7u + i;
        y[i] = threadIdx.x * 13u + 3u * i;
    }
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < NV; i++) ct_bfly(x[i], y[i], w, wp);
        w ^= (uint32_t)it & 1u;          // keep the twiddle loop-variant (uniform, cheap)
    }
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < NV; i++) s += x[i] ^ y[i];
    if (s == 0x12345678u) sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int NV>
__global__ void __launch_bounds__(256) mb_mac_kernel(uint64_t* sink, int iters, uint32_t b0) {
    uint64_t acc[NV];
    uint32_t d[NV];
#pragma unroll
    for (int i = 0; i < NV; i++) {
        acc[i] = 0;
        d[i] = threadIdx.x * 7u + i;
    }
    uint32_t b = b0 + threadIdx.x;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < NV; i++) acc[i] += (uint64_t)d[i] * b;
        b += 3u;
    }
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < NV; i++) s += acc[i];
    if (s == 0x123456789ull) sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// ---- Goldilocks field p = 2^64 - 2^32 + 1 (the north star's proposed NTT field; R1) -----------
// Register-resident butterflies over the 64-bit field, so that the field choice (30-bit Shoup field with the BK
// split in 3 parts vs Goldilocks with 8 transforms per CMux) rests on measured rates of this GPU, not on
// pipe-rate arithmetic.  Lazy representation in [0, 2^64); 2^64 = 2^32 - 1 and 2^96 = -1 (mod p).
__device__ __forceinline__ uint64_t gl_red128(uint64_t lo, uint64_t hi) {
    const uint32_t hl = (uint32_t)hi, hh = (uint32_t)(hi >> 32);
    uint64_t t0 = lo - hh;
    if (lo < hh) t0 -= 0xFFFFFFFFull;                    // borrow of 2^64 = 2^32 - 1
    const uint64_t t1 = ((uint64_t)hl << 32) - hl;       // hl (2^32 - 1)
    uint64_t r = t0 + t1;
    if (r < t1) r += 0xFFFFFFFFull;                      // carry of 2^64
    return r;
}
__device__ __forceinline__ uint64_t gl_add(uint64_t x, uint64_t y) {
    uint64_t r = x + y;
    if (r < x) r += 0xFFFFFFFFull;
    return r;
}
__device__ __forceinline__ uint64_t gl_sub(uint64_t x, uint64_t y) {
    uint64_t r = x - y;
    if (x < y) r -= 0xFFFFFFFFull;
    return r;
}
// CT butterfly with a general twiddle w (64 x 64 -> 128-bit product, then the reduction above)
__device__ __forceinline__ void gl_bfly(uint64_t& x, uint64_t& y, uint64_t w) {
    const uint64_t t = gl_red128(y * w, __umul64hi(y, w));
    const uint64_t x0 = x;
    x = gl_add(x0, t);
    y = gl_sub(x0, t);
}
// CT butterfly whose twiddle is 2^s, 0 < s < 32 (four-step NTT with psi^32 = 8: shift-only inner/outer DFTs)
__device__ __forceinline__ void gl_bfly_shift(uint64_t& x, uint64_t& y, int s) {
    const uint64_t t = gl_red128(y << s, y >> (64 - s));
    const uint64_t x0 = x;
    x = gl_add(x0, t);
    y = gl_sub(x0, t);
}
template <int NV, bool SHIFT>
__global__ void __launch_bounds__(256) mb_gl_kernel(uint64_t* sink, int iters, uint64_t w, int sh) {
    uint64_t x[NV], y[NV];
#pragma unroll
    for (int i = 0; i < NV; i++) {
        x[i] = threadIdx.x * 0x9E3779B97F4A7C15ull + i;
        y[i] = threadIdx.x * 0xC2B2AE3D27D4EB4Full + 3u * i;
    }
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < NV; i++) {
            if (SHIFT) gl_bfly_shift(x[i], y[i], sh);
            else gl_bfly(x[i], y[i], w);
        }
        w ^= (uint64_t)(it & 1);
        sh = (sh & 15) + 3;
    }
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < NV; i++) s += x[i] ^ y[i];
    if (s == 0x123456789ull) sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// rates[0] = 30-bit Shoup butterflies/s (the kernels' own), [1] Goldilocks general-twiddle butterflies/s,
// [2] Goldilocks shift-twiddle butterflies/s, [3] 64-bit MACs/s; all SMs, register resident
int run_microbench_fields(int iters, double* rates) {
    double b = 0, m = 0;
    if (run_microbench(iters, &b, &m)) return -1;
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return -1;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return -1;
    const int blocks = sms * 8, threads = 256;
    void* sink = nullptr;
    if (cudaMalloc(&sink, (size_t)blocks * threads * 8) != cudaSuccess) return -1;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best_g = 1e30f, best_s = 1e30f;
    for (int rep = 0; rep < 4; rep++) {
        float ms = 0;
        cudaEventRecord(e0);
        mb_gl_kernel<8, false><<<blocks, threads>>>((uint64_t*)sink, iters, 0x61E96455F799F0A0ull, 3);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) best_g = ms < best_g ? ms : best_g;
        cudaEventRecord(e0);
        mb_gl_kernel<8, true><<<blocks, threads>>>((uint64_t*)sink, iters, 0ull, 3);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) best_s = ms < best_s ? ms : best_s;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    if (cudaGetLastError() != cudaSuccess) return -1;
    const double ops = (double)blocks * threads * iters * 8.0;
    rates[0] = b;
    rates[1] = ops / (best_g * 1e-3);
    rates[2] = ops / (best_s * 1e-3);
    rates[3] = m;
    return 0;
}

int run_microbench(int iters, double* bfly, double* mac) {
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return -1;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return -1;
    const int blocks = sms * 8, threads = 256;
    void* sink = nullptr;
    if (cudaMalloc(&sink, (size_t)blocks * threads * 8) != cudaSuccess) return -1;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best_b = 1e30f, best_m = 1e30f;
    for (int rep = 0; rep < 4; rep++) {
        float ms = 0;
        cudaEventRecord(e0);
        mb_bfly_kernel<16><<<blocks, threads>>>((uint32_t*)sink, iters, 123456789u, 987654u);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) best_b = ms < best_b ? ms : best_b;
        cudaEventRecord(e0);
        mb_mac_kernel<16><<<blocks, threads>>>((uint64_t*)sink, iters, 77u);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) best_m = ms < best_m ? ms : best_m;
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    if (cudaGetLastError() != cudaSuccess) return -1;
    const double ops = (double)blocks * threads * iters * 16.0;
    *bfly = ops / (best_b * 1e-3);
    *mac = ops / (best_m * 1e-3);
    return 0;
}

}  // namespace tb

// ---- FP64 FFT variant: diagnostic exact product (same transforms as the FFT blind-rotation kernel) ------
#include "tb_fft.cuh"

namespace tb {

int set_fft_constants(const double2* zeta16) {
    return cudaMemcpyToSymbol(c_zeta, zeta16, 16 * sizeof(double2)) == cudaSuccess ? 0 : -1;
}

// signed 16-bit halves of a torus word: x = lo + 2^16 hi (mod 2^32), lo, hi in [-2^15, 2^15)
__device__ __forceinline__ void split16(uint32_t x, int32_t& lo, int32_t& hi) {
    lo = (int32_t)(int16_t)(x & 0xFFFFu);
    hi = (int32_t)(int16_t)((x - (uint32_t)lo) >> 16);
}

struct FftDiagSmem {
    double2 twB[kTwB];
    double2 twC[kTwC];
    double2 d[kRows][512];
    double2 b[kRows][2][512];
};

__global__ void __launch_bounds__(192) fft_muladd6_kernel(const int32_t* digits, const uint32_t* polys, uint32_t* res,
                                                          const double2* twB, const double2* twC) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    FftDiagSmem& S = *reinterpret_cast<FftDiagSmem*>(smem_raw);
    const int lane = threadIdx.x & 31, r = threadIdx.x >> 5;
    for (int k = threadIdx.x; k < kTwB; k += blockDim.x) S.twB[k] = twB[k];
    for (int k = threadIdx.x; k < kTwC; k += blockDim.x) S.twC[k] = twC[k];
    __syncthreads();
    dcplx x[16];
#pragma unroll
    for (int j = 0; j < 16; j++) {
        const int k = lay_a(lane, j);
        x[j] = dcplx{(double)digits[r * kN + k], (double)digits[r * kN + k + 512]};
    }
    fft_fwd(x, S.d[r], S.twB, S.twC, lane);
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 16; j++) S.d[r][fswz(lay_d(lane, j))] = make_double2(x[j].re, x[j].im);
    for (int h = 0; h < 2; h++) {
#pragma unroll
        for (int j = 0; j < 16; j++) {
            const int k = lay_a(lane, j);
            int32_t l0, h0, l1, h1;
            split16(polys[r * kN + k], l0, h0);
            split16(polys[r * kN + k + 512], l1, h1);
            x[j] = h == 0 ? dcplx{(double)l0, (double)l1} : dcplx{(double)h0, (double)h1};
        }
        fft_fwd(x, S.b[r][h], S.twB, S.twC, lane);
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 16; j++)
            S.b[r][h][fswz(lay_d(lane, j))] = make_double2(x[j].re * (1.0 / 512), x[j].im * (1.0 / 512));
    }
    __syncthreads();
    // MAC into d[0] (h = 0) and d[1] (h = 1): thread owns positions k
    for (int k = threadIdx.x; k < 512; k += blockDim.x) {
        const int sk = fswz(k);
        dcplx D[kRows];
#pragma unroll
        for (int rr = 0; rr < kRows; rr++) D[rr] = dcplx{S.d[rr][sk].x, S.d[rr][sk].y};
#pragma unroll
        for (int h = 0; h < 2; h++) {
            dcplx acc = {0.0, 0.0};
#pragma unroll
            for (int rr = 0; rr < kRows; rr++) {
                const dcplx B = {S.b[rr][h][sk].x, S.b[rr][h][sk].y};
                acc.re = fma(D[rr].re, B.re, fma(-D[rr].im, B.im, acc.re));
                acc.im = fma(D[rr].re, B.im, fma(D[rr].im, B.re, acc.im));
            }
            S.d[h][sk] = make_double2(acc.re, acc.im);
        }
    }
    __syncthreads();
    if (r < 2) {
#pragma unroll
        for (int j = 0; j < 16; j++) {
            const double2 v = S.d[r][fswz(lay_d(lane, j))];
            x[j] = dcplx{v.x, v.y};
        }
        fft_inv(x, S.d[r], S.twB, S.twC, lane);
        __syncwarp();
        uint32_t* part = reinterpret_cast<uint32_t*>(S.b[r][0]);   // 1024 u32 scratch per half
#pragma unroll
        for (int j = 0; j < 16; j++) {
            const int k = lay_a(lane, j);
            part[k] = round_mod32(x[j].re);
            part[k + 512] = round_mod32(x[j].im);
        }
    }
    __syncthreads();
    const uint32_t* lo = reinterpret_cast<const uint32_t*>(S.b[0][0]);
    const uint32_t* hi = reinterpret_cast<const uint32_t*>(S.b[1][0]);
    for (int c = threadIdx.x; c < kN; c += blockDim.x) res[c] = lo[c] + (hi[c] << 16);
}

int launch_fft_muladd6(const int32_t* digits, const uint32_t* polys, uint32_t* res, const double2* twB,
                       const double2* twC, cudaStream_t st) {
    const size_t smem = sizeof(FftDiagSmem);
    if (cudaFuncSetAttribute(fft_muladd6_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess)
        return -1;
    fft_muladd6_kernel<<<1, 192, smem, st>>>(digits, polys, res, twB, twC);
    return 0;
}

}  // namespace tb
