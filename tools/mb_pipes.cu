// Microbenchmark of the per-SM pipes an FP64 blind rotation would load (round 2 design study):
// DFMA, SHFL.32, LDS.128 / STS.128 (conflict-free), LDG.128 hitting L1, tcgen05.st / tcgen05.ld (32x32b.x32),
// and DFMA mixed with LDS.128 / SHFL.  One CTA of 512 threads (16 warps) per SM, clock64 around the loop;
// reports warp-instructions per SM clock (per sub-partition x4).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb_pipes tools/mb_pipes.cu
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void __launch_bounds__(512, 1) kern(double* sink, const double2* gsrc, long long* cyc, int iters) {
    __shared__ __align__(16) double2 buf[64 * 32];   // 32 KB
    __shared__ uint32_t tbase;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    double a[16];
#pragma unroll
    for (int i = 0; i < 16; i++) a[i] = 1.0 + 1e-9 * (tid + i);
    for (int k = tid; k < 64 * 32; k += 512) buf[k] = make_double2(k, -k);
    if (MODE >= 5 && MODE <= 6) {
        if (warp == 0) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase)) : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
        }
    }
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t taddr = tbase + ((uint32_t)(32 * (warp & 3)) << 16) + 32u * (warp >> 2);
    const long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        if (MODE == 0) {   // DFMA: 16 independent chains, 64 DFMA per iteration
#pragma unroll
            for (int r = 0; r < 4; r++)
#pragma unroll
                for (int i = 0; i < 16; i++) a[i] = fma(a[i], 0.999999, 1e-7);
        } else if (MODE == 1) {   // SHFL.32: 64 per iteration
#pragma unroll
            for (int r = 0; r < 2; r++)
#pragma unroll
                for (int i = 0; i < 16; i++) {
                    const int2 v = make_int2(__double2loint(a[i]), __double2hiint(a[i]));
                    a[i] = __hiloint2double(__shfl_xor_sync(0xffffffffu, v.y, 1 + (i & 3)), __shfl_xor_sync(0xffffffffu, v.x, 1 + (i & 3)));
                }
        } else if (MODE == 2) {   // LDS.128: 16 per iteration, conflict-free (consecutive lanes, 16 B each)
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const double2 v = buf[((it + warp * 16 + i) & 63) * 32 + lane];
                a[i] += v.x * v.y;
            }
        } else if (MODE == 3) {   // STS.128: 16 per iteration
#pragma unroll
            for (int i = 0; i < 16; i++) {
                double2* p = &buf[((it + warp * 16 + i) & 63) * 32 + lane];
                asm volatile("st.shared.v2.f64 [%0], {%1, %2};" ::"r"(smem_u32(p)), "d"(a[i]), "d"(a[(i + 1) & 15]) : "memory");
            }
            a[it & 15] += 1.0;
        } else if (MODE == 10) {   // STS.64: 32 per iteration (same bytes as 16 STS.128)
#pragma unroll
            for (int i = 0; i < 16; i++) {
                double* p = reinterpret_cast<double*>(&buf[((it + warp * 16 + i) & 63) * 32 + lane]);
                asm volatile("st.shared.f64 [%0], %1;" ::"r"(smem_u32(p)), "d"(a[i]) : "memory");
                asm volatile("st.shared.f64 [%0], %1;" ::"r"(smem_u32(p + 1)), "d"(a[(i + 1) & 15]) : "memory");
            }
            a[it & 15] += 1.0;
        } else if (MODE == 11) {   // STS.32: 64 per iteration (same bytes)
#pragma unroll
            for (int i = 0; i < 16; i++) {
                float* p = reinterpret_cast<float*>(&buf[((it + warp * 16 + i) & 63) * 32 + lane]);
#pragma unroll
                for (int w = 0; w < 4; w++)
                    asm volatile("st.shared.b32 [%0], %1;" ::"r"(smem_u32(p + w)), "r"(__double2loint(a[(i + w) & 15])) : "memory");
            }
            a[it & 15] += 1.0;
        } else if (MODE == 12) {   // STS.128 with a 16-B lane stride but lanes permuted within 8-lane groups
#pragma unroll
            for (int i = 0; i < 16; i++) {
                double2* p = &buf[((it + warp * 16 + i) & 63) * 32 + (lane ^ (i & 7))];
                asm volatile("st.shared.v2.f64 [%0], {%1, %2};" ::"r"(smem_u32(p)), "d"(a[i]), "d"(a[(i + 1) & 15]) : "memory");
            }
            a[it & 15] += 1.0;
        } else if (MODE == 4) {   // LDG.128 from a 32 KB block (L1 resident): 16 per iteration
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const double2 v = __ldg(gsrc + ((it * 16 + i) & 63) * 32 + lane);
                a[i] += v.x;
            }
        } else if (MODE == 5) {   // tcgen05.st 32x32b.x32 (32 words / thread), 2 per iteration + wait
#pragma unroll
            for (int h = 0; h < 4; h++) {
                uint32_t r[32];
#pragma unroll
                for (int i = 0; i < 16; i++) { r[2 * i] = __double2loint(a[i]); r[2 * i + 1] = __double2hiint(a[i]) + h; }
                asm volatile(
                    "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
                    "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr + 64u * (h & 1) + 256u * (h >> 1)),
                    "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
                    "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]),
                    "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]),
                    "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
                    : "memory");
            }
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            a[it & 15] += 1.0;
        } else if (MODE == 6) {   // tcgen05.ld 32x32b.x16, 4 in flight per wait (64 words / thread)
            uint32_t r[4][16];
#pragma unroll
            for (int h = 0; h < 4; h++)
                asm volatile(
                    "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                    : "=r"(r[h][0]), "=r"(r[h][1]), "=r"(r[h][2]), "=r"(r[h][3]), "=r"(r[h][4]), "=r"(r[h][5]),
                      "=r"(r[h][6]), "=r"(r[h][7]), "=r"(r[h][8]), "=r"(r[h][9]), "=r"(r[h][10]), "=r"(r[h][11]),
                      "=r"(r[h][12]), "=r"(r[h][13]), "=r"(r[h][14]), "=r"(r[h][15])
                    : "r"(taddr + 16u * h + 128u * (it & 1)));
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
            for (int h = 0; h < 4; h++)
#pragma unroll
                for (int i = 0; i < 4; i++) a[4 * h + i] += __hiloint2double(r[h][4 * i + 1] & 0x3FF00000, r[h][4 * i] ^ r[h][4 * i + 2]);
        } else if (MODE == 7) {   // mix: 64 DFMA + 16 LDS.128
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const double2 v = buf[((it + warp * 16 + i) & 63) * 32 + lane];
                a[i] = fma(a[i], v.x, 1e-7);
                a[i] = fma(a[i], 0.999999, v.y);
                a[i] = fma(a[i], 0.999999, 1e-7);
                a[i] = fma(a[i], 0.999999, 1e-7);
            }
        } else if (MODE == 8) {   // mix: 64 DFMA + 32 SHFL
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const int2 v = make_int2(__double2loint(a[i]), __double2hiint(a[i]));
                const double s = __hiloint2double(__shfl_xor_sync(0xffffffffu, v.y, 1), __shfl_xor_sync(0xffffffffu, v.x, 1));
                a[i] = fma(a[i], s, 1e-7);
                a[i] = fma(a[i], 0.999999, 1e-7);
                a[i] = fma(a[i], 0.999999, 1e-7);
                a[i] = fma(a[i], 0.999999, 1e-7);
            }
        } else if (MODE == 9) {   // mix: 64 DFMA + 16 LDG.128 (L1)
#pragma unroll
            for (int i = 0; i < 16; i++) {
                const double2 v = __ldg(gsrc + ((it * 16 + i) & 63) * 32 + lane);
                a[i] = fma(a[i], v.x, 1e-7);
                a[i] = fma(a[i], 0.999999, v.y);
                a[i] = fma(a[i], 0.999999, 1e-7);
                a[i] = fma(a[i], 0.999999, 1e-7);
            }
        }
    }
    const long long t1 = clock64();
    __syncthreads();
    if (tid == 0) cyc[blockIdx.x] = t1 - t0;
    double s = 0;
#pragma unroll
    for (int i = 0; i < 16; i++) s += a[i];
    if (s == 12345.678) sink[blockIdx.x * 512 + tid] = s;
    if (MODE >= 5 && MODE <= 6) {
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase) : "memory");
    }
}

template <int MODE>
static void run(const char* name, double per_iter, double* sink, const double2* g, long long* cyc, int nsm) {
    const int iters = 20000;
    for (int rep = 0; rep < 2; rep++) {
        kern<MODE><<<nsm, 512>>>(sink, g, cyc, iters);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(e)); return; }
    }
    long long h[1024];
    cudaMemcpy(h, cyc, nsm * sizeof(long long), cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (int i = 0; i < nsm; i++) mx = h[i] > mx ? h[i] : mx;
    // 16 warps per SM, per_iter warp-instructions of the measured kind per warp per iteration
    printf("{\"test\": \"%s\", \"warp_instr_per_sm_clk\": %.3f, \"cycles\": %lld}\n", name, 16.0 * per_iter * iters / mx, mx);
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    double* sink;
    double2* g;
    long long* cyc;
    cudaMalloc(&sink, (size_t)nsm * 512 * 8);
    cudaMalloc(&g, 64 * 32 * 16);
    cudaMemset(g, 0, 64 * 32 * 16);
    cudaMalloc(&cyc, nsm * sizeof(long long));
    run<0>("DFMA", 64, sink, g, cyc, nsm);
    run<1>("SHFL.32", 64, sink, g, cyc, nsm);
    run<2>("LDS.128", 16, sink, g, cyc, nsm);
    run<3>("STS.128", 16, sink, g, cyc, nsm);
    run<4>("LDG.128_L1hit", 16, sink, g, cyc, nsm);
    run<5>("tcgen05.st.32x32b.x32 (4 per wait)", 4, sink, g, cyc, nsm);
    run<6>("tcgen05.ld.32x32b.x16 (4 per wait)", 4, sink, g, cyc, nsm);
    run<7>("mix_DFMA64_LDS128x16 (DFMA count)", 64, sink, g, cyc, nsm);
    run<8>("mix_DFMA64_SHFLx32 (DFMA count)", 64, sink, g, cyc, nsm);
    run<9>("mix_DFMA64_LDG128x16 (DFMA count)", 64, sink, g, cyc, nsm);
    run<10>("STS.64 (x2 per 16 B)", 32, sink, g, cyc, nsm);
    run<11>("STS.32 (x4 per 16 B)", 64, sink, g, cyc, nsm);
    run<12>("STS.128 lane-permuted", 16, sink, g, cyc, nsm);
    run<3>("STS.128 (again)", 16, sink, g, cyc, nsm);
    return 0;
}
