// scratch microbenchmark: 30-bit Shoup butterfly vs a butterfly whose Shoup quotient comes from the FP64 pipe
#include <cstdio>
#include <cstdint>
constexpr uint32_t kP = 1073707009u, kTwoP = 2u * kP;
__device__ __forceinline__ uint32_t red_2p(uint32_t x) { return min(x, x - kTwoP); }
__device__ __forceinline__ uint32_t shoup(uint32_t y, uint32_t w, uint32_t wp) { return y * w - __umulhi(y, wp) * kP; }
__device__ __forceinline__ uint32_t fpq(uint32_t y, uint32_t w, double wd) {
    const double M = 6755399441055744.0;                  // 2^52 + 2^51
    const double r = fma((double)y, wd, M);               // M + round(y w / p)
    const uint32_t q = (uint32_t)__double2loint(r);
    return (y * w + kP) - q * kP;                          // in (0.5 p, 1.5 p)
}
template <int MODE>
__global__ void k(uint32_t* sink, int iters, uint32_t w, uint32_t wp, double wd) {
    uint32_t x[16], y[16];
    for (int i = 0; i < 16; i++) { x[i] = threadIdx.x * 7u + i; y[i] = threadIdx.x * 13u + 3u * i; }
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < 16; i++) {
            const uint32_t X = red_2p(x[i]);
            const uint32_t T = (MODE == 0 || (MODE == 2 && (i & 1)) || (MODE == 3 && (i % 4 != 0))) ? shoup(y[i], w, wp) : fpq(y[i], w, wd);
            x[i] = X + T;
            y[i] = X - T + kTwoP;
        }
        w ^= (uint32_t)it & 1u;
    }
    uint32_t s = 0;
    for (int i = 0; i < 16; i++) s += x[i] ^ y[i];
    if (s == 0x12345678u) sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void check(uint32_t* bad, uint32_t w, uint32_t wp, double wd) {
    uint32_t y = blockIdx.x * blockDim.x + threadIdx.x;
    for (int rep = 0; rep < 64; rep++, y = y * 2654435761u + 12345u) {
        const uint32_t a = shoup(y, w, wp), b = fpq(y, w, wd);
        const uint64_t t = (uint64_t)y * w % kP;
        if (a % kP != t || b % kP != t || b >= kTwoP) atomicAdd(bad, 1u);
    }
}
int main() {
    const uint32_t w = 123456789u % kP, wp = (uint32_t)(((uint64_t)w << 32) / kP);
    const double wd = (double)w / (double)kP;
    uint32_t *sink, *bad;
    cudaMalloc(&sink, 148 * 8 * 256 * 4);
    cudaMallocManaged(&bad, 4);
    *bad = 0;
    check<<<4096, 256>>>(bad, w, wp, wd);
    cudaDeviceSynchronize();
    printf("mismatches: %u\n", *bad);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int iters = 4096;
    for (int mode = 0; mode < 4; mode++)
        for (int rep = 0; rep < 3; rep++) {
            cudaEventRecord(e0);
            if (mode == 0) k<0><<<148 * 8, 256>>>(sink, iters, w, wp, wd);
            else if (mode == 1) k<1><<<148 * 8, 256>>>(sink, iters, w, wp, wd);
            else if (mode == 2) k<2><<<148 * 8, 256>>>(sink, iters, w, wp, wd);
            else k<3><<<148 * 8, 256>>>(sink, iters, w, wp, wd);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            printf("mode %d: %.3f ms, %.3f T butterflies/s\n", mode, ms, 148.0 * 8 * 256 * iters * 16 / (ms * 1e-3) / 1e12);
        }
}
