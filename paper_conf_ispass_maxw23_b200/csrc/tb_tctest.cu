// tb_tctest.cu -- diagnostic: one CTA computes D = A . B^T with tcgen05.mma kind::i8 through the same
// descriptor / TMEM helpers as the tensor-core blind rotation (tb_tc.cuh), so the operand layouts, the
// instruction descriptor and the TMEM read-back are checked against a plain integer matrix product.
#include "tb_kernels.cuh"
#include "tb_tc.cuh"

namespace tb {

// A: [128][K] bytes, B: [N][K] bytes (row-major in global memory), D: [128][N] s32.  K % 32 == 0, K <= 256,
// N % 16 == 0, N <= 256.  lbo = byte stride between K-adjacent core matrices (>= 128, multiple of 16).
__global__ void __launch_bounds__(128) tc_mma_test_kernel(const uint8_t* __restrict__ A, const uint8_t* __restrict__ B,
                                                          int K, int N, uint32_t idesc, int lbo, int32_t* __restrict__ D) {
    extern __shared__ __align__(1024) unsigned char tsm[];
    __shared__ uint64_t mbar;
    __shared__ uint32_t tbase;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const uint32_t sbo_a = (uint32_t)(K / 16) * lbo, sbo_b = sbo_a;
    unsigned char* sA = tsm;
    unsigned char* sB = tsm + 16 * sbo_a;                          // 128 rows = 16 row groups
    for (int e = tid; e < 128 * K; e += 128) sA[tc_off(e / K, e % K, lbo, sbo_a)] = A[e];
    for (int e = tid; e < N * K; e += 128) sB[tc_off(e / K, e % K, lbo, sbo_b)] = B[e];
    if (warp == 0) tc_alloc<256>(&tbase);
    if (tid == 0) {
        mbar_init(&mbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    fence_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tbase;
    if (tid == 0) {
        for (int s = 0; s < K / 32; s++) {
            const uint64_t da = tc_sdesc(smem_u32(sA) + s * 2 * lbo, lbo, sbo_a);
            const uint64_t db = tc_sdesc(smem_u32(sB) + s * 2 * lbo, lbo, sbo_b);
            tc_mma_i8(tmem, da, db, idesc, s > 0);
        }
        tc_commit(smem_u32(&mbar));
    }
    mbar_wait(&mbar, 0);
    tc_fence_after();
    for (int c = 0; c < N; c += 8) {
        uint32_t v[8];
        tc_ld8(tmem + ((uint32_t)(32 * warp) << 16) + c, v);
        tc_wait_ld();
#pragma unroll
        for (int k = 0; k < 8; k++) D[(32 * warp + lane) * N + c + k] = (int32_t)v[k];
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tc_dealloc<256>(tmem);
}

int run_tc_mma_test(const uint8_t* A, const uint8_t* B, int K, int N, int a_signed, int b_signed, int lbo, int32_t* D,
                    cudaStream_t st) {
    if (K % 32 || K <= 0 || K > 256 || N % 16 || N <= 0 || N > 256 || lbo < 128 || lbo % 16) return -2;
    const size_t smem = (size_t)(16 + N / 8) * (K / 16) * lbo;
    if (cudaFuncSetAttribute(tc_mma_test_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return -1;
    tc_mma_test_kernel<<<1, 128, smem, st>>>(A, B, K, N, tc_idesc_i8(128, N, a_signed, b_signed), lbo, D);
    return 0;
}

}  // namespace tb
