// tb_tc.cuh -- 5th-generation tensor-core (tcgen05) primitives for the integer NTT of the blind rotation.
//
// The negacyclic NTT of length 1024 over Z_p (p = 0x3FFF7801, tb_common.cuh) is evaluated in four steps: a
// 32-point DFT over the rows of the 32 x 32 coefficient matrix, a twiddle, a 32-point DFT over the columns
// (DESIGN.md "Tensor-core NTT").  Both DFTs are exact integer matrix products done by tcgen05.mma kind::i8 on
// byte limbs (u8 x u8 / s8 x u8 -> s32 in TMEM), the limb recombination and the reductions mod p by the CUDA
// cores.  Operands are K-major, no swizzle: an R x K (bytes) tile is made of 8-row x 16-byte core matrices,
// core matrix (g = row / 8, c = kbyte / 16) at g * SBO + c * LBO, row r of it at 16 r.
#pragma once
#include <cstdint>

namespace tb {

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// shared-memory matrix descriptor (sm_100 "version 1"), SWIZZLE_NONE, K-major; addresses / strides in bytes
__device__ __forceinline__ uint64_t tc_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}
// instruction descriptor of kind::i8 with an s32 accumulator: M x N, A / B signed (s8) or unsigned (u8), K-major
__host__ __device__ constexpr uint32_t tc_idesc_i8(int M, int N, bool a_signed, bool b_signed) {
    return (2u << 4) | ((a_signed ? 1u : 0u) << 7) | ((b_signed ? 1u : 0u) << 10) | ((uint32_t)(N >> 3) << 17) |
           ((uint32_t)(M >> 4) << 24);
}
// D[tmem] (+)= A[smem] . B[smem]^T, one thread issues for the CTA
__device__ __forceinline__ void tc_mma_i8(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    const uint32_t z = 0;
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
        " tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, {%5, %6, %7, %8}, p;\n}\n" ::"r"(tmem_d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc), "r"(z), "r"(z), "r"(z), "r"(z)
        : "memory");
}
// completion of every tcgen05.mma issued so far by this thread -> one arrive on the mbarrier
__device__ __forceinline__ void tc_commit(uint32_t mbar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(mbar)
                 : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
// generic-proxy shared-memory writes -> visible to the tensor core's (async proxy) operand reads
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// TMEM allocation by one full warp; the base address is written to *dst (shared memory)
template <int NCOLS>
__device__ __forceinline__ void tc_alloc(uint32_t* dst) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst)),
                 "n"(NCOLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
template <int NCOLS>
__device__ __forceinline__ void tc_dealloc(uint32_t taddr) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(NCOLS) : "memory");
}

// 32 lanes x 32-bit, 8 / 16 / 32 consecutive columns per thread (lane = TMEM lane of the warp's quadrant)
__device__ __forceinline__ void tc_ld8(uint32_t taddr, uint32_t (&v)[8]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(taddr));
}
__device__ __forceinline__ void tc_ld16(uint32_t taddr, uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
}

// mbarrier (CTA scope)
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
// try_wait with a suspend-time hint: a waiting thread sleeps in the barrier instead of re-issuing the test
// (the spinning MMA thread otherwise takes issue slots from the compute warps of its sub-partition)
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
#ifdef TB_NO_SUSPEND_HINT
    asm volatile(
        "{\n .reg .pred p;\n TCW_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra TCW_%=;\n}\n" ::"r"(smem_u32(b)),
        "r"(parity)
        : "memory");
#else
    asm volatile(
        "{\n .reg .pred p;\n TCW_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
        " @!p bra TCW_%=;\n}\n" ::"r"(smem_u32(b)),
        "r"(parity), "r"(0x100000u)
        : "memory");
#endif
}

// byte offset of (row, kbyte) in a K-major no-swizzle tile with the given core-matrix strides
__host__ __device__ constexpr uint32_t tc_off(uint32_t row, uint32_t kbyte, uint32_t lbo, uint32_t sbo) {
    return (row >> 3) * sbo + (kbyte >> 4) * lbo + (row & 7) * 16 + (kbyte & 15);
}

}  // namespace tb
