// tb_kernels.cuh -- kernel argument blocks and host launchers shared by the library's translation unit.
#pragma once
#include <cuda_runtime.h>

#include <atomic>

#include "tb_common.cuh"

namespace tb {

// The >48 KB dynamic shared-memory opt-in (cudaFuncSetAttribute) is per device: remembered per (kernel, device)
// so that contexts on several GPUs of one process each get it (one atomic bit per device).
template <auto Kern>
inline int ensure_smem_attr(size_t bytes) {
    static std::atomic<uint64_t> done{0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return -1;
    const uint64_t bit = 1ull << (dev & 63);
    if (done.load(std::memory_order_acquire) & bit) return 0;
    if (cudaFuncSetAttribute(Kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess) return -1;
    done.fetch_or(bit, std::memory_order_acq_rel);
    return 0;
}

// blind rotation + extraction over a batch of lanes (tb_bootstrap.cu)
struct BrArgs {
    const uint32_t* src0;
    const uint32_t* src1;
    const uint32_t* src2;
    int64_t src_stride;        // words between ciphertext rows (>= n + 1)
    const LaneDesc* lanes;
    int32_t nlanes;
    const uint32_t* bkhat;     // [n][6 rows][6 outs][N]  (u32 < p)
    const uint2* twF;          // [31][32] per-lane forward twiddles (w, w')
    const uint2* twI;          // [31][32] per-lane inverse twiddles
    uint32_t* out;             // [nlanes][out_stride] extracted LWE(N) samples
    int64_t out_stride;        // words between output rows (>= N + 1; kLaneStride for the lane buffer)
};

// key switch + MUX combine + NOT over a batch of gates (tb_keyswitch.cu)
struct KsArgs {
    const uint32_t* lanes;      // extracted samples from br_kernel
    int32_t lane_base;          // GateDesc.lane* - lane_base = row in `lanes`
    int64_t lane_stride;        // words between lane rows (kLaneStride for the lane buffer)
    const GateDesc* gates;
    int32_t ngates;
    const uint32_t* ksk;        // [N][t][3][kKsRow]  (digit-0 rows dropped)
    uint32_t* out;              // output ciphertext rows
    int64_t out_stride;
    const uint32_t* not_src;    // NOT input rows
    int64_t not_stride;
    // fused all-gather (multi-GPU level loop): every output row is also stored, at the same row offset, into the
    // npeers other ranks' wire arrays (peer memory mapped into this process); 0 = own array only
    uint32_t* const* peers;     // device array [npeers] of peer wire bases (same stride as out)
    int32_t npeers;
};

int launch_br6(const BrArgs& A, int G, cudaStream_t st);
int launch_br9(const BrArgs& A, cudaStream_t st);
void launch_bk_to_ntt(const uint32_t* bk, uint32_t* bkhat, const uint2* twF, uint32_t ninv, uint32_t ninvp,
                      cudaStream_t st);
void launch_build_gate_desc(int kind, int32_t wa, int32_t wb, uint32_t cst, int64_t count, LaneDesc* lanes,
                            GateDesc* gates, cudaStream_t st);
int launch_ks(const KsArgs& A, int tile, uint32_t* partial, int S, cudaStream_t st);   // S > 1: sliced + reduce
int ks_tile_slices(int64_t ngates, int tile);
int launch_ks_split(const KsArgs& A, uint32_t* partial, cudaStream_t st);   // narrow levels
size_t ks_split_scratch_words(int64_t ngates);
void launch_ksk_relayout(const uint32_t* src, uint32_t* dst, cudaStream_t st);
int set_ntt_constants(const uint32_t* fw, const uint32_t* fwp, const uint32_t* iw, const uint32_t* iwp,
                      const uint32_t* misc);
int launch_ntt_muladd6(const int32_t* digits, const uint32_t* polys, uint32_t* res, const uint2* twF,
                       const uint2* twI, uint32_t ninv, uint32_t ninvp, cudaStream_t st);
int run_microbench(int iters, double* bfly, double* mac);
int run_microbench_fields(int iters, double* rates);
int run_tc_mma_test(const uint8_t* A, const uint8_t* B, int K, int N, int a_signed, int b_signed, int lbo, int32_t* D,
                    cudaStream_t st);

}  // namespace tb


namespace tb {
int set_fft_constants(const double2* zeta16);
int launch_fft_muladd6(const int32_t* digits, const uint32_t* polys, uint32_t* res, const double2* twB,
                       const double2* twC, cudaStream_t st);
}  // namespace tb

namespace tb {
int launch_brf(const BrArgs& A, int G, const double2* bkf, const double2* twB, const double2* twC, cudaStream_t st);
void launch_bk_to_fft(const uint32_t* bk, double2* bkf, const double2* twB, const double2* twC, cudaStream_t st);
size_t bkf_bytes();
// latency mode, one bootstrap per 2-SM cluster on the FP64 pipe (tb_brl2.cu); brl2_wave_lanes = co-resident clusters
int launch_brl2(const BrArgs& A, const double2* bkf, const double2* twL, cudaStream_t st);
int brl2_wave_lanes();
int launch_brl(const BrArgs& A, const double2* bkf, const double2* twL, cudaStream_t st);
int brl_wave_lanes();
}  // namespace tb

namespace tb {
// tensor-core blind rotation (tb_brt.cu)
int launch_brt(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st);
// br6 with the forward NTT on the tensor cores (tb_br6t.cu): 2 lanes per CTA, NTT-domain BK (bkhat)
int launch_br6t(const BrArgs& A, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st);
// both NTT directions on the tensor cores in br6's shape (tb_brq.cu): 2 lanes per CTA, natural-order BK (bk4)
int launch_brq(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st);
int launch_brtl(const BrArgs& A, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw, cudaStream_t st);
int launch_brt_muladd(const int32_t* digits, const uint32_t* bk4, const unsigned char* tcB, const uint2* tcTw,
                      uint32_t* res, cudaStream_t st);
void launch_bk_to_bk4(const uint32_t* bk, uint32_t* bk4, const uint2* pts, uint32_t ninv, uint32_t ninvp, int n_i,
                      cudaStream_t st);
size_t bk4_bytes();
void brt_tables(uint32_t psi, unsigned char* B, uint2* tw, uint2* pts);
size_t brt_table_bytes();
}  // namespace tb
