// tb_common.cuh -- compile-time parameters, NTT field and device-side descriptors of the B200 path.
//
// Parameters: tfhe-lib's 128-bit gate-bootstrapping set, which PyTFHE uses ("the default parameter set as
// described in Section VIII of the TFHE paper [7]", Sec. II-D; n = 630 is pinned by the
// 2.46 KB ciphertext of P:241).  Nothing here is shared with oracle/: every constant is re-derived.
#pragma once
#include <cstdint>

namespace tb {

constexpr int kN = 1024;           // TRLWE ring degree
constexpr int kTwoN = 2 * kN;
constexpr int kn = 630;            // LWE dimension
constexpr int kL = 3;              // gadget length l
constexpr int kBgbit = 7;          // log2 Bg
constexpr int kRows = 2 * kL;      // TGSW rows (k+1) l
constexpr int kKsT = 8;            // key-switch digits t
constexpr int kKsBasebit = 2;      // key-switch base 4
constexpr int kKsBase = 1 << kKsBasebit;
constexpr uint32_t kMu = 1u << 29; // 1/8 on the torus

// Gadget decomposition offset sum_j (Bg/2) 2^(32 - Bgbit (j+1)) (tfhe-lib's truncating reading, R4)
constexpr uint32_t kDecompOffset = (64u << 25) + (64u << 18) + (64u << 11);
static_assert(kDecompOffset == 0x81020000u, "decomposition offset");

// ---- exact NTT field ----------------------------------------------------------------------------
// The torus-2^32 products of the external product are computed exactly as integers:
// each BK coefficient is split into 3 signed parts of <= 11 bits, |part| <= 2^10, so every coefficient of
// sum_{r<6} D_r (x) part_r has |value| <= 6 * 1024 * 64 * 1024 = 402,653,184 < p/2.  With p < 2^30 the
// lazy butterflies keep values below 4p < 2^32.
constexpr uint32_t kP = 1073707009u;               // 0x3FFF7801 = 524271 * 2^11 + 1, prime
constexpr uint32_t kTwoP = 2u * kP;
constexpr uint32_t kHalfP = (kP - 1u) / 2u;
constexpr int kParts = 3;                          // BK split: bits [0,11), [11,22), [22,32)
constexpr int kOuts = 2 * kParts;                  // MAC outputs per gate: (poly q in {a,b}) x part m
static_assert(2ull * kRows * kN * 64ull * 1024ull < kP, "exactness bound");
static_assert(4ull * kP < (1ull << 32), "lazy bound");

// ---- device layouts --------------------------------------------------------------------------------
constexpr int kLaneStride = 1028;       // extracted LWE(kN) sample: a[1024], b, 3 pad words (16 B rows)
constexpr int kKsRow = 632;             // device KSK row: n+1 = 631 words + 1 pad (16 B aligned)
constexpr int kPadRow = 33;             // padded 32x33 layout of one NTT slot (conflict-free transpose)
constexpr int kSlotWords = 32 * kPadRow;

// One blind-rotation lane = one bootstrap (a gate has 1 lane, MUX has 2): the linear combination
// wa * A[ia] + wb * B[ib] + (0, ..., 0, cst) over the source arrays selected by `sel`.
struct LaneDesc {
    int32_t ia, ib;         // source rows (ib < 0: no second input)
    int32_t wa, wb;         // small signed weights
    uint32_t cst;           // torus constant added to b
    uint32_t sel;           // bits 0-1: array of ia, bits 2-3: array of ib (0, 1, 2 = src0/src1/src2)
    uint32_t pad0, pad1;
};
// One output gate of the key-switch kernel: KS(lane0 [+ lane1 + (0, mu)]) or NOT (negate an input row).
enum : int32_t { kGateBoot = 0, kGateMux = 1, kGateNot = 2 };
struct GateDesc {
    int32_t out_row;        // destination row in the output array
    int32_t lane0;          // lane index (relative to the launch) or, for NOT, source row (array 0)
    int32_t lane1;          // second lane (MUX) else -1
    int32_t kind;
};

}  // namespace tb
