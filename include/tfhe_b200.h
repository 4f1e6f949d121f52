/*
 * tfhe_b200.h -- C ABI of the B200-native TFHE gate-bootstrapping library (libtfhe_b200.so).
 *
 * What it does: the data-parallel hot path of PyTFHE's execution backend (Ma, Xu, Wills, ISPASS 2023) --
 * batched bootstrapped gates over the independent gates of one level of a levelised netlist.
 *   P:N = /root/reference/PAPER.md line N.  "Cn" / "Rn" = readings listed in DESIGN.md.
 *   - Problem statement: the backend exposes "bootstrapped gate computations (e.g., bootstrapped-NAND,
 *     bootstrapped-XOR)" on ciphertexts; the key is broadcast to the workers before traversal
 *     (P:239); a program is a DAG of gates traversed level by level by Algorithm 1 and the
 *     output nodes are returned.
 *   - A bootstrapped gate = linear combination -> blind rotation -> sample extraction ->
 *     key switching, at the TFHE default 128-bit parameters: n=630 N=1024 k=1 l=3 Bgbit=7,
 *     KS t=8 base 4.  Only this parameter set is compiled; anything else -> TB_EUNSUPPORTED.
 *
 * Data types.  Torus32 values are uint32_t.  An LWE ciphertext is a[0..629], b (631 words) stored in a row
 * of `stride` >= 631 words.  Keys are produced by the client (secret keys never reach this library).
 *
 * Conventions.
 *   - Every function returns int status: 0 = TB_OK, < 0 = error; nothing throws across the ABI.  On error
 *     tb_last_error() returns a thread-local message.
 *   - Pointers named dev_* / wires / out / ca / cb / cc are DEVICE pointers (cudaMalloc or torch tensors'
 *     data_ptr()) on the context's device; host_* pointers are host memory (pinned for async copies).
 *   - The caller owns every ciphertext buffer; the context owns keys and scratch.
 *   - Run calls (tb_gates, tb_run_level, tb_run_netlist) are stream-ordered on `stream` and never
 *     synchronise the device.  Load calls and tb_gates_host synchronise.
 *   - Thread-compatible: a context may be used by one host thread / one stream at a time (it owns
 *     scratch buffers that a second concurrent stream would race on).
 */
#ifndef TFHE_B200_H
#define TFHE_B200_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* tb_stream;   /* == cudaStream_t; NULL = legacy default stream */

typedef struct {
    int32_t n, N, k, l, Bgbit, ks_t, ks_basebit;
} tb_params;

typedef struct tb_ctx tb_ctx;

enum {
    TB_OK = 0,
    TB_EINVAL = -1,        /* null pointer, bad count / stride / index / gate code */
    TB_EUNSUPPORTED = -2,  /* parameter set other than the compiled one, or device is not sm_100 */
    TB_ENOKEYS = -3,       /* a run call before tb_load_bk and tb_load_ksk */
    TB_ECUDA = -4,         /* CUDA runtime error (message in tb_last_error) */
    TB_ENOMEM = -5         /* device or host allocation failed */
};

/* Gate codes = the 4-bit PyTFHE type field, read as the truth table f(a,b) at bit (2a+b) (Fig. 5;
 * reading C15; XOR = 0110 is the one code the paper prints).  MUX is a 3-input extension. */
enum tb_gate {
    TB_NOR = 1, TB_ANDNY = 2, TB_NOT = 3, TB_ANDYN = 4, TB_XOR = 6, TB_NAND = 7, TB_AND = 8,
    TB_XNOR = 9, TB_ORNY = 11, TB_ORYN = 13, TB_OR = 14, TB_MUX = 16
};

/* Default parameters (n=630, N=1024, k=1, l=3, Bgbit=7, ks_t=8, ks_basebit=2). */
tb_params tb_default_params(void);

/* Create a context on CUDA device `cuda_device`.  Fails with TB_EUNSUPPORTED for any other parameter set
 * or a device without compute capability 10.0.  *out receives the context. */
int tb_ctx_create(const tb_params* params, int cuda_device, tb_ctx** out);
int tb_ctx_destroy(tb_ctx* ctx);

/* Bootstrapping key, HOST pointer, torus layout [i < n][row r = bloc*l + j < 2l][poly < 2][N] u32
 * (n_words must equal n*2l*2*N = 7,741,440).  The torus key stays on the device (31 MB) and only the transform
 * domains that the selected kernels read are built from it: the NTT domain (br6 / br6t / br9: each coefficient
 * split into 3 signed parts, 92.9 MB), the FFT domain (brf / brl / brl2, 123.9 MB), the four-step NTT domain
 * (brt / brq / brtl, 92.9 MB).
 * Selecting another kernel later (tb_set_br_variant / tb_set_narrow_kernel / tb_set_narrow_lanes) builds the
 * domains it needs then (synchronously).  No host copy is kept.  Synchronous. */
int tb_load_bk(tb_ctx* ctx, const uint32_t* host_bk, size_t n_words);
/* Key-switching key, HOST pointer, layout [i < N][j < t][d < 4][n+1] u32 (n_words = 10,338,304).  Digit-0
 * rows (encryptions of 0, never read, C9) are dropped and rows padded to 632 words (62.1 MB).  Synchronous. */
int tb_load_ksk(tb_ctx* ctx, const uint32_t* host_ksk, size_t n_words);

/* Batched single-type bootstrapped gates over DEVICE arrays: out[g] = gate(ca[g], cb[g] [, cc[g]]) for
 * g < count, rows `stride` words apart in every array.  cb is ignored for TB_NOT; cc is used by TB_MUX
 * only.  out must not alias the inputs.  Async on `stream`. */
int tb_gates(tb_ctx* ctx, int gate, const uint32_t* ca, const uint32_t* cb, const uint32_t* cc,
             uint32_t* out, int64_t count, int64_t stride, tb_stream stream);

/* Same, HOST arrays (end-to-end path: host->device copies, gates, device->host copy, synchronise).  Uses
 * context-owned device staging buffers.  On any error the call still returns only after every copy it queued
 * from / into the host arrays has finished. */
int tb_gates_host(tb_ctx* ctx, int gate, const uint32_t* host_ca, const uint32_t* host_cb,
                  const uint32_t* host_cc, uint32_t* host_out, int64_t count, int64_t stride);

/* ---- netlists (Algorithm 1) ------------------------------------------------------------
 * Wire ids: [0, n_inputs) are the program inputs, n_inputs + g is the output of gate g.  type[g] is a gate
 * code; in1 = -1 for NOT, in2 = -1 unless MUX.  Gates may be listed in any order (no topological order is
 * assumed, C15); a cycle or an out-of-range wire -> TB_EINVAL. */
typedef struct {
    int64_t n_inputs;
    int64_t n_gates;
    const int32_t* type;
    const int64_t* in0;
    const int64_t* in1;
    const int64_t* in2;
} tb_netlist;

/* Algorithm 1 on the host: level_of_gate[g] = 1 + max(level of its inputs), inputs at level 0 -- the
 * iteration of the while loop in which g first enters C - finished.  Writes *n_levels. */
int tb_levelise(const tb_netlist* net, int64_t* level_of_gate, int64_t* n_levels);

/* Host-only execution plan (no device needed): *n_levels; level_off[L] for L = 0..n_levels = offset of the
 * first gate of level L+1 in level-sorted order (level_off[n_levels] = n_gates); row_of_wire[w] = the wire
 * array row of wire w (inputs first, then level 1's outputs, level 2's, ...; ascending gate index inside a
 * level).  Pass level_off = row_of_wire = NULL to query n_levels first.  This is the layout
 * tb_netlist_upload uses and the one the multi-GPU level loop shards (contiguous output rows per level). */
int tb_netlist_plan(const tb_netlist* net, int64_t* n_levels, int64_t* level_off, int64_t* row_of_wire);
/* tb_netlist_plan with the capacity-aware level schedule of tb_set_level_capacity (`lanes` > 0; 0 = Algorithm 1,
 * i.e. tb_netlist_plan).  Host only.  lanes < 0: TB_EINVAL. */
int tb_netlist_plan_capacity(const tb_netlist* net, int64_t lanes, int64_t* n_levels, int64_t* level_off,
                             int64_t* row_of_wire);

typedef struct tb_dev_netlist tb_dev_netlist;   /* library-owned device copy of a levelised netlist */

/* Levelise, renumber wires so that every level's outputs form one contiguous block of rows (inputs first,
 * then level 1, level 2, ...; within a level, gates in ascending original index), build the per-level
 * lane and gate descriptors and upload them.  *out receives the handle. */
int tb_netlist_upload(tb_ctx* ctx, const tb_netlist* net, tb_dev_netlist** out);
int tb_netlist_free(tb_ctx* ctx, tb_dev_netlist* dnet);
/* n_levels; n_rows = n_inputs + n_gates = rows a wire array must hold. */
int tb_netlist_info(const tb_dev_netlist* dnet, int64_t* n_levels, int64_t* n_rows);
/* row_of_wire[w] for every wire id w < n_inputs + n_gates (inputs map to themselves). */
int tb_netlist_wire_rows(const tb_dev_netlist* dnet, int64_t* row_of_wire);
/* first output row and number of gates (rows) of level `level` (1-based, 1..n_levels); also the number
 * of bootstrapped gates and of blind-rotation lanes (MUX = 2 lanes, NOT = 0) in it. */
int tb_netlist_level(const tb_dev_netlist* dnet, int64_t level, int64_t* row0, int64_t* n_gates,
                     int64_t* n_boot, int64_t* n_lanes);
/* Evaluate gates [g0, g1) of level `level` (indices within the level): reads input rows of `wires`,
 * writes rows row0+g0 .. row0+g1-1.  `wires` is a DEVICE array of n_rows rows of `stride` words.  Async. */
int tb_run_level(tb_ctx* ctx, const tb_dev_netlist* dnet, int64_t level, int64_t g0, int64_t g1,
                 uint32_t* wires, int64_t stride, tb_stream stream);
/* Fused all-gather for the multi-GPU level loop (the paper's per-level exchange of output
 * ciphertexts): after this call, the key-switch kernels of tb_run_level calls on the DEVICE array
 * `own_wires` store every output row not only there but, at the same row offset, into each of the n arrays
 * peer_wires[0..n-1] (HOST array of DEVICE pointers valid in this process: the other ranks' wire arrays,
 * opened with tb_ipc_import; same rows and stride).  Runs on any other wire array are unaffected.  The transfer rides on the key switch's own stores (NVLink
 * peer writes), so each level needs only a barrier across ranks instead of an all-gather.  n = 0 disables.
 * The caller keeps the peer mappings alive while set.  Errors: TB_EINVAL (n < 0, null pointers), TB_ECUDA. */
int tb_set_peer_wires(tb_ctx* ctx, const uint32_t* own_wires, uint32_t* const* peer_wires, int n);
#define TB_IPC_HANDLE_BYTES 64
/* CUDA IPC export of a device pointer: handle (TB_IPC_HANDLE_BYTES bytes, caller-owned) of the allocation
 * containing dev_ptr and dev_ptr's byte offset in it.  Errors: TB_EINVAL, TB_ECUDA. */
int tb_ipc_export(const void* dev_ptr, unsigned char* handle, int64_t* offset);
/* Open a handle exported by another process (on ctx's device): *base = the mapped allocation (pass it to
 * tb_ipc_close), *dev_ptr = *base + offset.  A process cannot open its own handle (TB_ECUDA). */
int tb_ipc_import(tb_ctx* ctx, const unsigned char* handle, int64_t offset, void** dev_ptr, void** base);
int tb_ipc_close(tb_ctx* ctx, void* base);
/* All levels in order on one device (single-GPU path).  Async. */
int tb_run_netlist(tb_ctx* ctx, const tb_dev_netlist* dnet, uint32_t* wires, int64_t stride, tb_stream stream);

/* End-to-end netlist evaluation through HOST buffers: copies the n_inputs input ciphertexts (rows of
 * in_stride words, host) into a context-owned device wire array, runs every level, and copies the rows of
 * the n_outputs wires listed in output_wires (original wire ids, host array) to host_outputs (rows of
 * out_stride >= 631 words).  The input copies run on their own stream in the order of the level that first reads
 * them (level L waits only for its inputs) and the outputs of level L are copied back while level L + 1 runs
 * (SURVEY 8(f) f1); a level of more than 8 waves of the throughput kernel (a wave = 4 x SM-count gates) runs as
 * three launches (3 waves, the middle, the last 3-4 waves) so that the copies overlap inside a wide level too.
 * Pinned host buffers make the copies asynchronous.  Synchronous, also on error (no copy
 * from / into the host buffers is in flight when it returns). */
int tb_run_netlist_host(tb_ctx* ctx, const tb_dev_netlist* dnet, const uint32_t* host_inputs, int64_t in_stride,
                        const int64_t* output_wires, int64_t n_outputs, uint32_t* host_outputs, int64_t out_stride);
/* tb_run_netlist_host: overlap the copies with the level loop (1, default) or run copy, levels, copy back one
 * after the other (0) -- for measuring the overlap. */
int tb_set_host_overlap(tb_ctx* ctx, int enable);

/* ---- per-kernel timing (CUDA events recorded around every launch on the launching stream) ---------- */
/* enable != 0 starts recording (and clears previous records); 0 stops. */
int tb_profile_enable(tb_ctx* ctx, int enable);
/* Synchronises the recorded events and returns the summed device time (ms) and launch counts of the
 * blind-rotation kernel and of the key-switch kernel since tb_profile_enable(ctx, 1). */
int tb_profile_read(tb_ctx* ctx, double* br_ms, int64_t* br_launches, double* ks_ms, int64_t* ks_launches);

/* ---- diagnostics used by the parity tests ---------------------------------------------------------- */
/* Blind rotation + extraction only: out[g] (N+1 words, rows `out_stride` apart) = Extract(BlindRotate(
 * ModSwitch(in[g]))) with test vector mu = 1/8 -- SURVEY 8(a) a2-a5 without the key switch.  Async. */
int tb_bootstrap_wo_ks(tb_ctx* ctx, const uint32_t* in, int64_t in_stride, uint32_t* out, int64_t out_stride,
                       int64_t count, tb_stream stream);
/* Key switch only: out[g] (n+1 words) = KS(in[g]) for extracted samples in[g] (N+1 words).  Async. */
int tb_keyswitch(tb_ctx* ctx, const uint32_t* in, int64_t in_stride, uint32_t* out, int64_t out_stride,
                 int64_t count, tb_stream stream);
/* Exact negacyclic product through the kernels' NTT (diagnostic): res[c] = sum over the 6 "rows" r of
 * (digits[r] (x) polys[r])[c] mod 2^32, digits in [-64, 63], polys u32 torus.  All DEVICE pointers:
 * digits [6][N] int32, polys [6][N] u32, res [N] u32.  Synchronous. */
int tb_ntt_muladd6(tb_ctx* ctx, const int32_t* digits, const uint32_t* polys, uint32_t* res);
/* Same product through the FP64-pipe transform (folded 512-point complex negacyclic FFT, 16-bit signed BK
 * halves, rounding to the nearest integer).  Synchronous. */
int tb_fft_muladd6(tb_ctx* ctx, const int32_t* digits, const uint32_t* polys, uint32_t* res);

/* Blind-rotation lanes per CTA for the default kernel: 1..4 fixed, or 0 (default) = auto per launch: 1 or 2,
 * whichever leaves the busiest SM the least work for that lane count. */
int tb_set_lanes_per_cta(tb_ctx* ctx, int lanes);
/* The lanes per CTA the default kernel uses for a launch of `nlanes` lanes (>= 1), or < 0 (TB_EINVAL). */
int tb_br6_lanes_per_cta(tb_ctx* ctx, int64_t nlanes);
/* Blind-rotation kernel: 6 = br6_kernel (default: 6 warps/lane, 2 CTAs/SM, BK words from L2), 10 = brf_kernel
 * (FP64-pipe FFT), 12 = brt_kernel (four-step NTT on the tcgen05 tensor cores, DESIGN.md
 * "Tensor-core NTT"), 14 = br6t_kernel (br6 with its forward NTTs on the tensor cores), 15 = brq_kernel (both
 * NTT directions on the tensor cores in br6's 2-CTA-per-SM shape).  All are bit-identical; see
 * DESIGN.md "Kernels".  Anything else: TB_EINVAL. */
int tb_set_br_variant(tb_ctx* ctx, int variant);
/* Latency mode for narrow levels: a launch with <= `lanes` bootstraps runs a latency-mode kernel (below)
 * instead of the throughput kernel.  Default = the device's SM count; 0 disables. */
int tb_set_narrow_lanes(tb_ctx* ctx, int64_t lanes);
/* Latency-mode kernel: 0 = auto (default: brl while the level's bootstraps fit in one wave of brl clusters, else
 * brl2), 11 = brl_kernel (one bootstrap per cluster of 4 SMs on the FP64 path: each SM owns one output polynomial
 * and one 16-bit BK half; 1.9 ms per level on B200, 32 per wave), 16 = brl2_kernel (one bootstrap per cluster of 2
 * SMs on the FP64 path: each SM owns one output polynomial and both BK halves, tb_brl2.cu; 2.1 ms, 74 per wave),
 * 9 = br9_kernel (one bootstrap per cluster of 2 SMs, integer NTT, forward-NTT rows exchanged through distributed
 * shared memory; 3.5 ms, 74 per wave), 13 = brtl_kernel (one bootstrap per SM on the tensor cores, tb_brtl.cu;
 * 4.7 ms, 148 per wave).  All are bit-identical.  Anything else: TB_EINVAL. */
int tb_set_narrow_kernel(tb_ctx* ctx, int kernel);
/* Level schedule used by tb_netlist_upload: Algorithm 1 gives every gate its earliest level;
 * with lanes > 0 gates that have slack are moved to later levels (never past their latest level, so the number
 * of levels is unchanged) to keep each level within `lanes` bootstraps (MUX = 2, NOT = 0) where possible: a
 * narrow level then fits one wave of the latency kernel.  -1 = auto (default; the number of brl clusters that
 * fit on the device, 32 on B200), 0 = Algorithm 1 as is.  Output bytes are identical either way (each gate's
 * result depends only on its inputs).  Affects netlists uploaded afterwards.  lanes < -1: TB_EINVAL. */
int tb_set_level_capacity(tb_ctx* ctx, int64_t lanes);
/* Level order of netlists uploaded afterwards, for a level loop over `world` ranks (P:263's
 * dependency-driven batching carried across GPUs): every level is cut into `world` contiguous chunks of
 * ceil(n / world) gates (rank r evaluates chunk r), and each chunk begins with the gates whose inputs from the
 * previous level were all produced by the same rank -- those can run before the previous level's exchange
 * barrier.  Output bytes do not depend on the order.  Default 1 (ascending gate index).  world < 1: TB_EINVAL. */
int tb_set_plan_world(tb_ctx* ctx, int world);
/* Host-only plan of tb_netlist_upload for `world` ranks and capacity `lanes` (0 = Algorithm 1): level offsets
 * [n_levels + 1], row of every wire, and early[(level - 1) * world + rank] (see tb_netlist_early).  Call with
 * null arrays to get n_levels first.  Bad arguments: TB_EINVAL. */
int tb_netlist_plan_world(const tb_netlist* net, int64_t lanes, int world, int64_t* n_levels, int64_t* level_off,
                          int64_t* row_of_wire, int64_t* early);
/* The world size a device netlist was planned for (tb_set_plan_world at upload time). */
int tb_netlist_world(const tb_dev_netlist* dnet, int* world);
/* Number of "early" gates at the start of rank `rank`'s chunk of `level` (1-based): gates whose inputs are in
 * levels < level - 1 or in the same rank's chunk of level - 1, so rank `rank` can evaluate them right after its
 * own part of level - 1, before that level's exchange.  Level 1: the whole chunk.  Out of range: TB_EINVAL. */
int tb_netlist_early(const tb_dev_netlist* dnet, int64_t level, int rank, int64_t* n_early);
/* Gates per key-switch CTA (8, 16 or 32; default 8): each tile streams the 62 MB KSK once from L2. */
int tb_set_ks_tile(tb_ctx* ctx, int gates);
/* Device bytes a context holds for keys: the torus BK, the BK domains built so far, the KSK. */
int tb_key_bytes(const tb_ctx* ctx, size_t* bytes);

/* Integer-pipe microbenchmark (roofline denominator): runs the kernels' own lazy
 * butterfly, register resident, on all SMs for `iters` iterations; returns butterflies/s and the 64-bit
 * multiply-accumulate rate (MAC/s) measured with CUDA events.  Synchronous. */
int tb_microbench(tb_ctx* ctx, int iters, double* butterflies_per_s, double* macs_per_s);
/* Field microbenchmark behind the NTT-field choice (R1; the north star proposed the 64-bit Goldilocks
 * prime): register-resident rates on all SMs, written to rates[0..3] = 30-bit Shoup butterflies/s (the kernels'
 * own), Goldilocks general-twiddle butterflies/s, Goldilocks shift-twiddle (x 2^s) butterflies/s, 64-bit
 * MACs/s.  Synchronous; iters <= 0 or null pointers: TB_EINVAL. */
int tb_microbench_fields(tb_ctx* ctx, int iters, double* rates);
/* Tensor-core external-product core (diagnostic): for four lanes g and both output polynomials q,
 * res[g][q][.] = sum_{r<6} digits[g][r] (x) polys[r][q] mod 2^32 (negacyclic), computed exactly as one CMux step
 * of the tensor-core blind rotation does it (four-step NTT on tcgen05 kind::i8, MAC against the NTT-domain BK,
 * inverse, centred lift).  Device pointers: digits int32 [2][6][1024] in [-64, 63],
 * polys u32 [6][2][1024] (one BK_i), res u32 [2][2][1024].  Synchronous. */
int tb_tc_muladd(tb_ctx* ctx, const int32_t* digits, const uint32_t* polys, uint32_t* res);
/* Tensor-core check (diagnostic): D[128][N] = A[128][K] . B[N][K]^T as integers through tcgen05.mma kind::i8
 * (device pointers; A bytes signed if a_signed else unsigned, likewise B; D s32), with the operand tiles laid
 * out in shared memory as K-major core matrices whose K-adjacent stride is `lbo` bytes (the layout of the
 * tensor-core NTT).  Synchronous.  K % 32, N % 16, K <= 256, N <= 256, lbo >= 128
 * and lbo % 16 == 0, else TB_EINVAL. */
int tb_tc_mma_test(tb_ctx* ctx, const uint8_t* A, const uint8_t* B, int K, int N, int a_signed, int b_signed,
                   int lbo, int32_t* D);

const char* tb_last_error(void);
const char* tb_version(void);

#ifdef __cplusplus
}
#endif
#endif
