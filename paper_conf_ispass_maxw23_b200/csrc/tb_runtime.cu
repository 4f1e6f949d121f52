// tb_runtime.cu -- the C ABI (include/tfhe_b200.h): contexts, key upload, batched gates, Algorithm-1
// levelisation and the level executor.  Host-side C++17; every arithmetic step of a gate runs in the
// kernels of tb_bootstrap.cu / tb_keyswitch.cu.  There is no CPU fallback: without a usable sm_100 device
// every entry point fails with an error status.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: ranges cost a branch unless a tool (nsys, ncu) is attached
#include "../../include/tfhe_b200.h"
#include "tb_kernels.cuh"

namespace {
// NVTX range over one C-ABI call (levels, gate batches, host-buffer netlists), so that a profiler timeline groups
// each call's kernels
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace


using namespace tb;

// ------------------------------------------------------------------------------------------ errors
static thread_local std::string g_err;
static int fail(int code, const char* msg) {
    g_err = msg;
    return code;
}
static int cuda_fail(cudaError_t e, const char* where) {
    g_err = std::string(where) + ": " + cudaGetErrorString(e);
    return TB_ECUDA;
}
#define TB_CUDA(call)                                            \
    do {                                                         \
        cudaError_t e_ = (call);                                 \
        if (e_ != cudaSuccess) return cuda_fail(e_, #call);      \
    } while (0)

extern "C" const char* tb_last_error(void) { return g_err.c_str(); }
extern "C" const char* tb_version(void) { return "tfhe_b200 0.1 (sm_100a; n=630 N=1024 l=3 Bgbit=7 t=8 base=4)"; }

// ------------------------------------------------------------------------------------------ field setup
static uint32_t mulmod(uint64_t a, uint64_t b) { return (uint32_t)((a * b) % kP); }
static uint32_t powmod(uint64_t b, uint64_t e) {
    uint64_t r = 1;
    b %= kP;
    while (e) {
        if (e & 1) r = r * b % kP;
        b = b * b % kP;
        e >>= 1;
    }
    return (uint32_t)r;
}
static uint32_t shoup_of(uint32_t w) { return (uint32_t)(((uint64_t)w << 32) / kP); }
static uint32_t brv10(uint32_t k) {
    uint32_t r = 0;
    for (int b = 0; b < 10; b++) r |= ((k >> b) & 1u) << (9 - b);
    return r;
}

struct tb_ctx {
    int device = 0;
    int lanes_per_cta = 0;                  // br6 lanes per CTA (1..4), 0 = auto by wave quantisation (br6_lanes)
    int sms = 0;                            // SM count (queried on first use)
    int variant = 6;                        // blind-rotation kernel: 6 = br6, 10 = brf (FP64 pipe)
    int ks_tile = 8;                        // gates per key-switch CTA (8, 16, 32); 8 measured fastest
    int narrow_lanes = 0;                   // launches with <= this many lanes run in latency mode (= SM count)
    int narrow_kernel = 0;                  // latency-mode kernel: 9 = br9 (2-SM cluster per lane), 11 = brl
                                            // (4-SM cluster per lane, FP64 path), 13 = brtl (one SM per lane,
                                            // tensor cores), 16 = brl2 (2-SM cluster per lane, FP64 path),
                                            // 0 = auto: brl while the lanes fit one wave of its clusters, else brl2
    int brl_wave = -2;                      // co-resident brl clusters (queried on first use)
    int plan_world = 1;                     // netlist upload: order each level for this many ranks (early gates first)
    int64_t level_capacity = -1;            // netlist upload: re-levelise to <= this many lanes per level where
                                            // slack allows (0 = Algorithm 1 as is, -1 = auto: brl_wave)
    cudaStream_t own = nullptr;             // internal stream for load / host-buffer calls
    cudaStream_t h2d = nullptr, d2h = nullptr;   // tb_run_netlist_host copy streams (overlap with the levels)
    std::vector<cudaEvent_t> hev;           // tb_run_netlist_host events (per level: inputs landed, outputs ready)
    int overlap_host = 1;                   // tb_run_netlist_host: overlap copies with the level loop
    uint2* twF = nullptr;                   // [31][32]
    uint2* twI = nullptr;
    double2* fftB = nullptr;                // FP64 FFT per-lane twiddles: stages 5-8 [15][32], stage 9 [8][32]
    double2* fftC = nullptr;
    double2* fftL = nullptr;                // brl: [64][6] per-thread pass-2/3 twiddle bases
    uint32_t ninv = 0, ninvp = 0;
    unsigned char* tcB = nullptr;           // tensor-core NTT: constant B operands (tb_brt.cu)
    uint2* tcTw = nullptr;                  // [2][32][32] four-step twiddles (+ Shoup)
    uint2* tcPts = nullptr;                 // [N] psi^(2j+1) (+ Shoup): evaluation points of bk4
    uint32_t* bk4 = nullptr;                // [n][N][36] NTT-domain BK in the four-step order (brt_kernel)
    uint32_t* bkhat = nullptr;              // [n][6][6][N]
    double2* bkf = nullptr;                 // FP64 variant: [n][6][4][512] complex, scaled by 1/512
    uint32_t* ksk = nullptr;                // [N][t][3][632]
    bool have_bk = false, have_ksk = false;
    uint32_t* bk_raw = nullptr;             // the torus BK as loaded (31 MB): source of every domain built later
    unsigned domains = 0;                   // BK domains built from bk_raw (kDomNtt | kDomFft | kDomBk4)
    // scratch (grown on demand; growing synchronises the device)
    uint32_t* lanebuf = nullptr;
    int64_t lanebuf_rows = 0;
    LaneDesc* ldesc = nullptr;
    GateDesc* gdesc = nullptr;
    int64_t desc_rows = 0;
    uint32_t* stage = nullptr;              // tb_gates_host staging
    size_t stage_words = 0;
    uint32_t* hwires = nullptr;             // tb_run_netlist_host device wire array
    size_t hwires_words = 0;
    uint32_t** peers = nullptr;             // fused all-gather: device array of the other ranks' wire bases
    int32_t npeers = 0;
    const uint32_t* peer_own = nullptr;     // the local wire array the peers mirror (other arrays: no peer stores)
    uint32_t* ks_scratch = nullptr;         // split key-switch partial sums (narrow levels)
    size_t ks_scratch_words = 0;
    // per-kernel event timing (tb_profile_*)
    bool prof = false;
    std::vector<cudaEvent_t> ev_pool;
    size_t ev_used = 0;
    std::vector<std::pair<int, size_t>> ev_rec;   // (kind 0 = br / 1 = ks, index of start event)
};

static cudaEvent_t next_event(tb_ctx* c) {
    if (c->ev_used == c->ev_pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        c->ev_pool.push_back(e);
    }
    return c->ev_pool[c->ev_used++];
}
// record a start event before a launch of `kind`; returns the record slot or -1
static long prof_begin(tb_ctx* c, int kind, cudaStream_t st) {
    if (!c->prof) return -1;
    cudaEvent_t a = next_event(c), b = next_event(c);
    if (!a || !b) return -1;
    cudaEventRecord(a, st);
    c->ev_rec.push_back({kind, c->ev_used - 2});
    return (long)c->ev_rec.size() - 1;
}
static void prof_end(tb_ctx* c, long slot, cudaStream_t st) {
    if (slot < 0) return;
    cudaEventRecord(c->ev_pool[c->ev_rec[slot].second + 1], st);
}

struct tb_dev_netlist {
    int64_t n_inputs = 0, n_gates = 0, n_levels = 0;
    std::vector<int64_t> level_off;         // [n_levels + 1] gate offsets (level-sorted order)
    std::vector<int64_t> lane_off;          // [n_gates + 1] lane prefix over level-sorted gates
    std::vector<int64_t> boot_prefix;       // [n_gates + 1] bootstrapped gates (non-NOT) prefix
    std::vector<int64_t> row_of_wire;       // [n_inputs + n_gates]
    int world = 1;                          // ranks the level order was planned for
    std::vector<int64_t> in_level;          // [n_inputs] first level that reads the input (n_levels + 1: none)
    std::vector<int64_t> in_first;          // [n_inputs] first level-sorted gate position reading it (n_gates: none)
    std::vector<int64_t> early;             // [n_levels][world]: gates at the start of rank r's chunk of a level
                                            // whose inputs are local once r has run its part of the level before
    LaneDesc* ldesc = nullptr;
    GateDesc* gdesc = nullptr;
};

static int grow_lanes(tb_ctx* c, int64_t rows) {
    if (rows <= c->lanebuf_rows) return TB_OK;
    int64_t want = std::max<int64_t>(rows, c->lanebuf_rows * 3 / 2);
    if (c->lanebuf) cudaFree(c->lanebuf);
    c->lanebuf = nullptr;
    c->lanebuf_rows = 0;
    if (cudaMalloc(&c->lanebuf, (size_t)want * kLaneStride * 4) != cudaSuccess) {
        cudaGetLastError();
        return fail(TB_ENOMEM, "lane buffer allocation failed");
    }
    c->lanebuf_rows = want;
    return TB_OK;
}
static int grow_desc(tb_ctx* c, int64_t rows) {
    if (rows <= c->desc_rows) return TB_OK;
    int64_t want = std::max<int64_t>(rows, c->desc_rows * 3 / 2);
    if (c->ldesc) cudaFree(c->ldesc);
    if (c->gdesc) cudaFree(c->gdesc);
    c->ldesc = nullptr;
    c->gdesc = nullptr;
    c->desc_rows = 0;
    if (cudaMalloc(&c->ldesc, (size_t)want * 2 * sizeof(LaneDesc)) != cudaSuccess ||
        cudaMalloc(&c->gdesc, (size_t)want * sizeof(GateDesc)) != cudaSuccess) {
        cudaGetLastError();
        return fail(TB_ENOMEM, "descriptor allocation failed");
    }
    c->desc_rows = want;
    return TB_OK;
}

extern "C" tb_params tb_default_params(void) {
    tb_params p;
    p.n = kn; p.N = kN; p.k = 1; p.l = kL; p.Bgbit = kBgbit; p.ks_t = kKsT; p.ks_basebit = kKsBasebit;
    return p;
}

extern "C" int tb_ctx_create(const tb_params* P, int dev, tb_ctx** out) {
    if (!P || !out) return fail(TB_EINVAL, "null argument");
    *out = nullptr;
    if (P->n != kn || P->N != kN || P->k != 1 || P->l != kL || P->Bgbit != kBgbit || P->ks_t != kKsT ||
        P->ks_basebit != kKsBasebit)
        return fail(TB_EUNSUPPORTED, "only n=630 N=1024 k=1 l=3 Bgbit=7 ks_t=8 ks_basebit=2 is compiled");
    int ndev = 0;
    TB_CUDA(cudaGetDeviceCount(&ndev));
    if (dev < 0 || dev >= ndev) return fail(TB_EINVAL, "bad device index");
    cudaDeviceProp prop;
    TB_CUDA(cudaGetDeviceProperties(&prop, dev));
    if (prop.major != 10 || prop.minor != 0) return fail(TB_EUNSUPPORTED, "device is not sm_100 (B200)");
    TB_CUDA(cudaSetDevice(dev));
    tb_ctx* c = new (std::nothrow) tb_ctx();
    if (!c) return fail(TB_ENOMEM, "host allocation failed");
    c->device = dev;
    c->narrow_lanes = prop.multiProcessorCount;

    // psi: primitive 2N-th root of unity mod p (psi^N = -1)
    uint32_t psi = 0;
    for (uint32_t g = 2; g < 1000 && !psi; g++) {
        uint32_t cand = powmod(g, (kP - 1) / kTwoN);
        if (powmod(cand, kN) == kP - 1) psi = cand;
    }
    const uint32_t psi_inv = powmod(psi, kP - 2);
    uint32_t fw[32] = {0}, fwp[32] = {0}, iw[32] = {0}, iwp[32] = {0}, misc[4] = {0};
    for (uint32_t k = 1; k < 32; k++) {
        fw[k] = powmod(psi, brv10(k));
        iw[k] = powmod(psi_inv, brv10(k));
        fwp[k] = shoup_of(fw[k]);
        iwp[k] = shoup_of(iw[k]);
    }
    misc[0] = (uint32_t)((1ull << 32) % kP);
    misc[1] = shoup_of(misc[0]);
    misc[2] = kTwoP;
    misc[3] = kDecompOffset;
    std::vector<uint2> tf(31 * 32), ti(31 * 32);
    for (int s = 5; s < 10; s++)
        for (int bj = 0; bj < (1 << (s - 5)); bj++)
            for (int t = 0; t < 32; t++) {
                const uint32_t k = (1u << s) + (uint32_t)t * (1u << (s - 5)) + bj;
                const int e = (1 << (s - 5)) - 1 + bj;
                const uint32_t w = powmod(psi, brv10(k)), wi = powmod(psi_inv, brv10(k));
                tf[e * 32 + t] = make_uint2(w, shoup_of(w));
                ti[e * 32 + t] = make_uint2(wi, shoup_of(wi));
            }
    // FP64 FFT variant: psi = e^{i pi / 1024}; zeta_{s,b} = psi^brv10(2^s + b) (tb_fft.cuh), from long double
    std::vector<double2> zeta16(16), fb(kTwB), fc(kTwC);
    auto cpsi = [](uint32_t e) {
        const long double a = 3.14159265358979323846264338327950288L * (long double)e / 1024.0L;
        return make_double2((double)cosl(a), (double)sinl(a));
    };
    for (int s = 1; s <= 4; s++)
        for (int b = 0; b < (1 << (s - 1)); b++) zeta16[(1 << (s - 1)) - 1 + b] = cpsi(brv10((1u << s) + b));
    for (int s = 5; s <= 8; s++)
        for (int u = 0; u < 16; u++) fb[(s - 5) * 16 + u] = cpsi(brv10((1u << s) + (uint32_t)u * (1u << (s - 5))));
    for (int t = 0; t < 32; t++) fc[t] = cpsi(brv10(512u + (uint32_t)t * 8u));
    std::vector<double2> fl(64 * 6);       // brl pass bases (tb_brl.cu): zeta_{s,b} = psi^brv10(2^s + b)
    for (int t = 0; t < 64; t++) {
        const uint32_t T = (uint32_t)t >> 3;
        fl[t * 6 + 0] = cpsi(brv10(16u + T));
        fl[t * 6 + 1] = cpsi(brv10(32u + 2 * T));
        fl[t * 6 + 2] = cpsi(brv10(64u + 4 * T));
        fl[t * 6 + 3] = cpsi(brv10(128u + (uint32_t)t));
        fl[t * 6 + 4] = cpsi(brv10(256u + 2 * (uint32_t)t));
        fl[t * 6 + 5] = cpsi(brv10(512u + 4 * (uint32_t)t));
    }
    c->ninv = powmod(kN, kP - 2);
    c->ninvp = shoup_of(c->ninv);
    std::vector<unsigned char> tcb(brt_table_bytes());
    std::vector<uint2> tctw(2048), tcpts(kN);
    brt_tables(psi, tcb.data(), tctw.data(), tcpts.data());
    int rc = set_ntt_constants(fw, fwp, iw, iwp, misc);
    if (rc == 0) rc = set_fft_constants(zeta16.data());
    cudaError_t e = cudaSuccess;
    if (rc == 0) e = cudaMalloc(&c->fftB, fb.size() * sizeof(double2));
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->fftC, fc.size() * sizeof(double2));
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->fftB, fb.data(), fb.size() * sizeof(double2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->fftC, fc.data(), fc.size() * sizeof(double2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->fftL, fl.size() * sizeof(double2));
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->fftL, fl.data(), fl.size() * sizeof(double2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->tcB, tcb.size());
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->tcB, tcb.data(), tcb.size(), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->tcTw, tctw.size() * sizeof(uint2));
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->tcTw, tctw.data(), tctw.size() * sizeof(uint2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->tcPts, tcpts.size() * sizeof(uint2));
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->tcPts, tcpts.data(), tcpts.size() * sizeof(uint2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->own, cudaStreamNonBlocking);
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->twF, 31 * 32 * sizeof(uint2));
    if (rc == 0 && e == cudaSuccess) e = cudaMalloc(&c->twI, 31 * 32 * sizeof(uint2));
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->twF, tf.data(), tf.size() * sizeof(uint2), cudaMemcpyHostToDevice);
    if (rc == 0 && e == cudaSuccess) e = cudaMemcpy(c->twI, ti.data(), ti.size() * sizeof(uint2), cudaMemcpyHostToDevice);
    if (rc != 0 || e != cudaSuccess) {
        tb_ctx_destroy(c);
        return e != cudaSuccess ? cuda_fail(e, "tb_ctx_create") : fail(TB_ECUDA, "constant upload failed");
    }
    *out = c;
    return TB_OK;
}

extern "C" int tb_ctx_destroy(tb_ctx* c) {
    if (!c) return TB_OK;
    cudaSetDevice(c->device);
    cudaFree(c->twF);
    cudaFree(c->twI);
    cudaFree(c->fftB);
    cudaFree(c->fftC);
    cudaFree(c->fftL);
    cudaFree(c->bkhat);
    cudaFree(c->bk_raw);
    cudaFree(c->bk4);
    cudaFree(c->tcB);
    cudaFree(c->tcTw);
    cudaFree(c->tcPts);
    cudaFree(c->bkf);
    cudaFree(c->ksk);
    cudaFree(c->lanebuf);
    cudaFree(c->ldesc);
    cudaFree(c->gdesc);
    cudaFree(c->stage);
    cudaFree(c->hwires);
    cudaFree(c->ks_scratch);
    cudaFree(c->peers);
    for (cudaEvent_t e : c->ev_pool) cudaEventDestroy(e);
    if (c->own) cudaStreamDestroy(c->own);
    if (c->h2d) cudaStreamDestroy(c->h2d);
    if (c->d2h) cudaStreamDestroy(c->d2h);
    for (cudaEvent_t e : c->hev) cudaEventDestroy(e);
    delete c;
    return TB_OK;
}

// Lanes per br6 CTA for a launch of `nlanes` lanes.  Fixed if set; auto picks 1 or 2 from the busiest SM's
// lane count.  This is a CALIBRATION, not a model: the per-lane-slot times below were measured on a 148-SM
// B200 by tools/lanes_sweep.sh (profiles/r01f_lanes_sweep.txt: 592 / 1024 / 1536 / 2048 lanes x G = 1..4) and
// must be re-measured whenever br6_kernel changes.  G = 2 runs 2 CTAs (4 lanes) per SM at kBr6SlotG2 per
// lane-slot, G = 1 runs 4 CTAs per SM at kBr6SlotG1.  A full wave favours G = 2 by 6 %, but G = 1 schedules the
// ragged last wave lane by lane instead of pair by pair (1,024 lanes: 20.5 vs 21.9 ms).
constexpr int64_t kBr6SlotG1 = 296;   // ms x 100 per 630-step lane slot, G = 1 (4 CTAs/SM)
constexpr int64_t kBr6SlotG2 = 279;   // ms x 100 per lane slot, G = 2 (2 CTAs/SM)
static int br6_lanes(tb_ctx* c, int64_t nlanes) {
    if (c->lanes_per_cta > 0) return c->lanes_per_cta;
    if (c->sms == 0 && cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, c->device) != cudaSuccess)
        c->sms = 148;
    const int64_t s = c->sms;
    const int64_t t1 = kBr6SlotG1 * ((nlanes + s - 1) / s);              // busiest SM: lanes x slot time
    const int64_t t2 = 2 * kBr6SlotG2 * ((nlanes + 2 * s - 1) / (2 * s)); // busiest SM: 2 x CTAs x slot time
    return t1 < t2 ? 1 : 2;
}

extern "C" int tb_br6_lanes_per_cta(tb_ctx* c, int64_t nlanes) {
    if (!c || nlanes < 0) return fail(TB_EINVAL, "null context or negative lane count");
    return br6_lanes(c, nlanes);
}

extern "C" int tb_set_lanes_per_cta(tb_ctx* c, int lanes) {
    if (!c || lanes < 0 || lanes > 4) return fail(TB_EINVAL, "lanes per CTA must be 0 (auto) or 1..4");
    c->lanes_per_cta = lanes;
    return TB_OK;
}

// ---- BK domains: only those the selected kernels read are built (from the loaded torus BK) ----------------
enum : unsigned { kDomNtt = 1, kDomFft = 2, kDomBk4 = 4 };
static unsigned needed_domains(const tb_ctx* c) {
    unsigned m = c->variant == 10 ? kDomFft : ((c->variant == 12 || c->variant == 15) ? kDomBk4 : kDomNtt);
    if (c->narrow_lanes > 0) {                         // latency mode: brl (FFT domain) and / or br9 (NTT domain)
        if (c->narrow_kernel == 9) m |= kDomNtt;
        else if (c->narrow_kernel == 11) m |= kDomFft;
        else if (c->narrow_kernel == 13) m |= kDomBk4;
        else if (c->narrow_kernel == 16) m |= kDomFft;
        else m |= kDomFft;                             // auto: brl or brl2 by the level's width
    }
    return m;
}
static int build_domains(tb_ctx* c) {
    if (!c->have_bk) return TB_OK;
    const unsigned miss = needed_domains(c) & ~c->domains;
    if (!miss) return TB_OK;
    TB_CUDA(cudaSetDevice(c->device));
    if ((miss & kDomNtt) && !c->bkhat) TB_CUDA(cudaMalloc(&c->bkhat, (size_t)kn * kRows * kOuts * kN * 4));
    if ((miss & kDomFft) && !c->bkf) TB_CUDA(cudaMalloc(&c->bkf, bkf_bytes()));
    if ((miss & kDomBk4) && !c->bk4) TB_CUDA(cudaMalloc(&c->bk4, bk4_bytes()));
    if (miss & kDomNtt) launch_bk_to_ntt(c->bk_raw, c->bkhat, c->twF, c->ninv, c->ninvp, c->own);
    if (miss & kDomFft) launch_bk_to_fft(c->bk_raw, c->bkf, c->fftB, c->fftC, c->own);
    if (miss & kDomBk4) launch_bk_to_bk4(c->bk_raw, c->bk4, c->tcPts, c->ninv, c->ninvp, kn, c->own);
    TB_CUDA(cudaGetLastError());
    TB_CUDA(cudaStreamSynchronize(c->own));
    c->domains |= miss;
    return TB_OK;
}

extern "C" int tb_set_br_variant(tb_ctx* c, int variant) {
    if (!c || !(variant == 6 || variant == 10 || variant == 12 || variant == 14 || variant == 15))
        return fail(TB_EINVAL, "blind-rotation variant must be 6, 10, 12, 14 or 15");
    c->variant = variant;
    return build_domains(c);
}

extern "C" int tb_set_narrow_kernel(tb_ctx* c, int kernel) {
    if (!c || (kernel != 0 && kernel != 9 && kernel != 11 && kernel != 13 && kernel != 16))
        return fail(TB_EINVAL, "latency-mode kernel must be 0 (auto), 9, 11, 13 or 16");
    c->narrow_kernel = kernel;
    return build_domains(c);
}

extern "C" int tb_set_level_capacity(tb_ctx* c, int64_t lanes) {
    if (!c || lanes < -1) return fail(TB_EINVAL, "level capacity must be -1 (auto), 0 (off) or > 0");
    c->level_capacity = lanes;
    return TB_OK;
}

extern "C" int tb_set_narrow_lanes(tb_ctx* c, int64_t lanes) {
    if (!c || lanes < 0) return fail(TB_EINVAL, "narrow-level threshold must be >= 0");
    c->narrow_lanes = lanes;
    return build_domains(c);
}

extern "C" int tb_set_plan_world(tb_ctx* c, int world) {
    if (!c || world < 1 || world > 1024) return fail(TB_EINVAL, "world size must be 1..1024");
    c->plan_world = world;
    return TB_OK;
}

extern "C" int tb_netlist_early(const tb_dev_netlist* d, int64_t level, int rank, int64_t* n_early) {
    if (!d || !n_early) return fail(TB_EINVAL, "null argument");
    if (level < 1 || level > d->n_levels) return fail(TB_EINVAL, "level out of range");
    if (rank < 0 || rank >= d->world) return fail(TB_EINVAL, "rank outside the world size the netlist was planned for");
    *n_early = d->early[(size_t)(level - 1) * d->world + rank];
    return TB_OK;
}

extern "C" int tb_netlist_world(const tb_dev_netlist* d, int* world) {
    if (!d || !world) return fail(TB_EINVAL, "null argument");
    *world = d->world;
    return TB_OK;
}

extern "C" int tb_set_ks_tile(tb_ctx* c, int gates) {
    if (!c || (gates != 8 && gates != 16 && gates != 32)) return fail(TB_EINVAL, "key-switch tile must be 8, 16 or 32");
    c->ks_tile = gates;
    return TB_OK;
}

extern "C" int tb_key_bytes(const tb_ctx* c, size_t* bytes) {
    if (!c || !bytes) return fail(TB_EINVAL, "null argument");
    *bytes = (c->have_bk ? (size_t)kn * kRows * 2 * kN * 4 : 0) +                       // torus BK (source)
             ((c->domains & kDomNtt) ? (size_t)kn * kRows * kOuts * kN * 4 : 0) +
             ((c->domains & kDomFft) ? bkf_bytes() : 0) + ((c->domains & kDomBk4) ? bk4_bytes() : 0) +
             (c->have_ksk ? (size_t)kN * kKsT * (kKsBase - 1) * kKsRow * 4 : 0);
    return TB_OK;
}

extern "C" int tb_load_bk(tb_ctx* c, const uint32_t* host_bk, size_t n_words) {
    if (!c || !host_bk) return fail(TB_EINVAL, "null argument");
    const size_t want = (size_t)kn * kRows * 2 * kN;
    if (n_words != want) return fail(TB_EINVAL, "bootstrapping key must have n*2l*2*N words");
    TB_CUDA(cudaSetDevice(c->device));
    if (!c->bk_raw) TB_CUDA(cudaMalloc(&c->bk_raw, want * 4));
    TB_CUDA(cudaMemcpyAsync(c->bk_raw, host_bk, want * 4, cudaMemcpyHostToDevice, c->own));
    TB_CUDA(cudaStreamSynchronize(c->own));
    c->have_bk = true;
    c->domains = 0;                                  // a new key: every domain is rebuilt from it
    return build_domains(c);
}

extern "C" int tb_load_ksk(tb_ctx* c, const uint32_t* host_ksk, size_t n_words) {
    if (!c || !host_ksk) return fail(TB_EINVAL, "null argument");
    const size_t want = (size_t)kN * kKsT * kKsBase * (kn + 1);
    if (n_words != want) return fail(TB_EINVAL, "key-switching key must have N*t*base*(n+1) words");
    TB_CUDA(cudaSetDevice(c->device));
    if (!c->ksk) TB_CUDA(cudaMalloc(&c->ksk, (size_t)kN * kKsT * (kKsBase - 1) * kKsRow * 4));
    uint32_t* tmp = nullptr;
    TB_CUDA(cudaMalloc(&tmp, want * 4));
    cudaError_t e = cudaMemcpyAsync(tmp, host_ksk, want * 4, cudaMemcpyHostToDevice, c->own);
    if (e == cudaSuccess) {
        launch_ksk_relayout(tmp, c->ksk, c->own);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->own);
    cudaFree(tmp);
    if (e != cudaSuccess) return cuda_fail(e, "tb_load_ksk");
    c->have_ksk = true;
    return TB_OK;
}

// ------------------------------------------------------------------------------------------ gates
// (C_g, w_a, w_b) per two-input gate: tfhe-lib's bootstrapped gates (EXT[10]; SURVEY 8(c) gate table)
static bool gate_linear(int gate, uint32_t* C, int32_t* wa, int32_t* wb) {
    const uint32_t e8 = kMu, e4 = 2u * kMu;
    switch (gate) {
        case TB_NAND:  *C = e8;      *wa = -1; *wb = -1; return true;
        case TB_AND:   *C = 0u - e8; *wa = 1;  *wb = 1;  return true;
        case TB_OR:    *C = e8;      *wa = 1;  *wb = 1;  return true;
        case TB_NOR:   *C = 0u - e8; *wa = -1; *wb = -1; return true;
        case TB_XOR:   *C = e4;      *wa = 2;  *wb = 2;  return true;
        case TB_XNOR:  *C = 0u - e4; *wa = -2; *wb = -2; return true;
        case TB_ANDNY: *C = 0u - e8; *wa = -1; *wb = 1;  return true;
        case TB_ANDYN: *C = 0u - e8; *wa = 1;  *wb = -1; return true;
        case TB_ORNY:  *C = e8;      *wa = -1; *wb = 1;  return true;
        case TB_ORYN:  *C = e8;      *wa = 1;  *wb = -1; return true;
        default: return false;
    }
}
static bool gate_known(int g) {
    uint32_t C; int32_t a, b;
    return g == TB_NOT || g == TB_MUX || gate_linear(g, &C, &a, &b);
}

static int check_ready(tb_ctx* c) {
    if (!c) return fail(TB_EINVAL, "null context");
    if (!c->have_bk || !c->have_ksk) return fail(TB_ENOKEYS, "load the bootstrapping and key-switching keys first");
    return TB_OK;
}

static int run_br(tb_ctx* c, const uint32_t* s0, const uint32_t* s1, const uint32_t* s2, int64_t sstride,
                  const LaneDesc* lanes, int64_t nlanes, uint32_t* out, int64_t ostride, cudaStream_t st) {
    if (nlanes <= 0) return TB_OK;
    BrArgs A;
    A.src0 = s0; A.src1 = s1; A.src2 = s2; A.src_stride = sstride;
    A.lanes = lanes; A.nlanes = (int32_t)nlanes; A.bkhat = c->bkhat; A.twF = c->twF; A.twI = c->twI;
    A.out = out; A.out_stride = ostride;
    const long slot = prof_begin(c, 0, st);
    int rc;
    int nk = c->narrow_kernel;
    if (nk == 0) {   // auto (profiles/r02l2_latency.jsonl): brl while the lanes fit its 32 four-SM clusters
                     // (1.9-2.0 ms), beyond that brl2 on SM pairs (2.1 ms up to 74 lanes, 4.2 ms up to 148; br9 was
                     // 3.5 / 7.1 ms there and brtl 4.7 ms)
        if (c->brl_wave == -2) c->brl_wave = brl_wave_lanes();
        nk = nlanes <= c->brl_wave ? 11 : 16;
    }
    if (c->narrow_lanes > 0 && nlanes <= c->narrow_lanes)
        rc = nk == 9    ? launch_br9(A, st)                    // narrow level: one lane per 2-SM cluster
             : nk == 16 ? launch_brl2(A, c->bkf, c->fftL, st)  // or per 2-SM cluster (FP64)
             : nk == 13 ? launch_brtl(A, c->bk4, c->tcB, c->tcTw, st)   // or per SM on the tensor cores
                        : launch_brl(A, c->bkf, c->fftL, st);  // or per 4-SM cluster (FP64)
    else if (c->variant == 12)
        rc = launch_brt(A, c->bk4, c->tcB, c->tcTw, st);
    else if (c->variant == 14)
        rc = launch_br6t(A, c->tcB, c->tcTw, st);
    else if (c->variant == 15)
        rc = launch_brq(A, c->bk4, c->tcB, c->tcTw, st);
    else if (c->variant == 10)
        rc = launch_brf(A, c->lanes_per_cta ? std::min(c->lanes_per_cta, 3) : 2, c->bkf, c->fftB, c->fftC, st);
    else
        rc = launch_br6(A, br6_lanes(c, nlanes), st);
    prof_end(c, slot, st);
    if (rc) return fail(TB_ECUDA, "blind-rotation kernel attribute/launch failed");
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "br_kernel launch");
    return TB_OK;
}
static int run_ks(tb_ctx* c, const uint32_t* lanes, int64_t lane_base, int64_t lane_stride, const GateDesc* gates,
                  int64_t ngates, uint32_t* out, int64_t ostride, const uint32_t* not_src, int64_t not_stride,
                  cudaStream_t st, uint32_t* const* peers = nullptr, int32_t npeers = 0) {
    if (ngates <= 0) return TB_OK;
    KsArgs A;
    A.lanes = lanes; A.lane_base = (int32_t)lane_base; A.lane_stride = lane_stride; A.gates = gates;
    A.ngates = (int32_t)ngates; A.ksk = c->ksk; A.out = out; A.out_stride = ostride; A.not_src = not_src;
    A.not_stride = not_stride;
    A.peers = peers;
    A.npeers = npeers;
    const bool split = c->narrow_lanes > 0 && ngates <= c->narrow_lanes;   // narrow level: split each gate's KS
    // mid-size level: tiles sliced over the input coefficients so that the launch still fills the GPU
    const int slices = split ? 1 : ks_tile_slices(ngates, c->ks_tile);
    // the split launch writes ngates x ks_split_count(ngates) partial rows (the slice count falls as ngates grows)
    const size_t need = split ? ks_split_scratch_words(ngates)
                              : (slices > 1 ? (size_t)ngates * slices * kKsRow : 0);
    if (need > c->ks_scratch_words) {
        cudaFree(c->ks_scratch);
        c->ks_scratch = nullptr;
        c->ks_scratch_words = 0;
        if (cudaMalloc(&c->ks_scratch, need * 4) != cudaSuccess) {
            cudaGetLastError();
            return fail(TB_ENOMEM, "key-switch scratch allocation failed");
        }
        c->ks_scratch_words = need;
    }
    const long slot = prof_begin(c, 1, st);
    const int rc = split ? launch_ks_split(A, c->ks_scratch, st) : launch_ks(A, c->ks_tile, c->ks_scratch, slices, st);
    prof_end(c, slot, st);
    if (rc) return fail(TB_ECUDA, "key-switch kernel attribute/launch failed");
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "ks_kernel launch");
    return TB_OK;
}

extern "C" int tb_gates(tb_ctx* c, int gate, const uint32_t* ca, const uint32_t* cb, const uint32_t* cc,
                        uint32_t* out, int64_t count, int64_t stride, tb_stream stream) {
    NvtxRange nv("tb_gates");
    int rc = check_ready(c);
    if (rc) return rc;
    if (count < 0 || stride < kn + 1 || count > ((int64_t)1 << 29)) return fail(TB_EINVAL, "bad count or stride");
    if (!gate_known(gate)) return fail(TB_EINVAL, "unknown gate code");
    if (count == 0) return TB_OK;
    if (!ca || !out || (gate != TB_NOT && !cb) || (gate == TB_MUX && !cc)) return fail(TB_EINVAL, "null array");
    TB_CUDA(cudaSetDevice(c->device));
    cudaStream_t st = (cudaStream_t)stream;
    const int64_t nl = gate == TB_MUX ? 2 * count : (gate == TB_NOT ? 0 : count);
    if ((rc = grow_desc(c, count))) return rc;
    if ((rc = grow_lanes(c, std::max<int64_t>(nl, 1)))) return rc;
    uint32_t C = 0; int32_t wa = 0, wb = 0;
    gate_linear(gate, &C, &wa, &wb);
    const int kind = gate == TB_NOT ? kGateNot : (gate == TB_MUX ? kGateMux : kGateBoot);
    launch_build_gate_desc(kind, wa, wb, C, count, c->ldesc, c->gdesc, st);
    if ((rc = run_br(c, ca, cb, cc, stride, c->ldesc, nl, c->lanebuf, kLaneStride, st))) return rc;
    return run_ks(c, c->lanebuf, 0, kLaneStride, c->gdesc, count, out, stride, ca, stride, st);
}

static int gates_host_impl(tb_ctx* c, int gate, const uint32_t* hca, const uint32_t* hcb, const uint32_t* hcc,
                           uint32_t* hout, int64_t count, int64_t stride);
extern "C" int tb_gates_host(tb_ctx* c, int gate, const uint32_t* hca, const uint32_t* hcb, const uint32_t* hcc,
                             uint32_t* hout, int64_t count, int64_t stride) {
    const int rc = gates_host_impl(c, gate, hca, hcb, hcc, hout, count, stride);
    if (rc != TB_OK && c && c->own) {   // no copy from / into the caller's host buffers may still be in flight
        cudaStreamSynchronize(c->own);
        cudaGetLastError();
    }
    return rc;
}
static int gates_host_impl(tb_ctx* c, int gate, const uint32_t* hca, const uint32_t* hcb, const uint32_t* hcc,
                           uint32_t* hout, int64_t count, int64_t stride) {
    int rc = check_ready(c);
    if (rc) return rc;
    if (count < 0 || stride < kn + 1) return fail(TB_EINVAL, "bad count or stride");
    if (!gate_known(gate)) return fail(TB_EINVAL, "unknown gate code");
    if (count == 0) return TB_OK;
    if (!hca || !hout || (gate != TB_NOT && !hcb) || (gate == TB_MUX && !hcc)) return fail(TB_EINVAL, "null array");
    TB_CUDA(cudaSetDevice(c->device));
    const size_t words = (size_t)count * stride;
    if (c->stage_words < 4 * words) {
        cudaFree(c->stage);
        c->stage = nullptr;
        c->stage_words = 0;
        if (cudaMalloc(&c->stage, 4 * words * 4) != cudaSuccess) {
            cudaGetLastError();
            return fail(TB_ENOMEM, "staging allocation failed");
        }
        c->stage_words = 4 * words;
    }
    uint32_t *da = c->stage, *db = c->stage + words, *dc = c->stage + 2 * words, *dout = c->stage + 3 * words;
    TB_CUDA(cudaMemcpyAsync(da, hca, words * 4, cudaMemcpyHostToDevice, c->own));
    if (gate != TB_NOT) TB_CUDA(cudaMemcpyAsync(db, hcb, words * 4, cudaMemcpyHostToDevice, c->own));
    if (gate == TB_MUX) TB_CUDA(cudaMemcpyAsync(dc, hcc, words * 4, cudaMemcpyHostToDevice, c->own));
    rc = tb_gates(c, gate, da, db, dc, dout, count, stride, (tb_stream)c->own);
    if (rc) return rc;
    TB_CUDA(cudaMemcpyAsync(hout, dout, words * 4, cudaMemcpyDeviceToHost, c->own));
    TB_CUDA(cudaStreamSynchronize(c->own));
    return TB_OK;
}

extern "C" int tb_bootstrap_wo_ks(tb_ctx* c, const uint32_t* in, int64_t in_stride, uint32_t* out,
                                  int64_t out_stride, int64_t count, tb_stream stream) {
    if (!c) return fail(TB_EINVAL, "null context");
    if (!c->have_bk) return fail(TB_ENOKEYS, "load the bootstrapping key first");
    if (count < 0 || in_stride < kn + 1 || out_stride < kN + 1) return fail(TB_EINVAL, "bad count or stride");
    if (count == 0) return TB_OK;
    if (!in || !out) return fail(TB_EINVAL, "null array");
    TB_CUDA(cudaSetDevice(c->device));
    int rc = grow_desc(c, count);
    if (rc) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    launch_build_gate_desc(kGateBoot, 1, 0, 0u, count, c->ldesc, c->gdesc, st);
    return run_br(c, in, in, in, in_stride, c->ldesc, count, out, out_stride, st);
}

extern "C" int tb_keyswitch(tb_ctx* c, const uint32_t* in, int64_t in_stride, uint32_t* out, int64_t out_stride,
                            int64_t count, tb_stream stream) {
    if (!c) return fail(TB_EINVAL, "null context");
    if (!c->have_ksk) return fail(TB_ENOKEYS, "load the key-switching key first");
    if (count < 0 || in_stride < kN + 1 || out_stride < kn + 1) return fail(TB_EINVAL, "bad count or stride");
    if (count == 0) return TB_OK;
    if (!in || !out) return fail(TB_EINVAL, "null array");
    TB_CUDA(cudaSetDevice(c->device));
    int rc = grow_desc(c, count);
    if (rc) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    launch_build_gate_desc(kGateBoot, 1, 0, 0u, count, c->ldesc, c->gdesc, st);
    return run_ks(c, in, 0, in_stride, c->gdesc, count, out, out_stride, in, in_stride, st);
}

extern "C" int tb_ntt_muladd6(tb_ctx* c, const int32_t* digits, const uint32_t* polys, uint32_t* res) {
    if (!c || !digits || !polys || !res) return fail(TB_EINVAL, "null argument");
    TB_CUDA(cudaSetDevice(c->device));
    if (launch_ntt_muladd6(digits, polys, res, c->twF, c->twI, c->ninv, c->ninvp, c->own))
        return fail(TB_ECUDA, "ntt_muladd6 launch failed");
    TB_CUDA(cudaGetLastError());
    TB_CUDA(cudaStreamSynchronize(c->own));
    return TB_OK;
}

extern "C" int tb_fft_muladd6(tb_ctx* c, const int32_t* digits, const uint32_t* polys, uint32_t* res) {
    if (!c || !digits || !polys || !res) return fail(TB_EINVAL, "null argument");
    TB_CUDA(cudaSetDevice(c->device));
    if (launch_fft_muladd6(digits, polys, res, c->fftB, c->fftC, c->own))
        return fail(TB_ECUDA, "fft_muladd6 launch failed");
    TB_CUDA(cudaGetLastError());
    TB_CUDA(cudaStreamSynchronize(c->own));
    return TB_OK;
}

extern "C" int tb_microbench(tb_ctx* c, int iters, double* bfly, double* mac) {
    if (!c || !bfly || !mac || iters <= 0) return fail(TB_EINVAL, "bad argument");
    TB_CUDA(cudaSetDevice(c->device));
    if (run_microbench(iters, bfly, mac)) return fail(TB_ECUDA, "microbenchmark failed");
    return TB_OK;
}

extern "C" int tb_microbench_fields(tb_ctx* c, int iters, double* rates) {
    if (!c || !rates || iters <= 0) return fail(TB_EINVAL, "bad argument");
    TB_CUDA(cudaSetDevice(c->device));
    if (run_microbench_fields(iters, rates)) return fail(TB_ECUDA, "microbenchmark failed");
    return TB_OK;
}

extern "C" int tb_tc_muladd(tb_ctx* c, const int32_t* digits, const uint32_t* polys, uint32_t* res) {
    if (!c || !digits || !polys || !res) return fail(TB_EINVAL, "null argument");
    TB_CUDA(cudaSetDevice(c->device));
    uint32_t* b4 = nullptr;
    TB_CUDA(cudaMalloc(&b4, (size_t)kN * 36 * 4));
    launch_bk_to_bk4(polys, b4, c->tcPts, c->ninv, c->ninvp, 1, c->own);
    const int rc = launch_brt_muladd(digits, b4, c->tcB, c->tcTw, res, c->own);
    cudaError_t e = rc ? cudaErrorLaunchFailure : cudaGetLastError();
    if (e == cudaSuccess) e = cudaStreamSynchronize(c->own);
    cudaFree(b4);
    if (e != cudaSuccess) return cuda_fail(e, "tb_tc_muladd");
    return TB_OK;
}

extern "C" int tb_tc_mma_test(tb_ctx* c, const uint8_t* A, const uint8_t* B, int K, int N, int a_signed, int b_signed,
                              int lbo, int32_t* D) {
    if (!c || !A || !B || !D) return fail(TB_EINVAL, "null argument");
    TB_CUDA(cudaSetDevice(c->device));
    const int rc = run_tc_mma_test(A, B, K, N, a_signed, b_signed, lbo, D, c->own);
    if (rc == -2) return fail(TB_EINVAL, "K must be a multiple of 32 <= 256, N a multiple of 16 <= 256, lbo >= 128");
    if (rc) return fail(TB_ECUDA, "tensor-core test launch failed");
    TB_CUDA(cudaGetLastError());
    TB_CUDA(cudaStreamSynchronize(c->own));
    return TB_OK;
}

// ------------------------------------------------------------------------------------------ netlists
// Algorithm 1: starting from the inputs (ready = finished = I), each iteration computes every
// node whose predecessors are all ready.  The iteration in which gate g first enters C - finished is
// 1 + max(level of its predecessors) (inputs = level 0), computed here with one Kahn pass (C14: k = 1).
static int levelise_impl(const tb_netlist* net, std::vector<int64_t>& level, int64_t* n_levels) {
    if (!net || net->n_inputs < 0 || net->n_gates < 0) return fail(TB_EINVAL, "bad netlist");
    const int64_t ni = net->n_inputs, ng = net->n_gates, nw = ni + ng;
    if (ng > 0 && (!net->type || !net->in0 || !net->in1)) return fail(TB_EINVAL, "null netlist array");
    level.assign((size_t)ng, -1);
    std::vector<int32_t> pending((size_t)ng, 0);
    std::vector<int64_t> head((size_t)nw + 1, 0), adj;
    auto ins = [&](int64_t g, int64_t k) -> int64_t {
        if (k == 0) return net->in0[g];
        if (k == 1) return net->type[g] == TB_NOT ? -1 : net->in1[g];
        return (net->type[g] == TB_MUX && net->in2) ? net->in2[g] : -1;
    };
    for (int64_t g = 0; g < ng; g++) {
        const int t = net->type[g];
        if (!gate_known(t)) return fail(TB_EINVAL, "unknown gate code in netlist");
        for (int k = 0; k < 3; k++) {
            const int64_t w = ins(g, k);
            const bool needed = k == 0 || (k == 1 && t != TB_NOT) || (k == 2 && t == TB_MUX);
            if (!needed) continue;
            if (w < 0 || w >= nw) return fail(TB_EINVAL, "wire index out of range");
            if (w == ni + g) return fail(TB_EINVAL, "gate reads its own output (cycle)");
            if (w >= ni) {
                pending[g]++;
                head[w + 1]++;
            }
        }
    }
    for (int64_t w = 0; w < nw; w++) head[w + 1] += head[w];
    adj.resize((size_t)head[nw]);
    std::vector<int64_t> fill(head.begin(), head.end() - 1);
    for (int64_t g = 0; g < ng; g++) {
        const int t = net->type[g];
        for (int k = 0; k < 3; k++) {
            const bool needed = k == 0 || (k == 1 && t != TB_NOT) || (k == 2 && t == TB_MUX);
            if (!needed) continue;
            const int64_t w = ins(g, k);
            if (w >= ni) adj[fill[w]++] = g;
        }
    }
    std::vector<int64_t> ready;                 // the current C - finished frontier
    for (int64_t g = 0; g < ng; g++)
        if (pending[g] == 0) { level[g] = 1; ready.push_back(g); }
    int64_t done = 0, L = ready.empty() ? 0 : 1;
    std::vector<int64_t> next;
    while (!ready.empty()) {
        next.clear();
        for (int64_t g : ready) {
            done++;
            const int64_t w = ni + g;
            for (int64_t e = head[w]; e < head[w + 1]; e++) {
                const int64_t h = adj[e];
                if (--pending[h] == 0) { level[h] = L + 1; next.push_back(h); }
            }
        }
        if (!next.empty()) L++;
        ready.swap(next);
    }
    if (done != ng) return fail(TB_EINVAL, "netlist has a cycle");
    *n_levels = L;
    return TB_OK;
}

extern "C" int tb_levelise(const tb_netlist* net, int64_t* level_of_gate, int64_t* n_levels) {
    if (!level_of_gate || !n_levels) return fail(TB_EINVAL, "null argument");
    std::vector<int64_t> lv;
    int rc = levelise_impl(net, lv, n_levels);
    if (rc) return rc;
    std::copy(lv.begin(), lv.end(), level_of_gate);
    return TB_OK;
}

// Capacity-aware re-levelisation ("dependency-driven scheduling beyond strict levels").
// Algorithm 1 runs every gate at its earliest level (ASAP).  On a deep, narrow netlist a level whose
// bootstraps exceed one wave of the latency kernel costs a second wave although many of its gates have
// slack.  Here each gate g has a window [ASAP(g), ALAP(g)] (ALAP = latest level that keeps the depth); levels
// are built in order: every ready gate whose deadline is this level is taken, then ready gates by increasing
// deadline while the level's lanes (MUX = 2 bootstraps, NOT = 0) stay <= `cap`.  The depth is unchanged
// (every gate runs by its deadline), so the serial chain of levels is as short as Algorithm 1's.
static void relevel_capacity(const tb_netlist* net, std::vector<int64_t>& lv, int64_t nlev, int64_t cap) {
    const int64_t ni = net->n_inputs, ng = net->n_gates;
    auto need = [&](int64_t g, int k) {
        const int t = net->type[g];
        return k == 0 || (k == 1 && t != TB_NOT) || (k == 2 && t == TB_MUX);
    };
    auto src = [&](int64_t g, int k) { return k == 0 ? net->in0[g] : (k == 1 ? net->in1[g] : net->in2[g]); };
    // successor lists (gate -> consumers) and ALAP by a reverse sweep over the ASAP order
    std::vector<int64_t> head((size_t)ng + 1, 0), adj, pend((size_t)ng, 0);
    for (int64_t g = 0; g < ng; g++)
        for (int k = 0; k < 3; k++)
            if (need(g, k) && src(g, k) >= ni) { head[src(g, k) - ni + 1]++; pend[g]++; }
    for (int64_t g = 0; g < ng; g++) head[g + 1] += head[g];
    adj.resize((size_t)head[ng]);
    std::vector<int64_t> fill(head.begin(), head.end() - 1);
    for (int64_t g = 0; g < ng; g++)
        for (int k = 0; k < 3; k++)
            if (need(g, k) && src(g, k) >= ni) adj[fill[src(g, k) - ni]++] = g;
    std::vector<int64_t> byl((size_t)ng);
    for (int64_t g = 0; g < ng; g++) byl[g] = g;
    std::stable_sort(byl.begin(), byl.end(), [&](int64_t x, int64_t y) { return lv[x] > lv[y]; });
    std::vector<int64_t> alap((size_t)ng, nlev);
    for (int64_t g : byl)
        for (int64_t e = head[g]; e < head[g + 1]; e++) alap[g] = std::min(alap[g], alap[adj[e]] - 1);
    auto lanes = [&](int64_t g) { return net->type[g] == TB_MUX ? 2 : (net->type[g] == TB_NOT ? 0 : 1); };
    std::vector<std::vector<int64_t>> bucket((size_t)nlev + 2);    // ready gates by deadline
    for (int64_t g = 0; g < ng; g++)
        if (pend[g] == 0) bucket[alap[g]].push_back(g);
    std::vector<int64_t> took;
    for (int64_t L = 1; L <= nlev; L++) {
        took.clear();
        int64_t used = 0;
        for (int64_t g : bucket[L]) { took.push_back(g); used += lanes(g); }   // deadline now: always
        bucket[L].clear();
        for (int64_t a = L + 1; a <= nlev && used < cap; a++) {
            auto& B = bucket[a];
            size_t keep = 0;
            for (size_t j = 0; j < B.size(); j++) {
                const int64_t g = B[j];
                if (used + lanes(g) <= cap) { took.push_back(g); used += lanes(g); }
                else B[keep++] = g;
            }
            B.resize(keep);
        }
        for (int64_t g : took) {
            lv[g] = L;
            for (int64_t e = head[g]; e < head[g + 1]; e++)
                if (--pend[adj[e]] == 0) bucket[alap[adj[e]]].push_back(adj[e]);
        }
    }
}

// Levelise (Algorithm 1, then capacity-aware re-levelisation when cap > 0) and renumber: inputs keep rows
// [0, n_inputs); the gates of level L follow those of level L-1, ascending original index inside a level.
// level_off (0-based, n_levels + 1 entries) are gate offsets into that order; order[k] = original gate index
// of the k-th gate.
// Level order for R ranks (start a rank's locally ready gates before the level barrier).  Each
// level is cut into R contiguous chunks (parallel.shard: ceil(n / R) gates each).  A gate of level L is "early"
// for rank r if every input it reads from level L - 1 lies in r's chunk of level L - 1 (inputs of older levels
// were exchanged at earlier barriers).  Rank r's chunk of level L is filled with the gates that are early for r
// (affinity r, then gates with no level-(L-1) input), then with the rest; its early gates come first, so they
// are a prefix [g0, g0 + early) that r can run before the barrier of level L - 1.  Outputs do not depend on the
// order (each gate's result depends only on its input bytes); R = 1 keeps ascending original indices.
static void order_for_world(const tb_netlist* net, const std::vector<int64_t>& lv, int64_t nlev,
                            const std::vector<int64_t>& level_off, std::vector<int64_t>& order, int world,
                            std::vector<int64_t>& early) {
    const int64_t ni = net->n_inputs;
    early.assign((size_t)nlev * world, 0);
    std::vector<int64_t> rank_of_gate((size_t)net->n_gates, -1);   // rank owning the gate in its level
    auto ins = [&](int64_t g, int k) -> int64_t {
        const int t = net->type[g];
        if (k == 0) return net->in0[g];
        if (k == 1) return t == TB_NOT ? -1 : net->in1[g];
        return t == TB_MUX ? net->in2[g] : -1;
    };
    for (int64_t L = 1; L <= nlev; L++) {
        const int64_t a = level_off[L - 1], n = level_off[L] - a;
        const int64_t chunk = (n + world - 1) / world;
        // affinity: -1 = no input from level L - 1 ("free"), r = all such inputs on rank r, -2 = several ranks
        std::vector<std::vector<int64_t>> aff((size_t)world);
        std::vector<int64_t> freeg, mixed;
        for (int64_t k = 0; k < n; k++) {
            const int64_t g = order[a + k];
            int64_t r = -1;
            for (int q = 0; q < 3; q++) {
                const int64_t w = ins(g, q);
                if (w < ni || lv[w - ni] != L - 1) continue;
                const int64_t rw = rank_of_gate[w - ni];
                r = (r == -1 || r == rw) ? rw : -2;
            }
            if (r == -1) freeg.push_back(g);
            else if (r == -2) mixed.push_back(g);
            else aff[(size_t)r].push_back(g);
        }
        std::vector<std::vector<int64_t>> part((size_t)world);
        std::vector<int64_t> rest, cap((size_t)world);
        for (int r = 0; r < world; r++) {
            cap[r] = std::max<int64_t>(0, std::min<int64_t>((r + 1) * chunk, n) - std::min<int64_t>(r * chunk, n));
            for (int64_t g : aff[r]) {
                if ((int64_t)part[r].size() < cap[r]) part[r].push_back(g);
                else rest.push_back(g);
            }
        }
        size_t fi = 0;
        for (int r = 0; r < world; r++)
            while ((int64_t)part[r].size() < cap[r] && fi < freeg.size()) part[r].push_back(freeg[fi++]);
        for (int r = 0; r < world; r++) early[(size_t)(L - 1) * world + r] = (int64_t)part[r].size();
        for (; fi < freeg.size(); fi++) rest.push_back(freeg[fi]);
        rest.insert(rest.end(), mixed.begin(), mixed.end());
        std::sort(rest.begin(), rest.end());
        size_t ri = 0;
        int64_t k = a;
        for (int r = 0; r < world; r++) {
            while ((int64_t)part[r].size() < cap[r] && ri < rest.size()) part[r].push_back(rest[ri++]);
            for (int64_t g : part[r]) {
                order[k++] = g;
                rank_of_gate[g] = r;
            }
        }
    }
}

static int plan_impl(const tb_netlist* net, int64_t* n_levels, std::vector<int64_t>& level_off,
                     std::vector<int64_t>& order, std::vector<int64_t>& row_of_wire, int64_t cap = 0,
                     int world = 1, std::vector<int64_t>* early = nullptr) {
    std::vector<int64_t> lv;
    int64_t nlev = 0;
    int rc = levelise_impl(net, lv, &nlev);
    if (rc) return rc;
    if (cap > 0) relevel_capacity(net, lv, nlev, cap);
    const int64_t ni = net->n_inputs, ng = net->n_gates;
    std::vector<int64_t> cnt((size_t)nlev + 2, 0);
    for (int64_t g = 0; g < ng; g++) cnt[lv[g]]++;
    level_off.assign((size_t)nlev + 1, 0);
    for (int64_t L = 1; L <= nlev; L++) level_off[L] = level_off[L - 1] + cnt[L];
    std::vector<int64_t> pos(level_off.begin(), level_off.end());
    order.assign((size_t)ng, 0);
    for (int64_t g = 0; g < ng; g++) order[pos[lv[g] - 1]++] = g;
    if (early) {
        if (world > 1) {
            order_for_world(net, lv, nlev, level_off, order, world, *early);
        } else {
            early->assign((size_t)nlev, 0);
            for (int64_t L = 1; L <= nlev; L++) (*early)[L - 1] = L == 1 ? level_off[1] : 0;
        }
    }
    row_of_wire.resize((size_t)(ni + ng));
    for (int64_t w = 0; w < ni; w++) row_of_wire[w] = w;
    for (int64_t k = 0; k < ng; k++) row_of_wire[ni + order[k]] = ni + k;
    *n_levels = nlev;
    return TB_OK;
}

extern "C" int tb_netlist_plan(const tb_netlist* net, int64_t* n_levels, int64_t* level_off, int64_t* row_of_wire) {
    return tb_netlist_plan_capacity(net, 0, n_levels, level_off, row_of_wire);
}

extern "C" int tb_netlist_plan_capacity(const tb_netlist* net, int64_t lanes, int64_t* n_levels, int64_t* level_off,
                                        int64_t* row_of_wire) {
    if (!net || !n_levels) return fail(TB_EINVAL, "null argument");
    if (lanes < 0) return fail(TB_EINVAL, "capacity must be >= 0");
    std::vector<int64_t> lo, order, rows;
    int rc = plan_impl(net, n_levels, lo, order, rows, lanes);
    if (rc) return rc;
    if (level_off) std::copy(lo.begin(), lo.end(), level_off);
    if (row_of_wire) std::copy(rows.begin(), rows.end(), row_of_wire);
    return TB_OK;
}

extern "C" int tb_netlist_plan_world(const tb_netlist* net, int64_t lanes, int world, int64_t* n_levels,
                                     int64_t* level_off, int64_t* row_of_wire, int64_t* early) {
    if (!net || !n_levels) return fail(TB_EINVAL, "null argument");
    if (lanes < 0 || world < 1 || world > 1024) return fail(TB_EINVAL, "capacity must be >= 0, world 1..1024");
    std::vector<int64_t> lo, order, rows, ea;
    int rc = plan_impl(net, n_levels, lo, order, rows, lanes, world, &ea);
    if (rc) return rc;
    if (level_off) std::copy(lo.begin(), lo.end(), level_off);
    if (row_of_wire) std::copy(rows.begin(), rows.end(), row_of_wire);
    if (early) std::copy(ea.begin(), ea.end(), early);
    return TB_OK;
}

extern "C" int tb_netlist_upload(tb_ctx* c, const tb_netlist* net, tb_dev_netlist** out) {
    if (!c || !net || !out) return fail(TB_EINVAL, "null argument");
    *out = nullptr;
    if (net->n_inputs + net->n_gates > INT32_MAX) return fail(TB_EINVAL, "netlist too large for 32-bit rows");
    tb_dev_netlist* d = new (std::nothrow) tb_dev_netlist();
    if (!d) return fail(TB_ENOMEM, "host allocation failed");
    std::vector<int64_t> order;
    int64_t cap = c->level_capacity;
    if (cap < 0) {   // auto: one wave of the latency kernel brl (32 bootstraps on B200)
        if (c->brl_wave == -2) c->brl_wave = brl_wave_lanes();
        cap = c->brl_wave > 0 ? c->brl_wave : 0;
    }
    d->world = c->plan_world;
    int rc = plan_impl(net, &d->n_levels, d->level_off, order, d->row_of_wire, cap, d->world, &d->early);
    if (rc) {
        delete d;
        return rc;
    }
    const int64_t ni = net->n_inputs, ng = net->n_gates;
    d->n_inputs = ni; d->n_gates = ng;
    d->in_level.assign((size_t)ni, d->n_levels + 1);
    d->in_first.assign((size_t)ni, ng);
    for (int64_t L = 1; L <= d->n_levels; L++)
        for (int64_t k = d->level_off[L - 1]; k < d->level_off[L]; k++) {
            const int64_t g = order[k];
            const int t = net->type[g];
            const int64_t w[3] = {net->in0[g], t == TB_NOT ? -1 : net->in1[g], t == TB_MUX ? net->in2[g] : -1};
            for (int64_t x : w)
                if (x >= 0 && x < ni) {
                    d->in_level[x] = std::min(d->in_level[x], L);
                    d->in_first[x] = std::min(d->in_first[x], k);
                }
        }
    // descriptors in level-sorted order
    std::vector<GateDesc> gd((size_t)ng);
    std::vector<LaneDesc> ld;
    ld.reserve((size_t)ng);
    d->lane_off.assign((size_t)ng + 1, 0);
    d->boot_prefix.assign((size_t)ng + 1, 0);
    for (int64_t k = 0; k < ng; k++) {
        const int64_t g = order[k];
        const int t = net->type[g];
        const int32_t ra = (int32_t)d->row_of_wire[net->in0[g]];
        GateDesc G;
        G.out_row = (int32_t)(ni + k);
        G.lane1 = -1;
        if (t == TB_NOT) {
            G.kind = kGateNot;
            G.lane0 = ra;
        } else if (t == TB_MUX) {
            const int32_t rb = (int32_t)d->row_of_wire[net->in1[g]];
            const int32_t rc2 = (int32_t)d->row_of_wire[net->in2[g]];
            G.kind = kGateMux;
            G.lane0 = (int32_t)ld.size();
            ld.push_back(LaneDesc{ra, rb, 1, 1, 0u - kMu, 0u, 0u, 0u});      // AND(a, b)
            G.lane1 = (int32_t)ld.size();
            ld.push_back(LaneDesc{ra, rc2, -1, 1, 0u - kMu, 0u, 0u, 0u});    // ANDNY(a, c)
        } else {
            uint32_t C; int32_t wa, wb;
            gate_linear(t, &C, &wa, &wb);
            const int32_t rb = (int32_t)d->row_of_wire[net->in1[g]];
            G.kind = kGateBoot;
            G.lane0 = (int32_t)ld.size();
            ld.push_back(LaneDesc{ra, rb, wa, wb, C, 0u, 0u, 0u});
        }
        gd[k] = G;
        d->lane_off[k + 1] = (int64_t)ld.size();
        d->boot_prefix[k + 1] = d->boot_prefix[k] + (t == TB_NOT ? 0 : 1);
    }
    cudaError_t e = cudaSetDevice(c->device);
    if (e == cudaSuccess && ng > 0) e = cudaMalloc(&d->gdesc, gd.size() * sizeof(GateDesc));
    if (e == cudaSuccess && !ld.empty()) e = cudaMalloc(&d->ldesc, ld.size() * sizeof(LaneDesc));
    if (e == cudaSuccess && ng > 0) e = cudaMemcpy(d->gdesc, gd.data(), gd.size() * sizeof(GateDesc), cudaMemcpyHostToDevice);
    if (e == cudaSuccess && !ld.empty()) e = cudaMemcpy(d->ldesc, ld.data(), ld.size() * sizeof(LaneDesc), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        tb_netlist_free(c, d);
        return cuda_fail(e, "tb_netlist_upload");
    }
    *out = d;
    return TB_OK;
}

extern "C" int tb_netlist_free(tb_ctx* c, tb_dev_netlist* d) {
    if (!d) return TB_OK;
    if (c) cudaSetDevice(c->device);
    cudaFree(d->gdesc);
    cudaFree(d->ldesc);
    delete d;
    return TB_OK;
}

extern "C" int tb_netlist_info(const tb_dev_netlist* d, int64_t* n_levels, int64_t* n_rows) {
    if (!d) return fail(TB_EINVAL, "null netlist");
    if (n_levels) *n_levels = d->n_levels;
    if (n_rows) *n_rows = d->n_inputs + d->n_gates;
    return TB_OK;
}

extern "C" int tb_netlist_wire_rows(const tb_dev_netlist* d, int64_t* row_of_wire) {
    if (!d || !row_of_wire) return fail(TB_EINVAL, "null argument");
    std::copy(d->row_of_wire.begin(), d->row_of_wire.end(), row_of_wire);
    return TB_OK;
}

extern "C" int tb_netlist_level(const tb_dev_netlist* d, int64_t level, int64_t* row0, int64_t* n_gates,
                                int64_t* n_boot, int64_t* n_lanes) {
    if (!d) return fail(TB_EINVAL, "null netlist");
    if (level < 1 || level > d->n_levels) return fail(TB_EINVAL, "level out of range");
    const int64_t a = d->level_off[level - 1], b = d->level_off[level];
    if (row0) *row0 = d->n_inputs + a;
    if (n_gates) *n_gates = b - a;
    if (n_boot) *n_boot = d->boot_prefix[b] - d->boot_prefix[a];
    if (n_lanes) *n_lanes = d->lane_off[b] - d->lane_off[a];
    return TB_OK;
}

extern "C" int tb_run_level(tb_ctx* c, const tb_dev_netlist* d, int64_t level, int64_t g0, int64_t g1,
                            uint32_t* wires, int64_t stride, tb_stream stream) {
    NvtxRange nv("tb_run_level");
    int rc = check_ready(c);
    if (rc) return rc;
    if (!d || !wires) return fail(TB_EINVAL, "null argument");
    if (stride < kn + 1) return fail(TB_EINVAL, "stride < n + 1");
    if (level < 1 || level > d->n_levels) return fail(TB_EINVAL, "level out of range");
    const int64_t a = d->level_off[level - 1], b = d->level_off[level];
    if (g0 < 0 || g1 < g0 || a + g1 > b) return fail(TB_EINVAL, "gate range outside the level");
    if (g0 == g1) return TB_OK;
    TB_CUDA(cudaSetDevice(c->device));
    const int64_t G0 = a + g0, G1 = a + g1;
    const int64_t l0 = d->lane_off[G0], l1 = d->lane_off[G1];
    if ((rc = grow_lanes(c, std::max<int64_t>(l1 - l0, 1)))) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if ((rc = run_br(c, wires, wires, wires, stride, d->ldesc + l0, l1 - l0, c->lanebuf, kLaneStride, st))) return rc;
    const bool mirror = c->npeers > 0 && wires == c->peer_own;
    return run_ks(c, c->lanebuf, l0, kLaneStride, d->gdesc + G0, G1 - G0, wires, stride, wires, stride, st,
                  mirror ? c->peers : nullptr, mirror ? c->npeers : 0);
}

// ------------------------------------------------------------------------------------------ fused all-gather
// The multi-GPU level loop's exchange step: instead of a per-level NCCL all-gather, the
// key-switch kernels store every output row into all ranks' wire arrays over NVLink (peer memory opened with
// CUDA IPC), so the transfer overlaps the key switch tile by tile; the loop then only needs a barrier.
extern "C" int tb_set_peer_wires(tb_ctx* c, const uint32_t* own_wires, uint32_t* const* peer_wires, int n) {
    if (!c || n < 0 || (n > 0 && (!peer_wires || !own_wires))) return fail(TB_EINVAL, "bad peer list");
    for (int k = 0; k < n; k++)
        if (!peer_wires[k]) return fail(TB_EINVAL, "null peer wire array");
    TB_CUDA(cudaSetDevice(c->device));
    cudaFree(c->peers);
    c->peers = nullptr;
    c->npeers = 0;
    c->peer_own = nullptr;
    if (n == 0) return TB_OK;
    TB_CUDA(cudaMalloc(&c->peers, (size_t)n * sizeof(uint32_t*)));
    TB_CUDA(cudaMemcpy(c->peers, peer_wires, (size_t)n * sizeof(uint32_t*), cudaMemcpyHostToDevice));
    c->npeers = n;
    c->peer_own = own_wires;
    return TB_OK;
}

// base of the device allocation holding p (driver cuMemGetAddressRange through the runtime's entry-point query,
// so the library does not link libcuda)
static int alloc_base(const void* p, void** base) {
    using Fn = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
    static Fn fn = nullptr;
    if (!fn) {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess || !f ||
            q != cudaDriverEntryPointSuccess)
            return -1;
        fn = (Fn)f;
    }
    CUdeviceptr b = 0;
    size_t size = 0;
    if (fn(&b, &size, (CUdeviceptr)p) != CUDA_SUCCESS) return -1;
    *base = (void*)b;
    return 0;
}

extern "C" int tb_ipc_export(const void* dev_ptr, unsigned char* handle, int64_t* offset) {
    if (!dev_ptr || !handle || !offset) return fail(TB_EINVAL, "null argument");
    void* base = nullptr;
    if (alloc_base(dev_ptr, &base)) return fail(TB_ECUDA, "device allocation base lookup failed");
    cudaIpcMemHandle_t h;
    TB_CUDA(cudaIpcGetMemHandle(&h, base));
    static_assert(sizeof(h) == TB_IPC_HANDLE_BYTES, "IPC handle size");
    memcpy(handle, &h, sizeof(h));
    *offset = (int64_t)((const char*)dev_ptr - (const char*)base);
    return TB_OK;
}

extern "C" int tb_ipc_import(tb_ctx* c, const unsigned char* handle, int64_t offset, void** dev_ptr, void** base) {
    if (!c || !handle || !dev_ptr || !base || offset < 0) return fail(TB_EINVAL, "bad argument");
    TB_CUDA(cudaSetDevice(c->device));
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    void* b = nullptr;
    TB_CUDA(cudaIpcOpenMemHandle(&b, h, cudaIpcMemLazyEnablePeerAccess));
    *base = b;
    *dev_ptr = (char*)b + offset;
    return TB_OK;
}

extern "C" int tb_ipc_close(tb_ctx* c, void* base) {
    if (!c || !base) return fail(TB_EINVAL, "null argument");
    TB_CUDA(cudaSetDevice(c->device));
    TB_CUDA(cudaIpcCloseMemHandle(base));
    return TB_OK;
}


extern "C" int tb_run_netlist(tb_ctx* c, const tb_dev_netlist* d, uint32_t* wires, int64_t stride, tb_stream stream) {
    if (!d) return fail(TB_EINVAL, "null netlist");
    for (int64_t L = 1; L <= d->n_levels; L++) {
        const int64_t n = d->level_off[L] - d->level_off[L - 1];
        int rc = tb_run_level(c, d, L, 0, n, wires, stride, stream);
        if (rc) return rc;
    }
    return TB_OK;
}

// ------------------------------------------------------------------------------------------ profiling
extern "C" int tb_profile_enable(tb_ctx* c, int enable) {
    if (!c) return fail(TB_EINVAL, "null context");
    TB_CUDA(cudaSetDevice(c->device));
    if (enable) {
        c->ev_used = 0;
        c->ev_rec.clear();
    }
    c->prof = enable != 0;
    return TB_OK;
}

extern "C" int tb_profile_read(tb_ctx* c, double* br_ms, int64_t* br_n, double* ks_ms, int64_t* ks_n) {
    if (!c) return fail(TB_EINVAL, "null context");
    TB_CUDA(cudaSetDevice(c->device));
    double t[2] = {0, 0};
    int64_t n[2] = {0, 0};
    for (const auto& r : c->ev_rec) {
        TB_CUDA(cudaEventSynchronize(c->ev_pool[r.second + 1]));
        float ms = 0;
        TB_CUDA(cudaEventElapsedTime(&ms, c->ev_pool[r.second], c->ev_pool[r.second + 1]));
        t[r.first] += ms;
        n[r.first]++;
    }
    if (br_ms) *br_ms = t[0];
    if (br_n) *br_n = n[0];
    if (ks_ms) *ks_ms = t[1];
    if (ks_n) *ks_n = n[1];
    return TB_OK;
}

// ------------------------------------------------------------------------------------------ e2e host path
extern "C" int tb_set_host_overlap(tb_ctx* c, int enable) {
    if (!c) return fail(TB_EINVAL, "null context");
    c->overlap_host = enable != 0;
    return TB_OK;
}

// End to end through host buffers (the host side of one batch overlaps the device
// work of another).  The input rows are copied on their own stream in the order of the level that first reads
// them, and level L waits only for the inputs it reads; the requested outputs produced by level L are copied back
// on a second stream while level L + 1 runs.  With overlap off (tb_set_host_overlap(0)) everything is serial.
static int run_netlist_host_impl(tb_ctx* c, const tb_dev_netlist* d, const uint32_t* hin, int64_t in_stride,
                                 const int64_t* outw, int64_t n_out, uint32_t* hout, int64_t out_stride);
// tb_run_netlist_host: a level of more than kHostChunkMinWaves waves of br6 (4 lanes per SM) runs as a first and a
// last chunk of kHostEdgeWaves waves around the rest, so that the copies overlap inside a wide level as well
constexpr int64_t kHostChunkMinWaves = 8, kHostEdgeWaves = 3;
extern "C" int tb_run_netlist_host(tb_ctx* c, const tb_dev_netlist* d, const uint32_t* hin, int64_t in_stride,
                                   const int64_t* outw, int64_t n_out, uint32_t* hout, int64_t out_stride) {
    NvtxRange nv("tb_run_netlist_host");
    const int rc = run_netlist_host_impl(c, d, hin, in_stride, outw, n_out, hout, out_stride);
    if (rc != TB_OK && c) {   // no copy from / into the caller's host buffers may still be in flight on return
        for (cudaStream_t s : {c->own, c->h2d, c->d2h})
            if (s) cudaStreamSynchronize(s);
        cudaGetLastError();
    }
    return rc;
}
static int run_netlist_host_impl(tb_ctx* c, const tb_dev_netlist* d, const uint32_t* hin, int64_t in_stride,
                                 const int64_t* outw, int64_t n_out, uint32_t* hout, int64_t out_stride) {
    int rc = check_ready(c);
    if (rc) return rc;
    if (!d || (d->n_inputs > 0 && !hin) || (n_out > 0 && (!outw || !hout))) return fail(TB_EINVAL, "null argument");
    if (in_stride < kn + 1 || out_stride < kn + 1 || n_out < 0) return fail(TB_EINVAL, "bad stride or count");
    const int64_t nw = d->n_inputs + d->n_gates, nL = d->n_levels;
    std::vector<int64_t> rows((size_t)n_out);
    for (int64_t k = 0; k < n_out; k++) {
        if (outw[k] < 0 || outw[k] >= nw) return fail(TB_EINVAL, "output wire out of range");
        rows[k] = d->row_of_wire[outw[k]];
    }
    TB_CUDA(cudaSetDevice(c->device));
    const int64_t S = kKsRow;                        // 632-word device rows
    const size_t words = (size_t)nw * S + 1;
    if (c->hwires_words < words) {
        cudaFree(c->hwires);
        c->hwires = nullptr;
        c->hwires_words = 0;
        if (cudaMalloc(&c->hwires, words * 4) != cudaSuccess) {
            cudaGetLastError();
            return fail(TB_ENOMEM, "wire array allocation failed");
        }
        c->hwires_words = words;
    }
    const bool ov = c->overlap_host != 0;
    if (ov && !c->h2d) TB_CUDA(cudaStreamCreateWithFlags(&c->h2d, cudaStreamNonBlocking));
    if (ov && !c->d2h) TB_CUDA(cudaStreamCreateWithFlags(&c->d2h, cudaStreamNonBlocking));
    cudaStream_t cs = c->own, hs = ov ? c->h2d : c->own, ds = ov ? c->d2h : c->own;
    // ---- chunks: a level of more than 8 waves of the throughput kernel (W = 4 lanes x SM count) runs as three
    // launches -- 3 W, the middle (a multiple of W, so no wave is added), the rest (3 W .. 4 W) -- so that the
    // copies overlap inside a wide level too: the middle's inputs land while the first chunk runs, the middle's
    // outputs leave while the last chunk runs; only the first chunk's inputs and the last chunk's outputs are
    // exposed.  (Chunks of 16 W throughout were measured slower: each key-switch launch has its own tail.)
    if (c->sms == 0 && cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, c->device) != cudaSuccess)
        c->sms = 148;
    const int64_t W = 4 * (int64_t)c->sms;
    std::vector<int64_t> bnd{0};                      // chunk boundaries in level-sorted gate positions
    std::vector<int64_t> lvl_of_chunk;
    for (int64_t L = 1; L <= nL; L++) {
        const int64_t a0 = d->level_off[L - 1], a1 = d->level_off[L], n = a1 - a0;
        if (ov && n > kHostChunkMinWaves * W) {
            const int64_t mid = (n - 2 * kHostEdgeWaves * W) / W * W;
            for (int64_t e : {a0 + kHostEdgeWaves * W, a0 + kHostEdgeWaves * W + mid, a1}) {
                bnd.push_back(e);
                lvl_of_chunk.push_back(L);
            }
        } else if (n > 0) {
            bnd.push_back(a1);
            lvl_of_chunk.push_back(L);
        }
    }
    const int64_t nC = (int64_t)lvl_of_chunk.size();
    auto chunk_of = [&](int64_t k) {                  // chunk of gate position k (nC: none)
        return (int64_t)(std::upper_bound(bnd.begin(), bnd.end(), k) - bnd.begin()) - 1;
    };
    const size_t nev = 2 * (size_t)(nC + 2);
    while (c->hev.size() < nev) {
        cudaEvent_t e;
        TB_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        c->hev.push_back(e);
    }
    auto ev_in = [&](int64_t j) { return c->hev[(size_t)j]; };             // inputs of chunk j landed
    auto ev_out = [&](int64_t j) { return c->hev[(size_t)(nC + 2 + j)]; }; // chunk j's outputs are final
    // ---- inputs: runs of consecutive rows with the same first chunk, in chunk order
    std::vector<int64_t> in_chunk((size_t)d->n_inputs), by_chunk((size_t)d->n_inputs);
    for (int64_t w = 0; w < d->n_inputs; w++) {
        in_chunk[(size_t)w] = d->in_first[w] >= d->n_gates ? nC : chunk_of(d->in_first[w]);
        by_chunk[(size_t)w] = w;
    }
    if (!std::is_sorted(in_chunk.begin(), in_chunk.end()))     // (already in chunk order: the common layout)
        std::stable_sort(by_chunk.begin(), by_chunk.end(),
                         [&](int64_t x, int64_t y) { return in_chunk[(size_t)x] < in_chunk[(size_t)y]; });
    std::vector<char> has_in((size_t)nC + 1, 0);
    for (size_t a = 0; a < by_chunk.size();) {
        const int64_t j = in_chunk[(size_t)by_chunk[a]];
        size_t b = a + 1;
        while (b < by_chunk.size() && in_chunk[(size_t)by_chunk[b]] == j && by_chunk[b] == by_chunk[b - 1] + 1) b++;
        TB_CUDA(cudaMemcpy2DAsync(c->hwires + (size_t)by_chunk[a] * S, S * 4, hin + (size_t)by_chunk[a] * in_stride,
                                  in_stride * 4, (kn + 1) * 4, b - a, cudaMemcpyHostToDevice, hs));
        if (b == by_chunk.size() || in_chunk[(size_t)by_chunk[b]] != j) {
            TB_CUDA(cudaEventRecord(ev_in(j), hs));
            has_in[(size_t)j] = 1;
        }
        a = b;
    }
    // ---- outputs grouped by the chunk that produces them (index nC: an input passed through)
    std::vector<std::vector<int64_t>> outs_at((size_t)nC + 1);
    for (int64_t k = 0; k < n_out; k++) {
        const int64_t r = rows[k];
        outs_at[(size_t)(r >= d->n_inputs ? chunk_of(r - d->n_inputs) : nC)].push_back(k);
    }
    auto copy_outs = [&](int64_t j) -> int {
        const auto& ks = outs_at[(size_t)j];
        for (size_t a = 0; a < ks.size();) {
            size_t b = a + 1;
            while (b < ks.size() && ks[b] == ks[b - 1] + 1 && rows[ks[b]] == rows[ks[b - 1]] + 1) b++;
            TB_CUDA(cudaMemcpy2DAsync(hout + (size_t)ks[a] * out_stride, out_stride * 4,
                                      c->hwires + (size_t)rows[ks[a]] * S, S * 4, (kn + 1) * 4, b - a,
                                      cudaMemcpyDeviceToHost, ds));
            a = b;
        }
        return TB_OK;
    };
    // ---- the level loop on the compute stream, chunk by chunk
    for (int64_t j = 0; j < nC; j++) {
        if (has_in[(size_t)j]) TB_CUDA(cudaStreamWaitEvent(cs, ev_in(j), 0));
        const int64_t L = lvl_of_chunk[(size_t)j], a0 = d->level_off[L - 1];
        if ((rc = tb_run_level(c, d, L, bnd[(size_t)j] - a0, bnd[(size_t)j + 1] - a0, c->hwires, S, (tb_stream)cs)))
            return rc;
        if (!outs_at[(size_t)j].empty()) {
            TB_CUDA(cudaEventRecord(ev_out(j), cs));
            TB_CUDA(cudaStreamWaitEvent(ds, ev_out(j), 0));
            if ((rc = copy_outs(j))) return rc;
        }
    }
    if (!outs_at[(size_t)nC].empty()) {               // outputs that are inputs: after every input copy
        for (int64_t j = 0; j <= nC; j++)
            if (has_in[(size_t)j]) TB_CUDA(cudaStreamWaitEvent(ds, ev_in(j), 0));
        if ((rc = copy_outs(nC))) return rc;
    }
    TB_CUDA(cudaStreamSynchronize(hs));
    TB_CUDA(cudaStreamSynchronize(cs));
    TB_CUDA(cudaStreamSynchronize(ds));
    return TB_OK;
}
