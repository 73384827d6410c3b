// abacus.cu -- host side of the C ABI declared in include/abacus.h.
//
// Responsibilities: argument validation, the per-call launch plan (segments
// of the candidate space, see common.cuh), the a1 headroom/order step of a
// decision (Eq. 2 + Eq. 3, P:1170-1182 / P:1366-1376, on the host like the
// paper's controller), weight preparation at load time, kernel launches,
// the NCCL combine of sharded sweeps, and reading back the decision.
// Every step of a2..a7 runs in the kernels (kernels_simt.cu, kernels_tc.cu).
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdlib>
#include <mutex>
#include <set>
#include <unistd.h>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/abacus.h"
#include "common.cuh"
#include "device_common.cuh"
#include "internal.h"
#include "tc_ptx.cuh"

using namespace abacus;

// one decision of a batch after a1 (host): its grid, threshold, size and space
// one decision of a batch as the caller gave it (copied to pinned memory, then to the device)
struct BatchRaw {
    abacus_query_t q[ABACUS_K_MAX];
    double now, infl;
    int32_t k, pad;
};
// a1 of one decision of a batch, computed on the device: headroom order, H, error
struct BatchA1 {
    int32_t order[ABACUS_K_MAX];
    float H;
    int32_t err;  // A1 code | query i << 8 | query j << 16 (0 = valid)
};

struct abacus_ctx {
    int device = 0;
    int nsm = 0;
    int32_t n_models = 0, D = 0;
    std::vector<int32_t> L;
    cudaStream_t stream = nullptr;      // stream of the blocking calls (default: own_stream)
    cudaStream_t own_stream = nullptr;
    Scratch* S = nullptr;         // device
    MappedRec* host_result = nullptr;  // pinned, host-mapped: the kernels write the decision here
    MappedRec* dev_result = nullptr;   // device alias of host_result
    uint32_t seq = 0;
    std::string err;
    uint64_t launches = 0;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    bool timed = false;
    // predictor
    bool loaded = false;
    int precision = ABACUS_FP32;
    std::vector<float> params;    // host fp32 copy
    float* d_w1b1 = nullptr;      // device W1[32][D] + b1[32]
    W234 w234{};
    W1P w1p{};                    // layer 1 as a kernel parameter (D = 24 fp32 predictor)
    uint8_t* d_blob[2] = {nullptr, nullptr};  // tensor-core weight blobs (fp16, bf16)
    TcWeights tw[2]{};
    // batched decisions: staging and device buffers, grown on demand (first call of a larger batch)
    int32_t batch_cap = 0;
    Result* h_out = nullptr;     // pinned
    BatchDec* d_decs = nullptr;
    SegP* d_segs = nullptr;
    BatchAcc* d_acc = nullptr;
    float* d_y0 = nullptr;
    Result* d_out = nullptr;
    BatchRaw* h_raw = nullptr;     // pinned: the decisions as given
    BatchRaw* d_raw = nullptr;
    BatchA1* h_a1 = nullptr;       // pinned: a1 per decision (order, H, error), from the device
    BatchA1* d_a1 = nullptr;
    int32_t* d_L = nullptr;        // device copy of the registry's op counts
    uint64_t* d_pairs = nullptr;   // [n] tile pairs per decision, then [n] = total
    // a6 over peer memory: this rank's mailbox of kPeerMax tagged records (abacus_peer_export)
    MappedRec* d_mailbox = nullptr;
    // what-if sweeps (NEXT-4): host-planned grid plans of up to kMaxSeg segments
    int32_t whatif_cap = 0;
    BatchDec* h_wdecs = nullptr;   // pinned
    SegP* h_wsegs = nullptr;       // pinned, kMaxSeg per variant
    SegP* d_wsegs = nullptr;
    // NEXT-3 training state (abacus_train_begin)
    bool training = false;
    abacus_adam_t adam{};
    int64_t train_t = 0;          // Adam step counter
    float* t_p = nullptr;         // parameters, m, v (device, n_params each)
    float* t_m = nullptr;
    float* t_v = nullptr;
    float* t_partial = nullptr;   // [kTrainMaxBlocks][n_params]
    float* t_loss_part = nullptr;
    float* t_loss = nullptr;      // last step's loss (device scalar)
    unsigned* t_ticket = nullptr;
};

namespace {

int fail(abacus_ctx* c, int code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    return code;
}


// ---- NCCL, resolved at run time -------------------------------------------
// The library does not link libnccl: a process that already loaded NCCL
// (e.g. through torch.distributed) must keep using that copy, so the symbols
// are looked up with dlopen(RTLD_NOLOAD) first and only then loaded.
struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;
    ncclResult_t (*CommUserRank)(const ncclComm_t, int*) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

const NcclApi& nccl() {
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return api;
    api.GetUniqueId = (decltype(api.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    api.CommInitRank = (decltype(api.CommInitRank))dlsym(h, "ncclCommInitRank");
    api.CommDestroy = (decltype(api.CommDestroy))dlsym(h, "ncclCommDestroy");
    api.CommCount = (decltype(api.CommCount))dlsym(h, "ncclCommCount");
    api.CommUserRank = (decltype(api.CommUserRank))dlsym(h, "ncclCommUserRank");
    api.AllGather = (decltype(api.AllGather))dlsym(h, "ncclAllGather");
    api.GetErrorString = (decltype(api.GetErrorString))dlsym(h, "ncclGetErrorString");
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.CommCount && api.CommUserRank && api.AllGather &&
             api.GetErrorString;
    return api;
}

#define CUDA_TRY(ctx, call)                                                                         \
    do {                                                                                            \
        cudaError_t e__ = (call);                                                                   \
        if (e__ != cudaSuccess) return fail(ctx, ABACUS_E_CUDA, "%s: %s", #call, cudaGetErrorString(e__)); \
    } while (0)

__host__ __device__ FastDiv make_fastdiv(uint32_t d) {
    FastDiv f{};
    f.d = d;
    uint32_t p = 0;
    while ((1ull << p) < d) p++;
    f.shift = p;
    f.mul = (uint32_t)(((1ull << 32) * ((1ull << p) - d)) / d + 1);
    return f;
}

// ---- validation -----------------------------------------------------------
int validate_grid(abacus_ctx* c, const abacus_grid_t* g, uint64_t* T_out) {
    if (!g) return fail(c, ABACUS_E_INVALID, "grid is NULL");
    if (g->k < 1 || g->k > ABACUS_K_MAX) return fail(c, ABACUS_E_INVALID, "k=%d outside [1,4]", g->k);
    uint64_t T = 1;
    int64_t max_sum_n = 0;
    for (int j = 0; j < g->k; j++) {
        const abacus_slot_t& s = g->slot[j];
        if (s.model_id < 1 || s.model_id > c->n_models)
            return fail(c, ABACUS_E_INVALID, "slot %d: model_id %d outside [1,%d]", j, s.model_id, c->n_models);
        for (int i = 0; i < j; i++)
            if (g->slot[i].model_id == s.model_id)
                return fail(c, ABACUS_E_DUP_MODEL, "slots %d and %d share model %d", i, j, s.model_id);
        const int32_t L = c->L[s.model_id - 1];
        if (s.start_op < 1 || s.start_op > s.end_lo || s.end_lo > s.end_hi || s.end_hi > L)
            return fail(c, ABACUS_E_INVALID, "slot %d: need 1 <= start_op <= end_lo <= end_hi <= L=%d", j, L);
        if (s.batch < 1 || s.batch > 32767) return fail(c, ABACUS_E_INVALID, "slot %d: batch %d", j, s.batch);
        if (s.seqlen < 0 || s.seqlen > 32767) return fail(c, ABACUS_E_INVALID, "slot %d: seqlen %d", j, s.seqlen);
        if (s.allow_absent != 0 && s.allow_absent != 1)
            return fail(c, ABACUS_E_INVALID, "slot %d: allow_absent must be 0/1", j);
        const uint64_t rho = (uint64_t)s.allow_absent + (uint64_t)(s.end_hi - s.end_lo + 1);
        T *= rho;
        if (T >= (1ull << 40)) return fail(c, ABACUS_E_INVALID, "grid size >= 2^40");
        max_sum_n += s.end_hi - s.start_op + 1;
    }
    if (max_sum_n + 1 >= (1ll << 24)) return fail(c, ABACUS_E_INVALID, "sum_n + 1 >= 2^24");
    *T_out = T;
    return ABACUS_OK;
}

// ---- plans ------------------------------------------------------------------
__host__ __device__ void fill_strides(PlanHdr& P) {
    uint64_t b = 1;
    for (int j = kKMax - 1; j >= 0; j--) {
        P.slot[j].tstride = b;
        P.slot[j].rtstride = 1.0 / (double)b;
        if (j < P.k) b *= (uint64_t)P.slot[j].radix;
    }
}

__host__ __device__ void fill_slots(PlanHdr& P, const abacus_grid_t* g) {
    for (int j = 0; j < kKMax; j++) {
        SlotP& s = P.slot[j];
        if (j < g->k) {
            const abacus_slot_t& a = g->slot[j];
            const int32_t radix = a.allow_absent + a.end_hi - a.end_lo + 1;
            s = SlotP{a.model_id, a.start_op, a.batch, a.seqlen, a.end_lo, a.end_hi, a.allow_absent, radix,
                      1.0 / (double)radix};
        } else {
            s = SlotP{0, 0, 0, 0, 0, 0, 0, 1, 1.0};
        }
    }
    P.k = g->k;
    fill_strides(P);
}

__host__ __device__ void finish_box(SegP& s) {
    uint64_t b = 1;
    for (int j = kKMax - 1; j >= 0; j--) {
        s.bstride[j] = b;
        s.rbstride[j] = 1.0 / (double)b;
        s.fd[j] = make_fastdiv(s.cnt[j]);
        b *= s.cnt[j];
    }
}

__host__ __device__ uint64_t box_size(const SegP& s) {
    uint64_t b = 1;
    for (int j = 0; j < kKMax; j++) b *= s.cnt[j];
    return b;
}

// whole grid as one box: digits = grid digits (encode / select kernels)
__host__ __device__ Plan plan_whole_grid(int32_t n_models, int32_t D, const abacus_grid_t* g, uint64_t T) {
    Plan P{};
    P.k = g->k;
    P.n_models = n_models;
    P.D = D;
    P.mode = kModeGrid;
    P.T = T;
    fill_slots(P, g);
    P.n_seg = 1;
    SegP& s = P.seg[0];
    // slots right-aligned in the digits: digit kKMax-1 is the last (fastest) slot
    const int off = kKMax - g->k;
    for (int d = 0; d < kKMax; d++) s.cnt[d] = d < off ? 1u : (uint32_t)P.slot[d - off].radix;
    for (int j = 0; j < kKMax; j++) {
        s.pos[j] = -1;
        s.dpos[j] = j < g->k ? off + j : -1;
    }
    finish_box(s);
    return P;
}

// number of elements of segment box `s` with index < a.  Per SLOT j the box
// digit set is: present -> [dlo_j, dlo_j + cnt_j), absent -> {0}; elements
// are ordered lexicographically by slot (index order).
__host__ __device__ uint64_t box_count_lt(const PlanHdr& P, const SegP& s, const uint32_t* dlo, const uint32_t* scnt, uint64_t a) {
    if (a >= P.T) return box_size(s);
    uint32_t dig[kKMax] = {0, 0, 0, 0};
    uint64_t rem = a;
    for (int j = P.k - 1; j >= 0; j--) {
        dig[j] = (uint32_t)(rem % (uint64_t)P.slot[j].radix);
        rem /= (uint64_t)P.slot[j].radix;
    }
    uint64_t cnt = 0;
    for (int j = 0; j < P.k; j++) {
        const bool present = (s.mask >> j) & 1u;
        uint64_t after = 1;  // elements per value of slot j's digit
        for (int i = j + 1; i < P.k; i++)
            if ((s.mask >> i) & 1u) after *= scnt[i];
        uint64_t below;
        bool inside;
        if (present) {
            const int64_t b = (int64_t)dig[j] - (int64_t)dlo[j];
            below = (uint64_t)(b < 0 ? 0 : (b > (int64_t)scnt[j] ? (int64_t)scnt[j] : b));
            inside = dig[j] >= dlo[j] && dig[j] < dlo[j] + scnt[j];
        } else {
            below = dig[j] > 0 ? 1 : 0;
            inside = dig[j] == 0;
        }
        cnt += below * after;
        if (!inside) return cnt;
    }
    return cnt;
}

// Lay the per-slot box (scnt, sistride) out in digit order: slots with
// cnt == 1 first, then the varying ones in slot order (common.cuh).
__host__ __device__ void order_digits(SegP& s, int k, const uint32_t* scnt, const uint64_t* sistride) {
    int d = 0;
    for (int pass = 0; pass < 2; pass++)
        for (int j = 0; j < kKMax; j++) {
            const uint32_t cj = j < k ? scnt[j] : 1u;
            if ((pass == 0) != (cj == 1)) continue;
            s.dpos[j] = d;
            s.cnt[d] = cj;
            s.istride[d] = j < k ? sistride[j] : 0;
            d++;
        }
    finish_box(s);
    s.fast_carry = s.cnt[kKMax - 1] >= (uint32_t)kTileM ? 1u : 0u;
}

__host__ __device__ void set_positions(const PlanHdr& P, SegP& s) {
    for (int j = 0; j < kKMax; j++) {
        s.pos[j] = -1;
        if (j >= P.k || !((s.mask >> j) & 1u)) continue;
        int p = 0;
        for (int i = 0; i < P.k; i++)
            if (((s.mask >> i) & 1u) && P.slot[i].model_id < P.slot[j].model_id) p++;
        s.pos[j] = p;
    }
}

// GRID / sweep: one segment per presence pattern, restricted to [first, last)
// segment sink of a full Plan (host and single launches)
struct PlanSink {
    Plan* P;
    __host__ __device__ void operator()(int i, const SegP& s) const { P->seg[i] = s; }
};

// The segments go to `put(index, segment)`: the Plan's own table (host and
// single launches) or, on the device planner of a batch, straight to the
// decision's slots in global memory (no 3.7 KB Plan on the thread's stack).
template <class Put>
__host__ __device__ void plan_grid_segments_into(PlanHdr& P, Put&& put, int32_t n_models, int32_t D,
                                                 const abacus_grid_t* g, uint64_t T, uint64_t first, uint64_t last,
                                                 float H) {
    P = PlanHdr{};
    P.k = g->k;
    P.n_models = n_models;
    P.D = D;
    P.mode = kModeGrid;
    P.T = T;
    P.H = H;
    P.want_y0 = first == 0 && last > 0;
    fill_slots(P, g);
    uint64_t tstride[kKMax];
    {
        uint64_t b = 1;
        for (int j = kKMax - 1; j >= 0; j--) {
            tstride[j] = j < g->k ? b : 0;
            if (j < g->k) b *= (uint64_t)P.slot[j].radix;
        }
    }
    uint64_t tiles = 0, n_eval = 0;
    for (uint32_t mask = 0; mask < (1u << g->k); mask++) {
        bool ok = true;
        for (int j = 0; j < g->k; j++)
            if (!g->slot[j].allow_absent && !((mask >> j) & 1u)) ok = false;
        if (!ok) continue;
        SegP s{};
        s.mask = mask;
        uint32_t dlo[kKMax] = {0, 0, 0, 0}, scnt[kKMax] = {1, 1, 1, 1};
        uint64_t sist[kKMax] = {0, 0, 0, 0};
        s.n_base = 0;
        s.t_base = 0;
        for (int j = 0; j < kKMax; j++) {
            const bool present = j < g->k && ((mask >> j) & 1u);
            if (present) {
                const abacus_slot_t& a = g->slot[j];
                scnt[j] = (uint32_t)(a.end_hi - a.end_lo + 1);
                dlo[j] = a.allow_absent ? 1u : 0u;
                s.ope0[j] = a.end_lo;
                sist[j] = tstride[j];
                s.t_base += (uint64_t)dlo[j] * tstride[j];
                s.n_base += a.end_lo - a.start_op + 1;
            } else {
                s.ope0[j] = 0;
            }
        }
        order_digits(s, g->k, scnt, sist);
        set_positions(P, s);
        s.u_begin = box_count_lt(P, s, dlo, scnt, first);
        s.u_end = box_count_lt(P, s, dlo, scnt, last);
        if (s.u_end <= s.u_begin) continue;
        s.tile0 = tiles;
        tiles += (s.u_end - s.u_begin + kTileM - 1) / kTileM;
        n_eval += s.u_end - s.u_begin;
        put(P.n_seg++, s);
    }
    P.n_tiles = tiles;
    P.n_eval = n_eval;
}

__host__ __device__ Plan plan_grid_segments(int32_t n_models, int32_t D, const abacus_grid_t* g, uint64_t T,
                                            uint64_t first, uint64_t last, float H) {
    Plan P{};
    plan_grid_segments_into(static_cast<PlanHdr&>(P), PlanSink{&P}, n_models, D, g, T, first, last, H);
    return P;
}

// CHAIN (decision mode): u = 0 critical only; block j: slots < j full, slot j
// grows op by op, later slots absent
template <class Put>
__host__ __device__ void plan_chain_into(PlanHdr& P, Put&& put, int32_t n_models, int32_t D, const abacus_grid_t* g,
                                         float H, uint64_t* n_out) {
    P = PlanHdr{};
    P.k = g->k;
    P.n_models = n_models;
    P.D = D;
    P.mode = kModeChain;
    P.H = H;
    P.want_y0 = 1;
    fill_slots(P, g);
    uint64_t cum = 0;
    uint64_t tiles = 0;
    for (int j = 0; j < g->k; j++) {
        SegP s{};
        s.mask = (2u << j) - 1u;
        s.n_base = 0;
        uint32_t scnt[kKMax] = {1, 1, 1, 1};
        uint64_t sist[kKMax] = {0, 0, 0, 0};
        for (int i = 0; i < kKMax; i++) s.ope0[i] = 0;
        for (int i = 0; i < j; i++) {
            s.ope0[i] = g->slot[i].end_hi;
            s.n_base += g->slot[i].end_hi - g->slot[i].start_op + 1;
        }
        if (j == 0) {
            s.ope0[0] = g->slot[0].end_hi;
            s.n_base = g->slot[0].end_hi - g->slot[0].start_op + 1;
        } else {
            scnt[j] = (uint32_t)(g->slot[j].end_hi - g->slot[j].start_op + 1);
            s.ope0[j] = g->slot[j].start_op;
            sist[j] = 1;
            s.n_base += 1;
        }
        order_digits(s, g->k, scnt, sist);
        P.chain_cum[j] = cum;
        s.t_base = cum;
        set_positions(P, s);
        s.u_begin = 0;
        s.u_end = box_size(s);
        s.tile0 = tiles;
        tiles += (s.u_end + kTileM - 1) / kTileM;
        cum += s.u_end;
        put(P.n_seg++, s);
    }
    P.chain_cum[g->k] = cum;
    P.T = cum;
    P.n_tiles = tiles;
    P.n_eval = cum;
    *n_out = cum;
}

__host__ __device__ Plan plan_chain(int32_t n_models, int32_t D, const abacus_grid_t* g, float H, uint64_t* n_out) {
    Plan P{};
    plan_chain_into(static_cast<PlanHdr&>(P), PlanSink{&P}, n_models, D, g, H, n_out);
    return P;
}

// ---- weight preparation for the tensor-core path ----------------------------
uint16_t f2h_bits(float v) {
    __half h = __float2half_rn(v);
    uint16_t b;
    memcpy(&b, &h, 2);
    return b;
}
float h2f(uint16_t b) {
    __half h;
    memcpy(&h, &b, 2);
    return __half2float(h);
}
uint16_t f2b_bits(float v) {
    __nv_bfloat16 h = __float2bfloat16_rn(v);
    uint16_t b;
    memcpy(&b, &h, 2);
    return b;
}
float b2f(uint16_t b) {
    __nv_bfloat16 h;
    memcpy(&h, &b, 2);
    return __bfloat162float(h);
}

// smallest s >= 0 with bound * 2^-s <= 2^14 (fp16 activations stay < 65504)
int scale_exp(double bound) {
    int s = 0;
    while (bound / std::ldexp(1.0, s) > 16384.0 && s < 60) s++;
    return s;
}

// blob: [W2 chunks][W3 chunks][out chunks]; chunk = N rows x 16 K, b_offset layout
std::vector<uint8_t> build_blob(const abacus_ctx* c, int fmt, float* l1_scale, float* b4_out) {
    const int D = c->D;
    const float* p = c->params.data();
    const float* W1 = p;
    const float* b1 = W1 + kHidden * D;
    const float* W2 = b1 + kHidden;
    const float* b2 = W2 + kHidden * kHidden;
    const float* W3 = b2 + kHidden;
    const float* b3 = W3 + kHidden * kHidden;
    const float* w4 = b3 + kHidden;
    const float b4 = w4[kHidden];
    // exact power-of-two layer scales (fp16 only): worst-case activation bounds
    // with |x| <= 32768 (any int16 feature row)
    // bf16 (fmt 1): layer 1 runs on the same fp16 table / digit operand as the
    // fp16 path (so it takes the same s1); layers 2, 3 and the output are bf16
    // (no range limit: s2 = s3 = 1, W2 absorbs 1 / s1)
    double s1 = 1, s2 = 1, s3 = 1;
    {
        double B1 = 0, B2 = 0, B3 = 0;
        for (int i = 0; i < kHidden; i++) {
            double a = std::fabs((double)b1[i]);
            for (int j = 0; j < D; j++) a += std::fabs((double)W1[i * D + j]) * 32768.0;
            B1 = std::max(B1, a);
        }
        for (int i = 0; i < kHidden; i++) {
            double a = std::fabs((double)b2[i]);
            for (int j = 0; j < kHidden; j++) a += std::fabs((double)W2[i * kHidden + j]) * B1;
            B2 = std::max(B2, a);
        }
        for (int i = 0; i < kHidden; i++) {
            double a = std::fabs((double)b3[i]);
            for (int j = 0; j < kHidden; j++) a += std::fabs((double)W3[i * kHidden + j]) * B2;
            B3 = std::max(B3, a);
        }
        s1 = std::ldexp(1.0, -scale_exp(B1));
        if (fmt == 0) {
            s2 = std::ldexp(1.0, -scale_exp(B2));
            s3 = std::ldexp(1.0, -scale_exp(B3));
        }
    }
    *l1_scale = (float)s1;
    *b4_out = b4;
    const int nch = fmt == 0 ? 3 : 5;
    const size_t hid_bytes = (size_t)nch * tc::kChunkBytesN32;
    const size_t out_bytes = (size_t)nch * tc::kChunkBytesN16;
    std::vector<uint8_t> blob(2 * hid_bytes + out_bytes, 0);
    auto put = [&](size_t base, int n, int k, uint16_t v) {
        memcpy(blob.data() + base + tc::b_offset(n, k), &v, 2);
    };
    auto conv = [&](float v) { return fmt == 0 ? f2h_bits(v) : f2b_bits(v); };
    auto back = [&](uint16_t b) { return fmt == 0 ? h2f(b) : b2f(b); };
    // hidden layers: out unit n, input j; scale factor maps scaled-in -> scaled-out
    // bf16: W = W_hi + W_lo (lo chunks 2, 3) only for layer 3, the one layer
    // whose split the config-5 error budget needs (DESIGN.md r2); layer 2 and
    // the output run hi weights only (their lo chunks stay zero, never issued;
    // splitting the output too measured 8.6e-3 vs 8.1e-3 max error on config 5
    // and -5 % throughput)
    auto hidden = [&](size_t base, const float* W, const float* b, double sin, double sout, bool lo) {
        const double f = sout / sin;  // W' = W * (s_out / s_in) with s = 2^-e
        for (int n = 0; n < kHidden; n++) {
            for (int j = 0; j < kHidden; j++) {
                const float w = (float)((double)W[n * kHidden + j] * f);
                const int ch = j >> 4, k = j & 15;
                const uint16_t hi = conv(w);
                put(base + (size_t)ch * tc::kChunkBytesN32, n, k, hi);
                if (fmt == 1 && lo) put(base + (size_t)(2 + ch) * tc::kChunkBytesN32, n, k, conv(w - back(hi)));
            }
            const float bb = (float)((double)b[n] * sout);
            const uint16_t bh = conv(bb);
            const size_t cb = base + (size_t)(nch - 1) * tc::kChunkBytesN32;
            if (fmt == 0) {
                // fp16: no bias MMA; the chunk holds the f16 biases as 16 pairs (unit 2i
                // low, 2i + 1 high) that the epilogue adds with HFMA2.RELU
                memcpy(blob.data() + cb + 2 * (size_t)n, &bh, 2);
            } else {
                put(cb, n, 0, bh);
                put(cb, n, 1, conv(bb - back(bh)));
            }
        }
    };
    hidden(0, W2, b2, s1, s2, false);
    hidden(hid_bytes, W3, b3, s2, s3, true);
    // output layer: row 0 = w4 / s3, rows 1..15 zero (both paths add b4 in fp32
    // when y is read, so the blob's output bias chunk stays zero)
    {
        const size_t base = 2 * hid_bytes;
        for (int j = 0; j < kHidden; j++) {
            const float w = (float)((double)w4[j] / s3);
            const int ch = j >> 4, k = j & 15;
            const uint16_t hi = conv(w);
            put(base + (size_t)ch * tc::kChunkBytesN16, 0, k, hi);
        }
    }
    return blob;
}

cudaStream_t pick_stream(abacus_ctx* c, void* st) { return st ? (cudaStream_t)st : c->stream; }

// Wait until the kernel-side publish of sequence number `seq` is visible in
// the mapped record and copy it out (spin; the stream is polled now and then
// so a failed or finished-without-result launch is reported instead of
// hanging). Sequence numbers are unique per process, so a recycled pinned
// buffer can never hold chunks whose tags match a new number.
std::atomic<uint32_t> g_seq{0};
uint32_t next_seq(abacus_ctx*) {
    uint32_t s = ++g_seq;
    if (s == 0) s = ++g_seq;
    return s;
}

// A search that has not published after ABACUS_WAIT_TIMEOUT_S seconds (default
// 300: a full config-4 sweep in fp32 takes about 1 s) is reported as E_CUDA
// instead of spinning forever; the ctx's stream may still hold the hung work.
double wait_timeout_s() {
    static double t = [] {
        const char* e = getenv("ABACUS_WAIT_TIMEOUT_S");
        const double v = e ? atof(e) : 0.0;
        return v > 0.0 ? v : 300.0;
    }();
    return t;
}

int wait_result(abacus_ctx* c, uint32_t seq, Result* R) {
    const auto t0 = std::chrono::steady_clock::now();
    for (uint64_t spin = 1;; spin++) {
        if (rec_read(c->host_result, seq, R)) break;
        if ((spin & 1023) == 0) {
            const cudaError_t e = cudaStreamQuery(c->stream);
            if (e != cudaSuccess && e != cudaErrorNotReady)
                return fail(c, ABACUS_E_CUDA, "search kernel failed: %s", cudaGetErrorString(e));
            if (e == cudaSuccess && !rec_read(c->host_result, seq, R))
                return fail(c, ABACUS_E_CUDA, "search finished without publishing its result");
            const double dt = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            if (dt > wait_timeout_s())
                return fail(c, ABACUS_E_CUDA, "search did not publish its result within %.0f s "
                            "(ABACUS_WAIT_TIMEOUT_S); the ctx stream still holds the work", dt);
        }
    }
    std::atomic_thread_fence(std::memory_order_acquire);
    return ABACUS_OK;
}

// a1 (Eq. 2 + Eq. 3, sort) and the decision's slots in headroom order, shared by
// the host (single rounds) and the device planner of batches. Returns an A1_*
// code (0 = valid) and the offending query indices in *qi, *qj.
enum : int32_t { A1_OK = 0, A1_K, A1_TIME, A1_MODEL, A1_DUP, A1_NEXTOP, A1_SIZES, A1_QTIME, A1_T, A1_SUMN };
__host__ __device__ int32_t a1_slots(const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                                     const int32_t* L, int32_t n_models, int32_t* order, float* H_out,
                                     abacus_grid_t* g_out, uint64_t* T_out, int32_t* qi, int32_t* qj) {
    *qi = *qj = 0;
    if (k < 1 || k > ABACUS_K_MAX) return A1_K;
    if (!isfinite(now_ms) || !isfinite(inflight_pred_ms)) return A1_TIME;
    // a1: Eq. 2 + Eq. 3 headroom per query; ascending order, ties by model id
    double h[ABACUS_K_MAX];
    for (int i = 0; i < k; i++) {
        const abacus_query_t& a = q[i];
        *qi = i;
        if (a.model_id < 1 || a.model_id > n_models) return A1_MODEL;
        for (int j = 0; j < i; j++)
            if (q[j].model_id == a.model_id) {
                *qj = j;
                return A1_DUP;
            }
        if (a.next_op < 1 || a.next_op > L[a.model_id - 1]) return A1_NEXTOP;
        if (a.batch < 1 || a.batch > 32767 || a.seqlen < 0 || a.seqlen > 32767) return A1_SIZES;
        if (!isfinite(a.qos_ms) || !isfinite(a.t_start_ms)) return A1_QTIME;
        h[i] = (a.qos_ms - (now_ms - a.t_start_ms)) - inflight_pred_ms;
        order[i] = i;
    }
    // stable insertion sort of <= 4 entries (std::stable_sort would allocate a buffer per call)
    for (int i = 1; i < k; i++) {
        const int v = order[i];
        int j = i - 1;
        while (j >= 0 && (h[order[j]] > h[v] || (h[order[j]] == h[v] && q[order[j]].model_id > q[v].model_id))) {
            order[j + 1] = order[j];
            j--;
        }
        order[j + 1] = v;
    }
    *H_out = (float)h[order[0]];
    // a2: slots in headroom order; the critical query is fully included
    abacus_grid_t& g = *g_out;
    g = abacus_grid_t{};
    g.k = k;
    uint64_t T = 1;
    int64_t max_sum_n = 0;
    for (int j = 0; j < k; j++) {
        const abacus_query_t& a = q[order[j]];
        const int32_t Lm = L[a.model_id - 1];
        g.slot[j] = abacus_slot_t{a.model_id, a.next_op, a.batch, a.seqlen, j == 0 ? Lm : a.next_op, Lm, j == 0 ? 0 : 1};
        T *= (uint64_t)g.slot[j].allow_absent + (uint64_t)(g.slot[j].end_hi - g.slot[j].end_lo + 1);
        if (T >= (1ull << 40)) return A1_T;
        max_sum_n += Lm - a.next_op + 1;
    }
    if (max_sum_n + 1 >= (1ll << 24)) return A1_SUMN;
    *T_out = T;
    return A1_OK;
}

// host: the same with the library's error text
int a1_fail(abacus_ctx* c, int32_t code, int32_t qi, int32_t qj, const abacus_query_t* q, int32_t k) {
    switch (code) {
        case A1_K: return fail(c, ABACUS_E_INVALID, "k=%d outside [1,4]", k);
        case A1_TIME: return fail(c, ABACUS_E_INVALID, "non-finite time");
        case A1_MODEL: return fail(c, ABACUS_E_INVALID, "query %d: model_id %d", qi, q[qi].model_id);
        case A1_DUP: return fail(c, ABACUS_E_DUP_MODEL, "queries %d, %d share a model", qj, qi);
        case A1_NEXTOP: return fail(c, ABACUS_E_INVALID, "query %d: next_op %d", qi, q[qi].next_op);
        case A1_SIZES: return fail(c, ABACUS_E_INVALID, "query %d: batch/seqlen", qi);
        case A1_QTIME: return fail(c, ABACUS_E_INVALID, "query %d: non-finite time", qi);
        case A1_T: return fail(c, ABACUS_E_INVALID, "grid size >= 2^40");
        case A1_SUMN: return fail(c, ABACUS_E_INVALID, "sum_n + 1 >= 2^24");
        default: return ABACUS_OK;
    }
}

int decision_slots(abacus_ctx* c, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                   int32_t* order, float* H_out, abacus_grid_t* g_out, uint64_t* T_out = nullptr) {
    if (!c->loaded) return fail(c, ABACUS_E_NOT_LOADED, "no predictor loaded");
    if (!q) return fail(c, ABACUS_E_INVALID, "NULL argument");
    int32_t qi = 0, qj = 0;
    uint64_t T = 0;
    const int32_t code = a1_slots(q, k, now_ms, inflight_pred_ms, c->L.data(), c->n_models, order, H_out, g_out, &T,
                                  &qi, &qj);
    if (code) return a1_fail(c, code, qi, qj, q, k);
    if (T_out) *T_out = T;
    return ABACUS_OK;
}

unsigned long long* trace_ptr();

int launch_fused(abacus_ctx* c, Plan& P) {
    P.trace = trace_ptr();
    int grid = 0;
    cudaError_t e;
    if (c->timed) cudaEventRecord(c->ev0, c->stream);
    if (c->precision == ABACUS_FP32) {
        e = launch_fused_fp32(P, c->w234, c->d_w1b1, c->S, c->nsm, c->stream, &grid);
    } else {
        const int fmt = c->precision == ABACUS_FP16 ? 0 : 1;
        e = launch_fused_tc(P, c->tw[fmt], c->d_w1b1, c->S, c->nsm, c->stream, &grid);
    }
    if (c->timed) cudaEventRecord(c->ev1, c->stream);
    if (e != cudaSuccess) return fail(c, ABACUS_E_CUDA, "fused search launch: %s", cudaGetErrorString(e));
    c->launches++;
    return ABACUS_OK;
}

}  // namespace

static unsigned long long* g_trace_ptr = nullptr;
namespace {
unsigned long long* trace_ptr() { return g_trace_ptr; }
}  // namespace

// ============================================================================
// C ABI
// ============================================================================
// ---- batched decisions: planning on the device -----------------------------
// One thread per decision runs the same planner as the single-round path
// (plan_grid_segments / plan_chain, __host__ __device__) and writes the
// decision's header and segments (fixed slots of kMaxSegBatch) in place.
__global__ void batch_plan_kernel(const BatchRaw* __restrict__ raw, int32_t n, int32_t n_models, int32_t D,
                                  const int32_t* __restrict__ L, int32_t space, uint64_t grid_budget,
                                  BatchDec* __restrict__ decs, SegP* __restrict__ segs, uint64_t* __restrict__ pairs,
                                  BatchA1* __restrict__ a1) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const BatchRaw& rw = raw[i];
    // a1 (the host's function): headroom order, H, slots, validation
    BatchA1 r{};
    abacus_grid_t g;
    uint64_t T = 0;
    int32_t qi = 0, qj = 0;
    const int32_t code = a1_slots(rw.q, rw.k, rw.now, rw.infl, L, n_models, r.order, &r.H, &g, &T, &qi, &qj);
    r.err = code ? (code | (qi << 8) | (qj << 16)) : 0;
    a1[i] = r;
    if (code) {
        // an invalid decision gets a one-candidate placeholder plan (model 1 run to
        // its end) so the batch's tile walk stays well formed; the call reports the
        // error and writes no output
        g = abacus_grid_t{};
        g.k = 1;
        g.slot[0] = abacus_slot_t{1, 1, 1, 0, L[0], L[0], 0};
        T = 1;
    }
    const bool chain = !code && (space == ABACUS_SPACE_CHAIN || (space == ABACUS_SPACE_AUTO && T > grid_budget));
    uint64_t n_eval = 0;
    // segments go straight to this decision's slots in global memory
    SegP* my = segs + (size_t)kMaxSegBatch * i;
    auto put = [&](int sg, const SegP& sp) {
        if (sg < kMaxSegBatch) my[sg] = sp;
    };
    PlanHdr P;
    if (chain) {
        plan_chain_into(P, put, n_models, D, &g, r.H, &n_eval);
    } else {
        plan_grid_segments_into(P, put, n_models, D, &g, T, 0, T, r.H);
        n_eval = P.n_eval;
    }
    BatchDec& bd = decs[i];
    bd.h = P;
    bd.h.want_y0 = 1;
    bd.h.n_eval = n_eval;
    bd.h.mapped = nullptr;
    bd.h.trace = nullptr;
    bd.seg0 = (uint32_t)(kMaxSegBatch * i);
    pairs[i] = (P.n_tiles + 1) / 2;  // tiles padded to pairs (lock-step slots never straddle decisions)
}

// exclusive prefix sum of the tile pairs -> decs[i].pair0, pairs[n] = total (one block)
constexpr int kScanThreads = 1024;
__global__ void __launch_bounds__(kScanThreads) batch_scan_kernel(BatchDec* __restrict__ decs,
                                                                  uint64_t* __restrict__ pairs, int32_t n) {
    __shared__ uint64_t s[kScanThreads];
    const int t = threadIdx.x;
    const int per = (n + kScanThreads - 1) / kScanThreads;
    const int i0 = t * per, i1 = min(n, i0 + per);
    uint64_t sum = 0;
    for (int i = i0; i < i1; i++) sum += pairs[i];
    s[t] = sum;
    __syncthreads();
    for (int off = 1; off < kScanThreads; off <<= 1) {  // inclusive Hillis-Steele scan
        const uint64_t v = t >= off ? s[t - off] : 0;
        __syncthreads();
        s[t] += v;
        __syncthreads();
    }
    uint64_t run = s[t] - sum;
    for (int i = i0; i < i1; i++) {
        decs[i].pair0 = run;
        run += pairs[i];
    }
    if (t == kScanThreads - 1) pairs[n] = s[t];
}

namespace {
int grow_batch(abacus_ctx* c, int32_t n) {
    if (n <= c->batch_cap) return ABACUS_OK;
    int32_t cap = c->batch_cap ? c->batch_cap : 256;
    while (cap < n) cap *= 2;
    if (c->h_out) cudaFreeHost(c->h_out);
    cudaFree(c->d_decs);
    cudaFree(c->d_segs);
    cudaFree(c->d_acc);
    cudaFree(c->d_y0);
    cudaFree(c->d_out);
    if (c->h_raw) cudaFreeHost(c->h_raw);
    cudaFree(c->d_raw);
    if (c->h_a1) cudaFreeHost(c->h_a1);
    cudaFree(c->d_a1);
    cudaFree(c->d_pairs);
    c->h_raw = nullptr;
    c->d_raw = nullptr;
    c->h_a1 = nullptr;
    c->d_a1 = nullptr;
    c->d_pairs = nullptr;
    c->h_out = nullptr;
    c->d_decs = nullptr;
    c->d_segs = nullptr;
    c->d_acc = nullptr;
    c->d_y0 = nullptr;
    c->d_out = nullptr;
    c->batch_cap = 0;
    const size_t nd = (size_t)cap, ns = (size_t)cap * kMaxSegBatch;
    CUDA_TRY(c, cudaHostAlloc(&c->h_out, nd * sizeof(Result), cudaHostAllocDefault));
    CUDA_TRY(c, cudaMalloc(&c->d_decs, nd * sizeof(BatchDec)));
    CUDA_TRY(c, cudaMalloc(&c->d_segs, ns * sizeof(SegP)));
    CUDA_TRY(c, cudaMalloc(&c->d_acc, nd * sizeof(BatchAcc)));
    CUDA_TRY(c, cudaMalloc(&c->d_y0, nd * sizeof(float)));
    CUDA_TRY(c, cudaMalloc(&c->d_out, nd * sizeof(Result)));
    CUDA_TRY(c, cudaHostAlloc(&c->h_raw, nd * sizeof(BatchRaw), cudaHostAllocDefault));
    CUDA_TRY(c, cudaMalloc(&c->d_raw, nd * sizeof(BatchRaw)));
    CUDA_TRY(c, cudaHostAlloc(&c->h_a1, nd * sizeof(BatchA1), cudaHostAllocDefault));
    CUDA_TRY(c, cudaMalloc(&c->d_a1, nd * sizeof(BatchA1)));
    CUDA_TRY(c, cudaMalloc(&c->d_pairs, (nd + 1) * sizeof(uint64_t)));

    c->batch_cap = cap;
    return ABACUS_OK;
}

// a7 for one decision from its result record (shared by the single and batched searches)
// a7 on the host for records published to host-mapped memory: end op per slot of t*
void host_decode(const Plan& P, Result& R) {
    for (int j = 0; j < kKMax; j++)
        R.end_op[j] = (R.key && j < P.k) ? decode_slot_ope(P, R.key & ((1ull << 40) - 1), j) : 0;
}

// ---- a6 over peer memory (abacus_peer_comm_init) ------------------------------
struct PeerComm {
    abacus_ctx* ctx = nullptr;
    int32_t nranks = 0, rank = 0;
    uint32_t seq = 0;                 // per-communicator launch counter (same on every rank)
    PeerComb* d_comb = nullptr;       // device copy of the peer table
    std::vector<void*> opened;        // IPC-opened peer mailboxes
};
std::mutex g_peer_mu;
std::set<const void*> g_peer_comms;  // communicators this library created (type check of a void* comm)

PeerComm* as_peer(void* comm) {
    std::lock_guard<std::mutex> lk(g_peer_mu);
    return g_peer_comms.count(comm) ? static_cast<PeerComm*>(comm) : nullptr;
}

// (nranks, rank) of an NCCL communicator (the NCCL copy the process already loaded)
int comm_shape(abacus_ctx* c, void* comm, int* nranks, int* rank) {
    if (PeerComm* pc = as_peer(comm)) {
        if (pc->ctx != c) return fail(c, ABACUS_E_INVALID, "peer communicator of another ctx");
        *nranks = pc->nranks;
        *rank = pc->rank;
        return ABACUS_OK;
    }
    if (!nccl().ok) return fail(c, ABACUS_E_NCCL, "libnccl.so.2 not available");
    if (nccl().CommCount((ncclComm_t)comm, nranks) != ncclSuccess || *nranks < 1 || *nranks > 64 ||
        nccl().CommUserRank((ncclComm_t)comm, rank) != ncclSuccess || *rank < 0 || *rank >= *nranks)
        return fail(c, ABACUS_E_NCCL, "bad communicator");
    return ABACUS_OK;
}

// a6 after a fused launch whose last CTA left this rank's record in S->result
// (P.mapped == null, so end ops are decoded on the device): one ncclAllGather
// of the 56-byte records on the ctx stream, then one 1-thread kernel runs
// combine_results (common.cuh) and publishes the global record to the mapped
// copy tagged `seq`.
int combine_over_comm(abacus_ctx* c, void* comm, uint32_t seq) {
    int nranks = 0, rank = 0;
    int rc = comm_shape(c, comm, &nranks, &rank);
    if (rc) return rc;
    ncclResult_t nr =
        nccl().AllGather(&c->S->result, c->S->gathered, sizeof(Result), ncclUint8, (ncclComm_t)comm, c->stream);
    if (nr != ncclSuccess) return fail(c, ABACUS_E_NCCL, "ncclAllGather: %s", nccl().GetErrorString(nr));
    CUDA_TRY(c, launch_finalize_gather(c->S, nranks, c->dev_result, seq, c->stream));
    c->launches++;
    return ABACUS_OK;
}

// a sweep's decision from its result record (status OK / NONE, no drop test)
abacus_decision_t sweep_decision(const Result& R, int32_t k, float H) {
    abacus_decision_t d{};
    d.critical = 0;
    for (int j = 0; j < 4; j++) d.order[j] = j < k ? j : -1;
    d.headroom_ms = H;
    d.pred_critical_only_ms = R.y0;
    d.evaluated = R.evaluated;
    d.key = R.key;
    d.index = R.key & ((1ull << 40) - 1);
    d.status = R.key ? ABACUS_DECIDE_OK : ABACUS_DECIDE_NONE;
    d.pred_ms = R.key ? R.y_best : NAN;
    d.total_ops = R.key ? R.total_ops : 0;
    for (int j = 0; j < k; j++) d.end_op[j] = R.key ? R.end_op[j] : 0;
    return d;
}

abacus_decision_t assemble_decision(const Result& R, const int32_t* order, int32_t k, float H, uint64_t n_eval) {
    abacus_decision_t d{};
    d.critical = order[0];
    for (int j = 0; j < 4; j++) d.order[j] = j < k ? order[j] : -1;
    d.headroom_ms = H;
    d.pred_critical_only_ms = R.y0;
    d.evaluated = n_eval;
    d.key = R.key;
    d.index = R.key & ((1ull << 40) - 1);
    if (!(R.y0 <= H)) {  // drop mechanism
        d.status = ABACUS_DECIDE_DROP;
        d.pred_ms = R.y0;
        d.total_ops = 0;
    } else {
        d.status = ABACUS_DECIDE_OK;
        d.pred_ms = R.y_best;
        d.total_ops = R.total_ops;
        for (int j = 0; j < k; j++) d.end_op[order[j]] = R.end_op[j];
    }
    return d;
}
}  // namespace

extern "C" {

int abacus_abi_version(void) { return ABACUS_ABI_VERSION; }

int abacus_create(int device, int32_t n_models, const int32_t* ops_per_model, int32_t k_max, abacus_ctx** out) {
    if (!out || !ops_per_model) return ABACUS_E_INVALID;
    if (n_models < 1 || n_models > 64 || k_max != ABACUS_K_MAX) return ABACUS_E_INVALID;
    for (int i = 0; i < n_models; i++)
        if (ops_per_model[i] < 1 || ops_per_model[i] > 32767) return ABACUS_E_INVALID;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return ABACUS_E_DEVICE;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return ABACUS_E_CUDA;
    if (prop.major != 10 || prop.minor != 0) return ABACUS_E_DEVICE;  // sm_100 only: no fallback
    if (cudaSetDevice(device) != cudaSuccess) return ABACUS_E_CUDA;
    abacus_ctx* c = new abacus_ctx();
    c->device = device;
    c->nsm = prop.multiProcessorCount;
    c->n_models = n_models;
    c->D = n_models + 4 * ABACUS_K_MAX;
    c->L.assign(ops_per_model, ops_per_model + n_models);
    bool ok = cudaStreamCreateWithFlags(&c->own_stream, cudaStreamNonBlocking) == cudaSuccess &&
              cudaMalloc(&c->S, sizeof(Scratch)) == cudaSuccess &&
              cudaMemset(c->S, 0, sizeof(Scratch)) == cudaSuccess &&
              cudaHostAlloc(&c->host_result, sizeof(MappedRec), cudaHostAllocMapped) == cudaSuccess &&
              cudaHostGetDevicePointer(&c->dev_result, c->host_result, 0) == cudaSuccess &&
              cudaEventCreate(&c->ev0) == cudaSuccess && cudaEventCreate(&c->ev1) == cudaSuccess;
    if (ok) {
        const float nan = NAN;
        ok = cudaMemcpy(&c->S->y0, &nan, sizeof(float), cudaMemcpyHostToDevice) == cudaSuccess &&
             cudaMalloc(&c->d_L, sizeof(int32_t) * (size_t)n_models) == cudaSuccess &&
             cudaMemcpy(c->d_L, ops_per_model, sizeof(int32_t) * (size_t)n_models, cudaMemcpyHostToDevice) ==
                 cudaSuccess;
    }
    c->stream = c->own_stream;
    if (ok) memset(c->host_result, 0, sizeof(MappedRec));
    if (!ok) {
        abacus_destroy(c);
        return ABACUS_E_CUDA;
    }
    *out = c;
    return ABACUS_OK;
}

void abacus_destroy(abacus_ctx* c) {
    if (!c) return;
    cudaSetDevice(c->device);
    if (c->stream) cudaStreamSynchronize(c->stream);
    if (c->own_stream) cudaStreamSynchronize(c->own_stream);
    cudaFree(c->S);
    cudaFree(c->d_w1b1);
    cudaFree(c->d_blob[0]);
    cudaFree(c->d_blob[1]);
    if (c->host_result) cudaFreeHost(c->host_result);
    if (c->h_out) cudaFreeHost(c->h_out);
    cudaFree(c->d_decs);
    cudaFree(c->d_segs);
    cudaFree(c->d_acc);
    cudaFree(c->d_y0);
    cudaFree(c->d_out);
    if (c->h_raw) cudaFreeHost(c->h_raw);
    cudaFree(c->d_raw);
    if (c->h_a1) cudaFreeHost(c->h_a1);
    cudaFree(c->d_a1);
    cudaFree(c->d_L);
    cudaFree(c->d_pairs);
    if (c->h_wdecs) cudaFreeHost(c->h_wdecs);
    if (c->h_wsegs) cudaFreeHost(c->h_wsegs);
    cudaFree(c->d_wsegs);
    cudaFree(c->d_mailbox);
    cudaFree(c->t_p);
    cudaFree(c->t_m);
    cudaFree(c->t_v);
    cudaFree(c->t_partial);
    cudaFree(c->t_loss_part);
    cudaFree(c->t_loss);
    cudaFree(c->t_ticket);
    if (c->ev0) cudaEventDestroy(c->ev0);
    if (c->ev1) cudaEventDestroy(c->ev1);
    if (c->own_stream) cudaStreamDestroy(c->own_stream);
    delete c;
}

const char* abacus_last_error(const abacus_ctx* c) { return c ? c->err.c_str() : "null ctx"; }

uint64_t abacus_kernel_launches(const abacus_ctx* c) { return c ? c->launches : 0; }

float abacus_last_kernel_ms(const abacus_ctx* c) {
    if (!c || !c->timed) return -1.0f;
    float ms = -1.0f;
    if (cudaEventSynchronize(c->ev1) != cudaSuccess) return -1.0f;
    if (cudaEventElapsedTime(&ms, c->ev0, c->ev1) != cudaSuccess) return -1.0f;
    return ms;
}

int abacus_load_predictor(abacus_ctx* c, const float* params, size_t n_params, int precision) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    const size_t want = (size_t)kHidden * c->D + 2 * kHidden * kHidden + 4 * kHidden + 1;
    if (!params || n_params != want)
        return fail(c, ABACUS_E_INVALID, "n_params=%zu, expected %zu for D=%d", n_params, want, c->D);
    if (precision != ABACUS_FP32 && precision != ABACUS_BF16 && precision != ABACUS_FP16)
        return fail(c, ABACUS_E_INVALID, "unknown precision %d", precision);
    for (size_t i = 0; i < n_params; i++)
        if (!std::isfinite(params[i])) return fail(c, ABACUS_E_INVALID, "param %zu is not finite", i);
    CUDA_TRY(c, cudaSetDevice(c->device));
    // async predict / search work queued on any stream may still read the old
    // weights (W2..W4 travel by value, W1/b1 and the blobs by pointer): finish
    // it before the device copies are overwritten or freed
    CUDA_TRY(c, cudaDeviceSynchronize());
    c->params.assign(params, params + n_params);
    const int D = c->D;
    const float* p = c->params.data();
    if (!c->d_w1b1) CUDA_TRY(c, cudaMalloc(&c->d_w1b1, sizeof(float) * (kHidden * D + kHidden)));
    CUDA_TRY(c, cudaMemcpy(c->d_w1b1, p, sizeof(float) * (kHidden * D + kHidden), cudaMemcpyHostToDevice));
    const float* q = p + kHidden * D + kHidden;
    memcpy(&c->w234.W2[0][0], q, sizeof(float) * kHidden * kHidden);
    q += kHidden * kHidden;
    memcpy(c->w234.b2, q, sizeof(float) * kHidden);
    q += kHidden;
    memcpy(&c->w234.W3[0][0], q, sizeof(float) * kHidden * kHidden);
    q += kHidden * kHidden;
    memcpy(c->w234.b3, q, sizeof(float) * kHidden);
    q += kHidden;
    memcpy(c->w234.w4, q, sizeof(float) * kHidden);
    q += kHidden;
    c->w234.b4 = *q;
    if (D == 24) {
        memcpy(&c->w1p.W1[0][0], p, sizeof(float) * kHidden * 24);
        memcpy(c->w1p.b1, p + kHidden * 24, sizeof(float) * kHidden);
    }
    for (int fmt = 0; fmt < 2; fmt++) {
        float l1s = 1.0f;
        TcWeights tw{};
        std::vector<uint8_t> blob = build_blob(c, fmt, &l1s, &tw.b4);
        if (c->d_blob[fmt]) cudaFree(c->d_blob[fmt]);
        CUDA_TRY(c, cudaMalloc(&c->d_blob[fmt], blob.size()));
        CUDA_TRY(c, cudaMemcpy(c->d_blob[fmt], blob.data(), blob.size(), cudaMemcpyHostToDevice));
        tw.fmt = fmt;
        tw.nch_hidden = fmt == 0 ? 3 : 5;
        tw.nch_out = fmt == 0 ? 3 : 5;
        tw.bytes = (uint32_t)blob.size();
        tw.l1_scale = l1s;
        tw.blob = c->d_blob[fmt];
        c->tw[fmt] = tw;
    }
    c->precision = precision;
    c->loaded = true;
    return ABACUS_OK;
}

int abacus_encode_candidates(abacus_ctx* c, const abacus_grid_t* grid, uint64_t first, uint64_t count,
                             int16_t* d_features, void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    uint64_t T = 0;
    int rc = validate_grid(c, grid, &T);
    if (rc) return rc;
    if (first > T || count > T - first) return fail(c, ABACUS_E_INVALID, "range beyond T=%llu", (unsigned long long)T);
    if (count && !d_features) return fail(c, ABACUS_E_INVALID, "d_features is NULL");
    CUDA_TRY(c, cudaSetDevice(c->device));
    const Plan P = plan_whole_grid(c->n_models, c->D, grid, T);
    CUDA_TRY(c, launch_encode_grid(P, first, count, d_features, c->nsm, pick_stream(c, stream)));
    if (count) c->launches++;
    return ABACUS_OK;
}

int abacus_encode_groups(abacus_ctx* c, const abacus_group_t* d_groups, uint64_t count, int16_t* d_features,
                         uint32_t* d_bad, void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (count && (!d_groups || !d_features)) return fail(c, ABACUS_E_INVALID, "NULL device buffer");
    static_assert(sizeof(abacus_group_t) == 4 + 4 * 5 * 4, "group record layout");
    CUDA_TRY(c, cudaSetDevice(c->device));
    CUDA_TRY(c, launch_encode_groups(d_groups, count, c->n_models, c->D, d_features, d_bad, c->nsm,
                                     pick_stream(c, stream)));
    if (count) c->launches++;
    return ABACUS_OK;
}

int abacus_predict_batch(abacus_ctx* c, const int16_t* d_features, uint64_t count, float* d_latency_ms,
                         void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->loaded) return fail(c, ABACUS_E_NOT_LOADED, "no predictor loaded");
    if (count && (!d_features || !d_latency_ms)) return fail(c, ABACUS_E_INVALID, "NULL device buffer");
    CUDA_TRY(c, cudaSetDevice(c->device));
    cudaStream_t st = pick_stream(c, stream);
    if (c->precision == ABACUS_FP32) {
        CUDA_TRY(c, launch_predict_fp32(c->w234, c->D == 24 ? &c->w1p : nullptr, c->d_w1b1, c->D, d_features, count,
                                        d_latency_ms, c->nsm, st));
    } else {
        if (c->D > 31) return fail(c, ABACUS_E_INVALID, "tensor predict supports D <= 31 (N <= 15 models)");
        const int fmt = c->precision == ABACUS_FP16 ? 0 : 1;
        CUDA_TRY(c, launch_predict_tc(c->tw[fmt], c->w234, c->d_w1b1, c->D, d_features, count, d_latency_ms, c->nsm, st));
    }
    if (count) c->launches++;
    return ABACUS_OK;
}

int abacus_select_group(abacus_ctx* c, const abacus_grid_t* grid, uint64_t first, uint64_t count,
                        const float* d_latency_ms, float headroom_ms, unsigned long long* d_best_key,
                        void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    uint64_t T = 0;
    int rc = validate_grid(c, grid, &T);
    if (rc) return rc;
    if (first > T || count > T - first) return fail(c, ABACUS_E_INVALID, "range beyond T");
    if (!d_best_key || (count && !d_latency_ms)) return fail(c, ABACUS_E_INVALID, "NULL device buffer");
    if (std::isnan(headroom_ms)) return fail(c, ABACUS_E_INVALID, "headroom is NaN");
    CUDA_TRY(c, cudaSetDevice(c->device));
    const Plan P = plan_whole_grid(c->n_models, c->D, grid, T);
    CUDA_TRY(c, launch_select(P, first, count, d_latency_ms, headroom_ms, d_best_key, c->nsm,
                              pick_stream(c, stream)));
    if (count) c->launches++;
    return ABACUS_OK;
}

int abacus_search(abacus_ctx* c, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                  int32_t space, uint64_t grid_budget, abacus_decision_t* out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!out) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (space < ABACUS_SPACE_GRID || space > ABACUS_SPACE_AUTO) return fail(c, ABACUS_E_INVALID, "bad space");
    int32_t order[ABACUS_K_MAX];
    float H = 0.0f;
    abacus_grid_t g{};
    uint64_t T = 0;
    int rc = decision_slots(c, q, k, now_ms, inflight_pred_ms, order, &H, &g, &T);
    if (rc) return rc;
    const bool chain = space == ABACUS_SPACE_CHAIN || (space == ABACUS_SPACE_AUTO && T > grid_budget);
    // the plan is built in place (the segment table is written once, not returned by value)
    Plan P;
    const PlanSink put{&P};
    uint64_t n_eval = 0;
    if (chain) {
        plan_chain_into(static_cast<PlanHdr&>(P), put, c->n_models, c->D, &g, H, &n_eval);
    } else {
        plan_grid_segments_into(static_cast<PlanHdr&>(P), put, c->n_models, c->D, &g, T, 0, T, H);
        n_eval = P.n_eval;
    }
    P.want_y0 = 1;
    P.mapped = c->dev_result;
    P.seq = next_seq(c);
    CUDA_TRY(c, cudaSetDevice(c->device));
    rc = launch_fused(c, P);
    if (rc) return rc;
    Result R;
    rc = wait_result(c, P.seq, &R);
    if (rc) return rc;
    host_decode(P, R);
    *out = assemble_decision(R, order, k, H, n_eval);
    return ABACUS_OK;
}


int abacus_search_batch(abacus_ctx* c, const abacus_query_t* q, const int32_t* k, const double* now_ms,
                        const double* inflight_pred_ms, int32_t n, int32_t space, uint64_t grid_budget,
                        abacus_decision_t* out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!q || !k || !now_ms || !inflight_pred_ms || !out) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (n < 1 || n > ABACUS_BATCH_MAX) return fail(c, ABACUS_E_INVALID, "n=%d outside [1,%d]", n, ABACUS_BATCH_MAX);
    if (space < ABACUS_SPACE_GRID || space > ABACUS_SPACE_AUTO) return fail(c, ABACUS_E_INVALID, "bad space");
    if (!c->loaded) return fail(c, ABACUS_E_NOT_LOADED, "no predictor loaded");
    if (c->precision == ABACUS_FP32) {
        // the fp32 SIMT path has no batched kernel: one fused launch per decision.
        // Every decision is validated (a1) first and the results go to a scratch
        // array, so an error names its decision and leaves `out` untouched.
        for (int32_t i = 0; i < n; i++) {
            int32_t order[ABACUS_K_MAX];
            float H = 0.0f;
            abacus_grid_t g{};
            const int rc = decision_slots(c, q + 4 * (size_t)i, k[i], now_ms[i], inflight_pred_ms[i], order, &H, &g);
            if (rc) {
                c->err = "decision " + std::to_string(i) + ": " + c->err;
                return rc;
            }
        }
        std::vector<abacus_decision_t> tmp((size_t)n);
        for (int32_t i = 0; i < n; i++) {
            const int rc = abacus_search(c, q + 4 * (size_t)i, k[i], now_ms[i], inflight_pred_ms[i], space,
                                         grid_budget, &tmp[(size_t)i]);
            if (rc) {
                c->err = "decision " + std::to_string(i) + ": " + c->err;
                return rc;
            }
        }
        memcpy(out, tmp.data(), sizeof(abacus_decision_t) * (size_t)n);
        return ABACUS_OK;
    }
    CUDA_TRY(c, cudaSetDevice(c->device));
    int rc = grow_batch(c, n);
    if (rc) return rc;
    // The host copies the decisions to pinned memory and bounds the widest digit
    // (it selects the tensor kernels' split layer-1 layout); a1, validation and
    // planning run on the device, one thread per decision (batch_plan_kernel).
    // A failing decision is reported by its index (the first one) after the
    // launch; no output is written then.
    uint32_t maxcnt = 0;
    for (int32_t i = 0; i < n; i++) {
        BatchRaw& rw = c->h_raw[i];
        const int32_t ki = k[i];
        const int32_t kc = ki < 0 ? 0 : (ki > ABACUS_K_MAX ? ABACUS_K_MAX : ki);
        memcpy(rw.q, q + 4 * (size_t)i, sizeof(abacus_query_t) * ABACUS_K_MAX);
        rw.now = now_ms[i];
        rw.infl = inflight_pred_ms[i];
        rw.k = ki;
        // widest digit = L - next_op + 1 over the non-critical queries (the critical
        // query's slot is fixed): the same bound a single round derives from its
        // plan, so a batch picks the same layer-1 layout (and the same arithmetic)
        // as abacus_search of each of its rounds. The critical query is the
        // smallest headroom, ties to the smaller model id (a1, reading c10).
        int crit = 0;
        double hc = 0.0;
        for (int j = 0; j < kc; j++) {
            const abacus_query_t& a = rw.q[j];
            const double h = (a.qos_ms - (rw.now - a.t_start_ms)) - rw.infl;
            if (j == 0 || h < hc || (h == hc && a.model_id < rw.q[crit].model_id)) {
                crit = j;
                hc = h;
            }
        }
        for (int j = 0; j < kc; j++) {
            const abacus_query_t& a = rw.q[j];
            if (j != crit && a.model_id >= 1 && a.model_id <= c->n_models && a.next_op >= 1) {
                const int32_t w = c->L[a.model_id - 1] - a.next_op + 1;
                if (w > 0 && (uint32_t)w > maxcnt) maxcnt = (uint32_t)w;
            }
        }
    }
    cudaStream_t st = c->stream;
    CUDA_TRY(c, cudaMemcpyAsync(c->d_raw, c->h_raw, (size_t)n * sizeof(BatchRaw), cudaMemcpyHostToDevice, st));
    // one warp per block: the per-thread planner is latency-bound, so spread it over every SM
    batch_plan_kernel<<<(n + 31) / 32, 32, 0, st>>>(c->d_raw, n, c->n_models, c->D, c->d_L, space, grid_budget,
                                                       c->d_decs, c->d_segs, c->d_pairs, c->d_a1);
    batch_scan_kernel<<<1, kScanThreads, 0, st>>>(c->d_decs, c->d_pairs, n);
    CUDA_TRY(c, cudaGetLastError());
    c->launches += 2;
    CUDA_TRY(c, cudaMemsetAsync(c->d_acc, 0, (size_t)n * sizeof(BatchAcc), st));
    CUDA_TRY(c, cudaMemsetAsync(c->d_y0, 0xFF, (size_t)n * sizeof(float), st));  // NaN
    if (c->timed) cudaEventRecord(c->ev0, st);
    const int fmt = c->precision == ABACUS_FP16 ? 0 : 1;
    // the exact pair count is only known on the device: the grid covers every SM
    const uint64_t pairs_ub = ~0ull >> 8;
    cudaError_t e = launch_batch_tc(c->d_decs, c->d_segs, n, c->d_pairs + n, pairs_ub, maxcnt, c->D, c->tw[fmt],
                                    c->d_w1b1, c->d_acc, c->d_y0, c->d_out, c->nsm, st);
    if (c->timed) cudaEventRecord(c->ev1, st);
    if (e != cudaSuccess) return fail(c, ABACUS_E_CUDA, "batched search launch: %s", cudaGetErrorString(e));
    c->launches += 2;
    CUDA_TRY(c, cudaMemcpyAsync(c->h_a1, c->d_a1, (size_t)n * sizeof(BatchA1), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(c, cudaMemcpyAsync(c->h_out, c->d_out, (size_t)n * sizeof(Result), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(c, cudaStreamSynchronize(st));
    for (int32_t i = 0; i < n; i++) {
        const int32_t er = c->h_a1[i].err;
        if (er) {
            a1_fail(c, er & 0xFF, (er >> 8) & 0xFF, (er >> 16) & 0xFF, q + 4 * (size_t)i, k[i]);
            c->err = "decision " + std::to_string(i) + ": " + c->err;
            return (er & 0xFF) == A1_DUP ? ABACUS_E_DUP_MODEL : ABACUS_E_INVALID;
        }
    }
    for (int32_t i = 0; i < n; i++)
        out[i] = assemble_decision(c->h_out[i], c->h_a1[i].order, k[i], c->h_a1[i].H, c->h_out[i].evaluated);
    return ABACUS_OK;
}

int abacus_search_mway(abacus_ctx* c, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                       int32_t ways, abacus_decision_t* out, int32_t* rounds_out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!out) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (ways < 1 || ways > 128) return fail(c, ABACUS_E_INVALID, "ways=%d outside [1,128]", ways);
    int32_t order[ABACUS_K_MAX];
    float H = 0.0f;
    abacus_grid_t g{};
    int rc = decision_slots(c, q, k, now_ms, inflight_pred_ms, order, &H, &g);
    if (rc) return rc;
    uint64_t n_chain = 0;
    Plan P = plan_chain(c->n_models, c->D, &g, H, &n_chain);
    P.mapped = c->dev_result;
    P.seq = next_seq(c);
    CUDA_TRY(c, cudaSetDevice(c->device));
    CUDA_TRY(c, launch_mway(P, c->w234, c->d_w1b1, ways, c->S, c->stream));
    c->launches++;
    Result R;
    rc = wait_result(c, P.seq, &R);
    if (rc) return rc;
    abacus_decision_t d{};
    d.critical = order[0];
    for (int j = 0; j < 4; j++) d.order[j] = j < k ? order[j] : -1;
    d.headroom_ms = H;
    d.pred_critical_only_ms = R.y0;
    d.pred_ms = R.y_best;
    d.evaluated = R.evaluated;
    d.key = R.key;
    d.index = R.key & ((1ull << 40) - 1);
    d.status = R.status;
    d.total_ops = R.total_ops;
    if (R.status == ABACUS_DECIDE_OK)
        for (int j = 0; j < k; j++) d.end_op[order[j]] = R.end_op[j];
    if (rounds_out) *rounds_out = (int32_t)R.pad;
    *out = d;
    return ABACUS_OK;
}

int abacus_search_grid(abacus_ctx* c, const abacus_grid_t* grid, float headroom_ms, uint64_t first, uint64_t count,
                       void* nccl_comm, abacus_decision_t* out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->loaded) return fail(c, ABACUS_E_NOT_LOADED, "no predictor loaded");
    if (!out) return fail(c, ABACUS_E_INVALID, "out is NULL");
    uint64_t T = 0;
    int rc = validate_grid(c, grid, &T);
    if (rc) return rc;
    if (first > T || count > T - first) return fail(c, ABACUS_E_INVALID, "range beyond T");
    if (std::isnan(headroom_ms)) return fail(c, ABACUS_E_INVALID, "headroom is NaN");
    CUDA_TRY(c, cudaSetDevice(c->device));
    Plan P = plan_grid_segments(c->n_models, c->D, grid, T, first, first + count, headroom_ms);
    const uint32_t seq = next_seq(c);
    PeerComm* pc = nccl_comm ? as_peer(nccl_comm) : nullptr;
    // with an NCCL combine the finalize kernel publishes; with a peer combine the
    // fused kernel's last CTA combines and publishes itself
    const bool nccl_combine = nccl_comm && !pc;
    P.mapped = nccl_combine ? nullptr : c->dev_result;
    P.seq = seq;
    if (nccl_comm) {
        int nranks = 0, rank = 0;
        rc = comm_shape(c, nccl_comm, &nranks, &rank);
        if (rc) return rc;
    }
    if (pc) {
        P.peer = pc->d_comb;
        P.peer_seq = ++pc->seq;
    }
    rc = launch_fused(c, P);
    if (rc) return rc;
    if (nccl_combine) {
        rc = combine_over_comm(c, nccl_comm, seq);
        if (rc) return rc;
    }
    Result R;
    rc = wait_result(c, seq, &R);
    if (rc) return rc;
    if (R.status == 3) return fail(c, ABACUS_E_NCCL, "peer combine: a rank's record did not arrive in time");
    if (!nccl_comm) host_decode(P, R);
    *out = sweep_decision(R, grid->k, headroom_ms);
    return ABACUS_OK;
}

// Per-decision sharded search: every rank runs a1 on the same
// inputs (deterministic, so every rank derives the same grid, order and H), a
// GRID decision's index space is split into the contiguous shard of this rank,
// the fused kernel searches it, and one all-gather + combine_results gives every
// rank the global record; the drop test uses y(0) from the rank whose shard holds
// index 0.  A CHAIN decision (<= a few thousand candidates: launch-bound) is
// searched whole on every rank, with no collective.
int abacus_search_sharded(abacus_ctx* c, const abacus_query_t* q, int32_t k, double now_ms, double inflight_pred_ms,
                          int32_t space, uint64_t grid_budget, void* nccl_comm, abacus_decision_t* out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!out) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (space < ABACUS_SPACE_GRID || space > ABACUS_SPACE_AUTO) return fail(c, ABACUS_E_INVALID, "bad space");
    if (!nccl_comm) return abacus_search(c, q, k, now_ms, inflight_pred_ms, space, grid_budget, out);
    int32_t order[ABACUS_K_MAX];
    float H = 0.0f;
    abacus_grid_t g{};
    uint64_t T = 0;
    int rc = decision_slots(c, q, k, now_ms, inflight_pred_ms, order, &H, &g, &T);
    if (rc) return rc;
    const bool chain = space == ABACUS_SPACE_CHAIN || (space == ABACUS_SPACE_AUTO && T > grid_budget);
    if (chain) return abacus_search(c, q, k, now_ms, inflight_pred_ms, space, grid_budget, out);
    int nranks = 0, rank = 0;
    rc = comm_shape(c, nccl_comm, &nranks, &rank);
    if (rc) return rc;
    const uint64_t first = (uint64_t)rank * T / (uint64_t)nranks;  // T < 2^40, nranks <= 64: no overflow
    const uint64_t last = (uint64_t)(rank + 1) * T / (uint64_t)nranks;
    Plan P;
    plan_grid_segments_into(static_cast<PlanHdr&>(P), PlanSink{&P}, c->n_models, c->D, &g, T, first, last, H);
    PeerComm* pc = as_peer(nccl_comm);
    P.mapped = pc ? c->dev_result : nullptr;  // the finalize kernel (NCCL) or the last CTA (peer) publishes
    P.seq = next_seq(c);
    if (pc) {
        P.peer = pc->d_comb;
        P.peer_seq = ++pc->seq;
    }
    CUDA_TRY(c, cudaSetDevice(c->device));
    rc = launch_fused(c, P);
    if (rc) return rc;
    if (!pc) {
        rc = combine_over_comm(c, nccl_comm, P.seq);
        if (rc) return rc;
    }
    Result R;
    rc = wait_result(c, P.seq, &R);
    if (rc) return rc;
    if (R.status == 3) return fail(c, ABACUS_E_NCCL, "peer combine: a rank's record did not arrive in time");
    *out = assemble_decision(R, order, k, H, R.evaluated);
    return ABACUS_OK;
}

// a6 on the host (no device work): the same combine_results as the finalize
// kernel, over per-rank sweep decisions.
int abacus_combine_decisions(const abacus_decision_t* per_rank, int32_t nranks, int32_t drop_test,
                             abacus_decision_t* out) {
    if (!per_rank || !out || nranks < 1 || nranks > 64) return ABACUS_E_INVALID;
    Result r[64];
    for (int32_t i = 0; i < nranks; i++) {
        const abacus_decision_t& d = per_rank[i];
        if (memcmp(&d.headroom_ms, &per_rank[0].headroom_ms, sizeof(float)) != 0) return ABACUS_E_INVALID;
        if (d.status != ABACUS_DECIDE_OK && d.status != ABACUS_DECIDE_NONE) return ABACUS_E_INVALID;
        if ((d.key == 0) != (d.status == ABACUS_DECIDE_NONE)) return ABACUS_E_INVALID;
        Result& R = r[i];
        R = Result{};
        R.key = d.key;
        R.y_best = d.pred_ms;
        R.y0 = d.pred_critical_only_ms;
        R.evaluated = d.evaluated;
        for (int j = 0; j < kKMax; j++) R.end_op[j] = d.end_op[j];
        R.total_ops = d.total_ops;
    }
    const Result R = combine_results(r, nranks);
    abacus_decision_t d = per_rank[0];
    d.key = R.key;
    d.index = R.key & ((1ull << 40) - 1);
    d.evaluated = R.evaluated;
    d.pred_critical_only_ms = R.y0;
    d.total_ops = R.key ? R.total_ops : 0;
    d.pred_ms = R.key ? R.y_best : NAN;
    for (int j = 0; j < 4; j++) d.end_op[j] = R.key ? R.end_op[j] : 0;
    d.status = R.key ? ABACUS_DECIDE_OK : ABACUS_DECIDE_NONE;
    if (drop_test && !(R.y0 <= d.headroom_ms)) {  // drop mechanism (reading c14)
        d.status = ABACUS_DECIDE_DROP;
        d.pred_ms = R.y0;
        d.total_ops = 0;
        for (int j = 0; j < 4; j++) d.end_op[j] = 0;
    }
    *out = d;
    return ABACUS_OK;
}

// ---- NEXT-4: what-if sweeps over bs / seqlen ---------------------------------
namespace {
int grow_whatif(abacus_ctx* c, int32_t n) {
    int rc = grow_batch(c, n);
    if (rc) return rc;
    if (n <= c->whatif_cap) return ABACUS_OK;
    if (c->h_wdecs) cudaFreeHost(c->h_wdecs);
    if (c->h_wsegs) cudaFreeHost(c->h_wsegs);
    cudaFree(c->d_wsegs);
    c->h_wdecs = nullptr;
    c->h_wsegs = nullptr;
    c->d_wsegs = nullptr;
    c->whatif_cap = 0;
    int32_t cap = 256;  // own capacity: a large earlier decision batch must not size the plan staging
    while (cap < n) cap *= 2;
    CUDA_TRY(c, cudaHostAlloc(&c->h_wdecs, (size_t)cap * sizeof(BatchDec), cudaHostAllocDefault));
    CUDA_TRY(c, cudaHostAlloc(&c->h_wsegs, (size_t)cap * kMaxSeg * sizeof(SegP), cudaHostAllocDefault));
    CUDA_TRY(c, cudaMalloc(&c->d_wsegs, (size_t)cap * kMaxSeg * sizeof(SegP)));
    c->whatif_cap = cap;
    return ABACUS_OK;
}

// segment sink into a what-if variant's fixed slots (host staging)
struct ArraySink {
    SegP* segs;
    __host__ __device__ void operator()(int i, const SegP& sg) const { segs[i] = sg; }
};
}  // namespace

// What-if sweep (the load balancer picks
// batch sizes at run time and inputs vary in length): the grid's candidates
// under every (bs, seqlen) variant.  Tensor paths: every variant is one plan
// of a single batched search launch (the NEXT-4 batch kernel), planned on the
// host; fp32: one fused launch per variant.
int abacus_search_whatif(abacus_ctx* c, const abacus_grid_t* grid, const abacus_variant_t* variants, int32_t n_var,
                         float headroom_ms, abacus_decision_t* per_variant, abacus_decision_t* best,
                         int32_t* best_variant) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->loaded) return fail(c, ABACUS_E_NOT_LOADED, "no predictor loaded");
    if (!variants || (!per_variant && !best)) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (n_var < 1 || n_var > ABACUS_WHATIF_MAX)
        return fail(c, ABACUS_E_INVALID, "n_var=%d outside [1,%d]", n_var, ABACUS_WHATIF_MAX);
    if (std::isnan(headroom_ms)) return fail(c, ABACUS_E_INVALID, "headroom is NaN");
    uint64_t T = 0;
    int rc = validate_grid(c, grid, &T);
    if (rc) return rc;
    if ((unsigned __int128)T * (unsigned __int128)n_var >= ((unsigned __int128)1 << 40))
        return fail(c, ABACUS_E_INVALID, "n_var * |grid| >= 2^40");
    for (int32_t v = 0; v < n_var; v++)
        for (int j = 0; j < grid->k; j++) {
            const int32_t b = variants[v].batch[j], l = variants[v].seqlen[j];
            if (b < 1 || b > 32767 || l < 0 || l > 32767)
                return fail(c, ABACUS_E_INVALID, "variant %d slot %d: batch %d / seqlen %d", v, j, b, l);
        }
    CUDA_TRY(c, cudaSetDevice(c->device));
    auto variant_grid = [&](int32_t v) {
        abacus_grid_t g = *grid;
        for (int j = 0; j < g.k; j++) {
            g.slot[j].batch = variants[v].batch[j];
            g.slot[j].seqlen = variants[v].seqlen[j];
        }
        return g;
    };
    std::vector<Result> res((size_t)n_var);
    // Large variant grids run one fused single-search launch each: at >= 2^24
    // candidates the ~10 us launch + prologue is < 10 % of a variant, and the
    // single kernel's inner loop (plan in the constant bank, unrolled by two)
    // is ~1.2x the batch kernel's per candidate on the same grid
    // (tools/exp_whatif.py).  Smaller grids share one batched launch.
    const bool per_launch = c->precision == ABACUS_FP32 || T >= (1ull << 24);
    if (per_launch) {
        for (int32_t v = 0; v < n_var; v++) {
            const abacus_grid_t g = variant_grid(v);
            Plan P = plan_grid_segments(c->n_models, c->D, &g, T, 0, T, headroom_ms);
            P.mapped = c->dev_result;
            P.seq = next_seq(c);
            rc = launch_fused(c, P);
            if (rc) return rc;
            rc = wait_result(c, P.seq, &res[(size_t)v]);
            if (rc) return rc;
            host_decode(P, res[(size_t)v]);
        }
    } else {
        rc = grow_whatif(c, n_var);
        if (rc) return rc;
        uint64_t pairs = 0;
        uint32_t maxcnt = 0;
        for (int32_t v = 0; v < n_var; v++) {
            const abacus_grid_t g = variant_grid(v);
            BatchDec& bd = c->h_wdecs[v];
            SegP* segs = c->h_wsegs + (size_t)kMaxSeg * v;
            plan_grid_segments_into(bd.h, ArraySink{segs}, c->n_models, c->D, &g, T, 0, T, headroom_ms);
            bd.h.want_y0 = 1;
            bd.h.mapped = nullptr;
            bd.h.trace = nullptr;
            bd.pair0 = pairs;
            bd.seg0 = (uint32_t)(kMaxSeg * v);
            pairs += (bd.h.n_tiles + 1) / 2;  // tiles padded to pairs, as for decision batches
            for (int i = 0; i < bd.h.n_seg; i++)
                for (int j = 0; j < kKMax; j++) maxcnt = segs[i].cnt[j] > maxcnt ? segs[i].cnt[j] : maxcnt;
        }
        cudaStream_t st = c->stream;
        CUDA_TRY(c, cudaMemcpyAsync(c->d_decs, c->h_wdecs, (size_t)n_var * sizeof(BatchDec), cudaMemcpyHostToDevice,
                                    st));
        CUDA_TRY(c, cudaMemcpyAsync(c->d_wsegs, c->h_wsegs, (size_t)n_var * kMaxSeg * sizeof(SegP),
                                    cudaMemcpyHostToDevice, st));
        CUDA_TRY(c, cudaMemcpyAsync(c->d_pairs + n_var, &pairs, sizeof(uint64_t), cudaMemcpyHostToDevice, st));
        CUDA_TRY(c, cudaMemsetAsync(c->d_acc, 0, (size_t)n_var * sizeof(BatchAcc), st));
        CUDA_TRY(c, cudaMemsetAsync(c->d_y0, 0xFF, (size_t)n_var * sizeof(float), st));  // NaN
        if (c->timed) cudaEventRecord(c->ev0, st);
        const int fmt = c->precision == ABACUS_FP16 ? 0 : 1;
        cudaError_t e = launch_batch_tc(c->d_decs, c->d_wsegs, n_var, c->d_pairs + n_var, pairs, maxcnt, c->D,
                                        c->tw[fmt], c->d_w1b1, c->d_acc, c->d_y0, c->d_out, c->nsm, st);
        if (c->timed) cudaEventRecord(c->ev1, st);
        if (e != cudaSuccess) return fail(c, ABACUS_E_CUDA, "what-if search launch: %s", cudaGetErrorString(e));
        c->launches += 2;
        CUDA_TRY(c, cudaMemcpyAsync(c->h_out, c->d_out, (size_t)n_var * sizeof(Result), cudaMemcpyDeviceToHost, st));
        CUDA_TRY(c, cudaStreamSynchronize(st));
        memcpy(res.data(), c->h_out, (size_t)n_var * sizeof(Result));
    }
    // the global best: max (sum_n, v T + t) over the variants (NEXT-4 reading: the
    // variant is the most significant index digit)
    uint64_t bkey = 0;
    int32_t bv = -1;
    for (int32_t v = 0; v < n_var; v++) {
        const Result& R = res[(size_t)v];
        if (per_variant) per_variant[v] = sweep_decision(R, grid->k, headroom_ms);
        if (!R.key) continue;
        const uint64_t lifted = (R.key & ~((1ull << 40) - 1)) | ((uint64_t)v * T + (R.key & ((1ull << 40) - 1)));
        if (lifted > bkey) {
            bkey = lifted;
            bv = v;
        }
    }
    if (best) {
        Result R{};
        uint64_t ev = 0;
        for (int32_t v = 0; v < n_var; v++) ev += res[(size_t)v].evaluated;
        if (bv >= 0) R = res[(size_t)bv];
        R.y0 = res[0].y0;
        R.evaluated = ev;
        abacus_decision_t d = sweep_decision(R, grid->k, headroom_ms);
        d.key = bkey;
        d.index = bkey & ((1ull << 40) - 1);
        *best = d;
    }
    if (best_variant) *best_variant = bv;
    return ABACUS_OK;
}

// ---- NEXT-3: training (kernels_train.cu) ----------------------------------
static constexpr uint64_t kTrainMaxBatch = ABACUS_TRAIN_MAX_BATCH;
static constexpr unsigned kTrainMaxBlocks = (unsigned)(kTrainMaxBatch / 128);

int abacus_train_begin(abacus_ctx* c, const float* params, size_t n_params, const abacus_adam_t* opt) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!params || !opt) return fail(c, ABACUS_E_INVALID, "NULL argument");
    const int np = train_n_params(c->D);
    if (n_params != (size_t)np) return fail(c, ABACUS_E_INVALID, "n_params=%zu, expected %d", n_params, np);
    for (size_t i = 0; i < n_params; i++)
        if (!std::isfinite(params[i])) return fail(c, ABACUS_E_INVALID, "non-finite parameter %zu", i);
    if (!(opt->beta1 >= 0.0f && opt->beta1 < 1.0f && opt->beta2 >= 0.0f && opt->beta2 < 1.0f && opt->eps > 0.0f))
        return fail(c, ABACUS_E_INVALID, "bad Adam hyper-parameters");
    CUDA_TRY(c, cudaSetDevice(c->device));
    if (!c->t_p) {
        CUDA_TRY(c, cudaMalloc(&c->t_p, np * sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_m, np * sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_v, np * sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_partial, (size_t)kTrainMaxBlocks * np * sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_loss_part, kTrainMaxBlocks * sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_loss, sizeof(float)));
        CUDA_TRY(c, cudaMalloc(&c->t_ticket, sizeof(unsigned)));
        CUDA_TRY(c, cudaMemset(c->t_ticket, 0, sizeof(unsigned)));
    }
    CUDA_TRY(c, cudaMemcpyAsync(c->t_p, params, np * sizeof(float), cudaMemcpyHostToDevice, c->stream));
    CUDA_TRY(c, cudaMemsetAsync(c->t_m, 0, np * sizeof(float), c->stream));
    CUDA_TRY(c, cudaMemsetAsync(c->t_v, 0, np * sizeof(float), c->stream));
    CUDA_TRY(c, cudaMemsetAsync(c->t_loss, 0xFF, sizeof(float), c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    c->adam = *opt;
    c->train_t = 0;
    c->training = true;
    return ABACUS_OK;
}

namespace {
int train_one(abacus_ctx* c, const int16_t* d_x, const float* d_y, uint64_t count, float lr, float* d_grad,
              float* d_loss, cudaStream_t st) {
    c->train_t++;
    TrainArgs A{};
    A.p = c->t_p;
    A.m = c->t_m;
    A.v = c->t_v;
    A.x = d_x;
    A.t = d_y;
    A.count = count;
    A.D = c->D;
    A.inv_count = (float)(1.0 / (double)count);
    A.partial = c->t_partial;
    A.loss_part = c->t_loss_part;
    A.ticket = c->t_ticket;
    A.loss_last = c->t_loss;
    A.loss_out = d_loss;
    A.grad_out = d_grad;
    A.lr = lr;
    A.beta1 = c->adam.beta1;
    A.beta2 = c->adam.beta2;
    A.eps = c->adam.eps;
    A.bc1 = (float)(1.0 - std::pow((double)c->adam.beta1, (double)c->train_t));
    A.bc2 = (float)(1.0 - std::pow((double)c->adam.beta2, (double)c->train_t));
    const cudaError_t e = launch_train_step(A, st);
    if (e != cudaSuccess) return fail(c, ABACUS_E_CUDA, "train step launch: %s", cudaGetErrorString(e));
    c->launches++;
    return ABACUS_OK;
}
}  // namespace

int abacus_train_step(abacus_ctx* c, const int16_t* d_features, const float* d_latency_ms, uint64_t count,
                      float lr, float* d_grad, void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->training) return fail(c, ABACUS_E_NOT_LOADED, "abacus_train_begin not called");
    if (!d_features || !d_latency_ms) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (count < 1 || count > kTrainMaxBatch) return fail(c, ABACUS_E_INVALID, "count=%llu", (unsigned long long)count);
    if (!(lr >= 0.0f) || !std::isfinite(lr)) return fail(c, ABACUS_E_INVALID, "bad learning rate");
    CUDA_TRY(c, cudaSetDevice(c->device));
    return train_one(c, d_features, d_latency_ms, count, lr, d_grad, nullptr, pick_stream(c, stream));
}

int abacus_train_epoch(abacus_ctx* c, const int16_t* d_features, const float* d_latency_ms, uint64_t count,
                       uint32_t batch, float lr, float* d_losses, void* stream) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->training) return fail(c, ABACUS_E_NOT_LOADED, "abacus_train_begin not called");
    if (!d_features || !d_latency_ms) return fail(c, ABACUS_E_INVALID, "NULL argument");
    if (count < 1 || batch < 1 || batch > kTrainMaxBatch) return fail(c, ABACUS_E_INVALID, "count/batch");
    if (!(lr >= 0.0f) || !std::isfinite(lr)) return fail(c, ABACUS_E_INVALID, "bad learning rate");
    CUDA_TRY(c, cudaSetDevice(c->device));
    cudaStream_t st = pick_stream(c, stream);
    uint64_t step = 0;
    for (uint64_t s = 0; s < count; s += batch, step++) {
        const uint64_t n = count - s < batch ? count - s : batch;
        const int rc = train_one(c, d_features + s * (uint64_t)c->D, d_latency_ms + s, n, lr, nullptr,
                                 d_losses ? d_losses + step : nullptr, st);
        if (rc) return rc;
    }
    return ABACUS_OK;
}

int abacus_train_params(abacus_ctx* c, float* params_out, float* last_loss) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!c->training) return fail(c, ABACUS_E_NOT_LOADED, "abacus_train_begin not called");
    if (!params_out) return fail(c, ABACUS_E_INVALID, "NULL argument");
    CUDA_TRY(c, cudaSetDevice(c->device));
    CUDA_TRY(c, cudaDeviceSynchronize());
    CUDA_TRY(c, cudaMemcpy(params_out, c->t_p, train_n_params(c->D) * sizeof(float), cudaMemcpyDeviceToHost));
    if (last_loss) CUDA_TRY(c, cudaMemcpy(last_loss, c->t_loss, sizeof(float), cudaMemcpyDeviceToHost));
    return ABACUS_OK;
}

int abacus_nccl_unique_id(uint8_t* id128) {
    if (!id128) return ABACUS_E_INVALID;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId id;
    if (!nccl().ok || nccl().GetUniqueId(&id) != ncclSuccess) return ABACUS_E_NCCL;
    memcpy(id128, &id, 128);
    return ABACUS_OK;
}

int abacus_nccl_comm_init(abacus_ctx* c, int32_t nranks, int32_t rank, const uint8_t* id128, void** comm_out) {
    if (!c || !id128 || !comm_out || nranks < 1 || nranks > 64 || rank < 0 || rank >= nranks)
        return fail(c, ABACUS_E_INVALID, "bad NCCL init arguments");
    CUDA_TRY(c, cudaSetDevice(c->device));
    ncclUniqueId id;
    memcpy(&id, id128, 128);
    ncclComm_t comm;
    if (!nccl().ok) return fail(c, ABACUS_E_NCCL, "libnccl.so.2 not available");
    ncclResult_t nr = nccl().CommInitRank(&comm, nranks, id, rank);
    if (nr != ncclSuccess) return fail(c, ABACUS_E_NCCL, "ncclCommInitRank: %s", nccl().GetErrorString(nr));
    *comm_out = comm;
    return ABACUS_OK;
}

void abacus_nccl_comm_destroy(void* comm) {
    if (comm && nccl().ok) nccl().CommDestroy((ncclComm_t)comm);
}

// ---- a6 over peer memory ----------------------------------------------------
// blob: [0, 64) cudaIpcMemHandle_t of the mailbox, [64, 72) pid, [72, 80) the
// mailbox's device address in the exporting process, [80, 84) device ordinal,
// [84, 88) magic
static constexpr uint32_t kPeerMagic = 0x41425043u;  // "ABPC"

int abacus_peer_export(abacus_ctx* c, uint8_t* blob) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!blob) return fail(c, ABACUS_E_INVALID, "NULL argument");
    CUDA_TRY(c, cudaSetDevice(c->device));
    if (!c->d_mailbox) {
        CUDA_TRY(c, cudaMalloc(&c->d_mailbox, 2 * kPeerMax * sizeof(MappedRec)));
        CUDA_TRY(c, cudaMemset(c->d_mailbox, 0, 2 * kPeerMax * sizeof(MappedRec)));
    }
    memset(blob, 0, ABACUS_PEER_BLOB);
    cudaIpcMemHandle_t h;
    CUDA_TRY(c, cudaIpcGetMemHandle(&h, c->d_mailbox));
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    memcpy(blob, &h, 64);
    const uint64_t pid = (uint64_t)getpid(), addr = (uint64_t)(uintptr_t)c->d_mailbox;
    const int32_t dev = c->device;
    memcpy(blob + 64, &pid, 8);
    memcpy(blob + 72, &addr, 8);
    memcpy(blob + 80, &dev, 4);
    memcpy(blob + 84, &kPeerMagic, 4);
    return ABACUS_OK;
}

int abacus_peer_comm_init(abacus_ctx* c, int32_t nranks, int32_t rank, const uint8_t* blobs, void** comm_out) {
    if (!c) return ABACUS_E_INVALID;
    c->err.clear();
    if (!blobs || !comm_out || nranks < 1 || nranks > kPeerMax || rank < 0 || rank >= nranks)
        return fail(c, ABACUS_E_INVALID, "bad peer communicator arguments (1 <= nranks <= %d)", kPeerMax);
    if (!c->d_mailbox) return fail(c, ABACUS_E_INVALID, "abacus_peer_export was not called on this ctx");
    CUDA_TRY(c, cudaSetDevice(c->device));
    PeerComm* pc = new PeerComm();
    pc->ctx = c;
    pc->nranks = nranks;
    pc->rank = rank;
    PeerComb hc{};
    hc.nranks = nranks;
    hc.rank = rank;
    const char* e = getenv("ABACUS_PEER_TIMEOUT_MS");
    hc.timeout_ms = e && atoi(e) > 0 ? (uint32_t)atoi(e) : 10000u;
    hc.local = c->d_mailbox;
    auto cleanup = [&]() {
        for (void* p : pc->opened) cudaIpcCloseMemHandle(p);
        delete pc;
    };
    for (int32_t r = 0; r < nranks; r++) {
        const uint8_t* b = blobs + (size_t)r * ABACUS_PEER_BLOB;
        uint64_t pid, addr;
        int32_t dev;
        uint32_t magic;
        memcpy(&pid, b + 64, 8);
        memcpy(&addr, b + 72, 8);
        memcpy(&dev, b + 80, 4);
        memcpy(&magic, b + 84, 4);
        if (magic != kPeerMagic) {
            cleanup();
            return fail(c, ABACUS_E_INVALID, "rank %d: not a peer blob", r);
        }
        if (r == rank) {
            if (pid != (uint64_t)getpid() || addr != (uint64_t)(uintptr_t)c->d_mailbox) {
                cleanup();
                return fail(c, ABACUS_E_INVALID, "rank %d's blob is not this ctx's", r);
            }
            hc.dst[r] = c->d_mailbox;
        } else if (pid == (uint64_t)getpid()) {
            // same process (tests: two ctxs on one device): the address is valid
            // here; another device needs peer access
            if (dev != c->device) {
                const cudaError_t pe = cudaDeviceEnablePeerAccess(dev, 0);
                if (pe != cudaSuccess && pe != cudaErrorPeerAccessAlreadyEnabled) {
                    cleanup();
                    return fail(c, ABACUS_E_CUDA, "peer access to device %d: %s", dev, cudaGetErrorString(pe));
                }
                cudaGetLastError();
            }
            hc.dst[r] = reinterpret_cast<MappedRec*>((uintptr_t)addr);
        } else {
            cudaIpcMemHandle_t h;
            memcpy(&h, b, 64);
            void* ptr = nullptr;
            const cudaError_t oe = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
            if (oe != cudaSuccess) {
                cleanup();
                return fail(c, ABACUS_E_CUDA, "rank %d: cudaIpcOpenMemHandle: %s", r, cudaGetErrorString(oe));
            }
            pc->opened.push_back(ptr);
            hc.dst[r] = static_cast<MappedRec*>(ptr);
        }
    }
    if (cudaMalloc(&pc->d_comb, sizeof(PeerComb)) != cudaSuccess ||
        cudaMemcpy(pc->d_comb, &hc, sizeof(PeerComb), cudaMemcpyHostToDevice) != cudaSuccess) {
        cudaFree(pc->d_comb);
        cleanup();
        return fail(c, ABACUS_E_CUDA, "peer table allocation failed");
    }
    {
        std::lock_guard<std::mutex> lk(g_peer_mu);
        g_peer_comms.insert(pc);
    }
    *comm_out = pc;
    return ABACUS_OK;
}

void abacus_peer_comm_destroy(void* comm) {
    PeerComm* pc = nullptr;
    {
        std::lock_guard<std::mutex> lk(g_peer_mu);
        if (!comm || !g_peer_comms.count(comm)) return;
        g_peer_comms.erase(comm);
        pc = static_cast<PeerComm*>(comm);
    }
    cudaSetDevice(pc->ctx->device);
    cudaStreamSynchronize(pc->ctx->stream);
    for (void* p : pc->opened) cudaIpcCloseMemHandle(p);
    cudaFree(pc->d_comb);
    delete pc;
}

// not in the ABI header (tools/kernel_trace.py): device array of 8 globaltimer
// stamps the next fused launches write from CTA 0 (null disables)
int abacus_internal_set_trace(void* d_stamps) {
    g_trace_ptr = (unsigned long long*)d_stamps;
    return ABACUS_OK;
}

int abacus_set_stream(abacus_ctx* c, void* stream) {
    if (!c) return ABACUS_E_INVALID;
    // the blocking calls share the ctx's scratch, mapped record and batch /
    // training buffers: whenever the effective stream changes (including the
    // reset to the ctx's own stream), finish the work queued on the old one
    const cudaStream_t next = stream ? (cudaStream_t)stream : c->own_stream;
    if (next != c->stream) {
        cudaSetDevice(c->device);
        cudaStreamSynchronize(c->stream);
    }
    c->stream = next;
    return ABACUS_OK;
}

int abacus_set_timing(abacus_ctx* c, int on) {
    if (!c) return ABACUS_E_INVALID;
    c->timed = on != 0;
    return ABACUS_OK;
}

}  // extern "C"
