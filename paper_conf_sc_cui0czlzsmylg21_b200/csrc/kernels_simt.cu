// kernels_simt.cu -- SIMT kernels of the Abacus candidate search (sm_100a).
//
//   encode_grid_kernel      a2+a3  grid range -> Fig.-8 int16 rows
//   encode_groups_kernel    a3     explicit groups -> Fig.-8 rows
//   predict_fp32_kernel     a4     MLP forward, fp32 FFMA
//   select_kernel           a5     headroom mask + max key
//   fused_fp32_kernel       a2..a5 persistent fused search, fp32 SIMT path
//   finalize_gather_kernel  a6/a7  max over the ranks' gathered records
//
// The fused tensor-core path lives in kernels_tc.cu.
#include <cuda_runtime.h>
#include <math.h>

#include <cstring>

#include "common.cuh"
#include "device_common.cuh"
#include "internal.h"
#include "tc_ptx.cuh"

namespace abacus {

// ---------------------------------------------------------------------------
// shared device helpers
// ---------------------------------------------------------------------------

// Fig. 8 row for one candidate.  opeD[d] is the end op of the slot in digit d
// (slots right-aligned: slot j = d - (kKMax - k)); 0 = absent.  Positions:
// present slots in ascending model id.
__device__ __forceinline__ void write_fig8_row(const Plan& P, const int32_t (&opeD)[kKMax], int16_t* row) {
    for (int i = 0; i < P.D; i++) row[i] = 0;
    const int off = kKMax - P.k;
#pragma unroll
    for (int d = 0; d < kKMax; d++) {
        if (d < off || opeD[d] == 0) continue;
        const SlotP& s = P.slot[d - off];
        int p = 0;
#pragma unroll
        for (int e = 0; e < kKMax; e++)
            if (e >= off && opeD[e] != 0 && P.slot[e - off].model_id < s.model_id) p++;
        row[s.model_id - 1] = 1;
        int16_t* f = row + P.n_models + 4 * p;
        f[0] = (int16_t)s.ops;
        f[1] = (int16_t)opeD[d];
        f[2] = (int16_t)s.bs;
        f[3] = (int16_t)s.seqlen;
    }
}

// copy a block's staged rows (smem) to global with 16-byte stores where aligned
__device__ __forceinline__ void store_rows(const int16_t* sm, int16_t* gout, uint64_t nbytes) {
    const uintptr_t ga = reinterpret_cast<uintptr_t>(gout);
    if ((ga & 15) == 0) {
        const uint64_t n16 = nbytes / 16;
        const int4* s4 = reinterpret_cast<const int4*>(sm);
        int4* g4 = reinterpret_cast<int4*>(gout);
        for (uint64_t i = threadIdx.x; i < n16; i += blockDim.x) g4[i] = s4[i];
        const char* sb = reinterpret_cast<const char*>(sm);
        char* gb = reinterpret_cast<char*>(gout);
        for (uint64_t i = n16 * 16 + threadIdx.x; i < nbytes; i += blockDim.x) gb[i] = sb[i];
    } else {
        const uint64_t n2 = nbytes / 2;
        for (uint64_t i = threadIdx.x; i < n2; i += blockDim.x) gout[i] = sm[i];
    }
}

// ---------------------------------------------------------------------------
// a2 + a3: grid range encode.  One thread per candidate t; the block's rows
// are staged in shared memory and written with coalesced 16-byte stores.
// plan.seg[0] is the whole grid as one box (cnt = radix, digits = grid digits).
// ---------------------------------------------------------------------------
constexpr int kEncThreads = 128;

__global__ void __launch_bounds__(kEncThreads) encode_grid_kernel(const __grid_constant__ Plan P, uint64_t first,
                                                                  uint64_t count, int16_t* __restrict__ out) {
    extern __shared__ int16_t s_rows[];  // kEncThreads * D
    const SegP& g = P.seg[0];
    for (uint64_t base = (uint64_t)blockIdx.x * kEncThreads; base < count;
         base += (uint64_t)gridDim.x * kEncThreads) {
        const uint64_t idx = base + threadIdx.x;
        uint32_t v[kKMax];
        decode_box<kKMax>(g, first + base, threadIdx.x, v);
        int32_t opeD[kKMax];
        const int off = kKMax - P.k;
#pragma unroll
        for (int d = 0; d < kKMax; d++) opeD[d] = d >= off ? digit_to_ope(P.slot[d - off], v[d]) : 0;
        if (idx < count) write_fig8_row(P, opeD, s_rows + threadIdx.x * P.D);
        __syncthreads();
        const uint64_t nrows = min((uint64_t)kEncThreads, count - base);
        store_rows(s_rows, out + base * P.D, nrows * P.D * 2);
        __syncthreads();
    }
}


// ---------------------------------------------------------------------------
// a2 + a3 fast path for D = 24 (N = 8): per block 1024 consecutive candidates,
// thread t builds rows t, t + 256, ... in a shared-memory stage (3 x 16-byte
// stores for the bitmap and zeros, then 2 x 4-byte stores per present model at
// its Fig.-8 position, read from a per-presence-pattern table), and one thread
// writes the whole 48 KB stage to HBM with a TMA bulk store (double-buffered).
// ---------------------------------------------------------------------------
constexpr int kEnc24Threads = 256;
constexpr int kEnc24Rows = 1024;

__global__ void __launch_bounds__(kEnc24Threads) encode_grid24_kernel(const __grid_constant__ Plan P, uint64_t first,
                                                                      uint64_t count, int16_t* __restrict__ out) {
    extern __shared__ __align__(128) uint8_t s_enc[];
    uint4* stage = reinterpret_cast<uint4*>(s_enc);                  // 2 x 1024 rows x 3 uint4
    uint4* s_bm = stage + 2 * kEnc24Rows * 3;                          // [16] bitmap words per mask
    int8_t* s_pos = reinterpret_cast<int8_t*>(s_bm + 16);              // [16][4] Fig.-8 position per digit
    const SegP& g = P.seg[0];
    const int off = kKMax - P.k;
    if (threadIdx.x < 16) {
        const uint32_t mask = threadIdx.x;  // bit d: digit d present
        uint32_t w[4] = {0, 0, 0, 0};
        for (int d = 0; d < kKMax; d++) {
            int8_t p = -1;
            if (d >= off && ((mask >> d) & 1u)) {
                const int m = P.slot[d - off].model_id;
                w[(m - 1) >> 1] |= 1u << (16 * ((m - 1) & 1));
                p = 0;
                for (int e = off; e < kKMax; e++)
                    if (((mask >> e) & 1u) && P.slot[e - off].model_id < m) p++;
            }
            s_pos[threadIdx.x * 4 + d] = p;
        }
        s_bm[threadIdx.x] = make_uint4(w[0], w[1], w[2], w[3]);
    }
    // per digit: (ops | ope0 << 16) base word and the constant (bs | seqlen << 16) word
    uint32_t opsw[kKMax], bsw[kKMax];
    int32_t elo[kKMax];
    bool abs_[kKMax];
#pragma unroll
    for (int d = 0; d < kKMax; d++) {
        if (d < off) {
            opsw[d] = bsw[d] = 0;
            elo[d] = 0;
            abs_[d] = true;
            continue;
        }
        const SlotP& s = P.slot[d - off];
        opsw[d] = (uint32_t)(uint16_t)s.ops;
        bsw[d] = (uint32_t)(uint16_t)s.bs | ((uint32_t)(uint16_t)s.seqlen << 16);
        elo[d] = s.end_lo - s.absent;  // ope = elo + digit (for a present digit)
        abs_[d] = s.absent != 0;
    }
    __syncthreads();
    int it = 0;
    for (uint64_t base = (uint64_t)blockIdx.x * kEnc24Rows; base < count;
         base += (uint64_t)gridDim.x * kEnc24Rows, it++) {
        uint4* st = stage + (it & 1) * kEnc24Rows * 3;
        if (it >= 2 && threadIdx.x == 0)
            asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // stage reused two rounds later
        __syncthreads();
        const uint32_t nrows = (uint32_t)min((uint64_t)kEnc24Rows, count - base);
        // digits of row threadIdx.x (fp64 split of the stage base + carry), then
        // + kEnc24Threads per further row with a multiply-high carry chain
        uint32_t v[kKMax];
        decode_box<kKMax>(g, first + base, threadIdx.x, v);
        for (uint32_t r = threadIdx.x; r < nrows; r += kEnc24Threads) {
            if (r != threadIdx.x) {
                uint32_t carry = kEnc24Threads;
#pragma unroll
                for (int d = kKMax - 1; d >= 0; d--) {
                    const uint32_t x = v[d] + carry;
                    const uint32_t q = fastdiv(x, g.fd[d]);
                    v[d] = x - q * g.cnt[d];
                    carry = q;
                }
            }
            uint32_t mask = 0;
#pragma unroll
            for (int d = 0; d < kKMax; d++)
                if (d >= off && !(abs_[d] && v[d] == 0)) mask |= 1u << d;
            uint4* row = st + r * 3;
            row[0] = s_bm[mask];
            row[1] = make_uint4(0, 0, 0, 0);
            row[2] = make_uint4(0, 0, 0, 0);
            uint32_t* rw = reinterpret_cast<uint32_t*>(row);
#pragma unroll
            for (int d = 0; d < kKMax; d++) {
                const int p = s_pos[mask * 4 + d];
                if (p < 0) continue;
                rw[4 + 2 * p] = opsw[d] | ((uint32_t)(elo[d] + (int32_t)v[d]) << 16);
                rw[5 + 2 * p] = bsw[d];
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + base * 24),
                         "r"((uint32_t)__cvta_generic_to_shared(st)), "r"(nrows * 48u)
                         : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
    }
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// ---------------------------------------------------------------------------
// a3 for explicit groups (config-5 instance samples)
// ---------------------------------------------------------------------------
struct GroupRec {
    int32_t k;
    int32_t s[kKMax][5];  // model_id, ops, ope, batch, seqlen
};

__global__ void __launch_bounds__(kEncThreads) encode_groups_kernel(const GroupRec* __restrict__ groups,
                                                                    uint64_t count, int32_t n_models, int32_t D,
                                                                    int16_t* __restrict__ out,
                                                                    uint32_t* __restrict__ bad) {
    extern __shared__ int16_t s_rows[];
    for (uint64_t base = (uint64_t)blockIdx.x * kEncThreads; base < count;
         base += (uint64_t)gridDim.x * kEncThreads) {
        const uint64_t idx = base + threadIdx.x;
        int16_t* row = s_rows + threadIdx.x * D;
        if (idx < count) {
            const GroupRec g = groups[idx];
            for (int i = 0; i < D; i++) row[i] = 0;
            bool ok = g.k >= 0 && g.k <= kKMax;
            if (ok) {
                for (int j = 0; j < g.k; j++) {
                    int m = g.s[j][0];
                    ok = ok && m >= 1 && m <= n_models;
                    for (int i = 0; i < j; i++) ok = ok && g.s[i][0] != m;
                }
            }
            if (ok) {
                for (int j = 0; j < g.k; j++) {
                    int p = 0;
                    for (int i = 0; i < g.k; i++) p += g.s[i][0] < g.s[j][0];
                    row[g.s[j][0] - 1] = 1;
                    int16_t* f = row + n_models + 4 * p;
                    f[0] = (int16_t)g.s[j][1];
                    f[1] = (int16_t)g.s[j][2];
                    f[2] = (int16_t)g.s[j][3];
                    f[3] = (int16_t)g.s[j][4];
                }
            } else if (bad) {
                atomicAdd(bad, 1u);
            }
        }
        __syncthreads();
        const uint64_t nrows = min((uint64_t)kEncThreads, count - base);
        store_rows(s_rows, out + base * D, nrows * D * 2);
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// a4, fp32 SIMT: one thread per candidate row.  Layer 1 weights (runtime D)
// are staged in shared memory (broadcast reads); layers 2-4 are kernel
// parameters (constant bank: FFMA with a constant operand, no load).
// ---------------------------------------------------------------------------
constexpr int kPredThreads = 128;

__device__ __forceinline__ void mlp_tail_fp32(const W234& W, float (&h1)[kHidden], float& y) {
    float h2[kHidden];
#pragma unroll
    for (int i = 0; i < kHidden; i++) {
        float s = W.b2[i];
#pragma unroll
        for (int j = 0; j < kHidden; j++) s = fmaf(W.W2[i][j], h1[j], s);
        h2[i] = fmaxf(s, 0.0f);
    }
    float acc = W.b4;
#pragma unroll
    for (int i = 0; i < kHidden; i++) {
        float s = W.b3[i];
#pragma unroll
        for (int j = 0; j < kHidden; j++) s = fmaf(W.W3[i][j], h2[j], s);
        acc = fmaf(W.w4[i], fmaxf(s, 0.0f), acc);
    }
    y = acc;
}

__global__ void __launch_bounds__(kPredThreads) predict_fp32_kernel(const __grid_constant__ W234 W,
                                                                    const float* __restrict__ w1b1, int32_t D,
                                                                    const int16_t* __restrict__ x, uint64_t count,
                                                                    float* __restrict__ y) {
    extern __shared__ float s_w1[];  // W1[32][D] then b1[32]
    for (int i = threadIdx.x; i < kHidden * D + kHidden; i += blockDim.x) s_w1[i] = w1b1[i];
    __syncthreads();
    const float* b1 = s_w1 + kHidden * D;
    for (uint64_t idx = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < count;
         idx += (uint64_t)gridDim.x * blockDim.x) {
        const int16_t* row = x + idx * D;
        float h1[kHidden];
#pragma unroll
        for (int i = 0; i < kHidden; i++) h1[i] = 0.0f;
        for (int j = 0; j < D; j++) {
            const float xv = (float)row[j];
#pragma unroll
            for (int i = 0; i < kHidden; i++) h1[i] = fmaf(s_w1[i * D + j], xv, h1[i]);
        }
#pragma unroll
        for (int i = 0; i < kHidden; i++) h1[i] = fmaxf(h1[i] + b1[i], 0.0f);
        float out;
        mlp_tail_fp32(W, h1, out);
        y[idx] = out;
    }
}

// D = 24 (the registry's canonical width): layer 1 from the kernel parameters
// too, so every FFMA of the row takes its weight from the constant bank (no
// shared-memory load per FMA, which bound the generic kernel at 0.36 of the
// FP32 FMA rate).  Each thread runs R = 2 consecutive rows so every weight
// brought into a uniform register (LDCU) feeds two FFMAs; the 2 x 48-byte rows
// are read with six 16-byte streaming loads.
constexpr int kPred24Rows = 2;

__global__ void __launch_bounds__(kPredThreads) predict24_fp32_kernel(const __grid_constant__ W1P A,
                                                                      const __grid_constant__ W234 W,
                                                                      const int16_t* __restrict__ x, uint64_t count,
                                                                      float* __restrict__ y) {
    constexpr int D = 24, R = kPred24Rows;
    const uint64_t npair = (count + R - 1) / R;
    for (uint64_t pi = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; pi < npair;
         pi += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t row0 = pi * R;
        float xv[R][D];
#pragma unroll
        for (int rr = 0; rr < R; rr++) {
            // a missing last row re-reads row0 (its result is not stored)
            const uint64_t row = row0 + rr < count ? row0 + rr : row0;
            const uint4* rp = reinterpret_cast<const uint4*>(x + row * D);
#pragma unroll
            for (int q = 0; q < 3; q++) {
                const uint4 v = __ldcs(rp + q);
                const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                for (int i = 0; i < 4; i++) {
                    xv[rr][8 * q + 2 * i] = (float)(int16_t)(w[i] & 0xFFFFu);
                    xv[rr][8 * q + 2 * i + 1] = (float)(int16_t)(w[i] >> 16);
                }
            }
        }
        float h[R][kHidden];
#pragma unroll
        for (int i = 0; i < kHidden; i++) {
            float s[R];
#pragma unroll
            for (int rr = 0; rr < R; rr++) s[rr] = 0.0f;
#pragma unroll
            for (int j = 0; j < D; j++)
#pragma unroll
                for (int rr = 0; rr < R; rr++) s[rr] = fmaf(A.W1[i][j], xv[rr][j], s[rr]);
#pragma unroll
            for (int rr = 0; rr < R; rr++) h[rr][i] = fmaxf(s[rr] + A.b1[i], 0.0f);
        }
        float h2[R][kHidden];
#pragma unroll
        for (int i = 0; i < kHidden; i++) {
            float s[R];
#pragma unroll
            for (int rr = 0; rr < R; rr++) s[rr] = W.b2[i];
#pragma unroll
            for (int j = 0; j < kHidden; j++)
#pragma unroll
                for (int rr = 0; rr < R; rr++) s[rr] = fmaf(W.W2[i][j], h[rr][j], s[rr]);
#pragma unroll
            for (int rr = 0; rr < R; rr++) h2[rr][i] = fmaxf(s[rr], 0.0f);
        }
        float acc[R];
#pragma unroll
        for (int rr = 0; rr < R; rr++) acc[rr] = W.b4;
#pragma unroll
        for (int i = 0; i < kHidden; i++) {
            float s[R];
#pragma unroll
            for (int rr = 0; rr < R; rr++) s[rr] = W.b3[i];
#pragma unroll
            for (int j = 0; j < kHidden; j++)
#pragma unroll
                for (int rr = 0; rr < R; rr++) s[rr] = fmaf(W.W3[i][j], h2[rr][j], s[rr]);
#pragma unroll
            for (int rr = 0; rr < R; rr++) acc[rr] = fmaf(W.w4[i], fmaxf(s[rr], 0.0f), acc[rr]);
        }
#pragma unroll
        for (int rr = 0; rr < R; rr++)
            if (row0 + rr < count) __stcs(y + row0 + rr, acc[rr]);
    }
}

// ---------------------------------------------------------------------------
// a5: headroom mask + largest-group key over a grid range.  Each thread walks
// kSelPer consecutive candidates (two 16-byte loads of y), decoding only the
// first index; the following ones advance the fastest digit with a carry
// check.  Warp shuffle max -> shared -> one atomicMax(u64) per block.
// plan.seg[0] is the whole grid with the slots right-aligned in the digits
// (digit 3 = last slot), see plan_whole_grid.
// ---------------------------------------------------------------------------
constexpr int kSelThreads = 256;
constexpr int kSelPer = 32;
constexpr int kSelPad = kSelPer + 4;  // padded per-thread row of the load stage

__global__ void __launch_bounds__(kSelThreads) select_kernel(const __grid_constant__ Plan P, uint64_t first,
                                                             uint64_t count, const float* __restrict__ lat,
                                                             float H, unsigned long long* best) {
    __shared__ unsigned long long s_max[kSelThreads / 32];
    __shared__ __align__(16) float s_y[kSelThreads * kSelPad];
    const SegP& g = P.seg[0];
    const int off = kKMax - P.k;  // digit of slot j = off + j
    // n of slot j at digit value d: 0 if absent (d == 0 and absent allowed), else nb_j + d
    int32_t nb[kKMax];
    bool ab[kKMax];
#pragma unroll
    for (int d = 0; d < kKMax; d++) {
        const int j = d - off;
        if (j < 0) {
            nb[d] = 0;
            ab[d] = true;
            continue;
        }
        const SlotP& s = P.slot[j];
        ab[d] = s.absent != 0;
        nb[d] = s.end_lo - s.ops + 1 - s.absent;
    }
    const uint32_t cnt3 = g.cnt[kKMax - 1];
    unsigned long long mx = 0;
    const uint64_t chunk = (uint64_t)kSelThreads * kSelPer;
    for (uint64_t base = (uint64_t)blockIdx.x * chunk; base < count; base += (uint64_t)gridDim.x * chunk) {
        const uint64_t i0 = base + (uint64_t)threadIdx.x * kSelPer;
        const uint64_t w0 = base + (uint64_t)(threadIdx.x & ~31u) * kSelPer;  // the warp's 1024 candidates
        const float* wsrc = lat + w0;
        float y[kSelPer];
        if (w0 + 32 * kSelPer <= count && (reinterpret_cast<uintptr_t>(wsrc) & 15u) == 0) {
            // coalesced: 8 x 512 B per warp into a padded shared stage, then each
            // thread reads back its own 32 consecutive values (conflict-free)
            float* sw = s_y + (threadIdx.x >> 5) * (32 * kSelPad);
            const int lane = threadIdx.x & 31;
            float4 a[kSelPer / 4];
#pragma unroll
            for (int k = 0; k < kSelPer / 4; k++) a[k] = __ldcs(reinterpret_cast<const float4*>(wsrc) + k * 32 + lane);
#pragma unroll
            for (int k = 0; k < kSelPer / 4; k++) {
                const int idx4 = k * 32 + lane;
                *reinterpret_cast<float4*>(sw + (idx4 >> 3) * kSelPad + (idx4 & 7) * 4) = a[k];
            }
            __syncwarp();
#pragma unroll
            for (int k = 0; k < kSelPer / 4; k++) {
                const float4 b = *reinterpret_cast<const float4*>(sw + lane * kSelPad + 4 * k);
                y[4 * k] = b.x; y[4 * k + 1] = b.y; y[4 * k + 2] = b.z; y[4 * k + 3] = b.w;
            }
            __syncwarp();
        } else {
            if (i0 >= count) continue;
            const float* src = lat + i0;
#pragma unroll
            for (int q = 0; q < kSelPer; q++) y[q] = i0 + q < count ? src[q] : __int_as_float(0x7fc00000);
        }
        if (i0 >= count) continue;
        // feasibility bits of the thread's 32 consecutive candidates
        uint32_t fm = 0;
#pragma unroll
        for (int q = 0; q < kSelPer; q++) fm |= (y[q] <= H ? 1u : 0u) << q;
        if (!fm) continue;
        uint32_t v[kKMax];
        decode_box<kKMax>(g, first + base, threadIdx.x * kSelPer, v);
        auto nsum_rest = [&]() {
            int32_t r = 0;
#pragma unroll
            for (int d = 0; d < kKMax - 1; d++) r += (ab[d] && v[d] == 0) ? 0 : nb[d] + (int32_t)v[d];
            return r;
        };
        // A run = consecutive candidates with no carry out of the last digit.
        // Inside a run the index t and the last slot's n both grow with q, so
        // the key ((sum_n + 1) << 40) | t is strictly increasing: only the last
        // feasible candidate of each run can hold the run's maximum.
        const uint64_t t0 = first + i0;
        int32_t rest = nsum_rest();
        uint32_t qa = 0;
        while (true) {
            const uint32_t left = (uint32_t)kSelPer - qa, room = cnt3 - v[kKMax - 1];
            const uint32_t len = room < left ? room : left;
            const uint32_t runm = (len >= 32u ? 0xffffffffu : ((1u << len) - 1u)) << qa;
            const uint32_t m = fm & runm;
            if (m) {
                const uint32_t q = 31u - (uint32_t)__clz(m);
                const uint32_t v3 = v[kKMax - 1] + (q - qa);
                const int32_t n3 = (ab[kKMax - 1] && v3 == 0) ? 0 : nb[kKMax - 1] + (int32_t)v3;
                mx = umax64(mx, ((unsigned long long)(rest + n3 + 1) << 40) | (t0 + q));
            }
            qa += len;
            if (qa >= (uint32_t)kSelPer || !(fm >> qa)) break;
            // carry: the last digit wraps to 0, the others count up
            v[kKMax - 1] = 0;
#pragma unroll
            for (int d = kKMax - 2; d >= 0; d--) {
                if (++v[d] < g.cnt[d]) break;
                v[d] = 0;
            }
            rest = nsum_rest();
        }
    }
    mx = warp_max_u64(mx);
    if ((threadIdx.x & 31) == 0) s_max[threadIdx.x >> 5] = mx;
    __syncthreads();
    if (threadIdx.x < 32) {
        mx = threadIdx.x < kSelThreads / 32 ? s_max[threadIdx.x] : 0ull;
        mx = warp_max_u64(mx);
        if (threadIdx.x == 0 && mx) atomicMax(best, mx);
    }
}

// ---------------------------------------------------------------------------
// a2..a5 fused, fp32 SIMT path.  Persistent blocks of 128 threads, one
// 128-candidate tile per iteration.  Layer 1 is evaluated per segment as
//     z1 = c_P + sum_j v_j * w_P,j
// where c_P = b1 + W1 x0_P (x0_P: the Fig.-8 vector of the segment's v = 0
// group) and w_P,j = W1[:, N + 4 pos_P(j) + 1] (the ope column of slot j at its
// Fig.-8 position): x(v) = x0_P + sum_j v_j e_{N+4pos_P(j)+1} is affine in the
// digits, so this is W1 x + b1 exactly (up to fp32 rounding order).  The
// per-segment tables are built in the prologue, on device, from fp32 W1/b1.
// ---------------------------------------------------------------------------
constexpr int kFusedThreads = 128;
constexpr int kFusedBlocksPerSM = 3;

__device__ void build_l1_tables(const Plan& P, const float* __restrict__ w1b1, float* s_c, float* s_w) {
    // s_c[s][32], s_w[s][4][32]
    const int D = P.D;
    const float* b1 = w1b1 + kHidden * D;
    for (int e = threadIdx.x; e < P.n_seg * kHidden; e += blockDim.x) {
        const int s = e / kHidden, i = e % kHidden;
        const SegP& g = P.seg[s];
        const float* w = w1b1 + i * D;
        float c = b1[i];
        for (int dg = 0; dg < kKMax; dg++) s_w[(s * kKMax + dg) * kHidden + i] = 0.0f;
        for (int j = 0; j < P.k; j++) {
            if (!((g.mask >> j) & 1u)) continue;
            const SlotP& sl = P.slot[j];
            const int f = P.n_models + 4 * g.pos[j];
            c = fmaf(w[sl.model_id - 1], 1.0f, c);
            c = fmaf(w[f + 0], (float)sl.ops, c);
            c = fmaf(w[f + 1], (float)g.ope0[j], c);
            c = fmaf(w[f + 2], (float)sl.bs, c);
            c = fmaf(w[f + 3], (float)sl.seqlen, c);
            s_w[(s * kKMax + g.dpos[j]) * kHidden + i] = w[f + 1];  // digit of slot j
        }
        s_c[s * kHidden + i] = c;
    }
}

__global__ void __launch_bounds__(kFusedThreads, kFusedBlocksPerSM) fused_fp32_kernel(const __grid_constant__ Plan P,
                                                                      const __grid_constant__ W234 Wt,
                                                                      const float* __restrict__ w1b1, Scratch* S) {
    __shared__ float s_c[kMaxSeg * kHidden];
    __shared__ float s_w[kMaxSeg * kKMax * kHidden];
    build_l1_tables(P, w1b1, s_c, s_w);
    __syncthreads();

    const uint32_t r = threadIdx.x;
    unsigned long long best = 0;
    float best_y = __int_as_float(0x7fc00000);
    uint64_t wb, we;
    work_range(P.n_tiles, (uint64_t)blockIdx.x, (uint64_t)gridDim.x, wb, we);
    Walker W;
    if (wb < we) walker_begin(P, W, wb, r);
    for (uint64_t w = wb; w < we; w++) {
        if (w != wb) walker_next(P, W, w, r);
        const bool valid = W.u_end - W.ub > (uint64_t)r;
        const float* c = s_c + W.s * kHidden;
        const float* wc = s_w + W.s * kKMax * kHidden;
        float h1[kHidden];
#pragma unroll
        for (int i = 0; i < kHidden; i++) {
            float z = c[i];
#pragma unroll
            for (int j = 0; j < kKMax; j++) z = fmaf(wc[j * kHidden + i], (float)W.v[j], z);
            h1[i] = fmaxf(z, 0.0f);
        }
        float y;
        mlp_tail_fp32(Wt, h1, y);
        if (valid && walker_is_index0(W, r)) S->y0 = y;
        fold_candidate(W, valid, y, P.H, best, best_y);
    }
    cta_publish_and_finish(P, S, best, best_y);
}

// Two candidates per thread (rows r of tiles w and w + 1): each weight of
// layers 2-4 is read once from shared memory (LDS.128 broadcast, four weights)
// and feeds two FFMAs, so the kernel is bound by the FMA pipe instead of the
// constant cache that the one-candidate kernel reads every weight from.  The
// per-candidate arithmetic (FMA order) is the one-candidate kernel's.
constexpr int kFused2Threads = 128;
constexpr int kFused2BlocksPerSM = 2;

struct W234s {  // layers 2..4 in shared memory, rows 16-byte aligned
    float4 W2[kHidden][kHidden / 4];
    float4 W3[kHidden][kHidden / 4];
    float b2[kHidden], b3[kHidden], w4[kHidden];
    float b4;
};

__device__ __forceinline__ void mlp_tail_fp32_x2(const W234s& W, const float (&hx)[kHidden],
                                                 const float (&hy)[kHidden], float& yx, float& yy) {
    float gx[kHidden], gy[kHidden];
#pragma unroll
    for (int i = 0; i < kHidden; i++) {
        float sx = W.b2[i], sy = sx;
#pragma unroll
        for (int q = 0; q < kHidden / 4; q++) {
            const float4 w = W.W2[i][q];
            sx = fmaf(w.x, hx[4 * q + 0], sx); sy = fmaf(w.x, hy[4 * q + 0], sy);
            sx = fmaf(w.y, hx[4 * q + 1], sx); sy = fmaf(w.y, hy[4 * q + 1], sy);
            sx = fmaf(w.z, hx[4 * q + 2], sx); sy = fmaf(w.z, hy[4 * q + 2], sy);
            sx = fmaf(w.w, hx[4 * q + 3], sx); sy = fmaf(w.w, hy[4 * q + 3], sy);
        }
        gx[i] = fmaxf(sx, 0.0f);
        gy[i] = fmaxf(sy, 0.0f);
    }
    float ax = W.b4, ay = W.b4;
#pragma unroll
    for (int i = 0; i < kHidden; i++) {
        float sx = W.b3[i], sy = sx;
#pragma unroll
        for (int q = 0; q < kHidden / 4; q++) {
            const float4 w = W.W3[i][q];
            sx = fmaf(w.x, gx[4 * q + 0], sx); sy = fmaf(w.x, gy[4 * q + 0], sy);
            sx = fmaf(w.y, gx[4 * q + 1], sx); sy = fmaf(w.y, gy[4 * q + 1], sy);
            sx = fmaf(w.z, gx[4 * q + 2], sx); sy = fmaf(w.z, gy[4 * q + 2], sy);
            sx = fmaf(w.w, gx[4 * q + 3], sx); sy = fmaf(w.w, gy[4 * q + 3], sy);
        }
        ax = fmaf(W.w4[i], fmaxf(sx, 0.0f), ax);
        ay = fmaf(W.w4[i], fmaxf(sy, 0.0f), ay);
    }
    yx = ax;
    yy = ay;
}

__device__ __forceinline__ void layer1_fp32(const float* c, const float* wc, const uint32_t (&v)[kKMax],
                                            float (&h)[kHidden]) {
#pragma unroll
    for (int i = 0; i < kHidden; i++) {
        float z = c[i];
#pragma unroll
        for (int j = 0; j < kKMax; j++) z = fmaf(wc[j * kHidden + i], (float)v[j], z);
        h[i] = fmaxf(z, 0.0f);
    }
}

template <class PL>
__global__ void __launch_bounds__(kFused2Threads, kFused2BlocksPerSM) fused_fp32x2_kernel(
    const __grid_constant__ PL Pin, const __grid_constant__ W234 Wt, const float* __restrict__ w1b1, Scratch* S) {
    const Plan& P = *reinterpret_cast<const Plan*>(&Pin);  // PlanT<8> for decisions: same layout prefix
    __shared__ float s_c[kMaxSeg * kHidden];
    __shared__ float s_w[kMaxSeg * kKMax * kHidden];
    __shared__ W234s s_W;
    build_l1_tables(P, w1b1, s_c, s_w);
    for (int e = threadIdx.x; e < kHidden * kHidden; e += blockDim.x) {
        const int i = e / kHidden, j = e % kHidden;
        reinterpret_cast<float*>(&s_W.W2[i][0])[j] = Wt.W2[i][j];
        reinterpret_cast<float*>(&s_W.W3[i][0])[j] = Wt.W3[i][j];
    }
    if (threadIdx.x < kHidden) {
        s_W.b2[threadIdx.x] = Wt.b2[threadIdx.x];
        s_W.b3[threadIdx.x] = Wt.b3[threadIdx.x];
        s_W.w4[threadIdx.x] = Wt.w4[threadIdx.x];
    }
    if (threadIdx.x == 0) s_W.b4 = Wt.b4;
    __syncthreads();

    const uint32_t r = threadIdx.x;
    unsigned long long best = 0;
    float best_y = __int_as_float(0x7fc00000);
    uint32_t bsn = 1u;
    // work items are tile pairs (w, w + 1); the last pair may have only w.
    // The packed walker (device_common.cuh) carries each row's digits and sum_n;
    // rows past a segment's end have sn = 0, which no fold accepts.
    auto unpack = [](uint32_t a1, uint32_t a2, uint32_t (&v)[kKMax]) {
        v[0] = (a1 & 0xFFFFu) - 0x6400u;
        v[1] = (a1 >> 16) - 0x6400u;
        v[2] = (a2 & 0xFFFFu) - 0x6400u;
        v[3] = (a2 >> 16) - 0x6400u;
    };
    const uint64_t n_pairs = (P.n_tiles + 1) / 2;
    uint64_t pb, pe;
    work_range(n_pairs, (uint64_t)blockIdx.x, (uint64_t)gridDim.x, pb, pe);
    PackedWalker W;
    if (pb < pe) W.begin(P, 2 * pb, r);
    for (uint64_t p = pb; p < pe; p++) {
        const uint64_t w = 2 * p;
        if (p != pb) W.next(P, r);
        const uint32_t x1 = W.a1, x2 = W.a2, xs = W.sn;
        const int sX = W.s;
        uint32_t v[kKMax];
        unpack(x1, x2, v);
        float hx[kHidden], hy[kHidden];
        layer1_fp32(s_c + sX * kHidden, s_w + sX * kKMax * kHidden, v, hx);
        const bool hasY = w + 1 < P.n_tiles;
        if (hasY) W.next(P, r);
        const uint32_t ys = hasY ? W.sn : 0u;
        unpack(W.a1, W.a2, v);
        layer1_fp32(s_c + W.s * kHidden, s_w + W.s * kKMax * kHidden, v, hy);
        float yx, yy;
        mlp_tail_fp32_x2(s_W, hx, hy, yx, yy);
        if (w == 0 && P.want_y0 && r == 0) S->y0 = yx;
        fold_packed(P, sX, x1, x2, xs, yx, best, best_y, bsn);
        fold_packed(P, W.s, W.a1, W.a2, ys, yy, best, best_y, bsn);
    }
    cta_publish_and_finish(P, S, best, best_y);
}

// ---------------------------------------------------------------------------
// a6 tail: after the NCCL all-gather of the per-rank Result records, every
// rank reduces the same records to the same global decision.
// ---------------------------------------------------------------------------
__global__ void finalize_gather_kernel(Scratch* S, int nranks, MappedRec* mapped, uint32_t seq) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    S->result = combine_results(S->gathered, nranks);  // common.cuh, shared with the host
    if (mapped) publish_mapped(S->result, mapped, seq);
}


// ---------------------------------------------------------------------------
// NEXT-1: the paper's multi-way search (§7.7) in one
// CTA.  Round 1 predicts u = 0 (drop test) and the chain's block ends (queries
// fully added, "between queries"); later rounds probe the open interval
// (last fit, first miss) of the next query's operators at `ways` points
// p_i = lo + floor(i (hi - lo) / (ways + 1)) ("among the operators").  Each
// round is one batched prediction: thread i evaluates probe i with the fp32
// predictor (layer 1 from shared memory, layers 2-4 from the constant bank).
// ---------------------------------------------------------------------------
constexpr int kMwayThreads = 512;  // 16 warps: one warp per probe, lane = hidden unit

// y of chain position u, computed by one warp (lane i = hidden unit i; the
// activations are broadcast with shuffles; weights transposed in shared
// memory so the lanes read consecutive words).  Returns y in every lane.
struct MwaySmem {
    float w1t[80 * kHidden];  // W1^T [D][32]
    float w2t[kHidden * kHidden], w3t[kHidden * kHidden];
    float b1[kHidden], b2[kHidden], b3[kHidden], w4[kHidden];
    float b4;
};

__device__ float chain_candidate_y_warp(const Plan& P, const MwaySmem& W, uint64_t u, uint32_t lane) {
    int32_t ope[kKMax];
#pragma unroll
    for (int j = 0; j < kKMax; j++) ope[j] = j < P.k ? decode_slot_ope(P, u, j) : 0;
    float z = W.b1[lane];
    // Fig. 8 features: at most 5 non-zeros per present model
#pragma unroll
    for (int j = 0; j < kKMax; j++) {
        if (j >= P.k || ope[j] == 0) continue;
        int p = 0;
#pragma unroll
        for (int i = 0; i < kKMax; i++)
            if (i < P.k && ope[i] != 0 && P.slot[i].model_id < P.slot[j].model_id) p++;
        const SlotP& s = P.slot[j];
        const int f = P.n_models + 4 * p;
        z += W.w1t[(s.model_id - 1) * kHidden + lane];
        z = fmaf(W.w1t[(f + 0) * kHidden + lane], (float)s.ops, z);
        z = fmaf(W.w1t[(f + 1) * kHidden + lane], (float)ope[j], z);
        z = fmaf(W.w1t[(f + 2) * kHidden + lane], (float)s.bs, z);
        z = fmaf(W.w1t[(f + 3) * kHidden + lane], (float)s.seqlen, z);
    }
    float h = fmaxf(z, 0.0f);
    float acc = W.b2[lane];
#pragma unroll
    for (int j = 0; j < kHidden; j++) acc = fmaf(W.w2t[j * kHidden + lane], __shfl_sync(0xffffffffu, h, j), acc);
    h = fmaxf(acc, 0.0f);
    acc = W.b3[lane];
#pragma unroll
    for (int j = 0; j < kHidden; j++) acc = fmaf(W.w3t[j * kHidden + lane], __shfl_sync(0xffffffffu, h, j), acc);
    h = fmaxf(acc, 0.0f);
    float y = W.w4[lane] * h;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) y += __shfl_xor_sync(0xffffffffu, y, o);
    return y + W.b4;
}

__global__ void __launch_bounds__(kMwayThreads, 1) mway_kernel(const __grid_constant__ Plan P,
                                                                const __grid_constant__ W234 Wt,
                                                                const float* __restrict__ w1b1, int ways,
                                                                Scratch* S) {
    __shared__ MwaySmem W;
    __shared__ uint64_t s_probe[128];
    __shared__ float s_y[128];
    __shared__ int s_n, s_done, s_rounds, s_preds;
    __shared__ uint64_t s_lo, s_hi;
    __shared__ float s_ylo, s_y0;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    for (int i = threadIdx.x; i < kHidden * P.D; i += blockDim.x) {
        const int o = i / P.D, c = i % P.D;
        W.w1t[c * kHidden + o] = w1b1[i];
    }
    for (int i = threadIdx.x; i < kHidden * kHidden; i += blockDim.x) {
        const int o = i / kHidden, c = i % kHidden;
        W.w2t[c * kHidden + o] = Wt.W2[o][c];
        W.w3t[c * kHidden + o] = Wt.W3[o][c];
    }
    if (threadIdx.x < kHidden) {
        W.b1[threadIdx.x] = w1b1[kHidden * P.D + threadIdx.x];
        W.b2[threadIdx.x] = Wt.b2[threadIdx.x];
        W.b3[threadIdx.x] = Wt.b3[threadIdx.x];
        W.w4[threadIdx.x] = Wt.w4[threadIdx.x];
    }
    if (threadIdx.x == 0) W.b4 = Wt.b4;
    if (threadIdx.x == 0) {
        // round 1: u = 0 and the block ends B_j = chain_cum[j + 1] - 1
        int n = 0;
        s_probe[n++] = 0;
        for (int j = 1; j < P.k; j++) s_probe[n++] = P.chain_cum[j + 1] - 1;
        s_n = n;
        s_done = 0;
        s_rounds = 0;
        s_preds = 0;
    }
    __syncthreads();
    for (int round = 0;; round++) {
        const int n = s_n;
        for (int pi = (int)warp; pi < n; pi += (int)nwarps) {
            const float yv = chain_candidate_y_warp(P, W, s_probe[pi], lane);
            if (lane == 0) s_y[pi] = yv;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            s_rounds++;
            s_preds += n;
            uint64_t lo, hi;
            int lf = -1;
            if (round == 0) {
                s_y0 = s_y[0];
                if (!(s_y[0] <= P.H)) {  // drop mechanism
                    s_done = 2;
                } else {
                    lf = 0;
                    for (int i = 1; i < n; i++)
                        if (s_y[i] <= P.H) lf = i;
                    lo = s_probe[lf];
                    hi = P.chain_cum[P.k];
                    s_ylo = s_y[lf];
                }
            } else {
                lo = s_lo;
                hi = s_hi;
                for (int i = 0; i < n; i++)
                    if (s_y[i] <= P.H) lf = i;
                if (lf >= 0) {
                    lo = s_probe[lf];
                    s_ylo = s_y[lf];
                }
            }
            if (s_done == 0) {
                for (int i = lf + 1; i < n; i++)
                    if (!(s_y[i] <= P.H)) {
                        hi = s_probe[i];
                        break;
                    }
                s_lo = lo;
                s_hi = hi;
                // a chain holds < 2^17 positions: 32-bit probe arithmetic
                const uint32_t span = (uint32_t)(hi - lo);
                if (span <= 1) {
                    s_done = 1;
                } else {
                    int m = 0;
                    if (span - 1 <= (uint32_t)ways) {
                        for (uint32_t v = 1; v < span; v++) s_probe[m++] = lo + v;
                    } else {
                        const uint32_t den = (uint32_t)ways + 1u;
                        uint32_t prev = 0;
                        for (int i = 1; i <= ways; i++) {
                            const uint32_t v = (span * (uint32_t)i) / den;
                            if (v > prev && v < span) {
                                s_probe[m++] = lo + v;
                                prev = v;
                            }
                        }
                    }
                    s_n = m;
                }
            }
        }
        __syncthreads();
        if (s_done) break;
    }
    if (threadIdx.x < 32) {
        // a7: decision assembly (lane j decodes slot j)
        const bool drop = s_done == 2;
        const uint64_t u = drop ? 0 : s_lo;
        const int32_t my_ope = threadIdx.x < (unsigned)P.k ? decode_slot_ope(P, u, (int)threadIdx.x) : 0;
        int32_t ope[kKMax];
#pragma unroll
        for (int j = 0; j < kKMax; j++) ope[j] = __shfl_sync(0xffffffffu, my_ope, j);
        if (threadIdx.x == 0) {
            int32_t sum_n = 0;
            for (int j = 0; j < P.k; j++)
                if (ope[j]) sum_n += ope[j] - P.slot[j].ops + 1;
            Result& R = S->result;
            R.key = ((unsigned long long)(sum_n + 1) << 40) | u;
            R.y_best = drop ? s_y0 : s_ylo;
            R.y0 = s_y0;
            R.evaluated = (unsigned long long)s_preds;
            for (int j = 0; j < kKMax; j++) R.end_op[j] = drop ? 0 : ope[j];
            R.total_ops = drop ? 0 : sum_n;
            R.status = drop ? 1 : 0;
            R.pad = (uint32_t)s_rounds;
            if (P.mapped) publish_mapped(R, P.mapped, P.seq);
        }
    }
}

cudaError_t launch_mway(const Plan& P, const W234& W, const float* w1b1, int ways, Scratch* S, cudaStream_t st) {
    if (P.D > 80) return cudaErrorInvalidValue;
    mway_kernel<<<1, kMwayThreads, 0, st>>>(P, W, w1b1, ways, S);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// launchers
// ---------------------------------------------------------------------------
cudaError_t launch_encode_grid(const Plan& P, uint64_t first, uint64_t count, int16_t* out, int nsm,
                               cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    if (P.D == 24 && (reinterpret_cast<uintptr_t>(out) & 15u) == 0) {
        const size_t smem = 2 * kEnc24Rows * 3 * sizeof(uint4) + 16 * sizeof(uint4) + 64;
        cudaError_t e = cudaFuncSetAttribute(encode_grid24_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
        const uint64_t blocks = (count + kEnc24Rows - 1) / kEnc24Rows;
        const int grid = (int)(blocks < (uint64_t)nsm * 2 ? blocks : (uint64_t)nsm * 2);
        encode_grid24_kernel<<<grid, kEnc24Threads, smem, st>>>(P, first, count, out);
        return cudaGetLastError();
    }
    const uint64_t blocks = (count + kEncThreads - 1) / kEncThreads;
    const int grid = (int)(blocks < (uint64_t)nsm * 16 ? blocks : (uint64_t)nsm * 16);
    const size_t smem = (size_t)kEncThreads * P.D * sizeof(int16_t);
    encode_grid_kernel<<<grid, kEncThreads, smem, st>>>(P, first, count, out);
    return cudaGetLastError();
}

// a3 fast path for D = 24 (N = 8): persistent blocks stream tiles of 256
// records (84 B each, 21.5 KB): the next tile's records are loaded into
// registers (coalesced 16-byte loads) while the current tile is encoded from
// shared memory; each thread zeroes its 48-byte row in a stage and stores the
// bitmap entries and the (ops | ope << 16, bs | seqlen << 16) words of its
// present models at their Fig.-8 positions; the stage is written back with
// coalesced 16-byte streaming stores.
constexpr int kEncG24Threads = 256;
constexpr uint32_t kRecW = sizeof(GroupRec) / 4;                       // 21 words
constexpr int kTileV = kEncG24Threads * (int)sizeof(GroupRec) / 16;    // 1,344 x 16 B
constexpr int kPerV = (kTileV + kEncG24Threads - 1) / kEncG24Threads;  // 6

__device__ __forceinline__ bool group_row24(const uint32_t* r, uint4* row) {
    const int k = (int)r[0];
    int32_t m[kKMax];
    bool ok = k >= 0 && k <= kKMax;
#pragma unroll
    for (int j = 0; j < kKMax; j++) {
        m[j] = (int32_t)r[1 + 5 * j];
        if (j < k) {
            ok = ok && m[j] >= 1 && m[j] <= 8;
#pragma unroll
            for (int i = 0; i < j; i++) ok = ok && m[i] != m[j];
        }
    }
    row[0] = make_uint4(0, 0, 0, 0);
    row[1] = make_uint4(0, 0, 0, 0);
    row[2] = make_uint4(0, 0, 0, 0);
    if (ok) {
        uint32_t* rw = reinterpret_cast<uint32_t*>(row);
        uint16_t* rh = reinterpret_cast<uint16_t*>(row);
#pragma unroll
        for (int j = 0; j < kKMax; j++) {
            if (j >= k) continue;
            int p = 0;
#pragma unroll
            for (int i = 0; i < kKMax; i++) p += (i < k && m[i] < m[j]) ? 1 : 0;
            rh[m[j] - 1] = 1;  // bitmap x[m - 1] = 1
            rw[4 + 2 * p] = (r[2 + 5 * j] & 0xFFFFu) | (r[3 + 5 * j] << 16);  // ops | ope
            rw[5 + 2 * p] = (r[4 + 5 * j] & 0xFFFFu) | (r[5 + 5 * j] << 16);  // bs | seqlen
        }
    }
    return ok;
}

__global__ void __launch_bounds__(kEncG24Threads) encode_groups24_kernel(const GroupRec* __restrict__ groups,
                                                                         uint64_t count,
                                                                         int16_t* __restrict__ out,
                                                                         uint32_t* __restrict__ bad) {
    __shared__ __align__(16) uint32_t s_rec[kEncG24Threads * kRecW];
    __shared__ __align__(16) uint4 s_row[kEncG24Threads * 3];
    __shared__ uint32_t s_bad;
    const int tid = threadIdx.x;
    if (tid == 0) s_bad = 0;
    const uint64_t ntiles = (count + kEncG24Threads - 1) / kEncG24Threads;
    uint4 a[kPerV];
    auto load = [&](uint64_t t) {  // full tiles: into registers
        const uint4* src = reinterpret_cast<const uint4*>(groups + t * kEncG24Threads);
#pragma unroll
        for (int u = 0; u < kPerV; u++) {
            const int i = tid + u * kEncG24Threads;
            if (i < kTileV) a[u] = __ldcs(src + i);
        }
    };
    auto full = [&](uint64_t t) { return (t + 1) * kEncG24Threads <= count; };
    uint32_t nbad = 0;
    uint64_t t = blockIdx.x;
    if (t < ntiles && full(t)) load(t);
    for (; t < ntiles; t += gridDim.x) {
        const uint32_t n = (uint32_t)min((uint64_t)kEncG24Threads, count - t * kEncG24Threads);
        if (n == kEncG24Threads) {
#pragma unroll
            for (int u = 0; u < kPerV; u++) {
                const int i = tid + u * kEncG24Threads;
                if (i < kTileV) reinterpret_cast<uint4*>(s_rec)[i] = a[u];
            }
        } else {
            const uint32_t* s32 = reinterpret_cast<const uint32_t*>(groups + t * kEncG24Threads);
            for (uint32_t j = tid; j < n * kRecW; j += kEncG24Threads) s_rec[j] = __ldcs(s32 + j);
        }
        __syncthreads();
        const uint64_t tn = t + gridDim.x;
        if (tn < ntiles && full(tn)) load(tn);  // in flight while this tile is encoded
        if ((uint32_t)tid < n) nbad += group_row24(s_rec + tid * kRecW, s_row + tid * 3) ? 0u : 1u;
        __syncthreads();
        uint4* dst = reinterpret_cast<uint4*>(out + t * kEncG24Threads * 24);
        for (uint32_t j = tid; j < n * 3; j += kEncG24Threads) __stcs(dst + j, s_row[j]);
        __syncthreads();
    }
    if (nbad) atomicAdd(&s_bad, nbad);
    __syncthreads();
    if (tid == 0 && bad && s_bad) atomicAdd(bad, s_bad);
}

cudaError_t launch_encode_groups(const void* groups, uint64_t count, int32_t n_models, int32_t D, int16_t* out,
                                 uint32_t* bad, int nsm, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    if (D == 24 && n_models == 8 && (reinterpret_cast<uintptr_t>(out) & 15u) == 0 &&
        (reinterpret_cast<uintptr_t>(groups) & 15u) == 0) {
        const uint64_t blocks = (count + kEncG24Threads - 1) / kEncG24Threads;
        const int grid = (int)(blocks < (uint64_t)nsm * 6 ? blocks : (uint64_t)nsm * 6);
        encode_groups24_kernel<<<grid, kEncG24Threads, 0, st>>>(reinterpret_cast<const GroupRec*>(groups), count,
                                                                 out, bad);
        return cudaGetLastError();
    }
    const uint64_t blocks = (count + kEncThreads - 1) / kEncThreads;
    const int grid = (int)(blocks < (uint64_t)nsm * 16 ? blocks : (uint64_t)nsm * 16);
    const size_t smem = (size_t)kEncThreads * D * sizeof(int16_t);
    encode_groups_kernel<<<grid, kEncThreads, smem, st>>>(reinterpret_cast<const GroupRec*>(groups), count,
                                                           n_models, D, out, bad);
    return cudaGetLastError();
}

cudaError_t launch_predict_fp32(const W234& W, const W1P* w1p, const float* w1b1, int32_t D, const int16_t* x,
                                uint64_t count, float* y, int nsm, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    if (D == 24 && w1p && (reinterpret_cast<uintptr_t>(x) & 15u) == 0) {
        const uint64_t blocks = ((count + kPred24Rows - 1) / kPred24Rows + kPredThreads - 1) / kPredThreads;
        const int grid = (int)(blocks < (uint64_t)nsm * 16 ? blocks : (uint64_t)nsm * 16);
        predict24_fp32_kernel<<<grid, kPredThreads, 0, st>>>(*w1p, W, x, count, y);
        return cudaGetLastError();
    }
    const uint64_t blocks = (count + kPredThreads - 1) / kPredThreads;
    const int grid = (int)(blocks < (uint64_t)nsm * 8 ? blocks : (uint64_t)nsm * 8);
    const size_t smem = (size_t)(kHidden * D + kHidden) * sizeof(float);
    predict_fp32_kernel<<<grid, kPredThreads, smem, st>>>(W, w1b1, D, x, count, y);
    return cudaGetLastError();
}

cudaError_t launch_select(const Plan& P, uint64_t first, uint64_t count, const float* lat, float H,
                          unsigned long long* best, int nsm, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    const uint64_t blocks = (count + kSelThreads * kSelPer - 1) / (kSelThreads * kSelPer);
    const int grid = (int)(blocks < (uint64_t)nsm * 8 ? blocks : (uint64_t)nsm * 8);
    select_kernel<<<grid, kSelThreads, 0, st>>>(P, first, count, lat, H, best);
    return cudaGetLastError();
}

cudaError_t launch_fused_fp32(const Plan& P, const W234& W, const float* w1b1, Scratch* S, int nsm,
                              cudaStream_t st, int* grid_out) {
    uint32_t maxcnt = 0;
    for (int s = 0; s < P.n_seg; s++)
        for (int j = 0; j < kKMax; j++) maxcnt = P.seg[s].cnt[j] > maxcnt ? P.seg[s].cnt[j] : maxcnt;
#ifndef EXP_FP32X1
    if (maxcnt < 32768u) {  // the packed walker holds a digit as 0x6400 + v in 16 bits

        const uint64_t n_pairs = (P.n_tiles + 1) / 2;
        uint64_t g = (uint64_t)nsm * kFused2BlocksPerSM;
        if (n_pairs < g) g = n_pairs;
        if (g < 1) g = 1;
        *grid_out = (int)g;
        if (P.n_seg <= 8) {  // decisions: the short parameter block
            PlanDecision Ps;
            memcpy(&Ps, &P, sizeof(PlanDecision));
            fused_fp32x2_kernel<PlanDecision><<<(int)g, kFused2Threads, 0, st>>>(Ps, W, w1b1, S);
        } else {
            fused_fp32x2_kernel<Plan><<<(int)g, kFused2Threads, 0, st>>>(P, W, w1b1, S);
        }
        return cudaGetLastError();
    }
#endif
    uint64_t g = (uint64_t)nsm * kFusedBlocksPerSM;
    if (P.n_tiles < g) g = P.n_tiles;
    if (g < 1) g = 1;
    *grid_out = (int)g;
    fused_fp32_kernel<<<(int)g, kFusedThreads, 0, st>>>(P, W, w1b1, S);
    return cudaGetLastError();
}

cudaError_t launch_finalize_gather(Scratch* S, int nranks, MappedRec* mapped, uint32_t seq, cudaStream_t st) {
    finalize_gather_kernel<<<1, 32, 0, st>>>(S, nranks, mapped, seq);
    return cudaGetLastError();
}

}  // namespace abacus
