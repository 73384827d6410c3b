// kernels_tc.cu -- tensor-core (tcgen05 / TMEM) kernels of the Abacus search.
//
//   fused_tc_kernel        a2..a5 fused: enumerate -> layer-1 operand in TMEM ->
//                          layer 1, 2, 3 and output MMAs (ReLU + pack in the
//                          epilogues) -> headroom mask -> running max key
//
//   fused_batch_tc_kernel  the same for many independent plans per launch
//                          (NEXT-4 decision batches and what-if variants)
//   predict24_tc_kernel    a4 alone, D = 24: int16 Fig.-8 rows from HBM (TMA)
//   predict_tc_kernel      a4 alone, any D <= 31
//
// CTA = NG groups of 4 warps.  A group owns 128 candidate rows = the 128 TMEM
// lanes (warp q of a group reaches lanes 32q..32q+31) and a private slice of
// TMEM columns; one elected thread issues the group's MMAs (M = 128, N = 32,
// or 8 for the output layer, K = 16 per instruction, A from TMEM, B = weights
// resident in shared memory) and commits them to the group's mbarrier.
// Groups run independently, so while one group waits on its MMA the others
// run their epilogues.
//
// Numerics (reading r2, §4):
//   fp16 (FMT 0): weights and activations fp16 RNE; layers are rescaled by
//     exact powers of two so activations stay in fp16 range (ReLU is
//     positively homogeneous, so the output is unchanged).  The output
//     accumulates in fp32, hidden layers 2-3 in f16 with their biases added in
//     the f16 epilogue; b4 is added in fp32.  Layer 1 accumulates in f16 in the
//     search kernels (true digits v against an uncompensated table) and in fp32
//     in the standalone predict kernels (features as 1024 + v).
//   bf16 (FMT 1): layer 1 as in fp16 (fp16 digit / feature operand, fp16
//     table, fp32 accumulation), then bf16 activations; W2 and w4 bf16 (hi),
//     W3 = W3_hi + W3_lo (both multiplied); hidden biases as a (hi, lo) pair
//     against a constant-1 K column; fp32 accumulation; b4 in fp32.
//   Digits / features enter as the exact fp16 values 1024 + v (v < 1024), or
//   split as 256 hi + lo above (SPLIT).
#include <cuda_runtime.h>
#include <math.h>

#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "common.cuh"
#include "device_common.cuh"
#include "internal.h"
#include "tc_ptx.cuh"

namespace abacus {

using namespace tc;


struct TcParams {
    const uint8_t* blob;  // device weight blob (layer 2, layer 3, output chunks)
    uint32_t bytes;
    float l1_scale;
    float b4;             // output bias (fp32)
};


template <int FMT>
struct TcCfg {
    static constexpr int kNchL1 = 1;                     // layer-1 B chunks per segment (fused; fp16 table)
    static constexpr int kNchHid = FMT == 0 ? 3 : 5;     // hidden-layer B chunks
    static constexpr int kNchOut = FMT == 0 ? 3 : 5;     // output-layer B chunks
    static constexpr uint32_t kOne2 = FMT == 0 ? 0x3C003C00u : 0x3F803F80u;  // (1, 1)
};

// hi/lo split of an fp32 value into two 16-bit values (hi + lo ~ v)
template <int FMT>
__device__ __forceinline__ void split16(float v, uint16_t& hi, uint16_t& lo) {
    hi = to16<FMT>(v);
    lo = to16<FMT>(v - from16<FMT>(hi));
}

// Layer-1 B operand per segment: rows n = hidden unit, K columns
//   k0 = c_hi, k1 = c_lo, then per slot j:
//     SPLIT:   k(2+2j) = 256 w_j, k(3+2j) = w_j   (digit = 256 hi + lo)
//     !SPLIT:  k(2+j)  = w_j                      (digit exact in the format)
// The table is fp16 for both paths (FMT = 0 here; the bf16 path switches to
// bf16 operands from layer 2 on).
// c = b1 + W1 x0 (Fig.-8 vector of the segment's v = 0 group), w_j = the
// W1 column of slot j's ope at its Fig.-8 position.
template <int FMT, bool SPLIT, bool TRUEV = false>
__device__ void build_b1_fused(const Plan& P, const float* __restrict__ w1b1, float scale, uint8_t* s_b1, int t0,
                               int nt) {
    constexpr int NCH = TcCfg<FMT>::kNchL1;
    const int D = P.D;
    const float* b1 = w1b1 + kHidden * D;
    for (int e = t0; e < P.n_seg * kHidden; e += nt) {
        const int s = e / kHidden, n = e % kHidden;
        const SegP& g = P.seg[s];
        const float* w = w1b1 + n * D;
        float c = b1[n];
        float wj[kKMax] = {0.0f, 0.0f, 0.0f, 0.0f};  // per box digit
        for (int j = 0; j < kKMax; j++) {
            if (j >= P.k || !((g.mask >> j) & 1u)) continue;
            const SlotP& sl = P.slot[j];
            const int f = P.n_models + 4 * g.pos[j];
            c = fmaf(w[sl.model_id - 1], 1.0f, c);
            c = fmaf(w[f + 0], (float)sl.ops, c);
            c = fmaf(w[f + 1], (float)g.ope0[j], c);
            c = fmaf(w[f + 2], (float)sl.bs, c);
            c = fmaf(w[f + 3], (float)sl.seqlen, c);
            wj[g.dpos[j]] = w[f + 1] * scale;  // column of slot j's box digit
        }
        c *= scale;
        if (FMT == 0 && !SPLIT && !TRUEV) {  // digits enter as 1024 + v (store_a1): remove 1024 w_j as the MMA sees it
            for (int j = 0; j < kKMax; j++) c -= 1024.0f * from16<FMT>(to16<FMT>(wj[j]));
        }
        uint16_t ch, cl;
        split16<FMT>(c, ch, cl);
        uint8_t* base = s_b1 + (size_t)s * NCH * kChunkBytesN32;
        for (int k = 0; k < 16; k++) {
            uint16_t v0 = 0, v1 = 0;
            int j = -1;
            float m = 1.0f;
            if (k == 0) v0 = ch;
            else if (k == 1) v0 = cl;
            else if (SPLIT && k < 2 + 2 * kKMax) { j = (k - 2) >> 1; m = ((k - 2) & 1) ? 1.0f : 256.0f; }
            else if (!SPLIT && k < 2 + kKMax) { j = k - 2; }
            if (j >= 0) {
                uint16_t h, l;
                split16<FMT>(wj[j], h, l);
                if (FMT == 0) {
                    v0 = to16<FMT>(wj[j] * m);
                } else {
                    v0 = to16<FMT>(from16<FMT>(h) * m);
                    v1 = to16<FMT>(from16<FMT>(l) * m);
                }
            }
            *reinterpret_cast<uint16_t*>(base + b_offset(n, k)) = v0;
            if (NCH > 1) *reinterpret_cast<uint16_t*>(base + kChunkBytesN32 + b_offset(n, k)) = v1;
        }
    }
}

// shared-memory carve-up common to both kernels
struct TcSmem {
    uint32_t w2, w3, w4;  // byte offsets of the weight chunks
    uint32_t b1;          // layer-1 B tables
    uint32_t bars;        // mbarriers
    uint32_t tmem_slot;
    uint32_t stage;       // predict: per-group feature staging
    uint32_t total;
};

template <int FMT>
__host__ __device__ inline TcSmem tc_smem_layout(int n_l1_tables, uint32_t l1_table_bytes, int ng,
                                                  uint32_t stage_bytes_per_group) {
    TcSmem L{};
    uint32_t o = 0;
    L.w2 = o;
    o += TcCfg<FMT>::kNchHid * kChunkBytesN32;
    L.w3 = o;
    o += TcCfg<FMT>::kNchHid * kChunkBytesN32;
    L.w4 = o;
    o += TcCfg<FMT>::kNchOut * kChunkBytesN16;
    o = (o + 1023u) & ~1023u;
    L.b1 = o;
    o += (uint32_t)n_l1_tables * l1_table_bytes;
    o = (o + 15u) & ~15u;
    L.stage = o;
    o += (uint32_t)ng * stage_bytes_per_group;
    o = (o + 7u) & ~7u;
    L.bars = o;
    o += 8u * (uint32_t)ng;
    L.tmem_slot = o;
    o += 16;
    L.total = o;
    return L;
}

// per-"group" share of the stage area that holds W1 | b1 (fp32) for the table build
__host__ __device__ inline uint32_t w1_stage_bytes(int D, int ng) {
    const uint32_t total = (uint32_t)(kHidden * D + kHidden) * 4u;
    return (total + (uint32_t)ng * 16u - 1u) / ((uint32_t)ng * 16u) * 16u;
}

// ---------------------------------------------------------------------------
// fused search
//
// A group (4 warps = the 128 TMEM lanes, warp q reaching lanes 32q..32q+31)
// keeps TWO tiles in flight (TMEM slots X and Y) that move through the layers
// in lock step: one MMA commit covers both, so a stage costs one mbarrier
// wait, two overlapped tcgen05.ld, one tcgen05.st wait and one hand-off for
// two tiles, while the CTA's other groups keep the tensor pipe fed.
// Per group 96 TMEM columns: D_X [0,32) D_Y [32,64) A_X [64,80) A_Y [80,96);
// the layer-1 operand A1 aliases the first 8 columns of A.  One constant
// chunk (1, 1, 0, ...) at column 480 supplies the bias rows of every B operand.
// ---------------------------------------------------------------------------
struct TileIO {
    uint32_t d, a1, a;  // TMEM addresses (column part; lane 0)
};

// Layer-1 operand row.  fp16 unsplit (digits <= 1024): the digits enter as the
// exact fp16 values 1024 + v, built by integer adds on the bit patterns
// (0x6400 + v); build_b1_fused removes 1024 * sum_j w_j from the constant.
// Columns 3..7 are not written: their K rows of B are zero and the stale
// activations they hold are finite (the A regions are zeroed at start).
template <int FMT, bool SPLIT>
__device__ __forceinline__ void store_a1(uint32_t taddr, const uint32_t (&v)[kKMax]) {
    if (FMT == 0 && !SPLIT) {
        uint32_t a[4];
        a[0] = TcCfg<FMT>::kOne2;
        a[1] = 0x64006400u + v[0] + (v[1] << 16);  // exact up to v = 1024 (0x6800 = 2048)
        a[2] = 0x64006400u + v[2] + (v[3] << 16);
        a[3] = 0u;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(taddr), "r"(a[0]),
                     "r"(a[1]), "r"(a[2]), "r"(a[3])
                     : "memory");
        return;
    }
    uint32_t a[8];
    a[0] = TcCfg<FMT>::kOne2;
    if (SPLIT) {
#pragma unroll
        for (int j = 0; j < kKMax; j++) a[1 + j] = pack2<FMT>((float)(v[j] >> 8), (float)(v[j] & 255u));
        a[5] = a[6] = a[7] = 0;
    } else {
        a[1] = pack2<FMT>((float)v[0], (float)v[1]);
        a[2] = pack2<FMT>((float)v[2], (float)v[3]);
        a[3] = a[4] = a[5] = a[6] = a[7] = 0;
    }
    tmem_st8(taddr, a);
}

// The MMA pipeline of one group.  Operand hand-off: after writing its 32 rows
// a warp fences its tcgen05.st and ARRIVES on the group's named barrier
// without blocking; only the stage's issuing warp SYNCs (waits for all 128
// threads), then issues the MMAs from one elected lane and commits them to the
// group's mbarrier.  The issuer rotates over the group's 4 warps (one per
// SMSP): hand-off position p = 0 (issue layer 2), 1 (layer 3), 2 (output),
// 3 (layer 1 of the next tiles).
template <int FMT>
struct TcPipe {
    TileIO X, Y;
    uint32_t tCx, tCy, lane_off, bar_id, ph;  // bias constant chunk of X / Y (may be shared)
    uint64_t* bar;
    uint64_t db2, db3, db4;
#ifndef EXP_NO_PRE
    uint64_t db2u, db3u, db4u;  // the layers' second K chunk
    uint32_t xa8, ya8;          // the second half of A
#endif

    uint32_t hb_smem;  // fp16: shared address of layer 2's bias words (layer 3's follow one blob later)
    bool me[4];
    // fp16 unsplit kernels: layer 1 accumulates in f16 from the true digits v
    // (store_a1_true) against a table without the 1024 offset, so its epilogue is
    // a packed 16-bit TMEM load and a max.f16x2 ReLU (the bias is in the MMA)
    bool l1f16 = false;
    // fp16: the output layer runs without its bias K chunk and b4 is added to y
    // in fp32 when y is read (one MMA fewer per tile)
    bool outbias = false;
    float b4 = 0.0f;
    __device__ __forceinline__ void set_outbias(float bias) {
        outbias = true;  // both formats: b4 in fp32 at the read of y, no output bias chunk
        b4 = bias;
    }
    __device__ __forceinline__ uint32_t add_b4(uint32_t ybits) const {
        return outbias ? __float_as_uint(__uint_as_float(ybits) + b4) : ybits;
    }
#ifdef EXP_STAGETRACE
    unsigned long long* tr = nullptr;  // CTA 0, group 0, lane 0 of each warp
    uint32_t it = 0, wqq = 0;
    __device__ __forceinline__ void stamp(int st, int k) {
        if (tr && it >= 64 && it < 80 && (threadIdx.x & 31) == 0) {
            long long c;
            asm volatile("mov.u64 %0, %%clock64;" : "=l"(c));
            tr[16 + (((it - 64) * 4 + wqq) * 4 + st) * 3 + k] = (unsigned long long)c;
        }
    }
#else
    __device__ __forceinline__ void stamp(int, int) {}
#endif

    // fused layout: 96 columns per group, one constant chunk at 480 for all
    __device__ __forceinline__ void init(uint32_t tbase, int g, int wq, uint64_t* mbar, uint64_t d2, uint64_t d3,
                                         uint64_t d4) {
        const uint32_t col = tbase + (uint32_t)g * 96u;
        init_layout(TileIO{col + 0, col + 64, col + 64}, TileIO{col + 32, col + 80, col + 80}, tbase + 480,
                    tbase + 480, g, wq, mbar, d2, d3, d4);
    }
    __device__ __forceinline__ void init_layout(const TileIO& x, const TileIO& y, uint32_t cx, uint32_t cy, int g,
                                                int wq, uint64_t* mbar, uint64_t d2, uint64_t d3, uint64_t d4) {
        X = x;
        Y = y;
        tCx = cx;
        tCy = cy;
        lane_off = (uint32_t)(wq * 32) << 16;
        bar_id = 1 + (uint32_t)g;
        ph = 0;
        bar = mbar;
        db2 = d2;
        db3 = d3;
        db4 = d4;
        // opaque copies: the compiler keeps the descriptors live instead of
        // rebuilding them from the shared-memory base at every issue (~7 uniform
        // instructions per stage on the issuing warp: +1.3 % on config 4)
        asm volatile("mov.b64 %0, %0;" : "+l"(db2));
        asm volatile("mov.b64 %0, %0;" : "+l"(db3));
        asm volatile("mov.b64 %0, %0;" : "+l"(db4));
#ifndef EXP_NO_PRE
        db2u = db2 + (kChunkBytesN32 >> 4);
        db3u = db3 + (kChunkBytesN32 >> 4);
        db4u = db4 + (kChunkBytesN16 >> 4);
        xa8 = X.a + 8;
        ya8 = Y.a + 8;
        asm volatile("mov.b64 %0, %0;" : "+l"(db2u));
        asm volatile("mov.b64 %0, %0;" : "+l"(db3u));
        asm volatile("mov.b64 %0, %0;" : "+l"(db4u));
        asm volatile("mov.b32 %0, %0;" : "+r"(xa8));
        asm volatile("mov.b32 %0, %0;" : "+r"(ya8));
#endif

        // fp16: the bias chunk of each hidden layer holds its 16 f16 bias pairs instead
        hb_smem = ((uint32_t)(d2 & 0x3FFFu) << 4) + 2u * kChunkBytesN32;
#pragma unroll
        for (int p = 0; p < 4; p++) me[p] = ((g + p) & 3) == wq;
    }
    // zero this warp's lanes of the A regions once: columns the layer-1 row
    // leaves unwritten must hold finite values (their B rows are zero)
    __device__ __forceinline__ void zero_a() const {
        uint32_t z[16];
#pragma unroll
        for (int i = 0; i < 16; i++) z[i] = 0u;
        tmem_st16(X.a + lane_off, z);
        tmem_st16(Y.a + lane_off, z);
        tmem_wait_st();
    }
    __device__ __forceinline__ bool handoff(bool mine) const {
        fence_before();
        if (mine) {
            named_bar_sync(bar_id, 128);
            fence_after();
        } else {
            named_bar_arrive(bar_id, 128);
        }
        return mine;
    }
    __device__ __forceinline__ void wait() {
        mbar_wait(bar, ph);
        ph ^= 1u;
        fence_after();
    }
    // layer-1 MMA of one tile against its segment's B operand (no commit).  Both
    // formats: fp16 operands and an fp16 segment table; the fp16 search kernels
    // (l1f16) store the true digits v and accumulate in f16, the bf16 path the
    // digits as the exact fp16 1024 + v against a compensated table with fp32
    // accumulation, then bf16 operands from layer 2 on (its layer-1 epilogue
    // packs bf16)
    __device__ __forceinline__ void issue_l1(const TileIO& T, uint64_t db) const {
        constexpr uint32_t id32 = idesc_f16(0, 32);
        if (l1f16) {
            constexpr uint32_t id16 = idesc_f16(0, 32, false);
            mma_ts_elect(T.d, T.a1, db, id16, 0u);
            return;
        }
        mma_ts_elect(T.d, T.a1, db, id32, 0u);
    }
    __device__ __forceinline__ void commit() const { mma_commit_elect(bar); }
    // layer LAYER (0: layer 2, 1: layer 3, 2: output) of X (and Y), one commit
    template <int LAYER, bool TWO>
    __device__ __forceinline__ void issue_next() const {
        constexpr uint32_t CH = LAYER == 2 ? kChunkBytesN16 : kChunkBytesN32;
        // fp16: hidden layers 2 and 3 accumulate in f16 (their epilogues then read
        // half the TMEM bytes), the output layer in fp32 (layer 1: issue_l1)
        constexpr uint32_t ID = idesc_f16(FMT, LAYER == 2 ? 8 : 32, FMT != 0 || LAYER == 2);
        const uint64_t db = LAYER == 0 ? db2 : (LAYER == 1 ? db3 : db4);
        if (FMT == 1) {
            // bf16 (DESIGN.md r2): layer 2 = hi weights + bias chunk (chunks 0, 1, 4),
            // layer 3 = hi + lo weights + bias chunk (0..4), output = hi weights (0, 1),
            // b4 added in fp32 when y is read
            if (TWO) {
#ifndef EXP_NO_PRE
                const uint64_t dbu = LAYER == 0 ? db2u : (LAYER == 1 ? db3u : db4u);
                if (LAYER == 0)
                    issue_pair_bf16_pre<ID, (CH >> 4), 3>(X.d, X.a, xa8, Y.d, Y.a, ya8, tCx, tCy, db, dbu, bar);
                else if (LAYER == 1)
                    issue_pair_bf16_pre<ID, (CH >> 4), 5>(X.d, X.a, xa8, Y.d, Y.a, ya8, tCx, tCy, db, dbu, bar);
                else
                    issue_pair2_pre<ID>(X.d, X.a, xa8, Y.d, Y.a, ya8, db, dbu, bar);
#else
                if (LAYER == 0) issue_layer2_asm<1, ID, CH, true, 4>(X.d, X.a, Y.d, Y.a, tCx, tCy, db, bar);
                else if (LAYER == 1) issue_layer2x5_asm<ID, CH>(X.d, X.a, Y.d, Y.a, tCx, tCy, db, bar);
                else issue_layer2_asm<1, ID, CH, false>(X.d, X.a, Y.d, Y.a, tCx, tCy, db, bar);
#endif
            } else {
                if (LAYER == 0) issue_layer_asm<1, ID, CH, true, 4, false>(X.d, X.a, tCx, db, bar);
                else if (LAYER == 1) issue_layer_asm<1, ID, CH, true, 4, true>(X.d, X.a, tCx, db, bar);
                else issue_layer_asm<1, ID, CH, false, 2, false>(X.d, X.a, tCx, db, bar);
            }
            return;
        }
        // fp16: no bias MMA in any layer (hidden biases in the f16 epilogue, b4 in fp32)
#ifndef EXP_NO_PRE
        // every issue operand precomputed (+0.9 % on config 4)
        if (TWO) {
            const uint64_t dbu = LAYER == 0 ? db2u : (LAYER == 1 ? db3u : db4u);
            issue_pair2_pre<ID>(X.d, X.a, xa8, Y.d, Y.a, ya8, db, dbu, bar);
            return;
        }
#endif
        if (TWO) issue_layer2_asm<0, ID, CH, false>(X.d, X.a, Y.d, Y.a, tCx, tCy, db, bar);
        else issue_layer_asm<0, ID, CH, false>(X.d, X.a, tCx, db, bar);
    }
    // wait for the previous layer's MMAs, ReLU + pack into A, hand off, issue layer LAYER
    // CONST: also (re)write the per-tile constant chunks (layouts where the
    // chunk shares the columns of the consumed layer-1 operand)
    template <int LAYER, bool TWO, bool CONST = false>
    __device__ __forceinline__ void stage() {
        stage_as<LAYER, TWO, CONST>(me[LAYER]);
    }
    // the same with the issuer role given by the caller (a compile-time
    // constant in the fused kernel's role-specialised loop)
    template <int LAYER, bool TWO, bool CONST = false>
    __device__ __forceinline__ void stage_as(bool mine) {
        epilogue<LAYER, TWO, CONST>();
        tmem_wait_st();
        stamp(LAYER, 1);
        if (handoff(mine)) {
            stamp(LAYER, 2);
            issue_next<LAYER, TWO>();
        }
    }
    // wait for the previous layer's MMAs, ReLU + pack into A (no st wait)
    template <int LAYER, bool TWO, bool CONST = false>
    __device__ __forceinline__ void epilogue() {
        uint32_t hbw[16];
        // layer 3's bias words sit one hidden-layer blob (kNchHid chunks) after layer 2's
        if (FMT == 0 && LAYER >= 1)
            lds_words16(hb_smem + (LAYER == 1 ? 0u : (uint32_t)TcCfg<FMT>::kNchHid * kChunkBytesN32), hbw);
        wait();
        stamp(LAYER, 0);
        if (FMT == 0 && LAYER >= 1) {
            // f16 accumulators of layer 2 / 3 (no bias MMA): bias + ReLU on packed
            // pairs, one HFMA2.RELU per pair; the 16 bias words were loaded from
            // shared memory before the mbarrier wait
            uint32_t a[16], b[16];
            if (TWO) tmem_ld16p_x2(X.d + lane_off, Y.d + lane_off, a, b);
            else tmem_ld16p_x2(X.d + lane_off, X.d + lane_off, a, b);
            const uint32_t one = 0x3C003C00u;
#pragma unroll
            for (int c = 0; c < 16; c++) asm("fma.rn.relu.f16x2 %0, %1, %2, %0;" : "+r"(a[c]) : "r"(one), "r"(hbw[c]));
            tmem_st16(X.a + lane_off, a);
            if (TWO) {
#pragma unroll
                for (int c = 0; c < 16; c++)
                    asm("fma.rn.relu.f16x2 %0, %1, %2, %0;" : "+r"(b[c]) : "r"(one), "r"(hbw[c]));
                tmem_st16(Y.a + lane_off, b);
            }
        } else if (FMT == 0 && LAYER == 0 && TWO && l1f16) {
            // f16 layer-1 accumulator (c and the digits' terms in one MMA): ReLU only
            uint32_t a[16], b[16];
            tmem_ld16p_x2(X.d + lane_off, Y.d + lane_off, a, b);
#pragma unroll
            for (int c = 0; c < 16; c++) asm("max.f16x2 %0, %0, %1;" : "+r"(a[c]) : "r"(0u));
            tmem_st16(X.a + lane_off, a);
#pragma unroll
            for (int c = 0; c < 16; c++) asm("max.f16x2 %0, %0, %1;" : "+r"(b[c]) : "r"(0u));
            tmem_st16(Y.a + lane_off, b);
        } else if (FMT == 0 && LAYER == 0 && !TWO && l1f16) {
            uint32_t a[16], b[16];
            tmem_ld16p_x2(X.d + lane_off, X.d + lane_off, a, b);
#pragma unroll
            for (int c = 0; c < 16; c++) asm("max.f16x2 %0, %0, %1;" : "+r"(a[c]) : "r"(0u));
            tmem_st16(X.a + lane_off, a);
        } else if (TWO) {
            uint32_t a[32], b[32], h[16];
            tmem_ld32x2(X.d + lane_off, Y.d + lane_off, a, b);
#pragma unroll
            for (int c = 0; c < 16; c++) h[c] = pack2_relu<FMT>(a[2 * c], a[2 * c + 1]);
            tmem_st16(X.a + lane_off, h);
#pragma unroll
            for (int c = 0; c < 16; c++) h[c] = pack2_relu<FMT>(b[2 * c], b[2 * c + 1]);
            tmem_st16(Y.a + lane_off, h);
        } else {
            uint32_t a[32], h[16];
            tmem_ld32(X.d + lane_off, a);
#pragma unroll
            for (int c = 0; c < 16; c++) h[c] = pack2_relu<FMT>(a[2 * c], a[2 * c + 1]);
            tmem_st16(X.a + lane_off, h);
        }
        if (CONST) {
            uint32_t c8[8] = {TcCfg<FMT>::kOne2, 0, 0, 0, 0, 0, 0, 0};
            tmem_st8(tCx + lane_off, c8);
            if (TWO) tmem_st8(tCy + lane_off, c8);
        }
    }
    // the same with fixed issuer roles: stage p issued by warp wq == p of the group
    template <bool TWO>
    __device__ __forceinline__ void run_layers_fixed(int wq, uint32_t& yx, uint32_t& yy) {
        stage_as<0, TWO>(wq == 0);
        stage_as<1, TWO>(wq == 1);
        stage_as<2, TWO>(wq == 2);
        wait();
        if (TWO) tmem_ld1x2(X.d + lane_off, Y.d + lane_off, yx, yy);
        else tmem_ld1(X.d + lane_off, yx);
        yx = add_b4(yx);
        if (TWO) yy = add_b4(yy);
    }
    // the three hidden stages, then wait for the output MMA and read y (column 0 of D)
    template <bool TWO, bool CONST = false>
    __device__ __forceinline__ void run_layers(uint32_t& yx, uint32_t& yy) {
        stage<0, TWO, CONST>();
        stage<1, TWO>();
        stage<2, TWO>();
        wait();
        stamp(3, 0);
        if (TWO) tmem_ld1x2(X.d + lane_off, Y.d + lane_off, yx, yy);
        else tmem_ld1(X.d + lane_off, yx);
        yx = add_b4(yx);
        if (TWO) yy = add_b4(yy);
    }
};

// CTA prologue common to both fused kernels: weights -> smem, mbarriers,
// TMEM allocation, the constant chunk
template <int FMT, int NG>
__device__ __forceinline__ uint32_t fused_prologue_tmem(uint64_t* bars, uint32_t* tmem_slot, int warp, int g, int wq) {
    if (threadIdx.x == 0) {
        for (int i = 0; i < NG; i++) mbar_init(&bars[i], 1);
        mbar_fence_init();
    }
    if (warp == 0) {
        tmem_alloc(tmem_slot, 512);
        tmem_relinquish();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tbase = __shfl_sync(0xffffffffu, *tmem_slot, 0);
    if (g == 0) {
        uint32_t c8[8] = {TcCfg<FMT>::kOne2, 0, 0, 0, 0, 0, 0, 0};
        tmem_st8(tbase + 480 + ((uint32_t)(wq * 32) << 16), c8);
        tmem_wait_st();
    }
    fence_before();
    __syncthreads();
    fence_after();
    return tbase;
}

// layer-1 operand row (1, 1, v0 .. v3, 0, 0) of a packed tile row (the fp16
// search kernels: f16 layer-1 accumulation, uncompensated table)
__device__ __forceinline__ void store_a1_packed_true(uint32_t taddr, uint32_t a1, uint32_t a2) {
    // (1024 + v) - 1024 = v exactly in f16 (v < 1024)
    asm volatile(
        "{\n\t.reg .b32 t1, t2;\n\t"
        "sub.rn.f16x2 t1, %1, %3;\n\t"
        "sub.rn.f16x2 t2, %2, %3;\n\t"
        "tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%4, t1, t2, %5};\n\t}" ::"r"(taddr),
        "r"(a1), "r"(a2), "r"(0x64006400u), "r"(0x3C003C00u), "r"(0u)
        : "memory");
}
// layer-1 operand row (1, 1, 1024 + v0 .. 1024 + v3, 0, 0) of a packed tile row
// (the bf16 path: fp32 layer-1 accumulation, compensated table)
__device__ __forceinline__ void store_a1_packed(uint32_t taddr, uint32_t a1, uint32_t a2) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(taddr), "r"(0x3C003C00u),
                 "r"(a1), "r"(a2), "r"(0u)
                 : "memory");
}


template <int FMT, bool SPLIT, int NG, class PL = Plan>
__global__ void __launch_bounds__(NG * 128, 1) fused_tc_kernel(const __grid_constant__ PL Pin,
                                                               const __grid_constant__ TcParams TP,
                                                               const float* __restrict__ w1b1, Scratch* S) {
    const Plan& P = *reinterpret_cast<const Plan*>(&Pin);  // PlanT<8> for decisions: same layout prefix
    extern __shared__ __align__(1024) uint8_t smem[];
    using C = TcCfg<FMT>;
    const TcSmem L = tc_smem_layout<FMT>(P.n_seg, C::kNchL1 * kChunkBytesN32, NG, w1_stage_bytes(P.D, NG));
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);  // one per group
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem + L.tmem_slot);

    const int tid = threadIdx.x;
    const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);  // warp-uniform for the compiler
    const int g = warp >> 2, wq = warp & 3;
    trace_stamp(P, 0);
    // the mbarriers and the TMEM allocation are set up while the weights load
    if (tid == 0) {
        for (int i = 0; i < NG; i++) mbar_init(&bars[i], 1);
        mbar_fence_init();
    }
    if (warp == 0) {
        tmem_alloc(tmem_slot, 512);
        tmem_relinquish();
    }
    {
        const int4* src = reinterpret_cast<const int4*>(TP.blob);
        int4* dst = reinterpret_cast<int4*>(smem);
        for (uint32_t i = tid; i < TP.bytes / 16; i += blockDim.x) dst[i] = src[i];
        // stage W1 | b1 (fp32) for the layer-1 table build
        float* s_w1 = reinterpret_cast<float*>(smem + L.stage);
        for (int i = tid; i < kHidden * P.D + kHidden; i += blockDim.x) s_w1[i] = __ldg(w1b1 + i);
    }
    fence_before();
    __syncthreads();
    fence_after();
    trace_stamp(P, 1);
    const uint32_t tbase = __shfl_sync(0xffffffffu, *tmem_slot, 0);
    constexpr bool kL1 = FMT == 0 && !SPLIT;  // layer 1 in f16 from the true digits (TcPipe::l1f16)
    build_b1_fused<0, SPLIT, kL1>(P, reinterpret_cast<const float*>(smem + L.stage), TP.l1_scale, smem + L.b1, tid,
                               blockDim.x);
    if (g == 0) {  // the constant chunk (1, 1, 0, ...) of the bias rows
        uint32_t c8[8] = {TcCfg<FMT>::kOne2, 0, 0, 0, 0, 0, 0, 0};
        tmem_st8(tbase + 480 + ((uint32_t)(wq * 32) << 16), c8);
        tmem_wait_st();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // weights and tables -> tensor core
    fence_before();
    __syncthreads();
    fence_after();
    trace_stamp(P, 2);

    const uint32_t r = (uint32_t)(tid & 127);
    const uint32_t sbase = smem_u32(smem);
    TcPipe<FMT> pp;
    pp.init(tbase, g, wq, &bars[g], smem_desc(sbase + L.w2), smem_desc(sbase + L.w3), smem_desc(sbase + L.w4));
    pp.set_outbias(TP.b4);
    pp.zero_a();
    pp.l1f16 = kL1;
    auto st1 = [&](uint32_t taddr, uint32_t a1, uint32_t a2) {
        if constexpr (kL1) store_a1_packed_true(taddr, a1, a2);
        else store_a1_packed(taddr, a1, a2);
    };
    const uint64_t d1base = smem_desc(sbase + L.b1);
    constexpr uint32_t kSegStep = C::kNchL1 * (kChunkBytesN32 >> 4);
#ifndef EXP_NO_SEGLO
    // the segment's table descriptor differs from d1base only in its low word (the
    // start address field, < 2^14): one shuffle of that word, no 64-bit arithmetic
    const uint32_t d1lo = (uint32_t)d1base, d1hi = (uint32_t)(d1base >> 32);
    auto issue_l1 = [&](const TileIO& T, int s) {
        const uint32_t lo = __shfl_sync(0xffffffffu, d1lo + (uint32_t)s * kSegStep, 0);
        pp.issue_l1(T, ((uint64_t)d1hi << 32) | lo);
    };
#else
    auto issue_l1 = [&](const TileIO& T, int s) {
        const int su = __shfl_sync(0xffffffffu, s, 0);
        pp.issue_l1(T, d1base + (uint64_t)((uint32_t)su * kSegStep));
    };
#endif
    using T1 = std::integral_constant<bool, false>;
    using T2 = std::integral_constant<bool, true>;

    unsigned long long best = 0;
    float best_y = __int_as_float(0x7fc00000);
    uint64_t wb, we;
    work_range(P.n_tiles, (uint64_t)blockIdx.x * NG + g, (uint64_t)gridDim.x * NG, wb, we);
    if constexpr (!SPLIT) {
        if (wb < we) {
#ifdef EXP_STAGETRACE
            if (blockIdx.x == 0 && g == 0) pp.tr = P.trace;
            pp.wqq = wq;
#endif
            // issuer roles fixed per warp: stage p (0..2 = layers 2, 3, out; 3 =
            // the next layer 1) is issued by the group's warp wq == p, so every
            // SMSP issues one stage of every group; the role test is one
            // compare of the warp-uniform wq with an immediate
            PackedWalker W;
            W.begin(P, wb, r);
            // X rows alternate between two register sets (the loop is unrolled by
            // two with the roles swapped), so the next X row needs no copy
            struct Row {
                uint32_t a1, a2, sn;
                int s;
            };
            Row RA, RB{0u, 0u, 0u, 0};
            uint32_t y1 = 0, y2 = 0, ys = 0;  // Y row: a1, a2, sn
            int sY = 0;
            uint32_t bsn = 1u;
            auto takeY = [&]() { y1 = W.a1; y2 = W.a2; ys = W.sn; sY = W.s; st1(pp.Y.a1 + pp.lane_off, W.a1, W.a2); };
            const bool yLive = wb + 1 < we;  // warp-uniform
            RA = Row{W.a1, W.a2, W.sn, W.s};
            st1(pp.X.a1 + pp.lane_off, RA.a1, RA.a2);
            if (yLive) {
                W.next(P, r);
                takeY();
            }
            tmem_wait_st();
            if (pp.handoff(wq == 3)) {
                issue_l1(pp.X, RA.s);
                if (yLive) issue_l1(pp.Y, sY);
                pp.commit();
            }
            // 32-bit iteration state (a group's range is < 2^32 tiles); y(0) is owed
            // only by the row that holds index 0 (the plan's first tile)
            const uint32_t nw = (uint32_t)(we - wb);
            uint32_t w = 0;
            bool owe_y0 = wb == 0 && P.want_y0 && wq == 0;
            const float Tr = raw_threshold(P.H, pp.b4);  // pp.outbias: b4 is added to y in fp32
            auto iteration = [&](auto two_c, auto next_two_c, Row& cx, Row& nx) {
                constexpr bool TWO = decltype(two_c)::value;
                constexpr bool NTWO = decltype(next_two_c)::value;
                pp.template stage_as<0, TWO>(wq == 0);
                pp.template stage_as<1, TWO>(wq == 1);
                pp.template stage_as<2, TWO>(wq == 2);
                // the next tiles' operand rows are computed while the output MMA runs
                const bool more = w + 2 < nw;  // warp-uniform
                if (more) {
                    W.next(P, r);
                    nx = Row{W.a1, W.a2, W.sn, W.s};
                    if (NTWO) W.next(P, r);
                }
                pp.wait();
                pp.stamp(3, 0);
                uint32_t ybx, yby = 0;
                if (TWO) tmem_ld1x2(pp.X.d + pp.lane_off, pp.Y.d + pp.lane_off, ybx, yby);
                else tmem_ld1(pp.X.d + pp.lane_off, ybx);
                // raw outputs (before b4): the headroom test against Tr, b4 added on a fold
                if (owe_y0) {  // warp-uniform (warp 0 of the group holding index 0)
                    if (r == 0) S->y0 = __fadd_rn(__uint_as_float(ybx), pp.b4);
                    owe_y0 = false;
                }
                if (TWO)
                    fold_packed2_raw(P, Tr, pp.b4, cx.s, cx.a1, cx.a2, cx.sn, __uint_as_float(ybx), sY, y1, y2, ys,
                                     __uint_as_float(yby), best, best_y, bsn);
                else
                    fold_packed_raw(P, Tr, pp.b4, cx.s, cx.a1, cx.a2, cx.sn, __uint_as_float(ybx), best, best_y,
                                    bsn);
                if (more) {
                    st1(pp.X.a1 + pp.lane_off, nx.a1, nx.a2);
                    if (NTWO) takeY();
                    tmem_wait_st();
                    pp.stamp(3, 1);
                    if (pp.handoff(wq == 3)) {
                        pp.stamp(3, 2);
                        issue_l1(pp.X, nx.s);
                        if (NTWO) issue_l1(pp.Y, sY);
                        pp.commit();
                    }
                }
#ifdef EXP_STAGETRACE
                pp.it++;
#endif
                w += 2;
            };
            // the tail: at most one pair with a lone successor, then a lone X
            auto tail = [&](Row& cx, Row& nx) {
                if (w + 1 < nw) {
                    iteration(T2{}, T1{}, cx, nx);
                    if (w < nw) iteration(T1{}, T1{}, nx, cx);
                } else if (w < nw) {
                    iteration(T1{}, T1{}, cx, nx);
                }
            };
            for (;;) {
                if (!(w + 3 < nw)) {
                    tail(RA, RB);
                    break;
                }
                iteration(T2{}, T2{}, RA, RB);
                if (!(w + 3 < nw)) {
                    tail(RB, RA);
                    break;
                }
                iteration(T2{}, T2{}, RB, RA);
            }

        }
    } else if (wb < we) {
        Walker W;
        walker_begin(P, W, wb, r);
        uint32_t vX[kKMax], vY[kKMax];
        int sX = 0, sY = 0;
        bool okX = false, okY = false, zX = false, zY = false;
        // ok: the row is inside its segment (only a segment's last tile is partial)
        auto take = [&](uint32_t (&v)[kKMax], int& s, bool& ok, bool& z) {
            const uint64_t rem = W.u_end - W.ub;  // uniform
            ok = rem >= (uint64_t)kTileM || (uint64_t)r < rem;
            z = false;
#pragma unroll
            for (int j = 0; j < kKMax; j++) v[j] = W.v[j];
            s = W.s;
        };
        auto fold = [&](uint32_t yb, int s, const uint32_t (&v)[kKMax], bool ok, bool z) {
            const float y = __uint_as_float(yb);
            (void)z;
            if (ok) fold_tile(P, s, v, y, best, best_y);
        };
        // index 0 (the drop test's critical-only group) is row 0 of the plan's
        // first tile whenever the plan starts at index 0 (P.want_y0)
        // prologue: tile wb in slot X and (if the group has it) wb + 1 in slot Y
        const bool yLive = wb + 1 < we;  // warp-uniform
        take(vX, sX, okX, zX);
        store_a1<0, SPLIT>(pp.X.a1 + pp.lane_off, vX);
        if (yLive) {
            walker_next(P, W, wb + 1, r);
            take(vY, sY, okY, zY);
            store_a1<0, SPLIT>(pp.Y.a1 + pp.lane_off, vY);
        }
        tmem_wait_st();
        if (pp.handoff(pp.me[3])) {
            issue_l1(pp.X, sX);
            if (yLive) issue_l1(pp.Y, sY);
            pp.commit();
        }
        // one iteration = layers 2, 3, out of the tiles in X (and Y), fold (a5),
        // then tiles w + 2 (and w + 3) enter the slots.  The steady state has
        // both slots full before and after; the tail handles a lone X.
        uint64_t w = wb;
        auto iteration = [&](auto two_c, auto next_two_c) {
            constexpr bool TWO = decltype(two_c)::value;
            constexpr bool NTWO = decltype(next_two_c)::value;
            uint32_t ybx, yby = 0;
            pp.template run_layers<TWO>(ybx, yby);
            if (w == 0 && P.want_y0 && r == 0) S->y0 = __uint_as_float(ybx);
            fold(ybx, sX, vX, okX, zX);
            if (TWO) fold(yby, sY, vY, okY, zY);
            if (w + 2 < we) {
                walker_next(P, W, w + 2, r);
                take(vX, sX, okX, zX);
                store_a1<0, SPLIT>(pp.X.a1 + pp.lane_off, vX);
                if (NTWO) {
                    walker_next(P, W, w + 3, r);
                    take(vY, sY, okY, zY);
                    store_a1<0, SPLIT>(pp.Y.a1 + pp.lane_off, vY);
                }
                tmem_wait_st();
                if (pp.handoff(pp.me[3])) {
                    issue_l1(pp.X, sX);
                    if (NTWO) issue_l1(pp.Y, sY);
                    pp.commit();
                }
            }
            w += 2;
        };
        while (w + 3 < we) iteration(T2{}, T2{});  // both slots full, both continue
        if (w + 1 < we) iteration(T2{}, T1{});    // both full; at most X gets a successor
        if (w < we) iteration(T1{}, T1{});        // X alone
    }
    trace_stamp(P, 3);
    fence_before();
    __syncthreads();
    fence_after();
    if (warp == 0) tmem_dealloc(tbase, 512);
    trace_stamp(P, 4);
    cta_publish_and_finish(P, S, best, best_y);
}

// ---------------------------------------------------------------------------
// batched decisions (NEXT-4): one launch searches many independent decisions.
// The launch's tile PAIRS are split contiguously over all groups; a group
// walks its pairs decision by decision.  On entering a decision it copies the
// decision's plan (header + segments) into its own shared-memory slot and
// builds that decision's layer-1 B operands into its own table region (all
// of the group's MMAs have completed at that point), so the five groups of a
// CTA can be in five different decisions.  On leaving a decision it folds its
// best (key, y) into the decision's accumulator with a 128-bit CAS.
// ---------------------------------------------------------------------------
// a group's plan slot holds up to kMaxSeg segments: decision batches use <= 8
// (kMaxSegBatch), what-if sweeps (NEXT-4) whole grid plans of <= 16
constexpr int kMaxSegSlot = kMaxSeg;
constexpr uint32_t kPlanBatchBytes = (uint32_t)((sizeof(Plan) + 15) & ~size_t(15));

__device__ __forceinline__ void acc_fold(BatchAcc* a, unsigned long long key, float y) {
    unsigned long long ok = a->key, oy = __float_as_uint(a->y);
    while (key > ok) {
        unsigned long long rk, ry;
        const unsigned long long ny = __float_as_uint(y);
        asm volatile(
            "{\n\t"
            ".reg .b128 d, c, n;\n\t"
            "mov.b128 c, {%2, %3};\n\t"
            "mov.b128 n, {%4, %5};\n\t"
            "atom.global.cas.b128 d, [%6], c, n;\n\t"
            "mov.b128 {%0, %1}, d;\n\t"
            "}"
            : "=l"(rk), "=l"(ry)
            : "l"(ok), "l"(oy), "l"(key), "l"(ny), "l"(a)
            : "memory");
        if (rk == ok && ry == oy) return;
        ok = rk;
        oy = ry;
    }
}

template <int FMT>
__host__ __device__ inline TcSmem batch_smem_layout(int D, int ng, uint32_t* plans_off) {
    TcSmem L = tc_smem_layout<FMT>(ng * kMaxSegSlot, TcCfg<FMT>::kNchL1 * kChunkBytesN32, ng,
                                   w1_stage_bytes(D, ng));
    *plans_off = (L.total + 15u) & ~15u;
    L.total = *plans_off + (uint32_t)ng * kPlanBatchBytes;
    return L;
}

template <int FMT, bool SPLIT, int NG>
__global__ void __launch_bounds__(NG * 128, 1) fused_batch_tc_kernel(const BatchDec* __restrict__ decs,
                                                                     const SegP* __restrict__ segs, int32_t n_dec,
                                                                     const uint64_t* __restrict__ n_pairs_dev, int32_t D,
                                                                     const __grid_constant__ TcParams TP,
                                                                     const float* __restrict__ w1b1, BatchAcc* acc,
                                                                     float* y0s) {
    extern __shared__ __align__(1024) uint8_t smem[];
    using C = TcCfg<FMT>;
    uint32_t plans_off;
    const TcSmem L = batch_smem_layout<FMT>(D, NG, &plans_off);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem + L.tmem_slot);
    const int tid = threadIdx.x;
    const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
    const int g = warp >> 2, wq = warp & 3;
    const float* s_w1 = reinterpret_cast<const float*>(smem + L.stage);
    {
        const int4* src = reinterpret_cast<const int4*>(TP.blob);
        int4* dst = reinterpret_cast<int4*>(smem);
        for (uint32_t i = tid; i < TP.bytes / 16; i += blockDim.x) dst[i] = src[i];
        float* w = reinterpret_cast<float*>(smem + L.stage);
        for (int i = tid; i < kHidden * D + kHidden; i += blockDim.x) w[i] = __ldg(w1b1 + i);
    }
    __syncthreads();
    const uint32_t tbase = fused_prologue_tmem<FMT, NG>(bars, tmem_slot, warp, g, wq);

    const uint32_t r = (uint32_t)(tid & 127);
    const uint32_t sbase = smem_u32(smem);
    TcPipe<FMT> pp;
    pp.init(tbase, g, wq, &bars[g], smem_desc(sbase + L.w2), smem_desc(sbase + L.w3), smem_desc(sbase + L.w4));
    pp.set_outbias(TP.b4);
    pp.zero_a();
    constexpr bool kL1 = FMT == 0 && !SPLIT;  // as fused_tc_kernel: layer 1 in f16 from the true digits
    pp.l1f16 = kL1;
    auto st1 = [&](uint32_t taddr, uint32_t a1, uint32_t a2) {
        if constexpr (kL1) store_a1_packed_true(taddr, a1, a2);
        else store_a1_packed(taddr, a1, a2);
    };
    constexpr uint32_t kTable = C::kNchL1 * kChunkBytesN32;
    uint8_t* my_b1 = smem + L.b1 + (size_t)g * kMaxSegSlot * kTable;
    const uint64_t d1base = smem_desc(sbase + L.b1 + (uint32_t)g * kMaxSegSlot * kTable);
    constexpr uint32_t kSegStep = kTable >> 4;
    Plan& P = *reinterpret_cast<Plan*>(smem + plans_off + (size_t)g * kPlanBatchBytes);
    auto issue_l1 = [&](const TileIO& T, int s) {
        const int su = __shfl_sync(0xffffffffu, s, 0);
        pp.issue_l1(T, d1base + (uint64_t)((uint32_t)su * kSegStep));
    };

    const uint64_t n_pairs = *n_pairs_dev;  // written by the planning kernels
    uint64_t pb, pe;
    work_range(n_pairs, (uint64_t)blockIdx.x * NG + g, (uint64_t)gridDim.x * NG, pb, pe);
    if (pb < pe) {
        // decision holding pair pb: the last d with pair0 <= pb
        int d = 0;
        {
            int lo = 0, hi = n_dec - 1;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (decs[mid].pair0 <= pb) lo = mid;
                else hi = mid - 1;
            }
            d = lo;
        }
        uint64_t dec_pair0 = 0, dec_pair_end = 0;
        // plan + layer-1 tables of decision d into this group's slots
        auto load_decision = [&]() {
            named_bar_sync(pp.bar_id, 128);  // every warp is done with the previous plan
            const BatchDec& bd = decs[d];
            const int n_seg = bd.h.n_seg;
            const uint32_t* src = reinterpret_cast<const uint32_t*>(&bd.h);
            uint32_t* dst = reinterpret_cast<uint32_t*>(&P);
            for (uint32_t i = r; i < sizeof(PlanHdr) / 4; i += 128) dst[i] = src[i];
            const uint32_t* ss = reinterpret_cast<const uint32_t*>(segs + bd.seg0);
            uint32_t* sd = reinterpret_cast<uint32_t*>(&P.seg[0]);
            for (uint32_t i = r; i < (uint32_t)n_seg * (sizeof(SegP) / 4); i += 128) sd[i] = ss[i];
            dec_pair0 = bd.pair0;
            dec_pair_end = d + 1 < n_dec ? decs[d + 1].pair0 : n_pairs;
            named_bar_sync(pp.bar_id, 128);
            build_b1_fused<0, SPLIT, kL1>(P, s_w1, TP.l1_scale, my_b1, (int)r, 128);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            named_bar_sync(pp.bar_id, 128);
        };
        unsigned long long best = 0;
        float best_y = __int_as_float(0x7fc00000);
        auto flush = [&]() {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                const unsigned long long k2 = __shfl_xor_sync(0xffffffffu, best, o);
                const float y2 = __shfl_xor_sync(0xffffffffu, best_y, o);
                if (k2 > best) { best = k2; best_y = y2; }
            }
            if ((tid & 31) == 0 && best) acc_fold(&acc[d], best, best_y);
            best = 0;
        };
        if constexpr (!SPLIT) {
            // packed walker + three-instruction fold (as fused_tc_kernel)
            PackedWalkerT<true> W{};
            uint32_t x1 = 0, x2 = 0, xs = 0, y1 = 0, y2 = 0, ys = 0, bsn = 1u;
            int sX = 0, sY = 0;
            uint64_t ltX = 0;
            // move the walker to local tile lt (the next one); a decision's pad tile has no rows
            auto adv = [&](uint64_t lt) {
                if (lt >= P.n_tiles) W.sn = 0u;
                else W.next(P, r);
            };
            auto enter_pair = [&](uint64_t p, bool fresh) {
                const uint64_t lt = 2 * (p - dec_pair0);
                if (fresh) W.begin(P, lt, r);
                else adv(lt);
                x1 = W.a1; x2 = W.a2; xs = W.sn; sX = W.s; ltX = lt;
                st1(pp.X.a1 + pp.lane_off, W.a1, W.a2);
                adv(lt + 1);
                y1 = W.a1; y2 = W.a2; ys = W.sn; sY = W.s;
                st1(pp.Y.a1 + pp.lane_off, W.a1, W.a2);
                tmem_wait_st();
                if (pp.handoff(wq == 3)) {
                    issue_l1(pp.X, sX);
                    issue_l1(pp.Y, sY);
                    pp.commit();
                }
            };
            load_decision();
            enter_pair(pb, true);
            // 32-bit loop state: pairs left in this group's range and in the current decision
            // bit 31 of in_dec: this pair's X row 0 is the decision's index 0 (y(0) owed)
            constexpr uint32_t kOweY0 = 0x80000000u;
            uint32_t left = (uint32_t)(pe - pb), in_dec = (uint32_t)(dec_pair_end - pb) | (ltX == 0 ? kOweY0 : 0u);
            while (left) {
                pp.template stage_as<0, true>(wq == 0);
                pp.template stage_as<1, true>(wq == 1);
                pp.template stage_as<2, true>(wq == 2);
                // the next pair's rows are walked while the output MMA runs (inside a decision)
                const bool same = (in_dec & ~kOweY0) > 1 && left > 1;  // warp-uniform
                uint32_t n1 = 0, n2 = 0, ns = 0, m1 = 0, m2 = 0, ms = 0;
                int nsX = 0, nsY = 0;
                if (same) {
                    ltX += 2;
                    adv(ltX);
                    n1 = W.a1; n2 = W.a2; ns = W.sn; nsX = W.s;
                    adv(ltX + 1);
                    m1 = W.a1; m2 = W.a2; ms = W.sn; nsY = W.s;
                }
                pp.wait();
                uint32_t ybx, yby;
                tmem_ld1x2(pp.X.d + pp.lane_off, pp.Y.d + pp.lane_off, ybx, yby);
                ybx = pp.add_b4(ybx);
                yby = pp.add_b4(yby);
                if ((in_dec & kOweY0) && r == 0 && P.want_y0) y0s[d] = __uint_as_float(ybx);
                in_dec &= ~kOweY0;
                fold_packed2(P, sX, x1, x2, xs, __uint_as_float(ybx), sY, y1, y2, ys, __uint_as_float(yby), best,
                             best_y, bsn);
                left--;
                in_dec--;
                if (same) {
                    x1 = n1; x2 = n2; xs = ns; sX = nsX;
                    y1 = m1; y2 = m2; ys = ms; sY = nsY;
                    st1(pp.X.a1 + pp.lane_off, x1, x2);
                    st1(pp.Y.a1 + pp.lane_off, y1, y2);
                    tmem_wait_st();
                    if (pp.handoff(wq == 3)) {
                        issue_l1(pp.X, sX);
                        issue_l1(pp.Y, sY);
                        pp.commit();
                    }
                } else if (in_dec == 0) {  // leaving decision d
                    flush();
                    bsn = 1u;
                    if (left) {
                        const uint64_t p = pe - left;  // the next pair, first of decision d + 1
                        d++;
                        load_decision();
                        in_dec = (uint32_t)(dec_pair_end - p);
                        enter_pair(p, true);
                        if (ltX == 0) in_dec |= kOweY0;
                    }
                }
            }
            flush();
        } else {
        Walker W{};
        uint32_t vX[kKMax], vY[kKMax];
        int sX = 0, sY = 0;
        bool okX = false, okY = false, zX = false, zY = false;
        auto take = [&](uint32_t (&v)[kKMax], int& s, bool& ok, bool& z) {
            ok = W.u_end - W.ub > (uint64_t)r;
            z = walker_is_index0(W, r);
#pragma unroll
            for (int j = 0; j < kKMax; j++) v[j] = W.v[j];
            s = W.s;
        };
        auto fold = [&](uint32_t yb, int s, const uint32_t (&v)[kKMax], bool ok, bool z) {
            const float y = __uint_as_float(yb);
            if (ok && z) y0s[d] = y;
            if (ok) fold_tile(P, s, v, y, best, best_y);
        };
        // the pair p's two tiles enter the slots (local tiles of decision d)
        auto enter_pair = [&](uint64_t p, bool fresh) {
            const uint64_t lt = 2 * (p - dec_pair0);
            if (fresh) walker_begin(P, W, lt, r);
            else walker_next(P, W, lt, r);
            take(vX, sX, okX, zX);
            store_a1<0, SPLIT>(pp.X.a1 + pp.lane_off, vX);
            walker_next(P, W, lt + 1, r);
            take(vY, sY, okY, zY);
            store_a1<0, SPLIT>(pp.Y.a1 + pp.lane_off, vY);
            tmem_wait_st();
            if (pp.handoff(pp.me[3])) {
                issue_l1(pp.X, sX);
                issue_l1(pp.Y, sY);
                pp.commit();
            }
        };
        load_decision();
        enter_pair(pb, true);
        for (uint64_t p = pb; p < pe; p++) {
            uint32_t ybx, yby;
            pp.template run_layers<true>(ybx, yby);
            fold(ybx, sX, vX, okX, zX);
            fold(yby, sY, vY, okY, zY);
            if (p + 1 == dec_pair_end) {  // leaving decision d
                flush();
                if (p + 1 < pe) {
                    d++;
                    load_decision();
                    enter_pair(p + 1, true);
                }
            } else if (p + 1 < pe) {
                enter_pair(p + 1, false);
            }
        }
        flush();  // the last decision of the range (a no-op if it was flushed at its end)
        }
    }
    fence_before();
    __syncthreads();
    fence_after();
    if (warp == 0) tmem_dealloc(tbase, 512);
}

// a7 for a batch: one warp per decision, lane j decodes slot j of t*
__global__ void batch_finalize_kernel(const BatchDec* __restrict__ decs, const BatchAcc* __restrict__ acc,
                                      const float* __restrict__ y0s, int32_t n_dec, Result* out) {
    const int d = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int lane = threadIdx.x & 31;
    if (d >= n_dec) return;
    const PlanHdr& h = decs[d].h;
    const unsigned long long key = acc[d].key;
    const int32_t my = (lane < h.k && key) ? decode_slot_ope(h, key & ((1ull << 40) - 1), lane) : 0;
    int32_t ope[kKMax];
#pragma unroll
    for (int j = 0; j < kKMax; j++) ope[j] = __shfl_sync(0xffffffffu, my, j);
    if (lane) return;
    Result R{};
    R.key = key;
    R.y_best = key ? acc[d].y : __int_as_float(0x7fc00000);
    R.y0 = y0s[d];
    R.evaluated = h.n_eval;
    for (int j = 0; j < kKMax; j++) R.end_op[j] = ope[j];
    R.total_ops = key ? (int32_t)(key >> 40) - 1 : 0;
    R.status = key ? 0 : 2;
    out[d] = R;
}

// ---------------------------------------------------------------------------
// standalone predictor: rows from HBM
//   A1 row = [x_hi (D values), x_lo (D values), 1, 1, 0...], x = 256 x_hi + x_lo
//   B1     = [256 W1 | W1 | b1_hi | b1_lo]  (bf16: second set of chunks = lo halves)
// ---------------------------------------------------------------------------
// Fast layer-1 layout for even D (here D = 24): x = 2^S hi + lo with
// lo in [0, 2^S) entered as the exact value 2^S0 + lo built by bit operations
// (fp16: S = 10, 1024 + lo = bits 0x6400 | lo; bf16: S = 7, 128 + lo = bits
// 0x4300 | lo) and hi converted exactly.  B columns: lo -> w, hi -> 2^S w; the
// constant offset 2^S0 sum_j w_j of the lo entries is removed from the bias.
template <int FMT>
struct Split {
    static constexpr int S = FMT == 0 ? 10 : 7;
    static constexpr uint32_t LOMASK2 = FMT == 0 ? 0x03FF03FFu : 0x007F007Fu;
    static constexpr uint32_t MAGIC2 = FMT == 0 ? 0x64006400u : 0x43004300u;
    static constexpr float OFFSET = FMT == 0 ? 1024.0f : 128.0f;
};

template <int FMT>
__device__ void build_b1_predict_fast(const float* __restrict__ w1b1, int D, float scale, uint8_t* s_b1, int nch) {
    const float* b1 = w1b1 + kHidden * D;
    const int K = nch * 16;
    for (int e = threadIdx.x; e < kHidden * K; e += blockDim.x) {
        const int n = e / K, k = e % K;
        uint16_t v0 = 0, v1 = 0;
        if (k < 2 * D) {
            const float w = w1b1[n * D + (k % D)] * scale;
            const float m = k < D ? 1.0f : (float)(1 << Split<FMT>::S);
            uint16_t h, l;
            split16<FMT>(w, h, l);
            if (FMT == 0) {
                v0 = to16<FMT>(w * m);
            } else {
                v0 = to16<FMT>(from16<FMT>(h) * m);
                v1 = to16<FMT>(from16<FMT>(l) * m);
            }
        } else if (k < 2 * D + 2) {
            // bias minus the lo offsets (computed with the weights as the MMA sees them)
            double off = 0.0;
            for (int j = 0; j < D; j++) {
                const float w = w1b1[n * D + j] * scale;
                double wq;
                if (FMT == 0) {
                    wq = (double)from16<FMT>(to16<FMT>(w));
                } else {
                    uint16_t h, l;
                    split16<FMT>(w, h, l);
                    wq = (double)from16<FMT>(h) + (double)from16<FMT>(l);
                }
                off += wq * (double)Split<FMT>::OFFSET;
            }
            const float bb = (float)((double)b1[n] * (double)scale - off);
            uint16_t h, l;
            split16<FMT>(bb, h, l);
            v0 = k == 2 * D ? h : l;
        }
        const int ch = k >> 4, kk = k & 15;
        *reinterpret_cast<uint16_t*>(s_b1 + (size_t)ch * kChunkBytesN32 + b_offset(n, kk)) = v0;
        if (FMT == 1)
            *reinterpret_cast<uint16_t*>(s_b1 + (size_t)(nch + ch) * kChunkBytesN32 + b_offset(n, kk)) = v1;
    }
}

// layer-1 operand row for D = 24 from the 12 packed int16 pairs of a row
template <int FMT>
__device__ __forceinline__ void encode_row24(const uint32_t (&w)[12], uint32_t (&a)[32]) {
#pragma unroll
    for (int i = 0; i < 12; i++) {
        a[i] = (w[i] & Split<FMT>::LOMASK2) | Split<FMT>::MAGIC2;        // lo pair, exact 2^S0 + lo
        const int32_t x0 = (int32_t)(w[i] << 16) >> (16 + Split<FMT>::S);  // sign-extended hi parts
        const int32_t x1 = (int32_t)w[i] >> (16 + Split<FMT>::S);
        a[12 + i] = pack2<FMT>((float)x0, (float)x1);
    }
    a[24] = TcCfg<FMT>::kOne2;
#pragma unroll
    for (int i = 25; i < 32; i++) a[i] = 0;
}

template <int FMT>
__device__ void build_b1_predict(const float* __restrict__ w1b1, int D, float scale, uint8_t* s_b1, int nch) {
    const float* b1 = w1b1 + kHidden * D;
    const int K = nch * 16;
    for (int e = threadIdx.x; e < kHidden * K; e += blockDim.x) {
        const int n = e / K, k = e % K;
        uint16_t v0 = 0, v1 = 0;
        if (k < 2 * D) {
            const float w = w1b1[n * D + (k % D)] * scale;
            const float m = k < D ? 256.0f : 1.0f;
            uint16_t h, l;
            split16<FMT>(w, h, l);
            if (FMT == 0) {
                v0 = to16<FMT>(w * m);
            } else {
                v0 = to16<FMT>(from16<FMT>(h) * m);
                v1 = to16<FMT>(from16<FMT>(l) * m);
            }
        } else if (k < 2 * D + 2) {
            uint16_t h, l;
            split16<FMT>(b1[n] * scale, h, l);
            v0 = k == 2 * D ? h : l;
        }
        const int ch = k >> 4, kk = k & 15;
        *reinterpret_cast<uint16_t*>(s_b1 + (size_t)ch * kChunkBytesN32 + b_offset(n, kk)) = v0;
        if (FMT == 1)
            *reinterpret_cast<uint16_t*>(s_b1 + (size_t)(nch + ch) * kChunkBytesN32 + b_offset(n, kk)) = v1;
    }
}

// Pipelined like the fused kernel: NG groups x 2 tile slots (X, Y).  Per slot
// 64 TMEM columns: D [0,32) and an operand region U [32,64) that holds the
// layer-1 operand (features split 256 hi + lo, 4 K-chunks) and, after the
// layer-1 MMA, the activations A = U[0,16) plus the bias constant chunk
// U[16,24) = (1, 1, 0, ...).  Each slot's 128 feature rows are brought into
// shared memory by a 1-D TMA bulk copy one slot-cycle ahead of use.
template <int FMT, int NG>
__global__ void __launch_bounds__(NG * 128, 1) predict_tc_kernel(const __grid_constant__ TcParams TP,
                                                                 const float* __restrict__ w1b1, int32_t D,
                                                                 const int16_t* __restrict__ x, uint64_t count,
                                                                 float* __restrict__ y) {
    extern __shared__ __align__(1024) uint8_t smem[];
    using C = TcCfg<FMT>;
    const int nch = (2 * D + 2 + 15) / 16;  // layer-1 K chunks (<= 4 for D <= 31)
    const uint32_t row_bytes = (uint32_t)D * 2u;
    const uint32_t stage_bytes = (kTileM * row_bytes + 127u) & ~127u;
    const TcSmem L = tc_smem_layout<FMT>(FMT == 0 ? nch : 2 * nch, kChunkBytesN32, 2 * NG, stage_bytes);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);  // per group: mma X, mma Y
    uint64_t* tbars = reinterpret_cast<uint64_t*>(smem + L.tmem_slot + 16);  // per group: tma X, tma Y
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem + L.tmem_slot);
    const int tid = threadIdx.x;
    const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
    const int g = warp >> 2, wq = warp & 3;
    const uint32_t lane = (uint32_t)(tid & 31);

    {
        const int4* src = reinterpret_cast<const int4*>(TP.blob);
        int4* dst = reinterpret_cast<int4*>(smem);
        for (uint32_t i = tid; i < TP.bytes / 16; i += blockDim.x) dst[i] = src[i];
    }
    const bool fast24 = D == 24;  // magic-number layer-1 layout (encode_row24)
    if (fast24) build_b1_predict_fast<FMT>(w1b1, D, TP.l1_scale, smem + L.b1, nch);
    else build_b1_predict<FMT>(w1b1, D, TP.l1_scale, smem + L.b1, nch);
    if (tid == 0) {
        for (int i = 0; i < 2 * NG; i++) {
            mbar_init(&bars[i], 1);
            mbar_init(&tbars[i], 1);
        }
        mbar_fence_init();
    }
    if (warp == 0) {
        tmem_alloc(tmem_slot, 512);
        tmem_relinquish();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tbase = __shfl_sync(0xffffffffu, *tmem_slot, 0);

    // per group 128 columns: X = D [0,32) U [32,64), Y = D [64,96) U [96,128);
    // U holds the layer-1 operand, then A = U[0,16) and the constant chunk U[16,24)
    const uint32_t col = tbase + (uint32_t)g * 128u;
    const TileIO X{col + 0, col + 32, col + 32}, Y{col + 64, col + 96, col + 96};
    const uint32_t r = (uint32_t)(tid & 127);
    const uint32_t sbase = smem_u32(smem);
    constexpr uint32_t id32 = idesc_f16(FMT, 32);
    TcPipe<FMT> pp;
    pp.init_layout(X, Y, col + 48, col + 112, g, wq, &bars[g], smem_desc(sbase + L.w2), smem_desc(sbase + L.w3),
                   smem_desc(sbase + L.w4));
    pp.set_outbias(TP.b4);
    const uint32_t lane_off = pp.lane_off;
    uint64_t* tbX = &tbars[2 * g];
    uint64_t* tbY = &tbars[2 * g + 1];
    uint32_t tphX = 0, tphY = 0;
    uint8_t* stX = smem + L.stage + (uint32_t)(2 * g) * stage_bytes;
    uint8_t* stY = stX + stage_bytes;
    const uint64_t d1base = smem_desc(sbase + L.b1);
    const bool tma_ok = (row_bytes % 16u) == 0 && (reinterpret_cast<uintptr_t>(x) & 15u) == 0;

    auto issue_l1 = [&](const TileIO& T) {
        for (int cb = 0; cb < nch; cb++)
            mma_ts_elect(T.d, T.a1 + 8 * cb, d1base + (uint64_t)(cb * (kChunkBytesN32 >> 4)), id32,
                         cb > 0 ? 1u : 0u);
        if (FMT == 1)
            for (int cb = 0; cb < nch; cb++)
                mma_ts_elect(T.d, T.a1 + 8 * cb, d1base + (uint64_t)((nch + cb) * (kChunkBytesN32 >> 4)), id32, 1u);
    };
    const uint64_t n_tiles = (count + kTileM - 1) / kTileM;
    // feature rows of tile w: TMA bulk copy into a slot's stage (lane 0 of the issuing warp)
    auto fetch = [&](uint64_t w, uint8_t* st, uint64_t* tb) {
        if (!tma_ok || w >= n_tiles) return;
        if (lane == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of `st`
            const uint64_t row0 = w * kTileM;
            const uint32_t nrows = (uint32_t)min((uint64_t)kTileM, count - row0);
            mbar_arrive_expect_tx(tb, nrows * row_bytes);
            bulk_g2s(st, x + row0 * (uint64_t)D, nrows * row_bytes, tb);
        }
    };
    // layer-1 operand row from the staged features (no tcgen05.st wait)
    auto encode = [&](const TileIO& T, uint64_t w, uint8_t* st, uint64_t* tb, uint32_t& tph) {
        const uint64_t row0 = w * kTileM;
        const uint32_t nrows = (uint32_t)min((uint64_t)kTileM, count - row0);
        const int16_t* rowp;
        if (tma_ok) {
            mbar_wait(tb, tph);
            tph ^= 1u;
            rowp = reinterpret_cast<const int16_t*>(st) + (size_t)min(r, nrows - 1) * D;
        } else {
            rowp = x + (row0 + min(r, nrows - 1)) * (uint64_t)D;
        }
        if (fast24) {
            uint32_t wv[12];
            const uint4* rp = reinterpret_cast<const uint4*>(rowp);
            const bool al = (reinterpret_cast<uintptr_t>(rowp) & 15u) == 0;
#pragma unroll
            for (int q = 0; q < 3; q++) {
                uint4 v4;
                if (al) v4 = rp[q];
                else {
                    const uint32_t* r32 = reinterpret_cast<const uint32_t*>(rowp) + 4 * q;
                    v4 = make_uint4(r32[0], r32[1], r32[2], r32[3]);
                }
                wv[4 * q] = v4.x; wv[4 * q + 1] = v4.y; wv[4 * q + 2] = v4.z; wv[4 * q + 3] = v4.w;
            }
            uint32_t av[32];
            encode_row24<FMT>(wv, av);
#pragma unroll
            for (int cb = 0; cb < 4; cb++) {
                uint32_t a8[8];
#pragma unroll
                for (int i = 0; i < 8; i++) a8[i] = av[8 * cb + i];
                tmem_st8(T.a1 + lane_off + 8 * cb, a8);
            }
            return;
        }
        for (int cb = 0; cb < nch; cb++) {
            uint32_t a[8];
#pragma unroll
            for (int i = 0; i < 8; i++) {
                float v2[2];
#pragma unroll
                for (int h = 0; h < 2; h++) {
                    const int k = cb * 16 + 2 * i + h;
                    float val = 0.0f;
                    if (k < D) val = (float)(rowp[k] >> 8);
                    else if (k < 2 * D) val = (float)(rowp[k - D] & 255);
                    else if (k < 2 * D + 2) val = 1.0f;
                    v2[h] = val;
                }
                a[i] = pack2<FMT>(v2[0], v2[1]);
            }
            tmem_st8(T.a1 + lane_off + 8 * cb, a);
        }
    };
    // tiles w (and w + 1) enter the slots: encode, hand off, issue layer 1, refill the stages
    auto enter = [&](uint64_t w, bool two) {
        encode(X, w, stX, tbX, tphX);
        if (two) encode(Y, w + 1, stY, tbY, tphY);
        tmem_wait_st();
        if (pp.handoff(pp.me[3])) {
            issue_l1(X);
            if (two) issue_l1(Y);
            pp.commit();
            fetch(w + 2, stX, tbX);  // every thread has consumed the stages (hand-off)
            if (two) fetch(w + 3, stY, tbY);
        }
    };
    uint64_t wb, we;
    work_range(n_tiles, (uint64_t)blockIdx.x * NG + g, (uint64_t)gridDim.x * NG, wb, we);
    if (wb < we) {
        if (r == 0) {
            fetch(wb, stX, tbX);
            if (wb + 1 < we) fetch(wb + 1, stY, tbY);
        }
        enter(wb, wb + 1 < we);
        for (uint64_t w = wb; w < we; w += 2) {
            uint32_t yx, yy = 0;
            const bool two = w + 1 < we;
            if (two) pp.template run_layers<true, true>(yx, yy);
            else pp.template run_layers<false, true>(yx, yy);
            const uint64_t row = w * kTileM + r;
            if (row < count) y[row] = __uint_as_float(yx);
            if (two && row + kTileM < count) y[row + kTileM] = __uint_as_float(yy);
            if (w + 2 < we) enter(w + 2, w + 3 < we);
        }
    }
    fence_before();
    __syncthreads();
    fence_after();
    if (warp == 0) tmem_dealloc(tbase, 512);
}

// ---------------------------------------------------------------------------
// predict, fp16, D = 24 (N = 8, K_MAX = 4: the canonical width) -- the
// fused kernel's pipeline (5 groups x 2 lock-step tiles, 96 TMEM columns per
// group) fed from HBM instead of the walker.  A row's 24 features enter the
// layer-1 operand as the exact fp16 values 1024 + v (bit pattern
// 0x6400 | v, valid for 0 <= v < 1024: every Fig.-8 feature of the registry),
// so layer 1 is 2 K chunks (24 features + the (1, 1) bias pair) and the
// operand is exactly the 16-column A region.  Rows with a feature outside
// [0, 1024) are flagged (one OR over the 12 packed words) and recomputed on
// the CUDA cores in fp32 after the tile; their tensor result is discarded.
// The 128 rows (6 KB) of a tile come in by a 1-D TMA bulk copy into one of
// two stages per slot, issued two iterations ahead.
// ---------------------------------------------------------------------------
constexpr int kPred24NG = 5;
constexpr uint32_t kRow24 = 48;
constexpr uint32_t kStage24 = kTileM * kRow24;  // 6 KB

// layer-1 B operand (2 chunks): k < 24: w_nk s1; k = 24, 25: (b1_n s1 - 1024 sum_k w_nk s1) as (hi, lo)
__device__ void build_b1_predict24(const float* __restrict__ w1b1, float scale, uint8_t* s_b1) {
    constexpr int FMT = 0, D = 24;
    const float* b1 = w1b1 + kHidden * D;
    for (int e = threadIdx.x; e < kHidden * 32; e += blockDim.x) {
        const int n = e >> 5, k = e & 31;
        uint16_t v = 0;
        if (k < D) {
            v = to16<FMT>(w1b1[n * D + k] * scale);
        } else if (k < D + 2) {
            double off = 0.0;
            for (int j = 0; j < D; j++) off += (double)from16<FMT>(to16<FMT>(w1b1[n * D + j] * scale)) * 1024.0;
            const float bb = (float)((double)b1[n] * (double)scale - off);
            uint16_t h, l;
            split16<FMT>(bb, h, l);
            v = k == D ? h : l;
        }
        *reinterpret_cast<uint16_t*>(s_b1 + (size_t)(k >> 4) * kChunkBytesN32 + b_offset(n, k & 15)) = v;
    }
}

// fp32 SIMT forward of one row (the rare rows outside the tensor path's range)
__device__ __forceinline__ float predict_row_fp32(const W234& W, const float* __restrict__ w1b1,
                                               const int16_t* __restrict__ row) {
    constexpr int D = 24;
    float h1[kHidden], h2[kHidden];
#pragma unroll 1
    for (int i = 0; i < kHidden; i++) {
        float s = w1b1[kHidden * D + i];
        for (int k = 0; k < D; k++) s = fmaf(w1b1[i * D + k], (float)row[k], s);
        h1[i] = fmaxf(s, 0.0f);
    }
#pragma unroll 1
    for (int i = 0; i < kHidden; i++) {
        float s = W.b2[i];
        for (int j = 0; j < kHidden; j++) s = fmaf(W.W2[i][j], h1[j], s);
        h2[i] = fmaxf(s, 0.0f);
    }
    float acc = W.b4;
#pragma unroll 1
    for (int i = 0; i < kHidden; i++) {
        float s = W.b3[i];
        for (int j = 0; j < kHidden; j++) s = fmaf(W.W3[i][j], h2[j], s);
        acc = fmaf(W.w4[i], fmaxf(s, 0.0f), acc);
    }
    return acc;
}

// FMT 1 (bf16): the same fp16 layer-1 operand and table; layers 2, 3 and the
// output in bf16 (TcPipe<1>), as in the fused bf16 search.
template <int FMT, int NG>
__global__ void __launch_bounds__(NG * 128, 1) predict24_tc_kernel(const __grid_constant__ TcParams TP,
                                                                   const __grid_constant__ W234 W,
                                                                   const float* __restrict__ w1b1,
                                                                   const int16_t* __restrict__ x, uint64_t count,
                                                                   float* __restrict__ y) {
    extern __shared__ __align__(1024) uint8_t smem[];
    // stages: per group X0 X1 Y0 Y1 (4 x 6 KB); TMA mbarriers after the TMEM slot
    const TcSmem L = tc_smem_layout<FMT>(2, kChunkBytesN32, NG, 4 * kStage24);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem + L.tmem_slot);
    uint64_t* tbars = reinterpret_cast<uint64_t*>(smem + L.total);  // per group: X0 X1 Y0 Y1
    const int tid = threadIdx.x;
    const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
    const int g = warp >> 2, wq = warp & 3;
    {
        const int4* src = reinterpret_cast<const int4*>(TP.blob);
        int4* dst = reinterpret_cast<int4*>(smem);
        for (uint32_t i = tid; i < TP.bytes / 16; i += blockDim.x) dst[i] = src[i];
    }
    build_b1_predict24(w1b1, TP.l1_scale, smem + L.b1);
    if (tid == 0)
        for (int i = 0; i < 4 * NG; i++) mbar_init(&tbars[i], 1);
    const uint32_t tbase = fused_prologue_tmem<FMT, NG>(bars, tmem_slot, warp, g, wq);

    const uint32_t r = (uint32_t)(tid & 127);
    const uint32_t sbase = smem_u32(smem);
    TcPipe<FMT> pp;
    pp.init(tbase, g, wq, &bars[g], smem_desc(sbase + L.w2), smem_desc(sbase + L.w3), smem_desc(sbase + L.w4));
    pp.set_outbias(TP.b4);
    const uint64_t d1 = smem_desc(sbase + L.b1);
    uint8_t* stg = smem + L.stage + (uint32_t)g * 4u * kStage24;  // X0 X1 Y0 Y1
    uint64_t* tb = &tbars[4 * g];
    uint32_t tph = 0;  // phase bit per stage (bit i: stage i)
    const uint64_t n_tiles = (count + kTileM - 1) / kTileM;
    uint64_t wb, we;
    work_range(n_tiles, (uint64_t)blockIdx.x * NG + g, (uint64_t)gridDim.x * NG, wb, we);
    // stage index of tile w: slot (w - wb) & 1, buffer ((w - wb) >> 1) & 1
    auto sidx = [&](uint64_t w) -> int { return (int)(((w - wb) & 1u) * 2u + (((w - wb) >> 1) & 1u)); };
    auto fetch = [&](uint64_t w) {  // one thread of the group
        if (w >= we) return;
        const int si = sidx(w);
        const uint64_t row0 = w * kTileM;
        const uint32_t nrows = (uint32_t)min((uint64_t)kTileM, count - row0);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_arrive_expect_tx(&tb[si], nrows * kRow24);
        bulk_g2s(stg + (uint32_t)si * kStage24, x + row0 * 24u, nrows * kRow24, &tb[si]);
    };
    // operand words of this thread's row of tile w (after its stage landed)
    auto load = [&](uint64_t w, uint32_t (&a)[16], uint32_t& bad) {
        const int si = sidx(w);
        mbar_wait(&tb[si], (tph >> si) & 1u);
        tph ^= 1u << si;
        const uint64_t row0 = w * kTileM;
        const uint32_t nrows = (uint32_t)min((uint64_t)kTileM, count - row0);
        const uint4* rp = reinterpret_cast<const uint4*>(stg + (uint32_t)si * kStage24 + min(r, nrows - 1) * kRow24);
        const uint4 q0 = rp[0], q1 = rp[1], q2 = rp[2];
        a[0] = q0.x; a[1] = q0.y; a[2] = q0.z; a[3] = q0.w;
        a[4] = q1.x; a[5] = q1.y; a[6] = q1.z; a[7] = q1.w;
        a[8] = q2.x; a[9] = q2.y; a[10] = q2.z; a[11] = q2.w;
        const uint32_t o = (a[0] | a[1] | a[2] | a[3]) | (a[4] | a[5] | a[6] | a[7]) | (a[8] | a[9] | a[10] | a[11]);
        bad = (o & 0xFC00FC00u) != 0u ? 1u : 0u;  // a feature < 0 or >= 1024: recomputed in fp32
#pragma unroll
        for (int i = 0; i < 12; i++) a[i] |= 0x64006400u;
        a[12] = TcCfg<0>::kOne2;  // fp16 (1, 1): the layer-1 operand is fp16 in both formats
        a[13] = a[14] = a[15] = 0u;
    };
    auto issue_l1 = [&](const TileIO& T) {
        constexpr uint32_t id32 = idesc_f16(0, 32);
        mma_ts_elect(T.d, T.a1, d1, id32, 0u);
        mma_ts_elect(T.d, T.a1 + 8, d1 + (kChunkBytesN32 >> 4), id32, 1u);
    };
    auto put_y = [&](uint64_t w, uint32_t yb, uint32_t bad) {
        const uint64_t row = w * kTileM + r;
        if (row >= count) return;
        float v = __uint_as_float(yb);
        if (bad) v = predict_row_fp32(W, w1b1, x + row * 24u);
        y[row] = v;
    };
    using T1 = std::integral_constant<bool, false>;
    using T2 = std::integral_constant<bool, true>;
    if (wb < we) {
        if (r == 0)
            for (uint64_t w = wb; w < wb + 4; w++) fetch(w);
        uint32_t ax[16], ay[16];
        uint32_t badX = 0, badY = 0;
        const bool yLive = wb + 1 < we;
        load(wb, ax, badX);
        tmem_st16(pp.X.a + pp.lane_off, ax);
        if (yLive) {
            load(wb + 1, ay, badY);
            tmem_st16(pp.Y.a + pp.lane_off, ay);
        }
        tmem_wait_st();
        if (pp.handoff(pp.me[3])) {
            issue_l1(pp.X);
            if (yLive) issue_l1(pp.Y);
            pp.commit();
        }
        uint64_t w = wb;
        auto iteration = [&](auto two_c, auto next_two_c) {
            constexpr bool TWO = decltype(two_c)::value;
            constexpr bool NTWO = decltype(next_two_c)::value;
            pp.template stage<0, TWO>();
            pp.template stage<1, TWO>();
            pp.template stage<2, TWO>();
            // the next tiles' operand rows are read while the output MMA runs
            const bool more = w + 2 < we;
            uint32_t nbx = 0, nby = 0;
            if (more) load(w + 2, ax, nbx);
            pp.wait();
            uint32_t yx, yy = 0;
            if (TWO) tmem_ld1x2(pp.X.d + pp.lane_off, pp.Y.d + pp.lane_off, yx, yy);
            else tmem_ld1(pp.X.d + pp.lane_off, yx);
            yx = pp.add_b4(yx);
            if (TWO) yy = pp.add_b4(yy);
            if (more) {
                tmem_st16(pp.X.a + pp.lane_off, ax);
                if (NTWO) {
                    load(w + 3, ay, nby);
                    tmem_st16(pp.Y.a + pp.lane_off, ay);
                }
                tmem_wait_st();
                if (pp.handoff(pp.me[3])) {
                    issue_l1(pp.X);
                    if (NTWO) issue_l1(pp.Y);
                    pp.commit();
                    if ((tid & 31) == 0) {  // every thread has read these stages (hand-off barrier)
                        fetch(w + 4);
                        if (NTWO) fetch(w + 5);
                    }
                }
            }
            put_y(w, yx, badX);
            if (TWO) put_y(w + 1, yy, badY);
            badX = nbx;
            badY = nby;
            w += 2;
        };
        while (w + 3 < we) iteration(T2{}, T2{});
        if (w + 1 < we) iteration(T2{}, T1{});
        if (w < we) iteration(T1{}, T1{});
    }
    fence_before();
    __syncthreads();
    fence_after();
    if (warp == 0) tmem_dealloc(tbase, 512);
}

// ---------------------------------------------------------------------------
// launchers
// ---------------------------------------------------------------------------
constexpr int kFusedNG = 5;
#ifndef ABACUS_BATCH_NG
#define ABACUS_BATCH_NG 5
#endif
constexpr int kBatchNG = ABACUS_BATCH_NG;  // groups per CTA of the batch search kernel
constexpr int kPredictNG = 4;

template <int FMT, bool SPLIT>
static cudaError_t launch_fused_fmt(const Plan& P, const TcParams& tp, const float* w1b1, Scratch* S, int nsm,
                                    cudaStream_t st, int* grid_out) {
    using C = TcCfg<FMT>;
    const TcSmem L =
        tc_smem_layout<FMT>(P.n_seg, C::kNchL1 * kChunkBytesN32, kFusedNG, w1_stage_bytes(P.D, kFusedNG));
    // spread the tiles over as many SMs as possible (one tile per group first)
    uint64_t g = (P.n_tiles + kFusedNG - 1) / kFusedNG;
    if (g > (uint64_t)nsm) g = (uint64_t)nsm;
    if (g < 1) g = 1;
    *grid_out = (int)g;
    // the shared-memory opt-in is a host API call on the decision path: raise it
    // only when a launch needs more than this device has given the kernel so far
    auto optin = [&](auto kern, int* granted) -> cudaError_t {
        int dev = 0;
        cudaError_t e = cudaGetDevice(&dev);
        if (e != cudaSuccess) return e;
        if (dev < 0 || dev >= 64 || granted[dev] < (int)L.total) {
            e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L.total);
            if (e != cudaSuccess) return e;
            if (dev >= 0 && dev < 64) granted[dev] = (int)L.total;
        }
        return cudaSuccess;
    };
    if (P.n_seg <= 8) {  // decisions: the short parameter block
        static int s_granted8[64] = {};
        auto kern = fused_tc_kernel<FMT, SPLIT, kFusedNG, PlanDecision>;
        const cudaError_t e = optin(kern, s_granted8);
        if (e != cudaSuccess) return e;
        PlanDecision Ps;
        memcpy(&Ps, &P, sizeof(PlanDecision));
        kern<<<(int)g, kFusedNG * 128, L.total, st>>>(Ps, tp, w1b1, S);
        return cudaGetLastError();
    }
    static int s_granted[64] = {};
    auto kern = fused_tc_kernel<FMT, SPLIT, kFusedNG, Plan>;
    const cudaError_t e = optin(kern, s_granted);
    if (e != cudaSuccess) return e;
    kern<<<(int)g, kFusedNG * 128, L.total, st>>>(P, tp, w1b1, S);
    return cudaGetLastError();
}

// digits are < cnt: unsplit when exact as the fp16 1024 + v (v up to 1024); both
// formats enter layer 1 through the same fp16 digit operand
static bool need_split(int, uint32_t maxcnt) { return maxcnt > 1025; }

cudaError_t launch_fused_tc(const Plan& P, const TcWeights& TW, const float* w1b1, Scratch* S, int nsm,
                            cudaStream_t st, int* grid_out) {
    TcParams tp{TW.blob, TW.bytes, TW.l1_scale, TW.b4};
    uint32_t maxcnt = 0;
    for (int s = 0; s < P.n_seg; s++)
        for (int j = 0; j < kKMax; j++) maxcnt = P.seg[s].cnt[j] > maxcnt ? P.seg[s].cnt[j] : maxcnt;
    const bool split = need_split(TW.fmt, maxcnt);
    if (TW.fmt == 0) {
        if (!split) return launch_fused_fmt<0, false>(P, tp, w1b1, S, nsm, st, grid_out);
        return launch_fused_fmt<0, true>(P, tp, w1b1, S, nsm, st, grid_out);
    }
    if (!split) return launch_fused_fmt<1, false>(P, tp, w1b1, S, nsm, st, grid_out);
    return launch_fused_fmt<1, true>(P, tp, w1b1, S, nsm, st, grid_out);
}

template <int FMT, bool SPLIT>
static cudaError_t launch_batch_fmt(const BatchDec* decs, const SegP* segs, int32_t n_dec, const uint64_t* n_pairs,
                                    uint64_t pairs_ub, int32_t D, const TcParams& tp, const float* w1b1,
                                    BatchAcc* acc, float* y0s, int nsm, cudaStream_t st) {
    uint32_t plans_off;
    const TcSmem L = batch_smem_layout<FMT>(D, kBatchNG, &plans_off);
    auto kern = fused_batch_tc_kernel<FMT, SPLIT, kBatchNG>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L.total);
    if (e != cudaSuccess) return e;
    uint64_t g = (pairs_ub + kBatchNG - 1) / kBatchNG;  // the exact count is only known on the device
    if (g > (uint64_t)nsm) g = (uint64_t)nsm;
    if (g < 1) g = 1;
    kern<<<(int)g, kBatchNG * 128, L.total, st>>>(decs, segs, n_dec, n_pairs, D, tp, w1b1, acc, y0s);
    return cudaGetLastError();
}

cudaError_t launch_batch_tc(const BatchDec* d_decs, const SegP* d_segs, int32_t n_dec, const uint64_t* d_n_pairs,
                            uint64_t pairs_ub, uint32_t maxcnt, int32_t D, const TcWeights& TW, const float* w1b1,
                            BatchAcc* acc, float* y0s, Result* out, int nsm, cudaStream_t st) {
    TcParams tp{TW.blob, TW.bytes, TW.l1_scale, TW.b4};
    const bool split = need_split(TW.fmt, maxcnt);
    cudaError_t e;
#define ABACUS_BATCH_ARGS d_decs, d_segs, n_dec, d_n_pairs, pairs_ub, D, tp, w1b1, acc, y0s, nsm, st
    if (TW.fmt == 0)
        e = split ? launch_batch_fmt<0, true>(ABACUS_BATCH_ARGS) : launch_batch_fmt<0, false>(ABACUS_BATCH_ARGS);
    else
        e = split ? launch_batch_fmt<1, true>(ABACUS_BATCH_ARGS) : launch_batch_fmt<1, false>(ABACUS_BATCH_ARGS);
#undef ABACUS_BATCH_ARGS
    if (e != cudaSuccess) return e;
    const int threads = 256;
    const int blocks = (int)(((int64_t)n_dec * 32 + threads - 1) / threads);
    batch_finalize_kernel<<<blocks, threads, 0, st>>>(d_decs, acc, y0s, n_dec, out);
    return cudaGetLastError();
}

template <int FMT>
static cudaError_t launch_predict_fmt(const TcParams& tp, const float* w1b1, int32_t D, const int16_t* x,
                                      uint64_t count, float* y, int nsm, cudaStream_t st) {
    const int nch = (2 * D + 2 + 15) / 16;
    const uint32_t stage_bytes = (uint32_t)(kTileM * D * 2 + 127) & ~127u;
    TcSmem L = tc_smem_layout<FMT>(FMT == 0 ? nch : 2 * nch, kChunkBytesN32, 2 * kPredictNG, stage_bytes);
    const uint32_t total = L.total + 16 + 8 * 2 * kPredictNG;  // + TMA mbarriers after the TMEM slot
    auto kern = predict_tc_kernel<FMT, kPredictNG>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)total);
    if (e != cudaSuccess) return e;
    const uint64_t n_tiles = (count + kTileM - 1) / kTileM;
    uint64_t g = (n_tiles + kPredictNG - 1) / kPredictNG;
    if (g > (uint64_t)nsm) g = (uint64_t)nsm;
    if (g < 1) g = 1;
    kern<<<(int)g, kPredictNG * 128, total, st>>>(tp, w1b1, D, x, count, y);
    return cudaGetLastError();
}

cudaError_t launch_predict_tc(const TcWeights& TW, const W234& W, const float* w1b1, int32_t D, const int16_t* x,
                              uint64_t count, float* y, int nsm, cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    if (D > 31) return cudaErrorInvalidValue;  // layer-1 operand: 4 K-chunks = the 32-column U region
    TcParams tp{TW.blob, TW.bytes, TW.l1_scale, TW.b4};
    if (D == 24 && (reinterpret_cast<uintptr_t>(x) & 15u) == 0) {
        constexpr int NG = kPred24NG;
        const TcSmem L = TW.fmt == 0 ? tc_smem_layout<0>(2, kChunkBytesN32, NG, 4 * kStage24)
                                     : tc_smem_layout<1>(2, kChunkBytesN32, NG, 4 * kStage24);
        const uint32_t total = L.total + 8u * 4u * NG;  // + TMA mbarriers
        auto kern = TW.fmt == 0 ? predict24_tc_kernel<0, NG> : predict24_tc_kernel<1, NG>;
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)total);
        if (e != cudaSuccess) return e;
        const uint64_t n_tiles = (count + kTileM - 1) / kTileM;
        uint64_t g = (n_tiles + NG - 1) / NG;
        if (g > (uint64_t)nsm) g = (uint64_t)nsm;
        if (g < 1) g = 1;
        kern<<<(int)g, NG * 128, total, st>>>(tp, W, w1b1, x, count, y);
        return cudaGetLastError();
    }
    if (TW.fmt == 0) return launch_predict_fmt<0>(tp, w1b1, D, x, count, y, nsm, st);
    return launch_predict_fmt<1>(tp, w1b1, D, x, count, y, nsm, st);
}

}  // namespace abacus
