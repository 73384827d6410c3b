// device_common.cuh -- device helpers shared by the SIMT and tensor-core
// kernels (header-only: the library is built without relocatable device code).
#pragma once
#include <cuda_runtime.h>

#include "common.cuh"

namespace abacus {

// grid digit -> ope (0 = absent); SlotP carries the ABI digit definition
__host__ __device__ __forceinline__ int32_t digit_to_ope(const SlotP& s, uint32_t d) {
    if (s.absent) return d == 0 ? 0 : s.end_lo + (int32_t)d - 1;
    return s.end_lo + (int32_t)d;
}

__device__ __forceinline__ int find_segment(const Plan& P, uint64_t w) {
    int s = 0;
    for (int i = 1; i < P.n_seg; i++)
        if (w >= P.seg[i].tile0) s = i;
    return s;
}

// ---------------------------------------------------------------------------
// Tile walker: a worker (thread row r of a persistent group) walks a
// contiguous range of tiles [wb, we) of the plan.  The segment state lives in
// registers and the box digits v[] of its candidate advance by kTileM per tile
// with a carry chain, so the per-tile enumeration cost is a few integer ops;
// the slow decode (fp64 split of the tile base) runs only on entry and at
// segment boundaries.
// ---------------------------------------------------------------------------
struct Walker {
    uint32_t fast;        // segment's fast_carry flag
    uint64_t ub;          // box ordinal of the tile's row 0
    uint64_t u_end;       // segment end (box ordinal)
    uint64_t next_tile0;  // first work item of the next segment
    uint64_t t_base;
    uint64_t istride[kKMax];
    uint32_t cnt[kKMax];
    FastDiv fd[kKMax];
    int32_t n_base;
    int32_t s;            // segment index
    uint32_t v[kKMax];    // digits of this row's candidate
};

__device__ __forceinline__ void walker_enter(const Plan& P, Walker& W, int s, uint64_t w, uint32_t r) {
    const SegP& g = P.seg[s];
    W.s = s;
    W.u_end = g.u_end;
    W.next_tile0 = s + 1 < P.n_seg ? P.seg[s + 1].tile0 : ~0ull;
    W.t_base = g.t_base;
    W.n_base = g.n_base;
    W.fast = g.fast_carry;
#pragma unroll
    for (int j = 0; j < kKMax; j++) {
        W.istride[j] = g.istride[j];
        W.cnt[j] = g.cnt[j];
        W.fd[j] = g.fd[j];
    }
    W.ub = g.u_begin + (w - g.tile0) * kTileM;
    decode_box<kKMax>(g, W.ub, r, W.v);
}

__device__ __forceinline__ void walker_begin(const Plan& P, Walker& W, uint64_t w, uint32_t r) {
    walker_enter(P, W, find_segment(P, w), w, r);
}

// move to work item w + 1
__device__ __forceinline__ void walker_next(const Plan& P, Walker& W, uint64_t w_next, uint32_t r) {
    if (w_next == W.next_tile0) {
        walker_enter(P, W, W.s + 1, w_next, r);
        return;
    }
    W.ub += kTileM;
    if (W.fast) {
        // the fastest digit has cnt >= kTileM: every carry is 0 or 1
        uint32_t x = W.v[kKMax - 1] + kTileM;
        uint32_t c = x >= W.cnt[kKMax - 1] ? 1u : 0u;
        W.v[kKMax - 1] = c ? x - W.cnt[kKMax - 1] : x;
#pragma unroll
        for (int j = kKMax - 2; j >= 0; j--) {  // x <= cnt: a carry leaves exactly 0
            x = W.v[j] + c;
            c = x >= W.cnt[j] ? 1u : 0u;
            W.v[j] = c ? 0u : x;
        }
        return;
    }
    uint32_t carry = kTileM;
#pragma unroll
    for (int j = kKMax - 1; j >= 0; j--) {
        const uint32_t x = W.v[j] + carry;
        const uint32_t q = fastdiv(x, W.fd[j]);
        W.v[j] = x - q * W.cnt[j];
        carry = q;
    }
}

// contiguous work range of worker group `gid` out of `ngroups`
__device__ __forceinline__ void work_range(uint64_t n_tiles, uint64_t gid, uint64_t ngroups, uint64_t& wb,
                                           uint64_t& we) {
    const uint64_t per = n_tiles / ngroups, extra = n_tiles % ngroups;
    wb = gid * per + (gid < extra ? gid : extra);
    we = wb + per + (gid < extra ? 1 : 0);
}

// fold one evaluated candidate into the running best (key built lazily)
__device__ __forceinline__ void fold_candidate(const Walker& W, bool valid, float y, float H,
                                               unsigned long long& best, float& best_y) {
    if (valid && y <= H) {
        const uint32_t hi = (uint32_t)(W.n_base + (int32_t)(W.v[0] + W.v[1] + W.v[2] + W.v[3]) + 1);
        if (hi >= (uint32_t)(best >> 40)) {
            uint64_t idx = W.t_base;
#pragma unroll
            for (int j = 0; j < kKMax; j++) idx += (uint64_t)W.v[j] * W.istride[j];
            const unsigned long long key = ((unsigned long long)hi << 40) | idx;
            if (key > best) {
                best = key;
                best_y = y;
            }
        }
    }
}

// fold a finished candidate given its segment and digits (valid, y known)
__device__ __forceinline__ void fold_tile(const Plan& P, int s, const uint32_t (&v)[kKMax], float y,
                                          unsigned long long& best, float& best_y) {
    if (!(y <= P.H)) return;
    const SegP& g = P.seg[s];
    const uint32_t hi = (uint32_t)(g.n_base + (int32_t)(v[0] + v[1] + v[2] + v[3]) + 1);
    if (hi < (uint32_t)(best >> 40)) return;
    uint64_t idx = g.t_base;
#pragma unroll
    for (int j = 0; j < kKMax; j++) idx += (uint64_t)v[j] * g.istride[j];
    const unsigned long long key = ((unsigned long long)hi << 40) | idx;
    if (key > best) {
        best = key;
        best_y = y;
    }
}

__device__ __forceinline__ bool walker_is_index0(const Walker& W, uint32_t r) {
    return W.t_base == 0 && W.ub == 0 && r == 0;
}

// ---------------------------------------------------------------------------
// Packed tile walker (fp16 with unsplit digits, i.e. every box digit < 1024:
// the headline path).  A row keeps its layer-1 operand words directly,
//     a1 = (0x6400 + v0) | (0x6400 + v1) << 16,  a2 = (0x6400 + v2) | (0x6400 + v3) << 16
// (the exact fp16 values 1024 + v_j, store_a1's layout), and sn = sum_n + 1
// (reading c12, the key's high part).  A tile advance adds 128 to v3 and
// carries on the packed words with predicated adds; sn follows the carries.
// Segment changes are a uniform countdown of the segment's tiles, and the
// rows past the end of a segment's last tile get sn = 0, which no fold
// accepts (every candidate has sn >= 1).  The digits themselves are unpacked
// only when a fold has to build a key.
// ---------------------------------------------------------------------------
// GEN (the batch kernel): one add / compare / subtract chain for every
// segment (the tile advance as mixed-radix digits D_j < cnt_j, at most one
// carry per digit).  !GEN (the single search kernel, at its 96-register cap,
// where the three extra increment words spill): the chain for segments whose
// fastest digit has >= 128 options (D = (128, 0, 0, 0)), a radix division per
// digit otherwise.
template <bool GEN>
struct PackedWalkerT {
    uint32_t a1, a2, sn;  // per row: the most recently taken tile
    int32_t s;            // segment (uniform)
    uint32_t tl;          // tiles of the segment left, the current one included (uniform)
    uint32_t last_rows;   // valid rows of the segment's last tile (uniform)
    uint32_t fast;        // !GEN: cnt3 >= 128 (one carry at most per tile advance)
    uint32_t inc2, inc1, incsn;  // GEN: +128 rows as box digits, packed (v3, v2), (v1, v0) words and their sum
    uint32_t lim3, dec3, dsn3, lim2, cnt2, dsn2, lim1, dec1, dsn1;  // carry constants (uniform)
    uint64_t ub;          // box ordinal of the current tile's row 0 (general advance only)

    __device__ __forceinline__ void pack(const SegP& g, const uint32_t (&v)[kKMax], uint32_t r) {
        a1 = 0x64006400u + v[0] + (v[1] << 16);
        a2 = 0x64006400u + v[2] + (v[3] << 16);
        sn = (uint32_t)(g.n_base + 1) + v[0] + v[1] + v[2] + v[3];
        if (tl == 1 && r >= last_rows) sn = 0u;
    }
    __device__ __forceinline__ void enter(const Plan& P, int seg, uint64_t w, uint32_t r) {
        const SegP& g = P.seg[seg];
        s = seg;
        const uint64_t o = w - g.tile0;
        const uint64_t n = g.u_end - g.u_begin;
        const uint64_t nt = (n + kTileM - 1) / kTileM;
        tl = (uint32_t)(nt - o);
        last_rows = (uint32_t)(n - (nt - 1) * kTileM);
        ub = g.u_begin + o * kTileM;
        fast = g.fast_carry;
        // GEN: the tile advance (+128 box ordinals) as mixed-radix digits D_j <
        // cnt_j: adding them digit by digit needs at most one carry per digit
        // (v_j + D_j + 1 < 2 cnt_j), so every segment takes the same add /
        // compare / subtract chain
        if (GEN) {
            uint32_t rem = (uint32_t)kTileM, d[kKMax];
#pragma unroll
            for (int j = kKMax - 1; j >= 0; j--) {
                d[j] = j > 0 ? rem % g.cnt[j] : rem;
                rem = j > 0 ? rem / g.cnt[j] : 0u;
            }
            inc2 = (d[3] << 16) + d[2];
            inc1 = (d[1] << 16) + d[0];
            incsn = d[0] + d[1] + d[2] + d[3];
        }
        lim3 = (0x6400u + g.cnt[3]) << 16;
        dec3 = (g.cnt[3] << 16) - 1u;
        dsn3 = g.cnt[3] - 1u;
        lim2 = 0x6400u + g.cnt[2];
        cnt2 = g.cnt[2];
        dsn2 = g.cnt[2] - 1u;
        lim1 = (0x6400u + g.cnt[1]) << 16;
        dec1 = (g.cnt[1] << 16) - 1u;
        dsn1 = g.cnt[1] - 1u;
        uint32_t v[kKMax];
        decode_box<kKMax>(g, ub, r, v);
        pack(g, v, r);
    }
    __device__ __forceinline__ void begin(const Plan& P, uint64_t w, uint32_t r) { enter(P, find_segment(P, w), w, r); }
    // move to the next tile (w + 1 of the plan)
    __device__ __forceinline__ void next(const Plan& P, uint32_t r) {
        if (tl == 1) {
            const int ns = s + 1;
            enter(P, ns, P.seg[ns].tile0, r);
            return;
        }
        tl--;
        ub += kTileM;
        if (GEN || fast) {
            if (GEN) {
                a2 += inc2;  // v3 += D3, v2 += D2 (low half stays below bit 16: v2 + D2 + 1 < 2 cnt2 <= 2050)
                a1 += inc1;  // v1 += D1, v0 += D0
                sn += incsn;
            } else {
                a2 += (uint32_t)kTileM << 16;
                sn += kTileM;
            }
            if (!GEN) {
                // a carry out of v3 touches only some tiles of a warp's 32 consecutive
                // rows (cnt3 >= 128: a fraction (159 / cnt3) of them, 34 % on config 4);
                // the rest skip the carry chain with one vote (+1.6 % on config 4)
                const bool c3 = a2 >= lim3;
                if (__any_sync(0xffffffffu, c3)) {
                    if (c3) { a2 -= dec3; sn -= dsn3; }
                    const bool c2 = (a2 & 0xFFFFu) >= lim2;
                    if (c2) { a2 -= cnt2; a1 += 0x10000u; sn -= dsn2; }
                    const bool c1 = a1 >= lim1;
                    if (c1) { a1 -= dec1; sn -= dsn1; }
                }
                // the segment's last tile (uniform, rare): rows past its end never fold
                if (tl == 1 && last_rows < (uint32_t)kTileM) {
                    if (r >= last_rows) sn = 0u;
                }
                return;
            }
            const bool c3 = a2 >= lim3;  // v3 >= cnt3 (the low half never reaches bit 16)
            if (c3) { a2 -= dec3; sn -= dsn3; }  // v3 -= cnt3, v2 += 1
            const bool c2 = (a2 & 0xFFFFu) >= lim2;
            if (c2) { a2 -= cnt2; a1 += 0x10000u; sn -= dsn2; }  // v2 -= cnt2, v1 += 1
            const bool c1 = a1 >= lim1;
            if (c1) { a1 -= dec1; sn -= dsn1; }  // v1 -= cnt1, v0 += 1 (v0 stays in the box)
        } else {
            const SegP& g = P.seg[s];
            uint32_t v[kKMax] = {(a1 & 0xFFFFu) - 0x6400u, (a1 >> 16) - 0x6400u, (a2 & 0xFFFFu) - 0x6400u,
                                 (a2 >> 16) - 0x6400u};
            uint32_t carry = kTileM;
#pragma unroll
            for (int j = kKMax - 1; j >= 0; j--) {
                const uint32_t x = v[j] + carry;
                const uint32_t q = fastdiv(x, g.fd[j]);
                v[j] = x - q * g.cnt[j];
                carry = q;
            }
            a1 = 0x64006400u + v[0] + (v[1] << 16);
            a2 = 0x64006400u + v[2] + (v[3] << 16);
            sn = (uint32_t)(g.n_base + 1) + v[0] + v[1] + v[2] + v[3];
        }
        if (tl == 1 && last_rows < (uint32_t)kTileM && r >= last_rows) sn = 0u;
    }
};

using PackedWalker = PackedWalkerT<false>;

// fold one row of a packed tile: the key is built only when the row fits the
// headroom and its sum_n can reach the running best
__device__ __forceinline__ void fold_packed(const Plan& P, int s, uint32_t a1, uint32_t a2, uint32_t sn, float y,
                                            unsigned long long& best, float& best_y, uint32_t& bsn) {
    if (y <= P.H && sn >= bsn) {
        const SegP& g = P.seg[s];
        const uint64_t idx = g.t_base + (uint64_t)((a1 & 0xFFFFu) - 0x6400u) * g.istride[0] +
                             (uint64_t)((a1 >> 16) - 0x6400u) * g.istride[1] +
                             (uint64_t)((a2 & 0xFFFFu) - 0x6400u) * g.istride[2] +
                             (uint64_t)((a2 >> 16) - 0x6400u) * g.istride[3];
        const unsigned long long key = ((unsigned long long)sn << 40) | idx;
        if (key > best) {
            best = key;
            best_y = y;
            bsn = sn;
        }
    }
}

// The headroom test on the output accumulator before its fp32 bias: with
// y = fl(y_raw + b4) monotone in y_raw, {y_raw : fl(y_raw + b4) <= H} is
// {y_raw <= T} for T = the largest float with fl(T + b4) <= H, so testing
// y_raw <= T decides exactly what y <= H decides (and b4 is added only when a
// row folds).  H = NaN keeps NaN (no row fits), H = +inf gives +inf.
__host__ __device__ __forceinline__ float add_rn(float a, float b) {
#ifdef __CUDA_ARCH__
    return __fadd_rn(a, b);
#else
    volatile float r = a + b;  // one IEEE single rounding (no contraction)
    return r;
#endif
}
__host__ __device__ inline float raw_threshold(float H, float b4) {
    if (!(H == H) || isinf(H)) return H;
    float t = add_rn(H, -b4);
    while (add_rn(t, b4) > H) t = nextafterf(t, -INFINITY);
    for (;;) {
        const float u = nextafterf(t, INFINITY);
        if (isinf(u) || add_rn(u, b4) > H) break;
        t = u;
    }
    return t;
}

// fold_packed2 on raw outputs (yr = y - b4 before rounding; Tr = raw_threshold)
__device__ __forceinline__ void fold_packed2_raw(const Plan& P, float Tr, float b4, int sx, uint32_t x1, uint32_t x2,
                                                 uint32_t xs, float yrx, int sy, uint32_t y1, uint32_t y2,
                                                 uint32_t ys, float yry, unsigned long long& best, float& best_y,
                                                 uint32_t& bsn) {
    const bool cx = yrx <= Tr && xs >= bsn;
    const bool cy = yry <= Tr && ys >= bsn;
    if (cx || cy) {
        if (cx) fold_packed(P, sx, x1, x2, xs, __fadd_rn(yrx, b4), best, best_y, bsn);
        if (cy) fold_packed(P, sy, y1, y2, ys, __fadd_rn(yry, b4), best, best_y, bsn);
    }
}
__device__ __forceinline__ void fold_packed_raw(const Plan& P, float Tr, float b4, int s, uint32_t a1, uint32_t a2,
                                                uint32_t sn, float yr, unsigned long long& best, float& best_y,
                                                uint32_t& bsn) {
    if (yr <= Tr && sn >= bsn) fold_packed(P, s, a1, a2, sn, __fadd_rn(yr, b4), best, best_y, bsn);
}

// fold the two lock-step rows of a thread with one divergent branch: the cheap
// tests of both rows first, the key construction only for a row that passes
// (the key comparison inside is authoritative, so testing Y against the bsn
// from before X's fold is safe)
__device__ __forceinline__ void fold_packed2(const Plan& P, int sx, uint32_t x1, uint32_t x2, uint32_t xs, float yx,
                                             int sy, uint32_t y1, uint32_t y2, uint32_t ys, float yy,
                                             unsigned long long& best, float& best_y, uint32_t& bsn) {
    const bool cx = yx <= P.H && xs >= bsn;
    const bool cy = yy <= P.H && ys >= bsn;
    if (cx || cy) {
        if (cx) fold_packed(P, sx, x1, x2, xs, yx, best, best_y, bsn);
        if (cy) fold_packed(P, sy, y1, y2, ys, yy, best, best_y, bsn);
    }
}

// ---------------------------------------------------------------------------
// Last-CTA epilogue shared by the fused kernels (a5 cross-CTA + a7 decode).
// Each CTA publishes its best (key, y); the last CTA to arrive reduces them,
// decodes the winning index into end ops per slot and resets the ticket.
// ---------------------------------------------------------------------------
// q = floor(a / b) for a < 2^40 via an fp64 reciprocal (exact after one correction)
__host__ __device__ __forceinline__ unsigned long long div_rcp(unsigned long long a, unsigned long long b, double rb) {
    unsigned long long q = (unsigned long long)((double)a * rb);
    const long long rem = (long long)(a - q * b);
    if (rem < 0) q--;
    else if (rem >= (long long)b) q++;
    return q;
}

// End op of slot `j` of the candidate with index idx (GRID: digit j of the
// mixed-radix index, computed directly so lanes can decode slots in parallel;
// CHAIN: block structure).  0 = absent.  Also run by the host for searches
// whose record goes to host-mapped memory (the kernel then skips the decode).
__host__ __device__ __forceinline__ int32_t decode_slot_ope(const PlanHdr& P, unsigned long long idx, int j) {
    if (P.mode == kModeGrid) {
        const SlotP& s = P.slot[j];
        const unsigned long long q = div_rcp(idx, s.tstride, s.rtstride);
        const unsigned long long q2 = div_rcp(q, (unsigned long long)s.radix, s.rradix);
        return digit_to_ope(s, (uint32_t)(q - q2 * (unsigned long long)s.radix));
    }
    int blk = 0;
    for (int i = 1; i < P.k; i++)
        if (idx >= P.chain_cum[i]) blk = i;
    if (j < blk) return P.slot[j].end_hi;
    if (j == blk) return blk == 0 ? P.slot[0].end_hi : P.slot[j].ops + (int32_t)(idx - P.chain_cum[j]);
    return 0;
}

// optional timeline stamps (CTA 0, thread 0): tools/kernel_trace.py
__device__ __forceinline__ void trace_stamp(const PlanHdr& P, int slot) {
    if (P.trace && blockIdx.x == 0 && threadIdx.x == 0) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        P.trace[slot] = t;
    }
}

// copy a result record to host-mapped pinned memory as four tagged 16-byte
// chunks (MappedRec, common.cuh): no fence, the host validates the tags
__device__ __forceinline__ void publish_mapped(const Result& R, MappedRec* M, uint32_t seq) {
    uint32_t p[12];
    rec_payload(R, p);
#pragma unroll
    for (int i = 0; i < 4; i++)
        asm volatile("st.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(&M->w[4 * i]), "r"(p[3 * i]), "r"(p[3 * i + 1]),
                     "r"(p[3 * i + 2]), "r"(rec_tag(seq, p[3 * i], p[3 * i + 1], p[3 * i + 2], (uint32_t)i))
                     : "memory");
}

// device-side reader of a tagged record (the host's rec_read): volatile 16-byte
// loads, true once all four chunks carry the tag of `seq`
__device__ __forceinline__ bool rec_read_dev(const MappedRec* M, uint32_t seq, uint32_t (&p)[12]) {
    bool ok = true;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        uint32_t a, b, c, t;
        asm volatile("ld.volatile.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(a), "=r"(b), "=r"(c), "=r"(t)
                     : "l"(&M->w[4 * i])
                     : "memory");
        ok = ok && t == rec_tag(seq, a, b, c, (uint32_t)i);
        p[3 * i] = a;
        p[3 * i + 1] = b;
        p[3 * i + 2] = c;
    }
    return ok;
}

// a6 over peer memory, run by warp 0 of the last CTA with this rank's record R
// (every lane holds it): lane l sends R to rank l's mailbox, then waits for
// rank l's record in the local mailbox; the warp combines the nranks records
// exactly as combine_results does (max key with its y / end ops, evaluated
// summed, y(0) from the lowest rank that holds index 0).  A rank missing after
// the timeout makes the result status 3.
static __device__ __noinline__ Result peer_combine(const PeerComb& C, const Result& R, uint32_t seq) {
    const uint32_t lane = threadIdx.x & 31;
    const bool act = lane < (uint32_t)C.nranks;
    // two banks by launch parity: a rank that finished launch k and started k + 1
    // writes the other bank, so it never overwrites a launch-k record a slower
    // rank has not read yet (it cannot get two launches ahead: launch k + 1
    // needs every rank's k + 1 record)
    const uint32_t bank = (seq & 1u) * (uint32_t)kPeerMax;
    if (act) {
        publish_mapped(R, C.dst[lane] + bank + C.rank, seq);
        asm volatile("fence.acq_rel.sys;" ::: "memory");
    }
    Result mine{};
    mine.y0 = __int_as_float(0x7fc00000);
    bool timed_out = false;
    if (act) {
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        const unsigned long long limit = (unsigned long long)C.timeout_ms * 1000000ull;
        uint32_t p[12];
        for (;;) {
            if (rec_read_dev(C.local + bank + lane, seq, p)) break;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > limit) {
                timed_out = true;
                break;
            }
            __nanosleep(64);
        }
        if (!timed_out) rec_unpayload(p, mine);
    }
    // combine across the lanes (rank order = lane order)
    unsigned long long bk = mine.key;
    uint32_t win = lane;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long k2 = __shfl_xor_sync(0xffffffffu, bk, o);
        const uint32_t w2 = __shfl_xor_sync(0xffffffffu, win, o);
        if (k2 > bk || (k2 == bk && w2 < win)) { bk = k2; win = w2; }
    }
    unsigned long long ev = mine.evaluated;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ev += __shfl_xor_sync(0xffffffffu, ev, o);
    const uint32_t has_y0 = __ballot_sync(0xffffffffu, act && mine.y0 == mine.y0);
    const float y0 = __shfl_sync(0xffffffffu, mine.y0, has_y0 ? __ffs(has_y0) - 1 : 0);
    const uint32_t bad = __ballot_sync(0xffffffffu, timed_out);
    Result out;
    out.key = bk;
    out.y_best = __shfl_sync(0xffffffffu, mine.y_best, win);
    out.y0 = has_y0 ? y0 : __int_as_float(0x7fc00000);
    out.evaluated = ev;
#pragma unroll
    for (int j = 0; j < kKMax; j++) out.end_op[j] = __shfl_sync(0xffffffffu, mine.end_op[j], win);
    out.total_ops = __shfl_sync(0xffffffffu, mine.total_ops, win);
    out.status = bad ? 3 : (bk ? 0 : 2);
    out.seq = 0;
    out.pad = 0;
    return out;
}

static __device__ __noinline__ void cta_publish_and_finish(const Plan& P, Scratch* S, unsigned long long key, float y) {
    __shared__ unsigned long long s_key[32];
    __shared__ float s_y[32];
    __shared__ bool s_last;
    // warp (key, y) max: y follows its key
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long k2 = __shfl_xor_sync(0xffffffffu, key, o);
        const float y2 = __shfl_xor_sync(0xffffffffu, y, o);
        if (k2 > key) { key = k2; y = y2; }
    }
    const int warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    if ((threadIdx.x & 31) == 0) { s_key[warp] = key; s_y[warp] = y; }
    __syncthreads();
    if (threadIdx.x < 32) {
        unsigned long long bk = threadIdx.x < (unsigned)nwarps ? s_key[threadIdx.x] : 0ull;
        float by = threadIdx.x < (unsigned)nwarps ? s_y[threadIdx.x] : __int_as_float(0x7fc00000);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long k2 = __shfl_xor_sync(0xffffffffu, bk, o);
            const float y2 = __shfl_xor_sync(0xffffffffu, by, o);
            if (k2 > bk) { bk = k2; by = y2; }
        }
    if (threadIdx.x == 0) {
        S->cta_key[blockIdx.x] = bk;
        S->cta_y[blockIdx.x] = by;
        // one acquire-release ticket instead of fence + atomic (+ a fence in the
        // last CTA): the release publishes this CTA's record (and, through the
        // CTA barrier above, y(0) stored by another thread); the last CTA's
        // acquire, followed by the barrier below, orders its loads of every record
        unsigned int ticket;
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(ticket) : "l"(&S->counter) : "memory");
        s_last = ticket == gridDim.x - 1;
    }
    }
    __syncthreads();
    trace_stamp(P, 5);
    if (!s_last) return;
    trace_stamp(P, 8);
    if (threadIdx.x < 32) {
        // warp 0 reduces the per-CTA records (independent loads, then shuffles)
        unsigned long long bk = 0;
        float by = __int_as_float(0x7fc00000);
        const float y0 = __ldcg(&S->y0);
        constexpr int kPer = 16;  // grid <= 512 CTAs: all loads in flight at once
        unsigned long long kk[kPer];
        float yy[kPer];
#pragma unroll
        for (int i = 0; i < kPer; i++) {
            const unsigned int b = threadIdx.x + 32u * i;
            kk[i] = b < gridDim.x ? __ldcg(&S->cta_key[b]) : 0ull;
            yy[i] = b < gridDim.x ? __ldcg(&S->cta_y[b]) : 0.0f;
        }
#pragma unroll
        for (int i = 0; i < kPer; i++)
            if (kk[i] > bk) { bk = kk[i]; by = yy[i]; }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const unsigned long long k2 = __shfl_xor_sync(0xffffffffu, bk, o);
            const float y2 = __shfl_xor_sync(0xffffffffu, by, o);
            if (k2 > bk) { bk = k2; by = y2; }
        }
        trace_stamp(P, 9);
        // a7: lane j decodes slot j's end op of t*; a record that goes to host-mapped
        // memory is decoded by the host instead (off the kernel's critical path)
        const int32_t my_ope = ((!P.mapped || P.peer) && threadIdx.x < (unsigned)P.k && bk)
                                   ? decode_slot_ope(P, bk & ((1ull << 40) - 1), (int)threadIdx.x)
                                   : 0;
        int32_t ope[kKMax];
#pragma unroll
        for (int j = 0; j < kKMax; j++) ope[j] = __shfl_sync(0xffffffffu, my_ope, j);
        if (P.peer) {
            // this rank's record, then the in-kernel combine over the peers' mailboxes
            Result R{};
            R.key = bk;
            R.y_best = by;
            R.y0 = y0;
            R.evaluated = P.n_eval;
            for (int j = 0; j < kKMax; j++) R.end_op[j] = ope[j];
            R.total_ops = bk ? (int32_t)(bk >> 40) - 1 : 0;
            R.status = bk ? 0 : 2;
            const Result G = peer_combine(*P.peer, R, P.peer_seq);
            if (threadIdx.x != 0) return;
            S->result = G;
            S->y0 = __int_as_float(0x7fc00000);
            S->counter = 0;
            if (P.mapped) publish_mapped(G, P.mapped, P.seq);
            return;
        }
        if (threadIdx.x != 0) return;
        trace_stamp(P, 10);
        Result& R = S->result;
        R.key = bk;
        R.y_best = by;
        R.y0 = y0;
        R.evaluated = P.n_eval;
        for (int j = 0; j < kKMax; j++) R.end_op[j] = ope[j];
        R.total_ops = bk ? (int32_t)(bk >> 40) - 1 : 0;
        R.status = bk ? 0 : 2;
        S->y0 = __int_as_float(0x7fc00000);
        S->counter = 0;  // visible to the next launch (kernel boundary)
        trace_stamp(P, 6);
        if (P.mapped) publish_mapped(R, P.mapped, P.seq);
        trace_stamp(P, 7);
    }
}

}  // namespace abacus
