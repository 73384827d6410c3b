// common.cuh -- shared device/host definitions of the CUDA path (sm_100a).
//
// The "plan" describes a candidate space as a list of SEGMENTS.  A segment is
// one presence pattern P of the slots (which services are in the group) and
// the box of end-op digits of its present slots:
//     ope_j = ope0_j + v_j,  v_j in [0, cnt_j)          (present slots)
//     index = t_base + sum_j v_j * istride_j             (t for GRID, u for CHAIN)
//     sum_n = n_base + sum_j v_j                          (reading c12)
// Box-local ordinal u in [u_begin, u_end) enumerates the digits in mixed radix.
// The box digit order is: slots with cnt == 1 first, then the varying slots in
// slot order (dpos[j] = digit of slot j), so index(u) is increasing in u and
// digit kKMax-1 is always the fastest varying one.  Every candidate of the
// grid (ABI abacus_grid_t) lies in exactly one
// segment, and within a segment the Fig.-8 slot positions are
// uniform: this is what lets a 128-row tile share one layer-1 operand.
#pragma once
#include <cstdint>
#include <cstring>

namespace abacus {

constexpr int kHidden = 32;
constexpr int kKMax = 4;
constexpr int kMaxSeg = 16;
constexpr int kTileM = 128;  // candidates per tile = TMEM lanes = tcgen05 M

// floor(x / d) for x < 2^31 via multiply-high (Granlund-Montgomery round-up).
struct FastDiv {
    uint32_t mul, shift, d;
};

struct SegP {
    uint64_t u_begin, u_end;  // box-local ordinal range of this shard
    uint64_t tile0;           // first work item (tile) of the segment
    uint64_t t_base;          // index of the v = 0 element
    // per box DIGIT:
    uint64_t istride[kKMax];  // index stride (0 if absent)
    uint64_t bstride[kKMax];  // box stride (product of later cnt)
    double rbstride[kKMax];   // 1.0 / bstride (uniform fp64 split of the tile base)
    FastDiv fd[kKMax];        // divide by cnt
    uint32_t cnt[kKMax];      // box radix (1 if absent / fixed)
    int32_t ope0[kKMax];      // per SLOT: ope at v = 0, 0 if absent
    int32_t pos[kKMax];       // per SLOT: Fig.-8 position (rank by model id among present), -1 absent
    int32_t dpos[kKMax];      // per SLOT: its box digit
    int32_t n_base;           // sum_n at v = 0
    uint32_t mask;            // present slots
    uint32_t fast_carry;      // 1 if cnt[kKMax-1] >= kTileM (a tile advance carries <= 1)
    uint32_t pad;
};

struct SlotP {
    int32_t model_id, ops, bs, seqlen;
    int32_t end_lo, end_hi, absent, radix;  // grid digit definition (decode of t*)
    double rradix;                           // 1.0 / radix (fp64 quotient in the decode)
    uint64_t tstride;                        // product of the later radices
    double rtstride;                         // 1.0 / tstride
};

// result record written by the last CTA (and gathered across ranks)
struct Result {
    unsigned long long key;  // best key, 0 = none
    float y_best;            // y(t*)
    float y0;                // y(index 0), NaN if not evaluated
    unsigned long long evaluated;
    int32_t end_op[kKMax];   // decoded t* per slot (grid order), 0 absent
    int32_t total_ops;
    int32_t status;          // 0 OK, 2 NONE (set by host for decisions)
    uint32_t seq;            // unused in device records (the mapped copy carries tags)
    uint32_t pad;
};

__host__ __device__ inline float f32_from_bits(uint32_t b) {
    float f;
    memcpy(&f, &b, 4);
    return f;
}

// Host-mapped copy of a Result: four 16-byte chunks of three payload words and
// a tag, tag = seq ^ mix(payload, chunk index). The device writes it with four
// vector stores and no system fence; the host accepts the record once all four
// tags match the sequence number it waits for (a stale or torn chunk fails its
// tag), so no store ordering across the PCIe writes is needed.
struct alignas(64) MappedRec {
    uint32_t w[16];
};
__host__ __device__ inline uint32_t rec_tag(uint32_t seq, uint32_t a, uint32_t b, uint32_t c, uint32_t i) {
    uint32_t h = (a * 0x9E3779B1u) ^ ((b + 0x7F4A7C15u) * 0x85EBCA77u) ^ ((c + i) * 0xC2B2AE3Du) ^ (i * 0x27D4EB2Fu);
    h ^= h >> 15;
    h *= 0x2C1B3C6Du;
    h ^= h >> 12;
    return seq ^ h;
}
// payload words: key lo/hi, y_best, y0, evaluated lo/hi, end_op[4], total_ops,
// status | pad << 8 (pad: m-way rounds, < 2^24)
__host__ __device__ inline void rec_payload(const Result& R, uint32_t (&p)[12]) {
    p[0] = (uint32_t)R.key;
    p[1] = (uint32_t)(R.key >> 32);
    memcpy(&p[2], &R.y_best, 4);
    memcpy(&p[3], &R.y0, 4);
    p[4] = (uint32_t)R.evaluated;
    p[5] = (uint32_t)(R.evaluated >> 32);
    for (int j = 0; j < kKMax; j++) p[6 + j] = (uint32_t)R.end_op[j];
    p[10] = (uint32_t)R.total_ops;
    p[11] = ((uint32_t)R.status & 0xFFu) | (R.pad << 8);
}
__host__ __device__ inline void rec_unpayload(const uint32_t (&p)[12], Result& R) {
    R.key = (unsigned long long)p[0] | ((unsigned long long)p[1] << 32);
    memcpy(&R.y_best, &p[2], 4);
    memcpy(&R.y0, &p[3], 4);
    R.evaluated = (unsigned long long)p[4] | ((unsigned long long)p[5] << 32);
    for (int j = 0; j < kKMax; j++) R.end_op[j] = (int32_t)p[6 + j];
    R.total_ops = (int32_t)p[10];
    R.status = (int32_t)(p[11] & 0xFFu);
    R.pad = p[11] >> 8;
    R.seq = 0;
}

// host: all four chunks of a record carry the tag of `seq` -> payload into *R
// (volatile reads: the device may be writing the record concurrently)
inline bool rec_read(const MappedRec* M, uint32_t seq, Result* R) {
    const volatile uint32_t* w = M->w;
    uint32_t p[12];
    for (uint32_t i = 0; i < 4; i++) {
        const uint32_t a = w[4 * i], b = w[4 * i + 1], c = w[4 * i + 2], t = w[4 * i + 3];
        if (t != rec_tag(seq, a, b, c, i)) return false;
        p[3 * i] = a;
        p[3 * i + 1] = b;
        p[3 * i + 2] = c;
    }
    rec_unpayload(p, *R);
    return true;
}

// a6: the global result of a contiguously sharded candidate space from the
// per-rank records r[0..n) (rank order, shard r = [floor(rT/G), floor((r+1)T/G))).
// Max key (a key embeds its index, so two records never tie unless both are 0),
// y(t*) / end ops / total ops from the winning record, evaluated summed, and
// y(0) -- the drop test's prediction (reading c14) -- from the
// first record that evaluated index 0: only that rank's shard holds it, every
// other rank publishes NaN there.  Shared by the device finalize kernel (after
// the NCCL all-gather) and the host entry point abacus_combine_decisions.
__host__ __device__ inline Result combine_results(const Result* r, int n) {
    int best = 0;
    unsigned long long ev = 0;
    float y0 = f32_from_bits(0x7fc00000u);
    bool have_y0 = false;
    for (int i = 0; i < n; i++) {
        ev += r[i].evaluated;
        if (r[i].key > r[best].key) best = i;
        if (!have_y0 && r[i].y0 == r[i].y0) {
            y0 = r[i].y0;
            have_y0 = true;
        }
    }
    Result out = r[best];
    out.evaluated = ev;
    out.y0 = y0;
    out.status = out.key ? 0 : 2;
    return out;
}

enum PlanMode : int32_t { kModeGrid = 0, kModeChain = 1 };

// a6 over peer memory (abacus_peer_comm_init): every rank owns a mailbox of
// kPeerMax tagged records in its device memory; the last CTA of a rank's fused
// search writes its record into slot `rank` of every rank's mailbox (P2P stores
// through NVLink, or plain stores when the ranks share a device), then waits in
// its own mailbox for every rank's record of the same sequence number and
// combines them (combine_results) -- compute and collective in one kernel.
constexpr int kPeerMax = 32;  // ABACUS_PEER_MAX
struct PeerComb {
    int32_t nranks, rank;
    uint32_t timeout_ms;         // give up waiting for a peer after this long (status 3)
    uint32_t pad;
    MappedRec* local;            // this rank's mailbox (2 banks of kPeerMax slots)
    MappedRec* dst[kPeerMax];    // every rank's mailbox as mapped into this process
};

// header of a plan: everything but the segment table (decode of t*, a7)
struct PlanHdr {
    int32_t k, n_seg, n_models, D;
    int32_t mode;           // kModeGrid (t) or kModeChain (u)
    int32_t want_y0;        // 1 if index 0 is in range (decision drop test)
    float H;                // headroom threshold (inclusive)
    int32_t pad;
    uint64_t n_tiles;       // total work items
    uint64_t T;             // size of the whole space
    uint64_t n_eval;        // candidates in this plan (this shard)
    uint64_t chain_cum[kKMax + 1];  // CHAIN: first u of block j
    MappedRec* mapped;      // host-mapped pinned result record (device pointer) or null
    unsigned long long* trace;  // optional %globaltimer stamps (tools only), null in production
    uint32_t seq;           // sequence number the mapped copy is tagged with
    uint32_t peer_seq;      // tag of this launch's records in the peer mailboxes (with `peer`)
    const struct PeerComb* peer;  // in-kernel cross-GPU combine (a6 over peer memory) or null
    SlotP slot[kKMax];
};

struct Plan : PlanHdr {
    SegP seg[kMaxSeg];
};

// The same header with a shorter segment table: the launch parameter of the
// fused kernels for plans of <= 8 segments (every scheduling decision: 2^(k-1)
// presence patterns or k chain blocks), 2.1 KB instead of 4 KB of kernel
// parameters per launch (decision p99 -1.5 to -2 us).  The kernels read it
// through a `const Plan&` (same layout prefix; segments >= n_seg are never read).
template <int NSEG>
struct PlanT : PlanHdr {
    SegP seg[NSEG];
};
using PlanDecision = PlanT<8>;

// ---- batched decisions (NEXT-4): many independent decisions in one launch ----
// Decision d owns tiles [2 pair0, 2 pair0 + n_tiles) of the launch (n_tiles
// rounded up to even, so a group's two lock-step tiles never straddle two
// decisions); its segments are segs[seg0 .. seg0 + h.n_seg).
constexpr int kMaxSegBatch = 8;  // decision mode: <= 2^(k-1) presence patterns
struct BatchDec {
    PlanHdr h;
    uint64_t pair0;
    uint32_t seg0;
    uint32_t pad;
};
// per-decision running result, updated with a 128-bit compare-and-swap
struct __align__(16) BatchAcc {
    unsigned long long key;
    float y;   // y(t*) of the key
    float y0;  // y(index 0), written by the owner of the decision's first row
};

struct Scratch {             // device scratch owned by the ctx
    unsigned long long cta_key[1024];
    float cta_y[1024];
    float y0;
    unsigned int counter;    // last-CTA ticket, self-resetting
    unsigned int pad;
    Result result;
    Result gathered[64];
};

#ifdef __CUDACC__

__device__ __forceinline__ uint32_t fastdiv(uint32_t x, const FastDiv& f) {
    uint32_t q = __umulhi(x, f.mul);
    return (q + x) >> f.shift;
}

// digits v[j] of the box ordinal u = ub + r (ub uniform across the tile,
// r < 2^20 per thread): ub is split with an fp64 reciprocal (exact after one
// correction step since ub < 2^40), r is then added to the last digit and
// carried with 32-bit multiply-high divisions.
template <int K>
__device__ __forceinline__ void decode_box(const SegP& s, uint64_t ub, uint32_t r, uint32_t (&v)[kKMax]) {
    uint64_t rem = ub;
#pragma unroll
    for (int j = 0; j < K; j++) {
        uint64_t bs = s.bstride[j];
        uint64_t q;
        if (bs == 1) {
            q = rem;
        } else {
            q = (uint64_t)((double)rem * s.rbstride[j]);
            int64_t rr = (int64_t)(rem - q * bs);
            if (rr < 0) { q--; }
            else if ((uint64_t)rr >= bs) { q++; }
        }
        v[j] = (uint32_t)q;
        rem -= q * bs;
    }
    // add r to the last digit and carry
    uint32_t carry = r;
#pragma unroll
    for (int j = K - 1; j >= 0; j--) {
        uint32_t x = v[j] + carry;
        uint32_t q = fastdiv(x, s.fd[j]);
        v[j] = x - q * s.cnt[j];
        carry = q;
    }
}

__device__ __forceinline__ unsigned long long umax64(unsigned long long a, unsigned long long b) {
    return a > b ? a : b;
}

__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        unsigned long long w = __shfl_xor_sync(0xffffffffu, v, o);
        v = umax64(v, w);
    }
    return v;
}

#endif  // __CUDACC__

}  // namespace abacus
