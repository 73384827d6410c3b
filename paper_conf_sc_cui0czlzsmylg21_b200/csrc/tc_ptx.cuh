// tc_ptx.cuh -- thin inline-PTX wrappers for tcgen05 / TMEM / mbarrier /
// bulk copies on sm_100a, plus the operand layouts the kernels use.
#pragma once
#include <cstdint>

namespace abacus {
namespace tc {

// ---- operand layouts -------------------------------------------------------
// B operand (weights) in shared memory, K-major, SWIZZLE_NONE: a chunk holds
// N rows x 16 K of 16-bit values as 8x8 core matrices (8 rows x 16 bytes,
// 128 contiguous bytes); core matrices adjacent along K are kLBO bytes apart,
// along N kSBO bytes apart.
constexpr uint32_t kLBO = 128;
constexpr uint32_t kSBO = 256;
__host__ __device__ constexpr uint32_t b_offset(int n, int k) {
    return (uint32_t)((n >> 3) * kSBO + (k >> 3) * kLBO + (n & 7) * 16 + (k & 7) * 2);
}
constexpr uint32_t kChunkBytesN32 = 32 * 16 * 2;  // 1 KB
constexpr uint32_t kChunkBytesN16 = 16 * 16 * 2;  // 512 B

// instruction descriptor, kind::f16: D fp32 (or f16: f32_accum false), A/B fp16 (fmt 0) or bf16 (fmt 1),
// both K-major, M = 128.
__host__ __device__ constexpr uint32_t idesc_f16(int fmt, int N, bool f32_accum = true) {
    return ((uint32_t)f32_accum << 4) | ((uint32_t)fmt << 7) | ((uint32_t)fmt << 10) | ((uint32_t)(N >> 3) << 17) |
           ((uint32_t)(128 >> 4) << 24);
}

#ifdef __CUDACC__
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// shared-memory matrix descriptor (sm_100: version bits [46,48) = 1)
__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t lbo = kLBO, uint32_t sbo = kSBO) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}

// ---- mbarrier ----------------------------------------------------------------
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
#ifdef EXP_SUSPEND
    asm volatile(
        "{\n\t"
        ".reg .pred P1;\n\t"
        "LAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n\t"
        "@P1 bra DONE;\n\t"
        "bra LAB_WAIT;\n\t"
        "DONE:\n\t"
        "}" ::"r"(smem_u32(bar)),
        "r"(parity), "n"(EXP_SUSPEND)
        : "memory");
#else
    asm volatile(
        "{\n\t"
        ".reg .pred P1;\n\t"
        "LAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@P1 bra DONE;\n\t"
        "bra LAB_WAIT;\n\t"
        "DONE:\n\t"
        "}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
#endif
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

// ---- bulk copy global -> shared (TMA engine, 1-D), completes on an mbarrier --
__device__ __forceinline__ void bulk_g2s(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_u32(smem_dst)),
        "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
        : "memory");
}

// ---- shared-memory atomic with acquire-release semantics (CTA scope) --------
__device__ __forceinline__ uint32_t atom_add_acqrel(uint32_t* p, uint32_t v) {
    uint32_t old;
    asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(smem_u32(p)), "r"(v)
                 : "memory");
    return old;
}

// ---- named barrier over a subset of warps -----------------------------------
__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

__device__ __forceinline__ void named_bar_arrive(uint32_t id, uint32_t nthreads) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

// ---- TMEM allocation ----------------------------------------------------------
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
                 "r"(ncols)
                 : "memory");
}
__device__ __forceinline__ void tmem_relinquish() {
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}

// ---- ordering ---------------------------------------------------------------
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// ---- MMA: D[tmem] (+)= A[tmem] * B[smem]^T, kind::f16, M = 128 --------------
__device__ __forceinline__ void mma_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                       uint32_t accumulate) {
    asm volatile(
        "{\n\t"
        ".reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t"
        "}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}
// elect forms: called by ALL lanes of one warp inside a warp-uniform branch;
// elect.sync picks one lane to issue.  With warp-uniform operands the compiler
// emits a single ELECT + UTCHMMA (no per-lane waterfall loop).
__device__ __forceinline__ void mma_ts_elect(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                             uint32_t accumulate) {
    asm volatile(
        "{\n\t"
        ".reg .pred p, e;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t"
        "}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
        : "memory");
}
__device__ __forceinline__ void mma_commit_elect(uint64_t* bar) {
    asm volatile(
        "{\n\t"
        ".reg .pred e;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t"
        "}" ::"r"(smem_u32(bar))
        : "memory");
}

// One whole layer in one asm block (called by all lanes of the issuing warp):
// chunk descriptors are derived from the layer's base descriptor by 64-bit
// adds (a chunk = CHUNK bytes = CHUNK >> 4 descriptor units; no carry out of
// the 14-bit start-address field), the instruction descriptor is an
// immediate, one elected lane issues the MMAs and the commit.
//   FMT 0 (fp16):  D  = A[0:8) W_c0 + A[8:16) W_c1 + C bias
//   FMT 1 (bf16):  D  = A[0:8) Whi_c0 + A[8:16) Whi_c1 + A[0:8) Wlo_c0 + A[8:16) Wlo_c1 + C bias
// LO (bf16 only): also the lo chunks 2, 3; the bias chunk is then 4, else BCH.
template <int FMT, uint32_t IDESC, uint32_t CHUNK, bool BIAS = true, uint32_t BCH = 2, bool LO = (FMT == 1)>
__device__ __forceinline__ void issue_layer_asm(uint32_t tD, uint32_t tA, uint32_t tC, uint64_t dbase,
                                                uint64_t* bar) {
    constexpr uint32_t U = CHUNK >> 4;
    if (!LO && !BIAS) {  // the two data chunks only (the bias is added outside)
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d1;\n\t"
            ".reg .b32 a8;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d1, %2, %4;\n\t"
            "add.u32 a8, %1, 8;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %5, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [a8], d1, %5, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%3];\n\t"
            "}" ::"r"(tD),
            "r"(tA), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U), "n"(IDESC)
            : "memory");
        return;
    }
    if (!LO) {
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d1, d2;\n\t"
            ".reg .b32 a8;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d1, %3, %5;\n\t"
            "add.s64 d2, %3, %6;\n\t"
            "add.u32 a8, %1, 8;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %3, %7, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [a8], d1, %7, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], d2, %7, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%4];\n\t"
            "}" ::"r"(tD),
            "r"(tA), "r"(tC), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U), "n"((uint64_t)(BCH * U)),
            "n"(IDESC)
            : "memory");
    } else {
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d1, d2, d3, d4;\n\t"
            ".reg .b32 a8;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d1, %3, %5;\n\t"
            "add.s64 d2, %3, %6;\n\t"
            "add.s64 d3, %3, %7;\n\t"
            "add.s64 d4, %3, %8;\n\t"
            "add.u32 a8, %1, 8;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %3, %9, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [a8], d1, %9, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], d2, %9, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [a8], d3, %9, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], d4, %9, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%4];\n\t"
            "}" ::"r"(tD),
            "r"(tA), "r"(tC), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U), "n"((uint64_t)(2 * U)),
            "n"((uint64_t)(3 * U)), "n"((uint64_t)(4 * U)), "n"(IDESC)
            : "memory");
    }
}

// the MMAs of one layer for TWO tiles (same B operand) and ONE commit:
// chunks 0, 1 (the two K halves of the weights) and, with BIAS, the bias chunk
// BCH against the constant chunk (fp16 blob: BCH = 2; bf16 blob: BCH = 4, the
// lo chunks 2, 3 skipped -- layer 2 of the bf16 path runs hi weights only).
// IDESC carries the operand format (f16 or bf16).
template <int FMT, uint32_t IDESC, uint32_t CHUNK, bool BIAS = true, uint32_t BCH = 2>
__device__ __forceinline__ void issue_layer2_asm(uint32_t tDx, uint32_t tAx, uint32_t tDy, uint32_t tAy,
                                                 uint32_t tCx, uint32_t tCy, uint64_t dbase, uint64_t* bar) {
    constexpr uint32_t U = CHUNK >> 4;
    if (!BIAS) {  // the two data chunks only (the bias is added outside)
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d1;\n\t"
            ".reg .b32 ax8, ay8;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d1, %4, %6;\n\t"
            "add.u32 ax8, %1, 8;\n\t"
            "add.u32 ay8, %3, 8;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %4, %7, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ax8], d1, %7, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%3], %4, %7, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [ay8], d1, %7, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%5];\n\t"
            "}" ::"r"(tDx),
            "r"(tAx), "r"(tDy), "r"(tAy), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U), "n"(IDESC)
            : "memory");
        return;
    }
    asm volatile(
        "{\n\t"
        ".reg .pred e, pf, pt;\n\t"
        ".reg .b64 d1, d2;\n\t"
        ".reg .b32 ax8, ay8;\n\t"
        "setp.ne.b32 pf, 0, 0;\n\t"
        "setp.eq.b32 pt, 0, 0;\n\t"
        "add.s64 d1, %5, %7;\n\t"
        "add.s64 d2, %5, %8;\n\t"
        "add.u32 ax8, %1, 8;\n\t"
        "add.u32 ay8, %3, 8;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %5, %9, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ax8], d1, %9, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%4], d2, %9, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%3], %5, %9, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [ay8], d1, %9, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%10], d2, %9, pt;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n\t"
        "}" ::"r"(tDx),
        "r"(tAx), "r"(tDy), "r"(tAy), "r"(tCx), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U),
        "n"((uint64_t)(BCH * U)), "n"(IDESC), "r"(tCy)
        : "memory");
}

// issue_layer2_asm<.., false> with every operand precomputed by the caller
// (the second A half, the second chunk's descriptor): no address arithmetic
// between the barrier and the MMAs
template <uint32_t IDESC>
__device__ __forceinline__ void issue_pair2_pre(uint32_t tDx, uint32_t tAx, uint32_t tAx8, uint32_t tDy, uint32_t tAy,
                                                uint32_t tAy8, uint64_t d0, uint64_t d1, uint64_t* bar) {
    asm volatile(
        "{\n\t"
        ".reg .pred e, pf, pt;\n\t"
        "setp.ne.b32 pf, 0, 0;\n\t"
        "setp.eq.b32 pt, 0, 0;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %6, %9, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], %7, %9, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%4], %6, %9, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%5], %7, %9, pt;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%8];\n\t"
        "}" ::"r"(tDx),
        "r"(tAx), "r"(tAx8), "r"(tDy), "r"(tAy), "r"(tAy8), "l"(d0), "l"(d1), "r"(smem_u32(bar)), "n"(IDESC)
        : "memory");
}

// bf16 layer 2 / layer 3 for TWO tiles with the first two chunk descriptors and
// the second A halves precomputed (issue_pair2_pre's bf16 counterparts):
//   NCH 3: chunks 0, 1 and the bias chunk 4;  NCH 5: chunks 0..3 and the bias chunk 4
template <uint32_t IDESC, uint32_t U, int NCH>
__device__ __forceinline__ void issue_pair_bf16_pre(uint32_t tDx, uint32_t tAx, uint32_t tAx8, uint32_t tDy,
                                                    uint32_t tAy, uint32_t tAy8, uint32_t tCx, uint32_t tCy,
                                                    uint64_t d0, uint64_t d1, uint64_t* bar) {
    if (NCH == 3) {
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d4;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d4, %8, %12;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %8, %11, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], %9, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%6], d4, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%4], %8, %11, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%5], %9, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%7], d4, %11, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%10];\n\t"
            "}" ::"r"(tDx),
            "r"(tAx), "r"(tAx8), "r"(tDy), "r"(tAy), "r"(tAy8), "r"(tCx), "r"(tCy), "l"(d0), "l"(d1),
            "r"(smem_u32(bar)), "n"(IDESC), "n"((uint64_t)(4 * U))
            : "memory");
    } else {
        asm volatile(
            "{\n\t"
            ".reg .pred e, pf, pt;\n\t"
            ".reg .b64 d2, d3, d4;\n\t"
            "setp.ne.b32 pf, 0, 0;\n\t"
            "setp.eq.b32 pt, 0, 0;\n\t"
            "add.s64 d2, %8, %12;\n\t"
            "add.s64 d3, %9, %12;\n\t"
            "add.s64 d4, %8, %13;\n\t"
            "elect.sync _|e, 0xffffffff;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %8, %11, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], %9, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], d2, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%2], d3, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%6], d4, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%4], %8, %11, pf;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%5], %9, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%4], d2, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%5], d3, %11, pt;\n\t"
            "@e tcgen05.mma.cta_group::1.kind::f16 [%3], [%7], d4, %11, pt;\n\t"
            "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%10];\n\t"
            "}" ::"r"(tDx),
            "r"(tAx), "r"(tAx8), "r"(tDy), "r"(tAy), "r"(tAy8), "r"(tCx), "r"(tCy), "l"(d0), "l"(d1),
            "r"(smem_u32(bar)), "n"(IDESC), "n"((uint64_t)(2 * U)), "n"((uint64_t)(4 * U))
            : "memory");
    }
}

// bf16 layer 3 for TWO tiles: hi chunks 0, 1, lo chunks 2, 3 (W = W_hi + W_lo)
// and the bias chunk 4, one commit
template <uint32_t IDESC, uint32_t CHUNK>
__device__ __forceinline__ void issue_layer2x5_asm(uint32_t tDx, uint32_t tAx, uint32_t tDy, uint32_t tAy,
                                                   uint32_t tCx, uint32_t tCy, uint64_t dbase, uint64_t* bar) {
    constexpr uint32_t U = CHUNK >> 4;
    asm volatile(
        "{\n\t"
        ".reg .pred e, pf, pt;\n\t"
        ".reg .b64 d1, d2, d3, d4;\n\t"
        ".reg .b32 ax8, ay8;\n\t"
        "setp.ne.b32 pf, 0, 0;\n\t"
        "setp.eq.b32 pt, 0, 0;\n\t"
        "add.s64 d1, %5, %7;\n\t"
        "add.s64 d2, %5, %8;\n\t"
        "add.s64 d3, %5, %9;\n\t"
        "add.s64 d4, %5, %10;\n\t"
        "add.u32 ax8, %1, 8;\n\t"
        "add.u32 ay8, %3, 8;\n\t"
        "elect.sync _|e, 0xffffffff;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %5, %11, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ax8], d1, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], d2, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ax8], d3, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%4], d4, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%3], %5, %11, pf;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [ay8], d1, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%3], d2, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [ay8], d3, %11, pt;\n\t"
        "@e tcgen05.mma.cta_group::1.kind::f16 [%2], [%12], d4, %11, pt;\n\t"
        "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n\t"
        "}" ::"r"(tDx),
        "r"(tAx), "r"(tDy), "r"(tAy), "r"(tCx), "l"(dbase), "r"(smem_u32(bar)), "n"((uint64_t)U),
        "n"((uint64_t)(2 * U)), "n"((uint64_t)(3 * U)), "n"((uint64_t)(4 * U)), "n"(IDESC), "r"(tCy)
        : "memory");
}

// predicated forms: every lane of the issuing warps executes the instruction
// stream, only `pred != 0` issues (no divergent branch around the issue)
__device__ __forceinline__ void mma_ts_p(uint32_t pred, uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc,
                                         uint32_t idesc, uint32_t accumulate) {
    asm volatile(
        "{\n\t"
        ".reg .pred p, q;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "setp.ne.b32 q, %5, 0;\n\t"
        "@q tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t"
        "}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate), "r"(pred)
        : "memory");
}
__device__ __forceinline__ void mma_commit_p(uint32_t pred, uint64_t* bar) {
    asm volatile(
        "{\n\t"
        ".reg .pred q;\n\t"
        "setp.ne.b32 q, %1, 0;\n\t"
        "@q tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t"
        "}" ::"r"(smem_u32(bar)),
        "r"(pred)
        : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                     smem_u32(bar))
                 : "memory");
}

// ---- TMEM <-> registers (32 lanes per warp, 32-bit columns) -----------------
// loads include tcgen05.wait::ld in the same asm so no use can be hoisted above it
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]),
          "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]),
          "=r"(r[30]), "=r"(r[31])
        : "r"(taddr)
        : "memory");
}
// two 32-column loads (e.g. two tiles) with a single wait: the latencies overlap
__device__ __forceinline__ void tmem_ld32x2(uint32_t ta, uint32_t tb, uint32_t (&a)[32], uint32_t (&b)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%64];\n\t"
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
        "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%65];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]), "=r"(a[4]), "=r"(a[5]), "=r"(a[6]), "=r"(a[7]),
          "=r"(a[8]), "=r"(a[9]), "=r"(a[10]), "=r"(a[11]), "=r"(a[12]), "=r"(a[13]), "=r"(a[14]), "=r"(a[15]),
          "=r"(a[16]), "=r"(a[17]), "=r"(a[18]), "=r"(a[19]), "=r"(a[20]), "=r"(a[21]), "=r"(a[22]),
          "=r"(a[23]), "=r"(a[24]), "=r"(a[25]), "=r"(a[26]), "=r"(a[27]), "=r"(a[28]), "=r"(a[29]),
          "=r"(a[30]), "=r"(a[31]), "=r"(b[0]), "=r"(b[1]), "=r"(b[2]), "=r"(b[3]), "=r"(b[4]), "=r"(b[5]),
          "=r"(b[6]), "=r"(b[7]), "=r"(b[8]), "=r"(b[9]), "=r"(b[10]), "=r"(b[11]), "=r"(b[12]), "=r"(b[13]),
          "=r"(b[14]), "=r"(b[15]), "=r"(b[16]), "=r"(b[17]), "=r"(b[18]), "=r"(b[19]), "=r"(b[20]),
          "=r"(b[21]), "=r"(b[22]), "=r"(b[23]), "=r"(b[24]), "=r"(b[25]), "=r"(b[26]), "=r"(b[27]),
          "=r"(b[28]), "=r"(b[29]), "=r"(b[30]), "=r"(b[31])
        : "r"(ta), "r"(tb)
        : "memory");
}
// 16 consecutive 32-bit words from shared memory (four 16-byte loads); volatile
// so it stays ahead of a following mbarrier wait
__device__ __forceinline__ void lds_words16(uint32_t saddr, uint32_t (&w)[16]) {
    asm volatile(
        "ld.shared.v4.b32 {%0,%1,%2,%3}, [%16];\n\t"
        "ld.shared.v4.b32 {%4,%5,%6,%7}, [%16+16];\n\t"
        "ld.shared.v4.b32 {%8,%9,%10,%11}, [%16+32];\n\t"
        "ld.shared.v4.b32 {%12,%13,%14,%15}, [%16+48];"
        : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7]),
          "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]), "=r"(w[14]), "=r"(w[15])
        : "r"(saddr)
        : "memory");
}
// two 32-column loads of f16 accumulators (value in the low half of each
// column), adjacent columns packed into one register (.pack::16b)
__device__ __forceinline__ void tmem_ld16p_x2(uint32_t ta, uint32_t tb, uint32_t (&a)[16], uint32_t (&b)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.pack::16b.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%32];\n\t"
        "tcgen05.ld.sync.aligned.32x32b.x16.pack::16b.b32 "
        "{%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%33];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]), "=r"(a[4]), "=r"(a[5]), "=r"(a[6]), "=r"(a[7]),
          "=r"(a[8]), "=r"(a[9]), "=r"(a[10]), "=r"(a[11]), "=r"(a[12]), "=r"(a[13]), "=r"(a[14]), "=r"(a[15]),
          "=r"(b[0]), "=r"(b[1]), "=r"(b[2]), "=r"(b[3]), "=r"(b[4]), "=r"(b[5]), "=r"(b[6]), "=r"(b[7]),
          "=r"(b[8]), "=r"(b[9]), "=r"(b[10]), "=r"(b[11]), "=r"(b[12]), "=r"(b[13]), "=r"(b[14]), "=r"(b[15])
        : "r"(ta), "r"(tb)
        : "memory");
}
__device__ __forceinline__ void tmem_ld1x2(uint32_t ta, uint32_t tb, uint32_t& a, uint32_t& b) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%2];\n\t"
        "tcgen05.ld.sync.aligned.32x32b.x1.b32 {%1}, [%3];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(a), "=r"(b)
        : "r"(ta), "r"(tb)
        : "memory");
}
__device__ __forceinline__ void tmem_ld1(uint32_t taddr, uint32_t& r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];\n\ttcgen05.wait::ld.sync.aligned;"
                 : "=r"(r)
                 : "r"(taddr)
                 : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
        "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
        "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
        : "memory");
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t (&v)[8]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(v[0]),
        "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
        : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// ---- packing ------------------------------------------------------------------
// pack (lo, hi) -> 32 bits, element k = 2c in the low half
template <int FMT>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
    uint32_t d;
    if (FMT == 0) asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(d) : "f"(hi), "f"(lo));
    else asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(d) : "f"(hi), "f"(lo));
    return d;
}
template <int FMT>
__device__ __forceinline__ uint32_t pack2_relu(uint32_t lo_bits, uint32_t hi_bits) {
    uint32_t d;
    const float lo = __uint_as_float(lo_bits), hi = __uint_as_float(hi_bits);
    if (FMT == 0) asm("cvt.rn.relu.f16x2.f32 %0, %1, %2;" : "=r"(d) : "f"(hi), "f"(lo));
    else asm("cvt.rn.relu.bf16x2.f32 %0, %1, %2;" : "=r"(d) : "f"(hi), "f"(lo));
    return d;
}
template <int FMT>
__device__ __forceinline__ uint16_t to16(float v) {
    uint32_t d = pack2<FMT>(v, 0.0f);
    return (uint16_t)(d & 0xFFFFu);
}
template <int FMT>
__device__ __forceinline__ float from16(uint16_t h) {
    if (FMT == 0) {
        float f;
        asm("{ .reg .f16 t; mov.b16 t, %1; cvt.f32.f16 %0, t; }" : "=f"(f) : "h"(h));
        return f;
    }
    return __uint_as_float((uint32_t)h << 16);
}
#endif  // __CUDACC__

}  // namespace tc
}  // namespace abacus
