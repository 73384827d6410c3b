// probe_umma.cu -- TEST-ONLY library (libabacus_probe.so): one tcgen05.mma of
// M=128 x N x K=16 with A in TMEM and B in shared memory, to pin the operand
// layouts the product kernels assume (tc_ptx.cuh):
//   A (TMEM): lane m = row m, 32-bit column c holds k = 2c (low half), 2c+1 (high)
//   B (smem): K-major SWIZZLE_NONE core matrices, K-adjacent 128 B apart (LBO),
//             N-adjacent 256 B apart (SBO)
// variant 0: descriptor (LBO=128, SBO=256), A at column 32
// variant 1: descriptor fields swapped (LBO=256, SBO=128)
// variant 2: as 0 but A at column 40 (A address not 32-aligned)
// variant 3: as 0, and the same A/B issued twice with accumulate (D = 2 A B^T)
// variant 4: as 0 with an f16 accumulator (idesc c_format = F16); raw D words
// variant 5: as 4, issued twice with accumulate
// variant 6: as 0 with D columns [0, 32) pre-filled with a sentinel: an N < 32
//            MMA must leave columns [N, 32) untouched (N = 8 at M = 128)
#include <cuda_runtime.h>

#include <cstdint>

#include "tc_ptx.cuh"

using namespace abacus::tc;

__global__ void probe_kernel(int fmt, int variant, int N, const uint32_t* __restrict__ a_words,
                             const uint16_t* __restrict__ b, float* __restrict__ d_out) {
    __shared__ __align__(1024) uint8_t sb[4096];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int i = tid; i < 4096; i += blockDim.x) sb[i] = 0;
    __syncthreads();
    for (int e = tid; e < N * 16; e += blockDim.x) {
        const int n = e / 16, k = e % 16;
        *reinterpret_cast<uint16_t*>(sb + b_offset(n, k)) = b[n * 16 + k];
    }
    if (tid == 0) {
        mbar_init(&bar, 1);
        mbar_fence_init();
    }
    if (warp == 0) {
        tmem_alloc(&slot, 128);
        tmem_relinquish();
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tb = slot;
    const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
    const uint32_t acol = variant == 2 ? 40u : 32u;
    uint32_t a[8];
    for (int c = 0; c < 8; c++) a[c] = a_words[tid * 8 + c];
    tmem_st8(tb + acol + lane_off, a);
    if (variant == 6) {
        uint32_t z[16];
        for (int c = 0; c < 16; c++) z[c] = __float_as_uint(-777.0f);
        tmem_st16(tb + lane_off, z);
        tmem_st16(tb + 16 + lane_off, z);
    }
    tmem_wait_st();
    fence_before();
    __syncthreads();
    if (tid == 0) {
        fence_after();
        const uint32_t saddr = smem_u32(sb);
        const uint64_t desc = variant == 1 ? smem_desc(saddr, 256, 128) : smem_desc(saddr, 128, 256);
        uint32_t id = idesc_f16(fmt, N);
        if (variant == 4 || variant == 5) id &= ~(3u << 4);  // D format F16
        mma_ts(tb, tb + acol, desc, id, 0u);
        if (variant == 3 || variant == 5) mma_ts(tb, tb + acol, desc, id, 1u);
        mma_commit(&bar);
    }
    mbar_wait(&bar, 0);
    fence_after();
    uint32_t r[32];
    tmem_ld32(tb + lane_off, r);
    const int nout = variant == 6 ? 32 : N;
    for (int n = 0; n < nout; n++) d_out[tid * nout + n] = __uint_as_float(r[n]);
    fence_before();
    __syncthreads();
    fence_after();
    if (warp == 0) tmem_dealloc(tb, 128);
}

extern "C" int abacus_probe_mma(int fmt, int variant, int N, const uint32_t* a_words_host /*128x8*/,
                                const uint16_t* b_host /*N x 16*/, float* d_host /*128 x N*/) {
    uint32_t* da = nullptr;
    uint16_t* db = nullptr;
    float* dd = nullptr;
    cudaError_t e = cudaSuccess;
    if ((e = cudaMalloc(&da, 128 * 8 * 4)) != cudaSuccess) return (int)e;
    if ((e = cudaMalloc(&db, N * 16 * 2)) != cudaSuccess) return (int)e;
    const int nout = variant == 6 ? 32 : N;
    if ((e = cudaMalloc(&dd, 128 * nout * 4)) != cudaSuccess) return (int)e;
    cudaMemcpy(da, a_words_host, 128 * 8 * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(db, b_host, N * 16 * 2, cudaMemcpyHostToDevice);
    probe_kernel<<<1, 128>>>(fmt, variant, N, da, db, dd);
    e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaMemcpy(d_host, dd, 128 * nout * 4, cudaMemcpyDeviceToHost);
    cudaFree(da);
    cudaFree(db);
    cudaFree(dd);
    return (int)e;
}
