// kernels_train.cu -- NEXT-3: training the latency predictor on the GPU.
//
// One Adam step on a minibatch per launch (readings t1-t3):
//   loss = mean_s (y_s / t_s - 1)^2   (the smooth square of Eq. 1)
//   MLP  = D -> 32 -> 32 -> 32 -> 1, ReLU hidden, linear output (c1)
//   Adam (bias-corrected), learning rate per step.
//
// CTA = 128 samples x 4 threads.  Phase 1: forward pass and backward deltas in
// fp32, each thread owning 8 hidden units of its sample, weights in shared
// memory with padded rows, every per-sample vector in a padded shared row.
// Phase 2: the CTA's gradient partial sums dW_l[i][j] = sum_s delta_l[s][i]
// a_{l-1}[s][j] as register-blocked outer products over sample quarters,
// written to a per-CTA slot in global memory.  Phase 3 (the last CTA
// to finish, atomic ticket): sums the slots in CTA order (deterministic, no
// float atomics), applies Adam in place and records the loss.  The per-step
// contractions are 32 x 32 x 128 per CTA: the step is bound by latency and
// the cross-CTA reduction, not by FLOPs, so it runs on the FMA pipes.
#include <cuda_runtime.h>

#include <type_traits>

#include "common.cuh"
#include "internal.h"

namespace abacus {

namespace {
constexpr int kSamples = 128;                  // samples per CTA
constexpr int kQuad = 4;                       // threads per sample
constexpr int kTrainThreads = kSamples * kQuad;
constexpr int kUnits = kHidden / kQuad;        // hidden units per thread (8)
constexpr int kRow = kHidden + 1;              // padded shared rows (conflict-free quad access)
constexpr int kMaxD = 32;

struct TrainOffsets {
    int W1, b1, W2, b2, W3, b3, w4, b4, n;
};
__host__ __device__ inline TrainOffsets train_offsets(int D) {
    TrainOffsets o;
    o.W1 = 0;
    o.b1 = kHidden * D;
    o.W2 = o.b1 + kHidden;
    o.b2 = o.W2 + kHidden * kHidden;
    o.W3 = o.b2 + kHidden;
    o.b3 = o.W3 + kHidden * kHidden;
    o.w4 = o.b3 + kHidden;
    o.b4 = o.w4 + kHidden;
    o.n = o.b4 + 1;
    return o;
}

// shared memory (floats): padded weights | X0 | A1 A2 A3 D1 D2 D3 | G4 | quarter partials
// weights twice: transposed (forward: row = input j, the 8 units of a thread
// contiguous -> two 16-byte loads) and natural (backward: row = unit i)
struct TrainSmem {
    int W1T, W2T, W3T, W2, W3, vec, X0, A1, A2, A3, D1, D2, D3, G4, red, total;
};
__host__ __device__ inline TrainSmem train_smem(int D) {
    TrainSmem L;
    int o = 0;
    L.W1T = o; o += D * kHidden;
    L.W2T = o; o += kHidden * kHidden;
    L.W3T = o; o += kHidden * kHidden;
    L.W2 = o; o += kHidden * kHidden;
    L.W3 = o; o += kHidden * kHidden;
    L.vec = o; o += 4 * kHidden + 4;             // b1 b2 b3 w4 | b4
    L.X0 = o; o += kSamples * (D + 1);
    L.A1 = o; o += kSamples * kRow;
    L.A2 = o; o += kSamples * kRow;
    L.A3 = o; o += kSamples * kRow;
    L.D1 = o; o += kSamples * kRow;
    L.D2 = o; o += kSamples * kRow;
    L.D3 = o; o += kSamples * kRow;
    L.G4 = o; o += kSamples;
    L.red = o; o += kQuad * train_offsets(D).n;  // per sample-quarter gradient partials
    L.total = o;
    return L;
}
}  // namespace

// Thread (sample s, quad q) owns hidden units q*8 .. q*8+7 of every layer:
// it computes those units' pre-activations from the full previous-layer row
// (read from shared memory), writes its 8 results back to the sample's row,
// and the 4 threads of the sample (consecutive lanes) meet at __syncwarp.
__global__ void __launch_bounds__(kTrainThreads) train_step_kernel(const TrainArgs A) {
    extern __shared__ float sm[];
    const int D = A.D;
    const TrainOffsets o = train_offsets(D);
    const TrainSmem L = train_smem(D);
    const int XR = D + 1;
    float* W1T = sm + L.W1T;
    float* W2T = sm + L.W2T;
    float* W3T = sm + L.W3T;
    float* W2 = sm + L.W2;
    float* W3 = sm + L.W3;
    float* b1 = sm + L.vec;
    float* b2 = b1 + kHidden;
    float* b3 = b2 + kHidden;
    float* w4 = b3 + kHidden;
    float* b4 = w4 + kHidden;
    float* X0 = sm + L.X0;
    float* A1 = sm + L.A1;
    float* A2 = sm + L.A2;
    float* A3 = sm + L.A3;
    float* D1 = sm + L.D1;
    float* D2 = sm + L.D2;
    float* D3 = sm + L.D3;
    float* G4 = sm + L.G4;
    float* red = sm + L.red;
    __shared__ float s_loss[kTrainThreads / 32];
    __shared__ bool s_last;

    const int tid = threadIdx.x;
    for (int e = tid; e < o.n; e += kTrainThreads) {
        const float v = A.p[e];
        if (e < o.b1) W1T[(e % D) * kHidden + e / D] = v;
        else if (e < o.W2) b1[e - o.b1] = v;
        else if (e < o.b2) {
            const int i = (e - o.W2) >> 5, j = (e - o.W2) & 31;
            W2[i * kHidden + j] = v;
            W2T[j * kHidden + i] = v;
        } else if (e < o.W3) b2[e - o.b2] = v;
        else if (e < o.b3) {
            const int i = (e - o.W3) >> 5, j = (e - o.W3) & 31;
            W3[i * kHidden + j] = v;
            W3T[j * kHidden + i] = v;
        }
        else if (e < o.w4) b3[e - o.b3] = v;
        else if (e < o.b4) w4[e - o.w4] = v;
        else b4[0] = v;
    }
    const int sl = tid >> 2, q = tid & 3, u0 = q * kUnits;
    const uint64_t sidx = (uint64_t)blockIdx.x * kSamples + sl;
    const bool valid = sidx < A.count;
    // features of sample sl: the quad loads them together
    for (int j = q; j < D; j += kQuad) X0[sl * XR + j] = valid ? (float)A.x[sidx * (uint64_t)D + j] : 0.0f;
    __syncthreads();

    // ---- phase 1: forward + backward deltas ----
    float lossterm = 0.0f;
    {
        const float* xr = X0 + sl * XR;
        float* a1r = A1 + sl * kRow;
        float* a2r = A2 + sl * kRow;
        float* a3r = A3 + sl * kRow;
        float acc[kUnits];
#pragma unroll
        for (int k = 0; k < kUnits; k++) acc[k] = b1[u0 + k];
        for (int j = 0; j < D; j++) {
            const float xv = xr[j];
#pragma unroll
            for (int k = 0; k < kUnits; k++) acc[k] = fmaf(W1T[j * kHidden + u0 + k], xv, acc[k]);
        }
#pragma unroll
        for (int k = 0; k < kUnits; k++) a1r[u0 + k] = fmaxf(acc[k], 0.0f);
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kUnits; k++) acc[k] = b2[u0 + k];
#pragma unroll 8
        for (int j = 0; j < kHidden; j++) {
            const float av = a1r[j];
#pragma unroll
            for (int k = 0; k < kUnits; k++) acc[k] = fmaf(W2T[j * kHidden + u0 + k], av, acc[k]);
        }
#pragma unroll
        for (int k = 0; k < kUnits; k++) a2r[u0 + k] = fmaxf(acc[k], 0.0f);
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kUnits; k++) acc[k] = b3[u0 + k];
#pragma unroll 8
        for (int j = 0; j < kHidden; j++) {
            const float av = a2r[j];
#pragma unroll
            for (int k = 0; k < kUnits; k++) acc[k] = fmaf(W3T[j * kHidden + u0 + k], av, acc[k]);
        }
        float a3[kUnits];
        float y = 0.0f;
#pragma unroll
        for (int k = 0; k < kUnits; k++) {
            a3[k] = fmaxf(acc[k], 0.0f);
            a3r[u0 + k] = a3[k];
            y = fmaf(w4[u0 + k], a3[k], y);
        }
        y += __shfl_xor_sync(0xffffffffu, y, 1);
        y += __shfl_xor_sync(0xffffffffu, y, 2);
        y += b4[0];
        float g = 0.0f;
        if (valid) {
            const float t = A.t[sidx];
            const float r = y / t - 1.0f;
            if (q == 0) lossterm = r * r;
            g = 2.0f * r / t * A.inv_count;
        }
        if (q == 0) G4[sl] = g;
        // dL/dz3 = g w4 [a3 > 0] (a > 0 <=> z > 0)
        float* d3r = D3 + sl * kRow;
        float* d2r = D2 + sl * kRow;
        float* d1r = D1 + sl * kRow;
#pragma unroll
        for (int k = 0; k < kUnits; k++) d3r[u0 + k] = a3[k] > 0.0f ? g * w4[u0 + k] : 0.0f;
        __syncwarp();
        // dL/dz2[j] = [a2 > 0] sum_i W3[i][j] d3[i], j = own units
#pragma unroll
        for (int k = 0; k < kUnits; k++) acc[k] = 0.0f;
#pragma unroll 8
        for (int i = 0; i < kHidden; i++) {
            const float dv = d3r[i];
#pragma unroll
            for (int k = 0; k < kUnits; k++) acc[k] = fmaf(W3[i * kHidden + u0 + k], dv, acc[k]);
        }
#pragma unroll
        for (int k = 0; k < kUnits; k++) d2r[u0 + k] = a2r[u0 + k] > 0.0f ? acc[k] : 0.0f;
        __syncwarp();
#pragma unroll
        for (int k = 0; k < kUnits; k++) acc[k] = 0.0f;
#pragma unroll 8
        for (int i = 0; i < kHidden; i++) {
            const float dv = d2r[i];
#pragma unroll
            for (int k = 0; k < kUnits; k++) acc[k] = fmaf(W2[i * kHidden + u0 + k], dv, acc[k]);
        }
#pragma unroll
        for (int k = 0; k < kUnits; k++) d1r[u0 + k] = a1r[u0 + k] > 0.0f ? acc[k] : 0.0f;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) lossterm += __shfl_xor_sync(0xffffffffu, lossterm, off);
    if ((tid & 31) == 0) s_loss[tid >> 5] = lossterm;
    __syncthreads();

    // ---- phase 2: this CTA's gradient partial sums ----
    // dW[i][j] = sum_s delta[s][i] a[s][j] as register-blocked outer products:
    // thread = (sample quarter, 2 x JT tile); per sample 2 + JT shared loads
    // feed 2 JT independent FMAs; the quarters are summed through shared memory.
    const uint64_t left = A.count - (uint64_t)blockIdx.x * kSamples;
    const int ns = left < (uint64_t)kSamples ? (int)left : kSamples;
    const int quarter = tid >> 7, tt = tid & 127;
    const int sb = quarter * (kSamples / kQuad), se = min(sb + kSamples / kQuad, ns);
    float* myred = red + quarter * o.n;
    const int i0 = 2 * (tt >> 3), jb = tt & 7;
    auto outer = [&](auto jt_c, const float* dl, const float* al, int astride, int ncol, int off) {
        constexpr int JT = decltype(jt_c)::value;
        float acc[2][JT];
#pragma unroll
        for (int a2 = 0; a2 < 2; a2++)
#pragma unroll
            for (int b2 = 0; b2 < JT; b2++) acc[a2][b2] = 0.0f;
        const int j0 = jb * JT;
#pragma unroll 4
        for (int s2 = sb; s2 < se; s2++) {
            const float d0 = dl[s2 * kRow + i0], d1 = dl[s2 * kRow + i0 + 1];
#pragma unroll
            for (int b2 = 0; b2 < JT; b2++) {
                const float av = al[s2 * astride + j0 + b2];
                acc[0][b2] = fmaf(d0, av, acc[0][b2]);
                acc[1][b2] = fmaf(d1, av, acc[1][b2]);
            }
        }
#pragma unroll
        for (int b2 = 0; b2 < JT; b2++) {
            if (j0 + b2 < ncol) {
                myred[off + i0 * ncol + j0 + b2] = acc[0][b2];
                myred[off + (i0 + 1) * ncol + j0 + b2] = acc[1][b2];
            }
        }
    };
    if (D <= 24) outer(std::integral_constant<int, 3>{}, D1, X0, XR, D, o.W1);
    else outer(std::integral_constant<int, 4>{}, D1, X0, XR, D, o.W1);
    outer(std::integral_constant<int, 4>{}, D2, A1, kRow, kHidden, o.W2);
    outer(std::integral_constant<int, 4>{}, D3, A2, kRow, kHidden, o.W3);
    // biases b1, b2, b3 (3 x 32 threads), the output weights w4 and b4 (32 threads)
    if (tt < 96) {
        const float* dl = tt < 32 ? D1 : (tt < 64 ? D2 : D3);
        const int i = tt & 31;
        float acc0 = 0.0f;
        for (int s2 = sb; s2 < se; s2++) acc0 += dl[s2 * kRow + i];
        myred[(tt < 32 ? o.b1 : (tt < 64 ? o.b2 : o.b3)) + i] = acc0;
    } else {
        const int j = tt - 96;
        float acc0 = 0.0f, g0 = 0.0f;
        for (int s2 = sb; s2 < se; s2++) {
            acc0 = fmaf(G4[s2], A3[s2 * kRow + j], acc0);
            g0 += G4[s2];
        }
        myred[o.w4 + j] = acc0;
        if (j == 0) myred[o.b4] = g0;
    }
    __syncthreads();
    float* part = A.partial + (size_t)blockIdx.x * o.n;
    for (int e = tid; e < o.n; e += kTrainThreads)
        part[e] = (red[e] + red[o.n + e]) + (red[2 * o.n + e] + red[3 * o.n + e]);
    if (tid == 0) {
        float l = 0.0f;
        for (int w = 0; w < kTrainThreads / 32; w++) l += s_loss[w];
        A.loss_part[blockIdx.x] = l;
    }

    // ---- phase 3: the last CTA reduces over CTAs and applies Adam ----
    __threadfence();
    __syncthreads();
    if (tid == 0) s_last = atomicAdd(A.ticket, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    for (int e = tid; e < o.n; e += kTrainThreads) {
        // 8 independent partial sums keep 8 L2 loads in flight (fixed order: deterministic)
        float gs[8] = {0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f};
        unsigned b = 0;
        for (; b + 8 <= gridDim.x; b += 8) {
#pragma unroll
            for (int u = 0; u < 8; u++) gs[u] += __ldcg(&A.partial[(size_t)(b + u) * o.n + e]);
        }
        for (; b < gridDim.x; b++) gs[0] += __ldcg(&A.partial[(size_t)b * o.n + e]);
        const float gsum = ((gs[0] + gs[1]) + (gs[2] + gs[3])) + ((gs[4] + gs[5]) + (gs[6] + gs[7]));
        if (A.grad_out) A.grad_out[e] = gsum;
        const float m = A.beta1 * A.m[e] + (1.0f - A.beta1) * gsum;
        const float v = A.beta2 * A.v[e] + (1.0f - A.beta2) * gsum * gsum;
        A.m[e] = m;
        A.v[e] = v;
        const float mh = m / A.bc1, vh = v / A.bc2;
        A.p[e] = A.p[e] - A.lr * mh / (sqrtf(vh) + A.eps);
    }
    if (tid == 0) {
        float l = 0.0f;
        for (unsigned b = 0; b < gridDim.x; b++) l += __ldcg(&A.loss_part[b]);
        l *= A.inv_count;
        *A.loss_last = l;
        if (A.loss_out) *A.loss_out = l;
        *A.ticket = 0u;  // visible to the next launch (kernel boundary)
    }
}

int train_n_params(int D) { return train_offsets(D).n; }

cudaError_t launch_train_step(const TrainArgs& A, cudaStream_t st) {
    if (A.D < 1 || A.D > kMaxD) return cudaErrorInvalidValue;
    const size_t smem = (size_t)train_smem(A.D).total * sizeof(float);
    static size_t configured[64] = {};  // per device: set the attribute once per size
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64 || smem > configured[dev]) {
        cudaError_t e = cudaFuncSetAttribute(train_step_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        if (dev >= 0 && dev < 64) configured[dev] = smem;
    }
    const unsigned blocks = (unsigned)((A.count + kSamples - 1) / kSamples);
    train_step_kernel<<<blocks, kTrainThreads, smem, st>>>(A);
    return cudaGetLastError();
}

}  // namespace abacus
