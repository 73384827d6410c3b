// internal.h -- declarations shared by the host API and the kernel files.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "common.cuh"

namespace abacus {

// layers 2..4 in fp32, passed by value as a kernel parameter (constant bank)
struct W234 {
    float W2[kHidden][kHidden];
    float b2[kHidden];
    float W3[kHidden][kHidden];
    float b3[kHidden];
    float w4[kHidden];
    float b4;
};

// layer 1 in fp32 for the D = 24 SIMT predictor (kernel parameter, constant bank)
struct W1P {
    float W1[kHidden][24];
    float b1[kHidden];
};

// tensor-core weight blob: layer 2 / layer 3 / output chunks in the shared
// memory B-operand layout (tc_ptx.cuh b_offset), prepared at load time
struct TcWeights {
    int fmt;           // 0 fp16, 1 bf16
    int nch_hidden;    // B chunks per hidden layer (fp16 3, bf16 5)
    int nch_out;       // B chunks of the output layer (fp16 3, bf16 5)
    uint32_t bytes;    // blob size
    float l1_scale;    // 2^-s1 applied to layer-1 weights (fp16), 1 (bf16)
    float b4;
    const uint8_t* blob;  // device
};

cudaError_t launch_encode_grid(const Plan& P, uint64_t first, uint64_t count, int16_t* out, int nsm,
                               cudaStream_t st);
cudaError_t launch_encode_groups(const void* groups, uint64_t count, int32_t n_models, int32_t D, int16_t* out,
                                 uint32_t* bad, int nsm, cudaStream_t st);
cudaError_t launch_predict_fp32(const W234& W, const W1P* w1p, const float* w1b1, int32_t D, const int16_t* x,
                                uint64_t count, float* y, int nsm, cudaStream_t st);
cudaError_t launch_select(const Plan& P, uint64_t first, uint64_t count, const float* lat, float H,
                          unsigned long long* best, int nsm, cudaStream_t st);
cudaError_t launch_fused_fp32(const Plan& P, const W234& W, const float* w1b1, Scratch* S, int nsm,
                              cudaStream_t st, int* grid_out);
cudaError_t launch_mway(const Plan& P, const W234& W, const float* w1b1, int ways, Scratch* S, cudaStream_t st);
cudaError_t launch_finalize_gather(Scratch* S, int nranks, MappedRec* mapped, uint32_t seq, cudaStream_t st);

cudaError_t launch_fused_tc(const Plan& P, const TcWeights& TW, const float* w1b1, Scratch* S, int nsm,
                            cudaStream_t st, int* grid_out);
// batched decisions: d_decs[n_dec] and d_segs planned on the device, *d_n_pairs their tile-pair total
// (pairs_ub >= it sizes the grid); acc/y0s zeroed / NaN-filled by the caller
// NEXT-3: one Adam step on a minibatch (kernels_train.cu)
struct TrainArgs {
    float* p;                 // parameters (device, updated in place)
    float* m;                 // Adam first moment
    float* v;                 // Adam second moment
    const int16_t* x;         // count x D features
    const float* t;           // count target latencies (ms)
    uint64_t count;
    int32_t D;
    float inv_count;
    float* partial;           // [blocks][n_params] per-CTA gradient sums
    float* loss_part;         // [blocks]
    unsigned* ticket;         // zero between launches
    float* loss_last;         // device scalar
    float* loss_out;          // optional device scalar for this step
    float* grad_out;          // optional device [n_params]
    float lr, beta1, beta2, eps, bc1, bc2;  // bc = 1 - beta^t (bias corrections)
};
int train_n_params(int D);
cudaError_t launch_train_step(const TrainArgs& A, cudaStream_t st);

cudaError_t launch_batch_tc(const BatchDec* d_decs, const SegP* d_segs, int32_t n_dec, const uint64_t* d_n_pairs,
                            uint64_t pairs_ub, uint32_t maxcnt, int32_t D, const TcWeights& TW, const float* w1b1,
                            BatchAcc* acc, float* y0s, Result* out, int nsm, cudaStream_t st);
cudaError_t launch_predict_tc(const TcWeights& TW, const W234& W, const float* w1b1, int32_t D, const int16_t* x,
                              uint64_t count,
                              float* y, int nsm, cudaStream_t st);

}  // namespace abacus
