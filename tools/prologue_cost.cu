// prologue_cost.cu -- device-side fixed costs of the fused kernel's prologue,
// isolated: empty kernel vs. + TMEM alloc/dealloc, + mbarrier init, + system
// fence with a mapped store, + 25 KB dynamic shared memory, + 5 KB params.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

struct P5K { unsigned char b[5000]; };

template <int VARIANT>
__global__ void __launch_bounds__(640, 1) kern(const __grid_constant__ P5K p, int* out, volatile int* mapped) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint32_t slot;
    __shared__ uint64_t bar;
    const int warp = threadIdx.x >> 5;
    if (VARIANT & 1) {
        if (warp == 0) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        }
    }
    if (VARIANT & 2) {
        if (threadIdx.x == 0) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
            asm volatile("fence.mbarrier_init.release.cluster;");
        }
    }
    __syncthreads();
    if (VARIANT & 8) {
        for (int i = threadIdx.x; i < 25000 / 16; i += blockDim.x) reinterpret_cast<int4*>(smem)[i] = make_int4(i, 0, 0, 0);
        __syncthreads();
    }
    if (VARIANT & 1) {
        __syncthreads();
        if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
    }
    if (threadIdx.x == 0) {
        out[0] = p.b[4999] + ((VARIANT & 8) ? smem[7] : 0);
        if (VARIANT & 4) { __threadfence_system(); mapped[0] = 1; }
    }
}

template <int V>
void time_variant(const char* name, cudaStream_t s, int* d, int* dm) {
    P5K p{};
    const int smem = (V & 8) ? 25000 : 0;
    cudaFuncSetAttribute(kern<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, 32768);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float single = 0, batch = 0;
    for (int rep = 0; rep < 50; rep++) {
        cudaEventRecord(e0, s);
        kern<V><<<1, 640, smem, s>>>(p, d, dm);
        cudaEventRecord(e1, s);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep >= 10) single += ms;
    }
    cudaEventRecord(e0, s);
    for (int i = 0; i < 200; i++) kern<V><<<1, 640, smem, s>>>(p, d, dm);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&batch, e0, e1);
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) printf("error %s\n", cudaGetErrorString(err));
    printf("%-40s single launch (event) %7.2f us   back-to-back %7.2f us/launch\n", name, single / 40 * 1e3,
           batch / 200 * 1e3);
}

int main() {
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    int* d;
    cudaMalloc(&d, 64);
    int* hm;
    cudaHostAlloc(&hm, 64, cudaHostAllocMapped);
    int* dm;
    cudaHostGetDevicePointer(&dm, hm, 0);
    time_variant<0>("empty (5 KB params, 640 thr)", s, d, dm);
    time_variant<1>("+ tcgen05.alloc/dealloc 512", s, d, dm);
    time_variant<2>("+ mbarrier init + fence", s, d, dm);
    time_variant<4>("+ threadfence_system + mapped store", s, d, dm);
    time_variant<8>("+ 25 KB dynamic smem fill", s, d, dm);
    time_variant<15>("all of the above", s, d, dm);
    return 0;
}
