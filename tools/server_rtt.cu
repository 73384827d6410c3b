// server_rtt.cu -- microbenchmark for a persistent "search server" kernel:
// host writes a request (a plan-sized payload + sequence number) into pinned
// mapped memory; CTA 0 of a resident kernel polls it, reads the payload with
// 128 threads, wakes the other CTAs through a device-memory epoch, every CTA
// arrives on a ticket, the last one writes a 64-byte reply + sequence to mapped
// memory; the host spins on the reply.  Reports the round-trip percentiles.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <vector>
#include <atomic>
#include <cuda_runtime.h>

constexpr int kPayload = 3712;  // bytes (sizeof(Plan) class)
struct Req { unsigned seq; unsigned stop; unsigned pad[30]; unsigned char payload[kPayload]; };
struct Rep { unsigned seq; unsigned sum; unsigned pad[14]; };

__device__ unsigned g_epoch;
__device__ unsigned g_ticket;
__device__ unsigned g_sum[1024];

__global__ void server(volatile Req* req, volatile Rep* rep, int ctas) {
    __shared__ unsigned s_seq, s_stop;
    unsigned last = 0;
    for (;;) {
        if (blockIdx.x == 0) {
            if (threadIdx.x == 0) {
                unsigned s;
                do { s = req->seq; } while (s == last);
                __threadfence_system();
                s_seq = s;
                s_stop = req->stop;
            }
            __syncthreads();
            // read the payload (128 threads x 16 B chunks)
            unsigned acc = 0;
            const uint4* p = (const uint4*)req->payload;
            for (int i = threadIdx.x; i < kPayload / 16; i += blockDim.x) { uint4 v; asm volatile("ld.volatile.global.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p + i)); acc += v.x ^ v.w; }
            acc = __reduce_add_sync(0xffffffffu, acc);
            if ((threadIdx.x & 31) == 0) atomicAdd(&g_sum[0], acc);
            __syncthreads();
            if (threadIdx.x == 0) { __threadfence(); atomicExch(&g_epoch, s_seq); }
        } else {
            if (threadIdx.x == 0) {
                unsigned e;
                do { e = atomicAdd(&g_epoch, 0u); } while (e == last);
                s_seq = e;
            }
            __syncthreads();
        }
        const unsigned seq = s_seq;
        last = seq;
        if (blockIdx.x == 0 && s_stop) {  // stop: everyone must see it; simple: CTA 0 signals with a special epoch
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            const unsigned t = atomicAdd(&g_ticket, 1u);
            if (t == (unsigned)ctas - 1) {
                g_ticket = 0;
                __threadfence();
                rep->sum = g_sum[0];
                asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(&rep->seq), "r"(seq) : "memory");
            }
        }
        if (seq == 0xFFFFFFFFu) return;
    }
}

static double now() { return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count(); }

int main(int argc, char** argv) {
    int ctas = argc > 1 ? atoi(argv[1]) : 16;
    Req* req; Rep* rep;
    cudaHostAlloc(&req, sizeof(Req), cudaHostAllocMapped);
    cudaHostAlloc(&rep, sizeof(Rep), cudaHostAllocMapped);
    memset(req, 0, sizeof(Req)); memset(rep, 0, sizeof(Rep));
    Req* dreq; Rep* drep;
    cudaHostGetDevicePointer(&dreq, req, 0);
    cudaHostGetDevicePointer(&drep, rep, 0);
    cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    server<<<ctas, 128, 0, s>>>(dreq, drep, ctas);
    std::vector<double> t;
    for (unsigned i = 1; i <= 20000; i++) {
        double t0 = now();
        for (int j = 0; j < kPayload; j += 64) req->payload[j] = (unsigned char)i;
        std::atomic_thread_fence(std::memory_order_release);
        *(volatile unsigned*)&req->seq = i;
        while (*(volatile unsigned*)&rep->seq != i) {}
        double t1 = now();
        if (i > 1000) t.push_back(t1 - t0);
    }
    // stop
    *(volatile unsigned*)&req->seq = 0xFFFFFFFFu;
    while (*(volatile unsigned*)&rep->seq != 0xFFFFFFFFu) {}
    cudaStreamSynchronize(s);
    std::sort(t.begin(), t.end());
    printf("ctas %d: round trip p50 %.2f us  p90 %.2f  p99 %.2f  p999 %.2f  max %.2f  (%s)\n", ctas, t[t.size() / 2],
           t[t.size() * 9 / 10], t[t.size() * 99 / 100], t[t.size() * 999 / 1000], t.back(),
           cudaGetErrorString(cudaGetLastError()));
    return 0;
}
