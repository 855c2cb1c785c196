// queue_micro.cu -- SURVEY 8f N4: the paper's Fig. 1 queue microbenchmark on B200.
//
// PAPER.md:809-823 (Sec. III-A2) / Fig. 1: n threads each do 10 pushes,
// 10 pops, or 10 push-then-pop pairs on one shared device queue; the paper compares
// its warp-aggregated queue with a broker queue and a CAS queue.  Here the queue is
// the worker's own design (u64 monotone indices, tagged 8-byte slots {seq:32|item:32},
// DESIGN.md section 5.1) with four ways to reserve indices:
//   thread : one atomicAdd per thread per operation (no aggregation)
//   warp   : one atomicAdd per warp per round (ballot + popc)      -- the paper's
//   cta    : one atomicAdd per CTA per round (block scan)          -- this worker's
//   cas    : per-thread CAS loop on the counter (the paper's CAS baseline)
// Output: one JSON line per (mode, op, n) with Mops/s (device time, CUDA events).
//
// Build:  nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/queue_micro scripts/queue_micro.cu
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

enum Mode { kThread = 0, kWarp = 1, kCta = 2, kCas = 3 };
enum Op { kPush = 0, kPop = 1, kPushPop = 2 };
constexpr int kRounds = 10;

struct Q {
    unsigned long long *tail, *head;   // on separate 128-B lines
    uint64_t *ring;
    uint64_t cap;                      // power of two
};

__device__ __forceinline__ uint64_t reserve(Q q, unsigned long long *ctr, int mode, unsigned *smem_base) {
    const int lane = threadIdx.x & 31;
    if (mode == kThread) return atomicAdd(ctr, 1ull);
    if (mode == kCas) {
        unsigned long long o = *(volatile unsigned long long *)ctr, a;
        while ((a = atomicCAS(ctr, o, o + 1)) != o) o = a;
        return o;
    }
    if (mode == kWarp) {
        const unsigned m = __activemask();
        const int leader = __ffs(m) - 1;
        unsigned long long b = 0;
        if (lane == leader) b = atomicAdd(ctr, (unsigned long long)__popc(m));
        b = __shfl_sync(m, b, leader);
        return b + __popc(m & ((1u << lane) - 1));
    }
    // kCta: every thread of the block takes one index, one atomic per block
    __shared__ unsigned long long cbase;
    if (threadIdx.x == 0) cbase = atomicAdd(ctr, (unsigned long long)blockDim.x);
    __syncthreads();
    const uint64_t r = cbase + threadIdx.x;
    __syncthreads();
    return r;
}

__device__ __forceinline__ void push(Q q, uint64_t idx, uint32_t item) {
    uint64_t *p = &q.ring[idx & (q.cap - 1)];
    while ((uint32_t)(*(volatile uint64_t *)p >> 32) != (uint32_t)idx) { }          // slot free for idx
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(((uint64_t)(uint32_t)(idx + 1) << 32) | item));
}
__device__ __forceinline__ uint32_t pop(Q q, uint64_t idx) {
    uint64_t *p = &q.ring[idx & (q.cap - 1)];
    uint64_t v;
    do { asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p)); } while ((uint32_t)(v >> 32) != (uint32_t)(idx + 1));
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"((uint64_t)(uint32_t)(idx + q.cap) << 32));
    return (uint32_t)v;
}

__global__ void bench_kernel(Q q, int mode, int op, unsigned long long *sink) {
    uint32_t acc = 0;
    for (int r = 0; r < kRounds; ++r) {
        if (op == kPush || op == kPushPop) push(q, reserve(q, q.tail, mode, nullptr), threadIdx.x + r);
        if (op == kPop || op == kPushPop) acc += pop(q, reserve(q, q.head, mode, nullptr));
    }
    if (acc == 0xFFFFFFFFu) atomicAdd(sink, 1ull);
}

__global__ void init_ring(uint64_t *ring, uint64_t cap, uint64_t prefill) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x)
        ring[i] = i < prefill ? ((uint64_t)(uint32_t)(i + 1) << 32) | 7u : (uint64_t)(uint32_t)i << 32;
}

int main(int argc, char **argv) {
    const int block = 512;                       // the worker's CTA size
    const char *mname[] = {"thread", "warp", "cta", "cas"};
    const char *oname[] = {"push", "pop", "push_then_pop"};
    const int max_log = argc > 1 ? atoi(argv[1]) : 20;
    uint64_t cap = 1;
    while (cap < ((uint64_t)kRounds << max_log)) cap <<= 1;
    Q q{};
    unsigned long long *ctr = nullptr, *sink = nullptr;
    CK(cudaMalloc(&ctr, 256));
    CK(cudaMalloc(&sink, 8));
    CK(cudaMalloc(&q.ring, cap * 8));
    q.tail = ctr;
    q.head = ctr + 16;
    q.cap = cap;
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    for (int lg = 10; lg <= max_log; lg += 2) {
        const uint64_t n = 1ull << lg;
        for (int op = 0; op < 3; ++op)
            for (int mode = 0; mode < 4; ++mode) {
                if (mode == kCas && lg > 14) continue;   // retry storms: 2.9 s per launch at 2^16 threads
                float best = 1e30f;
                for (int rep = 0; rep < 3; ++rep) {
                    const uint64_t prefill = op == kPop ? (uint64_t)kRounds * n : 0;
                    init_ring<<<1024, 256>>>(q.ring, cap, prefill);
                    unsigned long long h[32] = {0};
                    h[0] = prefill;                  // tail
                    CK(cudaMemcpy(ctr, h, 256, cudaMemcpyHostToDevice));
                    CK(cudaDeviceSynchronize());
                    CK(cudaEventRecord(a));
                    bench_kernel<<<(unsigned)(n / block), block>>>(q, mode, op, sink);
                    CK(cudaEventRecord(b));
                    CK(cudaEventSynchronize(b));
                    CK(cudaGetLastError());
                    float ms = 0;
                    CK(cudaEventElapsedTime(&ms, a, b));
                    best = ms < best ? ms : best;
                }
                const double ops = (double)n * kRounds * (op == kPushPop ? 2 : 1);
                printf("{\"mode\": \"%s\", \"op\": \"%s\", \"threads\": %llu, \"ms\": %.4f, \"Mops\": %.1f}\n",
                       mname[mode], oname[op], (unsigned long long)n, best, ops / (best * 1e-3) / 1e6);
                fflush(stdout);
            }
    }
    return 0;
}
