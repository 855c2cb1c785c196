// micro.cu -- denominator microbenchmarks for the roofline.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o micro scripts/micro.cu
// Prints one JSON object: HBM copy GB/s, L2 random-load sectors/s and GB/s (4 B
// probes into arrays of several sizes), random fp64 atomicAdd-with-return ops/s
// into an 8 MB array (PageRank residuals at RMAT-20), random u32 atomicMin ops/s,
// and the dependent-chain latency of global loads (L2 hit) in ns.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__global__ void copy_k(const int4 *__restrict__ a, int4 *__restrict__ b, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

__global__ void probe_k(const uint32_t *__restrict__ a, uint64_t mask, uint64_t iters, uint32_t *out) {
    uint64_t s = mix(blockIdx.x * 1315423911ull + threadIdx.x);
    uint32_t acc = 0;
    for (uint64_t i = 0; i < iters; i += 8) {
        uint32_t v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) { s = mix(s + k); v[k] = a[s & mask]; }
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += v[k];
    }
    if (acc == 0xdeadbeef) *out = acc;
}

// BFS-shaped: stream 8 column entries per lane (coalesced rows), probe the
// state word they name (random), like one chunk of the worker's edge loop.
__global__ void chain_k(const uint32_t *__restrict__ colv, uint64_t ncol, const uint32_t *a, uint64_t iters,
                        uint32_t *out, int rnd = 0) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const int lane = threadIdx.x & 31;
    uint32_t acc = 0;
    for (uint64_t it = 0; it < iters; ++it) {
        uint64_t base = ((it * nwarps + warp) * 256) % (ncol - 256);
        if (rnd) base = (mix(it * nwarps + warp) % (ncol / 256 - 1)) * 256;   // random 1 KB segment
        uint32_t u[8], c[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) u[k] = __ldcs(colv + base + k * 32 + lane);
#pragma unroll
        for (int k = 0; k < 8; ++k) c[k] = a[u[k]];
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += c[k];
    }
    if (acc == 0xdeadbeef) *out = acc;
}

// Random 128-byte rows (one warp-wide coalesced 4-B load each) over an array of
// `n` u32: the shape of reading random adjacency-list segments.  8 rows per lane
// group in flight.  Measures rows/s; comparing array sizes exposes TLB reach.
__global__ void rows_k(const uint32_t *__restrict__ a, uint64_t nrows, uint64_t iters, uint32_t *out) {
    const int lane = threadIdx.x & 31;
    uint64_t s = mix(((blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5) * 7919ull + 17);
    uint32_t acc = 0;
    for (uint64_t it = 0; it < iters; ++it) {
        uint32_t v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) { s = mix(s + k); v[k] = __ldcs(a + (s & (nrows - 1)) * 32 + lane); }
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += v[k];
    }
    if (acc == 0xdeadbeef) *out = acc;
}

__global__ void atomadd_k(double *a, uint64_t mask, uint64_t iters, double *out) {
    uint64_t s = mix(blockIdx.x * 2654435761ull + threadIdx.x);
    double acc = 0;
    for (uint64_t i = 0; i < iters; i += 8) {
        double v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) { s = mix(s + k); v[k] = atomicAdd(a + (s & mask), 1e-12); }
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += v[k];
    }
    if (acc == -1.0) *out = acc;
}

__global__ void atommin_k(uint32_t *a, uint64_t mask, uint64_t iters, uint32_t *out) {
    uint64_t s = mix(blockIdx.x * 40503ull + threadIdx.x);
    uint32_t acc = 0;
    for (uint64_t i = 0; i < iters; i += 8) {
        uint32_t v[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) { s = mix(s + k); v[k] = atomicMin(a + (s & mask), (uint32_t)(s >> 40)); }
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += v[k];
    }
    if (acc == 0xdeadbeef) *out = acc;
}

__global__ void chase_k(const uint32_t *a, uint64_t steps, uint32_t *out) {
    uint32_t x = 0;
    for (uint64_t i = 0; i < steps; ++i) x = __ldcg(a + x);
    *out = x;
}

int main() {
    cudaDeviceProp p;
    CK(cudaGetDeviceProperties(&p, 0));
    const int grid = p.multiProcessorCount * 4, block = 512;
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    float ms;
    printf("{\"device\": \"%s\", \"sms\": %d", p.name, p.multiProcessorCount);
    // 1. HBM copy (read + write bytes)
    {
        size_t bytes = (size_t)4 << 30;
        int4 *a, *b;
        CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes));
        CK(cudaMemset(a, 1, bytes));
        copy_k<<<grid * 4, 256>>>(a, b, bytes / 16);
        float best = 1e30f;
        for (int r = 0; r < 5; ++r) {
            cudaEventRecord(e0); copy_k<<<grid * 4, 256>>>(a, b, bytes / 16); cudaEventRecord(e1);
            cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1); best = ms < best ? ms : best;
        }
        printf(", \"hbm_copy_gbs\": %.1f", 2.0 * bytes / (best * 1e-3) / 1e9);
        cudaFree(a); cudaFree(b);
    }
    uint32_t *out; CK(cudaMalloc(&out, 64));
    // 2. random 4-byte probes into arrays of 16 MB .. 1 GB
    for (size_t mb : {16, 64, 256, 1024}) {
        size_t n = mb << 18;   // u32 count
        uint32_t *a; CK(cudaMalloc(&a, n * 4)); CK(cudaMemset(a, 0, n * 4));
        const uint64_t iters = 1024;
        probe_k<<<grid, block>>>(a, n - 1, 64, out);
        cudaEventRecord(e0); probe_k<<<grid, block>>>(a, n - 1, iters, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        const double ops = (double)grid * block * iters;
        printf(", \"probe_%zuMB_gops\": %.1f", mb, ops / (ms * 1e-3) / 1e9);
        cudaFree(a);
    }
    // 2b. probes at the worker's occupancy (2 x 512 threads per SM) and the BFS-shaped chain
    {
        size_t n = (size_t)64 << 18;
        uint32_t *a; CK(cudaMalloc(&a, n * 4)); CK(cudaMemset(a, 0, n * 4));
        const int g2 = p.multiProcessorCount * 2;
        const uint64_t iters = 1024;
        cudaEventRecord(e0); probe_k<<<g2, 512>>>(a, n - 1, iters, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"probe_64MB_occ2x512_gops\": %.1f", (double)g2 * 512 * iters / (ms * 1e-3) / 1e9);
        const size_t ncol = (size_t)512 << 20;   // 2 GB of column ids
        uint32_t *colv; CK(cudaMalloc(&colv, ncol * 4));
        // random ids in [0, n)
        std::vector<uint32_t> hcol(1 << 20);
        uint64_t s = 99;
        for (auto &x : hcol) { s = s * 6364136223846793005ull + 1442695040888963407ull; x = (uint32_t)((s >> 33) % n); }
        for (size_t off = 0; off < ncol; off += hcol.size()) CK(cudaMemcpy(colv + off, hcol.data(), hcol.size() * 4, cudaMemcpyHostToDevice));
        const uint64_t it2 = 64;
        chain_k<<<g2, 512>>>(colv, ncol, a, 4, out);
        cudaEventRecord(e0); chain_k<<<g2, 512>>>(colv, ncol, a, it2, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"chain_col_probe_occ2x512_gedges\": %.1f", (double)g2 * 512 / 32 * 256 * it2 / (ms * 1e-3) / 1e9);
        const int g4 = p.multiProcessorCount * 4;
        cudaEventRecord(e0); chain_k<<<g4, 512>>>(colv, ncol, a, it2, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"chain_col_probe_occ4x512_gedges\": %.1f", (double)g4 * 512 / 32 * 256 * it2 / (ms * 1e-3) / 1e9);
        cudaEventRecord(e0); chain_k<<<g2, 512>>>(colv, ncol, a, it2, out, 1); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"chain_randseg_probe_occ2x512_gedges\": %.1f", (double)g2 * 512 / 32 * 256 * it2 / (ms * 1e-3) / 1e9);
        cudaFree(colv);
        cudaFree(a);
    }
    // 2c. random 128-B rows over 64 MB .. 4 GB (adjacency-segment reads; TLB reach)
    {
        const size_t maxb = (size_t)4 << 30;
        uint32_t *a; CK(cudaMalloc(&a, maxb)); CK(cudaMemset(a, 0, maxb));
        const int g2 = p.multiProcessorCount * 2;
        for (size_t mb : {64, 256, 512, 1024, 2048, 4096}) {
            const uint64_t nrows = (mb << 20) / 128;
            const uint64_t iters = 64;
            rows_k<<<g2, 512>>>(a, nrows, 4, out);
            cudaEventRecord(e0); rows_k<<<g2, 512>>>(a, nrows, iters, out); cudaEventRecord(e1);
            cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
            const double rows = (double)g2 * 512 / 32 * 8 * iters;
            printf(", \"rows128_%zuMB_grows\": %.2f", mb, rows / (ms * 1e-3) / 1e9);
        }
        cudaFree(a);
    }
    // 3. random fp64 atomicAdd with return into 8 MB (RMAT-20 residuals) and 64 MB
    for (size_t mb : {8, 64}) {
        size_t n = mb << 17;   // doubles
        double *a; CK(cudaMalloc(&a, n * 8)); CK(cudaMemset(a, 0, n * 8));
        const uint64_t iters = 256;
        atomadd_k<<<grid, block>>>(a, n - 1, 16, (double *)out);
        cudaEventRecord(e0); atomadd_k<<<grid, block>>>(a, n - 1, iters, (double *)out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"atomadd_f64_%zuMB_gops\": %.1f", mb, (double)grid * block * iters / (ms * 1e-3) / 1e9);
        cudaFree(a);
    }
    // 4. random u32 atomicMin with return into 64 MB
    {
        size_t n = (size_t)64 << 18;
        uint32_t *a; CK(cudaMalloc(&a, n * 4)); CK(cudaMemset(a, 0xff, n * 4));
        const uint64_t iters = 256;
        atommin_k<<<grid, block>>>(a, n - 1, 16, out);
        cudaEventRecord(e0); atommin_k<<<grid, block>>>(a, n - 1, iters, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"atommin_u32_64MB_gops\": %.1f", (double)grid * block * iters / (ms * 1e-3) / 1e9);
        cudaFree(a);
    }
    // 5. dependent-chain latency through L2 (16 MB ring, random cycle)
    {
        size_t n = (size_t)4 << 20;
        std::vector<uint32_t> h(n);
        for (size_t i = 0; i < n; ++i) h[i] = (uint32_t)i;
        uint64_t s = 12345;
        for (size_t i = n - 1; i > 0; --i) { s = s * 6364136223846793005ull + 1442695040888963407ull; size_t j = (s >> 33) % i; std::swap(h[i], h[j]); }
        std::vector<uint32_t> nxt(n);
        for (size_t i = 0; i < n; ++i) nxt[h[i]] = h[(i + 1) % n];
        uint32_t *a; CK(cudaMalloc(&a, n * 4)); CK(cudaMemcpy(a, nxt.data(), n * 4, cudaMemcpyHostToDevice));
        const uint64_t steps = 200000;
        chase_k<<<1, 1>>>(a, 1000, out);
        cudaEventRecord(e0); chase_k<<<1, 1>>>(a, steps, out); cudaEventRecord(e1);
        cudaEventSynchronize(e1); cudaEventElapsedTime(&ms, e0, e1);
        printf(", \"l2_chase_ns\": %.1f", ms * 1e6 / steps);
        cudaFree(a);
    }
    printf("}\n");
    return 0;
}
