// atos_qbench.cuh -- the queue microbenchmark of PAPER.md Fig. 1 (P:809-823,
// P:842-911), run on the worker's OWN ring code: the producer
// side is ring_store (tag check past the first lap, capacity error), the
// consumer side ring_read / slot_full_for / ring_release, exactly what
// warp_flush_local / batch_end and pop_batch execute.
//
// n threads, grouped into workers of worker_size threads (1 = thread, 32 =
// warp, 512 = CTA), each do `rounds` pushes, pops, or push-then-pop
// pairs.  A worker aggregates its threads' requests: its leader reserves up to
// `fetch` indices with ONE atomicAdd on the tail / head counter (
// the worker's FETCH_SIZE) -- or with a CAS loop (the paper's baseline).
// Pops are reserve-then-wait: a thread waits until the item of its index is
// published.  Every popped item is written to popped[] so that the caller can
// check multiset conservation (no item lost or duplicated).
#pragma once
// (included inside namespace atos by atos.cu, after atos_worker.cuh)

struct QBenchArgs {
    uint64_t *ring;
    uint64_t cap;
    Ctrl *ctrl;                 // head / tail / error lines of the benchmark queue
    uint32_t *popped;           // [n * rounds] or NULL
    int32_t worker, fetch, rounds, op, cas;
    uint64_t base;              // first index (tests start it just below 2^32)
};

enum QOp : int32_t { kQPush = 0, kQPop = 1, kQPushPop = 2 };

// Leader of a worker group: reserve `want` indices on *ctr (atomicAdd, or CAS).
__device__ __forceinline__ uint64_t qb_reserve(unsigned long long *ctr, uint64_t want, int cas) {
    if (!cas) return atomicAdd(ctr, (unsigned long long)want);
    unsigned long long o = *(volatile unsigned long long *)ctr, a;
    while ((a = atomicCAS(ctr, o, o + want)) != o) o = a;
    return o;
}

// The calling thread's index among the group's `gsz` threads gets index base+rank,
// where the group's leader reserved in chunks of `fetch` (ceil(gsz / fetch)
// atomics per round; each chunk is a separate reservation as in the worker).
__device__ __forceinline__ uint64_t qb_index(unsigned long long *ctr, const QBenchArgs &a, uint64_t *sh) {
    const int gsz = a.worker;
    const int rank = (int)(threadIdx.x % (unsigned)gsz);
    const int chunk = rank / a.fetch;
    const int nchunk = (gsz + a.fetch - 1) / a.fetch;
    if (gsz == 1) return qb_reserve(ctr, 1, a.cas);
    if (gsz == 32) {
        // warp worker: lane c (< nchunk) reserves chunk c, broadcast by shuffle
        const int lane = threadIdx.x & 31;
        uint64_t b = 0;
        if (lane < nchunk) b = qb_reserve(ctr, (uint64_t)min(a.fetch, gsz - lane * a.fetch), a.cas);
        b = __shfl_sync(0xffffffffu, b, chunk);
        return b + (uint64_t)(rank - chunk * a.fetch);
    }
    // CTA worker
    __syncthreads();
    if ((int)threadIdx.x < nchunk) sh[threadIdx.x] = qb_reserve(ctr, (uint64_t)min(a.fetch, gsz - (int)threadIdx.x * a.fetch), a.cas);
    __syncthreads();
    return sh[chunk] + (uint64_t)(rank - chunk * a.fetch);
}

__global__ void qbench_kernel(QBenchArgs a) {
    __shared__ uint64_t sh[kThreads];
    RankDev R{};
    R.ring = a.ring;
    R.ring_cap = a.cap;
    R.ctrl = a.ctrl;
    R.n_ranks = 1;
    const uint64_t gtid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int r = 0; r < a.rounds; ++r) {
        if (a.op == kQPush || a.op == kQPushPop) {
            const uint64_t idx = qb_index((unsigned long long *)&a.ctrl->tail.v, a, sh);
            ring_store(R, idx, (uint32_t)(gtid * (uint64_t)a.rounds + (uint64_t)r), a.base);   // the worker's push
        }
        if (a.op == kQPop || a.op == kQPushPop) {
            const uint64_t idx = qb_index((unsigned long long *)&a.ctrl->head.v, a, sh);
            uint64_t v;
            uint32_t spins = 0;
            while (!slot_full_for(v = ring_read(a.ring, a.cap, idx), idx)) {     // reserve-then-wait
                if (++spins > (1u << 26) || ld_relaxed_gpu(&a.ctrl->error.v)) { set_error(R, kErrTimeout); return; }
            }
            ring_release(a.ring, a.cap, idx);
            if (a.popped) a.popped[gtid * (uint64_t)a.rounds + (uint64_t)r] = lo32(v);
        }
    }
}

// Prepare the ring for indices starting at `base`: slot j free for the producer
// of the index idx in [base, base + cap) with idx = j (mod cap); with `prefill`
// items already published (item of index base + i is i).
__global__ void qbench_init_kernel(uint64_t *ring, uint64_t cap, uint64_t base, uint64_t prefill) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t idx = base + i;
        ring[idx & (cap - 1)] = i < prefill ? pack(lo32(idx + 1), (uint32_t)i) : pack(lo32(idx), 0u);
    }
}
