// atos_kernels.cuh -- the persistent Atos worker for sm_100a and its helper kernels.
//
// One CTA of 512 threads is one Atos "worker".
// The grid is persistent and co-resident (cooperative launch), one process per
// GPU; with virtual ranks, several ranks share one grid (blockIdx -> rank).
//
// Worker loop (Listing 3), per iteration:
//   1. claim one ready inbound packet from a peer channel and apply it
//      (owner-side atomicMin / atomicAdd, enqueue if improved / crossed)
//   2. else pop a batch of <= fetch vertices from the local ring
//      (reserve-then-wait, one leader atomic per worker)
//      and expand it with a CTA-wide load-balanced edge loop
//      (BFS: probe + atomicMin, Listing 5 PAPER.md:665-692;
//       PR: atomicAdd of alpha*r/outdeg with crossing enqueue)
//      - local discoveries go to a shared-memory staging buffer and are pushed
//        to the local ring with one atomic per flush (Listing 6 re-designed)
//      - remote discoveries become 8/16-byte messages in CTA-private staging and
//        are stored one-sided into the owner's channel over NVLink as packets,
//        flushed when full (size) or by age / at batch end (aggregation on/off,
//        PAPER.md:995-1065)
//   3. idle: termination detection (single rank: F == T; multi-rank:
//      coordinator double wave over per-rank counters), watchdog.
#pragma once
#include "atos_rt.cuh"

namespace atos {

constexpr int kApBfs = 0;
constexpr int kApPr = 1;
constexpr int kUnroll = 4;                      // edges per thread per round
constexpr int kRound = kThreads * kUnroll;      // edges per CTA round
constexpr int kOutCap = 2 * kRound;             // local push staging (u32 items)
constexpr int kHubWarps = 4;

template <int APP> struct AppTraits;
template <> struct AppTraits<kApBfs> { static constexpr int kMsgBytes = 8; };
template <> struct AppTraits<kApPr> { static constexpr int kMsgBytes = 16; };

struct Smem {
    RankDev R;
    uint32_t v[kThreads];          // batch: local vertex ids
    uint64_t val[kThreads];        // batch: depth (BFS) or delta bits (PR)
    int64_t beg[kThreads];         // batch: row begin (offset into col)
    int64_t off[kThreads + 1];     // batch: exclusive prefix of edge counts
    uint32_t out[kOutCap];         // local push staging
    int64_t wsum[kWarps];
    uint64_t res_lo, res_hi;       // outstanding ring reservation
    uint64_t b64[4];               // broadcast scratch
    uint32_t nout;                 // items in out[]
    int32_t minbad;
    int32_t flag;
    int32_t b32[4];
    uint32_t stail[kMaxRanks], shead[kMaxRanks];  // CTA staging ring per destination
    uint64_t st0[kMaxRanks];       // time the destination's staging became non-empty
    uint64_t staged_reported;
    uint64_t now;
    // coordinator double wave
    uint64_t wave[kMaxRanks][5];
    int32_t wave_valid;
    // per-CTA statistics
    unsigned long long c_pops, c_edges, c_pushes, c_msgs, c_packets, c_idle, c_hub;
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__device__ __forceinline__ void set_error(const RankDev &R, uint64_t code) {
    atomicCAS((unsigned long long *)&R.ctrl->error.v, 0ull, (unsigned long long)code);
}

__device__ __forceinline__ int owner_of(const Smem &s, int64_t u) {
    int r = 0;
#pragma unroll
    for (int k = 1; k < kMaxRanks; ++k)
        r += (k < s.R.n_ranks && s.R.part[k] <= u) ? 1 : 0;
    return r;
}

// Block-wide exclusive scan of one int64 per thread; returns the total.
__device__ __forceinline__ int64_t block_exscan(Smem &s, int64_t x, int64_t &excl) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t incl = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
        if (lane >= d) incl += y;
    }
    if (lane == 31) s.wsum[w] = incl;
    __syncthreads();
    if (w == 0) {
        int64_t t = lane < kWarps ? s.wsum[lane] : 0;
        int64_t ti = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int64_t y = __shfl_up_sync(0xffffffffu, ti, d);
            if (lane >= d) ti += y;
        }
        if (lane < kWarps) s.wsum[lane] = ti - t;   // exclusive warp offsets
        if (lane == kWarps - 1) s.b64[3] = (uint64_t)ti;
    }
    __syncthreads();
    excl = incl - x + s.wsum[w];
    int64_t total = (int64_t)s.b64[3];
    __syncthreads();
    return total;
}

// ---------------------------------------------------------------------------
// local ring push
// ---------------------------------------------------------------------------
// Single-item push from one thread (overflow path; rare).
__device__ void ring_push_one(const Smem &s, uint32_t item) {
    const RankDev &R = s.R;
    uint64_t idx = atomicAdd((unsigned long long *)&R.ctrl->tail.v, 1ull);
    uint64_t *p = &R.ring[idx & (R.ring_cap - 1)];
    uint32_t spins = 0;
    while (!slot_free_for(ld_relaxed_gpu(p), idx)) {
        if (++spins > (1u << 26)) { set_error(R, kErrCapacity); return; }
        __nanosleep(64);
    }
    fence_acq_rel_gpu();
    st_relaxed_gpu(p, pack(lo32(idx + 1), item));
}

// Push s.out[0..nout) with one leader atomic; whole CTA participates.
__device__ void ring_flush(Smem &s) {
    __syncthreads();
    const uint32_t cnt = s.nout;
    if (cnt == 0) return;
    const RankDev &R = s.R;
    if (threadIdx.x == 0) s.b64[0] = atomicAdd((unsigned long long *)&R.ctrl->tail.v, (unsigned long long)cnt);
    __syncthreads();
    const uint64_t base = s.b64[0];
    // release: the state updates (atomicMin / atomicAdd) made by this CTA before
    // the barrier must be visible before the item is (consumer reads depth[v]).
    fence_acq_rel_gpu();
    for (uint32_t i = threadIdx.x; i < cnt; i += kThreads) {
        const uint64_t idx = base + i;
        uint64_t *p = &R.ring[idx & (R.ring_cap - 1)];
        uint32_t spins = 0;
        while (!slot_free_for(ld_relaxed_gpu(p), idx)) {
            if (++spins > (1u << 26)) { set_error(R, kErrCapacity); break; }
            __nanosleep(64);
        }
        st_relaxed_gpu(p, pack(lo32(idx + 1), s.out[i]));
    }
    if (threadIdx.x == 0) { s.c_pushes += cnt; s.nout = 0; }
    __syncthreads();
}

// Append one local item to the CTA staging buffer (warp-aggregated smem atomic).
__device__ __forceinline__ void produce_local(Smem &s, uint32_t item) {
    const uint32_t m = __activemask();
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(m) - 1;
    const uint32_t rank = __popc(m & lanemask_lt());
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(&s.nout, (uint32_t)__popc(m));
    base = __shfl_sync(m, base, leader);
    const uint32_t pos = base + rank;
    if (pos < (uint32_t)kOutCap) s.out[pos] = item;
    else ring_push_one(s, item);   // overflow: direct push (never loses work)
}

// ---------------------------------------------------------------------------
// remote messages: CTA-private staging ring per destination, packets over NVLink
// ---------------------------------------------------------------------------
template <int APP>
__device__ __forceinline__ unsigned char *stage_base(const Smem &s, const KParams &kp, int cta, int dst) {
    const size_t slot = ((size_t)cta * kMaxRanks + dst) * (size_t)kp.stage_cap;
    return s.R.staging + slot * AppTraits<APP>::kMsgBytes;
}

template <int APP>
__device__ __forceinline__ void produce_remote(Smem &s, const KParams &kp, int cta, int dst,
                                               uint32_t v_local, uint64_t payload) {
    const uint32_t m = __activemask();
    const uint32_t grp = __match_any_sync(m, dst);
    const int lane = threadIdx.x & 31;
    const int leader = __ffs(grp) - 1;
    const uint32_t rank = __popc(grp & lanemask_lt());
    uint32_t base = 0;
    if (lane == leader) {
        base = atomicAdd(&s.stail[dst], (uint32_t)__popc(grp));
        if (base == s.shead[dst]) s.st0[dst] = globaltimer();   // staging became non-empty
    }
    base = __shfl_sync(grp, base, leader);
    const uint32_t pos = (base + rank) & (uint32_t)(kp.stage_cap - 1);
    unsigned char *b = stage_base<APP>(s, kp, cta, dst);
    if constexpr (APP == kApBfs) {
        ((uint64_t *)b)[pos] = pack((uint32_t)payload, v_local);
    } else {
        ((uint4 *)b)[pos] = make_uint4(v_local, 0u, (uint32_t)payload, (uint32_t)(payload >> 32));
    }
}

template <int APP> __device__ bool inbound_step(Smem &s, const KParams &kp, int cta);

// Send one packet of `cnt` staged messages to dst (whole CTA).  Returns false on error.
template <int APP>
__device__ bool send_packet(Smem &s, const KParams &kp, int cta, int dst, uint32_t cnt) {
    const RankDev &R = s.R;
    const uint32_t cp = (uint32_t)kp.cp;
    if (threadIdx.x == 0) {
        s.b64[1] = atomicAdd((unsigned long long *)&R.ctrl->out_reserve[dst].v, 1ull);
        s.flag = 0;
    }
    __syncthreads();
    const uint64_t pidx = s.b64[1];
    const uint32_t slot = (uint32_t)(pidx & (cp - 1));
    // wait until the receiver has released this packet slot; meanwhile keep
    // consuming inbound packets (which never produce remote sends) so that two
    // ranks with full channels cannot deadlock.
    uint64_t t_begin = 0;
    for (;;) {
        if (threadIdx.x == 0) {
            const uint64_t f = ld_acquire_sys(&R.free_mirror[dst][slot]);
            s.b32[0] = slot_free_for(pack(lo32(f), 0), pidx) ? 1 : 0;
            if (!s.b32[0]) {
                const uint64_t now = globaltimer();
                if (t_begin == 0) t_begin = now;
                if (ld_relaxed_gpu(&R.ctrl->error.v) != 0 ||
                    (now - t_begin) > 2000000000ull) {   // 2 s without a free slot
                    set_error(R, kErrCapacity);
                    s.b32[0] = 2;
                }
            }
        }
        __syncthreads();
        const int st = s.b32[0];
        __syncthreads();
        if (st == 1) break;
        if (st == 2) return false;
        inbound_step<APP>(s, kp, cta);
    }
    // payload: coalesced one-sided stores into dst's HBM over NVLink
    const unsigned char *src = stage_base<APP>(s, kp, cta, dst);
    const uint32_t h = s.shead[dst];
    const uint32_t mask = (uint32_t)(kp.stage_cap - 1);
    unsigned char *dpay = R.out_payload[dst] + (size_t)slot * kp.pkt * AppTraits<APP>::kMsgBytes;
    for (uint32_t i = threadIdx.x; i < cnt; i += kThreads) {
        const uint32_t q = (h + i) & mask;
        if constexpr (APP == kApBfs) {
            ((uint64_t *)dpay)[i] = ((const uint64_t *)src)[q];
        } else {
            ((uint4 *)dpay)[i] = ((const uint4 *)src)[q];
        }
    }
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd((unsigned long long *)&R.ctrl->sent.v, (unsigned long long)cnt);  // S before publish
        fence_acq_rel_sys();
        st_release_sys(&R.out_hdr[dst][slot], pack(lo32(pidx + 1), cnt));
        s.shead[dst] = h + cnt;
        if (s.shead[dst] == s.stail[dst]) s.st0[dst] = 0;
        s.c_msgs += cnt;
        s.c_packets += 1;
    }
    __syncthreads();
    return true;
}

// Flush staged messages: full packets always; partial ones when `force`, or
// when aggregation is off, or when the oldest staged message is older than
// agg_age_ns (the paper's BATCH_SIZE / WAIT_TIME triggers).
template <int APP>
__device__ void remote_flush(Smem &s, const KParams &kp, int cta, bool batch_end) {
    if (s.R.n_ranks <= 1) return;
    if (threadIdx.x == 0) s.now = globaltimer();
    __syncthreads();
    const uint64_t now = s.now;
    for (int d = 0; d < s.R.n_ranks; ++d) {
        if (d == s.R.rank) continue;
        for (;;) {
            const uint32_t pending = s.stail[d] - s.shead[d];
            if (pending == 0) break;
            bool go = pending >= (uint32_t)kp.pkt;
            if (!go && batch_end) {
                go = !kp.agg_on || (s.st0[d] != 0 && now - s.st0[d] >= (uint64_t)kp.agg_age_ns);
            }
            if (!go) break;
            const uint32_t cnt = pending < (uint32_t)kp.pkt ? pending : (uint32_t)kp.pkt;
            if (!send_packet<APP>(s, kp, cta, d, cnt)) return;
        }
    }
}

// Report this CTA's staged-message count change to the rank counter.
__device__ void report_staged(Smem &s) {
    if (s.R.n_ranks <= 1) return;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t cur = 0;
        for (int d = 0; d < s.R.n_ranks; ++d) cur += (uint64_t)(s.stail[d] - s.shead[d]);
        const uint64_t delta = cur - s.staged_reported;   // mod 2^64
        if (delta != 0) {
            fence_acq_rel_sys();
            atomicAdd((unsigned long long *)&s.R.ctrl->staged.v, (unsigned long long)delta);
            s.staged_reported = cur;
        }
    }
    __syncthreads();
}

// ---------------------------------------------------------------------------
// edge relaxation
// ---------------------------------------------------------------------------
template <int APP>
__device__ __forceinline__ void relax_remote(Smem &s, const KParams &kp, int cta, int64_t u, uint64_t payload) {
    const int d = owner_of(s, u);
    produce_remote<APP>(s, kp, cta, d, (uint32_t)(u - s.R.part[d]), payload);
}

// Expand the batch in smem (B vertices, E edges) with a load-balanced edge loop.
template <int APP>
__device__ void expand(Smem &s, const KParams &kp, int cta, int B, int64_t E) {
    const RankDev &R = s.R;
    const int tid = threadIdx.x;
    const int64_t vb = R.v_begin, ve = R.v_end;
    int j = 0;
    for (int64_t base = 0; base < E; base += kRound) {
        int32_t u[kUnroll];
        uint64_t val[kUnroll];
#pragma unroll
        for (int k = 0; k < kUnroll; ++k) {
            const int64_t e = base + (int64_t)k * kThreads + tid;
            u[k] = -1;
            if (e < E) {
                if (s.off[j + 1] <= e) {           // monotone search: off[j] <= e < off[j+1]
                    int lo = j + 1, hi = B - 1;
                    while (lo < hi) {
                        const int mid = (lo + hi + 1) >> 1;
                        if (s.off[mid] <= e) lo = mid; else hi = mid - 1;
                    }
                    j = lo;
                }
                u[k] = __ldg(R.col + s.beg[j] + (e - s.off[j]));   // coalesced within a row
                val[k] = s.val[j];
            }
        }
        if constexpr (APP == kApBfs) {
            uint32_t cur[kUnroll];
#pragma unroll
            for (int k = 0; k < kUnroll; ++k)
                cur[k] = (u[k] >= 0) ? R.depth[u[k]] : 0u;   // probe (stale = larger: safe)
#pragma unroll
            for (int k = 0; k < kUnroll; ++k) {
                const uint32_t nd = (uint32_t)val[k] + 1u;
                if (u[k] >= 0 && nd < cur[k]) {
                    const uint32_t old = atomicMin(R.depth + u[k], nd);
                    if (old > nd) {
                        if (u[k] >= vb && u[k] < ve) produce_local(s, (uint32_t)(u[k] - vb));
                        else relax_remote<APP>(s, kp, cta, u[k], nd);
                    }
                }
            }
        } else {
            const double eps = kp.eps;
#pragma unroll
            for (int k = 0; k < kUnroll; ++k) {
                if (u[k] < 0) continue;
                const double dlt = __longlong_as_double((long long)val[k]);
                if (u[k] >= vb && u[k] < ve) {
                    const uint32_t ul = (uint32_t)(u[k] - vb);
                    const double old = atomicAdd(R.pr_res + ul, dlt);
                    if (old < eps && old + dlt >= eps) produce_local(s, ul);   // crossing (R5)
                } else {
                    relax_remote<APP>(s, kp, cta, u[k], (uint64_t)__double_as_longlong(dlt));
                }
            }
        }
        __syncthreads();
        if (s.nout > (uint32_t)(kOutCap - kRound)) ring_flush(s);
        if (R.n_ranks > 1) {
            bool need = false;
            for (int d = 0; d < R.n_ranks; ++d)
                need |= (s.stail[d] - s.shead[d]) + (uint32_t)kRound > (uint32_t)kp.stage_cap - (uint32_t)kp.pkt;
            if (need) remote_flush<APP>(s, kp, cta, false);
        }
    }
    if (tid == 0) s.c_edges += (unsigned long long)E;
}

// Load per-vertex info of the popped batch s.v[0..B) and expand it.
template <int APP>
__device__ void process_batch(Smem &s, const KParams &kp, int cta, int B) {
    const RankDev &R = s.R;
    const int tid = threadIdx.x;
    int64_t deg = 0;
    if (tid < B) {
        const uint32_t v = s.v[tid];
        const int64_t b = R.row_ptr[v], e = R.row_ptr[v + 1];
        s.beg[tid] = b;
        deg = e - b;
        if constexpr (APP == kApBfs) {
            const uint32_t d = ld_relaxed_gpu_u32(R.depth + R.v_begin + v);
            s.val[tid] = d;
            if (d == kInf) deg = 0;
        } else {
            const double r = __longlong_as_double(
                (long long)atomicExch((unsigned long long *)(R.pr_res + v), 0ull));
            if (r != 0.0) atomicAdd(R.pr_rank + v, r);
            if (r == 0.0 || deg == 0) deg = 0;        // dangling vertices absorb (R4)
            else s.val[tid] = (uint64_t)__double_as_longlong(kp.alpha * r / (double)deg);
        }
    }
    int64_t excl;
    const int64_t E = block_exscan(s, deg, excl);
    if (tid < B) s.off[tid] = excl;
    if (tid == 0) s.off[B] = E;
    __syncthreads();
    if (E > 0) expand<APP>(s, kp, cta, B, E);
}

// ---------------------------------------------------------------------------
// pop from the local ring: reserve-then-wait
// ---------------------------------------------------------------------------
__device__ int pop_batch(Smem &s, const KParams &kp) {
    const RankDev &R = s.R;
    const int tid = threadIdx.x;
    if (tid == 0) {
        if (s.res_lo == s.res_hi) {
            const uint64_t t = ld_relaxed_gpu(&R.ctrl->tail.v);
            const uint64_t h = ld_relaxed_gpu(&R.ctrl->head.v);
            if (t > h) {
                uint64_t k = (t - h) / (uint64_t)kp.ctas_per_rank;
                k = k < 1 ? 1 : (k > (uint64_t)kp.fetch ? (uint64_t)kp.fetch : k);
                const uint64_t lo = atomicAdd((unsigned long long *)&R.ctrl->head.v, (unsigned long long)k);
                s.res_lo = lo;
                s.res_hi = lo + k;
            }
        }
        s.minbad = kThreads;
    }
    __syncthreads();
    const uint64_t lo = s.res_lo;
    const uint64_t avail = s.res_hi - lo;
    const int cnt = (int)(avail < (uint64_t)kp.fetch ? avail : (uint64_t)kp.fetch);
    uint64_t idx = lo + tid;
    uint64_t slot = 0;
    bool ready = false;
    if (tid < cnt) {
        slot = ld_relaxed_gpu(&R.ring[idx & (R.ring_cap - 1)]);
        ready = slot_full_for(slot, idx);
        if (!ready) atomicMin(&s.minbad, tid);
    }
    __syncthreads();
    const int B = cnt < s.minbad ? cnt : s.minbad;
    if (tid < B) {
        fence_acq_rel_gpu();   // acquire: see the producer's state update of this vertex
        s.v[tid] = lo32(slot);
        st_relaxed_gpu(&R.ring[idx & (R.ring_cap - 1)], pack(lo32(idx + R.ring_cap), 0u));
    }
    __syncthreads();
    if (tid == 0) s.res_lo = lo + (uint64_t)B;
    return B;
}

// ---------------------------------------------------------------------------
// inbound packets (owner-side receive)
// ---------------------------------------------------------------------------
template <int APP>
__device__ bool inbound_step(Smem &s, const KParams &kp, int cta) {
    const RankDev &R = s.R;
    if (R.n_ranks <= 1) return false;
    const uint32_t cp = (uint32_t)kp.cp;
    if (threadIdx.x == 0) {
        s.b32[1] = -1;
        const int p = R.n_ranks;
        const int start = (cta + (int)(s.c_idle & 7)) % p;
        for (int k = 0; k < p; ++k) {
            const int src = (start + k) % p;
            if (src == R.rank) continue;
            unsigned long long *cur = (unsigned long long *)&R.ctrl->in_cursor[src].v;
            const uint64_t c = ld_relaxed_gpu((const uint64_t *)cur);
            const uint64_t h = ld_acquire_sys(&R.in_hdr[src][c & (cp - 1)]);
            if (hi32(h) == lo32(c + 1) && atomicCAS(cur, c, c + 1) == c) {
                s.b32[1] = src;
                s.b32[2] = (int32_t)lo32(h);
                s.b64[2] = c;
                break;
            }
        }
    }
    __syncthreads();
    const int src = s.b32[1];
    if (src < 0) return false;
    const uint32_t cnt = (uint32_t)s.b32[2];
    const uint64_t c = s.b64[2];
    const uint32_t slot = (uint32_t)(c & (cp - 1));
    const unsigned char *pay = R.in_payload[src] + (size_t)slot * kp.pkt * AppTraits<APP>::kMsgBytes;
    for (uint32_t i = threadIdx.x; i < cnt; i += kThreads) {
        if constexpr (APP == kApBfs) {
            const uint64_t m = ld_cg_u64((const uint64_t *)pay + i);
            const uint32_t ul = lo32(m), nd = hi32(m);
            const uint32_t old = atomicMin(R.depth + R.v_begin + ul, nd);
            if (old > nd) produce_local(s, ul);
        } else {
            const uint4 m = ld_cg_u4((const uint4 *)pay + i);
            const double dlt = __longlong_as_double((long long)(((uint64_t)m.w << 32) | m.z));
            const double old = atomicAdd(R.pr_res + m.x, dlt);
            if (old < kp.eps && old + dlt >= kp.eps) produce_local(s, m.x);
        }
    }
    ring_flush(s);                     // T counts the new local work first
    if (threadIdx.x == 0) {
        // release the packet slot to the sender (after all payload reads; barrier above)
        st_release_sys(&R.peer_free[src][slot], c + cp);
        fence_acq_rel_sys();
        atomicAdd((unsigned long long *)&R.ctrl->recvd.v, (unsigned long long)cnt);   // R after effects
    }
    __syncthreads();
    return true;
}

// ---------------------------------------------------------------------------
// termination
// ---------------------------------------------------------------------------
// Multi-rank coordinator (rank 0, CTA 0): double wave over every rank's
// (F, R, T, staged, S); declare done when two consecutive waves are identical,
// every rank is passive (F == T, staged == 0) and sum S == sum R.
__device__ void coordinator_step(Smem &s, const KParams &kp) {
    const RankDev &R = s.R;
    if (threadIdx.x >= 32) return;
    const int lane = threadIdx.x;
    const int p = R.n_ranks;
    bool started = true;
    uint64_t F = 0, Rv = 0, T = 0, St = 0, S = 0;
    if (lane < p) {
        started = ld_acquire_sys(&R.ctrl->started[lane].v) == kp.epoch;
        const Ctrl *c = R.peer_ctrl[lane];
        F = ld_acquire_sys(&c->finished.v);
        Rv = ld_acquire_sys(&c->recvd.v);
        T = ld_acquire_sys(&c->tail.v);
        St = ld_acquire_sys(&c->staged.v);
        S = ld_acquire_sys(&c->sent.v);
    }
    const bool all_started = __all_sync(0xffffffffu, started);
    if (!all_started) {
        if (lane == 0) s.wave_valid = 0;
        __syncwarp();
        return;
    }
    bool same = true, passive = true;
    if (lane < p) {
        same = s.wave_valid && s.wave[lane][0] == F && s.wave[lane][1] == Rv && s.wave[lane][2] == T &&
               s.wave[lane][3] == St && s.wave[lane][4] == S;
        passive = (F == T) && (St == 0);
    }
    uint64_t sumS = S, sumR = Rv;
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) {
        sumS += __shfl_xor_sync(0xffffffffu, sumS, d);
        sumR += __shfl_xor_sync(0xffffffffu, sumR, d);
    }
    const bool all_same = __all_sync(0xffffffffu, same);
    const bool all_passive = __all_sync(0xffffffffu, passive);
    __syncwarp();
    if (lane < p) {
        s.wave[lane][0] = F; s.wave[lane][1] = Rv; s.wave[lane][2] = T;
        s.wave[lane][3] = St; s.wave[lane][4] = S;
    }
    if (lane == 0) {
        s.wave_valid = all_passive && sumS == sumR;
    }
    if (all_same && all_passive && sumS == sumR) {
        if (lane < p) st_release_sys(&R.peer_ctrl[lane]->done.v, kp.epoch);
    }
    if (lane == 0) atomicAdd((unsigned long long *)&R.ctrl->st_waves.v, 1ull);
    __syncwarp();
}

// ---------------------------------------------------------------------------
// the persistent worker
// ---------------------------------------------------------------------------
template <int APP>
__global__ void __launch_bounds__(kThreads, 2) worker_kernel(KParams kp) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem &s = *reinterpret_cast<Smem *>(smem_raw);
    const int lr = blockIdx.x / kp.ctas_per_rank;
    const int cta = blockIdx.x % kp.ctas_per_rank;
    const int tid = threadIdx.x;
    if (tid == 0) {
        s.R = kp.ranks[lr];
        s.nout = 0;
        s.res_lo = s.res_hi = 0;
        s.staged_reported = 0;
        s.wave_valid = 0;
        s.c_pops = s.c_edges = s.c_pushes = s.c_msgs = s.c_packets = s.c_idle = s.c_hub = 0;
        for (int d = 0; d < kMaxRanks; ++d) { s.stail[d] = s.shead[d] = 0; s.st0[d] = 0; }
    }
    __syncthreads();
    const bool multi = s.R.n_ranks > 1;
    const bool coordinator = multi && s.R.rank == 0 && cta == 0;
    if (tid == 0 && cta == 0) st_release_sys(&s.R.peer_ctrl[0]->started[s.R.rank].v, kp.epoch);
    const uint64_t t_start = globaltimer();
    uint32_t idle_streak = 0;

    for (;;) {
        if (tid == 0) {
            int f = 0;
            if (ld_relaxed_gpu(&s.R.ctrl->done.v) == kp.epoch) f = 1;
            if (ld_relaxed_gpu(&s.R.ctrl->error.v) != 0) f = 2;
            s.flag = f;
        }
        __syncthreads();
        if (s.flag) break;
        __syncthreads();

        bool worked = false;
        if (multi) worked = inbound_step<APP>(s, kp, cta);
        if (!worked) {
            const int B = pop_batch(s, kp);
            if (B > 0) {
                if (tid == 0) s.c_pops += B;
                process_batch<APP>(s, kp, cta, B);
                ring_flush(s);
                remote_flush<APP>(s, kp, cta, true);
                report_staged(s);
                if (tid == 0) {
                    if (multi) fence_acq_rel_sys(); else fence_acq_rel_gpu();
                    atomicAdd((unsigned long long *)&s.R.ctrl->finished.v, (unsigned long long)B);  // F last
                }
                worked = true;
            }
        }
        if (worked) { idle_streak = 0; continue; }

        // ---- idle: flush aged staging, detect termination, watchdog
        ++idle_streak;
        if (multi) {
            remote_flush<APP>(s, kp, cta, true);
            report_staged(s);
        }
        if (tid == 0) {
            s.c_idle++;
            if (!multi) {
                const uint64_t F = ld_acquire_gpu(&s.R.ctrl->finished.v);
                const uint64_t T = ld_acquire_gpu(&s.R.ctrl->tail.v);
                if (F == T) st_release_gpu(&s.R.ctrl->done.v, kp.epoch);
            }
            if (kp.watchdog_ns > 0 && globaltimer() - t_start > (uint64_t)kp.watchdog_ns)
                set_error(s.R, kErrTimeout);
        }
        if (coordinator) coordinator_step(s, kp);
        if (idle_streak > 4) __nanosleep(idle_streak > 64 ? 256 : 32);
    }
    __syncthreads();
    if (tid == 0) {
        Ctrl *c = s.R.ctrl;
        atomicAdd((unsigned long long *)&c->st_pops.v, s.c_pops);
        atomicAdd((unsigned long long *)&c->st_edges.v, s.c_edges);
        atomicAdd((unsigned long long *)&c->st_pushes.v, s.c_pushes);
        atomicAdd((unsigned long long *)&c->st_msgs.v, s.c_msgs);
        atomicAdd((unsigned long long *)&c->st_packets.v, s.c_packets);
        atomicAdd((unsigned long long *)&c->st_idle.v, s.c_idle);
        atomicAdd((unsigned long long *)&c->st_hub_chunks.v, s.c_hub);
    }
}

// ---------------------------------------------------------------------------
// helper kernels (setup / teardown of one solve)
// ---------------------------------------------------------------------------
// Cross-rank barrier: rank r writes `value` into every rank's bar[r] and waits
// until its own bar[*] all equal `value`.  One CTA.
__global__ void barrier_kernel(KParams kp, uint64_t value) {
    if (threadIdx.x != 0) return;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        for (int d = 0; d < R.n_ranks; ++d) st_release_sys(&R.peer_ctrl[d]->bar[R.rank].v, value);
    }
    const uint64_t t0 = globaltimer();
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        for (int d = 0; d < R.n_ranks; ++d) {
            while (ld_acquire_sys(&R.ctrl->bar[d].v) < value) {
                if (kp.watchdog_ns > 0 && globaltimer() - t0 > (uint64_t)kp.watchdog_ns) {
                    set_error(R, kErrTimeout);
                    return;
                }
                __nanosleep(128);
            }
        }
    }
}

__global__ void init_bfs_kernel(KParams kp) {
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        const int64_t n = R.n;
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
            R.depth[i] = kInf;
        if (blockIdx.x == 0 && threadIdx.x == 0) R.ctrl->error.v = 0;
    }
}

// Seed: owner of src sets depth[src] = 0 and enqueues it.  One thread.
__global__ void seed_bfs_kernel(KParams kp, int64_t src) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        if (src < R.v_begin || src >= R.v_end) continue;
        R.depth[src] = 0;
        const uint64_t idx = R.ctrl->tail.v;
        uint64_t *p = &R.ring[idx & (R.ring_cap - 1)];
        if (!slot_free_for(*p, idx)) { R.ctrl->error.v = kErrCapacity; return; }
        __threadfence();
        *p = pack(lo32(idx + 1), (uint32_t)(src - R.v_begin));
        __threadfence();
        R.ctrl->tail.v = idx + 1;
    }
}

// PR init: rank = 0, res = 1 - alpha, every owned vertex enqueued.
__global__ void init_pr_kernel(KParams kp) {
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        const int64_t nr = R.v_end - R.v_begin;
        const uint64_t base = R.ctrl->tail.v;     // not modified by this kernel
        const double r0 = 1.0 - kp.alpha;
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nr; i += (int64_t)gridDim.x * blockDim.x) {
            R.pr_rank[i] = 0.0;
            R.pr_res[i] = r0;
            const uint64_t idx = base + (uint64_t)i;
            R.ring[idx & (R.ring_cap - 1)] = pack(lo32(idx + 1), (uint32_t)i);
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) R.ctrl->error.v = 0;
    }
}

__global__ void bump_tail_kernel(KParams kp) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        R.ctrl->tail.v += (uint64_t)(R.v_end - R.v_begin);
    }
}

// After a solve: reservations that overshot the tail are retired so that the
// ring stays consistent for the next solve (slots marked consumed; T and F
// advanced by the same amount).  One CTA.
__global__ void fixup_kernel(KParams kp) {
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        const uint64_t h = R.ctrl->head.v, t = R.ctrl->tail.v;
        if (h > t) {
            for (uint64_t idx = t + threadIdx.x; idx < h; idx += blockDim.x)
                R.ring[idx & (R.ring_cap - 1)] = pack(lo32(idx + R.ring_cap), 0u);
        }
        __syncthreads();
        if (threadIdx.x == 0 && h > t) {
            R.ctrl->tail.v = h;
            R.ctrl->finished.v += h - t;
        }
        __syncthreads();
    }
}

// Gather owned results of every rank into full-size outputs (peer loads over NVLink).
__global__ void gather_bfs_kernel(KParams kp, int32_t *out) {
    const RankDev &R = kp.ranks[0];
    const int64_t n = R.n;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int o = 0;
        for (int k = 1; k < R.n_ranks; ++k) o += R.part[k] <= v ? 1 : 0;
        const uint32_t d = __ldcg(R.peer_depth[o] + v);
        out[v] = d == kInf ? -1 : (int32_t)d;
    }
}

__global__ void gather_pr_kernel(KParams kp, double *rank_out, double *res_out) {
    const RankDev &R = kp.ranks[0];
    const int64_t n = R.n;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int o = 0;
        for (int k = 1; k < R.n_ranks; ++k) o += R.part[k] <= v ? 1 : 0;
        const int64_t i = v - R.part[o];
        if (rank_out) rank_out[v] = __ldcg(R.peer_rank[o] + i);
        if (res_out) res_out[v] = __ldcg(R.peer_res[o] + i);
    }
}

// Min-id BFS parent: each rank scans its own rows u and
// atomicMins u into parent[v] for every edge u->v with depth(v) = depth(u)+1.
// depth_full = gathered depth (int32, -1 unreached), parent_acc = full-size int64.
__global__ void parent_init_kernel(int64_t *parent_acc, int64_t n) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        parent_acc[v] = INT64_MAX;
}

__global__ void parent_scan_kernel(KParams kp, const int32_t *depth_full, int64_t *parent_acc) {
    // one warp per owned row
    const int lane = threadIdx.x & 31;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        const int64_t nr = R.v_end - R.v_begin;
        for (int64_t i = warp; i < nr; i += nwarps) {
            const int64_t u = R.v_begin + i;
            const int32_t du = depth_full[u];
            if (du < 0) continue;
            for (int64_t e = R.row_ptr[i] + lane; e < R.row_ptr[i + 1]; e += 32) {
                const int32_t v = R.col[e];
                if (depth_full[v] == du + 1) atomicMin((long long *)(parent_acc + v), (long long)u);
            }
        }
    }
}

__global__ void parent_final_kernel(const int32_t *depth_full, int64_t *const *accs, int n_acc, int64_t n,
                                    int64_t src, int64_t *parent_out) {
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int64_t p = INT64_MAX;
        for (int k = 0; k < n_acc; ++k) {
            const int64_t q = __ldcg((const long long *)(accs[k] + v));
            p = q < p ? q : p;
        }
        if (depth_full[v] < 0) p = -1;
        else if (v == src) p = src;
        parent_out[v] = p;
    }
}

}  // namespace atos
