// atos_worker.cuh -- the persistent Atos worker for sm_100a.
//
// One CTA of 512 threads is one Atos "worker".
// The grid is persistent and co-resident (cooperative launch), one process per
// GPU; with virtual ranks, several ranks share one grid (blockIdx -> rank).
//
// Worker loop (Listing 3):
//   1. every warp tries to claim one ready inbound packet from a peer channel
//      and applies it (owner-side atomicMin / atomicAdd; enqueue if improved /
//      crossed)
//   2. otherwise the CTA pops a batch of <= fetch vertices from the local ring
//      (reserve-then-wait, one leader atomic per worker) and
//      expands it: the batch's edge space is cut into 256-edge chunks that the
//      16 warps process independently (no block barrier inside the edge loop),
//      8 edges per lane in flight:
//        BFS (Listing 5): probe depth[u], atomicMin if it
//          would improve, enqueue u if it did;
//        PR: atomicAdd alpha*r/outdeg into res[u],
//          enqueue on the crossing old < eps <= old+delta.
//      Local discoveries go to per-warp shared-memory staging; remote ones to
//      per-warp message staging that warps publish to the owner's channel as
//      packets with one-sided stores over NVLink (aggregation by size / age,
//      PAPER.md:995-1065).  At batch end the CTA enqueues its discoveries with
//      one leader atomic, or keeps up to `keep` of them as its next batch
//      (work-keeping chain: on latency-bound, high-diameter graphs a worker
//      follows its own discoveries without a queue round trip per level).
//   3. idle: flush aged staging, termination detection (single rank: F == T;
//      multi-rank: coordinator double wave), watchdog.
#pragma once
#include "atos_rt.cuh"

namespace atos {

#ifndef ATOS_MINB
#define ATOS_MINB (1024 / ATOS_THREADS)
#endif
constexpr int kMinBlocks = ATOS_MINB;   // resident CTAs per SM the register budget is sized for
constexpr int kApBfs = 0;
constexpr int kApPr = 1;
#ifndef ATOS_KU
#define ATOS_KU 4
#endif
constexpr int kU = ATOS_KU;          // edges per lane in flight
constexpr int kChunk = 32 * kU;      // edges per warp chunk
#ifndef ATOS_WOUT
#define ATOS_WOUT 128
#endif
constexpr int kWOut = ATOS_WOUT;     // per-warp local staging (items)
constexpr int kChunkMap = 1024;      // chunks whose first vertex is precomputed per batch
constexpr uint32_t kFull = 0xffffffffu;

// BFS row pieces.  A popped row longer than
// 2 x kp.split edges is cut: the popping worker expands the first kp.split edges
// and publishes the rest as ring items {1 | piece:15 | v:16} that any worker can
// pop, so a hub's adjacency list is scanned by many CTAs at once instead of
// serialising one of them.  Only ids < 2^16 of a rank block can be split -- after
// degree relabeling these are the block's highest-degree vertices.
constexpr uint32_t kPieceBit = 0x80000000u;
constexpr int64_t kPieceVMax = 1 << 16;
constexpr int64_t kPieceMax = 1 << 15;
constexpr int kKeepAuto = 128;       // work keeping on non-skewed graphs: measured best of 16..512 on the grid
constexpr int kSplitAuto = 1024;        // measured best of 512..8192 on RMAT-24/26

// PageRank sender-side residual combining (atos_config.pr_combine).
// A delta for a remote vertex u is added to this rank's ghost residual g[u]; the
// add that crosses eps_g (the local crossing rule R5 applied to g) exchanges g[u]
// with 0 and sends the accumulated value as one message.  Deltas below eps_g are
// thereby combined; quiescence leaves every g[u] < eps_g.

template <int APP> struct AppTraits;
template <> struct AppTraits<kApBfs> { static constexpr int kMsgBytes = 8; };
template <> struct AppTraits<kApPr> { static constexpr int kMsgBytes = 16; };

// One popped batch, set up for expansion.
// Edge -> vertex map of a batch with E <= kBitE edges (DESIGN.md 5.1 "edge map"):
// bit e of bm marks the first edge of a non-empty row, rowmap[w] is the (compacted)
// row holding edge 32w, nzslot[] maps compacted rows to batch slots.  A lane's row
// is then rowmap[w] + popc(bm[w] & lanes (0, lane]) -- one word per 32 edges
// instead of a per-lane binary search over the batch offsets.
constexpr int kBitW = 1024;
constexpr int64_t kBitE = (int64_t)kBitW * 32;

// One row of a popped batch in the single-rank BFS expansion (atos_bfs1.cuh).
struct alignas(16) BRec {
    int64_t base;    // short row: beg - (row's offset in the packed short edge space); long row: beg
    uint32_t nd;     // candidate depth of the row's targets (popped depth + 1)
    uint32_t len;    // long row: edges in the row (piece); short row: unused
};
constexpr int kLong = 64;            // rows of >= kLong edges are expanded as aligned chunks of kLongG x kCh1 edges
// (a batch's short rows -- up to kThreads rows of < kLong edges -- must fit the per-batch edge map
// of kBitW x 32 edges; kLong = 128 measured RMAT-24 2.425 -> 2.395 ms but overflows it)
static_assert((int64_t)(kLong - 1) * kThreads <= kBitE, "short rows of a batch must fit the edge map");
constexpr int kCh1 = 128;            // edges per warp chunk in atos_bfs1.cuh (32 lanes x 4)
#ifndef ATOS_LONGG
#define ATOS_LONGG 1
#endif
constexpr int kLongG = ATOS_LONGG;
constexpr int kLcv = 2048;           // long chunks whose row is precomputed per batch

struct BatchBuf {
    uint32_t v[kThreads];          // popped items (vertex ids / row pieces)
    uint32_t chunk_next;           // next unclaimed edge chunk
    int32_t use_bm;                // the edge map below is valid for this batch
    uint32_t bm[kBitW];
    uint16_t rowmap[kBitW];
    // The two expansions use disjoint per-row tables (a launch runs one of them),
    // so they share storage: shared memory not used here is L1 for the probes.
    union {
        struct {                   // generic expansion (PageRank, multi-rank, BFS options off the default)
            uint64_t val[kThreads];        // depth (BFS) or delta bits (PR)
            int64_t beg[kThreads];         // row begin (offset into col)
            int64_t off[kThreads + 1];     // exclusive prefix of edge counts
            uint16_t chunk_v[kChunkMap + 1];  // vertex (batch index) holding the first edge of each chunk
            uint16_t nzslot[kThreads];
        };
        struct {                   // single-rank BFS expansion (atos_bfs1.cuh): one 16-B record per row --
            BRec rec[kThreads];            // short rows at [0, NZ) in edge-map order, long rows at
            uint16_t lcv[kLcv];            // [kThreads - NL, kThreads) --, the long-chunk -> row map and
            uint32_t lq0[kThreads];        // the first chunk of every long row
        };
    };
};

// batch slot holding edge e (e = 32 * w + lane) from the edge map
__device__ __forceinline__ int bm_slot(const BatchBuf &bb, int64_t e, int lane) {
    const int w = (int)(e >> 5);
    const uint32_t below = lane == 31 ? 0xFFFFFFFEu : (((2u << lane) - 1u) & ~1u);
    return bb.nzslot[bb.rowmap[w] + __popc(bb.bm[w] & below)];
}

struct alignas(16) Smem {
    RankDev R;
    BatchBuf bb[1];
    uint32_t wout[kWarps][kWOut];  // per-warp local push staging
    uint32_t wn[kWarps];
    uint32_t wpre[kWarps + 1];
    uint32_t wst[kWarps][kMaxRanks], wsh[kWarps][kMaxRanks];   // per-warp message staging tail/head
    uint64_t wt0[kWarps][kMaxRanks];                           // time staging became non-empty
    int64_t wsum[kWarps];
    uint64_t res_lo, res_hi;       // outstanding ring reservation (ring 0)
    uint64_t res2_lo, res2_hi;     // priority queue: outstanding reservation on ring 1
    uint64_t ring2_base;           // ring 1 tail at the start of this solve
    uint64_t pq_st;                // priority queue: pq_state read at the last pop
    uint64_t pq_k0;                // priority queue: pq_state at the start of the solve (Ctrl::pq_k0)
    uint32_t pq_th;                // current threshold (kNoTh: FIFO, nothing is far)
    int32_t pq_q;                  // current ring (pq_state & 1; 0 without the priority queue)
    int32_t pop_q;                 // ring the current batch was popped from
    uint64_t limit;                // discrete mode: this launch pops indices < limit
    uint64_t ring_base;            // ring tail at the start of this solve
    uint64_t b64[4];
    int32_t b32[4];
    int32_t minbad;
    int32_t flag;
    uint64_t staged_reported;
    uint64_t wave[kMaxRanks][5];   // coordinator double wave
    int32_t wave_valid;
    // CTA-cooperative inbound claim (cta_inbound)
    int32_t in_got, in_src, in_r;
    // BFS hub bounds (atos_bfs1.cuh): TMA-copy completion barrier, its parity, batch counter
    alignas(8) uint64_t hub_mbar;
    uint32_t hub_par, hub_rnd;
    uint64_t in_cc;
    uint32_t in_off[33];
    unsigned long long c_pops, c_edges, c_pushes, c_msgs, c_packets, c_idle, c_hub, c_busy, c_batches, c_far;
#ifdef ATOS_PROF
    unsigned long long prof[10];
#endif
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Rank owning global vertex u: the largest r with part[r] <= u (binary search;
// an unrolled scan over all kMaxRanks entries was 12 % of the 8-rank BFS
// worker's instructions).
__device__ __forceinline__ int owner_of(const RankDev &R, int64_t u) {
    int lo = 0, hi = R.n_ranks - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (R.part[mid] <= u) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// Dynamic shared memory after Smem: the BFS hub bounds (atos_bfs1.cuh).
__device__ __forceinline__ uint8_t *hub_base(Smem &s) { return reinterpret_cast<uint8_t *>(&s + 1); }

// Streaming loads of the column array: bypass L1, evict-first in L2 so that the
// random-access state (depth / residual) stays L2-resident.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
#ifndef ATOS_COL_L1
#define ATOS_COL_L1 0
#endif
__device__ __forceinline__ int32_t ld_stream(const int32_t *ptr, uint64_t pol) {
    int32_t v;
#if ATOS_COL_L1 == 1
    asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(ptr), "l"(pol));
#elif ATOS_COL_L1 == 2
    v = __ldcs(ptr);
#elif ATOS_COL_L1 == 3
    v = __ldg(ptr);
#else
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(ptr), "l"(pol));
#endif
    return v;
}

#ifdef ATOS_PROF
// phase timing (debug builds only): wait until `x` is available, then timestamp
#define PROF_T(var, x) do { if ((x) == 0x7fffffff) __nanosleep(1); var = clock64(); } while (0)
#endif

// Block-wide exclusive scan of one int64 per thread; returns the total.
__device__ __forceinline__ int64_t block_exscan(Smem &s, int64_t x, int64_t &excl) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t incl = x;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const int64_t y = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += y;
    }
    if (lane == 31) s.wsum[w] = incl;
    __syncthreads();
    if (w == 0) {
        const int64_t t = lane < kWarps ? s.wsum[lane] : 0;
        int64_t ti = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int64_t y = __shfl_up_sync(kFull, ti, d);
            if (lane >= d) ti += y;
        }
        if (lane < kWarps) s.wsum[lane] = ti - t;
        if (lane == kWarps - 1) s.b64[3] = (uint64_t)ti;
    }
    __syncthreads();
    excl = incl - x + s.wsum[w];
    const int64_t total = (int64_t)s.b64[3];
    __syncthreads();
    return total;
}

// largest j in [lo, hi] with off[j] <= e   (off[lo] <= e holds)
__device__ __forceinline__ int upper_vertex(const BatchBuf &bb, int lo, int hi, int64_t e) {
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (bb.off[mid] <= e) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// ---------------------------------------------------------------------------
// local ring pushes
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t &res_lo_q(Smem &s, int q) { return q ? s.res2_lo : s.res_lo; }
__device__ __forceinline__ uint64_t &res_hi_q(Smem &s, int q) { return q ? s.res2_hi : s.res_hi; }
__device__ __forceinline__ uint64_t ring_base_q(const Smem &s, int q) { return q ? s.ring2_base : s.ring_base; }

__device__ __forceinline__ void ring_store(const RankDev &R, uint64_t idx, uint32_t item, uint64_t base, int q = 0) {
    uint64_t *p = &q_slots(R, q)[idx & (R.ring_cap - 1)];
    uint32_t spins = 0;
    // every index below the solve's base was consumed or retired, so slots of the
    // first lap of this solve are free without looking; later laps check the tag
    while (idx - base >= R.ring_cap && !slot_free_for(ld_relaxed_gpu(p), idx)) {
        if (++spins > (1u << 24)) { set_error(R, kErrCapacity); return; }
        __nanosleep(64);
    }
    st_relaxed_gpu(p, pack(lo32(idx + 1), item));
}

// Consumer of index idx: read its slot (published iff slot_full_for) and, once
// the item is taken, hand the slot to the producer of idx + cap.
__device__ __forceinline__ uint64_t ring_read(const uint64_t *ring, uint64_t cap, uint64_t idx) {
    return ld_relaxed_gpu(&ring[idx & (cap - 1)]);
}
__device__ __forceinline__ void ring_release(uint64_t *ring, uint64_t cap, uint64_t idx) {
    st_relaxed_gpu(&ring[idx & (cap - 1)], pack(lo32(idx + cap), 0u));
}

// warp_flush_local with the priority queue (N1): far-tagged items go to the other ring.
// (wn by value: a reference argument of a non-inlined call would live in local memory)
__device__ __noinline__ void warp_flush_local_pq(Smem &s, int w, uint32_t wn, bool fence) {
    const uint32_t cnt = wn;
    const int lane = threadIdx.x & 31;
    const int q = s.pq_q;
    uint32_t nf = 0;
    for (uint32_t i0 = 0; i0 < cnt; i0 += 32)
        nf += __popc(__ballot_sync(kFull, i0 + lane < cnt && pq_is_far(s.wout[w][i0 + lane])));
    unsigned long long bn = 0, bf = 0;
    if (lane == 0) {
        if (cnt > nf) bn = atomicAdd((unsigned long long *)q_tail(s.R, q), (unsigned long long)(cnt - nf));
        if (nf) bf = atomicAdd((unsigned long long *)q_tail(s.R, q ^ 1), (unsigned long long)nf);
        atomicAdd(&s.c_far, (unsigned long long)nf);
    }
    bn = __shfl_sync(kFull, bn, 0);
    bf = __shfl_sync(kFull, bf, 0);
    if (fence) fence_acq_rel_gpu();
    for (uint32_t i0 = 0; i0 < cnt; i0 += 32) {
        const uint32_t i = i0 + lane;
        const uint32_t it = i < cnt ? s.wout[w][i] : 0u;
        const bool far = i < cnt && pq_is_far(it);
        const uint32_t mf = __ballot_sync(kFull, far), mn = __ballot_sync(kFull, i < cnt && !far);
        if (far) ring_store(s.R, bf + __popc(mf & lanemask_lt()), it & ~kFarBit, ring_base_q(s, q ^ 1), q ^ 1);
        else if (i < cnt) ring_store(s.R, bn + __popc(mn & lanemask_lt()), it, ring_base_q(s, q), q);
        bf += __popc(mf);
        bn += __popc(mn);
    }
    if (lane == 0) atomicAdd(&s.c_pushes, (unsigned long long)cnt);
    wn = 0;
    __syncwarp();
}

// Whole warp: push wout[w][0..wn) with one leader atomic.
__device__ void warp_flush_local(Smem &s, int w, uint32_t &wn, bool fence) {
    __syncwarp();
    const uint32_t cnt = wn;
    if (cnt == 0) return;
    const int lane = threadIdx.x & 31;
    if (s.pq_th != kNoTh) {         // priority queue (N1): far-tagged items go to the other ring
        warp_flush_local_pq(s, w, wn, fence);
        wn = 0;
        return;
    }
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd((unsigned long long *)&s.R.ctrl->tail.v, (unsigned long long)cnt);
    base = __shfl_sync(kFull, base, 0);
    if (fence) fence_acq_rel_gpu();   // fire-and-forget relaxations must be performed first
    // No fence: every item was appended only after its improving atomic had
    // returned (the append is control-dependent on the returned value), so the
    // state update is already performed at L2, the coherence point, before this
    // store is issued; the consumer's claiming atomic on the same word is
    // address-dependent on the slot it reads.
    // A gpu-scope fence here would also invalidate L1 (CCTL.IVALL) and with it
    // the probe hits.
    for (uint32_t i = lane; i < cnt; i += 32) ring_store(s.R, base + i, s.wout[w][i], s.ring_base);
    if (lane == 0) atomicAdd(&s.c_pushes, (unsigned long long)cnt);
    wn = 0;
    __syncwarp();
}

// Whole warp: lanes with pred append item (caller guarantees wn + 32 <= kWOut).
__device__ __forceinline__ void warp_append_local(Smem &s, int w, uint32_t &wn, bool pred, uint32_t item) {
    const uint32_t m = __ballot_sync(kFull, pred);
    if (pred) s.wout[w][wn + __popc(m & lanemask_lt())] = item;
    wn += __popc(m);
}

// Whole warp: append the items whose bit is set in each lane's mask (bit k ->
// item[k]) with one warp scan per chunk instead of one ballot per row.
template <int N>
__device__ __forceinline__ void warp_append_mask(Smem &s, int w, uint32_t &wn, uint32_t msk, const uint32_t (&item)[N],
                                                 bool fence) {
    const int lane = threadIdx.x & 31;
    const uint32_t cnt = __popc(msk);
    uint32_t incl = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, incl, d);
        if (lane >= d) incl += y;
    }
    const uint32_t total = __shfl_sync(kFull, incl, 31);
    if (total == 0) return;
    if (wn + total > (uint32_t)kWOut) warp_flush_local(s, w, wn, fence);   // total <= 32*N <= kWOut
    uint32_t pos = wn + incl - cnt;
#pragma unroll
    for (int k = 0; k < N; ++k)
        if ((msk >> k) & 1u) s.wout[w][pos++] = item[k];
    wn += total;
}

// ---------------------------------------------------------------------------
// remote messages: per-warp staging per destination; packets over NVLink
// ---------------------------------------------------------------------------
template <int APP>
__device__ __forceinline__ unsigned char *wstage(const Smem &s, const KParams &kp, int cta, int w, int d) {
    const size_t slot = (((size_t)cta * kWarps + w) * kMaxRanks + d) * (size_t)kp.stage_cap;
    return s.R.staging + slot * AppTraits<APP>::kMsgBytes;
}

template <int APP> __device__ bool warp_inbound(Smem &s, const KParams &kp, int w, uint32_t &wn);

// Whole warp: publish `cnt` staged messages for dst as one packet.
// A channel (s -> d) is nsub independent sub-channels (rings of cps packets,
// own reserve counter and receive cursor); a sending warp always uses the same
// one, so receivers claiming on different cursors do not serialise on one CAS.
__device__ __forceinline__ uint32_t sub_slot(const KParams &kp, int k, uint64_t i) {
    return (uint32_t)k * (uint32_t)kp.cps + (uint32_t)(i & (uint64_t)(kp.cps - 1));
}

template <int APP>
__device__ bool warp_send_packet(Smem &s, const KParams &kp, int cta, int w, int d, uint32_t cnt, uint32_t &wn) {
    const RankDev &R = s.R;
    const int lane = threadIdx.x & 31;
    const int k = (cta * kWarps + w) % kp.nsub;
    unsigned long long pidx = 0;
    if (lane == 0) pidx = atomicAdd((unsigned long long *)&R.ctrl->out_reserve[d * kp.nsub + k].v, 1ull);
    pidx = __shfl_sync(kFull, pidx, 0);
    const uint32_t slot = sub_slot(kp, k, pidx);
    uint64_t t_begin = 0;
    for (;;) {   // wait for the receiver to free the slot; keep consuming inbound meanwhile
        int st = 0;
        if (lane == 0) {
            const uint64_t f = ld_acquire_peer(kp.sys, &R.free_mirror[d][slot]);
            if (lo32(f) == lo32(pidx)) st = 1;
            else {
                const uint64_t now = globaltimer();
                if (t_begin == 0) t_begin = now;
                if (ld_relaxed_gpu(&R.ctrl->error.v) != 0 || now - t_begin > 4000000000ull) {
                    set_error(R, kErrCapacity);
                    st = 2;
                }
            }
        }
        st = __shfl_sync(kFull, st, 0);
        if (st == 1) break;
        if (st == 2) return false;
        warp_inbound<APP>(s, kp, w, wn);
    }
    const unsigned char *src = wstage<APP>(s, kp, cta, w, d);
    const uint32_t h = s.wsh[w][d];
    const uint32_t mask = (uint32_t)(kp.stage_cap - 1);
    unsigned char *dpay = R.out_payload[d] + (size_t)slot * kp.pkt * AppTraits<APP>::kMsgBytes;
    for (uint32_t i = lane; i < cnt; i += 32) {     // coalesced one-sided stores into d's HBM
        const uint32_t q = (h + i) & mask;
        if constexpr (APP == kApBfs) ((uint64_t *)dpay)[i] = ((const uint64_t *)src)[q];
        else ((uint4 *)dpay)[i] = ((const uint4 *)src)[q];
    }
    // One system-scope release per packet: the warp barrier orders every lane's
    // payload stores before lane 0's st.release (cumulative), which also orders
    // the S increment before the header -- S is counted before any receiver can
    // count the messages in R (termination, section 6).
    __syncwarp();
    if (lane == 0) {
        atomicAdd((unsigned long long *)&R.ctrl->sent.v, (unsigned long long)cnt);   // S before publish
        st_release_peer(kp.sys, &R.out_hdr[d][slot], pack(lo32(pidx + 1), cnt));
        s.wsh[w][d] = h + cnt;
        if (s.wsh[w][d] == s.wst[w][d]) s.wt0[w][d] = 0;
        atomicAdd(&s.c_msgs, (unsigned long long)cnt);
        atomicAdd(&s.c_packets, 1ull);
    }
    __syncwarp();
    return true;
}

// Whole warp: send full packets (and partial ones when `partial`) for every destination.
template <int APP>
__device__ __noinline__ uint32_t warp_flush_remote(Smem &s, const KParams &kp, int cta, int w, bool batch_end, uint32_t wn) {
    const RankDev &R = s.R;
    if (R.n_ranks <= 1) return wn;
    const uint64_t now = globaltimer();
    for (int d = 0; d < R.n_ranks; ++d) {
        if (d == R.rank) continue;
        for (;;) {
            __syncwarp();
            const uint32_t pending = s.wst[w][d] - s.wsh[w][d];
            if (pending == 0) break;
            bool go = pending >= (uint32_t)kp.pkt;
            if (!go && batch_end) {
                const uint64_t t0 = s.wt0[w][d];
                go = !kp.agg_on || (t0 != 0 && now - t0 >= (uint64_t)kp.agg_age_ns);
            }
            go = __shfl_sync(kFull, go, 0);
            if (!go) break;
            const uint32_t cnt = pending < (uint32_t)kp.pkt ? pending : (uint32_t)kp.pkt;
            if (!warp_send_packet<APP>(s, kp, cta, w, d, cnt, wn)) return wn;
        }
    }
    return wn;
}

// Whole warp: lanes with pred stage a message (dst, v_local at dst, payload).
template <int APP>
__device__ __forceinline__ void warp_append_remote(Smem &s, const KParams &kp, int cta, int w, bool pred, int dst,
                                                   uint32_t v_local, uint64_t payload, uint32_t &wn) {
    uint32_t todo = __ballot_sync(kFull, pred);
    if (todo == 0) return;
    const int lane = threadIdx.x & 31;
    const uint32_t mask = (uint32_t)(kp.stage_cap - 1);
    // one round per destination present among the lanes (a loop over all
    // n_ranks destinations with a ballot each was 38 % of the 8-rank BFS
    // worker's instructions)
    while (todo) {
        const int d = __shfl_sync(kFull, dst, __ffs(todo) - 1);
        const bool mine = pred && dst == d;
        const uint32_t m = __ballot_sync(kFull, mine);
        todo &= ~m;
        __syncwarp();
        if (s.wst[w][d] - s.wsh[w][d] + 32 > (uint32_t)kp.stage_cap) {
            // full packets out first (keeps room for this row)
            wn = warp_flush_remote<APP>(s, kp, cta, w, false, wn);
            __syncwarp();
        }
        const uint32_t t = s.wst[w][d];
        if (mine) {
            unsigned char *b = wstage<APP>(s, kp, cta, w, d);
            const uint32_t pos = (t + __popc(m & lanemask_lt())) & mask;
            if constexpr (APP == kApBfs) ((uint64_t *)b)[pos] = pack((uint32_t)payload, v_local);
            else ((uint4 *)b)[pos] = make_uint4(v_local, 0u, (uint32_t)payload, (uint32_t)(payload >> 32));
        }
        __syncwarp();
        if (lane == 0) {
            if (t == s.wsh[w][d]) s.wt0[w][d] = globaltimer();
            s.wst[w][d] = t + __popc(m);
        }
        __syncwarp();
    }
    // aggregation off: the warp pushes what this 32-edge step produced right away
    // (Listing 5's per-warp remote push): packets of <= 32 messages
    if (!kp.agg_on) wn = warp_flush_remote<APP>(s, kp, cta, w, true, wn);
}

// Whole warp: claim the ready prefix (up to kClaim packets) of one inbound
// channel with ONE CAS on its cursor, apply the messages (owner-side receive),
// and release every packet slot to its sender.  Each lane probes one header, so
// a busy channel is drained kClaim packets per cursor round trip instead of one.
constexpr int kClaim = 8;
constexpr int kInU = 4;              // messages per lane in flight while applying

// Multi-rank BFS, a remote edge that improved this rank's ghost word of u: send u's new depth
// to its owner -- or, with bfs_ratom (virtual ranks), lower the owner's depth word here with one
// atomicMin (the paper's remote update) and send an activation only if it improved
// there.  Whole warp (warp_append_remote).
template <int APP>
__device__ __forceinline__ void bfs_send_remote(Smem &s, const KParams &kp, int cta, int w, bool rem, int64_t u,
                                                uint32_t nd, uint32_t &wn) {
    const RankDev &R = s.R;
    const int d = rem ? owner_of(R, u) : 0;
    uint64_t pay = nd;
    if (kp.bfs_ratom) {
        if (rem) {
            const uint32_t ndw = dw_make(nd);
            rem = atom_min_u32(R.peer_depth[d] + u, ndw) > ndw;
        }
        pay = nd | kBfsActivate;
    }
    warp_append_remote<APP>(s, kp, cta, w, rem, d, rem ? (uint32_t)(u - R.part[d]) : 0u, pay, wn);
}

#ifndef ATOS_INBOUND_WIDE
// experiment, off: 1 = poll every inbound channel at once (inbound_claim_wide).
// Measured slower (virtual ranks, same box: PR RMAT-20 2/4/8 ranks 51/75/109 ->
// 83/140/254 ms, BFS RMAT-24 2/8 ranks 10.9/20.6 -> 11.9/23.4 ms): every idle
// worker then claims the first ready channel in the same rotation order, and the
// claims collide on its cursor
#define ATOS_INBOUND_WIDE 0
#endif

// Whole warp, up to 32 inbound sub-channels (nc <= 32): poll them all at once --
// lane l takes channel (start + l) mod nc, loads its cursor, then the sequence
// words of its next kClaim packet headers (independent loads) -- pick the first
// channel (in rotation order) with a ready prefix and claim that prefix with ONE
// CAS on its cursor.  Two load round trips to look at every channel, where the
// one-by-one walk took two per channel (an idle 8-rank worker walked 7 channels,
// ~14 round trips, while the other 15 warps waited at the inbound barrier).
// Returns the claimed packet count (0: nothing claimed) with the channel and the
// cursor value; the caller acquires the claimed headers.
__device__ __forceinline__ int inbound_claim_wide(const Smem &s, const KParams &kp, int start, int &ch_out,
                                                  uint64_t &cc_out) {
    const RankDev &R = s.R;
    const int lane = threadIdx.x & 31;
    const int nc = R.n_ranks * kp.nsub;
    int ch = start + lane;
    if (ch >= nc) ch -= nc;
    const int sr = ch / kp.nsub, sk = ch - sr * kp.nsub;
    const bool valid = lane < nc && sr != R.rank;
    int r = 0;
    uint64_t cc = 0;
    if (valid) {
        cc = ld_relaxed_gpu(&R.ctrl->in_cursor[ch].v);
        const int lim = kClaim < kp.cps ? kClaim : kp.cps;
        uint32_t sq[kClaim];
#pragma unroll
        for (int k = 0; k < kClaim; ++k)     // the header's high word: the packet's sequence tag
            sq[k] = k < lim ? ld_relaxed_peer_u32(kp.sys, reinterpret_cast<const uint32_t *>(
                                                            &R.in_hdr[sr][sub_slot(kp, sk, cc + k)]) + 1)
                            : 0u;
#pragma unroll
        for (int k = 0; k < kClaim; ++k)
            if (r == k && k < lim && sq[k] == lo32(cc + k + 1)) r = k + 1;
    }
    const uint32_t m = __ballot_sync(kFull, r > 0);
    if (m == 0) return 0;
    const int src = __ffs(m) - 1;
    const int rr = __shfl_sync(kFull, r, src);
    const uint64_t c2 = __shfl_sync(kFull, cc, src);
    const int chs = __shfl_sync(kFull, ch, src);
    int won = 0;
    if (lane == 0)
        won = atomicCAS((unsigned long long *)&R.ctrl->in_cursor[chs].v, (unsigned long long)c2,
                        (unsigned long long)(c2 + (uint64_t)rr)) == c2;
    if (!__shfl_sync(kFull, won, 0)) return 0;
    ch_out = chs;
    cc_out = c2;
    return rr;
}

template <int APP>
__device__ bool warp_inbound(Smem &s, const KParams &kp, int w, uint32_t &wn) {
    const RankDev &R = s.R;
    if (R.n_ranks <= 1) return false;
    const int lane = threadIdx.x & 31;
    const uint32_t cps = (uint32_t)kp.cps;
    const int p = R.n_ranks, nc = p * kp.nsub;
    const int start = (w + (int)(s.c_idle & 7)) % nc;
    const bool wide = ATOS_INBOUND_WIDE && nc <= 32;
    // (channel ch = sr * nsub + sk walked incrementally: a div / mod per probed
    // channel was a third of a polling sender's instructions)
    int sr0 = start / kp.nsub, sk0 = start - sr0 * kp.nsub;
    for (int kk = 0; kk < (wide ? 1 : nc);
         ++kk, (++sk0 == kp.nsub) ? (sk0 = 0, sr0 = (sr0 + 1 == p ? 0 : sr0 + 1)) : 0) {
        int sr = sr0, sk = sk0, ch = sr * kp.nsub + sk, r = 0;
        uint64_t cc = 0;
        uint32_t cnt = 0;
        if (wide) {
            r = inbound_claim_wide(s, kp, start, ch, cc);
            if (r == 0) return false;
            sr = ch / kp.nsub;
            sk = ch - sr * kp.nsub;
        } else {
            if (sr == R.rank) continue;
            unsigned long long *cur = (unsigned long long *)&R.ctrl->in_cursor[ch].v;
            if (lane == 0) cc = ld_relaxed_gpu((const uint64_t *)cur);
            cc = __shfl_sync(kFull, cc, 0);
            bool ready = false;
            if (lane < kClaim && (uint32_t)lane < cps) {
                // relaxed poll: an acquire load also invalidates L1 (CCTL.IVALL), which
                // every idle warp would otherwise do on every poll of every channel
                const uint64_t h = ld_relaxed_peer(kp.sys, &R.in_hdr[sr][sub_slot(kp, sk, cc + lane)]);
                ready = hi32(h) == lo32(cc + lane + 1);
            }
            const uint32_t nready = __ballot_sync(kFull, ready);
            r = (~nready == 0u) ? 32 : __ffs(~nready) - 1;   // ready prefix
            if (r == 0) continue;
            int won = 0;
            if (lane == 0) won = atomicCAS(cur, (unsigned long long)cc, (unsigned long long)(cc + r)) == cc;
            if (!__shfl_sync(kFull, won, 0)) continue;
        }
        // acquire each claimed header (synchronises with its sender's st.release;
        // its low word is the packet's message count), then the warp barrier
        // orders every lane's payload reads after them
        if (lane < r) cnt = lo32(ld_acquire_peer(kp.sys, &R.in_hdr[sr][sub_slot(kp, sk, cc + lane)]));
        __syncwarp();
        uint32_t total = 0;
        for (int q = 0; q < r; ++q) {
            const uint32_t cq = __shfl_sync(kFull, cnt, q);
            const uint32_t slot = sub_slot(kp, sk, cc + q);
            const unsigned char *pay = R.in_payload[sr] + (size_t)slot * kp.pkt * AppTraits<APP>::kMsgBytes;
            for (uint32_t base = 0; base < cq; base += 32 * kInU) {
                bool pred[kInU];
                uint32_t ul[kInU];
                if constexpr (APP == kApBfs) {
                    uint64_t m[kInU];
#pragma unroll
                    for (int j = 0; j < kInU; ++j) {
                        const uint32_t i = base + j * 32 + lane;
                        m[j] = i < cq ? ld_cg_u64((const uint64_t *)pay + i) : 0ull;
                    }
#pragma unroll
                    for (int j = 0; j < kInU; ++j) {
                        const uint32_t i = base + j * 32 + lane;
                        ul[j] = lo32(m[j]);
                        pred[j] = false;
                        if (i < cq) {
                            const uint32_t hv = hi32(m[j]), dd = hv & ~kBfsActivate;
                            if (hv & kBfsActivate) {
                                pred[j] = true;          // lowered by the sender (bfs_ratom)
                            } else {
                                const uint32_t ndw = dw_make(dd);
                                pred[j] = atom_min_u32(R.depth + R.v_begin + ul[j], ndw) > ndw;
                            }
                            if (pred[j] && kp.filter) filt_put_fresh(R.filt, R.v_begin + ul[j], dd);
                            ul[j] = pq_tag(ul[j], dd, s.pq_th);
                        }
                    }
                } else {
                    uint4 m[kInU];
#pragma unroll
                    for (int j = 0; j < kInU; ++j) {
                        const uint32_t i = base + j * 32 + lane;
                        m[j] = i < cq ? ld_cg_u4((const uint4 *)pay + i) : make_uint4(0, 0, 0, 0);
                    }
#pragma unroll
                    for (int j = 0; j < kInU; ++j) {
                        const uint32_t i = base + j * 32 + lane;
                        ul[j] = m[j].x;
                        pred[j] = false;
                        if (i < cq) {
                            const uint64_t pv = ((uint64_t)m[j].w << 32) | m[j].z;
                            if (pv == kPrActivate) {
                                pred[j] = true;          // applied remotely by the sender (pr_ratom)
                            } else {
                                const double dlt = __longlong_as_double((long long)pv);
                                const double old = atom_add_f64(R.pr_res + pr_slot(ul[j], R.pr_q), dlt);
                                pred[j] = old < kp.eps && old + dlt >= kp.eps;
                            }
                        }
                    }
                }
#pragma unroll
                for (int j = 0; j < kInU; ++j) {
                    if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, false);
                    warp_append_local(s, w, wn, pred[j], ul[j]);
                }
            }
            total += cq;
        }
        warp_flush_local(s, w, wn, false);      // T counts the new local work before R
        __syncwarp();
        if (lane == 0) {
            // one system-scope fence per claim: every lane's payload reads and the
            // resulting state updates / enqueues are ordered before the slots are
            // handed back to the sender and before R counts the messages
            fence_peer(kp.sys);
            for (int q = 0; q < r; ++q)
                st_relaxed_peer(kp.sys, &R.peer_free[sr][sub_slot(kp, sk, cc + q)], cc + q + cps);   // slots free for the sender
            atomicAdd((unsigned long long *)&R.ctrl->recvd.v, (unsigned long long)total);
        }
        __syncwarp();
        return true;
    }
    return false;
}

// Whole CTA (the worker loop's receive step): warp 0 claims the ready prefix (up
// to kClaim packets) of one inbound channel with one CAS, then ALL 512 threads
// apply its messages -- a claimed set is expanded like a pop batch, instead of one
// warp applying it while the other 15 wait at the loop's barrier.  Returns
// whether anything was claimed (CTA-uniform).
template <int APP>
__device__ bool cta_inbound(Smem &s, const KParams &kp, int cta) {
    const RankDev &R = s.R;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint32_t cps = (uint32_t)kp.cps;
    if (w == 0) {
        const int nc = R.n_ranks * kp.nsub;
        const int start = (cta + (int)s.c_idle) % nc;
        int got = 0;
        const bool wide = ATOS_INBOUND_WIDE && nc <= 32;     // one look at every channel (inbound_claim_wide)
        int sr0 = start / kp.nsub, sk0 = start - sr0 * kp.nsub;
        for (int kk = 0; kk < (wide ? 1 : nc) && !got;
             ++kk, (++sk0 == kp.nsub) ? (sk0 = 0, sr0 = (sr0 + 1 == R.n_ranks ? 0 : sr0 + 1)) : 0) {
            int sr = sr0, sk = sk0, ch = sr * kp.nsub + sk, r = 0;
            uint64_t cc = 0;
            if (wide) {
                r = inbound_claim_wide(s, kp, start, ch, cc);
                if (r == 0) break;
                sr = ch / kp.nsub;
                sk = ch - sr * kp.nsub;
            } else {
                if (sr == R.rank) continue;
                unsigned long long *cur = (unsigned long long *)&R.ctrl->in_cursor[ch].v;
                if (lane == 0) cc = ld_relaxed_gpu((const uint64_t *)cur);
                cc = __shfl_sync(kFull, cc, 0);
                bool ready = false;
                if (lane < kClaim && (uint32_t)lane < cps) {
                    const uint64_t h = ld_relaxed_peer(kp.sys, &R.in_hdr[sr][sub_slot(kp, sk, cc + lane)]);   // relaxed poll
                    ready = hi32(h) == lo32(cc + lane + 1);
                }
                const uint32_t nready = __ballot_sync(kFull, ready);
                r = (~nready == 0u) ? 32 : __ffs(~nready) - 1;
                if (r == 0) continue;
                int won = 0;
                if (lane == 0) won = atomicCAS(cur, (unsigned long long)cc, (unsigned long long)(cc + r)) == cc;
                if (!__shfl_sync(kFull, won, 0)) continue;
            }
            // sync with each sender's release; the header's low word is the message count
            const uint32_t cnt = lane < r ? lo32(ld_acquire_peer(kp.sys, &R.in_hdr[sr][sub_slot(kp, sk, cc + lane)])) : 0u;
            uint32_t incl = lane < r ? cnt : 0u;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, d);
                if (lane >= d) incl += y;
            }
            if (lane < r) s.in_off[lane + 1] = incl;
            if (lane == 0) { s.in_off[0] = 0; s.in_src = ch; s.in_cc = cc; s.in_r = r; }
            got = 1;
        }
        if (lane == 0) s.in_got = got;
    }
    __syncthreads();      // also orders warp 0's acquires before every thread's payload reads
    if (!s.in_got) return false;
    const int ch = s.in_src, sr = ch / kp.nsub, sk = ch % kp.nsub, r = s.in_r;
    const uint64_t cc = s.in_cc;
    const uint32_t M = s.in_off[r];
    uint32_t wn = s.wn[w];
    for (uint32_t base = 0; base < M; base += kThreads * kInU) {
        bool pred[kInU];
        uint32_t ul[kInU];
        int q = 0;
#pragma unroll
        for (int j = 0; j < kInU; ++j) {
            const uint32_t m = base + j * kThreads + tid;
            pred[j] = false;
            ul[j] = 0;
            if (m < M) {
                while (q + 1 < r && s.in_off[q + 1] <= m) ++q;   // packet holding message m
                const uint32_t slot = sub_slot(kp, sk, cc + q);
                const unsigned char *pay = R.in_payload[sr] + (size_t)slot * kp.pkt * AppTraits<APP>::kMsgBytes;
                const uint32_t i = m - s.in_off[q];
                if constexpr (APP == kApBfs) {
                    const uint64_t msg = ld_cg_u64((const uint64_t *)pay + i);
                    ul[j] = lo32(msg);
                    const uint32_t hv = hi32(msg), dd = hv & ~kBfsActivate;
                    if (hv & kBfsActivate) {
                        pred[j] = true;                  // lowered by the sender (bfs_ratom)
                    } else {
                        const uint32_t ndw = dw_make(dd);
                        pred[j] = atom_min_u32(R.depth + R.v_begin + ul[j], ndw) > ndw;
                    }
                    if (pred[j] && kp.filter) filt_put_fresh(R.filt, R.v_begin + ul[j], dd);
                    ul[j] = pq_tag(ul[j], dd, s.pq_th);
                } else {
                    const uint4 msg = ld_cg_u4((const uint4 *)pay + i);
                    ul[j] = msg.x;
                    const uint64_t pv = ((uint64_t)msg.w << 32) | msg.z;
                    if (pv == kPrActivate) {
                        pred[j] = true;                  // applied remotely by the sender (pr_ratom)
                    } else {
                        const double dlt = __longlong_as_double((long long)pv);
                        const double old = atom_add_f64(R.pr_res + pr_slot(ul[j], R.pr_q), dlt);
                        pred[j] = old < kp.eps && old + dlt >= kp.eps;
                    }
                }
            }
        }
#pragma unroll
        for (int j = 0; j < kInU; ++j) {
            if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, false);
            warp_append_local(s, w, wn, pred[j], ul[j]);
        }
    }
    warp_flush_local(s, w, wn, false);        // T counts the new local work before R
    if (lane == 0) s.wn[w] = wn;
    __syncthreads();
    if (tid == 0) {
        // one system-scope fence per claim: payload reads and their effects are
        // ordered before the slots go back to the sender and before R counts them
        fence_peer(kp.sys);
        for (int q = 0; q < r; ++q)
            st_relaxed_peer(kp.sys, &R.peer_free[sr][sub_slot(kp, sk, cc + q)], cc + q + cps);
        atomicAdd((unsigned long long *)&R.ctrl->recvd.v, (unsigned long long)M);
        s.c_batches++;
    }
    return true;
}

// ---------------------------------------------------------------------------
// BFS relaxation of N edges per lane (u[k] = target or -1, nd[k] = candidate
// depth): probe (a stale word is larger, never smaller, so a probe can only
// cause a redundant atomic), then the relaxation.
// Retired edges come back with u[k] = -1 and imp[k] = false.  Whole warp.
// ---------------------------------------------------------------------------
template <int N, bool MULTI>
__device__ __forceinline__ void bfs_relax(Smem &s, const KParams &kp, int32_t (&u)[N],
                                          const uint32_t (&nd)[N], bool (&imp)[N]) {
    const RankDev &R = s.R;
    uint32_t *const depth = R.depth;
    uint8_t *const filt = R.filt;
    const bool fl = kp.filter;
    uint32_t cur[N];
    if (fl) {
#pragma unroll
        for (int k = 0; k < N; ++k) cur[k] = (u[k] >= 0) ? filt_probe(filt, u[k]) : 0u;     // probe the filter
    } else {
#pragma unroll
        for (int k = 0; k < N; ++k) {
#ifdef ATOS_NO_PROBE
            cur[k] = 0xFFFFFFFFu;
#else
            cur[k] = (u[k] >= 0) ? ldg_u32(depth + u[k]) : 0u;     // probe the word
#endif
        }
    }
    if (kp.relax_red) {
        // fire-and-forget relaxation: red.min, enqueue on the probe's verdict.
        // A racing improver may make the entry redundant (skipped at pop by the
        // pending bit); the flush fences before publishing the items.
#pragma unroll
        for (int k = 0; k < N; ++k) {
            const uint32_t ndw = dw_make(nd[k]);
            imp[k] = u[k] >= 0 && (fl ? filt_pass(cur[k], u[k], nd[k]) : ndw < cur[k]);
            if (imp[k]) {
                red_min_u32(depth + u[k], ndw);
                if (fl) filt_put(filt, u[k], nd[k], cur[k]);
            }
        }
    } else {
#pragma unroll
        for (int k = 0; k < N; ++k) {
            const uint32_t ndw = dw_make(nd[k]);
            imp[k] = false;
            if (u[k] >= 0 && (fl ? filt_pass(cur[k], u[k], nd[k]) : ndw < cur[k])) {
                imp[k] = atom_min_u32(depth + u[k], ndw) > ndw;
                if (fl && imp[k]) filt_put(filt, u[k], nd[k], cur[k]);
            }
        }
    }
}

// ---------------------------------------------------------------------------
// batch expansion
// ---------------------------------------------------------------------------
template <int APP, bool MULTI>
__device__ void expand_warp(Smem &s, BatchBuf &bb, const KParams &kp, int cta, int B, int64_t E, uint32_t &wn) {
    const RankDev &R = s.R;
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // register copies of the hot rank fields (s.R lives in smem)
    const int64_t vb = R.v_begin, ve = R.v_end;
    constexpr bool multi = MULTI;
    const int32_t *const col = R.col;
    double *const res = R.pr_res;
    const uint64_t pol = policy_evict_first();
    const uint32_t nch = (uint32_t)((E + kChunk - 1) / kChunk);
    const uint32_t th = s.pq_th;       // BFS priority queue threshold (kNoTh: off)
    int jprev = 0;
    uint32_t cs = (uint32_t)(threadIdx.x >> 5);   // static schedule: chunks w, w + 16, ...
    for (;;) {
        uint32_t c = 0;
        if (kp.static_chunks) {
            c = cs;
            cs += kWarps;
        } else {
            // dynamic chunk claim: a warp that finishes early takes the next chunk
            if (lane == 0) c = atomicAdd(&bb.chunk_next, 1u);
            c = __shfl_sync(kFull, c, 0);
        }
        if (c >= nch) break;
#ifdef ATOS_PROF
        long long pt0 = clock64(), pt1, pt2, pt3, pt4;
#endif
        const int64_t c0 = (int64_t)c * kChunk;
        const int64_t clast = (E < c0 + kChunk ? E : c0 + kChunk) - 1;
        int jlo, jhi;
        if (c + 1 < (uint32_t)kChunkMap) {      // precomputed in process_batch
            jlo = bb.chunk_v[c];
            jhi = c + 1 < nch ? bb.chunk_v[c + 1] : B - 1;
        } else {
            jlo = upper_vertex(bb, bb.off[jprev] <= c0 ? jprev : 0, B - 1, c0);
            jhi = upper_vertex(bb, jlo, B - 1, clast);
        }
        jprev = jlo;
        int32_t u[kU];
        using ValT = typename std::conditional<APP == kApBfs, uint32_t, uint64_t>::type;   // depth | delta bits
        ValT vv[kU];
        if (bb.use_bm) {
#pragma unroll
            for (int k = 0; k < kU; ++k) {
                const int64_t e = c0 + k * 32 + lane;
                u[k] = -1;
                vv[k] = 0;
                if (e <= clast) {
                    const int jj = bm_slot(bb, e, lane);
                    u[k] = ld_stream(col + bb.beg[jj] + (e - bb.off[jj]), pol);
                    vv[k] = (ValT)bb.val[jj];
                }
            }
        } else {
        int j = jlo;
        // the lane's current vertex in registers: column base (beg - off), value and the
        // next vertex's first edge; shared memory is read again only when a row ends
        int64_t cbase = bb.beg[j] - bb.off[j], nxt = j < jhi ? bb.off[j + 1] : INT64_MAX;
        ValT cval = (ValT)bb.val[j];
#pragma unroll
        for (int k = 0; k < kU; ++k) {
            const int64_t e = c0 + k * 32 + lane;
            u[k] = -1;
            vv[k] = 0;
            if (e <= clast) {
                if (e >= nxt) {                             // usually one step for skewed graphs
                    ++j;
                    if (j < jhi && bb.off[j + 1] <= e) j = upper_vertex(bb, j + 1, jhi, e);
                    cbase = bb.beg[j] - bb.off[j];
                    nxt = j < jhi ? bb.off[j + 1] : INT64_MAX;
                    cval = (ValT)bb.val[j];
                }
                u[k] = ld_stream(col + cbase + e, pol);
                vv[k] = cval;
            }
        }
        }
#ifdef ATOS_PROF
        { int32_t sk = 0; for (int k = 0; k < kU; ++k) sk |= u[k]; PROF_T(pt1, sk); }
#endif
#ifdef ATOS_DBG_COLONLY
        // diagnostic build: stream the columns, skip relaxation (wrong results)
        { int32_t sk = 0; for (int k = 0; k < kU; ++k) sk ^= u[k]; if (sk == 0x7fffffff) s.c_hub++;
#ifdef ATOS_PROF
          if (lane == 0) { atomicAdd(&s.prof[0], (unsigned long long)(pt1 - pt0)); atomicAdd(&s.prof[4], 1ull); }
#endif
          continue; }
#endif
        if constexpr (APP == kApBfs) {
            uint32_t nd[kU];
#pragma unroll
            for (int k = 0; k < kU; ++k) nd[k] = (uint32_t)vv[k] + 1u;
            bool imp[kU];
            bfs_relax<kU, MULTI>(s, kp, u, nd, imp);
#ifdef ATOS_PROF
            pt2 = pt3 = pt1;
            { int32_t sk = 0; for (int k = 0; k < kU; ++k) sk |= imp[k] ? 1 : 0; PROF_T(pt3, sk << 30); }
#endif
            if constexpr (!multi) {
                uint32_t msk = 0, item[kU];
#pragma unroll
                for (int k = 0; k < kU; ++k) {
                    msk |= (imp[k] ? 1u : 0u) << k;
                    item[k] = pq_tag((uint32_t)(u[k] - vb), nd[k], th);
                }
                warp_append_mask<kU>(s, w, wn, msk, item, kp.relax_red);
            } else {
#pragma unroll
                for (int k = 0; k < kU; ++k) {
                    const bool loc = imp[k] && u[k] >= vb && u[k] < ve;
                    if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, kp.relax_red);
                    warp_append_local(s, w, wn, loc, pq_tag((uint32_t)(u[k] - vb), nd[k], th));
                    bfs_send_remote<APP>(s, kp, cta, w, imp[k] && !loc, u[k], (uint32_t)vv[k] + 1u, wn);
                }
            }
#ifdef ATOS_PROF
            pt4 = clock64();
            if (lane == 0) {
                atomicAdd(&s.prof[0], (unsigned long long)(pt1 - pt0));
                atomicAdd(&s.prof[1], (unsigned long long)(pt2 - pt1));
                atomicAdd(&s.prof[2], (unsigned long long)(pt3 - pt2));
                atomicAdd(&s.prof[3], (unsigned long long)(pt4 - pt3));
                atomicAdd(&s.prof[4], 1ull);
            }
#endif
        } else {
            const double eps = kp.eps;
            bool cross[kU], gcross[kU];
            const bool comb = MULTI && kp.combine;
            const int64_t qn = pr_q_of(R.n);
#pragma unroll
            for (int k = 0; k < kU; ++k) {
                cross[k] = gcross[k] = false;
                const double dlt = __longlong_as_double((long long)vv[k]);
                if (u[k] >= vb && u[k] < ve) {
                    const double old = atom_add_f64(res + pr_slot(u[k] - vb, R.pr_q), dlt);
                    cross[k] = old < eps && old + dlt >= eps;        // crossing enqueue (R5)
                } else if (comb && u[k] >= 0) {                      // combine into the ghost residual (N2)
                    const double old = atom_add_f64(R.pr_ghost + pr_slot(u[k], qn), dlt);
                    gcross[k] = old < kp.eps_g && old + dlt >= kp.eps_g;
                } else if (MULTI && kp.pr_ratom && u[k] >= 0) {
                    // remote delta applied in the owner's memory (one-sided atomic, the
                    // paper's remote update); only a crossing becomes a message
                    const int d = owner_of(R, u[k]);
                    double *pr = R.peer_res[d] + pr_slot(u[k] - R.part[d], pr_q_of(R.part[d + 1] - R.part[d]));
                    const double old = kp.sys ? atom_add_f64_sys(pr, dlt) : atom_add_f64(pr, dlt);
                    gcross[k] = old < eps && old + dlt >= eps;
                }
            }
            if constexpr (!multi) {
                uint32_t msk = 0, item[kU];
#pragma unroll
                for (int k = 0; k < kU; ++k) {
                    msk |= (cross[k] ? 1u : 0u) << k;
                    item[k] = (uint32_t)(u[k] - vb);
                }
                warp_append_mask<kU>(s, w, wn, msk, item, false);
            } else {
#pragma unroll
                for (int k = 0; k < kU; ++k) {
                    if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, false);
                    warp_append_local(s, w, wn, cross[k], (uint32_t)(u[k] - vb));
                    if (comb) {   // the crossing add takes the whole ghost and sends it as one message
                        uint64_t gv = 0;
                        if (gcross[k]) gv = atom_exch_u64((uint64_t *)(R.pr_ghost + pr_slot(u[k], qn)), 0ull);
                        const int d = gcross[k] ? owner_of(R, u[k]) : 0;
                        warp_append_remote<APP>(s, kp, cta, w, gcross[k], d,
                                                gcross[k] ? (uint32_t)(u[k] - R.part[d]) : 0u, gv, wn);
                        continue;
                    }
                    if (kp.pr_ratom) {   // remote deltas already applied: activation messages for crossings only
                        const int d = gcross[k] ? owner_of(R, u[k]) : 0;
                        warp_append_remote<APP>(s, kp, cta, w, gcross[k], d,
                                                gcross[k] ? (uint32_t)(u[k] - R.part[d]) : 0u, kPrActivate, wn);
                        continue;
                    }
                    const bool rem = u[k] >= 0 && !(u[k] >= vb && u[k] < ve);
                    const int d = rem ? owner_of(R, u[k]) : 0;
                    warp_append_remote<APP>(s, kp, cta, w, rem, d, rem ? (uint32_t)(u[k] - R.part[d]) : 0u,
                                            (uint64_t)vv[k], wn);
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------
// BFS expansion, software-pipelined: each warp keeps two 128-edge chunks in
// flight -- the column loads of the next chunk are issued before the probes,
// atomics and appends of the current one, so the HBM latency of the column
// stream overlaps the L2 round trips of the relaxation.
// ---------------------------------------------------------------------------
constexpr int kPU = kU < 4 ? kU : 4;         // rows (of 32 edges) per pipelined stage
constexpr int kPChunk = 32 * kPU;            // 128 edges
static_assert(kChunk % kPChunk == 0, "pipelined chunks subdivide map chunks");

struct PipeStage {
    int32_t u[kPU];
    uint32_t nd[kPU];
};

__device__ __forceinline__ void pipe_load(const BatchBuf &bb, int B, int64_t E, uint32_t nchm, uint32_t c, PipeStage &st,
                                          const int32_t *col, uint64_t pol) {
    const int lane = threadIdx.x & 31;
    const int64_t c0 = (int64_t)c * kPChunk;
    const int64_t clast = (E < c0 + kPChunk ? E : c0 + kPChunk) - 1;
    if (bb.use_bm) {
#pragma unroll
        for (int k = 0; k < kPU; ++k) {
            const int64_t e = c0 + k * 32 + lane;
            st.u[k] = -1;
            st.nd[k] = 0;
            if (e <= clast) {
                const int jj = bm_slot(bb, e, lane);
                st.u[k] = ld_stream(col + bb.beg[jj] + (e - bb.off[jj]), pol);
                st.nd[k] = (uint32_t)bb.val[jj] + 1u;
            }
        }
        return;
    }
    const uint32_t m = (uint32_t)(c0 / kChunk);          // map chunk containing c0
    int jlo, jhi;
    if (m + 1 < (uint32_t)kChunkMap) {
        jlo = bb.chunk_v[m];                               // vertex of edge m*kChunk <= vertex of c0
        jhi = m + 1 < nchm ? bb.chunk_v[m + 1] : B - 1;
    } else {
        jlo = upper_vertex(bb, 0, B - 1, c0);
        jhi = upper_vertex(bb, jlo, B - 1, clast);
    }
    int j = jlo;
#pragma unroll
    for (int k = 0; k < kPU; ++k) {
        const int64_t e = c0 + k * 32 + lane;
        st.u[k] = -1;
        st.nd[k] = 0;
        if (e <= clast) {
            if (j < jhi && bb.off[j + 1] <= e) {
                ++j;
                if (j < jhi && bb.off[j + 1] <= e) j = upper_vertex(bb, j + 1, jhi, e);
            }
            st.u[k] = ld_stream(col + bb.beg[j] + (e - bb.off[j]), pol);
            st.nd[k] = (uint32_t)bb.val[j] + 1u;
        }
    }
}

template <int APP, bool MULTI>
__device__ __forceinline__ void pipe_relax(Smem &s, const KParams &kp, int cta, PipeStage &st, uint32_t &wn) {
    const RankDev &R = s.R;
    const int w = threadIdx.x >> 5;
    const int64_t vb = R.v_begin, ve = R.v_end;
    bool imp[kPU];
    bfs_relax<kPU, MULTI>(s, kp, st.u, st.nd, imp);
#pragma unroll
    for (int k = 0; k < kPU; ++k) {
        const bool loc = imp[k] && st.u[k] >= vb && st.u[k] < ve;
        if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, kp.relax_red);
        warp_append_local(s, w, wn, loc, pq_tag((uint32_t)(st.u[k] - vb), st.nd[k], s.pq_th));
        if constexpr (MULTI) bfs_send_remote<APP>(s, kp, cta, w, imp[k] && !loc, st.u[k], st.nd[k], wn);
    }
}

template <int APP, bool MULTI>
__device__ void expand_warp_pipe(Smem &s, BatchBuf &bb, const KParams &kp, int cta, int B, int64_t E, uint32_t &wn) {
    const int lane = threadIdx.x & 31;
    const int32_t *const col = s.R.col;
    const uint64_t pol = policy_evict_first();
    const uint32_t nchm = (uint32_t)((E + kChunk - 1) / kChunk);
    const uint32_t nch = (uint32_t)((E + kPChunk - 1) / kPChunk);
    uint32_t c = 0;
    if (lane == 0) c = atomicAdd(&bb.chunk_next, 1u);
    c = __shfl_sync(kFull, c, 0);
    if (c >= nch) return;
    PipeStage a, b;
    pipe_load(bb, B, E, nchm, c, a, col, pol);
    for (;;) {
        uint32_t c2 = 0;
        if (lane == 0) c2 = atomicAdd(&bb.chunk_next, 1u);
        c2 = __shfl_sync(kFull, c2, 0);
        const bool more = c2 < nch;
        if (more) pipe_load(bb, B, E, nchm, c2, b, col, pol);   // next chunk's columns in flight
        pipe_relax<APP, MULTI>(s, kp, cta, a, wn);
        if (!more) break;
        a = b;
    }
}

// ---------------------------------------------------------------------------
// BFS expansion, three-stage software pipeline (pipeline = 3): while chunk i
// is relaxed (compare, red/atomicMin, append), the probes of chunk i+1 and the
// column loads of chunk i+2 are already in flight, so a warp keeps two memory
// round trips outstanding instead of waiting on col -> probe per chunk.
// ---------------------------------------------------------------------------
template <bool MULTI>
__device__ __forceinline__ void probe_issue(const KParams &kp, const RankDev &R, const PipeStage &st,
                                            uint32_t (&cur)[kPU]) {
#pragma unroll
    for (int k = 0; k < kPU; ++k)
        cur[k] = st.u[k] < 0 ? 0u : (kp.filter ? filt_probe(R.filt, st.u[k]) : ldg_u32(R.depth + st.u[k]));
}

template <int APP, bool MULTI>
__device__ __forceinline__ void relax_finish(Smem &s, const KParams &kp, int cta, PipeStage &st,
                                             const uint32_t (&cur)[kPU], uint32_t &wn) {
    const RankDev &R = s.R;
    const int w = threadIdx.x >> 5;
    const int64_t vb = R.v_begin, ve = R.v_end;
    const bool fl = kp.filter;
    bool imp[kPU];
#pragma unroll
    for (int k = 0; k < kPU; ++k) {
        const uint32_t nd = st.nd[k], ndw = dw_make(nd);
        const bool maybe = st.u[k] >= 0 && (fl ? filt_pass(cur[k], st.u[k], nd) : ndw < cur[k]);
        imp[k] = false;
        if (maybe) {
            if (kp.relax_red) {
                red_min_u32(R.depth + st.u[k], ndw);
                imp[k] = true;
            } else {
                imp[k] = atom_min_u32(R.depth + st.u[k], ndw) > ndw;
            }
            if (fl && imp[k]) filt_put(R.filt, st.u[k], nd, cur[k]);
        }
    }
    if constexpr (!MULTI) {
        uint32_t msk = 0, item[kPU];
#pragma unroll
        for (int k = 0; k < kPU; ++k) {
            msk |= (imp[k] ? 1u : 0u) << k;
            item[k] = pq_tag((uint32_t)(st.u[k] - vb), st.nd[k], s.pq_th);
        }
        warp_append_mask<kPU>(s, w, wn, msk, item, kp.relax_red);
    } else {
#pragma unroll
        for (int k = 0; k < kPU; ++k) {
            const bool loc = imp[k] && st.u[k] >= vb && st.u[k] < ve;
            if (wn + 32 > (uint32_t)kWOut) warp_flush_local(s, w, wn, kp.relax_red);
            warp_append_local(s, w, wn, loc, pq_tag((uint32_t)(st.u[k] - vb), st.nd[k], s.pq_th));
            bfs_send_remote<APP>(s, kp, cta, w, imp[k] && !loc, st.u[k], st.nd[k], wn);
        }
    }
}

template <int APP, bool MULTI>
__device__ void expand_warp_pipe3(Smem &s, BatchBuf &bb, const KParams &kp, int cta, int B, int64_t E, uint32_t &wn) {
    const int lane = threadIdx.x & 31;
    const RankDev &R = s.R;
    const int32_t *const col = R.col;
    const uint64_t pol = policy_evict_first();
    const uint32_t nchm = (uint32_t)((E + kChunk - 1) / kChunk);
    const uint32_t nch = (uint32_t)((E + kPChunk - 1) / kPChunk);
    auto claim = [&]() {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(&bb.chunk_next, 1u);
        return __shfl_sync(kFull, c, 0);
    };
    PipeStage a, b, c;
    uint32_t ca = claim();
    if (ca >= nch) return;
    pipe_load(bb, B, E, nchm, ca, a, col, pol);
    uint32_t cb = claim();
    const bool hb = cb < nch;
    if (hb) pipe_load(bb, B, E, nchm, cb, b, col, pol);
    uint32_t cur_a[kPU], cur_b[kPU];
    probe_issue<MULTI>(kp, R, a, cur_a);
    bool have_b = hb;
    for (;;) {
        bool have_c = false;
        if (have_b) {
            const uint32_t cc = claim();
            have_c = cc < nch;
            if (have_c) pipe_load(bb, B, E, nchm, cc, c, col, pol);   // columns of chunk i+2
            probe_issue<MULTI>(kp, R, b, cur_b);                     // probes of chunk i+1
        }
        relax_finish<APP, MULTI>(s, kp, cta, a, cur_a, wn);          // chunk i
        if (!have_b) break;
        a = b;
#pragma unroll
        for (int k = 0; k < kPU; ++k) cur_a[k] = cur_b[k];
        b = c;
        have_b = have_c;
    }
}

// Load per-vertex info of the batch s.v[0..B) and expand it.
template <int APP, bool MULTI>
__device__ void process_batch(Smem &s, const KParams &kp, int cta, int B) {
    const RankDev &R = s.R;
    BatchBuf &bb = s.bb[0];
    const int tid = threadIdx.x;
#ifdef ATOS_PROF
    if (tid == 0) s.prof[7] -= (unsigned long long)clock64();
#endif
    int64_t deg = 0;
    uint32_t npc = 0;      // BFS: pieces of this row to publish
    if (tid < B) {
        const uint32_t it = bb.v[tid];
        if (APP == kApBfs && (it & kPieceBit)) {
            // a piece of a split row: edges [piece * split, (piece+1) * split) of v,
            // relaxed with v's current depth (a valid bound: depths only decrease,
            // and a newer depth re-expands the whole row anyway)
            const uint32_t v = it & 0xFFFFu, pc = (it >> 16) & 0x7FFFu;
            const int64_t rb = ldg_i64_nc(R.row_ptr + v), re = ldg_i64_nc(R.row_ptr + v + 1);
            const int64_t b = rb + (int64_t)pc * kp.split;
            bb.beg[tid] = b;
            deg = re - b < (int64_t)kp.split ? re - b : (int64_t)kp.split;
            const uint32_t d = dw_depth(ld_relaxed_gpu_u32(R.depth + R.v_begin + v));
            bb.val[tid] = d;
            if (d == kDepthInf || deg < 0) deg = 0;
        } else {
        const uint32_t v = it;
        const int64_t b = ldg_i64_nc(R.row_ptr + v), e = ldg_i64_nc(R.row_ptr + v + 1);
        bb.beg[tid] = b;
        deg = e - b;
        if constexpr (APP == kApBfs) {
            // claim the expansion of v at its current depth; stale duplicates see
            // the pending bit already cleared and are skipped
            const uint32_t old = atom_and_u32(R.depth + R.v_begin + v, ~1u);
            const uint32_t d = dw_depth(old);
            bb.val[tid] = d;
            if (!(old & 1u) || d == kDepthInf) deg = 0;
            if (kp.split > 0 && deg > 2 * (int64_t)kp.split && (int64_t)v < kPieceVMax &&
                deg <= (int64_t)kp.split * kPieceMax) {
                npc = (uint32_t)((deg - 1) / kp.split);   // pieces 1..npc go to the ring
                deg = kp.split;
            }
        } else {
            const int64_t sl = pr_slot(v, R.pr_q);
            const double r = __longlong_as_double((long long)atom_exch_u64((uint64_t *)(R.pr_res + sl), 0ull));
            if (r != 0.0) red_add_f64(R.pr_rank + sl, r);
            if (r == 0.0 || deg == 0) deg = 0;        // dangling vertices absorb (R4)
            else bb.val[tid] = (uint64_t)__double_as_longlong(kp.alpha * r / (double)deg);
        }
        }
    }
    if (APP == kApBfs && kp.split > 0 && __syncthreads_or(npc > 0)) {
        // publish the pieces before expanding, so idle workers start on them now;
        // T grows before this batch's F, so termination cannot be declared early
        int64_t pex;
        const int64_t ptot = block_exscan(s, (int64_t)npc, pex);
        if (tid == 0) {
            s.b64[2] = atomicAdd((unsigned long long *)q_tail(R, s.pq_q), (unsigned long long)ptot);
            s.c_pushes += (unsigned long long)ptot;
        }
        __syncthreads();
        const uint64_t pbase = s.b64[2] + (uint64_t)pex;
        for (uint32_t i = 0; i < npc; ++i)
            ring_store(R, pbase + i, kPieceBit | ((i + 1) << 16) | bb.v[tid], ring_base_q(s, s.pq_q), s.pq_q);
    }
    if (kp.prefetch && deg > 0) prefetch_l2_bulk(R.col + bb.beg[tid], (uint64_t)deg * 4);
    if (kp.edge_map)
        for (int i = tid; i < kBitW; i += kThreads) bb.bm[i] = 0u;   // ordered before the map by the scan's barriers
    // one scan for both the edge offsets and the compacted index of non-empty rows
    int64_t pexcl;
    const int64_t ptot = block_exscan(s, (deg << 16) | (deg > 0 ? 1 : 0), pexcl);
    const int64_t excl = pexcl >> 16, E = ptot >> 16;
    const bool use_bm = kp.edge_map && E <= kBitE;
    if (tid < B) {
        bb.off[tid] = excl;
        if (deg > 0) {   // chunk -> first vertex map: chunks starting inside this row
            const int64_t cl = (excl + deg - 1) / kChunk;
            for (int64_t c = (excl + kChunk - 1) / kChunk; c <= cl && c < kChunkMap; ++c) bb.chunk_v[c] = (uint16_t)tid;
            if (use_bm) {
                const int nz = (int)(pexcl & 0xFFFF);
                bb.nzslot[nz] = (uint16_t)tid;
                atomicOr(&bb.bm[excl >> 5], 1u << (excl & 31));
                for (int64_t w = (excl + 31) >> 5; w <= ((excl + deg - 1) >> 5); ++w) bb.rowmap[w] = (uint16_t)nz;
            }
        }
    }
    if (tid == 0) { bb.off[B] = E; s.c_edges += (unsigned long long)E; bb.chunk_next = 0; bb.use_bm = use_bm ? 1 : 0; }
    __syncthreads();
#ifdef ATOS_PROF
    if (tid == 0) s.prof[7] += (unsigned long long)clock64();   // minus entry below: setup+scan
#endif
#ifndef ATOS_NO_EARLY
    if (tid == 0 && kp.early && !kp.discrete && s.res_lo == s.res_hi) {
        // reserve the NEXT batch now, while this one is expanded, so the head
        // atomic's round trip leaves the critical path between batches -- only
        // when the ring holds plenty of work (an early reservation withholds
        // items from idle workers)
        const uint64_t t = ld_relaxed_gpu(&R.ctrl->tail.v), h = ld_relaxed_gpu(&R.ctrl->head.v);
        if (t > h && t - h >= 2ull * (uint64_t)kp.ctas_per_rank * (uint64_t)kp.fetch) {
            const uint64_t lo = atomicAdd((unsigned long long *)&R.ctrl->head.v, (unsigned long long)kp.fetch);
            s.res_lo = lo;
            s.res_hi = lo + (uint64_t)kp.fetch;
        }
    }
#endif
    if (E > 0) {
        const int w = tid >> 5;
        uint32_t wn = s.wn[w];
        // pipelined expansion pays off on low-degree (latency-bound, road-like) batches
#ifdef ATOS_PIPE3   // experimental: raises register pressure (stack spills) of the default paths
        if (APP == kApBfs && kp.pipe == 3)
            expand_warp_pipe3<APP, MULTI>(s, bb, kp, cta, B, E, wn);
        else
#endif
        if (APP == kApBfs && (kp.pipe == 1 || (kp.pipe == 2 && E < 16 * (int64_t)B)))
            expand_warp_pipe<APP, MULTI>(s, bb, kp, cta, B, E, wn);
        else expand_warp<APP, MULTI>(s, bb, kp, cta, B, E, wn);
        // without work keeping, each warp enqueues its discoveries as soon as its
        // chunks are done (one atomic per warp) instead of after the batch barrier
        if (kp.keep == 0 && kp.warp_flush) warp_flush_local(s, w, wn, APP == kApBfs && kp.relax_red);
        __syncwarp();
        if ((tid & 31) == 0) s.wn[w] = wn;
    }
}

// Priority-queue batch end (N1): the CTA's discoveries go to the current ring
// (depth below the threshold) or to the other one (far-tagged), one leader
// atomic per ring.  At most kWarps * kWOut = 4 * kThreads items.
__device__ __noinline__ void batch_end_pq(Smem &s, const KParams &kp) {
    const int tid = threadIdx.x;
    if (tid == 0) {
        uint32_t total = 0;
        for (int k = 0; k < kWarps; ++k) { s.wpre[k] = total; total += s.wn[k]; }
        s.wpre[kWarps] = total;
    }
    __syncthreads();
    const uint32_t total = s.wpre[kWarps];
    constexpr int kPer = kWarps * kWOut / kThreads;
    static_assert(kWarps * kWOut % kThreads == 0, "items per thread");
    uint32_t it[kPer];
    uint32_t nn = 0, nf = 0;
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        const uint32_t i = (uint32_t)tid + (uint32_t)j * kThreads;
        it[j] = 0;
        if (i < total) {
            int k = 0;
            while (k + 1 < kWarps && s.wpre[k + 1] <= i) ++k;
            it[j] = s.wout[k][i - s.wpre[k]];
            if (pq_is_far(it[j])) ++nf; else ++nn;
        }
    }
    int64_t ex;
    const int64_t tot = block_exscan(s, ((int64_t)nf << 32) | nn, ex);
    const int q = s.pq_q;
    if (tid == 0) {
        const uint64_t NN = (uint64_t)(tot & 0xFFFFFFFF), NF = (uint64_t)(tot >> 32);
        s.b64[0] = NN ? atomicAdd((unsigned long long *)q_tail(s.R, q), (unsigned long long)NN) : 0ull;
        s.b64[1] = NF ? atomicAdd((unsigned long long *)q_tail(s.R, q ^ 1), (unsigned long long)NF) : 0ull;
        s.c_pushes += NN + NF;
        s.c_far += NF;
    }
    __syncthreads();
    if (kp.relax_red && total > 0) fence_acq_rel_gpu();   // fire-and-forget relaxations are performed first
    uint64_t pn = s.b64[0] + (uint64_t)(ex & 0xFFFFFFFF), pf = s.b64[1] + (uint64_t)(ex >> 32);
#pragma unroll
    for (int j = 0; j < kPer; ++j) {
        const uint32_t i = (uint32_t)tid + (uint32_t)j * kThreads;
        if (i < total) {
            if (pq_is_far(it[j])) ring_store(s.R, pf++, it[j] & ~kFarBit, ring_base_q(s, q ^ 1), q ^ 1);
            else ring_store(s.R, pn++, it[j], ring_base_q(s, q), q);
        }
    }
    __syncthreads();
    if (tid < kWarps) s.wn[tid] = 0;
    __syncthreads();
}

// End of a batch: publish remote staging per policy, then enqueue this CTA's
// local discoveries with one leader atomic -- or keep up to kp.keep of them as
// the next batch (returned count, already in s.v) when the ring is nearly empty.
template <int APP, bool MULTI>
__device__ int batch_end(Smem &s, const KParams &kp, int cta, bool allow_keep) {
    const int tid = threadIdx.x, w = tid >> 5;
    BatchBuf &bb = s.bb[0];
    __syncthreads();
    if constexpr (MULTI) {
        uint32_t wn = s.wn[w];
        wn = warp_flush_remote<APP>(s, kp, cta, w, true, wn);
        __syncwarp();
        if ((tid & 31) == 0) s.wn[w] = wn;
        __syncthreads();
    }
    if (s.pq_th != kNoTh) {         // priority queue (N1): no keeping, split by bucket
        batch_end_pq(s, kp);
        return 0;
    }
    if (tid == 0) {
        uint32_t total = 0;
        for (int k = 0; k < kWarps; ++k) { s.wpre[k] = total; total += s.wn[k]; }
        s.wpre[kWarps] = total;
        uint32_t keep_n = 0;
        if (allow_keep && kp.keep > 0 && total > 0 && total <= (uint32_t)kp.keep) {
            // keep_always: follow the chain (road-like graphs: one queue round trip
            // per level costs more than the redundant relaxations it would avoid,
            // measured 2.1x faster on the grid); otherwise keep only in a
            // low-parallelism phase (T - F tiny) and keep FIFO order, which bounds
            // asynchronous redundancy.
            const uint64_t f = kp.keep_always ? 0 : ld_relaxed_gpu(&s.R.ctrl->finished.v);
            const uint64_t t = kp.keep_always ? 0 : ld_relaxed_gpu(&s.R.ctrl->tail.v);
            if (kp.keep_always || t - f <= (uint64_t)kp.keep) keep_n = total;
        }
        const uint32_t push_n = total - keep_n;
        s.b64[0] = push_n ? atomicAdd((unsigned long long *)&s.R.ctrl->tail.v, (unsigned long long)push_n) : 0ull;
        s.b32[0] = (int32_t)keep_n;
        s.b32[1] = (int32_t)total;
        s.c_pushes += push_n;
    }
    __syncthreads();
    const uint32_t keep_n = (uint32_t)s.b32[0], total = (uint32_t)s.b32[1];
    const uint64_t base = s.b64[0];
    // (no fence: see warp_flush_local; fire-and-forget relaxations need one)
    if (APP == kApBfs && kp.relax_red && total > keep_n) fence_acq_rel_gpu();
    for (uint32_t i = tid; i < total; i += kThreads) {
        int k = 0;
        while (k + 1 < kWarps && s.wpre[k + 1] <= i) ++k;
        const uint32_t item = s.wout[k][i - s.wpre[k]];
        if (i < keep_n) bb.v[i] = item;
        else ring_store(s.R, base + (i - keep_n), item, s.ring_base);
    }
    __syncthreads();
    if (tid < kWarps) s.wn[tid] = 0;
    __syncthreads();
    return (int)keep_n;
}

// Report this CTA's staged-message count change to the rank counter.
__device__ void report_staged(Smem &s, const KParams &kp) {
    if (s.R.n_ranks <= 1) return;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t cur = 0;
        for (int w = 0; w < kWarps; ++w)
            for (int d = 0; d < s.R.n_ranks; ++d) cur += (uint64_t)(s.wst[w][d] - s.wsh[w][d]);
        const uint64_t delta = cur - s.staged_reported;   // mod 2^64
        if (delta != 0) {
            fence_peer(kp.sys);
            atomicAdd((unsigned long long *)&s.R.ctrl->staged.v, (unsigned long long)delta);
            s.staged_reported = cur;
        }
    }
    __syncthreads();
}

#include "atos_bfs1.cuh"

// ---------------------------------------------------------------------------
// pop from the local ring: reserve-then-wait
// ---------------------------------------------------------------------------
// Priority queue (N1; Listing 4 threshold / threshold_delta), leader
// thread: choose the ring to pop from and make sure a reservation is open on it.
// The current ring q = pq_state & 1 holds the bucket below the threshold; the
// other ring collects the discoveries at or above it.  When ring q is drained
// (every item pushed to it finished: F_q == T_q) while the other ring holds
// work, the bucket advances: one CAS increments pq_state, which swaps the roles
// of the rings and raises the threshold by delta.  A reservation left open on
// the other ring (taken before a swap) is still served: every reserved index
// must be consumed.
__device__ __noinline__ void pq_choose(Smem &s, const KParams &kp) {
    const RankDev &R = s.R;
    const uint64_t st = ld_relaxed_gpu(&R.ctrl->pq_state.v);
    const int q = (int)(st & 1);
    const uint64_t k = st - s.pq_k0;
    const uint64_t th = (uint64_t)kp.pq_th0 + k * (uint64_t)kp.pq_delta;
    s.pq_st = st;
    s.pq_q = q;
    s.pq_th = th < (uint64_t)kNoTh ? (uint32_t)th : kNoTh - 1;
    s.pop_q = q;
    if (kp.discrete) {
        // one launch pops ring q up to the snapshot the step kernel took
        uint64_t *hd = q_head(R, q);
        if (s.res_lo == s.res_hi) {
            const uint64_t h = ld_relaxed_gpu(hd);
            if (h < s.limit) {
                uint64_t n = (s.limit - h) / (uint64_t)kp.ctas_per_rank;
                n = n < 1 ? 1 : (n > (uint64_t)kp.fetch ? (uint64_t)kp.fetch : n);
                const uint64_t lo = atomicAdd((unsigned long long *)hd, (unsigned long long)n);
                if (lo < s.limit) {
                    s.res_lo = lo;
                    s.res_hi = lo + n < s.limit ? lo + n : s.limit;
                }
            }
        }
        return;      // (the reservation lives in res_lo / res_hi; its ring is q)
    }
    uint64_t &lo = res_lo_q(s, q), &hi = res_hi_q(s, q);
    if (lo == hi) {
        const uint64_t t = ld_relaxed_gpu(q_tail(R, q)), h = ld_relaxed_gpu(q_head(R, q));
        if (t > h) {
            uint64_t n = (t - h) / (uint64_t)kp.ctas_per_rank;
            n = n < 1 ? 1 : (n > (uint64_t)kp.fetch ? (uint64_t)kp.fetch : n);
            lo = atomicAdd((unsigned long long *)q_head(R, q), (unsigned long long)n);
            hi = lo + n;
        }
    }
    if (lo != hi && slot_full_for(ld_relaxed_gpu(&q_slots(R, q)[lo & (R.ring_cap - 1)]), lo)) {
        // The item may belong to a later bucket if ring q was swapped out since st
        // was read (items still in a ring at a swap were all pushed after it: the
        // ring was drained).  Re-read the state (the load is issued after the slot
        // was seen full); if it moved, the batch goes back to its ring unexpanded.
        if (ld_relaxed_gpu(&R.ctrl->pq_state.v) != st) s.pq_q = q ^ 1;
        return;
    }
    // A reservation that overshot a ring's tail and is still open when the ring
    // becomes the other bucket's (after a swap) receives that bucket's items.  They
    // are popped (the reserved indices must be consumed) but not expanded -- their
    // depth may not be final yet -- and go back to the end of that ring
    // (pq_recycle), which also frees the worker's reservation.
    const int o = q ^ 1;
    const uint64_t lo2 = res_lo_q(s, o), hi2 = res_hi_q(s, o);
    if (lo2 != hi2 && slot_full_for(ld_relaxed_gpu(&q_slots(R, o)[lo2 & (R.ring_cap - 1)]), lo2)) {
        s.pop_q = o;
        return;
    }
    // nothing ready: advance the bucket if ring q is drained and ring o holds work
    const uint64_t f = ld_acquire_gpu(q_fin(R, q));
    const uint64_t t = ld_acquire_gpu(q_tail(R, q));
    if (f == t && ld_relaxed_gpu(q_tail(R, o)) > ld_relaxed_gpu(q_fin(R, o)))
        atomicCAS((unsigned long long *)&R.ctrl->pq_state.v, (unsigned long long)st, (unsigned long long)(st + 1));
}

// Priority queue: a batch popped from the NON-current ring (an old reservation,
// see pq_choose) goes back to the end of that ring unexpanded.  Whole CTA.
__device__ __noinline__ void pq_recycle(Smem &s, int B) {
    const int tid = threadIdx.x, q = s.pop_q;
    if (tid == 0) {
        s.b64[0] = atomicAdd((unsigned long long *)q_tail(s.R, q), (unsigned long long)B);
        s.c_pushes += (unsigned long long)B;
    }
    __syncthreads();
    if (tid < B) ring_store(s.R, s.b64[0] + (uint64_t)tid, s.bb[0].v[tid], ring_base_q(s, q), q);
    __syncthreads();
}

__device__ int pop_batch(Smem &s, const KParams &kp) {
    const RankDev &R = s.R;
    const int tid = threadIdx.x;
    BatchBuf &bb = s.bb[0];
    if (tid == 0) {
        if (kp.pq) {
            pq_choose(s, kp);
        } else if (s.res_lo == s.res_hi && kp.discrete) {
            // discrete mode: reserve with atomicAdd and clip at the launch's snapshot,
            // so every reserved slot is already published; head may overshoot the
            // limit and is set back to it by discrete_step_kernel (a CAS loop here
            // measured ~1.3 us per success under 296-way contention)
            const uint64_t h = ld_relaxed_gpu(&R.ctrl->head.v);
            if (h < s.limit) {
                uint64_t k = (s.limit - h) / (uint64_t)kp.ctas_per_rank;
                k = k < 1 ? 1 : (k > (uint64_t)kp.fetch ? (uint64_t)kp.fetch : k);
                const uint64_t lo = atomicAdd((unsigned long long *)&R.ctrl->head.v, (unsigned long long)k);
                if (lo < s.limit) {
                    s.res_lo = lo;
                    s.res_hi = lo + k < s.limit ? lo + k : s.limit;
                }
            }
        } else if (s.res_lo == s.res_hi) {
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
    // ring of this pop: 0 without the priority queue; in discrete pq mode the
    // reservation is kept in res_lo/hi for ring pq_q
    const int q = s.pop_q;
    const bool dq = kp.pq && kp.discrete;
    const uint64_t lo = dq ? s.res_lo : res_lo_q(s, q);
    const uint64_t avail = (dq ? s.res_hi : res_hi_q(s, q)) - lo;
    uint64_t *const ring = q_slots(R, q);
    const int cnt = (int)(avail < (uint64_t)kp.fetch ? avail : (uint64_t)kp.fetch);
    const uint64_t idx = lo + tid;
    uint64_t slot = 0;
    if (tid < cnt) {
        slot = ring_read(ring, R.ring_cap, idx);
        if (!slot_full_for(slot, idx)) atomicMin(&s.minbad, tid);
    }
    __syncthreads();
    const int B = cnt < s.minbad ? cnt : s.minbad;
    if (tid < B) {
        // no acquire fence: the vertex state is only accessed through L2 atomics
        // whose address depends on this slot value (see warp_flush_local)
        bb.v[tid] = lo32(slot);
        ring_release(ring, R.ring_cap, idx);
    }
    __syncthreads();
    if (tid == 0) {
        if (dq) s.res_lo = lo + (uint64_t)B;
        else res_lo_q(s, q) = lo + (uint64_t)B;
    }
    return B;
}

// ---------------------------------------------------------------------------
// termination (multi-rank): coordinator double wave
// ---------------------------------------------------------------------------
// Rank 0, CTA 0, warp 0 reads every rank's (F, R, T, staged, S); done when two
// consecutive waves are identical, every rank is passive (F == T, staged == 0)
// and sum S == sum R (Mattern's four-counter method).
__device__ void coordinator_step(Smem &s, const KParams &kp) {
    const RankDev &R = s.R;
    if (threadIdx.x >= 32) return;
    const int lane = threadIdx.x;
    const int p = R.n_ranks;
    bool started = true;
    uint64_t F = 0, Rv = 0, T = 0, St = 0, S = 0;
    if (lane < p) {
        started = ld_acquire_peer(kp.sys, &R.ctrl->started[lane].v) == kp.epoch;
        const Ctrl *c = R.peer_ctrl[lane];
        F = ld_acquire_peer(kp.sys, &c->finished.v);
        if (kp.pq) F += ld_acquire_peer(kp.sys, &c->pq_fin.v);
        Rv = ld_acquire_peer(kp.sys, &c->recvd.v);
        T = ld_acquire_peer(kp.sys, &c->tail.v);
        if (kp.pq) T += ld_acquire_peer(kp.sys, &c->pq_tail.v);
        St = ld_acquire_peer(kp.sys, &c->staged.v);
        S = ld_acquire_peer(kp.sys, &c->sent.v);
    }
    if (!__all_sync(kFull, started)) {
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
        sumS += __shfl_xor_sync(kFull, sumS, d);
        sumR += __shfl_xor_sync(kFull, sumR, d);
    }
    const bool all_same = __all_sync(kFull, same);
    const bool all_passive = __all_sync(kFull, passive);
    __syncwarp();
    if (lane < p) {
        s.wave[lane][0] = F; s.wave[lane][1] = Rv; s.wave[lane][2] = T;
        s.wave[lane][3] = St; s.wave[lane][4] = S;
    }
    if (lane == 0) s.wave_valid = all_passive && sumS == sumR;
    if (all_same && all_passive && sumS == sumR) {
        if (lane < p) st_release_peer(kp.sys, &R.peer_ctrl[lane]->done.v, kp.epoch);
    }
    if (lane == 0) atomicAdd((unsigned long long *)&R.ctrl->st_waves.v, 1ull);
    __syncwarp();
}

// ---------------------------------------------------------------------------
// the persistent worker
// ---------------------------------------------------------------------------
template <int APP, bool MULTI>
__device__ __forceinline__ void worker_body(Smem &s, const KParams &kp) {
    const int lr = blockIdx.x / kp.ctas_per_rank;
    const int cta = blockIdx.x % kp.ctas_per_rank;
    const int tid = threadIdx.x, w = tid >> 5;
    if (tid == 0) {
        s.R = kp.ranks[lr];
        s.res_lo = s.res_hi = 0;
        s.res2_lo = s.res2_hi = 0;
        s.ring_base = s.R.ctrl->ring_base.v;
        s.ring2_base = s.R.ctrl->pq_base.v;
        s.pq_q = s.pop_q = 0;
        s.pq_st = 0;
        s.pq_th = kNoTh;
        s.pq_k0 = 0;
        if (kp.pq) {        // the bucket at the start of the launch (pop_batch re-reads it)
            const uint64_t st = ld_relaxed_gpu(&s.R.ctrl->pq_state.v);
            s.pq_k0 = ld_relaxed_gpu(&s.R.ctrl->pq_k0.v);      // fixed for the solve (seed kernel)
            const uint64_t th = (uint64_t)kp.pq_th0 + (st - s.pq_k0) * (uint64_t)kp.pq_delta;
            s.pq_q = s.pop_q = (int)(st & 1);
            s.pq_th = th < (uint64_t)kNoTh ? (uint32_t)th : kNoTh - 1;
        }
        s.staged_reported = 0;
        s.wave_valid = 0;
        s.c_pops = s.c_edges = s.c_pushes = s.c_msgs = s.c_packets = s.c_idle = s.c_hub = s.c_far = 0;
        s.c_busy = s.c_batches = 0;
        s.limit = kp.discrete ? ld_relaxed_gpu(&s.R.ctrl->limit.v) : 0;
#ifdef ATOS_PROF
        for (int k = 0; k < 10; ++k) s.prof[k] = 0;
#endif
    }
    if (tid < kWarps) {
        s.wn[tid] = 0;
        for (int d = 0; d < kMaxRanks; ++d) { s.wst[tid][d] = s.wsh[tid][d] = 0; s.wt0[tid][d] = 0; }
    }
    if (APP == kApBfs && !MULTI && tid == 0) hub_mbar_init(s);   // hub bounds: TMA completion barrier
    if (APP == kApBfs && !MULTI && (kp.hub_dbg & 2)) hub_fill_unknown(s, kp);
    __syncthreads();
    constexpr bool multi = MULTI;
    const bool coordinator = multi && s.R.rank == 0 && cta == 0;
    if (tid == 0 && cta == 0) st_release_peer(kp.sys, &s.R.peer_ctrl[0]->started[s.R.rank].v, kp.epoch);
    const uint64_t t_start = globaltimer();
    uint32_t idle_streak = 0;

    if (kp.fault && tid == 0 && cta == 0 && s.R.rank == 0)     // test-only fault injection (T6 error paths)
        set_error(s.R, kp.fault == kFaultCapacity ? kErrCapacity : kErrTimeout);
    for (;;) {
        if (tid == 0) {
            int f = 0;
            if (ld_relaxed_gpu(&s.R.ctrl->done.v) == kp.epoch) f = 1;
            if (ld_relaxed_gpu(&s.R.ctrl->error.v) != 0) f = 2;
            // the watchdog is checked on every iteration, busy or idle: a solve that
            // never idles must still be stopped
            if (kp.watchdog_ns > 0 && globaltimer() - t_start > (uint64_t)kp.watchdog_ns) {
                set_error(s.R, kErrTimeout);
                f = 2;
            }
            s.flag = f;
        }
        __syncthreads();
        if (s.flag) break;

        const uint64_t t_work0 = (tid == 0) ? globaltimer() : 0;
        bool worked = false;
        if constexpr (multi) worked = cta_inbound<APP>(s, kp, cta);
        if (!worked) {
#ifdef ATOS_PROF
            const long long pb0 = clock64();
#endif
            int B = pop_batch(s, kp);
#ifdef ATOS_PROF
            if (tid == 0 && B > 0) s.prof[6] += (unsigned long long)(clock64() - pb0);
#endif
            if (B > 0) {
                const int B0 = B;
                if (kp.pq && s.pop_q != s.pq_q) {      // not this bucket's: back to its ring
                    pq_recycle(s, B);
                    B = 0;
                }
                int chain = 0;
                while (B > 0) {                 // work-keeping chain
                    if (tid == 0) s.c_pops += B;
#ifdef ATOS_PROF
                    const long long pb1 = clock64();
#endif
                    if constexpr (APP == kApBfs && !MULTI) {
                        if (kp.bfs1) process_batch_bfs1(s, kp, cta, B);
                        else process_batch<APP, MULTI>(s, kp, cta, B);
                    } else {
                        process_batch<APP, MULTI>(s, kp, cta, B);
                    }
#ifdef ATOS_PROF
                    const long long pb2 = clock64();
                    if (tid == 0) s.prof[8] += (unsigned long long)(pb2 - pb1);
#endif
                    // a chain of kept batches is bounded (keep_chain): an unbounded
                    // chain runs ahead of the wavefront and finds too-large depths
                    B = batch_end<APP, MULTI>(s, kp, cta, ++chain < kp.keep_chain);
#ifdef ATOS_PROF
                    if (tid == 0) s.prof[9] += (unsigned long long)(clock64() - pb2);
#endif
                }
                report_staged(s, kp);
#ifdef ATOS_PROF
                if (tid == 0) { s.prof[5] += (unsigned long long)(clock64() - pb0); }
#endif
                if (tid == 0) {
                    // T (returned by its atomic before the slot stores) is performed
                    // before this F update is issued; multi-rank adds a sys fence
                    // because the coordinator reads these counters over NVLink
                    if (multi) fence_peer(kp.sys);
                    atomicAdd((unsigned long long *)q_fin(s.R, s.pop_q), (unsigned long long)B0);  // F last
                }
                worked = true;
            }
        }
        if (worked) {
            if (tid == 0) { s.c_busy += globaltimer() - t_work0; s.c_batches++; }
            idle_streak = 0;
            continue;
        }

        // ---- idle: flush aged staging, detect termination, watchdog
        if (kp.discrete) break;   // discrete launch: the snapshot is drained (nothing reserved, head == limit)
        ++idle_streak;
        if constexpr (multi) {
            uint32_t wn = s.wn[w];
            wn = warp_flush_remote<APP>(s, kp, cta, w, true, wn);
            warp_flush_local(s, w, wn, false);
            if ((tid & 31) == 0) s.wn[w] = wn;
            report_staged(s, kp);
        }
        if (tid == 0) {
            s.c_idle++;
            if (!multi) {
                // F before T (per ring; F_q <= T_q always): equal sums mean every pushed
                // item had finished and nothing could produce more
                uint64_t F = ld_acquire_gpu(&s.R.ctrl->finished.v);
                if (kp.pq) F += ld_acquire_gpu(&s.R.ctrl->pq_fin.v);
                uint64_t T = ld_acquire_gpu(&s.R.ctrl->tail.v);
                if (kp.pq) T += ld_acquire_gpu(&s.R.ctrl->pq_tail.v);
                if (F == T) st_release_gpu(&s.R.ctrl->done.v, kp.epoch);
            }
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
        atomicAdd((unsigned long long *)&c->st_hub_hits.v, s.c_hub);
        atomicAdd((unsigned long long *)&c->st_busy_ns.v, s.c_busy);
        atomicAdd((unsigned long long *)&c->st_batches.v, s.c_batches);
        if (s.c_far) atomicAdd((unsigned long long *)&c->st_far.v, s.c_far);
#ifdef ATOS_PROF
        if (blockIdx.x < 4)
            printf("PROF cta %d chunks %llu col %llu probe %llu atom %llu append %llu (cyc/chunk/warp) | per batch: pop %llu setup %llu expand(t0) %llu end %llu total %llu batches %llu\n",
                   blockIdx.x, s.prof[4], s.prof[0] / (s.prof[4] + 1), s.prof[1] / (s.prof[4] + 1),
                   s.prof[2] / (s.prof[4] + 1), s.prof[3] / (s.prof[4] + 1), s.prof[6] / (s.c_batches + 1),
                   s.prof[7] / (s.c_batches + 1), s.prof[8] / (s.c_batches + 1), s.prof[9] / (s.c_batches + 1),
                   s.prof[5] / (s.c_batches + 1), s.c_batches);
#endif
    }
}

// The persistent worker (one cooperative launch per solve).
template <int APP, bool MULTI>
__global__ void __launch_bounds__(kThreads, kMinBlocks) worker_kernel(const __grid_constant__ KParams kp) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    worker_body<APP, MULTI>(*reinterpret_cast<Smem *>(smem_raw), kp);
}

// Discrete-kernel mode: one launch per queue snapshot, replayed by
// a CUDA-graph while-node; the per-solve parameters live in device memory so the
// instantiated graph never changes.
template <int APP>
__global__ void __launch_bounds__(kThreads, kMinBlocks) worker_discrete_kernel(const KParams *kpp) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ KParams kps;
    if (threadIdx.x == 0) kps = *kpp;
    __syncthreads();
    worker_body<APP, false>(*reinterpret_cast<Smem *>(smem_raw), kps);
}

// Between discrete launches: snapshot the tail as the next launch's limit and keep
// looping while the queue holds work (and no device error was raised).
__global__ void discrete_step_kernel(const KParams *kpp, cudaGraphConditionalHandle h, int after_launch) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const RankDev &R = kpp->ranks[0];
    // the ring of this launch: 0, or the current bucket's ring (priority queue)
    int q = kpp->pq ? (int)(R.ctrl->pq_state.v & 1) : 0;
    // after a launch every index below the old limit was consumed; reservations
    // past it were clipped, so head goes back to the limit
    if (after_launch && *q_head(R, q) > R.ctrl->limit.v) *q_head(R, q) = R.ctrl->limit.v;
    uint64_t t = ld_relaxed_gpu(q_tail(R, q)), hd = ld_relaxed_gpu(q_head(R, q));
    if (kpp->pq && t == hd && ld_relaxed_gpu(q_tail(R, q ^ 1)) > ld_relaxed_gpu(q_head(R, q ^ 1))) {
        // the bucket is drained (a launch retires everything below its limit):
        // advance it -- the other ring becomes current, the threshold grows by delta
        R.ctrl->pq_state.v += 1;
        q ^= 1;
        t = ld_relaxed_gpu(q_tail(R, q));
        hd = ld_relaxed_gpu(q_head(R, q));
    }
    R.ctrl->limit.v = t;
    const bool more = t > hd && ld_relaxed_gpu(&R.ctrl->error.v) == 0;
    if (more) R.ctrl->st_waves.v += 1;          // = worker launches of the solve
    cudaGraphSetConditional(h, more ? 1u : 0u);
}

}  // namespace atos
