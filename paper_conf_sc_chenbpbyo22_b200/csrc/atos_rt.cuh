// atos_rt.cuh -- device runtime primitives for the persistent Atos worker.
//
// Memory-model wrappers (system/gpu scope acquire/release, fences, globaltimer),
// the per-rank control block, the device-side rank view, and the lock-free
// ring queue (Sec. III-A2 + Listing 6) re-designed for
// sm_100a:  u64 monotone indices, one leader atomic per CTA worker, and
// self-validating 8-byte slots {seq:32 | item:32} so that publication needs no
// separate end/end_max/end_count counters (reading R15).
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace atos {

constexpr int kMaxRanks = 8;
constexpr int kMaxSub = 8;                    // sub-channels per (source, destination) pair
constexpr uint32_t kInf = 0xFFFFFFFFu;        // BFS word of an undiscovered vertex
constexpr uint32_t kDepthInf = 0x7FFFFFFFu;   // its depth field

// BFS per-vertex word: (depth << 1) | pending.  `pending` is set by every
// improving atomicMin and cleared (atomicAnd) by the one pop that expands the
// vertex at that depth, so stale duplicate queue entries are skipped without a
// second array.  Ordering by the word == ordering by depth for improvements:
// atomicMin(w, dw(nd)) > dw(nd)  <=>  depth(w) > nd.
__device__ __forceinline__ uint32_t dw_make(uint32_t d) { return (d << 1) | 1u; }
__device__ __forceinline__ uint32_t dw_depth(uint32_t w) { return w >> 1; }

// BFS probe filter (used when the depth words do not fit the L2 carve-out, e.g.
// RMAT-26: 268 MB of words vs 67 MB of filter): one byte per vertex holding an
// upper bound of its depth, saturated at 255.  It is written after every
// improvement with the new candidate depth; racing stores can only leave a larger
// value, never one below the true depth, so filt[u] <= nd (unsaturated) proves the
// edge cannot improve u.
__device__ __forceinline__ uint8_t filt_of(uint32_t d) { return d < 255u ? (uint8_t)d : (uint8_t)255; }
__device__ __forceinline__ bool filt_maybe(uint32_t f, uint32_t nd) { return nd < f || f == 255u; }
__device__ __forceinline__ uint32_t ldg_u8(const uint8_t *p) {
    uint16_t v;
    asm volatile("ld.global.u8 %0, [%1];" : "=h"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ void stg_u8(uint8_t *p, uint32_t x) {
    asm volatile("st.global.u8 [%0], %1;" ::"l"(p), "h"((uint16_t)x));
}
// Filter access.  Default: one byte per vertex.  ATOS_FILTER4 (experiment): one
// nibble per vertex (bound saturated at 15), half the footprint; the update is a
// racy read-modify-write of the byte, which can only leave an older -- still
// valid, larger -- bound in either nibble.  filt_probe returns the raw byte.
#ifndef ATOS_FILTER4
#define ATOS_FILTER4 0
#endif
__device__ __forceinline__ uint32_t filt_probe(const uint8_t *f, int64_t u) { return ldg_u8(f + (ATOS_FILTER4 ? (u >> 1) : u)); }
__device__ __forceinline__ uint32_t filt_val(uint32_t raw, int64_t u) {
    return ATOS_FILTER4 ? (raw >> ((u & 1) * 4)) & 15u : raw;
}
__device__ __forceinline__ bool filt_pass(uint32_t raw, int64_t u, uint32_t nd) {
    const uint32_t fv = filt_val(raw, u);
    return nd < fv || fv == (ATOS_FILTER4 ? 15u : 255u);
}
__device__ __forceinline__ void filt_put(uint8_t *f, int64_t u, uint32_t nd, uint32_t raw) {
    if (ATOS_FILTER4) {
        const int sh = (int)(u & 1) * 4;
        const uint32_t x = nd < 15u ? nd : 15u;
        stg_u8(f + (u >> 1), (raw & ~(15u << sh) & 0xFFu) | (x << sh));
    } else {
        stg_u8(f + u, filt_of(nd));
    }
}
__device__ __forceinline__ void filt_put_fresh(uint8_t *f, int64_t u, uint32_t nd) {
    filt_put(f, u, nd, ATOS_FILTER4 ? ldg_u8(f + (u >> 1)) : 0u);
}

#ifndef ATOS_THREADS
#define ATOS_THREADS 512
#endif
constexpr int kThreads = ATOS_THREADS;   // CTA worker
constexpr int kWarps = kThreads / 32;

// ---------------------------------------------------------------------------
// memory model
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_gpu_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_gpu(uint64_t *p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Peer-visible accesses at the scope the peers need: other GPUs / processes need
// .sys; virtual ranks (all peers on this device) need only .gpu, whose fences do
// not drain to the system level (MEMBAR.GPU instead of MEMBAR.SYS).  `sys` is
// uniform per launch (KParams::sys).
__device__ __forceinline__ uint64_t ld_acquire_peer(bool sys, const uint64_t *p) {
    return sys ? ld_acquire_sys(p) : ld_acquire_gpu(p);
}
__device__ __forceinline__ uint64_t ld_relaxed_peer(bool sys, const uint64_t *p) {
    return sys ? ld_relaxed_sys(p) : ld_relaxed_gpu(p);
}
__device__ __forceinline__ uint32_t ld_relaxed_peer_u32(bool sys, const uint32_t *p) {
    uint32_t v;
    if (sys) asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    else asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_peer(bool sys, uint64_t *p, uint64_t v) {
    if (sys) st_release_sys(p, v); else st_release_gpu(p, v);
}
__device__ __forceinline__ void st_relaxed_peer(bool sys, uint64_t *p, uint64_t v) {
    if (sys) st_relaxed_sys(p, v); else st_relaxed_gpu(p, v);
}
__device__ __forceinline__ void fence_peer(bool sys) {
    if (sys) fence_acq_rel_sys(); else fence_acq_rel_gpu();
}

// Explicit global-space accesses.  The rank view lives in shared memory, so the
// compiler cannot prove its pointers are global and would emit generic LD/ATOM;
// these force LDG / ATOMG without a "memory" clobber (no forced smem reloads).
#ifndef ATOS_PROBE_L1
#define ATOS_PROBE_L1 1
#endif
__device__ __forceinline__ uint32_t ldg_u32(const uint32_t *p) {   // weak load (probes)
    uint32_t v;
#if ATOS_PROBE_L1
    asm volatile("ld.global.b32 %0, [%1];" : "=r"(v) : "l"(p));
#else
    asm volatile("ld.global.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
#endif
    return v;
}
__device__ __forceinline__ uint32_t atom_min_u32(uint32_t *p, uint32_t x) {
    uint32_t o;
    asm volatile("atom.global.min.u32 %0, [%1], %2;" : "=r"(o) : "l"(p), "r"(x));
    return o;
}
__device__ __forceinline__ void red_min_u32(uint32_t *p, uint32_t x) {
    asm volatile("red.global.min.u32 [%0], %1;" ::"l"(p), "r"(x));
}
__device__ __forceinline__ uint32_t atom_and_u32(uint32_t *p, uint32_t x) {
    uint32_t o;
    asm volatile("atom.global.and.b32 %0, [%1], %2;" : "=r"(o) : "l"(p), "r"(x));
    return o;
}
__device__ __forceinline__ double atom_add_f64(double *p, double x) {
    double o;
    asm volatile("atom.global.add.f64 %0, [%1], %2;" : "=d"(o) : "l"(p), "d"(x));
    return o;
}
__device__ __forceinline__ double atom_add_f64_sys(double *p, double x) {
    double o;
    asm volatile("atom.sys.global.add.f64 %0, [%1], %2;" : "=d"(o) : "l"(p), "d"(x));
    return o;
}
__device__ __forceinline__ void red_add_f64(double *p, double x) {
    asm volatile("red.global.add.f64 [%0], %1;" ::"l"(p), "d"(x));
}
__device__ __forceinline__ uint64_t atom_exch_u64(uint64_t *p, uint64_t x) {
    uint64_t o;
    asm volatile("atom.global.exch.b64 %0, [%1], %2;" : "=l"(o) : "l"(p), "l"(x));
    return o;
}
__device__ __forceinline__ int64_t ldg_i64_nc(const int64_t *p) {   // read-only data (row offsets)
    int64_t v;
    asm volatile("ld.global.nc.b64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

// TMA bulk prefetch of [p, p+bytes) into L2 (sm_90+): one instruction per
// adjacency list, so the column stream is already in L2 when the warps reach it.
__device__ __forceinline__ void prefetch_l2_bulk(const void *p, uint64_t bytes) {
    const uint64_t end = ((uint64_t)p + bytes + 15) & ~(uint64_t)15;
    for (uint64_t x = (uint64_t)p & ~(uint64_t)15; x < end; x += (1u << 20)) {
        const uint32_t c = end - x > (1u << 20) ? (1u << 20) : (uint32_t)(end - x);
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(x), "r"(c));
    }
}

// L2-only (bypass the non-coherent L1) loads for data produced by other SMs/GPUs.
__device__ __forceinline__ uint64_t ld_cg_u64(const uint64_t *p) { return __ldcg((const unsigned long long *)p); }
__device__ __forceinline__ uint2 ld_cg_u2(const uint2 *p) { return __ldcg(p); }
__device__ __forceinline__ uint4 ld_cg_u4(const uint4 *p) { return __ldcg(p); }

__device__ __forceinline__ uint32_t lo32(uint64_t x) { return (uint32_t)x; }
__device__ __forceinline__ uint32_t hi32(uint64_t x) { return (uint32_t)(x >> 32); }
__device__ __forceinline__ uint64_t pack(uint32_t hi, uint32_t lo) { return ((uint64_t)hi << 32) | lo; }

// ---------------------------------------------------------------------------
// control block: every counter on its own 128-byte line
// ---------------------------------------------------------------------------
constexpr int kTimeline = 64;

struct alignas(128) Line {
    uint64_t v;
    uint64_t pad_[15];
};

enum DevError : uint64_t { kErrNone = 0, kErrCapacity = 4, kErrTimeout = 5 };
// test-only fault injection (KParams::fault, env ATOS_TEST_FAULT): raise this error at worker start
enum FaultKind : int32_t { kFaultNone = 0, kFaultCapacity = 1, kFaultTimeout = 2 };

struct Ctrl {
    Line head;                   // local ring: next index to reserve for pop
    Line tail;                   // local ring: next index to reserve for push (T)
    Line finished;               // local ring entries fully processed (F)
    Line staged;                 // messages sitting in CTA staging buffers
    Line sent;                   // messages published to peer channels (S)
    Line recvd;                  // inbound messages fully processed (R)
    Line done;                   // epoch of the finished solve (set by coordinator)
    Line error;                  // DevError of the current solve
    Line started[kMaxRanks];     // [coordinator only] epoch each rank started
    Line bar[kMaxRanks];         // pre-init barrier arrivals (epoch per rank)
    Line out_reserve[kMaxRanks * kMaxSub]; // packets reserved on sub-channel (this -> d, k) at [d * nsub + k]
    Line in_cursor[kMaxRanks * kMaxSub];   // next packet to consume on sub-channel (s -> this, k)
    Line ring_base;              // tail at the start of the current solve
    // priority queue (Listing 4's DistributedPriorityQueues,
    // P:629-639): a second ring with its own head / tail / finished counters.
    // pq_state counts bucket advances (monotone across solves): the CURRENT ring
    // is pq_state & 1, the threshold th0 + (pq_state - pq_k0) * delta.
    Line pq_head, pq_tail, pq_fin, pq_base, pq_state, pq_k0;
    Line limit;                  // discrete mode: queue snapshot this launch may pop up to
    Line st_pops, st_edges, st_pushes, st_msgs, st_packets, st_idle, st_hub_hits, st_waves;
    Line st_busy_ns, st_batches, st_far;
    // experiment (ATOS_TIMELINE=<bucket us>): edges / batches / pops started per time bucket of a solve
    uint64_t tl_t0;
    uint64_t tl_edges[kTimeline], tl_batches[kTimeline], tl_pops[kTimeline];
};

// Per-rank device view.  One per rank served by the grid (virtual ranks: many).
struct RankDev {
    int32_t rank, n_ranks;
    int64_t n;                   // global vertex count
    int64_t v_begin, v_end;      // owned global range [v_begin, v_end)
    int64_t part[kMaxRanks + 1]; // global partition offsets
    const int64_t *row_ptr;      // [n_r + 1] offsets into col (rank-local rows)
    const int32_t *col;          // [m_r] global vertex ids
    // application state (own memory)
    uint32_t *depth;             // BFS: [n] global-indexed words dw (owned + ghost filter)
    uint8_t *filt;               // BFS: [n] probe filter, an upper bound of depth saturated at 255
    uint8_t *hcb;                // BFS hub bounds: [hub_chunks] upper bound of max filt over 128 hub ids
    uint32_t *vis;               // BFS visited bitmap [n/32 + 1] (level-synchronous priority queue, KParams::vis)
    double *pr_rank;             // PR: [n_r], stored at pr_slot(local id)
    double *pr_res;              // PR: [n_r], stored at pr_slot(local id)
    double *pr_ghost;            // PR combining: [n] unsent residual for remote vertices, at pr_slot(global id, pr_q_of(n)); NULL = off
    int64_t pr_q;                // PR slot spreading: n_r / 8 (0 = identity), see pr_slot
    // local ring (own memory)
    uint64_t *ring;
    uint64_t *ring2;             // priority queue: the second ring (same capacity); NULL = FIFO
    uint64_t ring_cap;           // power of two
    Ctrl *ctrl;                  // own control block
    Ctrl *peer_ctrl[kMaxRanks];  // control block of every rank (own included)
    // channels; a packet = hdr word {seq:32|count:32} + payload of pkt msgs
    uint64_t *in_hdr[kMaxRanks];       // own memory: inbound from s
    unsigned char *in_payload[kMaxRanks];
    uint64_t *out_hdr[kMaxRanks];      // peer memory: d's in_hdr[rank]
    unsigned char *out_payload[kMaxRanks];
    uint64_t *free_mirror[kMaxRanks];  // own memory: free tags of packets of channel (this -> d)
    uint64_t *peer_free[kMaxRanks];    // peer memory: s's free_mirror[rank]
    // CTA-private staging of outbound messages [cta][dst][stage_cap] (own memory)
    unsigned char *staging;
    // degree relabeling (graph_load); NULL = identity.
    // Vertex ids inside the path are the NEW ids; outputs are mapped back.
    const int32_t *perm;         // [n] old id -> new id
    const int32_t *inv;          // [n] new id -> old id
    // peer state for the final gather
    uint32_t *peer_depth[kMaxRanks];
    double *peer_rank[kMaxRanks];
    double *peer_res[kMaxRanks];
    double *peer_ghost[kMaxRanks];
};

struct KParams {
    RankDev *ranks;          // device array, one per rank in this grid
    int32_t n_local;         // ranks served by this grid (virtual ranks)
    int32_t ctas_per_rank;
    int32_t fetch;           // vertices per pop batch (<= kThreads)
    int32_t pkt;             // messages per packet
    int32_t cp;              // packets per channel (pow2) = nsub sub-channels of cps packets
    int32_t nsub, cps;       // sub-channels per channel, packets per sub-channel (pow2)
    int32_t stage_cap;       // staging capacity per (cta, warp, dst), messages (pow2)
    int32_t agg_on;
    int32_t keep;            // max discovered items a worker keeps for itself (work-keeping chain)
    int32_t keep_always;     // 1: keep whenever <= keep discovered; 0: only when the rank's T - F <= keep
    int32_t keep_chain;      // max consecutive kept batches before the discoveries go to the ring
    int32_t prefetch;        // TMA bulk-prefetch each popped adjacency list into L2
    int32_t relax_red;       // BFS: fire-and-forget red.min, enqueue on the probe's verdict
    int32_t pipe;            // BFS: software-pipelined expansion (two 128-edge chunks in flight)
    int32_t filter;          // BFS: probe the u8 filter instead of the depth words
    int32_t hub_n;           // BFS hub bounds: vertex ids [0, hub_n) covered (multiple of 2048; 0 = off)
    int32_t hub_chunks;      // hub_n / 128
    int32_t bfs1;            // single-rank BFS: the lean expansion of atos_bfs1.cuh (else the generic one)
    int32_t hub_dbg;         // experiment (ATOS_HUB_DBG): 1 no re-scan, 2 no copy, 4 no per-edge test
    int64_t timeline_ns;     // experiment (ATOS_TIMELINE): bucket width of the per-solve work timeline (0 = off)
    int32_t split;           // BFS row pieces: edges per piece (0 = off), see kPieceBit
    int32_t combine;         // PR sender-side residual combining (multi-rank)
    int32_t discrete;        // discrete-kernel mode: pop only below ctrl->limit, exit when drained
    int32_t sys;             // peers are other devices/processes: system-scope ordering (else .gpu)
    int32_t early;           // reserve the next batch during expansion
    int32_t pq_early;        // level buckets: reserve the next batch on the current ring during expansion
    int32_t pr_ratom;        // multi-rank PR: remote deltas applied by atomics in the owner's memory, messages only for crossings
    int32_t bfs_ratom;       // multi-rank BFS: improvements applied by atomicMin in the owner's memory, activations only
    int32_t warp_flush;      // per-warp enqueue right after expansion (no keeping)
    int32_t edge_map;        // build the per-batch edge -> row bitmap map (batches <= kBitE edges)
    int32_t static_chunks;   // expand_warp: round-robin chunks per warp instead of claiming
    int32_t fault;           // test-only fault injection (FaultKind), raised by rank 0 CTA 0 at start
    int32_t pq;              // BFS priority queue (N1): items of depth >= threshold go to the other ring
    uint32_t pq_th0;         // initial threshold (depths < pq_th0 form the first bucket)
    uint32_t pq_delta;       // threshold_delta: the threshold grows by this at every bucket advance
    int32_t vis;             // single-rank BFS with pq_delta 1 (buckets = levels): visited bitmap instead
                             // of depth words + probe filter (see atos_bfs1.cuh "visited bitmap")
    int32_t vis_claim;       // with vis: discoveries are fire-and-forget red.or, the expansion is claimed
                             // at pop in a second bitmap (atos_bfs1.cuh "claim at pop")
    int64_t agg_age_ns;
    int64_t watchdog_ns;
    uint64_t epoch;
    double alpha, eps;       // PageRank
    double eps_g;            // PR combining: a ghost residual is sent when it crosses eps_g = eps / n_ranks
};

// ---------------------------------------------------------------------------
// ring slot encoding (Vyukov-style sequence numbers fused with the item)
//   free for the producer of index i : seq == lo32(i)
//   full, item of index i            : seq == lo32(i + 1)
// consumer of i sets seq = lo32(i + cap) (free for producer of i + cap).
// ---------------------------------------------------------------------------
__device__ __forceinline__ bool slot_full_for(uint64_t slot, uint64_t idx) { return hi32(slot) == lo32(idx + 1); }
__device__ __forceinline__ bool slot_free_for(uint64_t slot, uint64_t idx) { return hi32(slot) == lo32(idx); }

// The two rings of a rank (ring 1 exists only with the priority queue, N1):
// slots, reservation head, push tail (T) and finished count (F) of ring q.
__host__ __device__ __forceinline__ uint64_t *q_slots(const RankDev &R, int q) { return q ? R.ring2 : R.ring; }
__host__ __device__ __forceinline__ uint64_t *q_head(const RankDev &R, int q) { return q ? &R.ctrl->pq_head.v : &R.ctrl->head.v; }
__host__ __device__ __forceinline__ uint64_t *q_tail(const RankDev &R, int q) { return q ? &R.ctrl->pq_tail.v : &R.ctrl->tail.v; }
__host__ __device__ __forceinline__ uint64_t *q_fin(const RankDev &R, int q) { return q ? &R.ctrl->pq_fin.v : &R.ctrl->finished.v; }
__host__ __device__ __forceinline__ uint64_t *q_base(const RankDev &R, int q) { return q ? &R.ctrl->pq_base.v : &R.ctrl->ring_base.v; }

// Priority-queue item tag: a discovered vertex whose candidate depth is at or
// above the current threshold goes to the other ring (rank-local ids < 2^30 in
// this mode; pieces, bit 31, are never tagged).
constexpr uint32_t kFarBit = 0x40000000u;
constexpr uint32_t kNoTh = 0xFFFFFFFFu;      // threshold when the priority queue is off
__device__ __forceinline__ uint32_t pq_tag(uint32_t item, uint32_t nd, uint32_t th) {
    return nd >= th ? (item | kFarBit) : item;
}
__device__ __forceinline__ bool pq_is_far(uint32_t item) { return (item & (0x80000000u | kFarBit)) == kFarBit; }

// PR state placement: local id i lives at slot (i mod 8) * q + i / 8 (q = n_r / 8,
// identity on the tail), so that ids adjacent after degree relabeling -- the
// hubs, which receive most of the fp64 atomicAdds -- fall into different 32-B
// sectors and L2 slices instead of serialising in one atomic unit.  A bijection.
__host__ __device__ __forceinline__ int64_t pr_q_of(int64_t n_r) { return n_r >= 64 ? n_r / 8 : 0; }
// PR message payload meaning "the delta was already added in the owner's memory and crossed eps:
// enqueue the vertex" (KParams::pr_ratom); a real delta is never this NaN pattern
constexpr uint64_t kPrActivate = ~0ull;
// BFS message depth word flag: "the owner's depth word was already lowered to this depth by the
// sender (KParams::bfs_ratom): enqueue the vertex"
constexpr uint32_t kBfsActivate = 0x80000000u;
__device__ __forceinline__ int64_t pr_slot(int64_t i, int64_t q) {
    return (q > 0 && i < 8 * q) ? (i & 7) * q + (i >> 3) : i;
}

// Raise a device error for the current solve on this rank AND every peer, so
// that all ranks' workers leave the loop (a rank that only waited for the
// coordinator's done flag would otherwise spin until its own watchdog).  The
// first code wins on each rank; system-scope CAS reaches IPC-mapped peers.
__device__ __forceinline__ void set_error(const RankDev &R, uint64_t code) {
    atomicCAS((unsigned long long *)&R.ctrl->error.v, 0ull, (unsigned long long)code);
    for (int d = 0; d < R.n_ranks && d < kMaxRanks; ++d)
        if (d != R.rank && R.peer_ctrl[d])
            atomicCAS_system((unsigned long long *)&R.peer_ctrl[d]->error.v, 0ull, (unsigned long long)code);
}

}  // namespace atos
