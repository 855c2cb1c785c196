// atos_bfs1.cuh -- the single-rank BFS expansion of the persistent worker
// (Listing 5's neighbour loop, re-planned for sm_100a).
//
// Included by atos_worker.cuh; used by worker_body for BFS with one rank, the
// probe filter and fire-and-forget relaxation (the defaults on every graph).
//
// Two ideas, both aimed at the two limits ncu showed for the generic
// expansion: issued instructions per edge and the L1TEX wavefront rate of the
// per-edge random probe (one 128-B line per lane, ~1 per SM clock: 285 G
// probes/s measured, profiles/r1/micro_denominators.json).
//
// 1. Degree classes inside a batch (the paper's thread / warp / CTA load
//    balancing by degree).  Rows of >= kLong edges -- hub pieces
//    and long rows -- are cut into 128-edge chunks aligned to 16 B: a warp's
//    chunk belongs to ONE row, so the row record is read once per chunk
//    (warp-uniform candidate depth) and every lane loads its 4 edges with one
//    LDG.128.  Short rows share a packed edge space mapped by the per-batch edge
//    map (one bitmap word + one row index per 32 edges) to a 16-B row record.
//
// 2. Hub bounds.  After degree relabeling ids
//    [0, hub_n) are the graph's highest-degree vertices, which receive most edge
//    endpoints of a skewed graph (top 2^21 of RMAT-22: 0.97 of all endpoints).
//    Chunk c = ids [128c, 128c + 128) has a global byte hcb[c] holding an UPPER
//    BOUND of the largest probe-filter value in the chunk: every scan of the
//    filter gives one (filter values only decrease; racing plain stores of two
//    scans leave one of two valid bounds), and the warps of all workers re-scan
//    all chunks every few batches (hub_refresh).  Every worker copies the array
//    into shared memory per batch with one TMA bulk copy (hub_copy_issue).  An edge to a hub u with candidate
//    depth nd where hcb[u / 128] <= nd provably cannot improve u (depth(u) <=
//    filt(u) <= bound <= nd), so it is retired by one shared-memory byte load
//    instead of a global probe.  Exactness is unchanged: only edges that
//    cannot improve are skipped.
//
// 3. Visited bitmap (KParams::vis: the priority queue with threshold_delta 1,
//    i.e. buckets = BFS levels).  A bucket only holds vertices of
//    its level, and every vertex is discovered at its final depth (all vertices
//    of smaller depth were expanded in earlier buckets), so the state a probe
//    needs is ONE bit: visited or not.  The n-bit bitmap (8 MB at RMAT-26) stays
//    in L2 -- the 67 MB byte filter did not (45 % L2 hit rate, 22 GB DRAM reads
//    per RMAT-26 solve) -- and a stale L1 copy of a word only shows fewer bits,
//    which costs an extra atomicOr, never a wrong result.  The discoverer is the
//    one lane whose atomicOr set the bit: it stores the depth byte and enqueues,
//    so there are no duplicate queue entries, no claim at pop, and no 4-byte
//    depth words to read-modify-write in DRAM.  Hub bounds become "all 128 hubs
//    of the chunk visited" (0) or unknown (255).
#pragma once
// (included inside namespace atos by atos_worker.cuh)

__device__ __forceinline__ int4 ld_stream4(const int32_t *ptr, uint64_t pol) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                 : "l"(ptr), "l"(pol));
    return v;
}

// Re-scan this warp's hub chunks into the global bounds, all chunks of the
// graph once per batch of every worker: warp gw scans chunks gw + GW * j (up to
// 4 per warp with 2^21 hubs and 296 workers), loads first, then the reductions.
// Called after the warp's expansion, where it waits for the batch-end barrier.
__device__ __forceinline__ void hub_refresh(Smem &s, const KParams &kp, int cta) {
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t C = (uint32_t)kp.hub_n >> 7;            // (the array's padding stays 255)
    const uint32_t GW = (uint32_t)kp.ctas_per_rank * kWarps;
    const uint32_t c0 = (uint32_t)cta * kWarps + w;
    const uint32_t *f = reinterpret_cast<const uint32_t *>(s.R.filt);
    for (uint32_t cb = c0; cb < C; cb += 4 * GW) {
        uint32_t x[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const uint32_t c = cb + GW * j;
            x[j] = c < C ? __ldcg(f + (size_t)c * 32 + lane) : 0u;   // 128 B per chunk, from L2
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const uint32_t c = cb + GW * j;
            const uint32_t m = max(max(x[j] & 255u, (x[j] >> 8) & 255u), max((x[j] >> 16) & 255u, x[j] >> 24));
            const uint32_t cm = __reduce_max_sync(kFull, m);
            // store only a tighter bound than this worker's copy holds (most re-scans
            // change nothing; stores into the array every worker copies from cost)
            if (lane == 0 && c < C && cm < hub_base(s)[c]) s.R.hcb[c] = (uint8_t)cm;
        }
    }
}

// Visited-bitmap variant: chunk c (128 ids) = bitmap words 4c .. 4c+3; a warp
// checks 8 chunks per load (lane l: word 4 * (c0 + l/4) + l%4).
__device__ __forceinline__ void hub_refresh_vis(Smem &s, const KParams &kp, int cta) {
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t C = (uint32_t)kp.hub_n >> 7;
    const uint32_t GW = (uint32_t)kp.ctas_per_rank * kWarps;
    for (uint32_t cb = ((uint32_t)cta * kWarps + w) * 8u; cb < C; cb += GW * 8u) {
        const uint32_t c = cb + (uint32_t)(lane >> 2);
        const uint32_t x = c < C ? __ldcg(s.R.vis + 4 * (size_t)c + (lane & 3)) : 0u;
        const uint32_t full = __ballot_sync(kFull, x == 0xFFFFFFFFu);
        if ((lane & 3) == 0 && c < C && ((full >> lane) & 15u) == 15u && hub_base(s)[c] != 0) s.R.hcb[c] = 0;
    }
}

// Copy the global hub bounds into this worker's shared memory with one TMA bulk
// copy (cp.async.bulk, completion on an mbarrier), issued by one thread at the
// start of the batch setup and waited for just before the expansion, so it
// overlaps the row loads and the scans.  hub_chunks is a multiple of 16.
__device__ __forceinline__ uint32_t smem_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void hub_copy_issue(Smem &s, const KParams &kp) {
    const uint32_t bytes = (uint32_t)kp.hub_chunks;
    const uint32_t mb = smem_addr(&s.hub_mbar);
    // the previous batch's (generic-proxy) reads of the bounds precede this async-proxy overwrite
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_addr(hub_base(s))), "l"(s.R.hcb), "r"(bytes), "r"(mb) : "memory");
}

__device__ __forceinline__ void hub_copy_wait(const Smem &s, uint32_t parity) {
    const uint32_t mb = smem_addr(&s.hub_mbar);
    uint32_t done = 0;
    while (!done) {
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
                     : "=r"(done) : "r"(mb), "r"(parity) : "memory");
    }
}

__device__ __forceinline__ void hub_mbar_init(Smem &s) {   // one thread, before the loop's first barrier
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&s.hub_mbar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    s.hub_par = 0;
    s.hub_rnd = 0;
}

__device__ __forceinline__ void hub_fill_unknown(Smem &s, const KParams &kp) {   // (ATOS_HUB_DBG without the copy)
    for (int i = threadIdx.x; i < kp.hub_chunks; i += kThreads) hub_base(s)[i] = 255;
}

// Relaxation of N edges per lane in two phases, probe_* (hub-bound test, issue
// the probe loads) and finish_* (decide, relax), so that a pipelined expansion
// (ATOS_CHUNK_PIPE) can put the next chunk's column loads between them.
//
// Filter mode (u[k] < 0: no edge): hub-bound test, filter probe, red.min +
// filter store on the probe's verdict (relax_red; duplicates are skipped at pop
// by the pending bit, the flush fences before publishing).
template <int N>
__device__ __forceinline__ void probe_bfs1(const Smem &s, const KParams &kp, const uint8_t *hcs, int32_t (&u)[N],
                                           const uint32_t (&nd)[N], uint32_t (&f)[N], uint32_t &hits) {
    uint8_t *const filt = s.R.filt;
    const uint32_t H = (kp.hub_dbg & 4) ? 0u : (uint32_t)kp.hub_n;
    uint32_t hm = 0;                  // slots retired by the hub bound (statistics: one popc)
#pragma unroll
    for (int k = 0; k < N; ++k) {
        if ((uint32_t)u[k] < H) {     // (u < 0 is huge unsigned: not a hub)
            const uint32_t hb = hcs[(uint32_t)u[k] >> 7];
            if (hb <= nd[k] && hb != 255u) {
                u[k] = -1;
                hm |= 1u << k;
            }
        }
    }
    hits += __popc(hm);
#pragma unroll
    for (int k = 0; k < N; ++k) f[k] = u[k] >= 0 ? ldg_u8(filt + u[k]) : 0u;
}

template <int N>
__device__ __forceinline__ void finish_bfs1(const Smem &s, const int32_t (&u)[N], const uint32_t (&nd)[N],
                                            const uint32_t (&f)[N], uint32_t &msk) {
    uint32_t *const depth = s.R.depth;
    uint8_t *const filt = s.R.filt;
    msk = 0;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        if (u[k] >= 0 && (nd[k] < f[k] || f[k] == 255u)) {
            red_min_u32(depth + u[k], dw_make(nd[k]));
            stg_u8(filt + u[k], filt_of(nd[k]));
            msk |= 1u << k;
        }
    }
}

template <int N>
__device__ __forceinline__ void relax_bfs1(const Smem &s, const KParams &kp, const uint8_t *hcs, int32_t (&u)[N],
                                           const uint32_t (&nd)[N], uint32_t &msk, uint32_t &hits) {
    uint32_t f[N];
    probe_bfs1<N>(s, kp, hcs, u, nd, f, hits);
    finish_bfs1<N>(s, u, nd, f, msk);
}

// Visited-bitmap mode (all N edges at candidate depth nd): hub-bound test, bit
// probe (L1-cacheable: a stale word is conservative), then for clear bits
// either a fire-and-forget RED.OR (claim at pop, the default) or the
// atomicOr-with-return that decides the discoverer.  msk bit k = enqueue u[k].
template <int N>
__device__ __forceinline__ void probe_vis(const Smem &s, const KParams &kp, const uint8_t *hcs, int32_t (&u)[N],
                                          uint32_t (&wd)[N], uint32_t &hits) {
    uint32_t *const vis = s.R.vis;
    const uint32_t H = (kp.hub_dbg & 4) ? 0u : (uint32_t)kp.hub_n;
    uint32_t hm = 0;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        if ((uint32_t)u[k] < H && hcs[(uint32_t)u[k] >> 7] == 0) {
            u[k] = -1;
            hm |= 1u << k;
        }
    }
    hits += __popc(hm);
#pragma unroll
    for (int k = 0; k < N; ++k) wd[k] = u[k] >= 0 ? __ldca(vis + ((uint32_t)u[k] >> 5)) : 0xFFFFFFFFu;
}

template <int N>
__device__ __forceinline__ void finish_vis(const Smem &s, const KParams &kp, const int32_t (&u)[N], uint32_t nd,
                                           const uint32_t (&wd)[N], uint32_t &msk) {
    uint32_t *const vis = s.R.vis;
    if (kp.vis_claim) {
        // claim at pop: the bit is only a filter, set fire-and-forget (RED); a
        // vertex two lanes (or a stale probe) both see clear is enqueued twice and
        // the second pop loses the claim
        msk = 0;
#pragma unroll
        for (int k = 0; k < N; ++k) {
            const uint32_t bit = 1u << ((uint32_t)u[k] & 31u);
            if (u[k] >= 0 && !(wd[k] & bit)) {
                atomicOr(vis + ((uint32_t)u[k] >> 5), bit);
                msk |= 1u << k;
            }
        }
        return;
    }
    // all of the lane's atomics are issued before the first result is used (the
    // depth stores below would otherwise order each atomic after the previous
    // one's round trip: the compiler cannot tell the byte array from the bitmap)
    uint32_t old[N], cand = 0;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        const uint32_t bit = 1u << ((uint32_t)u[k] & 31u);
        old[k] = 0xFFFFFFFFu;
        if (u[k] >= 0 && !(wd[k] & bit)) {
            old[k] = atomicOr(vis + ((uint32_t)u[k] >> 5), bit);
            cand |= 1u << k;
        }
    }
    msk = 0;
#pragma unroll
    for (int k = 0; k < N; ++k) {
        if (((cand >> k) & 1u) && !(old[k] & (1u << ((uint32_t)u[k] & 31u)))) {
            if (nd < 255u) stg_u8(s.R.filt + u[k], nd);
            else s.R.depth[u[k]] = dw_make(nd);
            msk |= 1u << k;
        }
    }
}

template <int N>
__device__ __forceinline__ void relax_vis(const Smem &s, const KParams &kp, const uint8_t *hcs, int32_t (&u)[N],
                                          uint32_t nd, uint32_t &msk, uint32_t &hits) {
    uint32_t wd[N];
    probe_vis<N>(s, kp, hcs, u, wd, hits);
    finish_vis<N>(s, kp, u, nd, wd, msk);
}

// Largest li in [0, NL) with lq0[li] <= c, searched forward from li0 (a row
// with lq0[li0] <= c: the row of this warp's previous chunk).  The whole warp
// tests the next 32 rows at once; a warp's chunks are 16 apart and every row
// has at least one, so one round almost always suffices (a binary search over
// the batch's rows measured 10 % of the RMAT-26 worker's instructions).
__device__ __forceinline__ uint32_t long_row_from(const BatchBuf &bb, uint32_t NL, uint32_t c, uint32_t li0,
                                                  uint32_t lane) {
    uint32_t li = li0;
    for (;;) {
        const uint32_t j = li + 1 + lane;
        const uint32_t m = __ballot_sync(kFull, j < NL && bb.lq0[j] <= c);
        li += __popc(m);
        if (m != kFull) return li;
    }
}

// Expand the batch: each warp takes chunks w, w + 16, ...  A long-row chunk is
// kLongG groups of 128 edges of ONE row: every lane loads kLongG x 4 edges with
// kLongG independent LDG.128s, so a warp keeps kLongG x 512 B of the column
// stream in flight (memory-level parallelism is what bounds the stream: a
// warp's chunk is a dependent column -> probe -> relax chain).  A short chunk
// is 128 edges of the packed short-row edge space.
template <int G, bool VIS>
__device__ __forceinline__ void long_chunk(Smem &s, const BatchBuf &bb, const KParams &kp, const int32_t *col,
                                           uint64_t pol, uint32_t NL, uint32_t c, uint32_t lane, const uint8_t *hcs,
                                           int64_t vb, uint32_t &wn, uint32_t &hits, uint32_t &lcur) {
    const int w = threadIdx.x >> 5;
    const uint32_t li = c < (uint32_t)kLcv ? bb.lcv[c] : long_row_from(bb, NL, c, lcur, lane);
    lcur = li;
    const BRec r = bb.rec[kThreads - 1 - li];
    const uint32_t lo = (uint32_t)(r.base & 3);
    const int64_t a = r.base - lo;
    const uint32_t rel0 = (c - bb.lq0[li]) * (uint32_t)(kCh1 * G) + 4u * lane;   // edge offset from a
    const uint32_t end = lo + r.len;
    int32_t u[4 * G];
    uint32_t nd[4 * G];
#pragma unroll
    for (int g = 0; g < G; ++g) {
        const uint32_t rel = rel0 + (uint32_t)kCh1 * g;
        int4 v = make_int4(-1, -1, -1, -1);
        if (rel < end) v = ld_stream4(col + a + rel, pol);   // may read <= 3 entries past the row (padded array)
        u[4 * g + 0] = (rel >= lo && rel < end) ? v.x : -1;
        u[4 * g + 1] = (rel + 1 >= lo && rel + 1 < end) ? v.y : -1;
        u[4 * g + 2] = (rel + 2 >= lo && rel + 2 < end) ? v.z : -1;
        u[4 * g + 3] = (rel + 3 < end) ? v.w : -1;
    }
#pragma unroll
    for (int k = 0; k < 4 * G; ++k) nd[k] = r.nd;
    uint32_t msk;
    if constexpr (VIS) relax_vis<4 * G>(s, kp, hcs, u, r.nd, msk, hits);
    else relax_bfs1<4 * G>(s, kp, hcs, u, nd, msk, hits);
    if (__any_sync(kFull, msk != 0)) {
        uint32_t item[4 * G];
        const uint32_t tag = r.nd >= s.pq_th ? kFarBit : 0u;     // priority queue (N1): far bucket
#pragma unroll
        for (int k = 0; k < 4 * G; ++k) item[k] = (uint32_t)(u[k] - vb) | tag;
        warp_append_mask<4 * G>(s, w, wn, msk, item, kp.relax_red);
    }
}

#ifndef ATOS_CHUNK_PIPE
#define ATOS_CHUNK_PIPE 1     // 1 = next chunk's columns issued before this chunk's probes (default), 2 = after, 0 = off (A/B)
#endif

// One chunk's column ids in flight (pipelined expansion, ATOS_CHUNK_PIPE).
struct ChunkFetch {
    int32_t u[4];       // raw column ids (long chunk: valid where vm says so; short: -1 = no edge)
    uint32_t nd[4];     // candidate depth per slot
    uint32_t vm;        // valid-slot mask of a long chunk (0xF for short chunks)
};

__device__ __forceinline__ void fetch_chunk(const BatchBuf &bb, const int32_t *col, uint64_t pol, uint32_t NL,
                                            uint32_t NLC, uint32_t ES, uint32_t c, uint32_t lane, uint32_t below,
                                            uint32_t &lcur, ChunkFetch &f) {
    if (c < NLC) {
        const uint32_t li = c < (uint32_t)kLcv ? bb.lcv[c] : long_row_from(bb, NL, c, lcur, lane);
        lcur = li;
        const BRec r = bb.rec[kThreads - 1 - li];
        const uint32_t lo = (uint32_t)(r.base & 3);
        const int64_t a = r.base - lo;
        const uint32_t rel = (c - bb.lq0[li]) * (uint32_t)kCh1 + 4u * lane;
        const uint32_t end = lo + r.len;
        f.vm = (uint32_t)(rel >= lo && rel < end) | ((uint32_t)(rel + 1 >= lo && rel + 1 < end) << 1) |
               ((uint32_t)(rel + 2 >= lo && rel + 2 < end) << 2) | ((uint32_t)(rel + 3 < end) << 3);
        if (rel < end) {
            const int4 v = ld_stream4(col + a + rel, pol);
            f.u[0] = v.x; f.u[1] = v.y; f.u[2] = v.z; f.u[3] = v.w;
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) f.nd[k] = r.nd;
        return;
    }
    const uint32_t c0 = (c - NLC) * (uint32_t)kCh1;
    f.vm = 0xFu;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        const uint32_t e = c0 + 32u * k + lane;
        f.u[k] = -1;
        f.nd[k] = 0;
        if (e < ES) {
            const uint32_t wd = e >> 5;
            const BRec r = bb.rec[bb.rowmap[wd] + __popc(bb.bm[wd] & below)];
            f.u[k] = ld_stream(col + r.base + e, pol);
            f.nd[k] = r.nd;
        }
    }
}

template <bool VIS>
__device__ void expand_bfs1_pipe(Smem &s, BatchBuf &bb, const KParams &kp, uint32_t NL, uint32_t NLC, uint32_t ES,
                                 uint32_t &wn) {
    const int w = threadIdx.x >> 5;
    const uint32_t lane = threadIdx.x & 31;
    const int32_t *const col = s.R.col;
    const uint8_t *const hcs = hub_base(s);
    const uint64_t pol = policy_evict_first();
    const uint32_t below = lane == 31 ? 0xFFFFFFFEu : (((2u << lane) - 1u) & ~1u);
    const uint32_t ntot = NLC + (ES + kCh1 - 1) / kCh1;
    const int64_t vb = s.R.v_begin;
    uint32_t hits = 0, lcur = 0;
    ChunkFetch f;
    if ((uint32_t)w < ntot) fetch_chunk(bb, col, pol, NL, NLC, ES, (uint32_t)w, lane, below, lcur, f);
    for (uint32_t c = (uint32_t)w; c < ntot; c += kWarps) {
        int32_t u[4];
        uint32_t nd[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            u[k] = ((f.vm >> k) & 1u) ? f.u[k] : -1;
            nd[k] = f.nd[k];
        }
        uint32_t pv[4];
        if constexpr (ATOS_CHUNK_PIPE == 1)
            if (c + kWarps < ntot) fetch_chunk(bb, col, pol, NL, NLC, ES, c + kWarps, lane, below, lcur, f);
        if constexpr (VIS) probe_vis<4>(s, kp, hcs, u, pv, hits);
        else probe_bfs1<4>(s, kp, hcs, u, nd, pv, hits);
        if constexpr (ATOS_CHUNK_PIPE != 1)
            if (c + kWarps < ntot) fetch_chunk(bb, col, pol, NL, NLC, ES, c + kWarps, lane, below, lcur, f);
        uint32_t msk;
        if constexpr (VIS) finish_vis<4>(s, kp, u, s.pq_th, pv, msk);
        else finish_bfs1<4>(s, u, nd, pv, msk);
        if (__any_sync(kFull, msk != 0)) {
            uint32_t item[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) item[k] = pq_tag((uint32_t)(u[k] - vb), nd[k], s.pq_th);
            warp_append_mask<4>(s, w, wn, msk, item, kp.relax_red);
        }
    }
    if (kp.hub_n) {
        hits = __reduce_add_sync(kFull, hits);
        if (lane == 0 && hits) atomicAdd(&s.c_hub, (unsigned long long)hits);
    }
}

template <bool VIS>
__device__ void expand_bfs1(Smem &s, BatchBuf &bb, const KParams &kp, uint32_t NL, uint32_t NLC, uint32_t ES,
                            uint32_t &wn) {
    const int w = threadIdx.x >> 5;
    const uint32_t lane = threadIdx.x & 31;
    const int32_t *const col = s.R.col;
    const uint8_t *const hcs = hub_base(s);
    const uint64_t pol = policy_evict_first();
    const uint32_t below = lane == 31 ? 0xFFFFFFFEu : (((2u << lane) - 1u) & ~1u);
    const uint32_t ntot = NLC + (ES + kCh1 - 1) / kCh1;
    const int64_t vb = s.R.v_begin;
    uint32_t hits = 0, lcur = 0;
    for (uint32_t c = (uint32_t)w; c < ntot; c += kWarps) {
        if (c < NLC) {
            long_chunk<kLongG, VIS>(s, bb, kp, col, pol, NL, c, lane, hcs, vb, wn, hits, lcur);
            continue;
        }
        // short rows: packed edge space, coalesced 4-B column loads
        int32_t u[4];
        uint32_t nd[4];
        const uint32_t c0 = (c - NLC) * (uint32_t)kCh1;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const uint32_t e = c0 + 32u * k + lane;
            u[k] = -1;
            nd[k] = 0;
            if (e < ES) {
                const uint32_t wd = e >> 5;
                const BRec r = bb.rec[bb.rowmap[wd] + __popc(bb.bm[wd] & below)];
                u[k] = ld_stream(col + r.base + e, pol);
                nd[k] = r.nd;
            }
        }
        uint32_t msk;
        if constexpr (VIS) relax_vis<4>(s, kp, hcs, u, s.pq_th, msk, hits);     // one level per bucket
        else relax_bfs1<4>(s, kp, hcs, u, nd, msk, hits);
        if (__any_sync(kFull, msk != 0)) {
            uint32_t item[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) item[k] = pq_tag((uint32_t)(u[k] - vb), nd[k], s.pq_th);
            warp_append_mask<4>(s, w, wn, msk, item, kp.relax_red);
        }
    }
    if (kp.hub_n) {
        hits = __reduce_add_sync(kFull, hits);
        if (lane == 0 && hits) atomicAdd(&s.c_hub, (unsigned long long)hits);
    }
}

// Load per-vertex info of the batch s.v[0..B), classify rows, build the maps,
// refresh + copy the hub bounds, expand.  (Single rank, filter + relax_red.)
__device__ void process_batch_bfs1(Smem &s, const KParams &kp, int cta, int B) {
    const RankDev &R = s.R;
    BatchBuf &bb = s.bb[0];
    const int tid = threadIdx.x;
    const bool hub = kp.hub_chunks > 0;
    if (hub && tid == 0 && !(kp.hub_dbg & 2)) {
        s.hub_par ^= 1u;              // parity of this batch's copy (read by all threads after the scan's barriers)
        s.hub_rnd++;
        hub_copy_issue(s, kp);
    }
    int64_t deg = 0, b = 0;
    uint32_t npc = 0, nd = 0;
    if (tid < B) {
        const uint32_t it = bb.v[tid];
        if (it & kPieceBit) {
            // a piece of a split row: edges [piece * split, (piece+1) * split) of v,
            // relaxed with v's current depth (a valid bound: depths only decrease,
            // and a newer depth re-expands the whole row anyway)
            const uint32_t v = it & 0xFFFFu, pc = (it >> 16) & 0x7FFFu;
            const int64_t rb = ldg_i64_nc(R.row_ptr + v), re = ldg_i64_nc(R.row_ptr + v + 1);
            b = rb + (int64_t)pc * kp.split;
            deg = re - b < (int64_t)kp.split ? re - b : (int64_t)kp.split;
            if (kp.vis) {
                nd = s.pq_th;              // buckets are levels: every item of this one has depth th - 1
                if (deg < 0) deg = 0;
            } else {
                const uint32_t d = dw_depth(ld_relaxed_gpu_u32(R.depth + R.v_begin + v));
                nd = d + 1;
                if (d == kDepthInf || deg < 0) deg = 0;
            }
        } else {
            const uint32_t v = it;
            b = ldg_i64_nc(R.row_ptr + v);
            deg = ldg_i64_nc(R.row_ptr + v + 1) - b;
            if (kp.vis) {
                nd = s.pq_th;              // enqueued once, by its discoverer, at its final depth th - 1
                if (kp.vis_claim) {
                    // claim at pop: the first pop of v (in its own level's bucket) wins
                    // and stores v's depth; duplicates are skipped
                    const uint64_t gv = (uint64_t)(R.v_begin + v);
                    const uint32_t bit = 1u << (gv & 31u);
                    uint32_t *const claim = R.vis + ((uint64_t)R.n >> 5) + 1;
                    if (atomicOr(claim + (gv >> 5), bit) & bit) {
                        deg = 0;
                    } else if (nd - 1 < 255u) {
                        stg_u8(R.filt + gv, nd - 1);
                    } else {
                        R.depth[gv] = dw_make(nd - 1);
                    }
                }
            } else {
                // claim the expansion of v at its current depth; stale duplicates see
                // the pending bit already cleared and are skipped
                const uint32_t old = atom_and_u32(R.depth + R.v_begin + v, ~1u);
                const uint32_t d = dw_depth(old);
                nd = d + 1;
                if (!(old & 1u) || d == kDepthInf) deg = 0;
            }
            if (kp.split > 0 && deg > 2 * (int64_t)kp.split && (int64_t)v < kPieceVMax &&
                deg <= (int64_t)kp.split * kPieceMax) {
                npc = (uint32_t)((deg - 1) / kp.split);   // pieces 1..npc go to the ring
                deg = kp.split;
            }
        }
    }
    if (kp.split > 0 && __syncthreads_or(npc > 0)) {
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
    for (int i = tid; i < kBitW; i += kThreads) bb.bm[i] = 0u;
    // one scan for four counts: long chunks [40,64) | long rows [30,40) | short edges [10,30) | short rows [0,10)
    const bool lng = deg >= kLong;
    const uint32_t lo = (uint32_t)(b & 3);
    const uint32_t nch = lng ? (uint32_t)((deg + lo + kCh1 * kLongG - 1) / (kCh1 * kLongG)) : 0u;
    const int64_t x = lng ? (((int64_t)nch << 40) | (1ll << 30)) : ((deg << 10) | (deg > 0 ? 1 : 0));
    int64_t ex;
    const int64_t tot = block_exscan(s, x, ex);
    const uint32_t NLC = (uint32_t)(tot >> 40), NL = (uint32_t)((tot >> 30) & 1023), ES = (uint32_t)((tot >> 10) & 0xFFFFF);
    if (deg > 0) {
        if (lng) {
            const uint32_t li = (uint32_t)((ex >> 30) & 1023), q0 = (uint32_t)(ex >> 40);
            BRec r;
            r.base = b;
            r.nd = nd;
            r.len = (uint32_t)deg;
            bb.rec[kThreads - 1 - li] = r;
            bb.lq0[li] = q0;
            for (uint32_t q = q0; q < q0 + nch && q < (uint32_t)kLcv; ++q) bb.lcv[q] = (uint16_t)li;
        } else {
            const uint32_t off = (uint32_t)((ex >> 10) & 0xFFFFF), nz = (uint32_t)(ex & 1023);
            BRec r;
            r.base = b - (int64_t)off;
            r.nd = nd;
            r.len = 0;
            bb.rec[nz] = r;
            atomicOr(&bb.bm[off >> 5], 1u << (off & 31));
            for (uint32_t wd = (off + 31) >> 5; wd <= ((off + (uint32_t)deg - 1) >> 5); ++wd) bb.rowmap[wd] = (uint16_t)nz;
        }
    }
    // edges of the batch (statistics): per-warp sums, one smem atomic per warp
    unsigned long long de = (unsigned long long)deg;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) de += __shfl_xor_sync(kFull, de, o);
    if ((tid & 31) == 0 && de) atomicAdd(&s.c_edges, de);
    if (kp.timeline_ns && (tid & 31) == 0 && de) {        // experiment: work timeline of the solve
        const uint64_t b = (globaltimer() - R.ctrl->tl_t0) / (uint64_t)kp.timeline_ns;
        const int k = b < (uint64_t)kTimeline ? (int)b : kTimeline - 1;
        atomicAdd((unsigned long long *)&R.ctrl->tl_edges[k], de);
        if (tid == 0) {
            atomicAdd((unsigned long long *)&R.ctrl->tl_batches[k], 1ull);
            atomicAdd((unsigned long long *)&R.ctrl->tl_pops[k], (unsigned long long)B);
        }
    }
    if (hub && !(kp.hub_dbg & 2)) hub_copy_wait(s, s.hub_par ^ 1u);             // this batch's bounds have landed
    __syncthreads();
    if (tid == 0 && kp.pq_early) {
        // level buckets: reserve the NEXT batch on the current ring now, so the
        // head atomic leaves the critical path between batches -- only when the
        // ring holds plenty of work (a reservation withholds items from idle
        // workers).  An early reservation is an ordinary one taken sooner: if the
        // bucket advances first, pq_choose serves it as a stale one (pq_recycle).
        const int q = s.pq_q;
        uint64_t &lo = res_lo_q(s, q), &hi = res_hi_q(s, q);
        if (lo == hi) {
            const uint64_t t = ld_relaxed_gpu(q_tail(R, q)), h = ld_relaxed_gpu(q_head(R, q));
            if (t > h && t - h >= 2ull * (uint64_t)kp.ctas_per_rank * (uint64_t)kp.fetch) {
                lo = atomicAdd((unsigned long long *)q_head(R, q), (unsigned long long)kp.fetch);
                hi = lo + (uint64_t)kp.fetch;
            }
        }
    }
    if (NLC + ES > 0) {
        const int w = tid >> 5;
        uint32_t wn = s.wn[w];
        if constexpr (ATOS_CHUNK_PIPE != 0 && kLongG == 1) {
            if (kp.vis) expand_bfs1_pipe<true>(s, bb, kp, NL, NLC, ES, wn);
            else expand_bfs1_pipe<false>(s, bb, kp, NL, NLC, ES, wn);
        } else {
            if (kp.vis) expand_bfs1<true>(s, bb, kp, NL, NLC, ES, wn);
            else expand_bfs1<false>(s, bb, kp, NL, NLC, ES, wn);
        }
        __syncwarp();
        if ((tid & 31) == 0) s.wn[w] = wn;
    }
    if (hub && !(kp.hub_dbg & 1)) {
        if (kp.vis) hub_refresh_vis(s, kp, cta);
        else hub_refresh(s, kp, cta);
    }
}

