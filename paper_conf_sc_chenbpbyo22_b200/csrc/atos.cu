// atos.cu -- C ABI (include/atos.h) of the B200-native Atos hot path.
//
// Host runtime: graph ingest + 1-D partition, per-rank device
// arenas (state, ring, channels, control block) laid out identically on every
// rank so that peers can address each other after IPC mapping (the analogue of
// NVSHMEM's symmetric heap, Listing 5), kernel launch sequence of
// one solve (barrier -> init -> persistent worker -> fixup -> gather), error
// and statistics plumbing.
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include "../../include/atos.h"
#include "atos_aux.cuh"
#include "atos_worker.cuh"
namespace atos {
#include "atos_qbench.cuh"
}

using namespace atos;

constexpr int kColPad = 4;   // column arrays end with 4 spare entries (16-B loads of a row's last edges)
constexpr int64_t kHubAutoN = 3 << 19;   // hub bounds cover the top 1.5 M ids by default (12 KB of shared memory)
constexpr int64_t kHubMaxN = 1 << 22;


// ---------------------------------------------------------------------------
// errors
// ---------------------------------------------------------------------------
static thread_local char g_err[512] = "";

static atos_status fail(atos_status st, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return st;
}

#define CU(call)                                                                                  \
    do {                                                                                          \
        cudaError_t e_ = (call);                                                                  \
        if (e_ != cudaSuccess) {                                                                  \
            return fail(e_ == cudaErrorMemoryAllocation ? ATOS_ERR_OOM : ATOS_ERR_CUDA,         \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
        }                                                                                         \
    } while (0)

// Opt-in phase trace of graph_load (ATOS_LOAD_TRACE=1): syncs the stream at each
// mark and prints the host wall time of the phase to stderr.  Diagnostic only.
#include <chrono>
#include <cstdlib>
struct LoadTrace {
    bool on = std::getenv("ATOS_LOAD_TRACE") != nullptr;
    std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
    void mark(cudaStream_t st, const char *what) {
        if (!on) return;
        cudaStreamSynchronize(st);
        const auto now = std::chrono::steady_clock::now();
        fprintf(stderr, "[atos load] %-24s %8.2f ms\n", what, std::chrono::duration<double, std::milli>(now - t).count());
        t = now;
    }
};

extern "C" const char *atos_last_error(void) { return g_err; }
extern "C" int32_t atos_version(void) { return ATOS_ABI_VERSION; }

// ---------------------------------------------------------------------------
// config, partition, validation (host only)
// ---------------------------------------------------------------------------
extern "C" atos_status atos_config_init(atos_config *cfg) {
    if (!cfg) return fail(ATOS_ERR_INVALID_ARG, "cfg is NULL");
    std::memset(cfg, 0, sizeof(*cfg));
    cfg->worker_threads = kThreads;
    cfg->ctas_per_sm = 0;
    cfg->fetch_size = kThreads;
    cfg->keep_items = -1;
    cfg->l2_persist = 1;
    cfg->prefetch = 0;    // measured slower on RMAT-24 with both worker modes
    cfg->relax_red = 1;
    cfg->pipeline = 2;
    cfg->probe_filter = 2;
    cfg->ring_cap_factor = 2.0;
    cfg->agg_enabled = 1;
    // channel sweep, virtual ranks: PR RMAT-20 at 2 ranks 132 -> 59 ms with
    // 4096 packets per channel (senders stalled on full channels at batch end), 50 ms with
    // 1024-message packets; 8 ranks 115 -> 108 ms; BFS within noise
    cfg->agg_batch_msgs = 1024;
    cfg->agg_max_age_ns = 4000;      // ~the paper's eager WAIT_TIME for BFS
    cfg->channel_packets = 4096;
    cfg->watchdog_ms = 60000;
    cfg->rank = 0;
    cfg->n_ranks = 1;
    cfg->virtual_ranks = 1;
    cfg->device = 0;
    cfg->stream = nullptr;
    cfg->relabel = 2;
    cfg->hub_cache = -1;
    cfg->split_edges = -1;
    cfg->pr_combine = 0;
    cfg->pool_retain = 0;
    cfg->pq_threshold = 0;
    cfg->pq_delta = -1;
    return ATOS_OK;
}

extern "C" atos_status atos_partition_balanced(int64_t n, int32_t p, int64_t *part) {
    if (n < 0 || p < 1 || p > ATOS_MAX_RANKS || !part)
        return fail(ATOS_ERR_INVALID_ARG, "partition: need n>=0, 1<=p<=%d, part!=NULL", ATOS_MAX_RANKS);
    for (int r = 0; r <= p; ++r) part[r] = (int64_t)((__int128)r * n / p);
    return ATOS_OK;
}

extern "C" atos_status atos_validate_csr(const int64_t *row_ptr, const int32_t *col, int64_t n, int64_t nnz) {
    if (n < 1 || n > INT32_MAX || nnz < 0 || !row_ptr || (nnz > 0 && !col))
        return fail(ATOS_ERR_INVALID_ARG, "csr: need 1<=n<=2^31-1, nnz>=0, non-NULL arrays");
    if (row_ptr[0] != 0 || row_ptr[n] != nnz)
        return fail(ATOS_ERR_INVALID_ARG, "csr: row_ptr[0] must be 0 and row_ptr[n] == nnz");
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] < row_ptr[v]) return fail(ATOS_ERR_INVALID_ARG, "csr: row_ptr not monotone at %lld", (long long)v);
    for (int64_t e = 0; e < nnz; ++e)
        if (col[e] < 0 || col[e] >= n) return fail(ATOS_ERR_INVALID_ARG, "csr: col[%lld]=%d out of range", (long long)e, col[e]);
    return ATOS_OK;
}

// Priority-queue layout (second ring, visited + claim bitmaps): pq_delta > 0, or
// the auto choice (pq_delta = -1) on a single-rank graph of >= kPqAutoN
// vertices, where level buckets with the n-bit visited bitmap and claim at pop
// win over the FIFO queue with the byte filter (FIFO -> buckets, ms: RMAT-26
// 13.5 -> 8.62, RMAT-24 2.57 -> 2.42, RMAT-22 0.85 -> 0.81, RMAT-20 0.58 ->
// 0.41; RMAT-18 0.26 vs 0.27 and RMAT-16 0.14 vs 0.18 lose).
// Whether auto actually orders by level is decided per solve from the degree
// skew (make_params).
constexpr int64_t kPqAutoN = (int64_t)1 << 20;
static int pq_layout(const atos_config &c, int64_t n) {
    if (c.pq_delta > 0) return 1;
    return c.pq_delta == -1 && c.n_ranks == 1 && c.virtual_ranks == 1 && n >= kPqAutoN ? 1 : 0;
}

static bool valid_cfg(const atos_config &c) {
    auto pow2 = [](int64_t x) { return x > 0 && (x & (x - 1)) == 0; };
    return c.worker_threads == kThreads && c.fetch_size >= 1 && c.fetch_size <= kThreads &&
           c.keep_items >= -1 && c.keep_items <= kThreads && (c.keep_mode == 0 || c.keep_mode == 1) &&
           c.ring_cap_factor >= 1.0 && c.agg_batch_msgs >= 1 && c.agg_batch_msgs <= 4096 &&
           c.agg_max_age_ns >= 0 && pow2(c.channel_packets) && c.channel_packets <= (1 << 20) &&
           c.watchdog_ms >= 0 && c.n_ranks >= 1 && c.n_ranks <= ATOS_MAX_RANKS && c.rank >= 0 &&
           c.rank < c.n_ranks && c.virtual_ranks >= 1 && c.virtual_ranks <= ATOS_MAX_RANKS &&
           !(c.virtual_ranks > 1 && c.n_ranks > 1) && c.ctas_per_sm >= 0 && c.device >= 0 &&
           c.relabel >= 0 && c.relabel <= 2 && c.hub_cache >= -1 && c.hub_cache <= kHubMaxN &&
           (c.hub_cache <= 0 || c.hub_cache % 128 == 0) &&
           (c.split_edges == 0 || c.split_edges == -1 ||
            (c.split_edges >= 256 && c.split_edges <= (1 << 20) && pow2(c.split_edges))) &&
           (c.pr_combine == 0 || c.pr_combine == 1) && (c.pool_retain == 0 || c.pool_retain == 1) &&
           (c.discrete == 0 || (c.discrete == 1 && c.n_ranks == 1 && c.virtual_ranks == 1)) &&
           c.pq_threshold >= 0 && c.pq_delta >= -1;
}

// ---------------------------------------------------------------------------
// arena layout: identical computation on every rank
// ---------------------------------------------------------------------------
struct Layout {
    size_t ctrl, depth, filt, hcb, vis, rank, res, ring, ring2, in_hdr, in_pay, free_m, staging, parent, ghost, total;
    uint64_t ring_cap;
    int64_t n_r;
};

static uint64_t pow2_ceil(uint64_t x) {
    uint64_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

struct Shape {
    int64_t n;
    int p;
    int cp, pkt, stage_cap, ctas_per_rank, fetch;
    double ring_factor;
    int combine;       // PR ghost residuals allocated (n_ranks > 1 && pr_combine)
    int hub_chunks;    // BFS hub bounds array (single rank)
    int pq;            // priority queue (N1): second ring allocated
};

static Layout make_layout(const Shape &S, const int64_t *part, int r) {
    Layout L{};
    auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
    L.n_r = part[r + 1] - part[r];
    L.ring_cap = pow2_ceil(std::max<uint64_t>(1024, (uint64_t)(S.ring_factor * (double)L.n_r) +
                                                        (uint64_t)S.ctas_per_rank * (uint64_t)S.fetch));
    size_t o = 0;
    L.ctrl = o;    o = al(o + sizeof(Ctrl));
    L.depth = o;   o = al(o + (size_t)S.n * 4);
    L.filt = o;    o = al(o + (size_t)S.n);
    L.hcb = o;     o = al(o + (size_t)S.hub_chunks);
    L.vis = o;     o = al(o + (S.pq && S.p == 1 ? ((size_t)S.n / 32 + 1) * 8 : 0));   // visited + claimed bitmaps
    L.rank = o;    o = al(o + (size_t)L.n_r * 8);
    L.res = o;     o = al(o + (size_t)L.n_r * 8);
    L.ring = o;    o = al(o + (size_t)L.ring_cap * 8);
    L.ring2 = o;   o = al(o + (S.pq ? (size_t)L.ring_cap * 8 : 0));
    const bool multi = S.p > 1;
    L.in_hdr = o;  o = al(o + (multi ? (size_t)S.p * S.cp * 8 : 0));
    L.in_pay = o;  o = al(o + (multi ? (size_t)S.p * S.cp * S.pkt * 16 : 0));
    L.free_m = o;  o = al(o + (multi ? (size_t)S.p * S.cp * 8 : 0));
    L.staging = o; o = al(o + (multi ? (size_t)S.ctas_per_rank * kWarps * kMaxRanks * S.stage_cap * 16 : 0));
    L.parent = o;  o = al(o + (size_t)S.n * 8);
    L.ghost = o;   o = al(o + (multi && S.combine ? (size_t)S.n * 8 : 0));
    L.total = o;
    return L;
}

// sub-channels per channel: about 8 inbound cursors per rank in total (a single
// cursor serialised the receive side at 2 ranks), each sub-channel >= 2 packets
static int nsub_for(int p, int cp) {
    // about `rings` inbound rings per rank in total (ATOS_INBOUND_RINGS: A/B switch,
    // must be the same in every process of a multi-process run)
    static const int rings = std::getenv("ATOS_INBOUND_RINGS") ? std::max(1, std::atoi(std::getenv("ATOS_INBOUND_RINGS"))) : 8;
    int k = 1;
    while (k < kMaxSub && k * 2 * (p - 1) <= rings && cp / (k * 2) >= 2) k *= 2;
    return p > 1 ? k : 1;
}

static int stage_cap_for(int pkt) { return (int)pow2_ceil((uint64_t)std::max(2 * pkt, 64)); }

// ---------------------------------------------------------------------------
// handle
// ---------------------------------------------------------------------------
struct LocalRank {
    int rank = 0;
    Layout L{};
    unsigned char *arena = nullptr;
    int64_t *row_ptr = nullptr;
    int32_t *col = nullptr;
    int64_t m_r = 0;
    uint64_t snap[12] = {0};  // stat counters after the previous solve
};

struct atos_graph {
    atos_config cfg{};
    int64_t n = 0, nnz = 0;
    int p = 1;          // total ranks (virtual or processes)
    int n_local = 1;    // ranks served by this handle
    bool multiproc = false;
    bool connected = false;
    std::vector<int64_t> part;
    Shape S{};
    int sms = 0, occ = 0, grid = 0;
    size_t persist_max = 0, window_max = 0;   // L2 persisting-cache limits of the device
    size_t persist_set = (size_t)-1;          // carve-out last requested by this handle
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    LocalRank loc[kMaxRanks];
    unsigned char *peer_base[kMaxRanks] = {nullptr};
    bool peer_opened[kMaxRanks] = {false};
    RankDev *d_ranks = nullptr;
    int32_t *d_depth_full = nullptr;
    int32_t *d_perm = nullptr;     // degree relabeling: old -> new (NULL = identity)
    int32_t *d_inv = nullptr;      //                    new -> old
    int64_t *rp_dev_tmp = nullptr; // graph_load from host: device copy of the whole row_ptr made by
                                   // compute_relabel, reused for the ranks' rows, freed at the end of load
    int hub_n = 0;                 // BFS hub bounds: ids [0, hub_n) covered (single rank, relabeled graphs)
    int hub_chunks = 0;            // hub_n / 128 rounded up to a multiple of 16 (array size)
    bool skewed = true;            // max degree >= 32 x mean degree (set when an auto option needs it)
    int64_t **d_accs = nullptr;
    uint64_t epoch = 0;
    cudaEvent_t ev_begin = nullptr, ev_w0 = nullptr, ev_w1 = nullptr, ev_end = nullptr;
    bool pending = false;      // a solve is enqueued but not yet checked
    bool poisoned = false;     // multi-process handle after a device error: no further solves
    int app = kApBfs;          // application of the pending / last solve
    atos_stats last{};
    bool last_valid = false;
    // discrete-kernel mode: per-app instantiated graph
    // [step -> while(queue non-empty){ worker -> step }], parameters in d_kp
    KParams *d_kp = nullptr;
    cudaGraph_t dgraph[2] = {nullptr, nullptr};
    cudaGraphExec_t dexec[2] = {nullptr, nullptr};
};

// Device memory of a handle comes from a PRIVATE stream-ordered pool per device
// (cudaMemPoolCreate; never the device's default pool, so no other library's
// cudaMallocAsync is affected), allocated and freed on the handle's stream.  The
// pool's release threshold is unbounded so that memory freed by one handle can be
// reused by the next load in the same process without re-mapping (plain
// cudaMalloc / cudaFree of GB buffers measured 10-600 ms per call);
// atos_graph_free trims the pool back to zero unless cfg.pool_retain is set, so
// by default a freed graph's memory goes back to the device (and to torch's
// allocator).  The arena of a multi-process handle stays on cudaMalloc: it is
// exported with cudaIpcGetMemHandle.
#include <mutex>
static cudaMemPool_t pool_of(int device) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {nullptr};
    if (device < 0 || device >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[device]) {
        cudaMemPoolProps pr{};
        pr.allocType = cudaMemAllocationTypePinned;
        pr.location.type = cudaMemLocationTypeDevice;
        pr.location.id = device;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &pr) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[device] = p;
    }
    return pools[device];
}
// Exact-size cache of large blocks for handles with pool_retain = 1 (load/solve/free
// loops).  The pool alone kept the memory mapped but re-split it differently from one
// load to the next, and a request that no longer fit mapped new memory synchronously
// inside cudaMallocFromPoolAsync (40-800 ms stalls in random load phases, e2e trace).
// A retained handle's large blocks are parked here at free and handed out again for
// the same size; a handle with pool_retain = 0 empties the cache at its free.
constexpr size_t kCacheMin = (size_t)64 << 20;
struct BlockCache {
    std::mutex mu;
    std::vector<std::pair<size_t, void *>> parked;     // free blocks
    std::vector<std::pair<void *, size_t>> sizes;      // every cacheable block handed out
};
static BlockCache &block_cache(int device) {
    static BlockCache c[64];
    return c[device & 63];
}
template <typename T>
static cudaError_t dmalloc(const atos_graph *g, T **p, size_t bytes) {
    const bool cache = g->cfg.pool_retain && bytes >= kCacheMin;
    if (cache) {
        BlockCache &c = block_cache(g->cfg.device);
        std::lock_guard<std::mutex> lk(c.mu);
        for (size_t i = 0; i < c.parked.size(); ++i)
            if (c.parked[i].first == bytes) {
                *p = (T *)c.parked[i].second;
                c.parked.erase(c.parked.begin() + (long)i);
                return cudaSuccess;
            }
    }
    cudaMemPool_t pool = pool_of(g->cfg.device);
    const cudaError_t e = pool ? cudaMallocFromPoolAsync((void **)p, bytes, pool, g->stream)
                               : cudaMallocAsync((void **)p, bytes, g->stream);
    if (e == cudaSuccess && cache) {
        BlockCache &c = block_cache(g->cfg.device);
        std::lock_guard<std::mutex> lk(c.mu);
        c.sizes.emplace_back((void *)*p, bytes);
    }
    return e;
}
static void dfree(const atos_graph *g, void *p) {
    if (!p) return;
    if (g->cfg.pool_retain) {
        BlockCache &c = block_cache(g->cfg.device);
        std::lock_guard<std::mutex> lk(c.mu);
        for (const auto &x : c.sizes)
            if (x.first == p) {
                // the next user may be another handle on another stream: the block is
                // parked only once this handle's pending work on it is done
                cudaStreamSynchronize(g->stream);
                c.parked.emplace_back(x.second, p);
                return;
            }
    }
    cudaFreeAsync(p, g->stream);
}
// Release every parked block (a handle without pool_retain is being freed).
static void block_cache_release(const atos_graph *g) {
    BlockCache &c = block_cache(g->cfg.device);
    std::lock_guard<std::mutex> lk(c.mu);
    for (const auto &x : c.parked) {
        cudaFreeAsync(x.second, 0);     // (the handle's own stream may already be destroyed)
        for (size_t i = 0; i < c.sizes.size(); ++i)
            if (c.sizes[i].first == x.second) { c.sizes.erase(c.sizes.begin() + (long)i); break; }
    }
    c.parked.clear();
}

// dynamic shared memory of the worker: Smem, plus the BFS hub cache (one nibble per entry)
static size_t worker_smem(int app, int hub_chunks) {
    return sizeof(Smem) + (app == kApBfs ? (size_t)hub_chunks : 0);
}

// Dynamic smem limit, then the smallest shared-memory carve-out that still holds
// `want` CTAs per SM: the rest of the 256 KB unified L1/smem stays L1, which caches
// the hot (relabeled) part of the BFS depth words -- measured to matter.
template <typename F>
static cudaError_t kernel_setup_fn(F *fn, int &occ, size_t smem, int want) {
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const double need_kb = (double)want * ((double)(smem + 1024) / 1024.0);   // + 1 KB reserved per CTA
    int pct = (int)(need_kb / 228.0 * 100.0) + 1;
    pct = pct > 100 ? 100 : pct;
    e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kThreads, smem);
}
template <int APP, bool MULTI>
static cudaError_t kernel_setup(int &occ, size_t smem, int want) {
    return kernel_setup_fn(worker_kernel<APP, MULTI>, occ, smem, want);
}

static RankDev build_view(const atos_graph *g, int lr) {
    const LocalRank &me = g->loc[lr];
    const int r = me.rank;
    RankDev d{};
    d.rank = r;
    d.n_ranks = g->p;
    d.n = g->n;
    d.v_begin = g->part[r];
    d.v_end = g->part[r + 1];
    for (int k = 0; k <= kMaxRanks; ++k) d.part[k] = k <= g->p ? g->part[k] : g->n;
    d.row_ptr = me.row_ptr;
    d.col = me.col;
    unsigned char *b = me.arena;
    const Layout &L = me.L;
    d.depth = (uint32_t *)(b + L.depth);
    d.filt = (uint8_t *)(b + L.filt);
    d.hcb = (uint8_t *)(b + L.hcb);
    d.vis = (g->S.pq && g->p == 1) ? (uint32_t *)(b + L.vis) : nullptr;
    d.pr_rank = (double *)(b + L.rank);
    d.pr_res = (double *)(b + L.res);
    d.pr_q = pr_q_of(L.n_r);
    d.pr_ghost = (g->p > 1 && g->S.combine) ? (double *)(b + L.ghost) : nullptr;
    d.ring = (uint64_t *)(b + L.ring);
    d.ring2 = g->S.pq ? (uint64_t *)(b + L.ring2) : nullptr;
    d.ring_cap = L.ring_cap;
    d.ctrl = (Ctrl *)(b + L.ctrl);
    const size_t cp = (size_t)g->S.cp, pkt = (size_t)g->S.pkt;
    d.staging = b + L.staging;
    d.perm = g->d_perm;
    d.inv = g->d_inv;
    for (int s = 0; s < g->p; ++s) {
        // base pointer of rank s's arena as seen from this process
        unsigned char *bs = nullptr;
        if (!g->multiproc) bs = g->loc[s].arena;             // virtual ranks / single rank
        else bs = (s == r) ? b : g->peer_base[s];
        if (!bs) continue;
        const Layout Ls = g->multiproc ? make_layout(g->S, g->part.data(), s) : g->loc[s].L;
        d.peer_ctrl[s] = (Ctrl *)(bs + Ls.ctrl);
        d.peer_depth[s] = (uint32_t *)(bs + Ls.depth);
        d.peer_rank[s] = (double *)(bs + Ls.rank);
        d.peer_res[s] = (double *)(bs + Ls.res);
        d.peer_ghost[s] = (g->p > 1 && g->S.combine) ? (double *)(bs + Ls.ghost) : nullptr;
        if (g->p > 1) {
            d.in_hdr[s] = (uint64_t *)(b + L.in_hdr + (size_t)s * cp * 8);
            d.in_payload[s] = b + L.in_pay + (size_t)s * cp * pkt * 16;
            d.free_mirror[s] = (uint64_t *)(b + L.free_m + (size_t)s * cp * 8);
            d.out_hdr[s] = (uint64_t *)(bs + Ls.in_hdr + (size_t)r * cp * 8);
            d.out_payload[s] = bs + Ls.in_pay + (size_t)r * cp * pkt * 16;
            d.peer_free[s] = (uint64_t *)(bs + Ls.free_m + (size_t)r * cp * 8);
        }
    }
    return d;
}

__global__ void rebase_rows_kernel(int64_t *rp, int64_t n1, int64_t base) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n1; i += (int64_t)gridDim.x * blockDim.x)
        rp[i] -= base;
}

__global__ void check_rows_kernel(const int64_t *rp, int64_t nr, int64_t m, const int32_t *col, int64_t n,
                                  unsigned long long *bad) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nr; i += stride)
        if (rp[i + 1] < rp[i]) atomicOr(bad, 1ull);
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < m; e += stride)
        if (col[e] < 0 || col[e] >= n) atomicOr(bad, 2ull);
}

__global__ void init_arena_kernel(uint64_t *ring, uint64_t cap, uint64_t *free_m, uint64_t nfree, uint64_t cps) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += stride)
        ring[i] = pack(lo32(i), 0u);   // free for the producer of index i
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nfree; i += stride)
        free_m[i] = i % cps;           // slot of sub-channel packet index j (< cps) free for index j
}

// ---------------------------------------------------------------------------
// degree relabeling: inside every rank block, vertices
// are renumbered by out-degree, descending (ties by id), so that each block's
// hubs have its smallest ids -- the BFS hub cache covers them, and the hot part
// of the state arrays is compact in L2.  The partition itself is unchanged.
// ---------------------------------------------------------------------------
__global__ void degree_keys_kernel(const int64_t *rp, int64_t n, uint32_t *keys, int32_t *vals,
                                   unsigned long long *maxdeg) {
    unsigned long long mx = 0;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int64_t d = rp[v + 1] - rp[v];
        d = d < 0 ? 0 : (d > 0xFFFFFFFEll ? 0xFFFFFFFEll : d);
        keys[v] = 0xFFFFFFFFu - (uint32_t)d;      // ascending key == descending degree
        vals[v] = (int32_t)v;
        mx = (unsigned long long)d > mx ? (unsigned long long)d : mx;
    }
    atomicMax(maxdeg, mx);
}

__global__ void invert_perm_kernel(const int32_t *inv, int64_t n, int32_t *perm) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        perm[inv[i]] = (int32_t)i;
}

// deg_new[i] = out-degree of the vertex that gets local id i (old rows rebased to the rank)
__global__ void new_degrees_kernel(const int64_t *rp_old, const int32_t *inv, int64_t v0, int64_t nr,
                                   int64_t *deg_new) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= nr; i += (int64_t)gridDim.x * blockDim.x) {
        if (i == nr) { deg_new[i] = 0; continue; }
        const int64_t l = (int64_t)inv[v0 + i] - v0;
        deg_new[i] = rp_old[l + 1] - rp_old[l];
    }
}

// one warp per new row: copy the old row, mapping every target through perm
__global__ void permute_rows_kernel(const int64_t *rp_old, const int32_t *col_old, const int32_t *inv,
                                    const int32_t *perm, int64_t v0, int64_t nr, const int64_t *rp_new,
                                    int32_t *col_new) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < nr; i += nw) {
        const int64_t l = (int64_t)inv[v0 + i] - v0;
        const int64_t b = rp_old[l], d = rp_old[l + 1] - b, o = rp_new[i];
        for (int64_t k = lane; k < d; k += 32) col_new[o + k] = perm[col_old[b + k]];
    }
}

// Streamed variant for a host column array: old rows [l0, l1) restricted to the
// staged column range [c0, c1) (rank-relative offsets), one warp per old row;
// column ids are range-checked here (they are never checked elsewhere on this path).
// One warp per old row clipped to the chunk; a row with more than kPermLong
// edges in the chunk is deferred to permute_long_kernel (one CTA per row), so a
// hub row does not leave one warp running long after the rest of the grid (the
// last chunk of RMAT-24 took 11.8 ms against ~5 ms for the others).
constexpr int64_t kPermLong = 8192;
__global__ void permute_chunk_kernel(const int64_t *rp_old, const int32_t *stage, int64_t c0, int64_t c1,
                                     int64_t l0, int64_t l1, const int32_t *perm, int64_t v0,
                                     const int64_t *rp_new, int32_t *col_new, int64_t n, unsigned long long *bad,
                                     int64_t *long_rows, unsigned int *n_long) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t l = l0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); l < l1; l += nw) {
        const int64_t b = rp_old[l], e = rp_old[l + 1];
        const int64_t lo = b > c0 ? b : c0, hi = e < c1 ? e : c1;
        if (lo >= hi) continue;
        if (hi - lo > kPermLong) {
            if (lane == 0) long_rows[atomicAdd(n_long, 1u)] = l;
            continue;
        }
        const int64_t o = rp_new[perm[v0 + l] - v0] + (lo - b);
        for (int64_t k = lane; k < hi - lo; k += 32) {
            int32_t x = stage[lo - c0 + k];
            if (x < 0 || (int64_t)x >= n) { atomicOr(bad, 2ull); x = 0; }
            col_new[o + k] = perm[x];
        }
    }
}

__global__ void permute_long_kernel(const int64_t *rp_old, const int32_t *stage, int64_t c0, int64_t c1,
                                    const int32_t *perm, int64_t v0, const int64_t *rp_new, int32_t *col_new, int64_t n,
                                    unsigned long long *bad, const int64_t *long_rows, const unsigned int *n_long) {
    for (unsigned int i = blockIdx.x; i < *n_long; i += gridDim.x) {
        const int64_t l = long_rows[i];
        const int64_t b = rp_old[l], e = rp_old[l + 1];
        const int64_t lo = b > c0 ? b : c0, hi = e < c1 ? e : c1;
        const int64_t o = rp_new[perm[v0 + l] - v0] + (lo - b);
        for (int64_t k = threadIdx.x; k < hi - lo; k += blockDim.x) {
            int32_t x = stage[lo - c0 + k];
            if (x < 0 || (int64_t)x >= n) { atomicOr(bad, 2ull); x = 0; }
            col_new[o + k] = perm[x];
        }
    }
}

static bool is_device_ptr(const void *p) {
    if (!p) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

static atos_status upload_views(atos_graph *g) {
    std::vector<RankDev> v(g->n_local);
    for (int lr = 0; lr < g->n_local; ++lr) v[lr] = build_view(g, lr);
    CU(cudaMemcpyAsync(g->d_ranks, v.data(), sizeof(RankDev) * g->n_local, cudaMemcpyHostToDevice, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    return ATOS_OK;
}

static KParams make_params(atos_graph *g);

// hub bounds: vertices covered (multiple of 128, <= n) and the array size
static int hub_n_for(const atos_config &cfg, int64_t n) {
    int64_t h = cfg.hub_cache < 0 ? kHubAutoN : cfg.hub_cache;
    h = std::min<int64_t>(h, n);
    return (int)(h - h % 128);
}
static int hub_chunks_for(int hub_n) { return ((hub_n / 128 + 15) / 16) * 16; }

extern "C" atos_status atos_graph_free(atos_graph *g) {
    if (!g) return ATOS_OK;
    cudaSetDevice(g->cfg.device);
    if (g->stream) cudaStreamSynchronize(g->stream);
    if (g->multiproc && g->connected && !g->poisoned && g->d_ranks) {
        // peers may still be reading this rank's arena over NVLink (the gather and
        // parent passes of the last solve): every rank arrives here before any
        // rank unmaps or frees (epoch*4+2: above every barrier value of the solve)
        KParams kp = make_params(g);
        barrier_kernel<<<1, 32, 0, g->stream>>>(kp, g->epoch * 4 + 2);
        cudaStreamSynchronize(g->stream);
    }
    for (int s = 0; s < kMaxRanks; ++s)
        if (g->peer_opened[s]) cudaIpcCloseMemHandle(g->peer_base[s]);
    for (int lr = 0; lr < g->n_local; ++lr) {
        if (g->multiproc) cudaFree(g->loc[lr].arena);
        else dfree(g, g->loc[lr].arena);
        dfree(g, g->loc[lr].row_ptr);
        dfree(g, g->loc[lr].col);
    }
    dfree(g, g->d_ranks);
    dfree(g, g->d_depth_full);
    dfree(g, g->d_perm);
    dfree(g, g->d_inv);
    dfree(g, g->rp_dev_tmp);
    dfree(g, g->d_accs);
    if (g->stream) cudaStreamSynchronize(g->stream);
    for (int a = 0; a < 2; ++a) {
        if (g->dexec[a]) cudaGraphExecDestroy(g->dexec[a]);
        if (g->dgraph[a]) cudaGraphDestroy(g->dgraph[a]);
    }
    if (g->d_kp) cudaFree(g->d_kp);
    if (g->ev_begin) cudaEventDestroy(g->ev_begin);
    if (g->ev_w0) cudaEventDestroy(g->ev_w0);
    if (g->ev_w1) cudaEventDestroy(g->ev_w1);
    if (g->ev_end) cudaEventDestroy(g->ev_end);
    if (g->own_stream && g->stream) cudaStreamDestroy(g->stream);
    if (!g->cfg.pool_retain) {
        block_cache_release(g);
        cudaDeviceSynchronize();
        if (cudaMemPool_t pool = pool_of(g->cfg.device)) cudaMemPoolTrimTo(pool, 0);   // freed memory back to the device
    }
    delete g;
    return ATOS_OK;
}

struct GraphGuard {
    atos_graph *g;
    ~GraphGuard() { if (g) atos_graph_free(g); }
};

extern "C" atos_status atos_arena_bytes(int64_t n, const int64_t *part, int32_t n_ranks, int32_t rank,
                                        const atos_config *cfg_in, uint64_t *bytes_out) {
    atos_config cfg;
    if (cfg_in) cfg = *cfg_in; else atos_config_init(&cfg);
    if (!bytes_out || n < 1 || n_ranks < 1 || n_ranks > kMaxRanks || rank < 0 || rank >= n_ranks)
        return fail(ATOS_ERR_INVALID_ARG, "arena_bytes: bad arguments");
    std::vector<int64_t> pt(n_ranks + 1);
    if (part) std::copy(part, part + n_ranks + 1, pt.begin());
    else atos_partition_balanced(n, n_ranks, pt.data());
    Shape S{n, n_ranks, cfg.channel_packets, cfg.agg_batch_msgs, stage_cap_for(cfg.agg_batch_msgs),
            148 * (cfg.ctas_per_sm ? cfg.ctas_per_sm : 2) / (cfg.virtual_ranks > 1 ? cfg.virtual_ranks : 1),
            cfg.fetch_size, cfg.ring_cap_factor, cfg.pr_combine, 0, pq_layout(cfg, n)};
    *bytes_out = make_layout(S, pt.data(), rank).total;
    return ATOS_OK;
}

struct DevFrees {   // scratch device buffers of graph_load, freed on every exit path
    const atos_graph *g;
    std::vector<void *> p;
    explicit DevFrees(const atos_graph *g_) : g(g_) {}
    ~DevFrees() { for (void *x : p) dfree(g, x); }
};

// Compute g->d_inv / g->d_perm (all rank blocks, identically on every process).
// relabel == 2 decides from the degree skew and may leave them NULL.
static atos_status compute_relabel(atos_graph *g, const int64_t *row_ptr, bool rp_dev) {
    const int64_t n = g->n;
    cudaStream_t st = g->stream;
    DevFrees fr(g);
    const int64_t *rpf = row_ptr;
    if (!rp_dev) {
        int64_t *t = nullptr;
        CU(dmalloc(g, &t, (size_t)(n + 1) * 8));
        g->rp_dev_tmp = t;     // (graph_load copies the ranks' rows from it and frees it)
        CU(cudaMemcpyAsync(t, row_ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, st));
        rpf = t;
    }
    uint32_t *k0 = nullptr, *k1 = nullptr;
    int32_t *v0 = nullptr;
    unsigned long long *d_max = nullptr;
    CU(dmalloc(g, &k0, (size_t)n * 4)); fr.p.push_back(k0);
    CU(dmalloc(g, &k1, (size_t)n * 4)); fr.p.push_back(k1);
    CU(dmalloc(g, &v0, (size_t)n * 4)); fr.p.push_back(v0);
    CU(dmalloc(g, &d_max, 8)); fr.p.push_back(d_max);
    CU(cudaMemsetAsync(d_max, 0, 8, st));
    LoadTrace tr;
    tr.mark(st, "  relabel: row_ptr + scratch");
    degree_keys_kernel<<<1024, 256, 0, st>>>(rpf, n, k0, v0, d_max);
    CU(cudaGetLastError());
    unsigned long long mx = 0;
    CU(cudaMemcpyAsync(&mx, d_max, 8, cudaMemcpyDeviceToHost, st));
    CU(cudaStreamSynchronize(st));
    const double mean = (double)g->nnz / (double)n;
    g->skewed = (double)mx >= 32.0 * std::max(1.0, mean);
    if (g->cfg.relabel == 0) return ATOS_OK;                           // degree statistics only
    if (g->cfg.relabel == 2 && !g->skewed) return ATOS_OK;              // not skewed: keep the given order
    tr.mark(st, "  relabel: degree keys");
    CU(dmalloc(g, &g->d_inv, (size_t)n * 4));
    CU(dmalloc(g, &g->d_perm, (size_t)n * 4));
    int64_t maxlen = 0;
    for (int r = 0; r < g->p; ++r) maxlen = std::max(maxlen, g->part[r + 1] - g->part[r]);
    size_t tb = 0;
    CU(cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, v0, g->d_inv, (int)maxlen, 0, 32, st));
    void *tmp = nullptr;
    CU(dmalloc(g, &tmp, std::max<size_t>(tb, 16)));
    fr.p.push_back(tmp);
    for (int r = 0; r < g->p; ++r) {
        const int64_t b = g->part[r], len = g->part[r + 1] - b;
        if (len <= 0) continue;
        size_t t2 = tb;
        CU(cub::DeviceRadixSort::SortPairs(tmp, t2, k0 + b, k1 + b, v0 + b, g->d_inv + b, (int)len, 0, 32, st));
    }
    tr.mark(st, "  relabel: sort");
    invert_perm_kernel<<<1024, 256, 0, st>>>(g->d_inv, n, g->d_perm);
    CU(cudaGetLastError());
    CU(cudaStreamSynchronize(st));
    return ATOS_OK;
}

// Replace rank lr's (validated, rebased) rows by the relabeled ones.
static atos_status relabel_rows(atos_graph *g, LocalRank &me) {
    cudaStream_t st = g->stream;
    const int64_t v0 = g->part[me.rank], nr = me.L.n_r;
    DevFrees fr(g);
    int64_t *deg = nullptr, *rp_new = nullptr;
    int32_t *col_new = nullptr;
    CU(dmalloc(g, &deg, (size_t)(nr + 1) * 8)); fr.p.push_back(deg);
    CU(dmalloc(g, &rp_new, (size_t)(nr + 1) * 8)); fr.p.push_back(rp_new);
    CU(dmalloc(g, &col_new, ((size_t)me.m_r + kColPad) * 4)); fr.p.push_back(col_new);
    new_degrees_kernel<<<1024, 256, 0, st>>>(me.row_ptr, g->d_inv, v0, nr, deg);
    size_t tb = 0;
    CU(cub::DeviceScan::ExclusiveSum(nullptr, tb, deg, rp_new, (int64_t)(nr + 1), st));
    void *tmp = nullptr;
    CU(dmalloc(g, &tmp, std::max<size_t>(tb, 16)));
    fr.p.push_back(tmp);
    CU(cub::DeviceScan::ExclusiveSum(tmp, tb, deg, rp_new, (int64_t)(nr + 1), st));
    permute_rows_kernel<<<2048, 256, 0, st>>>(me.row_ptr, me.col, g->d_inv, g->d_perm, v0, nr, rp_new, col_new);
    CU(cudaGetLastError());
    CU(cudaStreamSynchronize(st));
    dfree(g, me.row_ptr);
    dfree(g, me.col);
    me.row_ptr = rp_new;
    me.col = col_new;
    fr.p.erase(std::remove(fr.p.begin(), fr.p.end(), (void *)rp_new), fr.p.end());
    fr.p.erase(std::remove(fr.p.begin(), fr.p.end(), (void *)col_new), fr.p.end());
    return ATOS_OK;
}

// Relabeled rows of rank `me` straight from a HOST column array: the columns are
// streamed in chunks through two device staging buffers on a second stream, and
// each chunk is permuted into place while the next one is copied, so the H2D
// transfer (the dominant cost of an end-to-end load) overlaps the permutation
// instead of preceding it.  me.row_ptr must be copied, rebased and validated.
static atos_status relabel_rows_streamed(atos_graph *g, LocalRank &me, const int64_t *rp_host, const int32_t *col_host,
                                         unsigned long long *d_bad) {
    cudaStream_t st = g->stream;
    const int r = me.rank;
    const int64_t v0 = g->part[r], nr = me.L.n_r, m = me.m_r, base = rp_host[v0];
    DevFrees fr(g);
    int64_t *deg = nullptr, *rp_new = nullptr;
    int32_t *col_new = nullptr;
    CU(dmalloc(g, &deg, (size_t)(nr + 1) * 8)); fr.p.push_back(deg);
    CU(dmalloc(g, &rp_new, (size_t)(nr + 1) * 8)); fr.p.push_back(rp_new);
    CU(dmalloc(g, &col_new, ((size_t)m + kColPad) * 4)); fr.p.push_back(col_new);
    new_degrees_kernel<<<1024, 256, 0, st>>>(me.row_ptr, g->d_inv, v0, nr, deg);
    size_t tb = 0;
    CU(cub::DeviceScan::ExclusiveSum(nullptr, tb, deg, rp_new, (int64_t)(nr + 1), st));
    void *tmp = nullptr;
    CU(dmalloc(g, &tmp, std::max<size_t>(tb, 16)));
    fr.p.push_back(tmp);
    CU(cub::DeviceScan::ExclusiveSum(tmp, tb, deg, rp_new, (int64_t)(nr + 1), st));
    int64_t ch = (int64_t)1 << 26;                  // 256 MB per stage
    if (const char *e = std::getenv("ATOS_LOAD_CHUNK")) ch = std::max<int64_t>(1, std::atoll(e));   // tests: many chunks
    const int64_t CH = std::min<int64_t>(std::max<int64_t>(m, 1), ch);
    int32_t *stage[2] = {nullptr, nullptr};
    for (int k = 0; k < 2; ++k) { CU(dmalloc(g, &stage[k], (size_t)CH * 4)); fr.p.push_back(stage[k]); }
    int64_t *long_rows = nullptr;            // rows deferred to permute_long_kernel (> kPermLong edges in a chunk)
    unsigned int *n_long = nullptr;
    CU(dmalloc(g, &long_rows, (size_t)(CH / kPermLong + 2) * 8)); fr.p.push_back(long_rows);
    CU(dmalloc(g, &n_long, sizeof(unsigned int))); fr.p.push_back(n_long);
    cudaStream_t cs = nullptr;
    CU(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    cudaEvent_t ev_in[2], ev_out[2], ev_ready;
    for (int k = 0; k < 2; ++k) {
        CU(cudaEventCreateWithFlags(&ev_in[k], cudaEventDisableTiming));
        CU(cudaEventCreateWithFlags(&ev_out[k], cudaEventDisableTiming));
    }
    CU(cudaEventCreateWithFlags(&ev_ready, cudaEventDisableTiming));
    CU(cudaEventRecord(ev_ready, st));           // rp_new and the row offsets are ready
    CU(cudaStreamWaitEvent(cs, ev_ready, 0));
    atos_status status = ATOS_OK;
    const bool trace = std::getenv("ATOS_LOAD_TRACE") != nullptr;
    std::vector<cudaEvent_t> tev;
    auto tmark = [&](cudaStream_t s_) {
        if (!trace) return;
        cudaEvent_t e_;
        cudaEventCreate(&e_);
        cudaEventRecord(e_, s_);
        tev.push_back(e_);
    };
    for (int64_t c0 = 0, k = 0; c0 < m && status == ATOS_OK; c0 += CH, ++k) {
        const int64_t c1 = std::min(m, c0 + CH);
        const int b = (int)(k & 1);
        // rows overlapping [c0, c1): first row ending after c0 .. first row starting at/after c1
        const int64_t *rp = rp_host + v0;
        const int64_t l0 = (int64_t)(std::upper_bound(rp, rp + nr + 1, base + c0) - rp) - 1;
        const int64_t l1 = (int64_t)(std::lower_bound(rp, rp + nr + 1, base + c1) - rp);
        if (k >= 2 && cudaStreamWaitEvent(cs, ev_out[b], 0) != cudaSuccess) status = fail(ATOS_ERR_CUDA, "stream wait");
        tmark(cs);
        if (cudaMemcpyAsync(stage[b], col_host + base + c0, (size_t)(c1 - c0) * 4, cudaMemcpyHostToDevice, cs) != cudaSuccess)
            status = fail(ATOS_ERR_CUDA, "cudaMemcpyAsync of a column chunk failed");
        tmark(cs);
        cudaEventRecord(ev_in[b], cs);
        cudaStreamWaitEvent(st, ev_in[b], 0);
        tmark(st);
        cudaMemsetAsync(n_long, 0, sizeof(unsigned int), st);
        permute_chunk_kernel<<<2048, 256, 0, st>>>(me.row_ptr, stage[b], c0, c1, std::max<int64_t>(l0, 0),
                                                  std::min(l1, nr), g->d_perm, v0, rp_new, col_new, g->n, d_bad,
                                                  long_rows, n_long);
        permute_long_kernel<<<1024, 512, 0, st>>>(me.row_ptr, stage[b], c0, c1, g->d_perm, v0, rp_new, col_new, g->n,
                                                 d_bad, long_rows, n_long);
        tmark(st);
        cudaEventRecord(ev_out[b], st);
    }
    const cudaError_t e = cudaStreamSynchronize(st);
    cudaStreamSynchronize(cs);
    for (size_t i = 0; i + 3 < tev.size(); i += 4) {
        float t[4] = {0, 0, 0, 0};
        for (int j = 0; j < 4; ++j) cudaEventElapsedTime(&t[j], tev[0], tev[i + j]);
        fprintf(stderr, "[atos load]   chunk %zu: copy %.2f ms, permute %.2f ms (copy %.2f-%.2f, permute %.2f-%.2f ms)\n",
                i / 4, t[1] - t[0], t[3] - t[2], t[0], t[1], t[2], t[3]);
    }
    for (cudaEvent_t x : tev) cudaEventDestroy(x);
    for (int k = 0; k < 2; ++k) { cudaEventDestroy(ev_in[k]); cudaEventDestroy(ev_out[k]); }
    cudaEventDestroy(ev_ready);
    cudaStreamDestroy(cs);
    if (status != ATOS_OK) return status;
    if (e != cudaSuccess) return fail(ATOS_ERR_CUDA, "streamed relabel: %s", cudaGetErrorString(e));
    dfree(g, me.row_ptr);
    me.row_ptr = rp_new;
    me.col = col_new;
    fr.p.erase(std::remove(fr.p.begin(), fr.p.end(), (void *)rp_new), fr.p.end());
    fr.p.erase(std::remove(fr.p.begin(), fr.p.end(), (void *)col_new), fr.p.end());
    return ATOS_OK;
}

extern "C" atos_status atos_graph_load(const int64_t *row_ptr, const int32_t *col, int64_t n, int64_t nnz,
                                       const int64_t *part, const atos_config *cfg_in, atos_graph **out) {
    if (!out) return fail(ATOS_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    atos_config cfg;
    if (cfg_in) cfg = *cfg_in; else atos_config_init(&cfg);
    if (!valid_cfg(cfg)) return fail(ATOS_ERR_INVALID_ARG, "invalid atos_config");
    if (!row_ptr || (nnz > 0 && !col) || n < 1 || n > INT32_MAX || nnz < 0)
        return fail(ATOS_ERR_INVALID_ARG, "graph_load: need 1<=n<=2^31-1, nnz>=0, non-NULL arrays");
    int ndev = 0;
    CU(cudaGetDeviceCount(&ndev));
    if (cfg.device >= ndev) return fail(ATOS_ERR_INVALID_ARG, "device %d not visible (%d devices)", cfg.device, ndev);
    CU(cudaSetDevice(cfg.device));

    atos_graph *g = new (std::nothrow) atos_graph();
    if (!g) return fail(ATOS_ERR_OOM, "host allocation failed");
    GraphGuard guard{g};
    g->cfg = cfg;
    g->n = n;
    g->nnz = nnz;
    g->multiproc = cfg.n_ranks > 1;
    g->p = g->multiproc ? cfg.n_ranks : cfg.virtual_ranks;
    g->n_local = g->multiproc ? 1 : cfg.virtual_ranks;
    g->part.resize(g->p + 1);
    if (part) {
        std::copy(part, part + g->p + 1, g->part.begin());
        if (g->part[0] != 0 || g->part[g->p] != n)
            return fail(ATOS_ERR_INVALID_ARG, "part must start at 0 and end at n");
        for (int r = 0; r < g->p; ++r)
            if (g->part[r + 1] < g->part[r]) return fail(ATOS_ERR_INVALID_ARG, "part not monotone");
    } else {
        atos_partition_balanced(n, g->p, g->part.data());
    }
    if (pq_layout(cfg, n))     // priority queue items carry a bucket tag in bit 30
        for (int r = 0; r < g->p; ++r)
            if (g->part[r + 1] - g->part[r] >= ((int64_t)1 << 30))
                return fail(ATOS_ERR_INVALID_ARG, "priority queue: rank blocks must hold < 2^30 vertices");

    // row offsets at partition boundaries (host copies of a few entries)
    const bool rp_dev = is_device_ptr(row_ptr);
    std::vector<int64_t> rb(g->p + 1);
    for (int r = 0; r <= g->p; ++r) {
        if (rp_dev) CU(cudaMemcpy(&rb[r], row_ptr + g->part[r], 8, cudaMemcpyDeviceToHost));
        else rb[r] = row_ptr[g->part[r]];
    }
    if (rb[0] != 0 || rb[g->p] != nnz) return fail(ATOS_ERR_INVALID_ARG, "row_ptr[0] must be 0 and row_ptr[n]==nnz");

    // device / occupancy
    cudaDeviceProp prop;
    CU(cudaGetDeviceProperties(&prop, cfg.device));
    g->sms = prop.multiProcessorCount;
    g->persist_max = (size_t)prop.persistingL2CacheMaxSize;
    g->window_max = (size_t)prop.accessPolicyMaxWindowSize;
    // (the persisting carve-out itself is sized per launch to the window, see launch_worker:
    //  a carve-out larger than the window would only shrink the L2 left to everything else)
    if (!prop.cooperativeLaunch) return fail(ATOS_ERR_CUDA, "device lacks cooperative launch");
    // hub bounds (atos_bfs1.cuh): the largest size they can take decides the BFS
    // kernel's shared memory; the actual size is set once relabeling is known
    const int hub_max = g->p == 1 ? hub_n_for(cfg, n) : 0;
    const int want = cfg.ctas_per_sm > 0 ? cfg.ctas_per_sm : 1024 / kThreads;
    const size_t smem_bfs = worker_smem(kApBfs, hub_chunks_for(hub_max)), smem_pr = worker_smem(kApPr, 0);
    int occ0 = 0, occ1 = 0, occ2 = 0, occ3 = 0;   // single- and multi-rank specialisations
    CU((kernel_setup<kApBfs, false>(occ0, smem_bfs, want)));
    CU((kernel_setup<kApPr, false>(occ1, smem_pr, want)));
    CU((kernel_setup<kApBfs, true>(occ2, smem_bfs, want)));
    CU((kernel_setup<kApPr, true>(occ3, smem_pr, want)));
    g->occ = std::min(std::min(occ0, occ1), std::min(occ2, occ3));
    if (cfg.discrete) {
        int occ4 = 0, occ5 = 0;
        CU(kernel_setup_fn(worker_discrete_kernel<kApBfs>, occ4, smem_bfs, want));
        CU(kernel_setup_fn(worker_discrete_kernel<kApPr>, occ5, smem_pr, want));
        g->occ = std::min(g->occ, std::min(occ4, occ5));
    }
    if (cfg.ctas_per_sm > 0) g->occ = std::min(g->occ, cfg.ctas_per_sm);
    if (g->occ < 1) return fail(ATOS_ERR_CUDA, "worker kernel cannot be resident (occupancy 0)");
    const int ctas_total = g->occ * g->sms;
    const int cpr = ctas_total / g->n_local;
    if (cpr < 1) return fail(ATOS_ERR_INVALID_ARG, "too many virtual ranks for the device");
    g->grid = cpr * g->n_local;
    g->S = Shape{n, g->p, cfg.channel_packets, cfg.agg_batch_msgs, stage_cap_for(cfg.agg_batch_msgs), cpr,
                 cfg.fetch_size, cfg.ring_cap_factor, cfg.pr_combine, 0, pq_layout(cfg, n)};

    if (cfg.stream) {
        g->stream = (cudaStream_t)cfg.stream;
    } else {
        CU(cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking));
        g->own_stream = true;
    }
    CU(cudaEventCreate(&g->ev_begin));
    CU(cudaEventCreate(&g->ev_w0));
    CU(cudaEventCreate(&g->ev_w1));
    CU(cudaEventCreate(&g->ev_end));

    LoadTrace tr;
    tr.mark(g->stream, "setup");
    if ((cfg.relabel != 0 || cfg.keep_items < 0 || (g->S.pq && cfg.pq_delta < 0)) && n > 1) {
        atos_status rs = compute_relabel(g, row_ptr, rp_dev);
        tr.mark(g->stream, "compute_relabel");
        if (rs != ATOS_OK) return rs;
    }

    // hub bounds only on relabeled (skewed) single-rank graphs: ids [0, hub_n) are the hubs
    if (hub_max > 0 && g->d_perm) {
        g->hub_n = hub_max;
        g->hub_chunks = hub_chunks_for(hub_max);
        g->S.hub_chunks = g->hub_chunks;
    }
    unsigned long long *d_bad = nullptr;
    CU(dmalloc(g, &d_bad, sizeof(unsigned long long)));   // (stream-ordered: cudaMalloc/cudaFree synchronise the device)
    CU(cudaMemsetAsync(d_bad, 0, sizeof(unsigned long long), g->stream));
    for (int lr = 0; lr < g->n_local; ++lr) {
        LocalRank &me = g->loc[lr];
        me.rank = g->multiproc ? cfg.rank : lr;
        const int r = me.rank;
        me.L = make_layout(g->S, g->part.data(), r);
        const int64_t nr = me.L.n_r;
        me.m_r = rb[r + 1] - rb[r];
        if (g->multiproc) CU(cudaMalloc(&me.arena, me.L.total));   // IPC-exported
        else CU(dmalloc(g, &me.arena, me.L.total));
        CU(cudaMemsetAsync(me.arena, 0, me.L.total, g->stream));
        tr.mark(g->stream, "arena");
        // host CSR + relabeling: stream the columns through the permutation (no
        // full-size device copy of the unpermuted columns)
        const char *se = std::getenv("ATOS_LOAD_STREAMED");
        const bool streamed = g->d_perm && me.m_r > 0 && !rp_dev && !is_device_ptr(col) && !(se && se[0] == '0');
        CU(dmalloc(g, &me.row_ptr, (size_t)(nr + 1) * 8));
        if (!streamed) CU(dmalloc(g, &me.col, ((size_t)me.m_r + kColPad) * 4));
        CU(cudaMemcpyAsync(me.row_ptr, (g->rp_dev_tmp ? g->rp_dev_tmp : row_ptr) + g->part[r], (size_t)(nr + 1) * 8,
                           cudaMemcpyDefault, g->stream));
        if (me.m_r > 0 && !streamed)
            CU(cudaMemcpyAsync(me.col, col + rb[r], (size_t)me.m_r * 4, cudaMemcpyDefault, g->stream));
        tr.mark(g->stream, "copy csr");
        rebase_rows_kernel<<<256, 256, 0, g->stream>>>(me.row_ptr, nr + 1, rb[r]);
        check_rows_kernel<<<1024, 256, 0, g->stream>>>(me.row_ptr, nr, streamed ? 0 : me.m_r, me.col, n, d_bad);
        tr.mark(g->stream, "check rows");
        if (streamed) {
            unsigned long long bad0 = 0;
            CU(cudaMemcpyAsync(&bad0, d_bad, sizeof(bad0), cudaMemcpyDeviceToHost, g->stream));
            CU(cudaStreamSynchronize(g->stream));
            if (bad0) { dfree(g, d_bad); return fail(ATOS_ERR_INVALID_ARG, "csr: row_ptr not monotone"); }
            atos_status rs = relabel_rows_streamed(g, me, row_ptr, col, d_bad);
            if (rs != ATOS_OK) { dfree(g, d_bad); return rs; }
            tr.mark(g->stream, "relabel rows (streamed)");
        } else if (g->d_perm) {   // rows must be valid before they are permuted
            unsigned long long bad0 = 0;
            CU(cudaMemcpyAsync(&bad0, d_bad, sizeof(bad0), cudaMemcpyDeviceToHost, g->stream));
            CU(cudaStreamSynchronize(g->stream));
            if (bad0) { dfree(g, d_bad); return fail(ATOS_ERR_INVALID_ARG, "csr: invalid row_ptr or column index"); }
            atos_status rs = relabel_rows(g, me);
            if (rs != ATOS_OK) { dfree(g, d_bad); return rs; }
            tr.mark(g->stream, "relabel rows");
        }
        const uint64_t nfree = g->p > 1 ? (uint64_t)g->p * g->S.cp : 0;
        init_arena_kernel<<<1024, 256, 0, g->stream>>>((uint64_t *)(me.arena + me.L.ring), me.L.ring_cap,
                                                       (uint64_t *)(me.arena + me.L.free_m), nfree,
                                                       (uint64_t)(g->S.cp / nsub_for(g->p, g->S.cp)));
        if (g->S.pq)
            init_arena_kernel<<<1024, 256, 0, g->stream>>>((uint64_t *)(me.arena + me.L.ring2), me.L.ring_cap,
                                                           nullptr, 0, 1);
        if (const char *e = std::getenv("ATOS_TEST_RING_BASE")) {
            // test-only: start every ring index at this value (tests start just below
            // 2^32 so that the 32-bit slot tags wrap during the solves)
            const uint64_t base = std::strtoull(e, nullptr, 0);
            for (int q = 0; q < (g->S.pq ? 2 : 1); ++q)
                qbench_init_kernel<<<1024, 256, 0, g->stream>>>((uint64_t *)(me.arena + (q ? me.L.ring2 : me.L.ring)),
                                                               me.L.ring_cap, base, 0);
            Ctrl *c = (Ctrl *)(me.arena + me.L.ctrl);
            for (uint64_t *f : {&c->head.v, &c->tail.v, &c->finished.v, &c->ring_base.v, &c->pq_head.v, &c->pq_tail.v,
                                &c->pq_fin.v, &c->pq_base.v})
                CU(cudaMemcpyAsync(f, &base, 8, cudaMemcpyHostToDevice, g->stream));
            CU(cudaStreamSynchronize(g->stream));
        }
        CU(cudaGetLastError());
    }
    dfree(g, g->rp_dev_tmp);
    g->rp_dev_tmp = nullptr;
    unsigned long long bad = 0;
    CU(cudaMemcpyAsync(&bad, d_bad, sizeof(bad), cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    dfree(g, d_bad);
    if (bad & 1) return fail(ATOS_ERR_INVALID_ARG, "csr: row_ptr not monotone");
    if (bad & 2) return fail(ATOS_ERR_INVALID_ARG, "csr: column index out of [0, n)");

    CU(dmalloc(g, &g->d_ranks, sizeof(RankDev) * g->n_local));
    CU(dmalloc(g, &g->d_depth_full, (size_t)n * 4));
    CU(dmalloc(g, &g->d_accs, sizeof(int64_t *) * kMaxRanks));
    g->connected = !g->multiproc;
    for (int lr = 0; lr < g->n_local; ++lr)    // the 16-B column loads of atos_bfs1.cuh need this
        if (((uintptr_t)g->loc[lr].col & 15) != 0)
            return fail(ATOS_ERR_CUDA, "column array not 16-B aligned (%p)", (void *)g->loc[lr].col);
    if (std::getenv("ATOS_DEBUG_PTRS"))
        for (int lr = 0; lr < g->n_local; ++lr)
            fprintf(stderr, "[atos] rank %d col %p row_ptr %p arena %p m_r %lld hub_n %d chunks %d smem %zu\n", lr,
                    (void *)g->loc[lr].col, (void *)g->loc[lr].row_ptr, (void *)g->loc[lr].arena,
                    (long long)g->loc[lr].m_r, g->hub_n, g->hub_chunks, worker_smem(kApBfs, g->hub_chunks));
    atos_status st = upload_views(g);
    if (st != ATOS_OK) return st;
    tr.mark(g->stream, "finish");
    guard.g = nullptr;
    *out = g;
    return ATOS_OK;
}

extern "C" atos_status atos_graph_export(atos_graph *g, void *handle_out) {
    if (!g || !handle_out) return fail(ATOS_ERR_INVALID_ARG, "export: NULL argument");
    if (!g->multiproc) return fail(ATOS_ERR_STATE, "export: handle is not multi-process (n_ranks == 1)");
    CU(cudaSetDevice(g->cfg.device));
    cudaIpcMemHandle_t h;
    static_assert(sizeof(h) == ATOS_IPC_HANDLE_BYTES, "IPC handle size");
    CU(cudaIpcGetMemHandle(&h, g->loc[0].arena));
    std::memcpy(handle_out, &h, sizeof(h));
    return ATOS_OK;
}

extern "C" atos_status atos_graph_connect(atos_graph *g, const void *handles) {
    if (!g || !handles) return fail(ATOS_ERR_INVALID_ARG, "connect: NULL argument");
    if (!g->multiproc) return fail(ATOS_ERR_STATE, "connect: handle is not multi-process");
    if (g->connected) return fail(ATOS_ERR_STATE, "connect: already connected");
    CU(cudaSetDevice(g->cfg.device));
    const unsigned char *hb = (const unsigned char *)handles;
    for (int s = 0; s < g->p; ++s) {
        if (s == g->cfg.rank) { g->peer_base[s] = g->loc[0].arena; continue; }
        cudaIpcMemHandle_t h;
        std::memcpy(&h, hb + (size_t)s * ATOS_IPC_HANDLE_BYTES, sizeof(h));
        void *ptr = nullptr;
        cudaError_t e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess)
            return fail(ATOS_ERR_PEER, "cudaIpcOpenMemHandle(rank %d) failed: %s", s, cudaGetErrorString(e));
        g->peer_base[s] = (unsigned char *)ptr;
        g->peer_opened[s] = true;
    }
    g->connected = true;
    return upload_views(g);
}

// ---------------------------------------------------------------------------
// solves
// ---------------------------------------------------------------------------
static KParams make_params(atos_graph *g) {
    KParams kp{};
    kp.ranks = g->d_ranks;
    kp.n_local = g->n_local;
    kp.ctas_per_rank = g->S.ctas_per_rank;
    kp.fetch = g->cfg.fetch_size;
    kp.pkt = g->S.pkt;
    kp.cp = g->S.cp;
    kp.nsub = nsub_for(g->p, g->S.cp);
    kp.cps = g->S.cp / kp.nsub;
    kp.stage_cap = g->S.stage_cap;
    kp.agg_on = g->cfg.agg_enabled;
    // auto keeping: only for a persistent single-rank solve on a non-skewed graph
    // (discrete launches chain without bound inside one launch: 87 edges per
    // m_reached on the grid; measured)
    kp.keep = g->cfg.keep_items >= 0 ? g->cfg.keep_items
                                     : ((g->skewed || g->cfg.discrete || g->p > 1) ? 0 : kKeepAuto);
    kp.keep_always = g->cfg.keep_items >= 0 ? g->cfg.keep_mode : 1;
    kp.keep_chain = 1 << 30;
    if (const char *e = std::getenv("ATOS_KEEP_CHAIN")) kp.keep_chain = std::max(1, std::atoi(e));   // experiment
    kp.prefetch = g->cfg.prefetch;
    kp.relax_red = g->cfg.relax_red;
    kp.pipe = g->cfg.pipeline;
    // probe filter: explicit, or automatically when the depth words do not fit the
    // L2 persisting carve-out (RMAT-26: 268 MB of words, 67 MB of filter)
    kp.filter = g->cfg.probe_filter == 1 ||
                (g->cfg.probe_filter == 2 && (g->skewed ||
                                              (size_t)g->n * 4 > (g->persist_max ? g->persist_max : (size_t)64 << 20)));
    kp.hub_n = g->hub_n;
    kp.hub_chunks = g->hub_chunks;
    // lean single-rank BFS expansion (atos_bfs1.cuh) for the default relaxation
    // (filter + red.min); ATOS_BFS_V1 selects the generic expansion (A/B)
    kp.bfs1 = g->p == 1 && kp.filter && kp.relax_red && !std::getenv("ATOS_BFS_V1");
    if (!kp.bfs1) kp.hub_n = kp.hub_chunks = 0;
    if (const char *e = std::getenv("ATOS_HUB_DBG")) kp.hub_dbg = std::atoi(e);   // experiment
    if (const char *e = std::getenv("ATOS_TIMELINE")) kp.timeline_ns = std::atoll(e) * 1000;   // experiment
    kp.split = g->cfg.split_edges < 0 ? kSplitAuto : g->cfg.split_edges;
    kp.combine = g->p > 1 && g->S.combine;
    // multi-rank PR with remote atomics: a delta for a remote vertex is added in the owner's
    // memory by the sender (one-sided atomic with return) and only a crossing of eps becomes a
    // message (PR RMAT-20, 2/4/8 virtual ranks: 56/84/121 -> 41/47/61 ms, same box; messages
    // 725 M -> 16 M at 2 ranks).  Virtual ranks only: their state is initialised before the one
    // grid starts, while separate processes would need a barrier between every rank's init and
    // any rank's first remote add, and cross-GPU atomics at system scope on every residual
    // update (the owner's own adds included).  ATOS_PR_NORATOM sends delta messages (A/B).
    kp.pr_ratom = g->p > 1 && !g->multiproc && !kp.combine && !std::getenv("ATOS_PR_NORATOM") ? 1 : 0;
    // multi-rank BFS the same way: a remote edge that improves the sender's ghost word lowers the
    // owner's depth word with atomicMin and sends an activation only on an improvement there
    // (RMAT-24 at 2/4/8 virtual ranks 12.2/16.5/21.6 -> 12.4/15.3/18.5 ms, same box; the grid at
    // 4 ranks unchanged).  Virtual ranks only, as pr_ratom; ATOS_BFS_NORATOM (A/B)
    kp.bfs_ratom = g->p > 1 && !g->multiproc && !std::getenv("ATOS_BFS_NORATOM") ? 1 : 0;
    kp.sys = g->multiproc ? 1 : 0;   // virtual ranks share this device: .gpu scope suffices
    // early next-batch reservation + per-warp enqueue: measured within noise
    // (RMAT-24/26 BFS, RMAT-20 PR); off unless ATOS_EARLY is set (experiment)
    kp.early = std::getenv("ATOS_EARLY") ? 1 : 0;
    kp.warp_flush = std::getenv("ATOS_WARP_FLUSH") ? 1 : 0;   // experiment
    kp.edge_map = std::getenv("ATOS_NO_EDGE_MAP") ? 0 : 1;     // A/B switch
    // round-robin chunks (no shared-memory claim per chunk): RMAT-24 3.06 -> 3.00 ms,
    // PR 12.65 -> 12.55 ms; ATOS_DYNAMIC_CHUNKS restores the claiming (A/B)
    kp.static_chunks = std::getenv("ATOS_DYNAMIC_CHUNKS") ? 0 : 1;
    if (const char *f = std::getenv("ATOS_TEST_FAULT"))   // test-only fault injection (T6 error paths)
        kp.fault = std::strcmp(f, "capacity") == 0 ? kFaultCapacity : std::strcmp(f, "timeout") == 0 ? kFaultTimeout : 0;
    if (g->S.pq && (g->cfg.pq_delta > 0 || g->skewed)) {
        // priority queue (N1): no work keeping (a kept chain would bypass the
        // buckets) and no early reservation (it is ring-0 only).  Auto
        // (pq_delta = -1, large single-rank graphs): level buckets on skewed
        // graphs; a non-skewed (high-diameter) graph keeps the FIFO queue and
        // work keeping, one bucket per level would serialise its ~10^4 levels
        const uint32_t delta = g->cfg.pq_delta > 0 ? (uint32_t)g->cfg.pq_delta : 1u;
        kp.pq = 1;
        kp.pq_delta = delta;
        kp.pq_th0 = g->cfg.pq_threshold > 0 ? (uint32_t)g->cfg.pq_threshold : delta;
        kp.keep = 0;
        kp.early = 0;
        // buckets = levels on one rank: the visited bitmap replaces the depth words
        // and the probe filter (atos_bfs1.cuh); ATOS_NO_VIS keeps them (A/B)
        kp.vis = kp.bfs1 && kp.pq_delta == 1 && kp.pq_th0 == 1 && !ATOS_FILTER4 && !std::getenv("ATOS_NO_VIS");
        if (kp.vis) kp.relax_red = 0;     // discoveries are decided by atomicOr with return: no fence before enqueue
        // claim at pop (RED discoveries, one atomicOr per pop): RMAT-26 9.81 -> 8.62 ms,
        // RMAT-24 2.72 -> 2.43 ms; ATOS_VIS_NOCLAIM restores the discoverer's atomicOr (A/B)
        if (kp.vis && !std::getenv("ATOS_VIS_NOCLAIM")) kp.vis_claim = 1;
        // next-batch reservation during the expansion (the leader's pop took ~5
        // dependent round trips with the whole CTA waiting); ATOS_NO_PQ_EARLY (A/B)
        kp.pq_early = kp.vis && !g->cfg.discrete && !std::getenv("ATOS_NO_PQ_EARLY");
    }
    kp.agg_age_ns = g->cfg.agg_max_age_ns;
    kp.watchdog_ns = g->cfg.watchdog_ms * 1000000ll;
    kp.epoch = g->epoch;
    return kp;
}

// L2 persisting window for the random-access state of the worker (BFS words or
// filter / PR residuals); sets the device's persisting carve-out to match.
// Returns false when no window applies.
template <int APP>
static bool l2_window(atos_graph *g, const KParams &kp, cudaAccessPolicyWindow &w) {
    if (!(g->cfg.l2_persist && g->n_local == 1 && g->persist_max > 0 && g->window_max > 0)) return false;
    // keep the random-access state resident in L2 while the CSR column stream
    // passes through
    const LocalRank &me = g->loc[0];
    void *base = APP == kApBfs ? (void *)(me.arena + (kp.vis ? me.L.vis : kp.filter ? me.L.filt : me.L.depth))
                               : (void *)(me.arena + me.L.res);
    size_t bytes = APP == kApBfs ? (kp.vis ? ((size_t)g->n / 32 + 1) * (kp.vis_claim ? 8 : 4) : (size_t)g->n * (kp.filter ? 1 : 4))
                                 : (size_t)me.L.n_r * 8;
    bytes = std::min(bytes, g->window_max);
#ifdef ATOS_CARVE_MAX   // experiment: the whole persisting limit as carve-out
    const size_t carve = g->persist_max;
#else
    const size_t carve = std::min(bytes, g->persist_max);   // carve-out == window, no more
#endif
    if (carve != g->persist_set) {
        if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, carve) != cudaSuccess) {
            cudaGetLastError();
            g->persist_max = 0;                              // not permitted: no window from now on
            return false;
        }
        g->persist_set = carve;
    }
    w.base_ptr = base;
    w.num_bytes = bytes;
    w.hitRatio = (float)std::min(1.0, (double)carve / (double)bytes);
    w.hitProp = cudaAccessPropertyPersisting;
    w.missProp = cudaAccessPropertyStreaming;
    return true;
}

// Build (once per handle and app) the discrete-mode graph:
//   step -> while (cond) { worker_discrete -> step }
// step snapshots tail into ctrl->limit and sets cond = (queue non-empty).
template <int APP>
static atos_status build_discrete_graph(atos_graph *g, const KParams &kp) {
    if (g->dexec[APP]) return ATOS_OK;
    if (!g->d_kp) CU(cudaMalloc(&g->d_kp, sizeof(KParams)));
    cudaGraph_t gr = nullptr;
    CU(cudaGraphCreate(&gr, 0));
    g->dgraph[APP] = gr;
    cudaGraphConditionalHandle h;
    CU(cudaGraphConditionalHandleCreate(&h, gr, 1, cudaGraphCondAssignDefault));
    KParams *dkp = g->d_kp;
    int first = 0, after = 1;
    void *step_args[] = {&dkp, &h, &first};
    void *step_args_after[] = {&dkp, &h, &after};
    cudaKernelNodeParams sk{};
    sk.func = (void *)discrete_step_kernel;
    sk.gridDim = dim3(1);
    sk.blockDim = dim3(32);
    sk.kernelParams = step_args;
    cudaGraphNode_t pre = nullptr, cond = nullptr, wnode = nullptr, post = nullptr;
    CU(cudaGraphAddKernelNode(&pre, gr, nullptr, 0, &sk));
    cudaGraphNodeParams cp{};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = h;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    CU(cudaGraphAddNode(&cond, gr, &pre, 1, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    void *w_args[] = {&dkp};
    cudaKernelNodeParams wk{};
    wk.func = (void *)worker_discrete_kernel<APP>;
    wk.gridDim = dim3(g->grid);
    wk.blockDim = dim3(kThreads);
    wk.sharedMemBytes = (unsigned)worker_smem(APP, kp.hub_chunks);
    wk.kernelParams = w_args;
    CU(cudaGraphAddKernelNode(&wnode, body, nullptr, 0, &wk));
    cudaAccessPolicyWindow win{};
    if (l2_window<APP>(g, kp, win)) {
        cudaKernelNodeAttrValue av{};
        av.accessPolicyWindow = win;
        CU(cudaGraphKernelNodeSetAttribute(wnode, cudaKernelNodeAttributeAccessPolicyWindow, &av));
    }
    sk.kernelParams = step_args_after;
    CU(cudaGraphAddKernelNode(&post, body, &wnode, 1, &sk));
    CU(cudaGraphInstantiate(&g->dexec[APP], gr, 0));
    return ATOS_OK;
}

template <int APP>
static atos_status launch_worker(atos_graph *g, KParams &kp) {
    if (g->cfg.discrete) {
        kp.discrete = 1;
        atos_status s = build_discrete_graph<APP>(g, kp);
        if (s != ATOS_OK) return s;
        CU(cudaMemcpyAsync(g->d_kp, &kp, sizeof(KParams), cudaMemcpyHostToDevice, g->stream));
        CU(cudaGraphLaunch(g->dexec[APP], g->stream));
        return ATOS_OK;
    }
    cudaLaunchConfig_t lc{};
    lc.gridDim = dim3(g->grid);
    lc.blockDim = dim3(kThreads);
    lc.dynamicSmemBytes = worker_smem(APP, kp.hub_chunks);
    lc.stream = g->stream;
    cudaLaunchAttribute at[2];
    int na = 0;
    at[na].id = cudaLaunchAttributeCooperative;          // co-residency of the persistent grid
    at[na].val.cooperative = 1;
    ++na;
    cudaAccessPolicyWindow win{};
    if (l2_window<APP>(g, kp, win)) {
        at[na].id = cudaLaunchAttributeAccessPolicyWindow;
        at[na].val.accessPolicyWindow = win;
        ++na;
    }
    lc.attrs = at;
    lc.numAttrs = na;
    if (g->p > 1) CU(cudaLaunchKernelEx(&lc, worker_kernel<APP, true>, kp));
    else CU(cudaLaunchKernelEx(&lc, worker_kernel<APP, false>, kp));
    return ATOS_OK;
}

static atos_status read_ctrl(atos_graph *g, int lr, Ctrl &c) {
    CU(cudaMemcpy(&c, g->loc[lr].arena + g->loc[lr].L.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost));
    return ATOS_OK;
}

// Wait for the enqueued solve, check device error flags, fill g->last.
static constexpr int kSnap = 12;

// Back to the state graph_load left: control blocks, rings, channel headers and
// free mirrors re-initialised, statistics snapshots cleared.  Single process only.
static atos_status reset_queues(atos_graph *g) {
    for (int lr = 0; lr < g->n_local; ++lr) {
        LocalRank &me = g->loc[lr];
        CU(cudaMemsetAsync(me.arena + me.L.ctrl, 0, sizeof(Ctrl), g->stream));
        CU(cudaMemsetAsync(me.arena + me.L.in_hdr, 0, me.L.in_pay - me.L.in_hdr, g->stream));
        const uint64_t nfree = g->p > 1 ? (uint64_t)g->p * g->S.cp : 0;
        init_arena_kernel<<<1024, 256, 0, g->stream>>>((uint64_t *)(me.arena + me.L.ring), me.L.ring_cap,
                                                       (uint64_t *)(me.arena + me.L.free_m), nfree,
                                                       (uint64_t)(g->S.cp / nsub_for(g->p, g->S.cp)));
        if (g->S.pq)
            init_arena_kernel<<<1024, 256, 0, g->stream>>>((uint64_t *)(me.arena + me.L.ring2), me.L.ring_cap,
                                                           nullptr, 0, 1);
        CU(cudaGetLastError());
        std::memset(me.snap, 0, sizeof(me.snap));
    }
    CU(cudaStreamSynchronize(g->stream));
    return ATOS_OK;
}

static atos_status finish_solve(atos_graph *g) {
    const int app = g->app;
    if (!g->pending) return ATOS_OK;
    g->pending = false;
    CU(cudaStreamSynchronize(g->stream));
    atos_stats st{};
    st.n_ranks = g->n_local;
    st.grid_ctas = g->S.ctas_per_rank;
    float ms = 0;
    CU(cudaEventElapsedTime(&ms, g->ev_w0, g->ev_w1));
    st.ms_worker = ms;
    CU(cudaEventElapsedTime(&ms, g->ev_begin, g->ev_end));
    st.ms_total = ms;
    uint64_t err = 0;
    for (int lr = 0; lr < g->n_local; ++lr) {
        Ctrl c;
        atos_status s = read_ctrl(g, lr, c);
        if (s != ATOS_OK) return s;
        if (c.error.v && !err) err = c.error.v;
        const uint64_t now[kSnap] = {c.st_pops.v, c.st_edges.v, c.st_pushes.v, c.st_msgs.v,
                                     c.st_packets.v, c.st_idle.v, c.st_hub_hits.v, c.st_busy_ns.v,
                                     c.st_batches.v, c.st_waves.v, c.st_far.v, c.pq_state.v};
        uint64_t *sn = g->loc[lr].snap;
        st.pops += now[0] - sn[0];
        st.edges += now[1] - sn[1];
        st.local_pushes += now[2] - sn[2];
        st.msgs_sent += now[3] - sn[3];
        st.packets_sent += now[4] - sn[4];
        st.idle_polls += now[5] - sn[5];
        st.hub_hits += now[6] - sn[6];
        st.busy_ns += now[7] - sn[7];
        st.batches += now[8] - sn[8];
        if (g->cfg.discrete) st.iterations += now[9] - sn[9];
        st.far_pushes += now[10] - sn[10];
        st.pq_buckets += now[11] - sn[11];
        std::memcpy(sn, now, sizeof(now));
    }
    st.bytes_sent = st.msgs_sent * (uint64_t)(app == kApBfs ? AppTraits<kApBfs>::kMsgBytes
                                                            : AppTraits<kApPr>::kMsgBytes);
    g->last = st;
    g->last_valid = true;
    if (err) {
        // The aborted solve left reserved-but-unconsumed ring slots, channel packets
        // and S/R/F/T counters that no later solve could reconcile.  A handle that
        // owns every rank (single rank or virtual ranks) is reset to its
        // just-loaded state; a multi-process handle cannot reset its peers' view of
        // the channels alone, so it is poisoned (later solves: ATOS_ERR_STATE).
        if (g->multiproc) g->poisoned = true;
        else {
            atos_status rs = reset_queues(g);
            if (rs != ATOS_OK) return rs;
        }
    }
    if (err == kErrCapacity) return fail(ATOS_ERR_CAPACITY, "device queue/channel capacity exceeded; result invalid");
    if (err == kErrTimeout) return fail(ATOS_ERR_TIMEOUT, "device watchdog (%lld ms) fired; result invalid",
                                        (long long)g->cfg.watchdog_ms);
    if (err) return fail(ATOS_ERR_STATE, "device error %llu", (unsigned long long)err);
    return ATOS_OK;
}

extern "C" atos_status atos_set_watchdog(atos_graph *g, int64_t ms) {
    if (!g || ms < 0) return fail(ATOS_ERR_INVALID_ARG, "set_watchdog: NULL handle or ms < 0");
    g->cfg.watchdog_ms = ms;
    return ATOS_OK;
}

extern "C" atos_status atos_sync(atos_graph *g) {
    if (!g) return fail(ATOS_ERR_INVALID_ARG, "sync: NULL handle");
    CU(cudaSetDevice(g->cfg.device));
    return finish_solve(g);
}

extern "C" atos_status atos_last_stats(atos_graph *g, atos_stats *stats) {
    if (!g || !stats) return fail(ATOS_ERR_INVALID_ARG, "last_stats: NULL argument");
    atos_status s = atos_sync(g);
    if (s != ATOS_OK && !g->last_valid) return s;
    if (!g->last_valid) return fail(ATOS_ERR_STATE, "no completed solve");
    *stats = g->last;
    return s;
}

static atos_status begin_solve(atos_graph *g, KParams &kp) {
    CU(cudaSetDevice(g->cfg.device));
    if (!g->connected) return fail(ATOS_ERR_PEER, "multi-process handle not connected (atos_graph_connect)");
    if (g->poisoned) return fail(ATOS_ERR_STATE, "multi-process handle poisoned by an earlier device error; free and reload it");
    atos_status s = finish_solve(g);   // a previous async solve must be retired first
    if (s != ATOS_OK) return s;
    g->epoch++;
    kp = make_params(g);
    CU(cudaEventRecord(g->ev_begin, g->stream));
    if (g->p > 1) barrier_kernel<<<1, 32, 0, g->stream>>>(kp, g->epoch * 4 + 0);
    return ATOS_OK;
}

static int grid_for(int64_t n, int threads, int cap) {
    int64_t b = (n + threads - 1) / threads;
    return (int)std::max<int64_t>(1, std::min<int64_t>(b, cap));
}

extern "C" atos_status atos_bfs(atos_graph *g, int64_t src, int32_t *depth_out, int64_t *parent_out,
                                atos_stats *stats) {
    if (!g) return fail(ATOS_ERR_INVALID_ARG, "bfs: NULL handle");
    if (src < 0 || src >= g->n) return fail(ATOS_ERR_INVALID_ARG, "bfs: src %lld not in [0, %lld)", (long long)src, (long long)g->n);
    if (!depth_out) return fail(ATOS_ERR_INVALID_ARG, "bfs: depth_out is NULL");
    KParams kp;
    atos_status s = begin_solve(g, kp);
    if (s != ATOS_OK) return s;
    const bool dev_depth = is_device_ptr(depth_out);
    const bool dev_parent = parent_out && is_device_ptr(parent_out);
    const int gblocks = g->sms * 4;
    init_bfs_kernel<<<gblocks, 512, 0, g->stream>>>(kp);
    seed_bfs_kernel<<<1, 1, 0, g->stream>>>(kp, src);
    CU(cudaGetLastError());
    CU(cudaEventRecord(g->ev_w0, g->stream));
    s = launch_worker<kApBfs>(g, kp);
    if (s != ATOS_OK) return s;
    CU(cudaEventRecord(g->ev_w1, g->stream));
    fixup_kernel<<<1, 512, 0, g->stream>>>(kp);
    int32_t *dfull = dev_depth ? depth_out : g->d_depth_full;
    gather_bfs_kernel<<<grid_for(g->n, 512, gblocks), 512, 0, g->stream>>>(kp, dfull);
    if (parent_out) {
        LocalRank &me = g->loc[0];
        int64_t *acc = (int64_t *)(me.arena + me.L.parent);
        parent_init_kernel<<<grid_for(g->n, 512, gblocks), 512, 0, g->stream>>>(acc, g->n);
        parent_scan_kernel<<<gblocks, 512, 0, g->stream>>>(kp, dfull, acc);
        int n_acc = 1;
        int64_t *accs[kMaxRanks];
        accs[0] = acc;
        if (g->multiproc) {
            barrier_kernel<<<1, 32, 0, g->stream>>>(kp, g->epoch * 4 + 1);
            n_acc = g->p;
            for (int r = 0; r < g->p; ++r)
                accs[r] = (int64_t *)(g->peer_base[r] + make_layout(g->S, g->part.data(), r).parent);
        }
        CU(cudaMemcpyAsync(g->d_accs, accs, sizeof(int64_t *) * n_acc, cudaMemcpyHostToDevice, g->stream));
        int64_t *pout = parent_out;
        int64_t *ptmp = nullptr;
        if (!dev_parent) {
            CU(dmalloc(g, &ptmp, (size_t)g->n * 8));
            pout = ptmp;
        }
        parent_final_kernel<<<grid_for(g->n, 512, gblocks), 512, 0, g->stream>>>(dfull, g->d_accs, n_acc, g->n,
                                                                                src, pout);
        if (!dev_parent) {
            CU(cudaMemcpyAsync(parent_out, ptmp, (size_t)g->n * 8, cudaMemcpyDeviceToHost, g->stream));
            dfree(g, ptmp);
        }
    }
    if (!dev_depth) CU(cudaMemcpyAsync(depth_out, dfull, (size_t)g->n * 4, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaGetLastError());
    CU(cudaEventRecord(g->ev_end, g->stream));
    g->pending = true;
    g->app = kApBfs;
    const bool async = dev_depth && (!parent_out || dev_parent) && !stats;
    if (async) return ATOS_OK;
    s = finish_solve(g);
    if (stats) *stats = g->last;
    return s;
}

extern "C" atos_status atos_pagerank(atos_graph *g, double alpha, double eps, double *rank_out,
                                     double *residual_out, atos_stats *stats) {
    if (!g) return fail(ATOS_ERR_INVALID_ARG, "pagerank: NULL handle");
    if (!(alpha >= 0.0 && alpha < 1.0)) return fail(ATOS_ERR_INVALID_ARG, "pagerank: alpha must be in [0,1)");
    if (!(eps > 0.0)) return fail(ATOS_ERR_INVALID_ARG, "pagerank: eps must be > 0");
    KParams kp;
    atos_status s = begin_solve(g, kp);
    if (s != ATOS_OK) return s;
    kp.pq = 0;                     // the priority queue orders BFS by depth only
    kp.vis = 0;
    kp.alpha = alpha;
    kp.eps = eps;
    kp.eps_g = eps / (double)g->p;
    const int gblocks = g->sms * 4;
    init_pr_kernel<<<gblocks, 512, 0, g->stream>>>(kp);
    bump_tail_kernel<<<1, 1, 0, g->stream>>>(kp);
    CU(cudaGetLastError());
    CU(cudaEventRecord(g->ev_w0, g->stream));
    s = launch_worker<kApPr>(g, kp);
    if (s != ATOS_OK) return s;
    CU(cudaEventRecord(g->ev_w1, g->stream));
    fixup_kernel<<<1, 512, 0, g->stream>>>(kp);
    const bool dev_r = !rank_out || is_device_ptr(rank_out);
    const bool dev_s = !residual_out || is_device_ptr(residual_out);
    double *tr = nullptr, *ts = nullptr;
    if (!dev_r || !dev_s) {
        // stage through the (idle) parent accumulator region: 8n bytes each is not
        // guaranteed, so use the full-depth buffer region only for one output.
        CU(dmalloc(g, &tr, (size_t)g->n * 8));
        CU(dmalloc(g, &ts, (size_t)g->n * 8));
    }
    gather_pr_kernel<<<grid_for(g->n, 512, gblocks), 512, 0, g->stream>>>(
        kp, rank_out ? (dev_r ? rank_out : tr) : nullptr, residual_out ? (dev_s ? residual_out : ts) : nullptr);
    if (rank_out && !dev_r) CU(cudaMemcpyAsync(rank_out, tr, (size_t)g->n * 8, cudaMemcpyDeviceToHost, g->stream));
    if (residual_out && !dev_s) CU(cudaMemcpyAsync(residual_out, ts, (size_t)g->n * 8, cudaMemcpyDeviceToHost, g->stream));
    dfree(g, tr);
    dfree(g, ts);
    CU(cudaGetLastError());
    CU(cudaEventRecord(g->ev_end, g->stream));
    g->pending = true;
    g->app = kApPr;
    const bool async = dev_r && dev_s && !stats;
    if (async) return ATOS_OK;
    s = finish_solve(g);
    if (stats) *stats = g->last;
    return s;
}

// ---------------------------------------------------------------------------
// queue microbenchmark (Fig. 1) on the worker's ring code
// ---------------------------------------------------------------------------
extern "C" atos_status atos_queue_bench(const atos_qbench_config *c, uint32_t *popped_out, double *ms_out) {
    if (!c || !ms_out) return fail(ATOS_ERR_INVALID_ARG, "queue_bench: NULL argument");
    auto pow2 = [](uint64_t x) { return x > 0 && (x & (x - 1)) == 0; };
    if (!(c->worker_size == 1 || c->worker_size == 32 || c->worker_size == kThreads) || c->fetch_size < 1 ||
        c->fetch_size > c->worker_size || c->rounds < 1 || c->op < 0 || c->op > 2 || c->threads < kThreads ||
        c->threads % kThreads != 0 || !pow2(c->ring_cap) || (c->reserve_cas != 0 && c->reserve_cas != 1))
        return fail(ATOS_ERR_INVALID_ARG, "queue_bench: bad configuration");
    const uint64_t total = (uint64_t)c->threads * (uint64_t)c->rounds;
    if (c->op != kQPushPop && c->ring_cap < total)
        return fail(ATOS_ERR_INVALID_ARG, "queue_bench: push / pop alone need ring_cap >= threads * rounds");
    if (c->op == kQPushPop && c->ring_cap < (uint64_t)c->threads)
        return fail(ATOS_ERR_INVALID_ARG, "queue_bench: push-then-pop needs ring_cap >= threads");
    CU(cudaSetDevice(c->device));
    int sms = 0, per_sm = 0;
    CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c->device));
    CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, qbench_kernel, kThreads, 0));
    if (c->threads > (int64_t)sms * per_sm * kThreads)
        return fail(ATOS_ERR_INVALID_ARG, "queue_bench: threads exceed the co-resident limit (%lld)",
                    (long long)sms * per_sm * kThreads);
    cudaStream_t st;
    CU(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    uint64_t *ring = nullptr;
    Ctrl *ctrl = nullptr;
    uint32_t *pop = nullptr;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    atos_status rs = ATOS_OK;
    auto done = [&](atos_status r) {
        cudaStreamSynchronize(st);
        cudaFree(ring); cudaFree(ctrl); cudaFree(pop);
        if (e0) cudaEventDestroy(e0);
        if (e1) cudaEventDestroy(e1);
        cudaStreamDestroy(st);
        return r;
    };
    auto ck = [&](cudaError_t e, const char *what) {
        if (e != cudaSuccess && rs == ATOS_OK)
            rs = fail(e == cudaErrorMemoryAllocation ? ATOS_ERR_OOM : ATOS_ERR_CUDA, "queue_bench: %s: %s", what,
                      cudaGetErrorString(e));
        return e == cudaSuccess;
    };
    if (!ck(cudaMalloc(&ring, c->ring_cap * 8), "ring") || !ck(cudaMalloc(&ctrl, sizeof(Ctrl)), "ctrl") ||
        (popped_out && !is_device_ptr(popped_out) && !ck(cudaMalloc(&pop, total * 4), "popped")) ||
        !ck(cudaEventCreate(&e0), "event") || !ck(cudaEventCreate(&e1), "event"))
        return done(rs);
    uint32_t *pdev = popped_out ? (is_device_ptr(popped_out) ? popped_out : pop) : nullptr;
    const uint64_t prefill = c->op == kQPop ? total : 0;
    ck(cudaMemsetAsync(ctrl, 0, sizeof(Ctrl), st), "memset");
    qbench_init_kernel<<<1024, 256, 0, st>>>(ring, c->ring_cap, c->index_base, prefill);
    Ctrl h{};
    h.head.v = c->index_base;
    h.tail.v = c->index_base + prefill;
    ck(cudaMemcpyAsync(&ctrl->head.v, &h.head.v, 8, cudaMemcpyHostToDevice, st), "head");
    ck(cudaMemcpyAsync(&ctrl->tail.v, &h.tail.v, 8, cudaMemcpyHostToDevice, st), "tail");
    QBenchArgs a{ring, c->ring_cap, ctrl, pdev, c->worker_size, c->fetch_size, c->rounds, c->op, c->reserve_cas,
                 c->index_base};
    ck(cudaEventRecord(e0, st), "record");
    qbench_kernel<<<(unsigned)(c->threads / kThreads), kThreads, 0, st>>>(a);
    ck(cudaGetLastError(), "launch");
    ck(cudaEventRecord(e1, st), "record");
    if (pdev && pdev != popped_out) ck(cudaMemcpyAsync(popped_out, pdev, total * 4, cudaMemcpyDeviceToHost, st), "copy");
    uint64_t err = 0;
    ck(cudaMemcpyAsync(&err, &ctrl->error.v, 8, cudaMemcpyDeviceToHost, st), "error");
    ck(cudaStreamSynchronize(st), "sync");
    float ms = 0;
    ck(cudaEventElapsedTime(&ms, e0, e1), "elapsed");
    *ms_out = ms;
    if (rs == ATOS_OK && err == kErrCapacity) rs = fail(ATOS_ERR_CAPACITY, "queue_bench: ring capacity exceeded");
    if (rs == ATOS_OK && err) rs = fail(ATOS_ERR_TIMEOUT, "queue_bench: a pop never saw its item");
    return done(rs);
}
