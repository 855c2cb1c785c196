/*
 * atos.h -- C ABI of the B200-native Atos hot path (GPU-initiated asynchronous
 * graph traversal).  Implemented by paper_conf_sc_chenbpbyo22_b200/csrc/ and
 * built as paper_conf_sc_chenbpbyo22_b200/libatos.so (sm_100a SASS).
 *
 * Citations are to /root/reference/PAPER.md (P:<lines>) and the repo's
 * SURVEY.md §8 / DESIGN.md readings.
 *
 * General conventions
 *  - Every function returns atos_status; no C++ exception crosses the ABI.
 *    On failure a human-readable message is available from atos_last_error()
 *    (thread-local, valid until the next ABI call on the same thread).
 *  - Vertex ids are int32 in [0, n) (n <= 2^31-1); CSR row offsets are int64
 *    (RMAT-26 symmetric has ~2.1e9 entries; reading R9).
 *  - Pointer arguments may be HOST or DEVICE memory unless stated otherwise;
 *    the library inspects them with cudaPointerGetAttributes and copies with
 *    cudaMemcpyDefault.  Input arrays are caller-owned and only read during
 *    the call.  Output arrays are caller-owned and caller-allocated.
 *  - The graph handle owns all device memory it allocates (CSR copy, state,
 *    queues, channels, control blocks) and frees it in atos_graph_free.
 *  - A handle is not thread-safe: one host thread drives one handle.
 */
#ifndef ATOS_H
#define ATOS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ATOS_ABI_VERSION 5
#define ATOS_MAX_RANKS 8          /* one NVSwitch box: 8 GPUs */
#define ATOS_IPC_HANDLE_BYTES 64  /* == sizeof(cudaIpcMemHandle_t) */

typedef enum {
    ATOS_OK = 0,
    ATOS_ERR_INVALID_ARG = 1,  /* bad argument; nothing was modified            */
    ATOS_ERR_CUDA = 2,         /* a CUDA runtime call failed                    */
    ATOS_ERR_OOM = 3,          /* device allocation failed                      */
    ATOS_ERR_CAPACITY = 4,     /* a queue/channel would have overflowed; the
                                  solve was aborted, outputs are invalid        */
    ATOS_ERR_TIMEOUT = 5,      /* device watchdog fired; outputs are invalid    */
    ATOS_ERR_PEER = 6,         /* peer mapping (IPC) failed or is missing       */
    ATOS_ERR_STATE = 7         /* call not valid in the handle's current state  */
} atos_status;

typedef struct atos_graph atos_graph;   /* opaque */

/* Launch / runtime configuration.  Obtain defaults with atos_config_init(). */
typedef struct {
    int32_t worker_threads;   /* CTA worker size; 512 as in all of the paper's
                                 runs. Must be 512 in ABI v1.  */
    int32_t ctas_per_sm;      /* persistent CTAs per SM; 0 = max co-resident */
    int32_t fetch_size;       /* max vertices popped per worker batch (the
                                 paper's FETCH_SIZE); <= worker_threads */
    int32_t keep_items;       /* max discovered vertices a worker keeps as its
                                 own next batch instead of enqueueing them
                                 (work-keeping; 0 = always enqueue; <= 512);
                                 -1 = auto: 128 with keep_mode 1 on graphs that
                                 are not skewed (high-diameter, road-like), 0 on
                                 skewed ones        */
    int32_t l2_persist;       /* 1: give the random-access state (BFS words /
                                 PR residuals) an L2 persisting access-policy
                                 window during the worker kernel; sets the
                                 device's persisting-L2 limit to its maximum  */
    int32_t prefetch;         /* 1: TMA bulk-prefetch (cp.async.bulk.prefetch
                                 .L2) each popped adjacency list into L2      */
    int32_t relax_red;        /* BFS: 1 = fire-and-forget relaxation (red.min,
                                 enqueue on the probe's verdict; duplicates are
                                 skipped at pop); 0 = atomicMin with return   */
    int32_t pipeline;         /* BFS: 1 = software-pipelined expansion (each
                                 warp keeps two 128-edge chunks in flight),
                                 2 = only for low-degree batches, 0 = never,
                                 3 = three-stage pipeline (probes of the next
                                 chunk and columns of the one after in flight
                                 while a chunk is relaxed; no hub cache)      */
    int32_t probe_filter;     /* BFS: 1 = probe a 1-byte-per-vertex depth upper
                                 bound instead of the 4-byte words, 0 = never,
                                 2 = auto: on skewed graphs (hub probes share
                                 4x fewer L1/L2 lines; measured 3 % faster on
                                 RMAT-24) or when the words exceed the L2
                                 persisting carve-out                         */
    double ring_cap_factor;   /* local ring capacity = pow2 >= factor*n_rank   */
    int32_t agg_enabled;      /* communication aggregation: 1 =
                                 each warp stages its remote messages per
                                 destination and sends a packet when
                                 agg_batch_msgs are staged, or at batch end /
                                 when idle once the oldest staged message is
                                 agg_max_age_ns old; 0 = every warp sends what
                                 each 32-edge step produced at once (Listing
                                 5's per-warp push; packets of <= 32
                                 messages)                                    */
    int32_t agg_batch_msgs;   /* packet size in messages (the BATCH_SIZE);
                                 default 1024 (channel sweep)      */
    int64_t agg_max_age_ns;   /* flush age (the WAIT_TIME) in ns of
                                 %globaltimer, checked at batch end and when
                                 idle                                          */
    int32_t channel_packets;  /* packets per (src->dst) channel ring, pow2;
                                 default 4096                                  */
    int64_t watchdog_ms;      /* device watchdog per solve; 0 = none           */
    int32_t rank;             /* SPMD: this process's rank                     */
    int32_t n_ranks;          /* SPMD: number of processes (1 = single GPU)    */
    int32_t virtual_ranks;    /* >1 (with n_ranks==1): emulate this many ranks
                                 inside one grid on one device; same protocol,
                                 peers are same-device pointers    */
    int32_t device;           /* CUDA device ordinal                           */
    void *stream;             /* cudaStream_t to launch on; NULL = the library
                                 creates its own non-blocking stream           */
    int32_t relabel;          /* internal vertex order (outputs and src always
                                 use the caller's ids): 0 = as given, 1 = by
                                 out-degree, descending, inside every rank block
                                 (ties by id; the partition is unchanged),
                                 2 = auto: 1 iff max degree >= 32 x mean degree
                                 (skewed graphs)      */
    int32_t hub_cache;        /* BFS: shared-memory depth-bound cache entries per
                                 worker CTA for the first ids of every rank
                                 block; multiple of 32
                                 x n_ranks, <= 65536; 0 = off; -1 = auto
                                 (currently off: the L1 already serves hub
                                 probes; kept as a measured option)           */
    int32_t split_edges;      /* BFS: a popped row longer than 2 x split_edges
                                 is cut into split_edges-edge pieces that any
                                 worker can pop (the popping worker keeps the
                                 first); only for the first 65536 ids of a rank
                                 block (the hubs after relabeling).  Power of
                                 two in [256, 1<<20]; 0 = off; -1 = auto       */
    int32_t keep_mode;        /* when a worker keeps (keep_items > 0): 0 = only
                                 while the rank's outstanding work is <=
                                 keep_items (low-parallelism phases), 1 =
                                 whenever its batch discovered <= keep_items
                                 (latency chains; may add redundant work).
                                 Ignored when keep_items == -1 (auto)         */
    int32_t discrete;         /* 0 = one persistent worker kernel per solve
                                 (the paper's default); 1 = discrete
                                 kernels: each launch
                                 processes the queue snapshot [head, tail) and
                                 exits; a CUDA-graph while-node relaunches it
                                 until the queue is empty, with no host round
                                 trip.  Single rank only (n_ranks == 1 and
                                 virtual_ranks == 1)                           */
    int32_t pr_combine;       /* PageRank, n_ranks > 1 (not in the
                                 paper): 1 = sender-side residual combining --
                                 deltas for a remote vertex accumulate in this
                                 rank's ghost residual, which is sent as ONE
                                 message when it crosses eps / n_ranks; the
                                 returned residual then includes the unsent
                                 ghost mass (< eps in total per vertex beyond
                                 the owner's own < eps).  0 = send every delta
                                 (the paper's push, with aggregation)          */
    int32_t pool_retain;      /* 0 = atos_graph_free trims the library's private
                                 stream-ordered memory pool back to zero (freed
                                 memory returns to the device); 1 = keep it
                                 reserved for the next graph_load in this
                                 process (load/solve/free loops)               */
    int32_t pq_delta;         /* BFS priority queue (Listing 4's
                                 DistributedPriorityQueues threshold_delta,
                                 P:629-639): 0 = FIFO queue;
                                 -1 = auto (the default): 1 on a skewed
                                 single-rank graph of >= 2^20 vertices, else
                                 FIFO; > 0 = every rank keeps two rings,
                                 the current bucket (candidate depth below the
                                 threshold) and the rest; workers pop only the
                                 current one, and when it is drained the rings
                                 swap and the threshold grows by pq_delta.
                                 1 = level-synchronous order, large = FIFO.
                                 Needs rank blocks of < 2^30 vertices; ignored
                                 by PageRank                                  */
    int32_t pq_threshold;     /* initial threshold (the paper's `threshold`):
                                 depths below it form the first bucket; 0 =
                                 pq_delta                                     */
} atos_config;

/* Per-solve statistics (device counters, summed over the ranks this handle
 * can see; multi-process callers reduce across processes themselves). */
typedef struct {
    double ms_worker;         /* device time of the persistent worker kernel
                                 (CUDA events on the launch stream)           */
    double ms_total;          /* device time barrier+init+worker+gather        */
    uint64_t pops;            /* queue entries processed                       */
    uint64_t edges;           /* edges relaxed (CSR entries scanned)           */
    uint64_t local_pushes;    /* local ring enqueues                           */
    uint64_t msgs_sent;       /* remote messages (one-sided peer stores)       */
    uint64_t packets_sent;    /* channel packets published                     */
    uint64_t bytes_sent;      /* payload bytes stored into peer channels       */
    uint64_t idle_polls;      /* worker iterations that found no work          */
    uint64_t hub_hits;        /* BFS edges retired by the shared-memory hub
                                 cache without an L2 probe                    */
    uint64_t busy_ns;         /* sum over workers of time spent on work (ns)   */
    uint64_t batches;         /* work units (pop batches + packets + chunks)   */
    uint64_t iterations;      /* discrete mode: worker launches in the solve   */
    uint64_t far_pushes;      /* priority queue: items enqueued into the next
                                 bucket's ring                                 */
    uint64_t pq_buckets;      /* priority queue: bucket advances in the solve  */
    int32_t n_ranks;          /* ranks covered by these counters               */
    int32_t grid_ctas;        /* persistent CTAs per rank                      */
} atos_stats;

/* Fill *cfg with defaults.  Host only; never touches the GPU. */
atos_status atos_config_init(atos_config *cfg);

/* 1-D contiguous vertex blocks: part[r] = floor(r*n/p), r = 0..p (SURVEY §8a-1,
 * reading R13).  part must hold p+1 entries.  Host only. */
atos_status atos_partition_balanced(int64_t n, int32_t p, int64_t *part);

/* Validate a CSR (row_ptr monotone from 0 to nnz, every col in [0,n)).
 * row_ptr/col must be HOST pointers.  Host only. */
atos_status atos_validate_csr(const int64_t *row_ptr, const int32_t *col, int64_t n, int64_t nnz);

/* Bytes of the rank-exported device arena for a given shape (host only).
 * Used by the Python layer to size checks; identical on every rank. */
atos_status atos_arena_bytes(int64_t n, const int64_t *part, int32_t n_ranks, int32_t rank,
                             const atos_config *cfg, uint64_t *bytes_out);

/* Load the graph for this process.  row_ptr [n+1] / col [nnz] describe the
 * WHOLE directed graph (out-edges, global ids; duplicates and self-loops are
 * kept as given).  part = n_ranks+1 vertex offsets (NULL = balanced); with
 * cfg->virtual_ranks = R > 1 the partition has R blocks.  The rank(s) served
 * by this handle copy only their own rows (Listing 5's CSR + findPE,
 * P:642-692).  Allocates all device state.  cfg NULL = defaults. */
atos_status atos_graph_load(const int64_t *row_ptr, const int32_t *col, int64_t n, int64_t nnz,
                            const int64_t *part, const atos_config *cfg, atos_graph **out);

/* Multi-process (n_ranks > 1) peer mapping, the analogue of nvshmem_malloc's
 * symmetric heap (Listing 5):  every rank exports one IPC handle for
 * its arena (ATOS_IPC_HANDLE_BYTES bytes into handle_out), the caller
 * all-gathers them (torch.distributed), and passes the n_ranks handles in
 * rank order to atos_graph_connect, which maps every peer over NVLink. */
atos_status atos_graph_export(atos_graph *g, void *handle_out);
atos_status atos_graph_connect(atos_graph *g, const void *handles);

/* Asynchronous push BFS from global vertex src (Listing 5,
 * P:641-699): depth_out[n] receives the hop distance (-1 = unreachable) of
 * every vertex (all ranks receive the gathered result).  parent_out[n]
 * (optional, may be NULL) receives the min-id parent (parent[src] = src,
 * -1 unreachable).  stats optional.  Blocks until the result is in the
 * output buffers unless all outputs are device pointers and stats == NULL,
 * in which case it only enqueues on the handle's stream (use atos_sync). */
atos_status atos_bfs(atos_graph *g, int64_t src, int32_t *depth_out, int64_t *parent_out,
                     atos_stats *stats);

/* Asynchronous push-residual PageRank: rank = 0,
 * residual = 1-alpha, every vertex enqueued; pop v -> rank += r, residual
 * alpha*r/outdeg pushed to each out-neighbour, re-enqueue on the crossing
 * old < eps <= old+delta (reading R5).  Outputs the raw (unnormalised)
 * rank_out[n] and residual_out[n] (either may be NULL).  0 <= alpha < 1,
 * eps > 0.  Same blocking rule as atos_bfs. */
atos_status atos_pagerank(atos_graph *g, double alpha, double eps, double *rank_out,
                          double *residual_out, atos_stats *stats);

/* Set the device watchdog of later solves (ms; 0 = none).  Host only. */
atos_status atos_set_watchdog(atos_graph *g, int64_t ms);

/* Wait for the last enqueued solve and return its device status.
 * After a device error (ATOS_ERR_CAPACITY / ATOS_ERR_TIMEOUT) the outputs of
 * that solve are invalid; a single-process handle (n_ranks == 1, any
 * virtual_ranks) is reset to its just-loaded state and can solve again, a
 * multi-process handle is poisoned: later solves return ATOS_ERR_STATE. */
atos_status atos_sync(atos_graph *g);

/* Counters of the last completed solve (synchronises). */
atos_status atos_last_stats(atos_graph *g, atos_stats *stats);

/* Release everything the handle owns.  NULL-safe. */
atos_status atos_graph_free(atos_graph *g);

/* Queue microbenchmark (Fig. 1, P:809-823 / P:842-911)
 * on the worker's own ring code (tagged 8-byte slots, u64 monotone indices,
 * reserve-then-wait pop).  `threads` threads in workers of worker_size threads
 * (1 thread, 32 warp, 512 CTA) each do `rounds` pushes (op 0), pops
 * of a prefilled ring (op 1) or push-then-pop pairs (op 2); a worker's leader
 * reserves fetch_size indices per atomicAdd (the worker's FETCH_SIZE),
 * or per CAS loop with reserve_cas = 1 (the paper's CAS-queue baseline).
 * Item of the push (thread t, round r) is t*rounds + r; prefilled item i is i.
 * popped_out (host or device, threads*rounds entries, or NULL) receives the
 * item each (thread, round) popped, for conservation checks.  index_base is
 * the queue's first index (tests start just below 2^32 to cross the 32-bit
 * slot tags).  ring_cap: pow2; >= threads*rounds for ops 0/1, >= threads for
 * op 2.  threads: multiple of 512, at most the co-resident thread count
 * (waiting pops need their producers resident).  *ms_out = device time of the
 * benchmark kernel (CUDA events).  Errors: ATOS_ERR_INVALID_ARG,
 * ATOS_ERR_CAPACITY (a push never found its slot free), ATOS_ERR_TIMEOUT (a
 * pop never saw its item), ATOS_ERR_CUDA / ATOS_ERR_OOM. */
typedef struct {
    int32_t worker_size;      /* 1, 32 or 512 threads per worker               */
    int32_t fetch_size;       /* indices per leader reservation, 1..worker_size */
    int32_t op;               /* 0 push, 1 pop, 2 push-then-pop                */
    int32_t rounds;           /* operations per thread (the paper: 10)         */
    int64_t threads;          /* concurrent threads (multiple of 512)          */
    uint64_t ring_cap;        /* ring slots (power of two)                     */
    uint64_t index_base;      /* first queue index                             */
    int32_t reserve_cas;      /* 1 = CAS-loop reservation                      */
    int32_t device;           /* CUDA device ordinal                           */
} atos_qbench_config;
atos_status atos_queue_bench(const atos_qbench_config *cfg, uint32_t *popped_out, double *ms_out);

/* Thread-local message describing the last failure on this thread. */
const char *atos_last_error(void);

/* ABI version (ATOS_ABI_VERSION). */
int32_t atos_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ATOS_H */
