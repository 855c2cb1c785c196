// atos_aux.cuh -- per-solve helper kernels around the persistent worker:
// cross-rank barrier, state init + seeding, ring fixup, gather of
// owned results over NVLink and the min-id parent post-pass.
#pragma once
#include "atos_rt.cuh"

namespace atos {

// Cross-rank barrier: rank r writes `value` into every rank's bar[r] and waits
// until its own bar[*] all equal `value`.  One CTA.
__global__ void barrier_kernel(KParams kp, uint64_t value) {
    if (threadIdx.x != 0) return;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        for (int d = 0; d < R.n_ranks; ++d) st_release_peer(kp.sys, &R.peer_ctrl[d]->bar[R.rank].v, value);
    }
    const uint64_t t0 = globaltimer();
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        for (int d = 0; d < R.n_ranks; ++d) {
            while (ld_acquire_peer(kp.sys, &R.ctrl->bar[d].v) < value) {
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
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
            R.depth[i] = kInf;
            R.filt[i] = 255;
        }
        for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < kp.hub_chunks; i += (int64_t)gridDim.x * blockDim.x)
            R.hcb[i] = 255;     // hub bounds: unknown
        if (kp.vis)             // visited bitmap: nothing visited
            for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < 2 * (n / 32 + 1); i += (int64_t)gridDim.x * blockDim.x)
                R.vis[i] = 0u;  // (and the claim bitmap behind it)
        if (blockIdx.x == 0 && threadIdx.x == 0) R.ctrl->error.v = 0;
    }
}

// Seed: owner of src sets depth[src] = 0 and enqueues it.  One thread.
__global__ void seed_bfs_kernel(KParams kp, int64_t src) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    if (kp.ranks[0].perm) src = kp.ranks[0].perm[src];   // relabeling keeps every vertex in its rank block
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        R.ctrl->ring_base.v = R.ctrl->tail.v;
        R.ctrl->pq_base.v = R.ctrl->pq_tail.v;
        R.ctrl->pq_k0.v = R.ctrl->pq_state.v;      // priority queue: first bucket of this solve
        if (kp.timeline_ns) {
            R.ctrl->tl_t0 = globaltimer();
            for (int k = 0; k < kTimeline; ++k) R.ctrl->tl_edges[k] = R.ctrl->tl_batches[k] = R.ctrl->tl_pops[k] = 0;
        }
        if (src < R.v_begin || src >= R.v_end) continue;
        R.depth[src] = dw_make(0);
        filt_put_fresh(R.filt, src, 0u);
        if (kp.vis) R.vis[src >> 5] |= 1u << (src & 31);
        const int q = kp.pq ? (int)(R.ctrl->pq_state.v & 1) : 0;   // the current bucket's ring
        const uint64_t idx = *q_tail(R, q);
        uint64_t *p = &q_slots(R, q)[idx & (R.ring_cap - 1)];
        if (!slot_free_for(*p, idx)) { R.ctrl->error.v = kErrCapacity; return; }
        __threadfence();
        *p = pack(lo32(idx + 1), (uint32_t)(src - R.v_begin));
        __threadfence();
        *q_tail(R, q) = idx + 1;
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
        if (R.pr_ghost) {   // combining: no unsent residual for any remote vertex
            for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < R.n; i += (int64_t)gridDim.x * blockDim.x)
                R.pr_ghost[i] = 0.0;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) R.ctrl->error.v = 0;
    }
}

__global__ void bump_tail_kernel(KParams kp) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        R.ctrl->ring_base.v = R.ctrl->tail.v;   // the init lap [base, base+n_r) is part of this solve
        R.ctrl->tail.v += (uint64_t)(R.v_end - R.v_begin);
    }
}

// After a solve: reservations that overshot the tail are retired so that the
// ring stays consistent for the next solve (slots marked consumed; T and F
// advanced by the same amount).  One CTA.
__global__ void fixup_kernel(KParams kp) {
    if (kp.timeline_ns && threadIdx.x == 0) {   // experiment: print the work timeline of rank 0
        const Ctrl *c = kp.ranks[0].ctrl;
        printf("TIMELINE bucket_us %lld:", (long long)(kp.timeline_ns / 1000));
        for (int k = 0; k < kTimeline; ++k)
            if (c->tl_batches[k]) printf(" [%d %llu %llu %llu]", k, (unsigned long long)c->tl_edges[k],
                                         (unsigned long long)c->tl_batches[k], (unsigned long long)c->tl_pops[k]);
        printf("\n");
    }
    for (int lr = 0; lr < kp.n_local; ++lr) {
        const RankDev &R = kp.ranks[lr];
        for (int q = 0; q < (R.ring2 ? 2 : 1); ++q) {      // both rings with the priority queue
            const uint64_t h = *q_head(R, q), t = *q_tail(R, q);
            if (h > t) {
                for (uint64_t idx = t + threadIdx.x; idx < h; idx += blockDim.x)
                    q_slots(R, q)[idx & (R.ring_cap - 1)] = pack(lo32(idx + R.ring_cap), 0u);
            }
            __syncthreads();
            if (threadIdx.x == 0 && h > t) {
                *q_tail(R, q) = h;
                *q_fin(R, q) += h - t;
            }
            __syncthreads();
        }
    }
}

// Gather owned results of every rank into full-size outputs (peer loads over NVLink),
// indexed by the caller's (original) vertex ids.
__global__ void gather_bfs_kernel(KParams kp, int32_t *out) {
    const RankDev &R = kp.ranks[0];
    const int64_t n = R.n;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int o = 0;
        for (int k = 1; k < R.n_ranks; ++k) o += R.part[k] <= v ? 1 : 0;
        const int64_t nv = R.perm ? R.perm[v] : v;
        uint32_t d = dw_depth(__ldcg(R.peer_depth[o] + nv));
        if (kp.vis) {            // visited-bitmap mode: depth bytes (the word only at depth >= 255)
            const uint32_t b = __ldcg(R.filt + nv);
            if (b < 255u) d = b;
        }
        out[v] = d == kDepthInf ? -1 : (int32_t)d;
    }
}

__global__ void gather_pr_kernel(KParams kp, double *rank_out, double *res_out) {
    const RankDev &R = kp.ranks[0];
    const int64_t n = R.n;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        int o = 0;
        for (int k = 1; k < R.n_ranks; ++k) o += R.part[k] <= v ? 1 : 0;
        const int64_t nv = R.perm ? R.perm[v] : v;
        const int64_t i = pr_slot(nv - R.part[o], pr_q_of(R.part[o + 1] - R.part[o]));
        if (rank_out) rank_out[v] = __ldcg(R.peer_rank[o] + i);
        if (res_out) {
            double r = __ldcg(R.peer_res[o] + i);
            if (R.pr_ghost) {   // combining: unsent ghost mass of every other rank belongs to v's residual
                const int64_t gi = pr_slot(nv, pr_q_of(n));
                for (int k = 0; k < R.n_ranks; ++k)
                    if (k != o) r += __ldcg(R.peer_ghost[k] + gi);
            }
            res_out[v] = r;
        }
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
            const int64_t u = R.inv ? R.inv[R.v_begin + i] : R.v_begin + i;   // original ids throughout
            const int32_t du = depth_full[u];
            if (du < 0) continue;
            for (int64_t e = R.row_ptr[i] + lane; e < R.row_ptr[i + 1]; e += 32) {
                const int32_t v = R.inv ? R.inv[R.col[e]] : R.col[e];
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
