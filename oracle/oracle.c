/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for the Atos hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, constant or helper with the CUDA path
 * (paper_conf_sc_chenbpbyo22_b200/csrc); neither includes the other.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md):
 *
 *  oracle_bfs  -- the plain definition the asynchronous push BFS of
 *      PAPER.md:1158-1166 (Sec. IV "BFS") and Listing 5
 *      converges to: depth(v) = minimum number of CSR out-edges on a path
 *      src -> v, -1 if unreachable.  Written as the textbook serial FIFO
 *      queue BFS.  Parity: bit-exact.
 *
 *  oracle_bfs_parents_minid -- canonical BFS parent: the smallest vertex id
 *      u with an edge u->v and depth(u) = depth(v)-1; parent(src) = src,
 *      -1 if unreached (SURVEY.md §8a-9 reading; parents are not unique in
 *      the paper, so GPU parents are also checked by rule in the tests).
 *
 *  oracle_pagerank -- the plain PageRank definition that the push-residual
 *      PageRank of PAPER.md:1168-1182 (Sec. IV "PageRank") approximates:
 *          p = (1-a)/n 1 + a (P^T p + (sum_{outdeg(v)=0} p_v)/n 1),  sum p = 1,
 *      P[v,u] = mult(v->u)/outdeg(v) (readings R2-R4), solved by
 *      synchronous pull (Jacobi) iteration over the transpose (CSC) until
 *      ||p_{k+1} - p_k||_1 <= tol.  Per-vertex sums run in a fixed order and
 *      the L1 norm / dangling mass are summed serially, so the result is
 *      bit-identical for every thread count.
 *
 * Pins (tests/test_oracle.py): exhaustive brute force on every 4-vertex
 * digraph, closed forms (path, star, cycle, K_n, disconnected), scipy /
 * networkx / dense linear solve agreement, invariants on RMAT instances.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_OK 0
#define ORACLE_EINVAL 1
#define ORACLE_ENOMEM 3
#define ORACLE_ENOTCONV 4   /* Jacobi stopped at max_iter with ||p_{k+1}-p_k||_1 > tol */

int oracle_version(void) { return 1; }

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Serial FIFO-queue BFS over directed out-edges. */
int oracle_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col,
               int64_t src, int32_t *depth)
{
    if (n < 0 || (n > 0 && (src < 0 || src >= n)) || !row_ptr || !depth) return ORACLE_EINVAL;
    for (int64_t v = 0; v < n; ++v) depth[v] = -1;
    if (n == 0) return ORACLE_OK;
    int64_t *queue = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    if (!queue) return ORACLE_ENOMEM;
    int64_t head = 0, tail = 0;
    depth[src] = 0;
    queue[tail++] = src;
    while (head < tail) {
        int64_t v = queue[head++];
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int64_t u = col[e];
            if (depth[u] < 0) {            /* first visit = shortest hop count */
                depth[u] = depth[v] + 1;
                queue[tail++] = u;
            }
        }
    }
    free(queue);
    return ORACLE_OK;
}

/* parent(v) = min id u with u->v and depth(u) == depth(v)-1. */
int oracle_bfs_parents_minid(int64_t n, const int64_t *row_ptr, const int32_t *col,
                             const int32_t *depth, int64_t src, int64_t *parent)
{
    if (n < 0 || !row_ptr || !depth || !parent) return ORACLE_EINVAL;
    for (int64_t v = 0; v < n; ++v) parent[v] = -1;
    for (int64_t u = 0; u < n; ++u) {          /* ascending u: first hit is the minimum */
        if (depth[u] < 0) continue;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            int64_t v = col[e];
            if (v != src && parent[v] < 0 && depth[v] == depth[u] + 1) parent[v] = u;
        }
    }
    if (n > 0 && src >= 0 && src < n && depth[src] == 0) parent[src] = src;
    return ORACLE_OK;
}

/* Synchronous pull Jacobi PageRank with uniform dangling redistribution. */
int oracle_pagerank(int64_t n, const int64_t *row_ptr, const int32_t *col,
                    double alpha, double tol, int max_iter, int nthreads,
                    double *p_out, int *iters_out, double *delta_out)
{
    if (n <= 0 || !row_ptr || !p_out || !(alpha >= 0.0 && alpha < 1.0) || !(tol > 0.0))
        return ORACLE_EINVAL;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
    int64_t nnz = row_ptr[n];
    /* transpose: in-edges of u listed in ascending source order */
    int64_t *in_ptr = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t *in_src = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    double *p = (double *)malloc(sizeof(double) * (size_t)n);
    double *q = (double *)malloc(sizeof(double) * (size_t)n);
    double *contrib = (double *)malloc(sizeof(double) * (size_t)n);
    double *absdiff = (double *)malloc(sizeof(double) * (size_t)n);
    if (!in_ptr || !in_src || !fill || !p || !q || !contrib || !absdiff) {
        free(in_ptr); free(in_src); free(fill); free(p); free(q); free(contrib); free(absdiff);
        return ORACLE_ENOMEM;
    }
    for (int64_t e = 0; e < nnz; ++e) in_ptr[col[e] + 1]++;
    for (int64_t u = 0; u < n; ++u) in_ptr[u + 1] += in_ptr[u];
    for (int64_t u = 0; u < n; ++u) fill[u] = in_ptr[u];
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e)
            in_src[fill[col[e]]++] = (int32_t)v;

    const double inv_n = 1.0 / (double)n;
    for (int64_t v = 0; v < n; ++v) p[v] = inv_n;
    int it = 0;
    double delta = INFINITY;
    while (it < max_iter) {
        double dangling = 0.0;                 /* serial: fixed summation order */
        for (int64_t v = 0; v < n; ++v) {
            int64_t deg = row_ptr[v + 1] - row_ptr[v];
            if (deg == 0) { dangling += p[v]; contrib[v] = 0.0; }
            else contrib[v] = p[v] / (double)deg;
        }
        const double base = (1.0 - alpha) * inv_n + alpha * dangling * inv_n;
        #pragma omp parallel for schedule(static)
        for (int64_t u = 0; u < n; ++u) {
            double s = 0.0;
            for (int64_t e = in_ptr[u]; e < in_ptr[u + 1]; ++e) s += contrib[in_src[e]];
            q[u] = base + alpha * s;
            absdiff[u] = fabs(q[u] - p[u]);
        }
        delta = 0.0;
        for (int64_t u = 0; u < n; ++u) delta += absdiff[u];
        double *t = p; p = q; q = t;
        ++it;
        if (delta <= tol) break;
    }
    double sum = 0.0;
    for (int64_t v = 0; v < n; ++v) sum += p[v];
    for (int64_t v = 0; v < n; ++v) p_out[v] = p[v] / sum;
    if (iters_out) *iters_out = it;
    if (delta_out) *delta_out = delta;
    free(in_ptr); free(in_src); free(fill); free(p); free(q); free(contrib); free(absdiff);
    /* the definition is the FIXED POINT (north_star: "iterated to a 1e-12 L1
     * residual"); an iterate that has not reached tol is not the oracle's answer */
    return delta <= tol ? ORACLE_OK : ORACLE_ENOTCONV;
}
