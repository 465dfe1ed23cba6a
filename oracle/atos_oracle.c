/*
 * atos_oracle.c -- serial CPU oracle for the Atos hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (libatos.so and its Python binding) never links, imports
 * or calls anything here, and nothing here is shared with csrc/.
 *
 * Paper: Chen, Brock, Porumbescu, Buluc, Yelick, Owens, "Atos: A Task-Parallel
 * GPU Scheduler for Graph Analytics", ICPP'22 -- /root/reference/PAPER.md,
 * cited as P:<line>.  Readings of silent/garbled passages are listed in
 * DESIGN.md section "Readings" (R-BFS-*, R-PR-*, R-GC-*).
 *
 * Everything is single-threaded, plain C, no blocking or fusion.  Graphs are
 * CSR: row_ptr[n+1] (int64), col[m] (int32); row v lists the out-neighbours
 * of v (Listing 4 get_neighbor_list_start/length).
 *
 * Pins (tests/test_oracle_*.py): Floyd-Warshall, closed forms (path, cycle,
 * star, complete, grid, regular graphs, star PageRank), dense LU solve,
 * brute-force chromatic numbers, hand-solved 3-vertex PageRank, JP literal
 * round simulation == JP-by-priority greedy; the PageRank residual against
 * hand values (tests/golden/pr_residual_3vertex.json), the star closed form,
 * the dense matrix, and the push oracle's own residue array.  The colour-count of the GPU
 * path is "parity unpinned" (any proper colouring is correct).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define ORACLE_UNREACHED 0xFFFFFFFFu

/* ------------------------------------------------------------------------ */
/* BFS                                                                       */
/* ------------------------------------------------------------------------ */

/*
 * Definition ("BSP BFS is exactly Dijkstra's algorithm"; P:653-656
 * speculative BFS converges to the same depths): depth[v] = number of edges
 * on a shortest directed src->v path following CSR out-edges, depth[src]=0
 * (R-BFS-1), 0xFFFFFFFF when unreachable (Alg.1 init "MAX_UINT32", P:725,
 * R-BFS-2).  Written out as the textbook FIFO breadth-first search.
 * Returns 0, or -1 on bad arguments / allocation failure.
 */
int oracle_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col,
               int64_t src, uint32_t *depth)
{
    if (n < 0 || (n > 0 && (src < 0 || src >= n)) || !depth) return -1;
    for (int64_t v = 0; v < n; ++v) depth[v] = ORACLE_UNREACHED;
    if (n == 0) return 0;
    int64_t *fifo = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    if (!fifo) return -1;
    int64_t qh = 0, qt = 0;
    depth[src] = 0;
    fifo[qt++] = src;
    while (qh < qt) {
        int64_t v = fifo[qh++];
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int64_t w = col[e];
            if (depth[w] == ORACLE_UNREACHED) {
                depth[w] = depth[v] + 1;
                fifo[qt++] = w;
            }
        }
    }
    free(fifo);
    return 0;
}

/*
 * Graph500-style BFS validator (independent of any BFS implementation):
 *  (1) depth[src] == 0;
 *  (2) every edge (u,w) with u reached has w reached and depth[w] <= depth[u]+1;
 *  (3) every reached v != src has an in-neighbour u with depth[u] == depth[v]-1.
 * These three properties characterise shortest-path depths exactly.
 * Returns 0 when valid, otherwise a positive code naming the failed rule.
 */
int oracle_validate_bfs(int64_t n, const int64_t *row_ptr, const int32_t *col,
                        int64_t src, const uint32_t *depth)
{
    if (n == 0) return 0;
    if (depth[src] != 0) return 1;
    unsigned char *has_parent = (unsigned char *)calloc((size_t)n, 1);
    if (!has_parent) return 99;
    int rc = 0;
    for (int64_t u = 0; u < n && !rc; ++u) {
        if (depth[u] == ORACLE_UNREACHED) continue;
        for (int64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            int64_t w = col[e];
            if (depth[w] == ORACLE_UNREACHED) { rc = 2; break; }
            if ((uint64_t)depth[w] > (uint64_t)depth[u] + 1) { rc = 2; break; }
            if ((uint64_t)depth[w] == (uint64_t)depth[u] + 1) has_parent[w] = 1;
        }
    }
    for (int64_t v = 0; v < n && !rc; ++v)
        if (v != src && depth[v] != ORACLE_UNREACHED && !has_parent[v]) rc = 3;
    free(has_parent);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* PageRank                                                                  */
/* ------------------------------------------------------------------------ */

/*
 * Definition (R-PR-1): x solves x = (1-alpha)*1 + alpha * P^T x, P_{vw} =
 * (multiplicity of v->w)/deg(v), dangling rows zero; the result is x/n.
 * This is the fixed point of the paper's push iteration: rank starts at
 * 1-lambda (Alg.3) and every push adds lambda*res/deg to each
 * neighbour; lambda == alpha.
 *
 * Computed by Jacobi power iteration in double, written out plainly:
 *   x^0 = (1-alpha) 1
 *   x^{k+1}_w = (1-alpha) + alpha * sum_{v->w} x^k_v / deg(v)
 * stopping when max_w |x^{k+1}_w - x^k_w| <= tol or after max_iter sweeps.
 * The iterates increase monotonically to x*, so the stop rule bounds
 * 0 <= x_star - x <= tol * x_star / (1-alpha) elementwise (DESIGN.md R-PR-oracle).
 * rank_out[v] = x_v / n.  *iters_out = sweeps performed.  Returns 0 when the
 * tolerance was met, 1 when max_iter was hit, -1 on bad arguments.
 */
int oracle_pagerank_jacobi(int64_t n, const int64_t *row_ptr, const int32_t *col,
                           double alpha, double tol, int max_iter,
                           double *rank_out, int *iters_out)
{
    if (n < 0 || !(alpha > 0.0 && alpha < 1.0) || !(tol > 0.0) || !rank_out) return -1;
    if (n == 0) { if (iters_out) *iters_out = 0; return 0; }
    double *x = (double *)malloc(sizeof(double) * (size_t)n);
    double *y = (double *)malloc(sizeof(double) * (size_t)n);
    if (!x || !y) { free(x); free(y); return -1; }
    for (int64_t v = 0; v < n; ++v) x[v] = 1.0 - alpha;
    int k = 0, rc = 1;
    while (k < max_iter) {
        for (int64_t w = 0; w < n; ++w) y[w] = 0.0;
        for (int64_t v = 0; v < n; ++v) {
            int64_t deg = row_ptr[v + 1] - row_ptr[v];
            if (deg == 0) continue;                    /* dangling: zero row */
            double share = x[v] / (double)deg;
            for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) y[col[e]] += share;
        }
        double diff = 0.0;
        for (int64_t w = 0; w < n; ++w) {
            double nx = (1.0 - alpha) + alpha * y[w];
            double d = fabs(nx - x[w]);
            if (d > diff) diff = d;
            x[w] = nx;
        }
        ++k;
        if (diff <= tol) { rc = 0; break; }
    }
    for (int64_t v = 0; v < n; ++v) rank_out[v] = x[v] / (double)n;
    if (iters_out) *iters_out = k;
    free(x); free(y);
    return rc;
}

/*
 * Serial push PageRank following Algorithm 3's initialisation (P:761-767,
 * with the garbled P:766 read as R-PR-init: for each v, for each out-neighbour
 * w, residue[w] += (1-alpha)*alpha/deg(v)) and Algorithm 4's loop:
 *   vertex = frontier.pop(); res = residue[v]; residue[v] = 0;
 *   rank[v] += res; res = res*alpha/deg(v); residue[w] += res for neighbours.
 * Activation reading R-PR-6: a vertex is appended to the FIFO frontier when
 * its residue crosses eps from below (old <= eps < new); the initial frontier
 * holds, in ID order, every vertex whose residue exceeds eps (R-PR-7);
 * dangling vertices absorb their residue into rank (R-PR-3).  Stops when the
 * frontier is empty, i.e. every residue <= eps.
 * Outputs rank_out = rank/n; residue_out (optional) = final residues, not
 * normalised; *pops_out = number of pops.  Returns 0 / -1.
 */
int oracle_pagerank_push(int64_t n, const int64_t *row_ptr, const int32_t *col,
                         double alpha, double eps,
                         double *rank_out, double *residue_out, int64_t *pops_out)
{
    if (n < 0 || !(alpha > 0.0 && alpha < 1.0) || !(eps > 0.0) || !rank_out) return -1;
    if (pops_out) *pops_out = 0;
    if (n == 0) return 0;
    double *rank = (double *)malloc(sizeof(double) * (size_t)n);
    double *res = (double *)malloc(sizeof(double) * (size_t)n);
    /* FIFO ring: a vertex is queued at most once at a time (crossing rule), so n slots suffice */
    int64_t *q = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    unsigned char *inq = (unsigned char *)calloc((size_t)n, 1);
    if (!rank || !res || !q || !inq) { free(rank); free(res); free(q); free(inq); return -1; }
    for (int64_t v = 0; v < n; ++v) { rank[v] = 1.0 - alpha; res[v] = 0.0; }
    for (int64_t v = 0; v < n; ++v) {
        int64_t deg = row_ptr[v + 1] - row_ptr[v];
        if (deg == 0) continue;
        double add = (1.0 - alpha) * alpha / (double)deg;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) res[col[e]] += add;
    }
    int64_t qh = 0, qcount = 0, pops = 0;
    for (int64_t v = 0; v < n; ++v)
        if (res[v] > eps) { q[(qh + qcount) % n] = v; ++qcount; inq[v] = 1; }
    while (qcount > 0) {
        int64_t v = q[qh]; qh = (qh + 1) % n; --qcount; inq[v] = 0; ++pops;
        double r = res[v];
        res[v] = 0.0;
        rank[v] += r;
        int64_t deg = row_ptr[v + 1] - row_ptr[v];
        if (deg == 0) continue;
        double d = r * alpha / (double)deg;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int64_t w = col[e];
            double old = res[w];
            res[w] = old + d;
            if (old <= eps && res[w] > eps && !inq[w]) {
                q[(qh + qcount) % n] = w; ++qcount; inq[w] = 1;
            }
        }
    }
    for (int64_t v = 0; v < n; ++v) rank_out[v] = rank[v] / (double)n;
    if (residue_out) for (int64_t v = 0; v < n; ++v) residue_out[v] = res[v];
    if (pops_out) *pops_out = pops;
    free(rank); free(res); free(q); free(inq);
    return 0;
}

/*
 * PageRank residual of a candidate x (R-PR-1 definition, written out):
 *   r_w = (1-alpha) + alpha * sum_{v->w} x_v / deg(v)  -  x_w
 * one pass over the CSR rows, dangling rows contributing nothing (R-PR-3).
 * This is the residue of Alg.4 as a function of the ranks alone:
 * the push iteration keeps x* = x + (I - alpha P^T)^{-1} r at every step, and
 * stops when every residue <= eps.  So a candidate x whose
 * residual satisfies 0 <= r <= eps elementwise obeys
 *   0 <= x_star - x <= eps x_star / (1-alpha)
 * (because (I - alpha P^T)^{-1} >= 0 and (I - alpha P^T)^{-1} 1 = x_star / (1-alpha))
 * without solving for x*: one SpMV certifies the north-star tolerance at a
 * size where Jacobi to 1e-13 would take ~185 sweeps.  The in-neighbour sums
 * are accumulated in long double (x87 extended, 64-bit mantissa) so the
 * certificate's own rounding (<= indeg * 2^-64 * sum) stays far below eps
 * even at in-degrees of 10^6; the final subtraction is rounded to double.
 * x[n] is the UNNORMALISED rank (x = rank_out * n).  Returns 0 / -1.
 */
int oracle_pagerank_residual(int64_t n, const int64_t *row_ptr, const int32_t *col,
                             double alpha, const double *x, double *r_out)
{
    if (n < 0 || !(alpha > 0.0 && alpha < 1.0) || !x || !r_out) return -1;
    if (n == 0) return 0;
    long double *y = (long double *)malloc(sizeof(long double) * (size_t)n);
    if (!y) return -1;
    for (int64_t w = 0; w < n; ++w) y[w] = 0.0L;
    for (int64_t v = 0; v < n; ++v) {
        int64_t deg = row_ptr[v + 1] - row_ptr[v];
        if (deg == 0) continue;                        /* dangling: zero row */
        long double share = (long double)x[v] / (long double)deg;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) y[col[e]] += share;
    }
    for (int64_t w = 0; w < n; ++w)
        r_out[w] = (double)((1.0L - (long double)alpha) + (long double)alpha * y[w] - (long double)x[w]);
    free(y);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Graph colouring                                                           */
/* ------------------------------------------------------------------------ */

/*
 * Sequential greedy first-fit colouring in the given order (NULL = vertex-ID
 * order, the paper's initial queue order P:1231-1232).  This is Algorithm 5's
 * assign kernel (forbidden[] = neighbours' colours, colour =
 * find_min_color) run by a single worker, where no two vertices are coloured
 * concurrently and so no conflict is ever collected.  Self-loops
 * are ignored (R-GC-7); colours are 0-based, -1 = uncoloured.
 * Returns the number of colours used, or -1.
 */
int64_t oracle_color_greedy(int64_t n, const int64_t *row_ptr, const int32_t *col,
                            const int64_t *order, int32_t *color)
{
    if (n < 0 || !color) return -1;
    for (int64_t v = 0; v < n; ++v) color[v] = -1;
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] - row_ptr[v] > maxdeg) maxdeg = row_ptr[v + 1] - row_ptr[v];
    /* forbidden[c] == stamp  <=>  colour c is used by a neighbour of the current vertex */
    int64_t *forbidden = (int64_t *)malloc(sizeof(int64_t) * (size_t)(maxdeg + 2));
    if (!forbidden) return -1;
    for (int64_t c = 0; c < maxdeg + 2; ++c) forbidden[c] = -1;
    int64_t ncolors = 0;
    for (int64_t i = 0; i < n; ++i) {
        int64_t v = order ? order[i] : i;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int64_t w = col[e];
            if (w == v) continue;
            int32_t c = color[w];
            if (c >= 0 && c <= maxdeg + 1) forbidden[c] = v;
        }
        int32_t c = 0;
        while (forbidden[c] == v) ++c;
        color[v] = c;
        if (c + 1 > ncolors) ncolors = c + 1;
    }
    free(forbidden);
    return ncolors;
}

/*
 * splitmix64 (Steele, Lea, Flood 2014) -- the counter-based priority
 * pi(v) = splitmix64(seed ^ v) used for Jones-Plassmann and, independently
 * re-implemented on the GPU side, for the loser-recolours policy (R-GC-2).
 */
uint64_t oracle_splitmix64(uint64_t x)
{
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* priority order: larger pi first, ties broken by larger id */
static int jp_higher(uint64_t seed, int64_t a, int64_t b)
{
    uint64_t pa = oracle_splitmix64(seed ^ (uint64_t)a), pb = oracle_splitmix64(seed ^ (uint64_t)b);
    if (pa != pb) return pa > pb;
    return a > b;
}

static uint64_t g_sort_seed;
static int jp_cmp(const void *x, const void *y)
{
    int64_t a = *(const int64_t *)x, b = *(const int64_t *)y;
    if (a == b) return 0;
    return jp_higher(g_sort_seed, a, b) ? -1 : 1;
}

/*
 * Jones-Plassmann colouring with priority pi(v) = splitmix64(seed ^ v):
 * computed serially as greedy first-fit in decreasing-priority order (the
 * classical equivalence; cross-checked by oracle_color_jp_rounds).
 * Returns #colours or -1.  Not thread-safe (qsort comparator state).
 */
int64_t oracle_color_jp(int64_t n, const int64_t *row_ptr, const int32_t *col,
                        uint64_t seed, int32_t *color)
{
    if (n < 0 || !color) return -1;
    int64_t *order = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!order) return -1;
    for (int64_t v = 0; v < n; ++v) order[v] = v;
    g_sort_seed = seed;
    qsort(order, (size_t)n, sizeof(int64_t), jp_cmp);
    int64_t k = oracle_color_greedy(n, row_ptr, col, order, color);
    free(order);
    return k;
}

/*
 * Literal round-based Jones-Plassmann: in each round every uncoloured vertex
 * whose uncoloured neighbours all have lower priority takes the smallest
 * colour not used by its coloured neighbours.  O(rounds * m); tiny graphs.
 * Returns #colours or -1.
 */
int64_t oracle_color_jp_rounds(int64_t n, const int64_t *row_ptr, const int32_t *col,
                               uint64_t seed, int32_t *color)
{
    if (n < 0 || !color) return -1;
    for (int64_t v = 0; v < n; ++v) color[v] = -1;
    unsigned char *sel = (unsigned char *)malloc((size_t)(n > 0 ? n : 1));
    if (!sel) return -1;
    int64_t remaining = n, ncolors = 0;
    while (remaining > 0) {
        for (int64_t v = 0; v < n; ++v) {
            sel[v] = 0;
            if (color[v] >= 0) continue;
            int local_max = 1;
            for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
                int64_t w = col[e];
                if (w == v || color[w] >= 0) continue;
                if (jp_higher(seed, w, v)) { local_max = 0; break; }
            }
            sel[v] = (unsigned char)local_max;
        }
        for (int64_t v = 0; v < n; ++v) {
            if (!sel[v]) continue;
            int32_t c = 0;
            for (;;) {
                int used = 0;
                for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
                    int64_t w = col[e];
                    if (w != v && color[w] == c) { used = 1; break; }
                }
                if (!used) break;
                ++c;
            }
            color[v] = c;
            if (c + 1 > ncolors) ncolors = c + 1;
            --remaining;
        }
    }
    free(sel);
    return ncolors;
}

/*
 * Colouring validator: every colour >= 0, color[v] <= deg(v) (first-fit
 * bound, R-GC-4), and color[u] != color[w] for every edge u != w.
 * Returns 0 when valid, 1 uncoloured/out of range, 2 conflict.
 */
int oracle_validate_color(int64_t n, const int64_t *row_ptr, const int32_t *col,
                          const int32_t *color)
{
    for (int64_t v = 0; v < n; ++v) {
        int64_t deg = row_ptr[v + 1] - row_ptr[v];
        if (color[v] < 0 || (int64_t)color[v] > deg) return 1;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            int64_t w = col[e];
            if (w != v && color[w] == color[v]) return 2;
        }
    }
    return 0;
}
