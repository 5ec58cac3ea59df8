/*
 * oracle/oracle.c -- plain, slow, obviously-correct CPU oracle for GUM's hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. The product path (paper_conf_icde_menggltyz23_b200)
 * never imports, links or calls it, and shares no code with it: the two meet only at the seeded
 * edge lists produced by inputs/.
 *
 * What it computes (PAPER.md cited as P:<line>):
 *   The paper runs GAS algorithms in BSP mode over a frontier f_k (§II "Graph algorithms")
 *   for BFS, WCC, PR and SSSP (§VI-A "Baseline"). The paper never defines the outputs;
 *   DESIGN.md "Readings" #1 fixes them. BFS, SSSP and WCC are monotone min-fixpoints, so any
 *   schedule (including FSteal/OSteal) reaches the unique textbook answer; the oracle is that
 *   textbook definition:
 *     oracle_bfs         queue BFS hop depth from s                      (c-1; P:75 Example 2)
 *     oracle_sssp        binary-heap Dijkstra with lazy deletion, u64    (c-2; P:25 Example 1)
 *     oracle_wcc         union-find, union by smaller root id, halving   (c-3; Tab. III WCC)
 *     oracle_pagerank    fixed-K power iteration, fp64, dangling mass
 *                        redistributed uniformly                          (c-4)
 *   Graph semantics (c-0): directed multigraph, self-loops and parallel edges kept; BFS/SSSP/PR
 *   follow out-edges, WCC ignores direction. INF = 0xFFFFFFFF.
 *
 * Pins (tests/test_oracle_*.py, -m "not gpu"): closed forms (path, cycle, star, grid i+j,
 * torus x=1/V), scipy.sparse.csgraph (shortest_path, dijkstra, connected_components),
 * networkx.pagerank, brute force (Floyd-Warshall, reachability powers, dense PR) on tiny graphs.
 * No function here is "parity unpinned".
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC. Every function is single-threaded by design (SURVEY.md §8(d)
 * "Oracle timing") except oracle_pagerank_pull, the OpenMP variant §8(d) allows for full-size PR
 * checks ("an optional OpenMP pull variant reports its thread count").
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <omp.h>

#define ORACLE_INF 0xFFFFFFFFu

/* ---- own adjacency: counting sort of the raw edge list by source (stable) ---------------- */
/* row_ptr: uint64[V+1]; adj: uint32[E]; wadj: uint32[E] (may be NULL if w == NULL).           */
int oracle_build_adj(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, const uint32_t* w,
                     uint64_t* row_ptr, uint32_t* adj, uint32_t* wadj) {
    memset(row_ptr, 0, sizeof(uint64_t) * ((size_t)V + 1));
    for (uint64_t i = 0; i < E; i++) {
        if (src[i] >= V || dst[i] >= V) return -1;
        row_ptr[src[i] + 1]++;
    }
    for (uint32_t v = 0; v < V; v++) row_ptr[v + 1] += row_ptr[v];
    uint64_t* fill = (uint64_t*)malloc(sizeof(uint64_t) * ((size_t)V + 1));
    if (!fill) return -2;
    memcpy(fill, row_ptr, sizeof(uint64_t) * ((size_t)V + 1));
    for (uint64_t i = 0; i < E; i++) {
        uint64_t pos = fill[src[i]]++;
        adj[pos] = dst[i];
        if (w && wadj) wadj[pos] = w[i];
    }
    free(fill);
    return 0;
}

/* ---- c-1 BFS: FIFO queue ------------------------------------------------------------------ */
int oracle_bfs(uint32_t V, const uint64_t* row_ptr, const uint32_t* adj, uint32_t s, uint32_t* depth) {
    if (s >= V) return -1;
    uint32_t* queue = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(V ? V : 1));
    if (!queue) return -2;
    for (uint32_t v = 0; v < V; v++) depth[v] = ORACLE_INF;
    size_t head = 0, tail = 0;
    depth[s] = 0;
    queue[tail++] = s;
    while (head < tail) {
        uint32_t u = queue[head++];
        for (uint64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            uint32_t v = adj[e];
            if (depth[v] == ORACLE_INF) {
                depth[v] = depth[u] + 1;
                queue[tail++] = v;
            }
        }
    }
    free(queue);
    return 0;
}

/* ---- c-2 SSSP: binary-heap Dijkstra with lazy deletion, u64 arithmetic -------------------- */
typedef struct { uint64_t d; uint32_t v; } heap_item;

static void heap_push(heap_item* h, size_t* n, heap_item x) {
    size_t i = (*n)++;
    h[i] = x;
    while (i > 0) {
        size_t p = (i - 1) / 2;
        if (h[p].d <= h[i].d) break;
        heap_item t = h[p]; h[p] = h[i]; h[i] = t;
        i = p;
    }
}

static heap_item heap_pop(heap_item* h, size_t* n) {
    heap_item top = h[0];
    h[0] = h[--(*n)];
    size_t i = 0;
    for (;;) {
        size_t l = 2 * i + 1, r = l + 1, m = i;
        if (l < *n && h[l].d < h[m].d) m = l;
        if (r < *n && h[r].d < h[m].d) m = r;
        if (m == i) break;
        heap_item t = h[m]; h[m] = h[i]; h[i] = t;
        i = m;
    }
    return top;
}

/* Returns 0 ok, -1 bad source, -2 oom, -3 a finite distance >= 2^32-1 (ERANGE). */
int oracle_sssp(uint32_t V, const uint64_t* row_ptr, const uint32_t* adj, const uint32_t* wadj, uint32_t s,
                uint32_t* dist_out) {
    if (s >= V) return -1;
    uint64_t E = row_ptr[V];
    uint64_t* dist = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(V ? V : 1));
    heap_item* heap = (heap_item*)malloc(sizeof(heap_item) * (size_t)(E + 1));
    if (!dist || !heap) { free(dist); free(heap); return -2; }
    for (uint32_t v = 0; v < V; v++) dist[v] = UINT64_MAX;
    size_t n = 0;
    dist[s] = 0;
    heap_push(heap, &n, (heap_item){0, s});
    while (n > 0) {
        heap_item it = heap_pop(heap, &n);
        if (it.d != dist[it.v]) continue; /* stale entry (lazy deletion) */
        uint32_t u = it.v;
        for (uint64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            uint32_t v = adj[e];
            uint64_t nd = dist[u] + (uint64_t)wadj[e];
            if (nd < dist[v]) {
                dist[v] = nd;
                heap_push(heap, &n, (heap_item){nd, v});
            }
        }
    }
    int rc = 0;
    for (uint32_t v = 0; v < V; v++) {
        if (dist[v] == UINT64_MAX) dist_out[v] = ORACLE_INF;
        else if (dist[v] >= (uint64_t)ORACLE_INF) { dist_out[v] = ORACLE_INF; rc = -3; }
        else dist_out[v] = (uint32_t)dist[v];
    }
    free(dist);
    free(heap);
    return rc;
}

/* ---- c-3 WCC: union-find over every edge ignoring direction -------------------------------- */
static uint32_t uf_find(uint32_t* parent, uint32_t x) {
    while (parent[x] != x) {
        parent[x] = parent[parent[x]]; /* path halving */
        x = parent[x];
    }
    return x;
}

int oracle_wcc(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, uint32_t* label) {
    for (uint32_t v = 0; v < V; v++) label[v] = v;
    for (uint64_t i = 0; i < E; i++) {
        if (src[i] >= V || dst[i] >= V) return -1;
        uint32_t a = uf_find(label, src[i]);
        uint32_t b = uf_find(label, dst[i]);
        if (a == b) continue;
        if (a < b) label[b] = a; /* union by smaller root id: the root is the component minimum */
        else label[a] = b;
    }
    for (uint32_t v = 0; v < V; v++) label[v] = uf_find(label, v);
    return 0;
}

/* ---- c-4 PageRank: fixed-K power iteration (fp64) -------------------------------------------
 *   x_0[v] = 1/V
 *   D_k    = sum_{u : outdeg(u) = 0} x_k[u]
 *   x_{k+1}[v] = (1-d)/V + d * ( sum_{(u,v) in E} x_k[u]/outdeg(u) + D_k/V )
 *   resid[k] = sum_v |x_{k+1}[v] - x_k[v]|
 * Multiplicity counts in outdeg and in contributions (c-0). Edge-list push, in edge order.      */
int oracle_pagerank(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, int K, double d,
                    double* x_out, double* resid) {
    if (V == 0) return 0;
    uint64_t* outdeg = (uint64_t*)calloc((size_t)V, sizeof(uint64_t));
    double* x = (double*)malloc(sizeof(double) * V);
    double* y = (double*)malloc(sizeof(double) * V);
    if (!outdeg || !x || !y) { free(outdeg); free(x); free(y); return -2; }
    for (uint64_t i = 0; i < E; i++) {
        if (src[i] >= V || dst[i] >= V) { free(outdeg); free(x); free(y); return -1; }
        outdeg[src[i]]++;
    }
    for (uint32_t v = 0; v < V; v++) x[v] = 1.0 / (double)V;
    for (int k = 0; k < K; k++) {
        double D = 0.0;
        for (uint32_t u = 0; u < V; u++)
            if (outdeg[u] == 0) D += x[u];
        for (uint32_t v = 0; v < V; v++) y[v] = 0.0;
        for (uint64_t i = 0; i < E; i++) y[dst[i]] += x[src[i]] / (double)outdeg[src[i]];
        double r = 0.0;
        for (uint32_t v = 0; v < V; v++) {
            double nx = (1.0 - d) / (double)V + d * (y[v] + D / (double)V);
            r += fabs(nx - x[v]);
            x[v] = nx;
        }
        if (resid) resid[k] = r;
    }
    memcpy(x_out, x, sizeof(double) * V);
    free(outdeg);
    free(x);
    free(y);
    return 0;
}

/* ---- c-4 PageRank, OpenMP pull variant ("an optional OpenMP pull variant reports its
 * thread count"). The same recurrence as oracle_pagerank, computed per destination:
 *   y[v] = sum over the in-edges (u, v) of x_k[u]/outdeg(u)
 * with the in-edges of v taken from a STABLE counting sort of the raw edge list by destination, i.e. in
 * increasing edge index -- the order in which oracle_pagerank's edge loop adds them into y[v]. Each term
 * is the same double (x[u]/outdeg(u), one division) and each sum has the same order, so x_K is identical
 * to oracle_pagerank's (D_k is summed serially in vertex order as there); only the residual is reduced
 * in another order (pinned in tests/test_oracle.py). nthreads <= 0 => omp_get_max_threads(); *threads_used reports it.           */
int oracle_pagerank_pull(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, int K, double d,
                         int nthreads, double* x_out, double* resid, int* threads_used) {
    if (V == 0) return 0;
    const int T = nthreads > 0 ? nthreads : omp_get_max_threads();
    if (threads_used) *threads_used = T;
    uint64_t* outdeg = (uint64_t*)calloc((size_t)V, sizeof(uint64_t));
    uint64_t* in_ptr = (uint64_t*)calloc((size_t)V + 1, sizeof(uint64_t));
    uint32_t* in_src = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(E ? E : 1));
    double* x = (double*)malloc(sizeof(double) * V);
    double* cx = (double*)malloc(sizeof(double) * V);
    double* y = (double*)malloc(sizeof(double) * V);
    if (!outdeg || !in_ptr || !in_src || !x || !cx || !y) {
        free(outdeg); free(in_ptr); free(in_src); free(x); free(cx); free(y);
        return -2;
    }
    for (uint64_t i = 0; i < E; i++) {
        if (src[i] >= V || dst[i] >= V) {
            free(outdeg); free(in_ptr); free(in_src); free(x); free(cx); free(y);
            return -1;
        }
        outdeg[src[i]]++;
        in_ptr[dst[i] + 1]++;
    }
    for (uint32_t v = 0; v < V; v++) in_ptr[v + 1] += in_ptr[v];
    {
        uint64_t* fill = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)V);
        if (!fill) {
            free(outdeg); free(in_ptr); free(in_src); free(x); free(cx); free(y);
            return -2;
        }
        memcpy(fill, in_ptr, sizeof(uint64_t) * (size_t)V);
        for (uint64_t i = 0; i < E; i++) in_src[fill[dst[i]]++] = src[i]; /* stable: edge order per v */
        free(fill);
    }
    for (uint32_t v = 0; v < V; v++) x[v] = 1.0 / (double)V;
    for (int k = 0; k < K; k++) {
        double D = 0.0; /* serial, in vertex order: the same D_k as oracle_pagerank */
        for (uint32_t u = 0; u < V; u++)
            if (outdeg[u] == 0) D += x[u];
#pragma omp parallel for num_threads(T) schedule(static)
        for (int64_t u = 0; u < (int64_t)V; u++) cx[u] = outdeg[u] ? x[u] / (double)outdeg[u] : 0.0;
#pragma omp parallel for num_threads(T) schedule(dynamic, 4096)
        for (int64_t v = 0; v < (int64_t)V; v++) {
            double acc = 0.0;
            for (uint64_t e = in_ptr[v]; e < in_ptr[v + 1]; e++) acc += cx[in_src[e]];
            y[v] = acc;
        }
        double r = 0.0;
#pragma omp parallel for num_threads(T) schedule(static) reduction(+ : r)
        for (int64_t v = 0; v < (int64_t)V; v++) {
            double nx = (1.0 - d) / (double)V + d * (y[v] + D / (double)V);
            r += fabs(nx - x[v]);
            x[v] = nx;
        }
        if (resid) resid[k] = r;
    }
    memcpy(x_out, x, sizeof(double) * V);
    free(outdeg); free(in_ptr); free(in_src); free(x); free(cx); free(y);
    return 0;
}

/* ---- NEXT-4 delta-PageRank (§I: "delta-PageRank, SSSP, and BFS" suffer the long tail) ----
 * DESIGN.md reading #27. The paper names the algorithm without defining it; the reading is the
 * residual-push ("delta") formulation of PageRank run as frontier-driven BSP rounds:
 *   target  x* = the unique solution of x = (1-d)/V + d * sum_{(u,v) in E} x_u / outdeg(u)
 *           (a dangling vertex's mass is not redistributed -- the delta-based variant of the literature);
 *   state   x = 0, residual r = (1-d)/V for every vertex;
 *   round   F = { u : r_u > eps } in vertex order. Every u in F first hands its residual over
 *           (x_u += r_u, push_u = d*r_u/outdeg(u) or 0 if dangling, r_u = 0); then for each u in F and each
 *           out-edge (u, v) in edge order, r_v += push_u.
 *   stop    F empty. rounds_out = number of rounds with a non-empty F.
 * The identity x + (I - d P^T)^{-1} r = x* holds after every round, so 0 <= x* - x componentwise and
 * sum(x* - x) <= sum(r) / (1 - d) <= V * eps / (1 - d) at the end (pinned in tests/test_oracle.py).        */
int oracle_delta_pagerank(uint32_t V, uint64_t E, const uint32_t* src, const uint32_t* dst, double d, double eps,
                          double* x, double* r, uint32_t* rounds_out, uint64_t* work_out) {
    if (V == 0) return 0;
    uint64_t* row_ptr = (uint64_t*)calloc((size_t)V + 1, sizeof(uint64_t));
    uint32_t* adj = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(E ? E : 1));
    double* push = (double*)malloc(sizeof(double) * V);
    uint32_t* F = (uint32_t*)malloc(sizeof(uint32_t) * V);
    if (!row_ptr || !adj || !push || !F) {
        free(row_ptr); free(adj); free(push); free(F);
        return -2;
    }
    if (oracle_build_adj(V, E, src, dst, NULL, row_ptr, adj, NULL) != 0) {
        free(row_ptr); free(adj); free(push); free(F);
        return -1;
    }
    for (uint32_t v = 0; v < V; v++) {
        x[v] = 0.0;
        r[v] = (1.0 - d) / (double)V;
    }
    uint32_t rounds = 0;
    uint64_t work = 0; /* edges pushed along (the work rate's numerator) */
    for (;;) {
        size_t nf = 0;
        for (uint32_t v = 0; v < V; v++)
            if (r[v] > eps) F[nf++] = v;
        if (nf == 0) break;
        rounds++;
        for (size_t i = 0; i < nf; i++) {
            uint32_t u = F[i];
            uint64_t od = row_ptr[u + 1] - row_ptr[u];
            x[u] += r[u];
            push[u] = od ? d * r[u] / (double)od : 0.0;
            r[u] = 0.0;
        }
        for (size_t i = 0; i < nf; i++) {
            uint32_t u = F[i];
            for (uint64_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) r[adj[e]] += push[u];
            work += row_ptr[u + 1] - row_ptr[u];
        }
    }
    if (rounds_out) *rounds_out = rounds;
    if (work_out) *work_out = work;
    free(row_ptr); free(adj); free(push); free(F);
    return 0;
}
