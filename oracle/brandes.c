/*
 * oracle/brandes.c -- CPU ORACLE for the TurboBC hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (paper_conf_icppw_artiless21_b200/)
 * never links, imports or calls it, and shares no source with it.
 *
 * What it computes (PAPER.md = Artiles & Saeed, ICPPW'21, cited as P:<line>):
 *   BC(v) = sum_{s in sources, s != v} delta_s(v)                 Eq. 3
 *   delta_s(v) = sum_{w : d(s,w) = d(s,v)+1} sigma_sv/sigma_sw (1 + delta_s(w))   Eq. 4
 *   halved per source for undirected graphs
 * i.e. textbook Brandes (Eq. 2-4), which is what Algorithm 1
 * computes with SpMVs.  It is written as a queue BFS + reverse-order accumulation,
 * deliberately NOT in the paper's linear-algebra form, so that it is an independent
 * statement of the same definition.
 *
 * Conventions (SURVEY.md 8(c) readings, listed in DESIGN.md):
 *   - input is the CSC of the boolean adjacency matrix A: column v
 *     lists the rows u with A(u,v)=1, i.e. the edges u->v.  Duplicate entries collapse
 *     (A is boolean); self-loops are harmless.
 *   - depth(s)=0, unreachable = -1 (reading 3); sigma in fp64 (reading 9).
 *   - backward uses out-neighbours, i.e. A*delta_u, not A^T (reading 1: the printed
 *     A^T on Alg.1 l.37, is wrong for directed graphs).
 *   - the sources list may repeat; each occurrence counts (sum over the list).
 *
 * Parity status: every function here is pinned by tests/test_oracle.py against
 * brute-force Eq. 1 (exact rationals), closed forms, invariants and networkx.
 */
#define _POSIX_C_SOURCE 199309L
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <pthread.h>
#include <time.h>

typedef struct {
    int64_t n;
    int64_t *out_ptr;   /* CSR of A: out-neighbours (built here by counting sort) */
    int32_t *out_idx;
    int64_t *in_ptr;    /* CSC of A, deduplicated copy: in-neighbours */
    int32_t *in_idx;
} og_graph;

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* sort + unique each adjacency list in place; returns new nnz, compacts arrays */
static int64_t og_dedup(int64_t n, int64_t *ptr, int32_t *idx) {
    int64_t w = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t b = ptr[v], e = ptr[v + 1];
        qsort(idx + b, (size_t)(e - b), sizeof(int32_t), cmp_i32);
        ptr[v] = w;
        for (int64_t k = b; k < e; ++k)
            if (k == b || idx[k] != idx[k - 1]) idx[w++] = idx[k];
    }
    ptr[n] = w;
    return w;
}

static void og_free(og_graph *g) {
    free(g->out_ptr); free(g->out_idx); free(g->in_ptr); free(g->in_idx);
}

/* Build deduplicated in- and out-adjacency from the caller's CSC (CP_A, row_A). */
static int og_build(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, og_graph *g) {
    int64_t nnz = col_ptr[n];
    g->n = n;
    g->in_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    g->in_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    g->out_ptr = (int64_t *)calloc((size_t)(n + 1), sizeof(int64_t));
    g->out_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
    if (!g->in_ptr || !g->in_idx || !g->out_ptr || !g->out_idx) { og_free(g); return -1; }
    memcpy(g->in_ptr, col_ptr, sizeof(int64_t) * (size_t)(n + 1));
    memcpy(g->in_idx, row_idx, sizeof(int32_t) * (size_t)nnz);
    nnz = og_dedup(n, g->in_ptr, g->in_idx);
    /* transpose: edge u->v is row u in column v */
    for (int64_t v = 0; v < n; ++v)
        for (int64_t k = g->in_ptr[v]; k < g->in_ptr[v + 1]; ++k) g->out_ptr[g->in_idx[k] + 1]++;
    for (int64_t u = 0; u < n; ++u) g->out_ptr[u + 1] += g->out_ptr[u];
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!fill) { og_free(g); return -1; }
    memcpy(fill, g->out_ptr, sizeof(int64_t) * (size_t)n);
    for (int64_t v = 0; v < n; ++v)
        for (int64_t k = g->in_ptr[v]; k < g->in_ptr[v + 1]; ++k)
            g->out_idx[fill[g->in_idx[k]]++] = (int32_t)v;
    free(fill);
    return 0;
}

typedef struct {
    int32_t *dist;
    double *sigma;
    double *acc;      /* sum over children w of (1+delta(w))/sigma(w) */
    int32_t *order;   /* BFS visiting order (the stack of Brandes' algorithm) */
} og_work;

static int og_work_alloc(int64_t n, og_work *w) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    w->dist = (int32_t *)malloc(sizeof(int32_t) * nn);
    w->sigma = (double *)malloc(sizeof(double) * nn);
    w->acc = (double *)malloc(sizeof(double) * nn);
    w->order = (int32_t *)malloc(sizeof(int32_t) * nn);
    return (w->dist && w->sigma && w->acc && w->order) ? 0 : -1;
}
static void og_work_free(og_work *w) { free(w->dist); free(w->sigma); free(w->acc); free(w->order); }

/* Forward stage: BFS from s counting shortest paths.  Alg.1 l.11-28,
 * P:176-178; depth/sigma semantics of Alg.1 l.9-10, l.24-25.  Returns |order|. */
static int64_t og_forward(const og_graph *g, int32_t s, og_work *w) {
    int64_t n = g->n;
    for (int64_t v = 0; v < n; ++v) { w->dist[v] = -1; w->sigma[v] = 0.0; w->acc[v] = 0.0; }
    w->dist[s] = 0;
    w->sigma[s] = 1.0;                                   /* Alg.1 l.17 */
    int64_t head = 0, tail = 0;
    w->order[tail++] = s;
    while (head < tail) {
        int32_t v = w->order[head++];
        for (int64_t k = g->out_ptr[v]; k < g->out_ptr[v + 1]; ++k) {
            int32_t x = g->out_idx[k];
            if (w->dist[x] < 0) { w->dist[x] = w->dist[v] + 1; w->order[tail++] = x; }
            if (w->dist[x] == w->dist[v] + 1) w->sigma[x] += w->sigma[v];
        }
    }
    return tail;
}

/* Backward stage + accumulation for one source.  Eq. 4 evaluated in reverse BFS
 * order; Alg.1 l.31-47 with A (not A^T) on l.37; halving per P:180.
 * If delta_out != NULL it receives delta_s(v) (0 for s and unreachable vertices). */
static void og_backward(const og_graph *g, int32_t s, og_work *w, int64_t reached, int directed,
                        double *bc, double *delta_out) {
    if (delta_out) for (int64_t v = 0; v < g->n; ++v) delta_out[v] = 0.0;
    for (int64_t i = reached - 1; i >= 0; --i) {
        int32_t x = w->order[i];
        double delta_x = w->sigma[x] * w->acc[x];         /* Alg.1 l.39: delta = sigma * (A delta_u) */
        if (x != s) {                                       /* Alg.1 l.44 */
            bc[x] += directed ? delta_x : 0.5 * delta_x;    /* Alg.1 l.45 */
            if (delta_out) delta_out[x] = delta_x;
        }
        double coef = (1.0 + delta_x) / w->sigma[x];        /* Alg.1 l.35: delta_u */
        for (int64_t k = g->in_ptr[x]; k < g->in_ptr[x + 1]; ++k) {
            int32_t v = g->in_idx[k];                       /* edge v->x */
            if (w->dist[v] == w->dist[x] - 1) w->acc[v] += coef;
        }
    }
}

/* ---------------------------------------------------------------- public API */

/* BFS depth and sigma from one source (forward stage only). Returns 0, or -1 on bad input. */
int oracle_bfs(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int32_t source,
               int32_t *depth_out, double *sigma_out) {
    if (n <= 0 || source < 0 || source >= n) return -1;
    og_graph g; og_work w;
    if (og_build(n, col_ptr, row_idx, &g)) return -1;
    if (og_work_alloc(n, &w)) { og_free(&g); return -1; }
    og_forward(&g, source, &w);
    if (depth_out) memcpy(depth_out, w.dist, sizeof(int32_t) * (size_t)n);
    if (sigma_out) memcpy(sigma_out, w.sigma, sizeof(double) * (size_t)n);
    og_work_free(&w); og_free(&g);
    return 0;
}

/* One-sided dependencies delta_s(v) (Eq. 2) for one source, unhalved. */
int oracle_delta(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int32_t source,
                 double *delta_out) {
    if (n <= 0 || source < 0 || source >= n) return -1;
    og_graph g; og_work w;
    if (og_build(n, col_ptr, row_idx, &g)) return -1;
    if (og_work_alloc(n, &w)) { og_free(&g); return -1; }
    double *scratch = (double *)calloc((size_t)n, sizeof(double));
    int64_t r = og_forward(&g, source, &w);
    og_backward(&g, source, &w, r, 1, scratch, delta_out);
    free(scratch); og_work_free(&w); og_free(&g);
    return 0;
}

typedef struct {
    const og_graph *g;
    const int32_t *sources;
    int64_t lo, hi;
    int directed;
    double *bc;       /* private partial, n entries */
    int status;
} og_task;

static void *og_thread(void *arg) {
    og_task *t = (og_task *)arg;
    og_work w;
    if (og_work_alloc(t->g->n, &w)) { t->status = -1; return NULL; }
    for (int64_t i = t->lo; i < t->hi; ++i) {               /* Alg.1 l.6: for each source */
        int64_t r = og_forward(t->g, t->sources[i], &w);
        og_backward(t->g, t->sources[i], &w, r, t->directed, t->bc, NULL);
    }
    og_work_free(&w);
    t->status = 0;
    return NULL;
}

/* bc over an explicit source list (Alg.1 l.6 generalised to a list), nthreads >= 1
 * threads over contiguous source ranges, partials reduced in thread order.
 * Returns 0, or -1 on bad input / allocation failure. */
int oracle_bc_timed(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int directed,
                    const int32_t *sources, int64_t k, int nthreads, double *bc_out,
                    double *compute_seconds);

int oracle_bc(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int directed,
              const int32_t *sources, int64_t k, int nthreads, double *bc_out) {
    return oracle_bc_timed(n, col_ptr, row_idx, directed, sources, k, nthreads, bc_out, NULL);
}

/* Same as oracle_bc; if compute_seconds != NULL it receives the wall time of the source loop
 * alone (graph build excluded) -- a measurement hook for bench.py's cpu_baseline. */
int oracle_bc_timed(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int directed,
                    const int32_t *sources, int64_t k, int nthreads, double *bc_out,
                    double *compute_seconds) {
    if (n <= 0 || k < 0 || !bc_out) return -1;
    for (int64_t i = 0; i < k; ++i) if (sources[i] < 0 || sources[i] >= n) return -1;
    og_graph g;
    if (og_build(n, col_ptr, row_idx, &g)) return -1;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > k) nthreads = (int)(k > 0 ? k : 1);
    og_task *tasks = (og_task *)calloc((size_t)nthreads, sizeof(og_task));
    pthread_t *th = (pthread_t *)calloc((size_t)nthreads, sizeof(pthread_t));
    int rc = 0;
    for (int t = 0; t < nthreads; ++t) {
        tasks[t].g = &g; tasks[t].sources = sources; tasks[t].directed = directed;
        tasks[t].lo = k * t / nthreads; tasks[t].hi = k * (t + 1) / nthreads;
        tasks[t].bc = (double *)calloc((size_t)n, sizeof(double));
        if (!tasks[t].bc) rc = -1;
    }
    struct timespec t0, t1;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    if (!rc) {
        for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, og_thread, &tasks[t]);
        for (int t = 0; t < nthreads; ++t) { pthread_join(th[t], NULL); if (tasks[t].status) rc = -1; }
    }
    clock_gettime(CLOCK_MONOTONIC, &t1);
    if (compute_seconds)
        *compute_seconds = (double)(t1.tv_sec - t0.tv_sec) + 1e-9 * (double)(t1.tv_nsec - t0.tv_nsec);
    if (!rc) {
        for (int64_t v = 0; v < n; ++v) bc_out[v] = 0.0;
        for (int t = 0; t < nthreads; ++t)
            for (int64_t v = 0; v < n; ++v) bc_out[v] += tasks[t].bc[v];
    }
    for (int t = 0; t < nthreads; ++t) free(tasks[t].bc);
    free(tasks); free(th); og_free(&g);
    return rc;
}

/* ---------------------------------------------------------------- extended range (NEXT-2)
 * The same textbook Brandes in C long double (x86-64: 64-bit mantissa, 15-bit exponent, range
 * ~2^16383), for graphs whose shortest-path counts overflow fp64: on a P_a x P_b mesh sigma from a
 * corner is C(i+j, i), ~2^8190 at 4096 x 4096 (the paper's int sigma, and fp64
 * both overflow).  Same passages as og_forward / og_backward (Alg.1, Eq. 4); only the
 * number type differs.  sigma is exported as mantissa in [0.5, 1) and a binary exponent (frexpl). */

typedef struct {
    int32_t *dist;
    long double *sigma;
    long double *acc;
    int32_t *order;
} og_work_ld;

static int og_work_ld_alloc(int64_t n, og_work_ld *w) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    w->dist = (int32_t *)malloc(sizeof(int32_t) * nn);
    w->sigma = (long double *)malloc(sizeof(long double) * nn);
    w->acc = (long double *)malloc(sizeof(long double) * nn);
    w->order = (int32_t *)malloc(sizeof(int32_t) * nn);
    return (w->dist && w->sigma && w->acc && w->order) ? 0 : -1;
}
static void og_work_ld_free(og_work_ld *w) { free(w->dist); free(w->sigma); free(w->acc); free(w->order); }

static int64_t og_forward_ld(const og_graph *g, int32_t s, og_work_ld *w) {
    int64_t n = g->n;
    for (int64_t v = 0; v < n; ++v) { w->dist[v] = -1; w->sigma[v] = 0.0L; w->acc[v] = 0.0L; }
    w->dist[s] = 0;
    w->sigma[s] = 1.0L;                                  /* Alg.1 l.17 */
    int64_t head = 0, tail = 0;
    w->order[tail++] = s;
    while (head < tail) {
        int32_t v = w->order[head++];
        for (int64_t k = g->out_ptr[v]; k < g->out_ptr[v + 1]; ++k) {
            int32_t x = g->out_idx[k];
            if (w->dist[x] < 0) { w->dist[x] = w->dist[v] + 1; w->order[tail++] = x; }
            if (w->dist[x] == w->dist[v] + 1) w->sigma[x] += w->sigma[v];
        }
    }
    return tail;
}

static void og_backward_ld(const og_graph *g, int32_t s, og_work_ld *w, int64_t reached, int directed,
                           long double *bc) {
    for (int64_t i = reached - 1; i >= 0; --i) {
        int32_t x = w->order[i];
        long double delta_x = w->sigma[x] * w->acc[x];      /* Alg.1 l.39 */
        if (x != s) bc[x] += directed ? delta_x : 0.5L * delta_x;   /* Alg.1 l.45 */
        long double coef = (1.0L + delta_x) / w->sigma[x];  /* Alg.1 l.35 */
        for (int64_t k = g->in_ptr[x]; k < g->in_ptr[x + 1]; ++k) {
            int32_t v = g->in_idx[k];
            if (w->dist[v] == w->dist[x] - 1) w->acc[v] += coef;
        }
    }
}

/* depth and sigma (as mantissa * 2^exponent) from one source, long double. */
int oracle_bfs_ld(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int32_t source,
                  int32_t *depth_out, double *sigma_mant, int32_t *sigma_exp) {
    if (n <= 0 || source < 0 || source >= n) return -1;
    og_graph g; og_work_ld w;
    if (og_build(n, col_ptr, row_idx, &g)) return -1;
    if (og_work_ld_alloc(n, &w)) { og_free(&g); return -1; }
    og_forward_ld(&g, source, &w);
    for (int64_t v = 0; v < n; ++v) {
        int e = 0;
        long double m = frexpl(w.sigma[v], &e);
        if (depth_out) depth_out[v] = w.dist[v];
        if (sigma_mant) sigma_mant[v] = (double)m;
        if (sigma_exp) sigma_exp[v] = (int32_t)e;
    }
    og_work_ld_free(&w); og_free(&g);
    return 0;
}

/* bc over a source list, long double accumulation, rounded to double at the end (single thread). */
int oracle_bc_ld(int64_t n, const int64_t *col_ptr, const int32_t *row_idx, int directed,
                 const int32_t *sources, int64_t k, double *bc_out) {
    if (n <= 0 || k < 0 || !bc_out) return -1;
    for (int64_t i = 0; i < k; ++i) if (sources[i] < 0 || sources[i] >= n) return -1;
    og_graph g; og_work_ld w;
    if (og_build(n, col_ptr, row_idx, &g)) return -1;
    if (og_work_ld_alloc(n, &w)) { og_free(&g); return -1; }
    long double *bc = (long double *)calloc((size_t)n, sizeof(long double));
    if (!bc) { og_work_ld_free(&w); og_free(&g); return -1; }
    for (int64_t i = 0; i < k; ++i) {                        /* Alg.1 l.6 */
        int64_t r = og_forward_ld(&g, sources[i], &w);
        og_backward_ld(&g, sources[i], &w, r, directed, bc);
    }
    for (int64_t v = 0; v < n; ++v) bc_out[v] = (double)bc[v];
    free(bc); og_work_ld_free(&w); og_free(&g);
    return 0;
}
