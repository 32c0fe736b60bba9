/*
 * tbc.h -- C ABI of the B200-native TurboBC hot path (libturbobc.so).
 *
 * The method: Brandes betweenness centrality written as linear algebra, PAPER.md
 * (Artiles & Saeed, "TurboBC", ICPP Workshops '21), cited as P:<line>:
 *   Algorithm 1 BC-LA: per source s a forward BFS stage of masked SpMV
 *   f_t = A^T f producing sigma (shortest-path counts) and S (depth)  (l.11-28), then a
 *   backward stage over the levels in reverse with delta_u = (1+delta)/sigma, one SpMV
 *   and delta += sigma * (SpMV result)  (l.29-42), then bc(v) += delta(v), v != s
 *   (l.43-47), halved for undirected graphs.
 *
 * Conventions (all functions):
 *   - vertex ids are int32_t, 0-based (the paper's CSC is 1-based); sizes int64_t.
 *   - the graph is the boolean n x n adjacency matrix A: A(u,v) = 1 <=> edge u->v.
 *     CSC column v lists the ROWS u with A(u,v)=1, i.e. the in-neighbours of v.
 *     Duplicates collapse (A is boolean); self-loops are accepted and change nothing.
 *   - depth(s) = 0, unreachable = -1 (the paper's S is max(depth,0), R3).
 *   - sigma and bc are IEEE fp64.  sigma is exact while < 2^53.
 *   - the backward SpMV uses A (out-neighbours); the printed A^T of Alg.1 l.37
 *     is only right for undirected graphs (R1).
 *   - no normalisation, no n/k extrapolation (Eq. 1-3); each occurrence of a
 *     source in the list counts.
 *
 * Errors: every function returns a tbc_status; nothing crosses the ABI as an exception.
 * On error the outputs are untouched (create: *out = NULL), nothing leaks, and
 * tbc_last_error() holds a thread-local detail message.
 *
 * Threading: a tbc_graph is not re-entrant (it owns one workspace); distinct graphs may
 * be used from distinct host threads.
 */
#ifndef TBC_H
#define TBC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tbc_graph tbc_graph; /* opaque; owns device memory on its device */

typedef enum {
    TBC_OK = 0,
    TBC_ERR_INVALID = 1,     /* bad argument or malformed graph (see tbc_last_error) */
    TBC_ERR_OOM = 2,         /* cudaMalloc failed */
    TBC_ERR_CUDA = 3,        /* any other CUDA runtime error (message in tbc_last_error) */
    TBC_ERR_UNSUPPORTED = 4  /* valid request this build does not implement */
} tbc_status;

/* engine: which SpMV formulation drives both stages */
enum {
    TBC_ENGINE_CSC = 0,  /* frontier-compacted push/pull over CSC (+CSR for directed graphs) */
    TBC_ENGINE_COOT = 1  /* scCOOC: edge-parallel over the transposed-COO arrays every level
                            (Alg. 2) */
};

/* create flags */
enum {
    TBC_FLAG_ONE_FORMAT = 1u << 0,  /* strict single format: a directed
                                       TBC_ENGINE_CSC graph keeps its CSC alone -- no CSR copy, no
                                       owner arrays (graph ~ 16 n + 4 m bytes: col_ptr, row_idx,
                                       degrees).  bc then runs the batched engine only: every forward
                                       level is a pull over in-edges (Alg.3's masked A^T f) and the
                                       backward pushes delta_u over in-edges with fp64 atomics;
                                       TBC_OPT_BATCH must stay 1.  No effect on undirected graphs. */
    TBC_FLAG_NO_VALIDATE = 1u << 1, /* skip host-side input validation (caller guarantees it) */
    TBC_FLAG_NO_REORDER = 1u << 2   /* keep the caller's vertex labels internally (default: relabel by
                                       decreasing degree when the degree distribution is skewed --
                                       max degree > 16 x mean -- so hubs share cache lines; flat
                                       graphs keep their labels; all inputs and outputs stay in the
                                       caller's labels either way) */
};

/* options for tbc_graph_set_option.  Every forward level is run as one of five passes, chosen
 * by a per-item cost model: push over the frontier list,
 * push over all stored entries (edge stream, the scCOOC form of Alg. 2), pull over the
 * survivors of the previous pull, pull over all stored entries, or a candidate scan followed
 * by a pull over the candidates; every backward level L as a pull over the out-edges of level
 * L (list pass or edge stream) or a push from level L+1 over its in-edges (list pass, fp64
 * atomics).  The options restrict or re-weight that choice. */
enum {
    TBC_OPT_DIRECTION = 1,   /* forward: 0 auto (default), 1 push only, 2 pull whenever possible (level >= 2) */
    TBC_OPT_BWD_DIRECTION = 2, /* backward: 0 auto (default), 1 pull over the out-edges of level L only,
                                  2 push from level L+1 over its in-edges whenever possible (list passes) */
    TBC_OPT_TRACE = 3,       /* index in the next calls' source lists whose per-level timeline is
                                recorded (-1 = off, default) */
    TBC_OPT_FORMAT = 4,      /* 0 auto (default), 1 list passes only, 2 edge streams only
                                (TBC_ENGINE_COOT always streams) */
    TBC_OPT_COST_LIST = 5,   /* cost model, picoseconds per item: list-pass item (default 12) */
    TBC_OPT_COST_STREAM = 6, /*   stream-pass stored entry (default 4) */
    TBC_OPT_COST_ATOMIC = 7, /*   push contribution (fp64 atomic) (default 18) */
    TBC_OPT_COST_VERTEX = 8, /*   vertex of a whole-graph owner pass (default 10) */
    TBC_OPT_COST_SCAN = 9,   /*   vertex of a candidate scan before a pull that follows a push (default 3) */
    TBC_OPT_COST_BPUSH = 10, /*   extra per in-edge of a backward push level over a list item (default 6) */
    TBC_OPT_PARTITIONS = 11, /* SM partitions (1..8, default 8): the source list is dealt round-robin
                                to this many disjoint groups of SMs, each running its sources with its
                                own workspace and partition-local barriers; the partial bc vectors
                                are summed in partition order at the end of the call (deterministic
                                for a given value).  Costs one workspace (~50 B/vertex + 8 B/edge/64)
                                per partition.  Per-source engine only. */
    TBC_OPT_BATCH = 12,      /* bc engine (TBC_ENGINE_CSC graphs):
                                -1 (default) auto: the first call with sources runs a level-width probe (a
                                   forward BFS from its first source by one CTA, stopped after 65536
                                   vertices; synchronises the stream once per graph) and picks 2 when
                                   the probe's vertices per level < TBC_OPT_NARROW_WIDTH, else 1;
                                 0 the per-source grid engine (k_bc);
                                 1 batched -- W sources per sweep (W = 32 or 64, TBC_OPT_BATCH_WIDTH), A^T
                                   times an n x W frontier block;
                                 2 narrow-level -- one source per CTA, CTA barriers between levels, as
                                   many sources at once as CTAs fit (20 B/vertex of workspace each).
                                tbc_bfs and TBC_ENGINE_COOT always use the per-source engine. */
    TBC_OPT_BATCH_PULL = 13, /* batched engine: a forward level is pulled (candidates' in-edges)
                                when the frontier's out-edges x this value > nnz, else pushed
                                (default 8; must be >= 0) */
    TBC_OPT_BATCH_WIDTH = 14, /* batched engine: sources per sweep, 32 (one per warp lane) or 64
                                (two per lane), or 0 (default, settled once per graph) = 64 up to 8 M
                                vertices, and above that for average degree >= 8 when the W = 64
                                workspace fits 85 % of the free memory, else 32 (measured, DESIGN.md
                                4.5); a W = 64 workspace that then fails to allocate falls back to 32.
                                Workspace per SM partition ~ 16 W B/vertex of (sigma, delta_u) rows
                                (8 W + the split accumulator with TBC_OPT_BATCH_INPLACE) +
                                TBC_OPT_BATCH_LIST x (12 + W/8) B/vertex of level lists + tile starts. */
    TBC_OPT_BATCH_PARTS = 16, /* batched engine: SM partitions (1..8, or 0 = auto, the default: 1 for
                                graphs whose sigma rows overflow 1 GiB with average degree >= 8 or
                                with average degree >= 64, else up to 4 (average degree >= 8) or 8
                                fitting 80 % of free memory); partition q runs
                                batches q, q + P, ... on its own SMs, workspace and barrier (one
                                workspace each); bc accumulates with fp64 atomics from all of them */
    TBC_OPT_BATCH_ORDER = 17, /* batched engine: 1 (default) cut the call's sources into batches after a
                                stable sort by 2-hop out-volume class, then out-degree (bc is a sum
                                over sources, so only the floating-point summation order changes),
                                0 in the given order */
    TBC_OPT_NARROW_WIDTH = 18, /* auto engine: probe vertices per level below which the narrow-level
                                engine runs (default 4096; setting it re-runs the probe next call) */
    TBC_OPT_BATCH_LIST = 19, /* batched engine: level-list entries allocated per vertex (1..64, default 2;
                                capped at W).  A sweep whose lists outgrow them is re-run as two half
                                sweeps (tbc_stats.list_overflows) and the next call doubles them (in
                                place, TBC_OPT_BATCH_INPLACE: likewise a sweep whose split-owner
                                accumulator is too small; the next call sizes it to the need). */
    TBC_OPT_NARROW_SLOTS = 22, /* narrow-level engine: sources run concurrently (one CTA each), 0 = auto
                                (default: as many CTAs as are resident, within 60 % of the free memory,
                                40 B/vertex each) */
    TBC_OPT_SIGMA = 21,      /* narrow-level engine: 0 (default) fp64 sigma, and a source whose sigma
                                leaves the fp64 range (inf; meshes: sigma = C(i+j, i) from a corner) is
                                re-run with extended-range sigma and delta_u (mantissa + int32
                                exponent, exact below 2^53 like fp64; tbc_stats.xr_sources); 1 always
                                extended range.  The other engines compute in fp64 only. */
    TBC_OPT_BATCH_INPLACE = 23, /* batched engine, two-format graphs: 1 the backward overwrites sigma with
                                delta_u in place (8 W B/vertex of rows instead of 16 W, plus a split-owner
                                accumulator sized to the largest level's need; one more grid barrier
                                per backward level: ~6 % slower on Kronecker 22/25), 0 separate delta_u
                                rows, -1 (default) auto: in place when the separate rows would not fit
                                85 % of the free device memory (settled once per graph) */
    TBC_OPT_STAGE = 20       /* measurement: 0 (default) forward + backward; 1 forward stage only --
                                the batched and narrow-level engines run Alg.1 l.11-28 and skip the
                                backward stage, leaving bc untouched (per-stage HBM traffic with ncu) */
};

/* counters accumulated on the device by every tbc_bc / tbc_bc_device / tbc_bfs call since
 * the last tbc_stats_reset; TEPS/roofline bookkeeping for the bench. */
typedef struct {
    int64_t sources;     /* sources processed */
    int64_t reached;     /* sum over sources of reached vertices (s included) */
    int64_t reached_edges; /* sum over sources of the out-edges of the reached vertices */
    int64_t fwd_edges;   /* stored entries examined by forward levels (push: frontier
                            out-edges, pull: candidate in-edges, coot: nnz per level) */
    int64_t bwd_edges;   /* stored entries examined by backward levels */
    int64_t levels;      /* forward levels run (incl. the final empty one) */
    int64_t pull_levels; /* forward levels run as pull */
    int64_t scans;       /* candidate scans (first pull level of a source) */
    int64_t max_depth;   /* deepest BFS height seen */
    int64_t list_peak;   /* batched engine: most level-list entries one batch used (sizing) */
    int64_t bad_sources; /* tbc_bc_device: out-of-range entries of d_sources that were skipped */
    int64_t batch_width; /* batched engine: sources per sweep of the latest call (0: none yet) */
    int64_t batch_parts; /* batched engine: SM partitions of the latest call */
    int64_t workspace_bytes; /* device bytes of the engine workspaces now allocated (included in
                                tbc_graph_info's device_bytes); not reset by tbc_stats_reset */
    int64_t engine;      /* engine of the latest bc call: 0 per source, 1 batched, 2 narrow-level, -1 none */
    int64_t list_overflows; /* batched engine: sweeps whose level lists outgrew the workspace and were
                               re-run as two half sweeps (the next call grows the lists) */
    int64_t probe_width; /* auto engine: the probe's vertices per level (0 before the probe) */
    int64_t xr_sources;  /* narrow-level engine: sources run with extended-range sigma (TBC_OPT_SIGMA) */
} tbc_stats;

/* Create a graph from the CSC of A (CP_A = col_ptr, row_A = row_idx, here 0-based).
 *   n       : number of vertices, 1 <= n < 2^31
 *   nnz     : col_ptr[n]; entries in row_idx
 *   col_ptr : host int64[n+1], col_ptr[0] = 0, non-decreasing, col_ptr[n] = nnz
 *   row_idx : host int32[nnz], rows in [0, n); any order within a column; duplicates ok
 *   directed: 0 = undirected (pattern must be symmetric; validated unless NO_VALIDATE;
 *             bc halved per P:180), 1 = directed
 *   engine  : TBC_ENGINE_CSC or TBC_ENGINE_COOT
 *   device  : CUDA device ordinal
 *   out     : receives the handle (NULL on error)
 * The host arrays are copied; the caller may free them on return.  The graph is
 * canonicalised on the device (sorted, deduplicated columns; CSR copy for directed graphs).
 * Errors: TBC_ERR_INVALID (arguments/malformed/asymmetric), TBC_ERR_OOM, TBC_ERR_CUDA. */
tbc_status tbc_graph_create_csc(int64_t n, int64_t nnz, const int64_t *col_ptr,
                                const int32_t *row_idx, int directed, int engine,
                                unsigned flags, int device, tbc_graph **out);

/* Create a graph from an edge list: edge k is src[k] -> dst[k], i.e. A(src,dst) = 1,
 * stored as row src[k] of column dst[k] (the COOC arrays row_A = src, col_A = dst).
 * Arguments and errors as tbc_graph_create_csc; nnz >= 0 entries, ids in [0, n). */
tbc_status tbc_graph_create_coo(int64_t n, int64_t nnz, const int32_t *src, const int32_t *dst,
                                int directed, int engine, unsigned flags, int device,
                                tbc_graph **out);

/* Betweenness centrality over a source list (Alg.1 l.6 generalised to a list).
 *   sources: host int32[k], each in [0, n) (validated; TBC_ERR_INVALID otherwise); k >= 0
 *   bc_out : host double[n], OVERWRITTEN with bc(v) = sum_{s in list} delta_s(v)
 *            (x 1/2 per source if undirected).  k = 0 gives all zeros.
 * Synchronous. */
tbc_status tbc_bc(tbc_graph *g, const int32_t *sources, int64_t k, double *bc_out);

/* Device-pointer variant for framework integration (PyTorch tensors, multi-GPU ranks).
 *   d_sources   : device int32[k] on the graph's device; out-of-range entries are skipped
 *                 and counted (not validated on the host)
 *   d_bc        : device double[n]; the result is ACCUMULATED into it (bc += ...)
 *   cuda_stream : cudaStream_t to run on (NULL = legacy default stream)
 * Asynchronous with respect to the host; errors of the launch itself are returned. */
tbc_status tbc_bc_device(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc,
                         void *cuda_stream);

/* Forward stage only (Alg.1 l.11-28) from one source, by the per-source engine.
 *   depth_out: host int32[n] or NULL; sigma_out: host double[n] or NULL.  Synchronous. */
tbc_status tbc_bfs(tbc_graph *g, int32_t source, int32_t *depth_out, double *sigma_out);

/* Forward stage (Alg.1 l.11-28) of the engine tbc_bc runs on this graph -- batched (W sources per
 * sweep, W as TBC_OPT_BATCH_WIDTH; sources cut into sweeps in the given order, not grouped) or
 * narrow-level (TBC_OPT_BATCH) -- for a list of sources.
 *   sources  : host int32[k], each in [0, n) (validated)
 *   depth_out: host int32[k * n]; depth_out[i * n + v] = depth of v from sources[i] (0 at the
 *              source, -1 unreachable)
 *   sigma_out: host double[k * n]; sigma_out[i * n + v] = number of shortest paths (0 unreachable)
 * Synchronous.  Device scratch of 12 k n bytes is kept for reuse until tbc_destroy.
 * TBC_ERR_UNSUPPORTED for TBC_ENGINE_COOT graphs and for TBC_OPT_BATCH = 0 (use tbc_bfs). */
tbc_status tbc_bfs_batch(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out,
                         double *sigma_out);

/* tbc_bfs_batch with sigma as mantissa and binary exponent, for sigma beyond the fp64 range
 * (NEXT-2): sigma = sigma_mant_out[i n + v] * 2^sigma_exp_out[i n + v], mantissa in [0.5, 1) or 0.
 * The narrow-level engine exports its extended-range values; the fp64 engines split fp64 sigma. */
tbc_status tbc_bfs_batch_ext(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out,
                             double *sigma_mant_out, int32_t *sigma_exp_out);

/* Graph properties after canonicalisation; any output pointer may be NULL.
 *   nnz = stored entries of A after deduplication; device_bytes = device memory owned now: the
 *   graph arrays plus every engine workspace allocated so far (they are sized at the first call). */
tbc_status tbc_graph_info(const tbc_graph *g, int64_t *n, int64_t *nnz, int *directed,
                          size_t *device_bytes);

/* Engine options (TBC_OPT_*); TBC_ERR_INVALID for an unknown key or value. */
tbc_status tbc_graph_set_option(tbc_graph *g, int key, double value);

/* Read (synchronises the graph's device) / reset the accumulated counters. */
tbc_status tbc_stats_get(tbc_graph *g, tbc_stats *out);
tbc_status tbc_stats_reset(tbc_graph *g);

/* Per-level timeline of the traced source (TBC_OPT_TRACE) of the last call that reached it:
 *   out  : host int64[8 * cap]; entry i = {globaltimer ns, kind, level, N, E, a, b, 0} with
 *          kind 0 init, 1 candidate scan, 2 push level, 3 pull edge pass, 4 backward edge pass,
 *          5 owner pass (pull mask / backward delta); N/E = list size / out-edges produced
 *          (fwd) or processed (bwd),
 *          a/b = owners / edges the level traversed.  Timestamps are taken after each grid
 *          barrier, so consecutive differences are level durations.
 *   count: receives the number of entries recorded (<= 65536).  Synchronises the device. */
tbc_status tbc_trace_get(tbc_graph *g, int64_t *out, int64_t cap, int64_t *count);

/* Diagnostic region profile (libraries built with -DTBC_PROF only; TBC_ERR_UNSUPPORTED otherwise):
 * warp-cycles spent per code region of the persistent kernel since the last call, summed over
 * warps (lane 0 clock64 deltas).  out: host uint64[cap]; count receives 32.  Entry 0 grid
 * barriers, 1 + 4*mode + {window, index issue, gather/op, tail} for list passes (mode 0 push,
 * 1 pull, 2 backward pull, 3 backward push), 17 + mode stream passes, 20 pull owner pass,
 * 21 candidate scan, 22 backward owner pass, 23 the rest.  Reading resets the counters. */
tbc_status tbc_profile_get(tbc_graph *g, uint64_t *out, int64_t cap, int64_t *count);

/* Free everything the handle owns.  NULL is a no-op. */
tbc_status tbc_destroy(tbc_graph *g);

const char *tbc_status_string(tbc_status s);
const char *tbc_last_error(void); /* thread-local; "" if none */

#ifdef __cplusplus
}
#endif
#endif /* TBC_H */
