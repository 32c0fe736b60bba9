// tbc_internal.cuh -- shared definitions of libturbobc (graph object, workspace, params).
// Product code: shares nothing with oracle/.
#pragma once
#include <cstdint>
#include <cstddef>
#include <cuda_runtime.h>
#include "tbc.h"

namespace tbc {

#ifndef TBC_BLOCK
#define TBC_BLOCK 1024
#endif
#ifndef TBC_LANE_ITEMS
#define TBC_LANE_ITEMS 4
#endif
constexpr int kBlock = TBC_BLOCK;  // threads per CTA of the persistent kernel (one CTA per SM)
constexpr int64_t kTraceCap = 65536; // trace entries (one per barrier of the traced source)

// Device-side counters of one graph; all fields are touched by the persistent kernel only.
struct Ctrs {
    unsigned long long list;      // packed (count << ebits) | edge_sum of the BFS-order list
    unsigned long long cand[2];   // packed counters of the two pull-candidate buffers
    unsigned long long ilist;     // packed (count << ebits) | in-edge sum of the in-degree list (directed)
    unsigned int bar_count;       // grid barrier arrival counter
    unsigned int bar_gen;         // grid barrier generation
    // {list, ilist, cand[0], cand[1]} as the last arriver of the latest barrier saw them: CTAs
    // read the level sizes from here, never from the live counters, which a faster CTA may
    // already be appending to (next push level) or zeroing (candidate reset)
    unsigned long long snap[4];
    unsigned long long bad_sources;
    unsigned long long dyn[2];    // batched engine: dynamic tile counters of consecutive edge passes
    unsigned int ovf;             // batched engine: a level list outgrew the workspace (re-run in halves)
    unsigned long long ovf_total; // batched engine: such re-runs since the workspace was allocated
    unsigned long long salloc[2]; // batched engine (in place): split-accumulator allocation, by level parity
    unsigned long long split_need;// batched engine (in place): most split lanes of one level seen (sizes sacc)
    unsigned long long trace_n;   // entries written to the trace buffer
    // accumulated statistics (tbc_stats)
    long long st_sources, st_reached, st_reached_edges, st_fwd_edges, st_bwd_edges, st_levels, st_pull_levels,
        st_scans, st_max_depth, st_list_peak, st_overflows, st_xr_sources;
    unsigned long long prof[32];  // TBC_PROF builds: warp-cycles per code region (gctr only)
};

struct Params {
    int64_t n, m;
    const int64_t *__restrict__ in_ptr;   // CSC: in-neighbours (column v = rows u with u->v)
    const int32_t *__restrict__ in_idx;
    const int64_t *__restrict__ out_ptr;  // CSR: out-neighbours (== in_* when undirected)
    const int32_t *__restrict__ out_idx;
    const int2 *__restrict__ deg2;        // {out-degree, in-degree}
    int32_t *depth;                       // -1 unvisited
    double *sigma;                        // path counts, 0 when not on the current BFS
    double *du;                           // signed delta_u, sign = parity of the level
    double *gacc;                         // per-owner sums handed from edge to owner pass (0 between)
    int32_t *list_v;                      // BFS-order vertex list (levels concatenated)
    uint32_t *list_pre;                   // exclusive out-degree prefix along list_v (< m < 2^32)
    uint32_t *list_beg;                   // out_ptr[v] of each list entry (written at append)
    int32_t *tiles;                       // per level: owner index starting each tile
    // in-degree list (directed CSC engine): the same vertices per level as list_*, keyed by
    // in-degree (prefix over in_ptr) -- the owners of the backward push pass; == list_* otherwise
    int32_t *ilist_v;
    uint32_t *ilist_pre;
    uint32_t *ilist_beg;
    int32_t *itiles;
    int in_list;                          // 1: ilist_* is a separate list appended beside list_*
    int64_t n_scan;                       // vertices [0, n_scan) can have in-edges (degree-sorted labels)
    int64_t n_in;                         // vertices with in-degree > 0
    int32_t *cand_v[2];                   // pull candidate buffers
    uint32_t *cand_pre[2];
    uint32_t *cand_beg[2];
    int32_t *cand_tiles[2];
    int64_t *lvl;                         // per level: p0, N, e0, E, tile_base, ie0, IE, itile_base
    Ctrs *ctr;                            // this partition's counters and barrier
    Ctrs *gctr;                           // shared: full-grid barrier, trace counter
    int cta_base;                         // first CTA of this SM partition
    double *bc;                           // indexed by caller labels (a partition's partial bc
                                          // when the launch has several partitions)
    const int32_t *sources;               // caller labels
    const int32_t *__restrict__ perm;     // caller -> internal label (nullptr: identity)
    const int32_t *__restrict__ inv;      // internal -> caller label
    int64_t k;
    double bc_scale;                      // 0.5 undirected, 1 directed
    int ebits;                            // low bits of packed counters hold edge sums
    int bfs_only;                         // forward stage only (tbc_bfs)
    int directed;
    int coot;                             // TBC_ENGINE_COOT: edge-stream passes only
    int dir_mode;                         // 0 auto, 1 push only, 2 pull whenever possible
    int bwd_mode;                         // 0 auto, 1 pull only, 2 push whenever possible
    int64_t *trace;                       // per-level timeline of one source (8 int64 per entry)
    int64_t trace_cap, trace_src;
    // edge-stream passes (the scCOOC form of Alg. 2): owner of every stored entry
    const int32_t *__restrict__ in_col;   // column of each CSC entry (sorted)
    const int32_t *__restrict__ out_row;  // row of each CSR entry (sorted); nullptr for COO^T directed
    int fmt_mode;                         // 0 auto, 1 list passes only, 2 stream passes only
    double c_list, c_stream, c_atom, c_vert;  // per-item cost model (ps) for the per-level choice
    double c_scan, c_bpush;
};

}  // namespace tbc

namespace tbc {
// per-SM-partition workspace: each partition runs its own sources with these arrays
struct Workspace {
    int32_t *depth = nullptr;
    double *sigma = nullptr, *du = nullptr, *gacc = nullptr;
    int32_t *list_v = nullptr;
    uint32_t *list_pre = nullptr;
    uint32_t *list_beg = nullptr;
    int32_t *tiles = nullptr;
    int32_t *ilist_v = nullptr;   // in-degree list (directed CSC engine only)
    uint32_t *ilist_pre = nullptr;
    uint32_t *ilist_beg = nullptr;
    int32_t *itiles = nullptr;
    int32_t *cand_v[2] = {nullptr, nullptr};
    uint32_t *cand_pre[2] = {nullptr, nullptr};
    uint32_t *cand_beg[2] = {nullptr, nullptr};
    int32_t *cand_tiles[2] = {nullptr, nullptr};
    int64_t *lvl = nullptr;
    Ctrs *ctr = nullptr;
    double *bc_part = nullptr;    // partial bc of this partition (zero between calls)
};
constexpr int kMaxPartitions = 8;

// device buffers of the batched engine's source grouping (grow-only)
struct BatchOrder {
    void *keys = nullptr;   // 2 x cap uint32 keys + 2 x cap int32 values
    void *temp = nullptr;   // cub temp storage
    int64_t cap = 0;
    size_t temp_bytes = 0;
};

// workspace of the batched engine (tbc_batch.cu): W = 32 or 64 sources per sweep, lane l of a
// warp holding sources l (and l + 32); masks are W-bit words (W / 32 uint32 words)
struct BatchWorkspace {
    int width = 0;               // W the workspace was sized for
    size_t bytes = 0;
    double *sig = nullptr;       // [n][W] sigma of (vertex, source)
    double *du = nullptr;        // [n][W] delta_u accumulators (strict one-format graphs only; else the
                                 // backward overwrites sigma with delta_u in place, see k_bcb)
    double *sacc = nullptr;      // [2][sacc_cap] split owners' partial sums, by level parity (in place)
    int64_t *scnt = nullptr;     // [n + 2] split lanes per level of the current sweep (in place)
    int64_t sacc_cap = 0;
    uint32_t *vis = nullptr;     // [n] sources that have reached the vertex (W-bit words)
    uint32_t *fr[2] = {nullptr, nullptr};  // [n] dense level masks, by level parity (W-bit words)
    int32_t *list_v = nullptr;   // level lists (levels concatenated), capacity list_cap
    uint32_t *list_pre = nullptr;  // out-degree prefix, relative to the level
    uint32_t *list_beg = nullptr;  // out_ptr of the entry
    uint32_t *list_m = nullptr;    // sources on this level (W-bit words)
    int32_t *tiles = nullptr;      // per level: owner starting each warp tile, capacity tiles_cap
    int32_t *cand_v = nullptr;     // pull candidates (in-degree prefix)
    uint32_t *cand_pre = nullptr;
    uint32_t *cand_beg = nullptr;
    int32_t *cand_tiles = nullptr;
    int64_t *lvl = nullptr;        // per level: p0, N, E, tile base
    Ctrs *ctr = nullptr;
    int64_t list_cap = 0, tiles_cap = 0, cand_tiles_cap = 0;
    bool ready = false;
};
// workspace of the narrow-level engine (tbc_single.cu): one slot of per-vertex arrays per
// concurrently running source (one per resident CTA)
// per (slot, vertex) state of the narrow-level engine: one 32-byte DRAM sector
struct __align__(32) VRec {
    double sd;     // sigma (forward), then delta_u (backward); 0 between sources (extended range:
                   // the mantissa)
    int32_t depth; // -1 between sources
    int32_t sexp;  // extended range (NEXT-2): binary exponent of sd (value = sd * 2^sexp), else 0
    double bc;     // the slot's partial bc, summed into the caller's bc after each call
    double pad2;
};
static_assert(sizeof(VRec) == 32, "one sector per vertex record");
struct SingleWorkspace {
    int slots = 0;
    size_t bytes = 0;
    VRec *rec = nullptr;         // [slots][n]
    int32_t *order = nullptr;    // [slots][n]
    int32_t *lvl = nullptr;      // [slots][n + 2]
    Ctrs *ctr = nullptr;
    int64_t *probe_out = nullptr;
};
}  // namespace tbc

struct tbc_graph {
    int device = 0;
    int64_t n = 0, m = 0;
    int directed = 0;
    int engine = 0;
    unsigned flags = 0;
    // graph (device)
    int64_t *in_ptr = nullptr;
    int32_t *in_idx = nullptr;
    int64_t *out_ptr = nullptr;  // aliases in_ptr when undirected
    int32_t *out_idx = nullptr;
    int2 *deg2 = nullptr;
    int32_t *perm = nullptr;     // caller label -> internal label (degree-descending); nullptr = identity
    int32_t *inv = nullptr;      // internal label -> caller label
    int32_t *in_col = nullptr;   // column (owner) of every CSC entry: with in_idx, the COOC arrays
    int32_t *out_row = nullptr;  // row (owner) of every CSR entry (== in_col when undirected)
    // workspaces (device), one per SM partition; ws_count allocated so far
    tbc::Workspace ws[tbc::kMaxPartitions];
    int ws_count = 0;
    size_t ws_bytes = 0;          // device bytes of the per-source engine's workspaces
    int nparts = 8;               // TBC_OPT_PARTITIONS
    tbc::Ctrs *gctr = nullptr;    // shared counters: full-grid barrier, trace
    int64_t n_scan = 0, n_in = 0;
    double *bc_tmp = nullptr;
    int32_t *src_tmp = nullptr;
    int64_t src_cap = 0;
    // launch
    int grid = 0;
    int ebits = 38;
    int dir_mode = 0;
    int bwd_mode = 0;
    int fmt_mode = 0;
    double c_list = 12.0, c_stream = 4.0, c_atom = 18.0, c_vert = 10.0, c_scan = 3.0, c_bpush = 6.0;
    int sigma_mode = 0;           // TBC_OPT_SIGMA: 0 fp64 + extended re-run on overflow, 1 extended range
    int stage = 0;                // TBC_OPT_STAGE: 0 forward + backward, 1 forward only (measurement)
    int batch = -1;               // TBC_OPT_BATCH: -1 auto, 0 per source, 1 batched, 2 narrow-level
    int narrow = -1;              // auto choice, settled by the first call's probe: 1 narrow-level engine
    int narrow_slots = 0;         // TBC_OPT_NARROW_SLOTS: concurrent sources of the narrow engine (0 auto)
    double narrow_width = 4096.0; // TBC_OPT_NARROW_WIDTH: probe's vertices per level below which auto is narrow
    double probe_width = 0.0;     // the probe's measured vertices per level (tbc_stats)
    int last_mode = -1;           // engine of the latest bc call (0 per source, 1 batched, 2 narrow-level)
    tbc::SingleWorkspace sws;
    int batch_width = 0;          // TBC_OPT_BATCH_WIDTH: sources per sweep (32 or 64; 0 auto)
    double batch_pull = 8.0;      // TBC_OPT_BATCH_PULL: pull when frontier out-edges x this > m
    tbc::BatchWorkspace bws[tbc::kMaxPartitions];  // one per SM partition of the batched engine
    int batch_parts = 0;          // TBC_OPT_BATCH_PARTS: SM partitions of the batched engine (0 auto)
    int batch_order = 1;          // TBC_OPT_BATCH_ORDER: group the sources by out-degree into batches
    tbc::BatchOrder border;
    int bgrid = 0;
    int auto_width = 0;           // batch width the auto rule settled on for this graph (0: not yet)
    int last_width = 0, last_parts = 0;  // of the latest batched call (tbc_stats)
    int64_t blist_factor = 2;     // batched engine: level-list entries per vertex allocated (grows x2)
    unsigned long long *h_bovf = nullptr;  // pinned [2][kMaxPartitions]: per-partition list-overflow totals
                                           // and split-accumulator needs (largest level) after the latest call
    int binplace = -1;            // TBC_OPT_BATCH_INPLACE (-1 auto, 0 off, 1 on)
    int binplace_eff = -1;        // auto: settled at the first allocation (0 / 1)
    int64_t bsacc_cap = 0;        // batched engine (in place): split-accumulator values per level parity
                                  // (0 = initial W n / 16; grows to the largest level seen x 5/4)
    unsigned long long bovf_seen[tbc::kMaxPartitions] = {};
    tbc::Ctrs retired = {};       // statistics of freed batched workspaces (kept for tbc_stats)
    int32_t *bfs_depth = nullptr; // tbc_bfs_batch device outputs (grow-only)
    double *bfs_sigma = nullptr;
    int32_t *bfs_sexp = nullptr;  // tbc_bfs_batch_ext: sigma exponents
    int64_t bfs_cap = 0;          // elements of bfs_depth / bfs_sigma
    int64_t *trace = nullptr;     // device, 8 * kTraceCap int64
    int64_t trace_src = -1;       // index in the next call's source list to trace (-1: off)
    cudaStream_t stream = nullptr;  // internal stream for the synchronous host API
    size_t device_bytes = 0;
};

namespace tbc {
// error plumbing (tbc_api.cu)
tbc_status set_error(tbc_status s, const char *fmt, ...);
tbc_status cuda_error(cudaError_t e, const char *what);
// engine entry points (tbc_engine.cu)
tbc_status engine_setup(tbc_graph *g);
tbc_status engine_workspaces(tbc_graph *g, int count);  // allocate partitions [ws_count, count)
void engine_free(tbc_graph *g);                          // workspaces + shared counters
tbc_status engine_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc,
                      cudaStream_t stream, int bfs_only);
// batched engine (tbc_batch.cu)
tbc_status batch_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                     int32_t *bfs_depth = nullptr, double *bfs_sigma = nullptr);
int batch_width(const tbc_graph *g);  // sources per sweep the next batched call uses
// narrow-level engine (tbc_single.cu)
tbc_status single_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                      int32_t *bfs_depth = nullptr, double *bfs_sigma = nullptr, int32_t *bfs_sexp = nullptr);
tbc_status single_probe(tbc_graph *g, const int32_t *d_sources, cudaStream_t stream, double *width);
void single_free(tbc_graph *g);
// engine the next bc call on these sources runs (auto: probes once per graph): 0 per source,
// 1 batched, 2 narrow-level
tbc_status engine_choose(tbc_graph *g, const int32_t *d_sources, int64_t k, cudaStream_t stream, int *mode);
void batch_free(tbc_graph *g);
void batch_free_one(tbc_graph *g, int q);
}  // namespace tbc
