// tbc_engine.cu -- the per-source hot path of TurboBC (Algorithm 1) as one
// persistent, cooperative sm_100a kernel per tbc_bc call.
//
//   forward  (Alg.1 l.11-28):  level-synchronous masked SpMV.  Each level is either
//            PUSH  -- frontier (level d-1 list) scatters sigma along out-edges (CSR), claiming
//                     undiscovered targets with a CAS on depth (K1' + K2 of DESIGN.md), or
//            PULL  -- every still-undiscovered candidate sums sigma over in-edges (CSC) from
//                     the frontier: exactly the masked f_t = A^T f of l.19-22 / Alg.3.
//            Direction is chosen per level from frontier out-edges vs candidate in-edges.
//   backward (Alg.1 l.29-47): for L = D..1, owners on level L sum delta_u of their
//            out-neighbours on level L+1 (A delta_u, reading R1), delta = sigma * sum,
//            bc += delta (x 1/2 undirected), delta_u = (1+delta)/sigma (l.35).
//
// Every level is one merge-path pass over (owner list, out/in-edges): the diagonal of
// (owner end items + edges) is cut into warp tiles of kWT items, so a 600k-edge hub and a million
// degree-1 vertices cost the same per tile.  Tile start owners are written by the producers
// of the list at append time (warp-aggregated append, see warp_append), so no search is
// needed.  Levels are separated by a grid barrier inside the kernel: no host round trip per
// level (the paper's per-level host loop), one launch per call for all sources.
#include <cooperative_groups.h>
#include <cstdio>

#include "tbc_internal.cuh"

namespace tbc {
namespace {

constexpr unsigned FULL = 0xffffffffu;
enum { MODE_PUSH = 0, MODE_PULL = 1, MODE_BWD = 2 };

constexpr int kLaneItems = 8;              // items per lane per warp tile
constexpr int kWT = 32 * kLaneItems;        // diagonal items per warp tile
constexpr int kWarpsPerBlock = kBlock / 32;

struct __align__(16) WarpSmem {
    int64_t beg[kWT + 1];    // adjacency position of the owner's first in-tile edge
    double val[kWT + 1];     // PUSH: owner sigma; PULL/BWD: owner partial sum
    int32_t first[kWT + 2];  // slot of the owner's first in-tile edge (+ sentinel = ne)
    int32_t deg[kWT + 1];    // owner degree in the traversed direction
    int32_t own[kWT];        // owner (window index) of each edge slot
    int32_t start0;          // owner 0 begins inside the tile
};

constexpr size_t kSmemBytes = sizeof(WarpSmem) * kWarpsPerBlock;

// ------------------------------------------------------------------ memory-model helpers

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// streaming read of graph indices: read-only for the whole kernel, L1 no-allocate, L2 evict-first
__device__ __forceinline__ int ld_stream(const int32_t *ptr, uint64_t pol) {
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(ptr), "l"(pol));
    return v;
}

__device__ __forceinline__ void fence_acq_rel() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long *p) {
    return *(volatile const unsigned long long *)p;
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

constexpr unsigned long long kWatchdogNs = 20ull * 1000 * 1000 * 1000;  // 20 s at one barrier

// Grid-wide barrier for a cooperative (co-resident) grid.  Sense by generation counter.
__device__ __forceinline__ void grid_sync(Ctrs *c, unsigned &gen) {
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned g0 = gen;
        __threadfence();
        unsigned arrived = atomicAdd(&c->bar_count, 1u);
        if (arrived == gridDim.x - 1) {
            c->bar_count = 0;
            __threadfence();
            atomicExch(&c->bar_gen, g0 + 1);
        } else {
            const unsigned long long t0 = globaltimer_ns();
            while (ld_acquire(&c->bar_gen) == g0) {
                __nanosleep(32);
                if (globaltimer_ns() - t0 > kWatchdogNs) __trap();  // never hang the GPU
            }
        }
        __threadfence();  // acquire side; also invalidates this SM's L1 (CCTL.IVALL)
    }
    gen += 1;
    __syncthreads();
}

// ------------------------------------------------------------------ warp-aggregated append

// Append the lanes with pred to a list (v, exclusive degree prefix) through ONE packed 64-bit
// atomic per warp: (count << ebits) | degree_sum.  Because count and prefix are reserved
// together, list order and prefix order agree, and each appended owner knows its merge-path
// diagonal span [k0, k0+deg] inside its level, so it writes the start owner of every tile
// whose first diagonal lies in that span.  All 32 lanes must call this.
__device__ __forceinline__ void warp_append(bool pred, int32_t v, int64_t deg, unsigned long long *ctr,
                                            int ebits, int32_t *lv, int64_t *lpre, int32_t *tiles,
                                            int64_t p0, int64_t e0) {
    unsigned mask = __ballot_sync(FULL, pred);
    if (!mask) return;
    const int lane = threadIdx.x & 31;
    int64_t dg = pred ? deg : 0;
    int64_t inc = dg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int64_t t = __shfl_up_sync(FULL, inc, o);
        if (lane >= o) inc += t;
    }
    int64_t tot = __shfl_sync(FULL, inc, 31);
    unsigned long long old = 0;
    if (lane == 0)
        old = atomicAdd(ctr, ((unsigned long long)__popc(mask) << ebits) + (unsigned long long)tot);
    old = __shfl_sync(FULL, old, 0);
    if (pred) {
        int64_t p = (int64_t)(old >> ebits) + __popc(mask & ((1u << lane) - 1u));
        int64_t e = (int64_t)(old & ((1ull << ebits) - 1ull)) + inc - dg;
        lv[p] = v;
        lpre[p] = e;
        int64_t k0 = (e - e0) + (p - p0);
        int64_t k1 = k0 + dg;
        for (int64_t i = (k0 + kWT - 1) / kWT; i <= k1 / kWT; ++i) tiles[i] = (int32_t)(p - p0);
    }
}

// Warp-aggregated counter add (one atomic per warp); all 32 lanes must call this.
__device__ __forceinline__ void warp_add(unsigned long long val, unsigned long long *ctr) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) val += __shfl_xor_sync(FULL, val, o);
    if ((threadIdx.x & 31) == 0 && val) atomicAdd(ctr, val);
}

// ------------------------------------------------------------------ level descriptors

struct Level {
    int64_t p0, N, e0, E, tbase;
};

struct AppendTarget {
    unsigned long long *ctr;
    int32_t *v;
    int64_t *pre;
    int32_t *tiles;  // already offset to this level's tile base
    int64_t p0, e0;  // level start within the list (list position, edge prefix)
};

__device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

__device__ __forceinline__ double atomic_exch_d(double *p, double v) {
    unsigned long long r = atomicExch((unsigned long long *)p, __double_as_longlong(v));
    return __longlong_as_double(r);
}

// ------------------------------------------------------------------ merge-path level pass
//
// One WARP processes one tile of kWT diagonal items (owner end items + edges) with no block
// barrier: tiles are assigned round-robin to the grid's warps (every tile holds the same number
// of items, so the static assignment is balanced), the owner window lives in the warp's slice
// of shared memory, each lane keeps kLaneItems index loads and kLaneItems gathers in flight.
//
// Owners: ov[0..N) with exclusive degree prefix opre[] (minus e0), tile starts otiles[].
// adj_ptr/adj_idx: the traversed adjacency (CSR out-edges for PUSH/BWD, CSC in-edges for PULL).
// d: the level being discovered (push/pull), or the owners' level L (bwd).
// NOTE: ov/opre/otiles are written earlier in this same kernel (previous phases): they must
// NOT be declared __restrict__ const, or the compiler may read them through the
// non-coherent (ld.global.nc) path and see stale lines.
template <int MODE>
__device__ __forceinline__ void level_pass(const Params &P, WarpSmem &ws, const int32_t *ov,
                                           const int64_t *opre, const int32_t *otiles, int64_t N, int64_t E,
                                           int64_t e0, const int64_t *__restrict__ adj_ptr,
                                           const int32_t *__restrict__ adj_idx, int d, int64_t gwarp,
                                           int64_t nwarps, AppendTarget lvl_out, AppendTarget cand_out) {
    const int lane = threadIdx.x & 31;
    const int64_t K = N + E;
    const int64_t ntiles = ceil_div(K, kWT);
    const uint64_t pol_stream = policy_evict_first();
    for (int64_t tile = gwarp; tile < ntiles; tile += nwarps) {
        const int64_t ks = tile * kWT;
        const int64_t ke = min(ks + (int64_t)kWT, K);
        const int64_t ps = otiles[tile];
        const int64_t pe = (tile + 1 < ntiles) ? (int64_t)otiles[tile + 1] : N;
        const int64_t es = ks - ps, ee = ke - pe;
        const int nwin = (int)(min(pe, N - 1) - ps + 1);
        const int ne = (int)(ee - es);

        // ---- owner window: slot of the first in-tile edge, adjacency position of that edge
        for (int j = lane; j < nwin; j += 32) {
            const int32_t v = ov[ps + j];
            const int64_t pre = opre[ps + j] - e0;
            const int64_t b = adj_ptr[v];
            const int64_t deg = adj_ptr[v + 1] - b;
            const int64_t f = max(pre, es);
            ws.first[j] = (int32_t)(f - es);
            ws.beg[j] = b + (f - pre);
            ws.deg[j] = (int32_t)deg;
            if (MODE == MODE_PUSH) ws.val[j] = P.sigma[v];
            else ws.val[j] = 0.0;
            if (j == 0) ws.start0 = (pre >= es) ? 1 : 0;  // owner 0 begins inside this tile
        }
        if (lane == 0) ws.first[nwin] = ne;
        for (int sl = lane; sl < ne; sl += 32) ws.own[sl] = -1;
        __syncwarp();
        for (int j = lane; j < nwin; j += 32)
            if (ws.first[j] < ws.first[j + 1]) ws.own[ws.first[j]] = j;
        __syncwarp();
        // inclusive running max over own[0..ne): lane l scans slots [l*kLaneItems, +kLaneItems)
        {
            int loc[kLaneItems];
            int run = -1;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                const int sl = lane * kLaneItems + i;
                run = max(run, sl < ne ? ws.own[sl] : -1);
                loc[i] = run;
            }
            int incl = run;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(FULL, incl, o);
                if (lane >= o) incl = max(incl, t);
            }
            int prev = __shfl_up_sync(FULL, incl, 1);
            if (lane == 0) prev = -1;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                const int sl = lane * kLaneItems + i;
                if (sl < ne) ws.own[sl] = max(prev, loc[i]);
            }
        }
        __syncwarp();

        // ---- edges: slot = i*32 + lane (consecutive lanes -> consecutive adjacency entries)
        int xs[kLaneItems];
        int js[kLaneItems];
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            const int sl = i * 32 + lane;
            js[i] = -1;
            xs[i] = 0;
            if (sl < ne) {
                const int j = ws.own[sl];
                js[i] = j;
                xs[i] = ld_stream(adj_idx + ws.beg[j] + (sl - ws.first[j]), pol_stream);
            }
        }
        if (MODE == MODE_PUSH) {
            // masked scatter f_t(x) += f(u) for undiscovered x (Alg.1 l.19-25 as a push)
            int dxs[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) dxs[i] = js[i] >= 0 ? P.depth[xs[i]] : -2;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                bool claim = false;
                if (dxs[i] == -1) {
                    const int old = atomicCAS(&P.depth[xs[i]], -1, d);
                    claim = (old == -1);
                    dxs[i] = claim ? d : old;
                }
                if (dxs[i] == d) atomicAdd(&P.sigma[xs[i]], ws.val[js[i]]);
                if (__any_sync(FULL, claim)) {
                    int2 dg = make_int2(0, 0);
                    if (claim) {
                        P.du[xs[i]] = 0.0;
                        dg = P.deg2[xs[i]];
                    }
                    warp_append(claim, xs[i], dg.x, lvl_out.ctr, P.ebits, lvl_out.v, lvl_out.pre, lvl_out.tiles,
                                lvl_out.p0, lvl_out.e0);
                    warp_add((unsigned long long)dg.y, &P.ctr->indeg_vis);  // visited in-edge mass
                }
            }
        } else {
            double vals[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                vals[i] = 0.0;
                if (js[i] >= 0) {
                    if (MODE == MODE_PULL) {
                        // f_t(w) = sum over in-neighbours x on level d-1 of sigma(x)  (Alg.3 l.9-11)
                        if (P.depth[xs[i]] == d - 1) vals[i] = P.sigma[xs[i]];
                    } else {
                        // (A delta_u)(v): out-neighbour x on level d+1; the level parity is the sign
                        // of the stored delta_u, so concurrent same-level writes are rejected.
                        const double u = P.du[xs[i]];
                        const double want = ((d + 1) & 1) ? -u : u;
                        vals[i] = want > 0.0 ? want : 0.0;
                    }
                }
            }
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                // segmented (by owner) warp reduction; owners are non-decreasing across lanes
                double val = vals[i];
                const int ow = js[i];
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const double v2 = __shfl_down_sync(FULL, val, o);
                    const int o2 = __shfl_down_sync(FULL, ow, o);
                    if (lane + o < 32 && o2 == ow) val += v2;
                }
                const int up = __shfl_up_sync(FULL, ow, 1);
                if ((lane == 0 || up != ow) && ow >= 0 && val != 0.0) ws.val[ow] += val;
                __syncwarp();
            }

            // ---- owner finalisation (warp-uniform loop: appends are warp collectives)
            for (int base = 0; base < nwin; base += 32) {
                const int j = base + lane;
                bool fin = false;
                double total = 0.0;
                int32_t v = 0;
                if (j < nwin) {
                    v = ov[ps + j];
                    const bool end_in = ps + j < pe;
                    const bool start_in = j > 0 || ws.start0;
                    if (end_in && start_in) {
                        fin = true;
                        total = ws.val[j];
                    } else {
                        // owner split across tiles: partial sums meet in gacc[v]; the tile that
                        // completes the item count (deg + 1) finalises and resets the slots
                        const int c = (ws.first[j + 1] - ws.first[j]) + (end_in ? 1 : 0);
                        if (c > 0) {
                            if (ws.val[j] != 0.0) atomicAdd(&P.gacc[v], ws.val[j]);
                            fence_acq_rel();
                            const int old = atomicAdd(&P.gcnt[v], c);
                            if (old + c == ws.deg[j] + 1) {
                                fence_acq_rel();
                                total = atomic_exch_d(&P.gacc[v], 0.0);
                                P.gcnt[v] = 0;
                                fin = true;
                            }
                        }
                    }
                }
                if (MODE == MODE_PULL) {
                    // mask of Alg.1 l.20-25 / Alg.3 l.12-13: discovered iff the sum is non-zero
                    const bool disc = fin && total > 0.0;
                    const bool keep = fin && !(total > 0.0);
                    int2 dg = make_int2(0, 0);
                    if (disc) {
                        P.depth[v] = d;
                        P.sigma[v] = total;
                        P.du[v] = 0.0;
                        dg = P.deg2[v];
                    }
                    warp_append(disc, v, dg.x, lvl_out.ctr, P.ebits, lvl_out.v, lvl_out.pre, lvl_out.tiles,
                                lvl_out.p0, lvl_out.e0);
                    warp_add((unsigned long long)dg.y, &P.ctr->indeg_vis);
                    warp_append(keep, v, keep ? (int64_t)ws.deg[j] : 0, cand_out.ctr, P.ebits, cand_out.v,
                                cand_out.pre, cand_out.tiles, cand_out.p0, cand_out.e0);
                } else if (fin) {
                    // Alg.1 l.38-39 (delta = sigma * A delta_u), l.45 + P:180, then l.35 for level d
                    const double sg = P.sigma[v];
                    const double delta = sg * total;
                    P.bc[v] += delta * P.bc_scale;
                    const double dun = (1.0 + delta) / sg;
                    P.du[v] = (d & 1) ? -dun : dun;
                    P.sigma[v] = 0.0;
                    P.depth[v] = -1;
                }
            }
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------ the persistent kernel

__global__ void __launch_bounds__(kBlock, 3) k_bc(Params P) {
    extern __shared__ __align__(16) unsigned char dyn_smem[];
    WarpSmem *smem = reinterpret_cast<WarpSmem *>(dyn_smem);
    WarpSmem &ws = smem[threadIdx.x >> 5];
    const int64_t nwarps = (int64_t)gridDim.x * kWarpsPerBlock;
    const int64_t gwarp = (int64_t)blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    const int tid = threadIdx.x;
    const bool cta0 = blockIdx.x == 0;
    const int64_t nthreads = (int64_t)gridDim.x * kBlock;
    const int64_t gtid = (int64_t)blockIdx.x * kBlock + tid;
    Ctrs *C = P.ctr;
    // barrier generation: only thread 0 uses it (the first barrier cannot complete before
    // every CTA has read the current value, so reading it here is race-free)
    unsigned gen = (tid == 0) ? ld_acquire(&C->bar_gen) : 0u;
    const unsigned long long emask = (1ull << P.ebits) - 1ull;
    int32_t prev_s = -1;

    for (int64_t si = 0; si < P.k; ++si) {
        const int32_t s = P.sources[si];
        if (s < 0 || s >= P.n) {
            if (cta0 && tid == 0) atomicAdd(&C->bad_sources, 1ull);
            continue;
        }
        // ---------------- init (Alg.1 l.7-10, l.15-18): depth(s)=0, sigma(s)=1, frontier={s}
        const int64_t dego = P.deg2[s].x;
        if (cta0) {
            if (tid == 0) {
                if (prev_s >= 0) {
                    P.depth[prev_s] = -1;
                    P.sigma[prev_s] = 0.0;
                }
                P.depth[s] = 0;
                P.sigma[s] = 1.0;
                P.du[s] = 0.0;
                P.list_v[0] = s;
                P.list_pre[0] = 0;
                C->list = (1ull << P.ebits) | (unsigned long long)dego;
                C->indeg_vis = (unsigned long long)P.deg2[s].y;
                C->cand[0] = 0;
                C->cand[1] = 0;
            }
            for (int64_t i = tid; i <= dego / kWT; i += kBlock) P.tiles[i] = 0;
        }
        prev_s = s;
        grid_sync(C, gen);

        Level cur{0, 1, 0, dego, 0};  // level d-1 (frontier)
        int d = 1;
        bool cand_valid = false;
        int cb = 0;
        int64_t candN = 0, candE = 0;
        int64_t fwd_edges = 0, pulls = 0, scans = 0;
        for (;;) {
            const int64_t ntiles_f = ceil_div(cur.N + cur.E, kWT);
            Level nxt{cur.p0 + cur.N, 0, cur.e0 + cur.E, 0, cur.tbase + ntiles_f};
            // ---- direction (push cost = frontier out-edges, pull cost = in-edges
            //      of the undiscovered candidates (+ a scan of n vertices to list them))
            bool pull = false;
            if (P.dir_mode == 2) {
                pull = d >= 2;
            } else if (P.dir_mode == 0 && d >= 2) {
                const double pull_cost = cand_valid
                    ? (double)candE
                    : (double)(P.m - (int64_t)ld_volatile_u64(&C->indeg_vis)) + 0.25 * (double)P.n;
                pull = P.alpha * pull_cost < (double)cur.E;
            }
            if (pull && !cand_valid) {
                // candidate scan: undiscovered vertices with in-edges, in-degree prefix + tiles
                AppendTarget ct{&C->cand[cb], P.cand_v[cb], P.cand_pre[cb], P.cand_tiles[cb], 0, 0};
                for (int64_t base = gtid - (tid & 31); base < P.n; base += nthreads) {
                    const int64_t v = base + (tid & 31);
                    bool pr = false;
                    int64_t ind = 0;
                    if (v < P.n && P.depth[v] == -1) {
                        ind = P.deg2[v].y;
                        pr = ind > 0;
                    }
                    warp_append(pr, (int32_t)v, pr ? ind : 0, ct.ctr, P.ebits, ct.v, ct.pre, ct.tiles, 0, 0);
                }
                grid_sync(C, gen);
                const unsigned long long cv = ld_volatile_u64(&C->cand[cb]);
                candN = (int64_t)(cv >> P.ebits);
                candE = (int64_t)(cv & emask);
                cand_valid = true;
                ++scans;
            }
            AppendTarget lo{&C->list, P.list_v, P.list_pre, P.tiles + nxt.tbase, nxt.p0, nxt.e0};
            if (pull) {
                AppendTarget co{&C->cand[cb ^ 1], P.cand_v[cb ^ 1], P.cand_pre[cb ^ 1], P.cand_tiles[cb ^ 1], 0, 0};
                level_pass<MODE_PULL>(P, ws, P.cand_v[cb], P.cand_pre[cb], P.cand_tiles[cb], candN, candE, 0,
                                      P.in_ptr, P.in_idx, d, gwarp, nwarps, lo, co);
                fwd_edges += candE;
                ++pulls;
            } else {
                level_pass<MODE_PUSH>(P, ws, P.list_v + cur.p0, P.list_pre + cur.p0, P.tiles + cur.tbase, cur.N,
                                      cur.E, cur.e0, P.out_ptr, P.out_idx, d, gwarp, nwarps, lo, lo);
                fwd_edges += cur.E;
                if (cta0 && tid == 0) {
                    C->cand[0] = 0;  // candidate lists are stale after a push level
                    C->cand[1] = 0;
                }
                cand_valid = false;
            }
            grid_sync(C, gen);
            {
                const unsigned long long lv = ld_volatile_u64(&C->list);
                nxt.N = (int64_t)(lv >> P.ebits) - nxt.p0;
                nxt.E = (int64_t)(lv & emask) - nxt.e0;
            }
            if (pull) {
                const unsigned long long cv = ld_volatile_u64(&C->cand[cb ^ 1]);
                candN = (int64_t)(cv >> P.ebits);
                candE = (int64_t)(cv & emask);
                if (cta0 && tid == 0) C->cand[cb] = 0;  // consumed; next append target after cb flips
                cb ^= 1;
            }
            if (cta0 && tid == 0) {
                int64_t *l = P.lvl + 5 * (int64_t)d;
                l[0] = nxt.p0; l[1] = nxt.N; l[2] = nxt.e0; l[3] = nxt.E; l[4] = nxt.tbase;
            }
            if (nxt.N == 0) break;
            if (d > P.n + 1) __trap();  // impossible for a correct BFS: fail loudly, never spin
            cur = nxt;
            ++d;
        }
        const int D = d - 1;  // height of the BFS tree (levels 0..D non-empty)
        if (cta0 && tid == 0) {
            int64_t *l0 = P.lvl;
            l0[0] = 0; l0[1] = 1; l0[2] = 0; l0[3] = dego; l0[4] = 0;
            C->st_sources += 1;
            C->st_reached += cur.p0 + cur.N;
            C->st_reached_edges += cur.e0 + cur.E;
            C->st_fwd_edges += fwd_edges;
            C->st_levels += d;
            C->st_pull_levels += pulls;
            C->st_scans += scans;
            if (D > C->st_max_depth) C->st_max_depth = D;
        }
        if (P.bfs_only) break;

        // ---------------- backward (Alg.1 l.29-47): L = D (owner-only) down to 1
        int64_t bwd_edges = 0;
        for (int L = D; L >= 1; --L) {
            Level lv;
            if (L == D) {
                lv = cur;
            } else {
                const int64_t *l = P.lvl + 5 * (int64_t)L;
                lv = Level{l[0], l[1], l[2], l[3], l[4]};
            }
            if (L == D) {
                // deepest level: delta = 0, so delta_u = 1/sigma (Alg.1 l.35) and bc += 0
                for (int64_t i = gtid; i < lv.N; i += nthreads) {
                    const int32_t v = P.list_v[lv.p0 + i];
                    const double dun = 1.0 / P.sigma[v];
                    P.du[v] = (L & 1) ? -dun : dun;
                    P.sigma[v] = 0.0;
                    P.depth[v] = -1;
                }
            } else {
                AppendTarget none{nullptr, nullptr, nullptr, nullptr, 0, 0};
                level_pass<MODE_BWD>(P, ws, P.list_v + lv.p0, P.list_pre + lv.p0, P.tiles + lv.tbase, lv.N, lv.E,
                                     lv.e0, P.out_ptr, P.out_idx, L, gwarp, nwarps, none, none);
                bwd_edges += lv.E;
            }
            grid_sync(C, gen);
        }
        if (cta0 && tid == 0) C->st_bwd_edges += bwd_edges;
    }
    // leave the workspace all-unvisited for the next call (bfs_only keeps it for the caller)
    if (!P.bfs_only && cta0 && tid == 0 && prev_s >= 0) {
        P.depth[prev_s] = -1;
        P.sigma[prev_s] = 0.0;
    }
}

}  // namespace

// ------------------------------------------------------------------ host side

tbc_status engine_setup(tbc_graph *g) {
    const int64_t n = g->n, m = g->m;
    cudaStream_t s = g->stream;
    cudaError_t e;
    auto alloc = [&](auto **p, size_t count) -> cudaError_t {
        size_t bytes = sizeof(**p) * (count > 0 ? count : 1);
        cudaError_t r = cudaMalloc((void **)p, bytes);
        if (r == cudaSuccess) g->device_bytes += bytes;
        return r;
    };
    // packed counters: high bits count (<= n), low bits edge sum (<= m)
    int cbits = 1;
    while ((1ll << cbits) <= n) ++cbits;
    g->ebits = 64 - cbits;
    if (g->ebits < 63 && (m >> g->ebits) != 0)
        return set_error(TBC_ERR_UNSUPPORTED, "nnz %lld too large for n %lld", (long long)m, (long long)n);
    const int64_t list_tiles = (n + m) / kWT + n + 2;
    const int64_t cand_tiles = (n + m) / kWT + 2;
    if ((e = alloc(&g->depth, n)) || (e = alloc(&g->sigma, n)) || (e = alloc(&g->du, n)) ||
        (e = alloc(&g->gacc, n)) || (e = alloc(&g->gcnt, n)) || (e = alloc(&g->list_v, n + 1)) ||
        (e = alloc(&g->list_pre, n + 1)) || (e = alloc(&g->tiles, list_tiles)) ||
        (e = alloc(&g->lvl, 5 * (n + 2))) || (e = alloc(&g->ctr, 1)))
        return cuda_error(e, "workspace cudaMalloc");
    if (g->engine == TBC_ENGINE_CSC) {
        for (int b = 0; b < 2; ++b)
            if ((e = alloc(&g->cand_v[b], n + 1)) || (e = alloc(&g->cand_pre[b], n + 1)) ||
                (e = alloc(&g->cand_tiles[b], cand_tiles)))
                return cuda_error(e, "workspace cudaMalloc");
    }
    if ((e = cudaMemsetAsync(g->depth, 0xff, sizeof(int32_t) * n, s)) ||
        (e = cudaMemsetAsync(g->sigma, 0, sizeof(double) * n, s)) ||
        (e = cudaMemsetAsync(g->du, 0, sizeof(double) * n, s)) ||
        (e = cudaMemsetAsync(g->gacc, 0, sizeof(double) * n, s)) ||
        (e = cudaMemsetAsync(g->gcnt, 0, sizeof(int32_t) * n, s)) ||
        (e = cudaMemsetAsync(g->ctr, 0, sizeof(Ctrs), s)) || (e = cudaStreamSynchronize(s)))
        return cuda_error(e, "workspace init");
    int per_sm = 0, sms = 0;
    if ((e = cudaFuncSetAttribute(k_bc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes)) ||
        (e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_bc, kBlock, kSmemBytes)) ||
        (e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device)))
        return cuda_error(e, "occupancy query");
    if (per_sm < 1) return set_error(TBC_ERR_CUDA, "k_bc cannot be resident (occupancy 0)");
    g->grid = per_sm * sms;
    return TBC_OK;
}

tbc_status engine_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                      int bfs_only) {
    if (g->engine != TBC_ENGINE_CSC)
        return set_error(TBC_ERR_UNSUPPORTED, "engine %d not available in this build", g->engine);
    Params P{};
    P.n = g->n;
    P.m = g->m;
    P.in_ptr = g->in_ptr;
    P.in_idx = g->in_idx;
    P.out_ptr = g->out_ptr;
    P.out_idx = g->out_idx;
    P.deg2 = g->deg2;
    P.depth = g->depth;
    P.sigma = g->sigma;
    P.du = g->du;
    P.gacc = g->gacc;
    P.gcnt = g->gcnt;
    P.list_v = g->list_v;
    P.list_pre = g->list_pre;
    P.tiles = g->tiles;
    for (int b = 0; b < 2; ++b) {
        P.cand_v[b] = g->cand_v[b];
        P.cand_pre[b] = g->cand_pre[b];
        P.cand_tiles[b] = g->cand_tiles[b];
    }
    P.lvl = g->lvl;
    P.ctr = g->ctr;
    P.bc = d_bc;
    P.sources = d_sources;
    P.k = k;
    P.bc_scale = g->directed ? 1.0 : 0.5;
    P.ebits = g->ebits;
    P.bfs_only = bfs_only;
    P.dir_mode = g->dir_mode;
    P.alpha = g->alpha;
    void *args[] = {&P};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_bc, dim3(g->grid), dim3(kBlock), args, kSmemBytes, stream);
    if (e != cudaSuccess) return cuda_error(e, "cudaLaunchCooperativeKernel(k_bc)");
    return TBC_OK;
}

}  // namespace tbc
