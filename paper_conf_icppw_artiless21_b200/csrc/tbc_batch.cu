// tbc_batch.cu -- the batched multi-source engine (north star (c)): Algorithm 1
// of PAPER.md for 32 sources at once, one source per warp lane.  The per-source
// SpMV f_t = A^T f of l.19 becomes the product of A^T with a tall-skinny n x 32 frontier block
// (sparse times tall-skinny, still CUDA cores: irregular gathers, not a dense contraction), and
// the backward SpMV of l.37 (A delta_u, R1) likewise.  One stream of the adjacency
// serves all 32 sources of a level, and the per-level fixed costs (barriers, small levels,
// tails) are paid once per 32 sources instead of once per source.
//
// State (vertex-major, source-minor, so a warp's 32 lanes touch one 256-byte row):
//   sig[v][s]  sigma_s(v)             (fp64, exact integers < 2^53)
//   du[v][s]   delta_u_s(v) = (1 + delta_s(v)) / sigma_s(v) = 1/sigma_s(v) + acc_s(v)  (l.35)
//   vis[v]     lanes s with depth_s(v) <= the current level
//   fr[p][v]   lanes s with depth_s(v) = d, for the levels d of parity p in flight
//   level list d: vertices with any lane on level d, with that lane mask (M_d) and their
//              out-degree prefix, plus per-warp-tile start owners (merge path, as tbc_engine.cu)
//
// Forward level d+1 (Alg.1 l.19-27):
//   PUSH  owners = level list d; lanes M_d(u) & ~vis(x) of each out-edge u->x:
//         sig[x][s] += sig[u][s] (fp64 atomic), fr[x] |= lanes; the atomicOr that lifts fr[x]
//         from 0 appends x to level list d+1.
//   PULL  owners = candidates w (any active lane unvisited); lanes M_d(u) & ~vis(w) of each
//         in-edge u->w: acc[s] += sig[u][s]; discovered lanes = acc > 0 (the mask of l.20-25).
//   then an owner phase: list_m = M_{d+1}, vis |= M_{d+1}, retire M_d's dense masks.
// Backward level L = D..1 (Alg.1 l.29-47): owners = level list L; lanes M_L(v) & M_{L+1}(w) of
// each out-edge v->w: acc[s] += du[w][s]; then bc(v) += scale * sum_s sigma_s(v) acc_s
// (l.39, l.45, 1/2 if undirected P:180) and du[v][s] = 1/sigma_s(v) + acc_s.  A vertex whose
// out-edges span several warp tiles is "split": its partial sums are added with fp64 atomics
// (both bc and du are linear in acc), the tile holding its first item adds the 1/sigma term.
#include <algorithm>
#include <cstdio>

#include <cub/device/device_radix_sort.cuh>

#include "tbc_internal.cuh"
#include "tbc_device.cuh"

namespace tbc {
namespace {

constexpr unsigned FULL = 0xffffffffu;
#ifndef TBC_BBLOCK
#define TBC_BBLOCK 1024
#endif
constexpr int kBB = TBC_BBLOCK;  // threads per CTA (one CTA per SM)
constexpr int kBWarps = kBB / 32;
constexpr int kBI = 2;           // tile items per lane (window / index phases)
constexpr int kBT = 32 * kBI;    // diagonal items (owner end items + edges) per warp tile
constexpr int kPad = 8;
#ifndef TBC_BUNROLL
#define TBC_BUNROLL 6
#endif
#ifndef TBC_BUNROLL64
#define TBC_BUNROLL64 8
#endif
#ifndef TBC_STATIC_PCT
#define TBC_STATIC_PCT 80  // share of a pass's tiles dealt statically (the rest: dynamic); A/B on B200
                           // (round 2): 80 vs 60 -- Kronecker 22 379 vs 369 GTEPS, RMAT 18 404 vs 401,
                           // Kronecker 25 475 vs 476, mycielski19 1095 vs 1100; 90 loses on RMAT / mycielski
#endif
#ifndef TBC_DYN_CHUNK
#define TBC_DYN_CHUNK 1    // tiles taken per atomic in the dynamic share
#endif
#ifndef TBC_DYN_BIG
#define TBC_DYN_BIG 4      // chunk multiplier on passes of > 4 M tiles
#endif
// gathers in flight per lane in the slot loop, by batch width (A/B on B200: W = 32 best at 6 --
// Kronecker 25: 394 vs 389 at 4, 373 at 8; W = 64 best at 8, i.e. 4 per source -- Kronecker 22:
// 332 vs 318 at 6, RMAT 18: 359 vs 350)
constexpr int kBU = TBC_BUNROLL;
constexpr int kBU64 = TBC_BUNROLL64;

enum { B_PUSH = 0, B_PULL = 1, B_BWD = 2, B_BPUSH = 3 };  // B_BPUSH: one-format backward push

// lane-mask word of a batch of W sources: lane l of a warp holds sources l and (W = 64) l + 32
template <int W> struct MaskT { using T = uint32_t; };
template <> struct MaskT<64> { using T = unsigned long long; };

// TBC_PROF builds: lane 0 of every warp sums clock64 deltas per region into gctr->prof[0..15]:
// 0 barrier, 1 B phase, 2 push pass, 3 pull pass, 4 backward pass, 5 retire, 6 init/other,
// 8 + {0 window, 1 index+masks, 2 claims/append, 3 owner loop} inside the edge passes
enum { BR_BAR = 0, BR_BPHASE = 1, BR_PASS = 2, BR_CLEAR = 5, BR_OTHER = 6, BR_WIN = 8, BR_IDX = 9, BR_APP = 10,
       BR_OWN = 11, BR_OGATH = 12, BR_OEPI = 13, BR_SLOTS = 16 };
#ifdef TBC_PROF
__shared__ unsigned long long tbc_bprof[kBWarps][BR_SLOTS];
#define BPROF_START() unsigned long long _bt = clock64()
#define BPROF(slot)                                                              \
    do {                                                                         \
        const unsigned long long _n = clock64();                                 \
        if ((threadIdx.x & 31) == 0) tbc_bprof[threadIdx.x >> 5][(slot)] += _n - _bt; \
        _bt = _n;                                                                \
    } while (0)
#else
#define BPROF_START() ((void)0)
#define BPROF(slot) ((void)0)
#endif

struct BParams {
    int64_t n, m;
    const int64_t *__restrict__ in_ptr;
    const int32_t *__restrict__ in_idx;
    const int64_t *__restrict__ out_ptr;
    const int32_t *__restrict__ out_idx;
    const int2 *__restrict__ deg2;
    double *sig, *du;  // du == sig when the backward runs in place (two-format graphs)
    double *sacc;      // in place: [2][sacc_cap] split owners' partial sums by level parity
    int64_t *scnt;     // in place: split lanes per level of the sweep
    int64_t sacc_cap;
    int inplace;
    void *vis;        // MaskT<W>[n]
    void *fr0, *fr1;  // MaskT<W>[n]
    int32_t *list_v;
    uint32_t *list_pre, *list_beg;
    void *list_m;     // MaskT<W>[list_cap]
    int32_t *tiles;
    int32_t *cand_v;
    uint32_t *cand_pre, *cand_beg;
    int32_t *cand_tiles;
    int64_t *lvl;
    Ctrs *ctr;
    Ctrs *gctr;  // TBC_PROF builds: slot statistics in gctr->prof[24..31]
    double *bc;
    const int32_t *sources;
    int src_internal;  // sources already in internal labels (the grouped order), else caller labels
    const int32_t *__restrict__ perm;
    const int32_t *__restrict__ inv;
    int64_t k, n_scan, list_cap, tiles_cap, cand_tiles_cap;
    double bc_scale, pull_ratio;
    int ebits, dir_mode;
    int64_t *trace;  // per-phase timeline of batch trace_b (TBC_OPT_TRACE: source index / W)
    int64_t trace_cap, trace_b;
    // tbc_bfs_batch: forward stage only; depth / sigma of source i (list order, caller labels)
    // exported to bfs_depth[i n + v], bfs_sigma[i n + v] (pre-set to -1 / 0 by the host)
    int32_t *bfs_depth;
    double *bfs_sigma;
    int fwd_only;  // TBC_OPT_STAGE = 1: forward stage only (measurement), bc untouched
    // TBC_FLAG_ONE_FORMAT (directed): the CSC is the only adjacency -- list entries carry in-edge
    // spans (adj_ptr = in_ptr), every forward level is a pull, the backward pushes delta_u of level
    // L+1 over its in-edges into level L's rows, then an owner pass finishes level L
    int one_format;
    const int64_t *__restrict__ adj_ptr;  // spans of list entries: out_ptr, or in_ptr (one format)
};

// one launch: a BParams per SM partition (its own workspace and counters/barrier); partition q
// runs the batches q, q + nparts, ... on CTAs [q * cta_per_part, (q + 1) * cta_per_part)
constexpr int kBParts = 8;
struct BParamSet {
    BParams p[kBParts];
    int nparts, cta_per_part;
};

struct __align__(16) BWarpSmem {
    uint32_t beg[kBT + 2];   // adjacency position of the owner's first in-tile edge
    int32_t first[kBT + 2];  // slot of that edge (+ sentinel ne)
    int32_t v[kBT + 2];      // owner vertex
    unsigned long long msk[kBT + 2];  // owner lanes
    int32_t fl[kBT + 2];     // bit 0: the tile holds the owner's first item; bit 1: whole owner
    int32_t own[kBT + 2];    // owner (window index) of each slot
    int32_t x[kBT];          // other end of each slot
    int32_t claim[kBT + 2];  // vertices discovered by this tile (PULL); BWD in place: split owners' offsets
};
constexpr size_t kBSmem = sizeof(BWarpSmem) * kBWarps;

struct Lv {
    int64_t p0, N, E, tb;
};

// list entries used by a batch whose deepest level is D (levels 0..D are concatenated)
__device__ __forceinline__ int64_t nxt_p0_end(const BParams &P, int D) {
    const int64_t *l = P.lvl + 4 * (int64_t)D;
    return l[0] + l[1];
}

__device__ __forceinline__ int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// timeline entry {t_ns, kind, level, N, E, a, b, 0} after a barrier (CTA 0, thread 0; traced batch)
// kinds as tbc_trace_get: 0 init, 1 level masks + candidates (B phase), 2 push, 3 pull, 4 backward
__device__ __forceinline__ void btrace(const BParams &P, bool on, int kind, int64_t level, int64_t N, int64_t E,
                                       int64_t a, int64_t b) {
    if (!on || threadIdx.x != 0) return;  // on: the traced batch, CTA 0 of its partition
    const unsigned long long i = P.gctr->trace_n;
    if ((int64_t)i >= P.trace_cap) return;
    int64_t *t = P.trace + 8 * i;
    t[0] = (int64_t)globaltimer_ns(); t[1] = kind; t[2] = level; t[3] = N; t[4] = E; t[5] = a; t[6] = b; t[7] = 0;
    P.gctr->trace_n = i + 1;
}

// grid barrier (as tbc_engine.cu): the last arriver snapshots {list, active, cand} counters
__device__ __forceinline__ void bsync(Ctrs *c, unsigned &gen, unsigned nblocks) {
    BPROF_START();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned g0 = gen;
        fence_acq_rel();
        const unsigned arrived = atomicAdd(&c->bar_count, 1u);
        if (arrived == nblocks - 1) {
            c->bar_count = 0;
            fence_acq_rel();
            const unsigned long long s0 = ld_volatile_u64(&c->list), s1 = ld_volatile_u64(&c->ilist),
                                     s2 = ld_volatile_u64(&c->cand[0]);
            c->snap[0] = s0;
            c->snap[1] = s1;
            c->snap[2] = s2;
            fence_acq_rel();
            atomicExch(&c->bar_gen, g0 + 1);
        } else {
            const unsigned long long t0 = globaltimer_ns();
            while (ld_acquire(&c->bar_gen) == g0) {
                __nanosleep(20);
                if (globaltimer_ns() - t0 > kWatchdogNs) __trap();
            }
        }
        fence_acq_rel();
    }
    gen += 1;
    __syncthreads();
    BPROF(BR_BAR);
}

// a list being appended to: relative packed counter (count << ebits) | degree sum, arrays
// offset to the level start, capacities left
struct BOut {
    unsigned long long *ctr;
    int32_t *v;
    uint32_t *pre, *beg;
    int32_t *tiles;
    int64_t cap, tcap;
    unsigned *ovf;  // set when an entry or a tile start does not fit (the batch is re-run in halves)
};

// warp-aggregated append of the entries lanes hold (item i of lane l: v[i], degree dg[i],
// adjacency begin bg[i] if take[i]); one packed atomic per warp; the appender of an owner writes
// the start owner of every tile whose first item lies in its merge-path span (tbc_engine.cu)
__device__ __forceinline__ void bappend(const bool (&take)[kBI], const int32_t (&v)[kBI], const uint32_t (&dg)[kBI],
                                        const uint32_t (&bg)[kBI], const BOut &o, int ebits) {
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    unsigned cnt = 0;
    unsigned long long esum = 0;
#pragma unroll
    for (int i = 0; i < kBI; ++i) {
        cnt += __popc(__ballot_sync(FULL, take[i]));
        esum += __reduce_add_sync(FULL, take[i] ? dg[i] : 0u);
    }
    if (cnt == 0) return;
    unsigned long long old = 0;
    if (lane == 0) old = atomicAdd(o.ctr, ((unsigned long long)cnt << ebits) + esum);
    old = __shfl_sync(FULL, old, 0);
    int64_t p = (int64_t)(old >> ebits);
    int64_t e = (int64_t)(old & ((1ull << ebits) - 1ull));
#pragma unroll
    for (int i = 0; i < kBI; ++i) {
        const unsigned msk = __ballot_sync(FULL, take[i]);
        if (msk == 0) continue;
        const uint32_t x = take[i] ? dg[i] : 0u;
        uint32_t inc = x;
#pragma unroll
        for (int k = 1; k < 32; k <<= 1) {
            const uint32_t t = __shfl_up_sync(FULL, inc, k);
            if (lane >= k) inc += t;
        }
        if (take[i]) {
            const int64_t pp = p + __popc(msk & lt);
            const int64_t ee = e + (int64_t)(inc - x);
            const int64_t k0 = ee + pp, k1 = k0 + x;
            if (pp < o.cap && k1 / kBT < o.tcap) {
                o.v[pp] = v[i];
                o.pre[pp] = (uint32_t)ee;
                o.beg[pp] = bg[i];
                for (int64_t t = (k0 + kBT - 1) / kBT; t <= k1 / kBT; ++t) o.tiles[t] = (int32_t)pp;
            } else {  // capacity exceeded: the kernel re-runs the batch in halves (k_bcb)
                *o.ovf = 1u;
            }
        }
        p += __popc(msk);
        e += __shfl_sync(FULL, inc, 31);
    }
}

__device__ __forceinline__ void span(const int64_t *ptr, int32_t v, uint32_t &dg, uint32_t &bg) {
    const int64_t b = ptr[v];
    bg = (uint32_t)b;
    dg = (uint32_t)(ptr[v + 1] - b);
}

// 32 x 32 bit transpose across the warp: lane l holds row l (bit c = column c); afterwards lane c
// holds column c (bit l = row l).  Five rounds of block swaps with the partner lane l ^ j.
__device__ __forceinline__ uint32_t transpose32(uint32_t x) {
    const int lane = threadIdx.x & 31;
    constexpr uint32_t hi[5] = {0xFFFF0000u, 0xFF00FF00u, 0xF0F0F0F0u, 0xCCCCCCCCu, 0xAAAAAAAAu};
#pragma unroll
    for (int r = 0; r < 5; ++r) {
        const int j = 16 >> r;
        const uint32_t y = __shfl_xor_sync(FULL, x, j);
        x = (lane & j) ? ((x & hi[r]) | ((y >> j) & ~hi[r])) : ((x & ~hi[r]) | ((y << j) & hi[r]));
    }
    return x;
}

__device__ __forceinline__ uint64_t slot_range(int s0, int s1) {
    if (s0 >= 64 || s1 <= s0) return 0ull;
    const uint64_t hi = s1 >= 64 ? ~0ull : ((1ull << s1) - 1ull);
    return hi & ~((1ull << s0) - 1ull);
}

// One merge-path pass over an owner list (ov/opre/obeg/omsk/otiles, N owners, E edges):
//   PUSH: frontier owners, out-edges;  PULL: candidates, in-edges;  BWD: level-L owners, out-edges.
// emsk: per-vertex lane mask of the other end (PULL: M_d, BWD: M_{L+1}; PUSH uses ~vis).
// fr_out: PUSH/PULL the next level's dense mask, BWD the owners' level (scattered M_L).
template <int MODE, int W, bool IP = false>
__device__ __forceinline__ void bpass(const BParams &P, BWarpSmem &ws, const int32_t *ov, const uint32_t *opre,
                                      const uint32_t *obeg, const void *omsk_, const int32_t *otiles, int64_t N,
                                      int64_t E, const int32_t *__restrict__ adj_idx, const void *emsk_,
                                      void *fr_out_, unsigned long long active_, int64_t gwarp, int64_t nwarps,
                                      const BOut &out, unsigned long long *dyn, const uint32_t *soff = nullptr,
                                      double *sacc_l = nullptr) {
    using MT = typename MaskT<W>::T;
    constexpr int NS = W / 32;                 // sources per lane
    constexpr int U2 = (NS == 1 ? kBU : kBU64) / NS > 0 ? (NS == 1 ? kBU : kBU64) / NS : 1;  // gathers in flight per lane and source
    const MT *omsk = static_cast<const MT *>(omsk_);
    const MT *emsk = static_cast<const MT *>(emsk_);
    MT *fr_out = static_cast<MT *>(fr_out_);
    const MT *vis = static_cast<const MT *>(P.vis);
    const MT active = (MT)active_;
    const int lane = threadIdx.x & 31;
    const int64_t K = N + E;
    const int64_t ntiles = cdiv(K, kBT);
    const uint64_t pol = policy_evict_first();
    double *const sig = P.sig;
    // tiles [0, nstat) are dealt round-robin; the rest are taken one at a time from the pass's
    // counter by warps that ran out, so the costly tiles (many active lanes) do not leave most
    // warps waiting at the next grid barrier
    const int64_t nstat = (ntiles * TBC_STATIC_PCT) / 100;
    // dynamic chunk: 1 tile per atomic, 4 on passes of > 4 M tiles (A/B on B200: Kronecker 22, whose
    // largest passes have ~1 M tiles, is best at 1; Kronecker 25, ~16 M, at 4: 402 -> 426 GTEPS)
    const int chunk = ntiles > (4ll << 20) ? TBC_DYN_BIG * TBC_DYN_CHUNK : TBC_DYN_CHUNK;
    int64_t dend = -1;  // end of the warp's current dynamic chunk
    for (int64_t tile = gwarp;;) {
        if (tile >= nstat && tile >= dend) {
            unsigned long long t = 0;
            if (lane == 0) t = atomicAdd(dyn, 1ull);
            tile = nstat + (int64_t)__shfl_sync(FULL, t, 0) * chunk;
            dend = tile + chunk;
        }
        if (tile >= ntiles) break;
        BPROF_START();
        const int64_t ks = tile * kBT;
        const int64_t ke = min(ks + (int64_t)kBT, K);
        const int64_t ps = otiles[tile];
        const int64_t pe = (tile + 1 < ntiles) ? (int64_t)otiles[tile + 1] : N;
        const int64_t es = ks - ps, ee = ke - pe;
        const int nwin = (int)(min(pe, N - 1) - ps + 1);
        const int ne = (int)(ee - es);
        // ---- owner window
        for (int j = lane; j < nwin; j += 32) {
            const int64_t p = ps + j;
            const int64_t pre = (int64_t)opre[p];
            const int64_t f = max(pre, es);
            const int32_t v = ov[p];
            ws.first[j] = (int32_t)(f - es);
            ws.beg[j] = obeg[p] + (uint32_t)(f - pre);
            ws.v[j] = v;
            const int64_t kf = pre + p;  // the owner's first diagonal item
            const bool isf = kf >= ks && kf < ke;
            const bool whole = isf && p < pe;
            ws.msk[j] = (MODE == B_PULL) ? (MT)(~vis[v] & active) : omsk[p];
            ws.fl[j] = (isf ? 1 : 0) | (whole ? 2 : 0);
            if (MODE == B_BWD && IP) ws.claim[j] = whole ? 0 : (int32_t)soff[p];
        }
        for (int sl = lane; sl < kBT; sl += 32) ws.own[sl] = -1;
        if (lane == 0) ws.first[nwin] = ne;
        __syncwarp();
        for (int j = lane; j < nwin; j += 32)
            if (ws.first[j] < ws.first[j + 1]) ws.own[ws.first[j]] = j;
        __syncwarp();
        {  // owner of every slot: running max of the head marks over lane-contiguous slots
            int o[kBI];
            int run = -1;
#pragma unroll
            for (int i = 0; i < kBI; ++i) {
                const int sl = lane * kBI + i;
                run = max(run, sl < ne ? ws.own[sl] : -1);
                o[i] = run;
            }
            int incl = run;
#pragma unroll
            for (int k = 1; k < 32; k <<= 1) {
                const int t = __shfl_up_sync(FULL, incl, k);
                if (lane >= k) incl = max(incl, t);
            }
            int prev = __shfl_up_sync(FULL, incl, 1);
            if (lane == 0) prev = -1;
            __syncwarp();
#pragma unroll
            for (int i = 0; i < kBI; ++i) {
                const int sl = lane * kBI + i;
                if (sl < ne) ws.own[sl] = max(prev, o[i]);
            }
        }
        __syncwarp();
        BPROF(BR_WIN);
        // ---- edges, coalesced (slot = i*32 + lane): other end and its lanes
        int xs[kBI];
        MT ems[kBI];
        uint64_t act = 0;
#pragma unroll
        for (int i = 0; i < kBI; ++i) {
            const int sl = i * 32 + lane;
            xs[i] = 0;
            ems[i] = 0;
            if (sl < ne) {
                const int j = ws.own[sl];
                xs[i] = ld_stream(adj_idx + ws.beg[j] + (uint32_t)(sl - ws.first[j]), pol);
            }
        }
#pragma unroll
        for (int i = 0; i < kBI; ++i) {
            const int sl = i * 32 + lane;
            if (sl < ne) {
                const MT g = (MODE == B_PUSH) ? (MT)~vis[xs[i]] : emsk[xs[i]];  // BPUSH: M_L(u)
                ems[i] = g & (MT)ws.msk[ws.own[sl]];
            }
            ws.x[sl] = xs[i];
            act |= (uint64_t)__ballot_sync(FULL, ems[i] != (MT)0) << (32 * i);
        }
        // this lane's slots per source: the transpose of the slots' lane masks
        static_assert(kBI == 2, "64 slots per tile: two 32 x 32 transposes per source word");
        uint64_t lm[NS];
#pragma unroll
        for (int k = 0; k < NS; ++k)
            lm[k] = (uint64_t)transpose32((uint32_t)(ems[0] >> (32 * k))) |
                    ((uint64_t)transpose32((uint32_t)(ems[1] >> (32 * k))) << 32);
#ifdef TBC_PROF
        {
            unsigned pairs = 0;
#pragma unroll
            for (int i = 0; i < kBI; ++i) pairs += __popcll((unsigned long long)ems[i]);
            pairs = __reduce_add_sync(FULL, pairs);
            if (lane == 0) {
                atomicAdd(&P.gctr->prof[24 + 2 * MODE], (unsigned long long)__popcll(act));
                atomicAdd(&P.gctr->prof[25 + 2 * MODE], (unsigned long long)pairs);
                atomicAdd(&P.gctr->prof[30], (unsigned long long)ne);
                atomicAdd(&P.gctr->prof[31], (unsigned long long)nwin);
            }
        }
#endif
        BPROF(BR_IDX);
        if (MODE == B_PUSH) {
            // claims: the atomicOr that lifts fr_out[x] from 0 appends x to the next level
            bool cl[kBI];
            uint32_t cdg[kBI], cbg[kBI];
#pragma unroll
            for (int i = 0; i < kBI; ++i) {
                cl[i] = false;
                cdg[i] = 0;
                cbg[i] = 0;
                if (ems[i] != (MT)0) cl[i] = atomicOr(&fr_out[xs[i]], ems[i]) == (MT)0;
                if (cl[i]) span(P.adj_ptr, xs[i], cdg[i], cbg[i]);
            }
            bappend(cl, xs, cdg, cbg, out, P.ebits);
        }
        __syncwarp();
        BPROF(BR_APP);
        int nc = 0;  // PULL: discovered owners of this tile
#ifdef TBC_PROF
        unsigned n_own = 0;
#endif
        uint64_t leaf = 0;  // BWD: owners first seen here without an active slot (below)
        for (int j = 0; j < nwin; ++j) {
            uint64_t bits = act & slot_range(ws.first[j], ws.first[j + 1]);
            const int fl = ws.fl[j];
            if (MODE != B_BWD && bits == 0) continue;
            if (MODE == B_BWD && bits == 0) {
                if (!(fl & 1)) continue;
                if (j < 64) {  // (window entry 64 never starts in the tile; kept on the path below)
                    leaf |= 1ull << j;
                    continue;
                }
            }
            (void)fl;
#ifdef TBC_PROF
            ++n_own;
#endif
            const int32_t v = ws.v[j];
            const MT m = (MT)ws.msk[j];
            const int64_t row = (int64_t)v * W + lane;  // + 32 k: the lane's word of source k
            bool in[NS];
            uint64_t mine[NS];
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                in[k] = (m >> (32 * k + lane)) & 1u;
                // each lane walks only its own sources' slots of this owner (divergent loop, no
                // collectives inside): warp iterations = the busiest lane's count, not the slots'
                mine[k] = lm[k] & bits;
            }
            if (MODE == B_PUSH || MODE == B_BPUSH) {
                // PUSH: sigma(x) += sigma(u) (Alg.1 l.19 as a scatter); BPUSH (one format): the owner
                // w of level L+1 adds delta_u(w) into the accumulator row of each in-neighbour u on
                // level L (A delta_u of l.37, R1, as a scatter over the CSC)
                double *const dst = MODE == B_PUSH ? sig : P.du;
#pragma unroll
                for (int k = 0; k < NS; ++k) {
                    const double su = in[k] ? (MODE == B_PUSH ? sig : P.du)[row + 32 * k] : 0.0;
#pragma unroll
                    for (int h = 0; h < kBI; ++h) {
                        uint32_t mm = (uint32_t)(mine[k] >> (32 * h));
                        while (mm) {
                            const int sl = 32 * h + __ffs(mm) - 1;
                            mm &= mm - 1;
                            atomicAdd(&dst[(int64_t)ws.x[sl] * W + 32 * k + lane], su);
                        }
                    }
                }
                continue;
            }
            const double *src = (MODE == B_PULL) ? sig : P.du;
            double sv[NS], acc[NS];
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                sv[k] = (MODE == B_BWD && in[k]) ? sig[row + 32 * k] : 1.0;
                acc[k] = 0.0;
            }
            // the two 32-slot halves of the tile, U2 gathers in flight per lane and source;
            // __ffs(0) = 0 marks the exhausted positions
            BPROF(BR_OWN);
#pragma unroll
            for (int h = 0; h < kBI; ++h) {
                uint32_t mm[NS];
                uint32_t any = 0;
#pragma unroll
                for (int k = 0; k < NS; ++k) {
                    mm[k] = (uint32_t)(mine[k] >> (32 * h));
                    any |= mm[k];
                }
                const int32_t *xh = ws.x + 32 * h;
                while (any) {
                    int sl[NS][U2];
                    double a[NS][U2];
                    any = 0;
#pragma unroll
                    for (int k = 0; k < NS; ++k) {
#pragma unroll
                        for (int q = 0; q < U2; ++q) {
                            sl[k][q] = __ffs(mm[k]) - 1;
                            mm[k] &= mm[k] - 1;
                        }
                        any |= mm[k];
                    }
#pragma unroll
                    for (int k = 0; k < NS; ++k)
#pragma unroll
                        for (int q = 0; q < U2; ++q)
                            a[k][q] = sl[k][q] >= 0 ? src[(int64_t)xh[sl[k][q]] * W + 32 * k + lane] : 0.0;
#pragma unroll
                    for (int k = 0; k < NS; ++k)
#pragma unroll
                        for (int q = 0; q < U2; ++q) acc[k] += a[k][q];
                }
            }
            BPROF(BR_OGATH);
            if (MODE == B_PULL) {
                // Alg.1 l.20-25: lanes with a non-zero masked sum are discovered on this level
                MT newm = 0;
#pragma unroll
                for (int k = 0; k < NS; ++k) newm |= (MT)__ballot_sync(FULL, acc[k] > 0.0) << (32 * k);
                if (newm == (MT)0) continue;
                bool claimed;
                if (fl & 2) {
#pragma unroll
                    for (int k = 0; k < NS; ++k)
                        if (acc[k] > 0.0) sig[row + 32 * k] = acc[k];
                    if (lane == 0) fr_out[v] = newm;
                    claimed = true;
                } else {
#pragma unroll
                    for (int k = 0; k < NS; ++k)
                        if (acc[k] > 0.0) atomicAdd(&sig[row + 32 * k], acc[k]);
                    MT old = 0;
                    if (lane == 0) old = atomicOr(&fr_out[v], newm);
                    claimed = __shfl_sync(FULL, old, 0) == (MT)0;
                }
                if (claimed) {
                    if (lane == 0) ws.claim[nc] = v;
                    ++nc;
                }
            } else {
                // Alg.1 l.38-39, l.45 (x 1/2 undirected) and l.35
                double c = 0.0;
#pragma unroll
                for (int k = 0; k < NS; ++k) c += in[k] ? sv[k] * acc[k] : 0.0;
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
#pragma unroll
                for (int k = 0; k < NS; ++k) {
                    if (fl & 2) {
                        if (in[k]) P.du[row + 32 * k] = __drcp_rn(sv[k]) + acc[k];
                    } else if (IP) {
                        // in place: a split owner's sigma row stays intact until every tile has read
                        // it; the partial sums meet in the split accumulator, bsplit_fin writes delta_u
                        const int b = 32 * k + lane;
                        if (in[k] && acc[k] != 0.0)
                            atomicAdd(&sacc_l[(uint32_t)ws.claim[j] + __popcll((unsigned long long)m & ((1ull << b) - 1ull))],
                                      acc[k]);
                    } else {
                        const double t = acc[k] + ((fl & 1) ? __drcp_rn(sv[k]) : 0.0);
                        if (in[k] && t != 0.0) atomicAdd(&P.du[row + 32 * k], t);
                    }
                }
                if (lane == 0) {
                    if (c != 0.0) atomicAdd(&P.bc[P.inv ? P.inv[v] : v], c * P.bc_scale);
                    if (fl & 1) atomicOr(&fr_out[v], m);
                }
            }
            BPROF(BR_OEPI);
        }
#ifdef TBC_PROF
        if (lane == 0) atomicAdd(&P.gctr->prof[16 + MODE], (unsigned long long)n_own);
#endif
        if (MODE == B_PULL) {
            __syncwarp();
            bool cl[kBI];
            int32_t cv[kBI];
            uint32_t cdg[kBI], cbg[kBI];
#pragma unroll
            for (int i = 0; i < kBI; ++i) {
                const int q = i * 32 + lane;
                cl[i] = q < nc;
                cv[i] = cl[i] ? ws.claim[q] : 0;
                cdg[i] = 0;
                cbg[i] = 0;
                if (cl[i]) span(P.adj_ptr, cv[i], cdg[i], cbg[i]);
            }
            bappend(cl, cv, cdg, cbg, out, P.ebits);
        }
        if (MODE == B_BWD) {
            // owners whose first item is in this tile and that have no active slot here (all their
            // lanes are DAG leaves of this level, e.g. out-degree 0): delta_u = 1/sigma (l.35 with acc
            // = 0; added by the first tile if split), no bc term, their lanes scattered to fr_out.
            // Independent rows, so kLeafU owners per round with their sigma loads in flight together
            // instead of one round trip per owner in the loop above
            constexpr int kLeafU = 4;
            while (leaf) {
                int jq[kLeafU];
                double s[kLeafU][NS];
#pragma unroll
                for (int q = 0; q < kLeafU; ++q) {
                    jq[q] = __ffsll((long long)leaf) - 1;
                    leaf &= leaf - 1;
                }
#pragma unroll
                for (int q = 0; q < kLeafU; ++q) {
#pragma unroll
                    for (int k = 0; k < NS; ++k) {
                        s[q][k] = 1.0;
                        if (jq[q] >= 0 && (((MT)ws.msk[jq[q]] >> (32 * k + lane)) & 1u))
                            s[q][k] = sig[(int64_t)ws.v[jq[q]] * W + 32 * k + lane];
                    }
                }
#pragma unroll
                for (int q = 0; q < kLeafU; ++q) {
                    if (jq[q] < 0) continue;
                    const int32_t v = ws.v[jq[q]];
                    const MT m = (MT)ws.msk[jq[q]];
                    const bool whole = ws.fl[jq[q]] & 2;
#pragma unroll
                    for (int k = 0; k < NS; ++k) {
                        if (!((m >> (32 * k + lane)) & 1u)) continue;
                        double *const d = P.du + (int64_t)v * W + 32 * k + lane;
                        if (whole) *d = __drcp_rn(s[q][k]);
                        else if (!IP) atomicAdd(d, __drcp_rn(s[q][k]));  // in place: bsplit_fin
                    }
                    if (lane == 0) atomicOr(&fr_out[v], m);
                }
            }
        }
        __syncwarp();
        BPROF(BR_OWN);
        tile += tile < nstat ? nwarps : 1;
    }
}

// zero the (vertex, source) state of a level list's entries: sigma, delta_u, visited lanes and
// the dense mask of its parity (atomicAnd: a concurrent scatter of another level may share the word).
// EXPORT (tbc_bfs_batch): first write depth = level and sigma of every (vertex, lane) of the list to
// the caller's [source][vertex] arrays (source index b W + lane word)
template <int W, bool EXPORT = false, bool IP = false>
__device__ __forceinline__ void bclear(const BParams &P, const Lv &l, void *fr_, int64_t gwarp, int64_t nwarps,
                                       int level = 0, int64_t b = 0) {
    using MT = typename MaskT<W>::T;
    constexpr int NS = W / 32;
    MT *fr = static_cast<MT *>(fr_);
    MT *vis = static_cast<MT *>(P.vis);
    const MT *lm = static_cast<const MT *>(P.list_m);
    const int lane = threadIdx.x & 31;
    for (int64_t base = gwarp * 32; base < l.N; base += nwarps * 32) {
        const int64_t p = base + lane;
        int32_t v = -1;
        MT m = 0;
        if (p < l.N) {
            v = P.list_v[l.p0 + p];
            m = lm[l.p0 + p];
            atomicAnd(&fr[v], ~m);
            vis[v] = 0;
        }
        const int cnt = (int)min((int64_t)32, l.N - base);
        for (int q = 0; q < cnt; ++q) {
            const int32_t vq = __shfl_sync(FULL, v, q);
            const MT mq = __shfl_sync(FULL, m, q);
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                if ((mq >> (32 * k + lane)) & 1u) {
                    const int64_t row = (int64_t)vq * W + 32 * k + lane;
                    if (EXPORT) {
                        const int64_t o = (b * W + 32 * k + lane) * P.n + (P.inv ? P.inv[vq] : vq);
                        P.bfs_depth[o] = level;
                        P.bfs_sigma[o] = P.sig[row];
                    }
                    P.sig[row] = 0.0;
                    if (!IP) P.du[row] = 0.0;
                }
            }
        }
    }
}

// ---- in-place backward (two-format graphs): sigma and delta_u share one [n][W] array.  Pass L
// overwrites the level-L lanes of a whole owner's row with delta_u = 1/sigma + acc (l.35) right
// after reading sigma; the lanes of a split owner (its items span several tiles, so several warps
// need its sigma for the bc term) keep sigma through pass L while the tiles add their partial acc
// into a split accumulator, and bsplit_fin writes their delta_u after the pass.  Offsets into the
// accumulator (popc of the entry's lane mask each) are assigned one level ahead, per level parity
// (soff: cand_pre for even levels, cand_beg for odd ones -- the candidate lists are idle in the
// backward).

// list entry p (index in its level) is split: its merge-path items -- the first at pre + p, the
// end item out-degree items later -- fall in more than one tile
__device__ __forceinline__ bool bsplit(const BParams &P, int64_t p0, int64_t p, int32_t v) {
    const int64_t kf = (int64_t)P.list_pre[p0 + p] + p;
    return kf / kBT != (kf + P.deg2[v].x) / kBT;
}

// split-accumulator offsets of level L's split entries (warp-aggregated allocation from
// salloc[L & 1]); count: also add the level's split lanes to scnt[L]
template <int W>
__device__ __forceinline__ void bsplit_enum(const BParams &P, int L, bool count, bool alloc, int64_t gwarp,
                                            int64_t nwarps) {
    using MT = typename MaskT<W>::T;
    const MT *lm = static_cast<const MT *>(P.list_m);
    const int lane = threadIdx.x & 31;
    const int64_t *l = P.lvl + 4 * (int64_t)L;
    const int64_t p0 = l[0], N = l[1];
    uint32_t *soff = (L & 1) ? P.cand_beg : P.cand_pre;
    for (int64_t base = gwarp * 32; base < N; base += nwarps * 32) {
        const int64_t p = base + lane;
        unsigned c = 0;
        if (p < N && bsplit(P, p0, p, P.list_v[p0 + p])) c = __popcll((unsigned long long)lm[p0 + p]);
        unsigned incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        const unsigned tot = __shfl_sync(FULL, incl, 31);
        if (tot == 0) continue;
        unsigned long long b0 = 0;
        if (lane == 0) {
            if (alloc) b0 = atomicAdd(&P.ctr->salloc[L & 1], (unsigned long long)tot);
            if (count) atomicAdd((unsigned long long *)&P.scnt[L], (unsigned long long)tot);
        }
        if (!alloc) continue;
        b0 = __shfl_sync(FULL, b0, 0);
        if (c) soff[p] = (uint32_t)(b0 + incl - c);
    }
}

// the split lanes of every level 1..D into scnt (a sweep whose largest level needs more than
// sacc_cap is re-run in halves), with the offsets of level D
template <int W>
__device__ __forceinline__ void bsplit_count(const BParams &P, int D, int64_t gwarp, int64_t nwarps) {
    for (int L = 1; L <= D; ++L) bsplit_enum<W>(P, L, true, L == D, gwarp, nwarps);
}

// after pass L: delta_u of the split entries' level-L lanes = 1/sigma + sacc (l.35), the accumulator
// entries re-zeroed; then the offsets of level L-1
template <int W>
__device__ __forceinline__ void bsplit_fin(const BParams &P, int L, int64_t gwarp, int64_t nwarps) {
    using MT = typename MaskT<W>::T;
    constexpr int NS = W / 32;
    const MT *lm = static_cast<const MT *>(P.list_m);
    const int lane = threadIdx.x & 31;
    const int64_t *l = P.lvl + 4 * (int64_t)L;
    const int64_t p0 = l[0], N = l[1];
    const uint32_t *soff = (L & 1) ? P.cand_beg : P.cand_pre;
    double *const sacc = P.sacc + (L & 1) * P.sacc_cap;
    for (int64_t base = gwarp * 32; base < N; base += nwarps * 32) {
        const int64_t p = base + lane;
        int32_t v = -1;
        MT m = 0;
        uint32_t off = 0;
        bool sp = false;
        if (p < N) {
            v = P.list_v[p0 + p];
            sp = bsplit(P, p0, p, v);
            if (sp) {
                m = lm[p0 + p];
                off = soff[p];
            }
        }
        unsigned todo = __ballot_sync(FULL, sp);
        while (todo) {
            const int q = __ffs(todo) - 1;
            todo &= todo - 1;
            const int32_t vq = __shfl_sync(FULL, v, q);
            const MT mq = __shfl_sync(FULL, m, q);
            const uint32_t oq = __shfl_sync(FULL, off, q);
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                const int b = 32 * k + lane;
                if ((mq >> b) & 1u) {
                    const int64_t row = (int64_t)vq * W + b;
                    const uint32_t r = oq + __popcll((unsigned long long)mq & ((1ull << b) - 1ull));
                    P.sig[row] = __drcp_rn(P.sig[row]) + sacc[r];
                    sacc[r] = 0.0;
                }
            }
        }
    }
    if (L >= 2) bsplit_enum<W>(P, L - 1, false, true, gwarp, nwarps);
}

// one-format owner pass of level L: for each (v, lane s) on level L the row of du holds
// acc_s(v) = sum of delta_u over v's level-(L+1) out-neighbours (pushed there by B_BPUSH);
// bc(v) += scale * sum_s sigma_s(v) acc_s(v) (Alg.1 l.39, l.45) and du_s(v) = 1/sigma + acc (l.35)
template <int W>
__device__ __forceinline__ void bowner(const BParams &P, const Lv &l, int64_t gwarp, int64_t nwarps) {
    using MT = typename MaskT<W>::T;
    constexpr int NS = W / 32;
    const MT *lm = static_cast<const MT *>(P.list_m);
    const int lane = threadIdx.x & 31;
    for (int64_t base = gwarp * 32; base < l.N; base += nwarps * 32) {
        const int64_t p = base + lane;
        int32_t v = -1;
        MT m = 0;
        if (p < l.N) {
            v = P.list_v[l.p0 + p];
            m = lm[l.p0 + p];
        }
        const int cnt = (int)min((int64_t)32, l.N - base);
        for (int q = 0; q < cnt; ++q) {
            const int32_t vq = __shfl_sync(FULL, v, q);
            const MT mq = __shfl_sync(FULL, m, q);
            double c = 0.0;
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                if ((mq >> (32 * k + lane)) & 1u) {
                    const int64_t row = (int64_t)vq * W + 32 * k + lane;
                    const double sv = P.sig[row], acc = P.du[row];
                    c += sv * acc;
                    P.du[row] = __drcp_rn(sv) + acc;
                }
            }
#pragma unroll
            for (int o = 16; o >= 1; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
            if (lane == 0 && c != 0.0) atomicAdd(&P.bc[P.inv ? P.inv[vq] : vq], c * P.bc_scale);
        }
    }
}

// MULTI = false: one partition, every parameter at a static offset (S.p[0]); MULTI = true: the
// partition's parameters are indexed by blockIdx (costs registers, so only used when P > 1)
template <int W, bool MULTI, bool IP>
__global__ void __launch_bounds__(kBB, 1) k_bcb(const __grid_constant__ BParamSet S) {
    using MT = typename MaskT<W>::T;
    constexpr int NS = W / 32;
    const int part = MULTI ? (int)blockIdx.x / S.cta_per_part : 0;
    const BParams &P = S.p[part];
    const int lcta = MULTI ? (int)blockIdx.x - part * S.cta_per_part : (int)blockIdx.x;  // CTA in the partition
    extern __shared__ __align__(16) unsigned char bsm[];
    // the warp's smem block from an opaque copy of tid.x: the compiler keeps its address in a
    // register instead of re-deriving it from S2R before every shared access under register
    // pressure (~18 % of the instructions; A/B on B200: Kronecker 22 357 -> 366, RMAT 18 ~370 -> 404)
    const unsigned wtid = tid_opaque();
    BWarpSmem &ws = reinterpret_cast<BWarpSmem *>(bsm)[wtid >> 5];
    const int tid = threadIdx.x, lane = tid & 31;
    const bool cta0 = lcta == 0;
    const unsigned ncta = MULTI ? (unsigned)S.cta_per_part : gridDim.x;
    const int64_t nwarps = (int64_t)ncta * kBWarps;
    const int64_t gwarp = (int64_t)lcta * kBWarps + (tid >> 5);
    const int64_t nthreads = (int64_t)ncta * kBB;
    const int64_t gtid = (int64_t)lcta * kBB + tid;
    Ctrs *C = P.ctr;
    unsigned gen = (tid == 0) ? ld_acquire(&C->bar_gen) : 0u;
    const unsigned long long emask = (1ull << P.ebits) - 1ull;
    MT *fr[2] = {static_cast<MT *>(P.fr0), static_cast<MT *>(P.fr1)};
    MT *vis = static_cast<MT *>(P.vis);
    MT *list_m = static_cast<MT *>(P.list_m);
    const int64_t nb = (P.k + W - 1) / W;

#ifdef TBC_PROF
    for (int i = tid; i < kBWarps * BR_SLOTS; i += kBB) (&tbc_bprof[0][0])[i] = 0;
    __syncthreads();
    const unsigned long long t_kernel0 = clock64();
#endif
    for (int64_t b = part; b < nb; b += MULTI ? S.nparts : 1) {
      // the batch's lane sets still to run: all W lanes, or -- after a level list or its tile starts
      // outgrew the workspace (BOut::ovf) -- the two halves of the set that overflowed (a single
      // source always fits: batch_alloc sizes the lists for at least n entries)
      MT pend[8];
      int npend = 0;
      pend[npend++] = ~(MT)0;
      unsigned valid = 0;  // thread 0 of CTA 0: valid sources of the lane set being run
      while (npend > 0) {
        const MT bmask = pend[--npend];
        // ---------------- level 0: the batch's sources (Alg.1 l.15-18): source b*W + 32k + l is
        // lane l's source k; a vertex repeated in the batch is appended once, by its lowest source
        if (cta0 && tid < 32) {
            int32_t s[NS];
            valid = 0;
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                const int64_t si = b * W + 32 * k + lane;
                s[k] = -1;
                if (si < P.k && ((bmask >> (32 * k + lane)) & 1u)) {
                    const int32_t sc = P.sources[si];
                    if (sc >= 0 && sc < P.n) s[k] = (P.perm && !P.src_internal) ? P.perm[sc] : sc;
                    else if (bmask == ~(MT)0) atomicAdd(&C->bad_sources, 1ull);
                }
                if (s[k] >= 0) {
                    atomicOr(&fr[0][s[k]], (MT)1 << (32 * k + lane));
                    P.sig[(int64_t)s[k] * W + 32 * k + lane] = 1.0;
                }
                valid += __popc(__ballot_sync(FULL, s[k] >= 0));
            }
            int pos0 = 0;
            uint32_t e0 = 0;
#pragma unroll
            for (int k = 0; k < NS; ++k) {
                bool take = s[k] >= 0;
                for (int l = 0; l < 32; ++l) {
#pragma unroll
                    for (int k2 = 0; k2 <= k; ++k2) {
                        const int32_t t = __shfl_sync(FULL, s[k2], l);
                        if ((k2 < k || l < lane) && t == s[k]) take = false;
                    }
                }
                uint32_t dg = 0, bg = 0;
                if (take) span(P.adj_ptr, s[k], dg, bg);
                const unsigned tm = __ballot_sync(FULL, take);
                uint32_t inc = take ? dg : 0u;
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t t = __shfl_up_sync(FULL, inc, o);
                    if (lane >= o) inc += t;
                }
                if (take) {
                    const int pos = pos0 + __popc(tm & ((1u << lane) - 1u));
                    const uint32_t ee = e0 + inc - dg;
                    P.list_v[pos] = s[k];
                    P.list_pre[pos] = ee;
                    P.list_beg[pos] = bg;
                    const int64_t k0 = (int64_t)ee + pos, k1 = k0 + dg;
                    for (int64_t t = (k0 + kBT - 1) / kBT; t <= k1 / kBT; ++t) P.tiles[t] = pos;
                }
                pos0 += __popc(tm);
                e0 += __shfl_sync(FULL, inc, 31);
            }
            if (lane == 0) {
                C->list = ((unsigned long long)pos0 << P.ebits) | e0;
                C->ilist = 0;
                C->cand[0] = 0;
                C->dyn[0] = C->dyn[1] = 0;
                C->salloc[0] = C->salloc[1] = 0;
            }
        }
        unsigned ph = 0;  // edge passes of this batch so far (selects the dynamic-tile counter)
        const bool tr = b == P.trace_b && cta0;
        if (tr && cta0 && tid == 0) P.gctr->trace_n = 0;
        bsync(C, gen, ncta);
        btrace(P, tr, 0, 0, 0, 0, 0, 0);
        Lv cur{0, (int64_t)(ld_volatile_u64(&C->snap[0]) >> P.ebits), (int64_t)(ld_volatile_u64(&C->snap[0]) & emask), 0};
        if (cur.N == 0) continue;  // every lane invalid: nothing was written
        if (cta0 && tid == 0) {
            int64_t *l = P.lvl;
            l[0] = cur.p0; l[1] = cur.N; l[2] = cur.E; l[3] = cur.tb;
        }
        Lv prev{0, 0, 0, 0};
        int d = 0;
        MT active = ~(MT)0;
        int64_t fwd_edges = 0, pulls = 0;
        bool overflow = false;
        for (;;) {
            // direction of level d+1 (uniform: every CTA computes it from the same snapshot)
            const bool pull = P.one_format || (d + 1 >= 2 && P.dir_mode != 1 &&
                              (P.dir_mode == 2 || (double)cur.E * P.pull_ratio > (double)P.m));
            // ---- B(d): lanes of level d -> list masks and visited; retire M_{d-1}; candidates
            BPROF_START();
            if (cta0 && tid == 0) C->list = 0;  // relative counter of level d+1 (snapshot already taken)
            {
                unsigned long long orr = 0;
                long long rc = 0, re = 0;
                MT *frd = fr[d & 1];
                for (int64_t p = gtid; p < cur.N; p += nthreads) {
                    const int32_t v = P.list_v[cur.p0 + p];
                    const MT m = frd[v];
                    list_m[cur.p0 + p] = m;
                    vis[v] |= m;
                    orr |= (unsigned long long)m;
                    rc += __popcll((unsigned long long)m);
                    re += (long long)__popcll((unsigned long long)m) * P.deg2[v].x;
                }
                orr = (unsigned long long)__reduce_or_sync(FULL, (unsigned)orr) |
                      ((unsigned long long)__reduce_or_sync(FULL, (unsigned)(orr >> 32)) << 32);
                rc = __reduce_add_sync(FULL, (unsigned)rc);
                for (int k = 16; k >= 1; k >>= 1) re += __shfl_xor_sync(FULL, re, k);
                if (lane == 0) {
                    if (orr) atomicOr((unsigned long long *)&C->ilist, orr);
                    if (rc) atomicAdd((unsigned long long *)&C->st_reached, (unsigned long long)rc);
                    if (re) atomicAdd((unsigned long long *)&C->st_reached_edges, (unsigned long long)re);
                }
                if (d >= 1) {
                    MT *frp = fr[(d + 1) & 1];
                    for (int64_t p = gtid; p < prev.N; p += nthreads) frp[P.list_v[prev.p0 + p]] = 0;
                }
                if (pull) {  // candidates: vertices with in-edges and an unvisited active lane
                    const BOut co{&C->cand[0], P.cand_v, P.cand_pre, P.cand_beg, P.cand_tiles, P.n + kPad,
                                  P.cand_tiles_cap, &C->ovf};
                    for (int64_t base = gwarp * kBT; base < P.n_scan; base += nwarps * kBT) {
                        bool tk[kBI];
                        int32_t vv[kBI];
                        uint32_t dg[kBI], bg[kBI];
#pragma unroll
                        for (int i = 0; i < kBI; ++i) {
                            const int64_t w = base + i * 32 + lane;
                            vv[i] = (int32_t)w;
                            tk[i] = w < P.n_scan && (~vis[w] & active) != (MT)0;
                            dg[i] = 0;
                            bg[i] = 0;
                            if (tk[i]) {
                                span(P.in_ptr, vv[i], dg[i], bg[i]);
                                tk[i] = dg[i] > 0;
                            }
                        }
                        bappend(tk, vv, dg, bg, co, P.ebits);
                    }
                }
            }
            BPROF(BR_BPHASE);
            bsync(C, gen, ncta);
            btrace(P, tr, 1, d, cur.N, cur.E, pull, 0);
            active = (MT)ld_volatile_u64(&C->snap[1]);
            const unsigned long long cs = ld_volatile_u64(&C->snap[2]);
            // ---- A(d+1)
            if (cta0 && tid == 0) {
                C->cand[0] = 0;
                C->ilist = 0;
            }
            Lv nxt{cur.p0 + cur.N, 0, 0, cur.tb + cdiv(cur.N + cur.E, kBT)};
            const BOut lo{&C->list, P.list_v + nxt.p0, P.list_pre + nxt.p0, P.list_beg + nxt.p0, P.tiles + nxt.tb,
                          P.list_cap - nxt.p0, P.tiles_cap - nxt.tb, &C->ovf};
            MT *fro = fr[(d + 1) & 1];
            if (cta0 && tid == 0) C->dyn[(ph + 1) & 1] = 0;  // the next pass's counter (its last user is done)
            if (pull) {
                const int64_t cN = (int64_t)(cs >> P.ebits), cE = (int64_t)(cs & emask);
                bpass<B_PULL, W>(P, ws, P.cand_v, P.cand_pre, P.cand_beg, nullptr, P.cand_tiles, cN, cE, P.in_idx,
                              fr[d & 1], fro, (unsigned long long)active, gwarp, nwarps, lo, &C->dyn[ph & 1]);
                fwd_edges += cE;
                ++pulls;
            } else {
                bpass<B_PUSH, W>(P, ws, P.list_v + cur.p0, P.list_pre + cur.p0, P.list_beg + cur.p0, list_m + cur.p0,
                              P.tiles + cur.tb, cur.N, cur.E, P.out_idx, nullptr, fro, 0u, gwarp, nwarps, lo,
                              &C->dyn[ph & 1]);
                fwd_edges += cur.E;
            }
            ++ph;
            bsync(C, gen, ncta);
            if (*(volatile unsigned *)&C->ovf) {  // level d+1 did not fit (uniform: read after the barrier)
                overflow = true;
                break;
            }
            {
                const unsigned long long lv = ld_volatile_u64(&C->snap[0]);
                nxt.N = (int64_t)(lv >> P.ebits);
                nxt.E = (int64_t)(lv & emask);
            }
            btrace(P, tr, pull ? 3 : 2, d + 1, nxt.N, nxt.E, pull ? (int64_t)(cs >> P.ebits) : cur.N,
                   pull ? (int64_t)(cs & emask) : cur.E);
            if (nxt.N == 0) break;
            ++d;
            if (cta0 && tid == 0) {
                int64_t *l = P.lvl + 4 * (int64_t)d;
                l[0] = nxt.p0; l[1] = nxt.N; l[2] = nxt.E; l[3] = nxt.tb;
            }
            if (d > P.n + 1) __trap();  // impossible for a correct BFS: fail loudly, never spin
            prev = cur;
            cur = nxt;
        }
        bool split_ovf = false;  // the split accumulator, not a level list, was outgrown (no list growth)
        if (IP && !overflow && !P.bfs_depth && !P.fwd_only) {
            // in-place backward: split lanes per level and level D's accumulator offsets; a sweep whose
            // largest level needs more than the accumulator holds is re-run in halves (nothing of the
            // backward has been written yet)
            bsplit_count<W>(P, d, gwarp, nwarps);
            bsync(C, gen, ncta);
            __shared__ int s_sovf;
            if (tid == 0) {
                long long mx = 0;
                for (int L = 1; L <= d; ++L) mx = max(mx, (long long)ld_volatile_u64((const unsigned long long *)&P.scnt[L]));
                s_sovf = mx > P.sacc_cap;
                if (cta0 && (unsigned long long)mx > C->split_need) C->split_need = (unsigned long long)mx;
            }
            __syncthreads();
            overflow = s_sovf != 0;
            split_ovf = overflow;
            __syncthreads();
        }
        if (overflow) {
            // drop the lane set's partial forward state (grid-wide, no list needed), then run its halves
            for (int64_t i = gtid; i < P.n * W; i += nthreads) P.sig[i] = 0.0;
            for (int64_t i = gtid; i < P.n; i += nthreads) {
                vis[i] = 0;
                fr[0][i] = 0;
                fr[1][i] = 0;
            }
            bsync(C, gen, ncta);
            if (cta0 && tid == 0) {  // every CTA has read the flag (before the barrier above)
                C->ovf = 0;
                C->st_overflows += 1;
                if (!split_ovf) C->ovf_total += 1;
            }
            // split-lane counts: zeroed only after the barrier above -- every CTA has taken its
            // overflow decision from them by then (done before the re-run's next barrier)
            if (P.scnt)
                for (int64_t i = gtid; i < P.n + 2; i += nthreads) P.scnt[i] = 0;
            MT lo = 0, x = bmask;
            for (int i = __popcll((unsigned long long)bmask) / 2; i > 0; --i) {
                lo |= x & (~x + 1);
                x &= x - 1;
            }
            if (lo == 0 || npend + 2 > 8) __trap();  // one source always fits (batch_alloc)
            pend[npend++] = bmask ^ lo;
            pend[npend++] = lo;
            continue;
        }
        const int D = d;  // deepest non-empty level of the batch
        if (cta0 && tid == 0) {
            C->st_levels += D + 2;
            C->st_pull_levels += pulls;
            C->st_fwd_edges += fwd_edges;
            if (D > C->st_max_depth) C->st_max_depth = D;
            const int64_t used = nxt_p0_end(P, D);
            if (used > C->st_list_peak) C->st_list_peak = used;
        }
        if (P.bfs_depth || P.fwd_only) {  // tbc_bfs_batch (export depth / sigma) or forward-only
            for (int L = 0; L <= D; ++L) {  // measurement (TBC_OPT_STAGE): retire, next batch
                const int64_t *l = P.lvl + 4 * (int64_t)L;
                if (P.bfs_depth) bclear<W, true>(P, Lv{l[0], l[1], l[2], l[3]}, fr[L & 1], gwarp, nwarps, L, b);
                else bclear<W>(P, Lv{l[0], l[1], l[2], l[3]}, fr[L & 1], gwarp, nwarps);
            }
            if (cta0 && tid == 0) {
                C->st_scans += pulls;
                C->st_sources += valid;
            }
            bsync(C, gen, ncta);
            continue;
        }
        // ---------------- backward, L = D..1 (Alg.1 l.29-47); level L+2 retired on the way
        int64_t bwd_edges = 0;
        for (int L = D; L >= 1 && P.one_format; --L) {
            // one format (CSC only): P(L) pushes delta_u of level L+1 over its in-edges into the rows
            // of level L (masked M_{L+1}(w) & M_L(u)); O(L) finishes level L (owner pass)
            const BOut none{nullptr, nullptr, nullptr, nullptr, nullptr, 0, 0, nullptr};
            if (L < D) {
                const int64_t *l1 = P.lvl + 4 * (int64_t)(L + 1);
                const Lv lw{l1[0], l1[1], l1[2], l1[3]};
                if (cta0 && tid == 0) C->dyn[(ph + 1) & 1] = 0;
                bpass<B_BPUSH, W>(P, ws, P.list_v + lw.p0, P.list_pre + lw.p0, P.list_beg + lw.p0, list_m + lw.p0,
                                  P.tiles + lw.tb, lw.N, lw.E, P.in_idx, fr[L & 1], nullptr, 0u, gwarp, nwarps, none,
                                  &C->dyn[ph & 1]);
                ++ph;
                bwd_edges += lw.E;
                bsync(C, gen, ncta);
            }
            const int64_t *l = P.lvl + 4 * (int64_t)L;
            bowner<W>(P, Lv{l[0], l[1], l[2], l[3]}, gwarp, nwarps);
            {  // scatter M_{L-1} (P(L-1)'s in-neighbour masks) and drop M_{L+1}: the same parity array
                const int64_t *lp = P.lvl + 4 * (int64_t)(L - 1);
                for (int64_t p = gtid; p < lp[1]; p += nthreads) atomicOr(&fr[(L - 1) & 1][P.list_v[lp[0] + p]], list_m[lp[0] + p]);
                if (L + 1 <= D) {
                    const int64_t *ln = P.lvl + 4 * (int64_t)(L + 1);
                    for (int64_t p = gtid; p < ln[1]; p += nthreads)
                        atomicAnd(&fr[(L + 1) & 1][P.list_v[ln[0] + p]], ~list_m[ln[0] + p]);
                }
            }
            if (L + 2 <= D) {
                const int64_t *l2 = P.lvl + 4 * (int64_t)(L + 2);
                bclear<W, false, IP>(P, Lv{l2[0], l2[1], l2[2], l2[3]}, fr[L & 1], gwarp, nwarps);
            }
            bsync(C, gen, ncta);
            btrace(P, tr, 4, L, l[1], l[2], 0, 0);
        }
        for (int L = D; L >= 1 && !P.one_format; --L) {
            const int64_t *l = P.lvl + 4 * (int64_t)L;
            const Lv lv{l[0], l[1], l[2], l[3]};
            const BOut none{nullptr, nullptr, nullptr, nullptr, nullptr, 0, 0, nullptr};
            if (cta0 && tid == 0) {
                C->dyn[(ph + 1) & 1] = 0;  // the next pass's counter (its last user is done)
                if (IP) C->salloc[(L + 1) & 1] = 0;  // for level L-1's offsets (bsplit_fin)
            }
            bpass<B_BWD, W, IP>(P, ws, P.list_v + lv.p0, P.list_pre + lv.p0, P.list_beg + lv.p0, list_m + lv.p0,
                         P.tiles + lv.tb, lv.N, lv.E, P.out_idx, fr[(L + 1) & 1], fr[L & 1], 0u, gwarp, nwarps, none,
                         &C->dyn[ph & 1], IP ? ((L & 1) ? P.cand_beg : P.cand_pre) : nullptr,
                         IP ? P.sacc + (L & 1) * P.sacc_cap : nullptr);
            ++ph;
            bwd_edges += lv.E;
            if (L + 2 <= D) {
                BPROF_START();
                const int64_t *l2 = P.lvl + 4 * (int64_t)(L + 2);
                bclear<W, false, IP>(P, Lv{l2[0], l2[1], l2[2], l2[3]}, fr[L & 1], gwarp, nwarps);
                BPROF(BR_CLEAR);
            }
            bsync(C, gen, ncta);
            btrace(P, tr, 4, L, lv.N, lv.E, 0, 0);
            if (IP) {
                bsplit_fin<W>(P, L, gwarp, nwarps);
                bsync(C, gen, ncta);
            }
        }
        // retire levels 0..min(2, D)
        for (int L = 0; L <= min(2, D); ++L) {
            const int64_t *l = P.lvl + 4 * (int64_t)L;
            bclear<W, false, IP>(P, Lv{l[0], l[1], l[2], l[3]}, fr[L & 1], gwarp, nwarps);
        }
        if (P.scnt)
            for (int64_t L = gtid + 1; L <= D; L += nthreads) P.scnt[L] = 0;
        if (cta0 && tid == 0) {
            C->st_bwd_edges += bwd_edges;
            C->st_scans += pulls;
            C->st_sources += valid;
        }
        bsync(C, gen, ncta);
        btrace(P, tr, 5, 0, 0, 0, 0, 0);
      }
    }
#ifdef TBC_PROF
    if ((tid & 31) == 0) {
        unsigned long long busy = 0;
        for (int r = 0; r < BR_OTHER; ++r) busy += tbc_bprof[tid >> 5][r];
        for (int r = BR_WIN; r <= BR_OEPI; ++r) busy += tbc_bprof[tid >> 5][r];
        tbc_bprof[tid >> 5][BR_OTHER] = clock64() - t_kernel0 - busy;
        for (int r = 0; r < BR_SLOTS; ++r) atomicAdd(&P.gctr->prof[r], tbc_bprof[tid >> 5][r]);
    }
#endif
}

}  // namespace

// ------------------------------------------------------------------ host side

static int64_t batch_ws_bytes(const tbc_graph *g, int W, bool inplace);

// in-place backward (TBC_OPT_BATCH_INPLACE): forced, or auto when the separate delta_u rows would not
// fit 85 % of the free memory (with the workspaces already held); settled once per graph
static bool batch_inplace(tbc_graph *g, int W) {
    if (!g->out_idx) return false;  // one format: the backward pushes into separate accumulators
    if (g->binplace >= 0) return g->binplace == 1;
    if (g->binplace_eff < 0) {
        size_t fr = 0, tot = 0;
        double have = cudaMemGetInfo(&fr, &tot) == cudaSuccess ? 0.85 * (double)fr : 0.0;
        for (int q = 0; q < kMaxPartitions; ++q) have += g->bws[q].ready ? (double)g->bws[q].bytes : 0.0;
        g->binplace_eff = (double)batch_ws_bytes(g, W, false) > have ? 1 : 0;
    }
    return g->binplace_eff == 1;
}

static tbc_status batch_alloc(tbc_graph *g, int q, int W) {
    BatchWorkspace &w = g->bws[q];
    if (w.ready && w.width == W) return TBC_OK;
    if (w.ready) batch_free_one(g, q);  // other width: reallocate
    const int64_t n = g->n, m = g->m;
    const int64_t nw = W / 32;  // 32-bit words per mask
    cudaStream_t s = g->stream;
    cudaError_t e = cudaSuccess;
    auto alloc = [&](auto **p, size_t cnt) -> cudaError_t {
        size_t bytes = sizeof(**p) * (cnt > 0 ? cnt : 1);
        cudaError_t r = cudaMalloc((void **)p, bytes);
        if (r == cudaSuccess) w.bytes += bytes;
        return r;
    };
    // level lists: a batch uses one entry per (vertex, level) with any of its sources on it -- at most
    // W n, but about n on low-diameter graphs (cfg 3: 1.07 n); sized at blist_factor n (>= n: one
    // source always fits) and grown by the next call after a sweep overflowed (k_bcb re-runs it in
    // halves).  Tile starts: <= (entries + their out-edges) / kBT + one partial tile per level.
    w.width = W;
    const int64_t f = g->blist_factor < W ? g->blist_factor : W;
    w.list_cap = f * n + kPad;
    w.tiles_cap = (w.list_cap + f * m) / kBT + n + 2 + kPad;
    w.cand_tiles_cap = (n + m) / kBT + 2 + kPad;
    // sigma and delta_u share one [n][W] array (the backward overwrites sigma in place); the owners
    // whose out-edges span several tiles sum their partial accumulators in sacc first, f n values per
    // level parity (grown with the lists; a sweep that needs more is re-run in halves)
    const bool inplace = batch_inplace(g, W);
    w.sacc_cap = inplace ? (g->bsacc_cap ? g->bsacc_cap : W * n / 16) + kPad : 0;
    if ((e = alloc(&w.sig, (size_t)n * W)) || (!inplace && (e = alloc(&w.du, (size_t)n * W))) ||
        (inplace && (e = alloc(&w.sacc, 2 * (size_t)w.sacc_cap))) || (inplace && (e = alloc(&w.scnt, n + 2))) ||
        (e = alloc(&w.vis, n * nw)) ||
        (e = alloc(&w.fr[0], n * nw)) || (e = alloc(&w.fr[1], n * nw)) || (e = alloc(&w.list_v, w.list_cap)) ||
        (e = alloc(&w.list_pre, w.list_cap)) || (e = alloc(&w.list_beg, w.list_cap)) ||
        (e = alloc(&w.list_m, w.list_cap * nw)) || (e = alloc(&w.tiles, w.tiles_cap)) ||
        (e = alloc(&w.cand_v, n + kPad)) || (e = alloc(&w.cand_pre, n + kPad)) || (e = alloc(&w.cand_beg, n + kPad)) ||
        (e = alloc(&w.cand_tiles, w.cand_tiles_cap)) || (e = alloc(&w.lvl, 4 * (n + 2))) || (e = alloc(&w.ctr, 1))) {
        g->device_bytes += w.bytes;
        batch_free_one(g, q);  // release the arrays that were allocated (no leak, device_bytes exact)
        return cuda_error(e, "batch workspace cudaMalloc");
    }
    g->device_bytes += w.bytes;
    if ((e = cudaMemsetAsync(w.sig, 0, sizeof(double) * n * W, s)) ||
        (w.du && (e = cudaMemsetAsync(w.du, 0, sizeof(double) * n * W, s))) ||
        (w.sacc && (e = cudaMemsetAsync(w.sacc, 0, sizeof(double) * 2 * w.sacc_cap, s))) ||
        (w.scnt && (e = cudaMemsetAsync(w.scnt, 0, sizeof(int64_t) * (n + 2), s))) ||
        (e = cudaMemsetAsync(w.vis, 0, sizeof(uint32_t) * n * nw, s)) ||
        (e = cudaMemsetAsync(w.fr[0], 0, sizeof(uint32_t) * n * nw, s)) ||
        (e = cudaMemsetAsync(w.fr[1], 0, sizeof(uint32_t) * n * nw, s)) ||
        (e = cudaMemsetAsync(w.ctr, 0, sizeof(Ctrs), s)) || (e = cudaStreamSynchronize(s))) {
        batch_free_one(g, q);
        return cuda_error(e, "batch workspace init");
    }
    if (!g->bgrid) {
        int per_sm = 0, sms = 0;
        for (const void *fn : {(const void *)k_bcb<32, false, false>, (const void *)k_bcb<64, false, false>,
                               (const void *)k_bcb<32, true, false>, (const void *)k_bcb<64, true, false>,
                               (const void *)k_bcb<32, false, true>, (const void *)k_bcb<64, false, true>,
                               (const void *)k_bcb<32, true, true>, (const void *)k_bcb<64, true, true>})
            if ((e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBSmem)))
                return cuda_error(e, "batch smem attribute");
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void *)k_bcb<64, true, true>, kBB, kBSmem)) ||
            (e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device)))
            return cuda_error(e, "batch occupancy query");
        if (per_sm < 1) return set_error(TBC_ERR_CUDA, "k_bcb cannot be resident (occupancy 0)");
        g->bgrid = per_sm * sms;
    }
    w.ready = true;
    return TBC_OK;
}

void batch_free_one(tbc_graph *g, int q) {
    BatchWorkspace &w = g->bws[q];
    if (w.ctr) {  // keep the partition's accumulated statistics (tbc_stats) across a reallocation
        Ctrs c;
        if (cudaMemcpy(&c, w.ctr, sizeof c, cudaMemcpyDeviceToHost) == cudaSuccess) {
            g->retired.st_sources += c.st_sources;
            g->retired.st_reached += c.st_reached;
            g->retired.st_reached_edges += c.st_reached_edges;
            g->retired.st_fwd_edges += c.st_fwd_edges;
            g->retired.st_bwd_edges += c.st_bwd_edges;
            g->retired.st_levels += c.st_levels;
            g->retired.st_pull_levels += c.st_pull_levels;
            g->retired.st_scans += c.st_scans;
            g->retired.st_overflows += c.st_overflows;
            g->retired.bad_sources += c.bad_sources;
            if (c.st_max_depth > g->retired.st_max_depth) g->retired.st_max_depth = c.st_max_depth;
            if (c.st_list_peak > g->retired.st_list_peak) g->retired.st_list_peak = c.st_list_peak;
        }
        (void)cudaGetLastError();
    }
    void *ps[] = {w.sig, w.du, w.sacc, w.scnt, w.vis, w.fr[0], w.fr[1], w.list_v, w.list_pre, w.list_beg, w.list_m, w.tiles,
                  w.cand_v, w.cand_pre, w.cand_beg, w.cand_tiles, w.lvl, w.ctr};
    for (void *p : ps) cudaFree(p);
    g->device_bytes -= w.bytes;
    w = BatchWorkspace{};
    // the partition's overflow total restarts with its counters (after cudaFree: a copy still in
    // flight from the last launch has landed by now)
    if (g->h_bovf) g->h_bovf[q] = g->h_bovf[kMaxPartitions + q] = 0;
    g->bovf_seen[q] = 0;
}

void batch_free(tbc_graph *g) {
    for (int q = 0; q < kMaxPartitions; ++q) batch_free_one(g, q);
    cudaFree(g->border.keys);
    cudaFree(g->border.temp);
    g->border = BatchOrder{};
}

// auto width (measured with grouped sources): 64 sources per sweep up to 8 M
// vertices (faster on RMAT 18, Kronecker 22 and the mycielski graphs) and above it for average
// degree >= 8 while the W = 64 workspace fits 85 % of the free memory (Kronecker 25: 400 vs 389
// GTEPS), else 32 (the 16 M-vertex lattice: 2.03 vs 1.91, at half the workspace).  The choice is
// made once per graph (a later change in free memory cannot flip it and reallocate), and falls
// back to 32 if the W = 64 workspace then fails to allocate (batch_run).
static int64_t batch_ws_bytes(const tbc_graph *g, int W, bool inplace) {  // batch_alloc's sizes, one partition
    const int64_t n = g->n, m = g->m, nw = W / 32;
    const int64_t f = g->blist_factor < W ? g->blist_factor : W;
    const int64_t list_cap = f * n + kPad;
    const int64_t tiles_cap = (list_cap + f * m) / kBT + n + 2 + kPad;
    const int64_t sacc = 2 * 8 * (g->bsacc_cap ? g->bsacc_cap : W * n / 16);
    const int64_t rows = inplace ? 8 * W * n + sacc + 8 * n : 16 * W * n;  // in place: + sacc, scnt
    return rows + 12 * n * nw + list_cap * (12 + 4 * nw) + 4 * tiles_cap + 16 * (n + kPad) +
           4 * ((n + m) / kBT + 2 + kPad) + 32 * (n + 2) + (int64_t)sizeof(Ctrs);
}

int batch_width(const tbc_graph *g) {
    if (g->batch_width) return g->batch_width;
    if (g->auto_width) return g->auto_width;
    const int64_t n = g->n, m = g->m;
    if (n <= (8ll << 20)) return 64;
    if (m < 8 * n) return 32;
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) return 32;
    double have = 0.85 * (double)fr;
    for (int q = 0; q < kMaxPartitions; ++q) have += g->bws[q].ready ? (double)g->bws[q].bytes : 0.0;
    return (double)batch_ws_bytes(g, 64, g->binplace == 1) <= have ? 64 : 32;
}

// source grouping key of each source (one warp per source): its 2-hop out-volume V = sum of the
// out-degrees of its out-neighbours, in classes floor(4 log2(V + 1)) (bits 31..24), then its own
// out-degree (bits 23..0); value = internal label.  Out-of-range entries get (0, INT32_MAX) and
// are counted as bad sources by the kernel.
__global__ void k_source_keys(int64_t k, int64_t n, const int32_t *__restrict__ src, const int32_t *__restrict__ perm,
                              const int2 *__restrict__ deg2, const int64_t *__restrict__ out_ptr,
                              const int32_t *__restrict__ out_idx, uint32_t *keys, int32_t *vals) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); i < k; i += nw) {
        const int32_t sc = src[i];
        if (sc < 0 || sc >= n) {
            if (lane == 0) {
                keys[i] = 0;
                vals[i] = INT32_MAX;
            }
            continue;
        }
        const int32_t v = perm ? perm[sc] : sc;
        unsigned long long vol = 0;
        if (out_idx)  // one-format graphs (no CSR): the out-degree alone
            for (int64_t e = out_ptr[v] + lane; e < out_ptr[v + 1]; e += 32) vol += (unsigned)deg2[out_idx[e]].x;
#pragma unroll
        for (int o = 16; o >= 1; o >>= 1) vol += __shfl_xor_sync(0xffffffffu, vol, o);
        if (lane == 0) {
            const uint32_t cls = (uint32_t)floorf(4.0f * log2f((float)vol + 1.0f));
            const uint32_t od = (uint32_t)min(deg2[v].x, 0xFFFFFF);
            keys[i] = (min(cls, 255u) << 24) | od;
            vals[i] = v;
        }
    }
}

// Group the call's sources by their 2-hop out-volume class (then out-degree) before cutting them
// into batches of W: bc is a sum over sources, so the batches' composition is free, and sources with
// similar fan-out have similar level profiles, so each vertex sits on fewer distinct levels per batch
// (fewer list entries and edge visits; measured +60 % GTEPS on Kronecker 22)
static tbc_status batch_group_sources(tbc_graph *g, const int32_t *d_sources, int64_t k, cudaStream_t stream,
                                      const int32_t **grouped) {
    BatchOrder &o = g->border;
    cudaError_t e = cudaSuccess;
    size_t tb = 0;
    if ((e = cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, (uint32_t *)nullptr, (uint32_t *)nullptr,
                                                       (int32_t *)nullptr, (int32_t *)nullptr, (int)k, 0, 32, stream)))
        return cuda_error(e, "source grouping (size query)");
    if (k > o.cap || tb > o.temp_bytes) {
        cudaFree(o.keys);
        cudaFree(o.temp);
        o = BatchOrder{};
        const int64_t cap = k + 1024;
        size_t need = 0;
        if ((e = cub::DeviceRadixSort::SortPairsDescending(nullptr, need, (uint32_t *)nullptr, (uint32_t *)nullptr,
                                                           (int32_t *)nullptr, (int32_t *)nullptr, (int)cap, 0, 32,
                                                           stream)))
            return cuda_error(e, "source grouping (size query)");
        need = need > tb ? need : tb;
        if ((e = cudaMalloc(&o.keys, (size_t)cap * 16)) || (e = cudaMalloc(&o.temp, need)))
            return cuda_error(e, "source grouping cudaMalloc");
        o.cap = cap;
        o.temp_bytes = need;
    }
    uint32_t *k0 = (uint32_t *)o.keys, *k1 = k0 + o.cap;
    int32_t *v0 = (int32_t *)(k1 + o.cap), *v1 = v0 + o.cap;
    const int blocks = (int)((k + 7) / 8 < 4096 ? (k + 7) / 8 : 4096);  // 8 warps per block
    k_source_keys<<<blocks, 256, 0, stream>>>(k, g->n, d_sources, g->perm, g->deg2, g->out_ptr, g->out_idx, k0, v0);
    size_t tbytes = o.temp_bytes;
    if ((e = cudaGetLastError()) ||
        (e = cub::DeviceRadixSort::SortPairsDescending(o.temp, tbytes, k0, k1, v0, v1, (int)k, 0, 32, stream)))
        return cuda_error(e, "source grouping");
    *grouped = v1;
    return TBC_OK;
}

// auto partitions (measured): wide-level graphs -- sigma rows beyond 1 GiB with
// average degree >= 8 (Kronecker 22/25), or average degree >= 64 (mycielski) -- keep the whole GPU
// on one batch; the others (RMAT 18, high-diameter lattices) run up to 8 batches side by side, as
// many as fit in 80 % of the free device memory
static int batch_auto_parts(tbc_graph *g, int W) {
    const int64_t n = g->n, m = g->m;
    if ((n * 32ll * 16 > (1ll << 30) && m >= 8 * n) || m >= 64 * n) return 1;
    const int cap = m >= 8 * n ? 4 : kMaxPartitions;  // RMAT 18: 4 beats 8; lattices: 8
    const double per = (double)batch_ws_bytes(g, W, g->out_idx && (g->binplace == 1 || g->binplace_eff == 1));
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) return 1;
    double have = 0.8 * (double)fr;
    for (int q = 0; q < kMaxPartitions; ++q) have += g->bws[q].ready ? (double)g->bws[q].bytes : 0.0;
    int np = 1;
    while (np < cap && (np * 2) * per <= have) np *= 2;
    return np;
}

tbc_status batch_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                     int32_t *bfs_depth, double *bfs_sigma) {
    int W = batch_width(g);
    const int32_t *src = d_sources;
    {  // sweeps of earlier calls that outgrew the level lists: grow them (x2) before this call
        bool grew = false;
        for (int q = 0; q < kMaxPartitions; ++q) grew |= g->h_bovf && g->h_bovf[q] > g->bovf_seen[q];
        if (grew && g->blist_factor < W) {
            g->blist_factor *= 2;
            for (int q = 0; q < kMaxPartitions; ++q) batch_free_one(g, q);  // reallocated below
        }
        for (int q = 0; q < kMaxPartitions; ++q) g->bovf_seen[q] = g->h_bovf ? g->h_bovf[q] : 0;
        // a level of an earlier call needed more split-accumulator values than allocated: resize
        // (to the largest need x 5/4, never shrinking) the partitions that were short
        int64_t need = 0;
        for (int q = 0; q < kMaxPartitions; ++q)
            if (g->h_bovf && g->bws[q].ready && g->bws[q].sacc &&
                (int64_t)g->h_bovf[kMaxPartitions + q] > g->bws[q].sacc_cap - kPad)
                need = std::max(need, (int64_t)g->h_bovf[kMaxPartitions + q]);
        if (need > 0) {
            g->bsacc_cap = std::max(g->bsacc_cap, need + need / 4 + 1024);
            for (int q = 0; q < kMaxPartitions; ++q)
                if (g->bws[q].ready && g->bws[q].sacc && g->bws[q].sacc_cap - kPad < g->bsacc_cap) batch_free_one(g, q);
        }
    }
    // tbc_bfs_batch exports per list index: batches are cut from the list as given
    const bool grouped = g->batch_order && k > 1 && k < (1ll << 31) && !bfs_depth;
    if (grouped) {
        tbc_status st = batch_group_sources(g, d_sources, k, stream, &src);
        if (st != TBC_OK) return st;
    }
    if (!g->batch_width && !g->auto_width) {  // settle the auto width once, with an OOM fallback
        tbc_status st = batch_alloc(g, 0, W);
        if (st == TBC_ERR_OOM && W == 64) {
            (void)cudaGetLastError();
            W = 32;
            st = batch_alloc(g, 0, W);
        }
        if (st != TBC_OK) return st;
        g->auto_width = W;
    }
    const int64_t nb = (k + W - 1) / W;
    int np = g->batch_parts ? g->batch_parts : batch_auto_parts(g, W);
    if (np > nb) np = (int)nb;
    if (np < 1) np = 1;
    for (int q = 0; q < np; ++q) {
        tbc_status st = batch_alloc(g, q, W);
        if (st == TBC_ERR_OOM && q > 0) {  // run on the partitions that fit
            (void)cudaGetLastError();
            np = q;
            break;
        }
        if (st != TBC_OK) return st;
    }
    if (np > g->bgrid) np = g->bgrid;
    static_assert(sizeof(BParamSet) <= 32000, "kernel parameter space");
    BParamSet S{};
    S.nparts = np;
    S.cta_per_part = g->bgrid / np;
    for (int q = 0; q < np; ++q) {
        const BatchWorkspace &w = g->bws[q];
        BParams &P = S.p[q];
        P.n = g->n;
        P.m = g->m;
        P.in_ptr = g->in_ptr;
        P.in_idx = g->in_idx;
        P.out_ptr = g->out_ptr;
        P.out_idx = g->out_idx;
        P.deg2 = g->deg2;
        P.sig = w.sig;
        P.du = w.du ? w.du : w.sig;
        P.sacc = w.sacc;
        P.scnt = w.scnt;
        P.sacc_cap = w.sacc_cap;
        P.inplace = w.du ? 0 : 1;
        P.vis = w.vis;
        P.fr0 = w.fr[0];
        P.fr1 = w.fr[1];
        P.list_v = w.list_v;
        P.list_pre = w.list_pre;
        P.list_beg = w.list_beg;
        P.list_m = w.list_m;
        P.tiles = w.tiles;
        P.cand_v = w.cand_v;
        P.cand_pre = w.cand_pre;
        P.cand_beg = w.cand_beg;
        P.cand_tiles = w.cand_tiles;
        P.lvl = w.lvl;
        P.ctr = w.ctr;
        P.gctr = g->gctr;
        P.bc = d_bc;  // shared by the partitions: every bc update is an fp64 atomic add
        P.sources = src;
        P.src_internal = grouped ? 1 : 0;
        P.perm = g->perm;
        P.inv = g->inv;
        P.k = k;
        P.n_scan = g->n_scan;
        P.list_cap = w.list_cap;
        P.tiles_cap = w.tiles_cap;
        P.cand_tiles_cap = w.cand_tiles_cap;
        P.bc_scale = g->directed ? 1.0 : 0.5;
        P.pull_ratio = g->batch_pull;
        P.ebits = g->ebits;
        P.dir_mode = g->dir_mode;
        P.trace = g->trace;
        P.trace_cap = g->trace ? kTraceCap : 0;
        P.trace_b = g->trace_src >= 0 ? g->trace_src / W : -1;
        P.bfs_depth = bfs_depth;
        P.bfs_sigma = bfs_sigma;
        P.fwd_only = g->stage == 1;
        P.one_format = g->out_idx == nullptr ? 1 : 0;
        P.adj_ptr = P.one_format ? g->in_ptr : g->out_ptr;
    }
    g->last_width = W;
    g->last_parts = np;
    void *args[] = {&S};
    const bool ip = S.p[0].inplace != 0;
    const void *fn = ip ? (np > 1 ? (W == 64 ? (const void *)k_bcb<64, true, true> : (const void *)k_bcb<32, true, true>)
                                  : (W == 64 ? (const void *)k_bcb<64, false, true> : (const void *)k_bcb<32, false, true>))
                        : (np > 1 ? (W == 64 ? (const void *)k_bcb<64, true, false> : (const void *)k_bcb<32, true, false>)
                                  : (W == 64 ? (const void *)k_bcb<64, false, false> : (const void *)k_bcb<32, false, false>));
    cudaError_t e = cudaLaunchCooperativeKernel(fn, dim3(S.cta_per_part * np), dim3(kBB), args, kBSmem, stream);
    if (e != cudaSuccess) return cuda_error(e, "cudaLaunchCooperativeKernel(k_bcb)");
    if (!g->h_bovf && (e = cudaMallocHost(&g->h_bovf, sizeof(unsigned long long) * 2 * kMaxPartitions)) == cudaSuccess)
        for (int q = 0; q < 2 * kMaxPartitions; ++q) g->h_bovf[q] = 0;
    (void)cudaGetLastError();
    if (g->h_bovf)  // overflow totals, read by the next call (no synchronisation here)
        for (int q = 0; q < np; ++q)
            if ((e = cudaMemcpyAsync(&g->h_bovf[q], &g->bws[q].ctr->ovf_total, sizeof(unsigned long long),
                                     cudaMemcpyDeviceToHost, stream)) ||
                (e = cudaMemcpyAsync(&g->h_bovf[kMaxPartitions + q], &g->bws[q].ctr->split_need,
                                     sizeof(unsigned long long), cudaMemcpyDeviceToHost, stream)))
                return cuda_error(e, "overflow counter copy");
    return TBC_OK;
}

}  // namespace tbc
