// tbc_engine.cu -- the per-source hot path of TurboBC (Algorithm 1) as one
// persistent, cooperative sm_100a kernel per tbc_bc call (all sources, all levels).
//
//   forward  (Alg.1 l.11-28): level-synchronous masked SpMV.  Each level is either
//            PUSH  -- the frontier (level d-1 list) scatters sigma along its out-edges (CSR);
//                     the fp64 atomic that lifts sigma(x) from 0 claims x for level d, or
//            PULL  -- every still-undiscovered candidate sums sigma over its in-edges (CSC)
//                     from the frontier: the masked f_t = A^T f of l.19-22 / Alg.3,
//                     then an owner pass applies the mask of l.20-25 (discovered iff sum > 0).
//            Direction per level: frontier out-edges vs candidate in-edges.
//   backward (Alg.1 l.29-47): for L = D..1 an edge pass sums delta_u of the
//            out-neighbours on level L+1 (A delta_u, reading R1) into acc(v), then an owner
//            pass sets delta = sigma * acc, bc += delta (x 1/2 undirected) and
//            delta_u = (1+delta)/sigma (l.35), and resets the vertex for the next source.
//
// Edge passes are merge-path passes over (owner list, adjacency): the diagonal of (owner end
// items + edges) is cut into warp tiles of kWT items, so a 600k-edge hub and a million
// degree-1 vertices cost the same per tile.  The producer of a list writes the start owner of
// every tile while appending (warp_append), so no search is needed, and tiles are dealt to
// warps round-robin (equal items per tile => balanced).  Phases are separated by a grid
// barrier inside the kernel: no host round trip per level (cf. the paper's per-level kernels
// and host loop).
#include <cstdio>

#include "tbc_internal.cuh"
#include "tbc_device.cuh"

namespace tbc {
namespace {

constexpr unsigned FULL = 0xffffffffu;

#ifdef TBC_DEBUG
#define TBC_CHECK(cond, ...)                                                           \
    do {                                                                               \
        if (!(cond)) {                                                                 \
            printf("TBC_CHECK failed %s:%d (%s) ", __FILE__, __LINE__, #cond);          \
            printf(__VA_ARGS__);                                                       \
            printf("\n");                                                              \
            __trap();                                                                  \
        }                                                                              \
    } while (0)
#else
#define TBC_CHECK(cond, ...) ((void)0)
#endif
// PUSH/PULL: forward level; BWD: backward level pulled over the owners' out-edges;
// BPUSH: backward level pushed from level L+1 over its in-edges (fp64 atomics into level L)
enum { MODE_PUSH = 0, MODE_PULL = 1, MODE_BWD = 2, MODE_BPUSH = 3 };

constexpr int kLaneItems = TBC_LANE_ITEMS;  // items per lane per warp tile
constexpr int kWT = 32 * kLaneItems;   // diagonal items per warp tile
constexpr int kWarpsPerBlock = kBlock / 32;

constexpr int kListPad = 8;  // spare entries at the end of every list array
// per-warp slice of shared memory (owner window of one tile; reused as append buffers)
struct __align__(16) WarpSmem {
    int64_t beg[kWT + 2];    // adjacency position of the owner's first in-tile edge
    double val[kWT + 2];     // PUSH: owner sigma; PULL/BWD: owner partial sum
    int32_t first[kWT + 2];  // slot of the owner's first in-tile edge (+ sentinel = ne)
    int32_t own[kWT + 2];    // owner (window index) of each edge slot
    int32_t v[kWT + 2];      // owner vertex id
};
constexpr size_t kSmemBytes = sizeof(WarpSmem) * kWarpsPerBlock;

// ------------------------------------------------------------------ region profiler (TBC_PROF)
// Diagnostic builds only: lane 0 of every warp adds clock64 deltas per code region into a
// per-warp shared-memory row; the rows are summed into gctr->prof at the end of the kernel.
enum {
    PR_BARRIER = 0, PR_EDGE = 1,  // PR_EDGE + 4 * MODE + {0 window, 1 index issue, 2 gather/op, 3 tail}
    PR_STREAM = 17,               // + MODE (PUSH, PULL, BWD)
    PR_PULL_OWNER = 20, PR_SCAN = 21, PR_BWD_OWNER = 22, PR_OTHER = 23, PR_SLOTS = 24
};
#ifdef TBC_PROF
__shared__ unsigned long long tbc_sprof[kWarpsPerBlock][PR_SLOTS];
#define PROF_START() unsigned long long _pt = clock64()
#define PROF(slot)                                                              \
    do {                                                                        \
        const unsigned long long _n = clock64();                                \
        if ((threadIdx.x & 31) == 0) tbc_sprof[threadIdx.x >> 5][(slot)] += _n - _pt; \
        _pt = _n;                                                               \
    } while (0)
#else
#define PROF_START() ((void)0)
#define PROF(slot) ((void)0)
#endif

// ------------------------------------------------------------------ memory-model helpers

// ---- TMA bulk copies (cp.async.bulk) completing on an mbarrier: the edge-stream pipeline
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_inval(uint64_t *bar) {
    asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, unsigned parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

// global -> shared bulk copy (TMA), bytes a multiple of 16, both addresses 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }

// Grid-wide barrier of the cooperative (co-resident) grid: release fence + arrival atomic,
// the last arriver bumps the generation; waiters acquire it.  The acquire-side gpu fence also
// invalidates this SM's L1, so plain loads after the barrier see other CTAs' writes.
// The last arriver also snapshots the list / candidate counters into c->snap (every CTA's
// appends are complete then): after the barrier CTAs read the snapshot, which nobody writes
// before the next barrier, while the live counters may already move (a CTA released early
// starts the next push level's appends or resets the candidate counters).
__device__ __forceinline__ void grid_sync(Ctrs *c, unsigned &gen, unsigned nblocks) {
    PROF_START();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned g0 = gen;
        fence_acq_rel();
        const unsigned arrived = atomicAdd(&c->bar_count, 1u);
        if (arrived == nblocks - 1) {
            c->bar_count = 0;
            fence_acq_rel();
            const unsigned long long s0 = ld_volatile_u64(&c->list), s1 = ld_volatile_u64(&c->ilist),
                                     s2 = ld_volatile_u64(&c->cand[0]), s3 = ld_volatile_u64(&c->cand[1]);
            c->snap[0] = s0;
            c->snap[1] = s1;
            c->snap[2] = s2;
            c->snap[3] = s3;
            fence_acq_rel();
            atomicExch(&c->bar_gen, g0 + 1);
        } else {
            const unsigned long long t0 = globaltimer_ns();
            while (ld_acquire(&c->bar_gen) == g0) {
                __nanosleep(20);
                if (globaltimer_ns() - t0 > kWatchdogNs) __trap();  // never hang the GPU
            }
        }
        fence_acq_rel();
    }
    gen += 1;
    __syncthreads();
    PROF(PR_BARRIER);
}

// ------------------------------------------------------------------ warp-aggregated append

// A list being appended to: packed counter (count << ebits) | degree_sum, the arrays, the
// level's tile table, and the level's start (list position, degree prefix).
struct ListOut {
    unsigned long long *ctr;
    int32_t *v;
    uint32_t *pre;
    uint32_t *beg;
    int32_t *tiles;  // already offset to this level's tile base
    int64_t p0, e0;  // level start within the list (list position, edge prefix)
};

// Append the entries a warp holds in registers (lane l, item i: vertex v[i], degree dg[i],
// adjacency begin bg[i], if take[i]) with ONE packed 64-bit atomic for the whole warp:
// (count << ebits) | degree_sum, so list order and degree-prefix order agree and every
// appended owner knows its merge-path span [k0, k0 + deg] inside its level: it writes the start
// owner of every tile whose first diagonal item lies in that span.  Entries are ordered
// item-major, lane-minor, so each item's stores are coalesced across the warp; the prefix is
// one warp scan per item.  Degrees of distinct vertices sum to <= m < 2^32 (engine_setup).
// All 32 lanes call this (warp-uniform control flow).
__device__ __forceinline__ void warp_append(const bool (&take)[kLaneItems], const int32_t (&v)[kLaneItems],
                                            const uint32_t (&dg)[kLaneItems], const uint32_t (&bg)[kLaneItems],
                                            const ListOut &o, int ebits) {
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    unsigned cnt = 0;
    unsigned long long esum = 0;
#pragma unroll
    for (int i = 0; i < kLaneItems; ++i) {
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
    for (int i = 0; i < kLaneItems; ++i) {
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
            TBC_CHECK(v[i] >= 0, "append v %d", v[i]);
            o.v[pp] = v[i];
            o.pre[pp] = (uint32_t)ee;
            o.beg[pp] = bg[i];
            const int64_t k0 = (ee - o.e0) + (pp - o.p0);
            const int64_t k1 = k0 + x;
            for (int64_t t = (k0 + kWT - 1) / kWT; t <= k1 / kWT; ++t) o.tiles[t] = (int32_t)(pp - o.p0);
        }
        p += __popc(msk);
        e += __shfl_sync(FULL, inc, 31);
    }
}

// degree and adjacency begin of v in a pointer array (CSC in_ptr or CSR out_ptr)
__device__ __forceinline__ void adj_span(const int64_t *ptr, int32_t v, uint32_t &dg, uint32_t &bg) {
    const int64_t b = ptr[v];
    bg = (uint32_t)b;
    dg = (uint32_t)(ptr[v + 1] - b);
}

// ------------------------------------------------------------------ level descriptors

// a BFS level: list positions [p0, p0+N) (both lists), out-edge prefix base e0 and sum E with
// its tile base, in-edge prefix base ie0 and sum IE of the in-degree list with its tile base
struct Level {
    int64_t p0, N, e0, E, tbase, ie0, IE, itbase;
};
constexpr int kLvlWords = 8;

__device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------------------------ merge-path edge pass
//
// One WARP processes one tile of kWT diagonal items with no block barrier.  Lane l owns the
// kLaneItems CONSECUTIVE edge slots [l*kLaneItems, +kLaneItems) of the tile, so its owners come
// out of the owner scan in registers and its per-owner sums are local runs; a single segmented
// warp scan over the lanes' trailing runs joins owners that straddle lanes.  Each lane keeps
// kLaneItems index loads and then kLaneItems gathers / atomics in flight.
// Owners: ov[0..N) with exclusive degree prefix opre[] (minus e0), adjacency begin obeg[],
// tile starts otiles[].  adj_idx: the traversed adjacency (CSR out-edges for PUSH/BWD, CSC
// in-edges for PULL).  d: the level being discovered (PUSH/PULL) or the owners' level (BWD).
// PULL/BWD hand each owner's sum to gacc[v]: a plain store when the whole owner lies in the
// tile, an fp64 atomic add for the (at most two) owners cut by the tile's ends.  The owner
// pass after the next barrier consumes and re-zeroes gacc.
// NOTE: ov/opre/obeg/otiles are written earlier in this same kernel (previous phases): they
// must NOT be declared __restrict__ const, or the compiler may read them through the
// non-coherent (ld.global.nc) path and see stale lines.
template <int MODE>
__device__ __forceinline__ void edge_pass(const Params &P, WarpSmem &ws, const int32_t *ov, const uint32_t *opre,
                                          const uint32_t *obeg, const int32_t *otiles, int64_t N, int64_t E,
                                          int64_t e0, const int64_t *__restrict__ adj_ptr,
                                          const int32_t *__restrict__ adj_idx, int d, int64_t gwarp, int64_t nwarps,
                                          ListOut out, ListOut out_in) {
    const int lane = threadIdx.x & 31;
    const int64_t K = N + E;
    const int64_t ntiles = ceil_div(K, kWT);
    const uint64_t pol_stream = policy_evict_first();
    PROF_START();
    for (int64_t tile = gwarp; tile < ntiles; tile += nwarps) {
        const int64_t ks = tile * kWT;
        const int64_t ke = min(ks + (int64_t)kWT, K);
        const int64_t ps = otiles[tile];
        const int64_t pe = (tile + 1 < ntiles) ? (int64_t)otiles[tile + 1] : N;
        const int64_t es = ks - ps, ee = ke - pe;
        const int nwin = (int)(min(pe, N - 1) - ps + 1);
        const int ne = (int)(ee - es);
        TBC_CHECK(nwin >= 1 && nwin <= kWT + 1 && ne >= 0 && ne <= kWT && ps >= 0 && pe <= N && ps <= pe,
                  "mode %d tile %lld/%lld N %lld E %lld ps %lld pe %lld nwin %d ne %d", MODE, (long long)tile,
                  (long long)ntiles, (long long)N, (long long)E, (long long)ps, (long long)pe, nwin, ne);

        // ---- owner window (three coalesced list reads): first in-tile slot, its adjacency position
        bool start0 = true;
        for (int j = lane; j < nwin; j += 32) {
            const int64_t pre = (int64_t)opre[ps + j] - e0;
            const int64_t f = max(pre, es);
            const int32_t v = ov[ps + j];
            TBC_CHECK(v >= 0 && v < P.n && f - es >= 0 && f - es <= kWT, "mode %d v %d f-es %lld", MODE, v,
                      (long long)(f - es));
            ws.first[j] = (int32_t)(f - es);
            ws.beg[j] = (int64_t)obeg[ps + j] + (f - pre);
            ws.v[j] = v;
            ws.own[j] = -1;
            if (MODE == MODE_PUSH) {
                ws.val[j] = P.sigma[v];
            } else if (MODE == MODE_BPUSH) {  // owner on level d+1: its delta_u, sign by parity
                const double u = P.du[v];
                ws.val[j] = ((d + 1) & 1) ? -u : u;
            } else {
                ws.val[j] = 0.0;
            }
            if (j == 0) start0 = pre >= es;  // owner 0 begins inside this tile

        }
        start0 = __shfl_sync(FULL, start0, 0);
        for (int sl = nwin + lane; sl < ne; sl += 32) ws.own[sl] = -1;
        if (lane == 0) ws.first[nwin] = ne;
        __syncwarp();
        for (int j = lane; j < nwin; j += 32)
            if (ws.first[j] < ws.first[j + 1]) ws.own[ws.first[j]] = j;
        __syncwarp();
        // owners of this lane's slots [l*kLaneItems, +kLaneItems): running max of the head marks
        int o[kLaneItems];
        {
            int run = -1;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                const int sl = lane * kLaneItems + i;
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
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                const int sl = lane * kLaneItems + i;
                o[i] = sl < ne ? max(prev, o[i]) : -1;
                if (sl < ne) ws.own[sl] = o[i];
            }
        }
        __syncwarp();

        PROF(PR_EDGE + 4 * MODE + 0);
        // ---- edges in coalesced order: slot = i*32 + lane (consecutive lanes -> consecutive entries)
        int xs[kLaneItems];
        int js[kLaneItems];
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            const int sl = i * 32 + lane;
            js[i] = -1;
            xs[i] = 0;
            if (sl < ne) {
                const int j = ws.own[sl];
                TBC_CHECK(j >= 0 && j < nwin, "mode %d own %d nwin %d sl %d", MODE, j, nwin, sl);
                js[i] = j;
                xs[i] = ld_stream(adj_idx + ws.beg[j] + (sl - ws.first[j]), pol_stream);
                TBC_CHECK(xs[i] >= 0 && xs[i] < P.n, "mode %d x %d pos %lld", MODE, xs[i],
                          (long long)(ws.beg[j] + (sl - ws.first[j])));
            }
        }
        PROF(PR_EDGE + 4 * MODE + 1);
        if (MODE == MODE_PUSH) {
            // masked scatter f_t(x) += f(u) for x on levels {-1, d} (Alg.1 l.19-25 as a push).
            // sigma is 0 off the current BFS, so the atomic that lifts sigma(x) from 0 is the
            // unique claim of x.  All kLaneItems atomics are issued before any result is used.
            int dxs[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) dxs[i] = js[i] >= 0 ? P.depth[xs[i]] : -2;
            double olds[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                olds[i] = 1.0;
                if (dxs[i] == -1 || dxs[i] == d) olds[i] = atomicAdd(&P.sigma[xs[i]], ws.val[js[i]]);
            }
            PROF(PR_EDGE + 4 * MODE + 2);
            bool claim[kLaneItems];
            uint32_t cdg[kLaneItems];
            uint32_t cbg[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                claim[i] = olds[i] == 0.0;
                cdg[i] = 0;
                cbg[i] = 0;
                if (claim[i]) {
                    P.depth[xs[i]] = d;
                    P.du[xs[i]] = 0.0;
                    adj_span(adj_ptr, xs[i], cdg[i], cbg[i]);
                }
            }
            warp_append(claim, xs, cdg, cbg, out, P.ebits);
            if (out_in.ctr) {
#pragma unroll
                for (int i = 0; i < kLaneItems; ++i)
                    if (claim[i]) adj_span(P.in_ptr, xs[i], cdg[i], cbg[i]);
                warp_append(claim, xs, cdg, cbg, out_in, P.ebits);
            }
        } else if (MODE == MODE_BPUSH) {
            // transposed SpMV of Alg.1 l.37 (reading R1: A delta_u) as a push: every in-edge
            // v -> w of an owner w on level d+1 adds delta_u(w) to acc(v) when v is on level d
            int dxs[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) dxs[i] = js[i] >= 0 ? P.depth[xs[i]] : -2;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i)
                if (dxs[i] == d) atomicAdd(&P.gacc[xs[i]], ws.val[js[i]]);
            PROF(PR_EDGE + 4 * MODE + 2);
        } else {
            double vals[kLaneItems];
            if (MODE == MODE_PULL) {
                // f_t(w) = sum over in-neighbours x of sigma(x) (Alg.3 l.9-11).  No level test: an
                // in-neighbour of a still-undiscovered w is on level d-1 or undiscovered (sigma = 0),
                // so sigma itself is the masked frontier vector f.
#pragma unroll
                for (int i = 0; i < kLaneItems; ++i) vals[i] = js[i] >= 0 ? P.sigma[xs[i]] : 0.0;
            } else {
                // (A delta_u)(v): out-neighbour x on level d+1.  The level parity is the sign of
                // the stored delta_u, so neighbours on other levels contribute exactly 0.
#pragma unroll
                for (int i = 0; i < kLaneItems; ++i) {
                    const double u = js[i] >= 0 ? P.du[xs[i]] : 0.0;
                    const double want = ((d + 1) & 1) ? -u : u;
                    vals[i] = want > 0.0 ? want : 0.0;
                }
            }
            PROF(PR_EDGE + 4 * MODE + 2);
            // transpose the values to lane-contiguous slots through shared memory (beg[] is dead)
            double *vb = reinterpret_cast<double *>(ws.beg);
            __syncwarp();
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) vb[i * 32 + lane] = vals[i];
            __syncwarp();
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) vals[i] = vb[lane * kLaneItems + i];
            // per-lane runs: interior runs are complete owners of this lane; the head run may
            // continue an owner from the previous lane, the tail run may continue into the next
            int head_o = o[0], tail_o = o[0];
            double head_sum = 0.0, run = 0.0;
            bool single = true;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                if (o[i] < 0) continue;
                if (o[i] != tail_o) {
                    if (single) head_sum = run;
                    else ws.val[tail_o] = run;
                    single = false;
                    run = 0.0;
                    tail_o = o[i];
                }
                run += vals[i];
            }
            // segmented inclusive scan of the tail runs across lanes (segment = same owner
            // carried through lanes that hold a single run)
            const int prev_tail = __shfl_up_sync(FULL, tail_o, 1);
            bool flag = !(single && lane > 0 && prev_tail == tail_o && tail_o >= 0);
            double S = run;
#pragma unroll
            for (int k = 1; k < 32; k <<= 1) {
                const double s_up = __shfl_up_sync(FULL, S, k);
                const bool f_up = __shfl_up_sync(FULL, flag, k);
                if (lane >= k && !flag) {
                    S += s_up;
                    flag = f_up;
                }
            }
            const double S_prev = __shfl_up_sync(FULL, S, 1);
            if (!single && head_o >= 0)
                ws.val[head_o] = head_sum + ((lane > 0 && prev_tail == head_o) ? S_prev : 0.0);
            const int next_head = __shfl_down_sync(FULL, head_o, 1);
            if (tail_o >= 0 && (lane == 31 || next_head != tail_o)) ws.val[tail_o] = S;
            __syncwarp();
            // ---- hand each owner's sum to the owner pass (this and the reduction: region 3)
            for (int j = lane; j < nwin; j += 32) {
                const double t = ws.val[j];
                if (t == 0.0) continue;
                const bool whole = (j > 0 || start0) && (ps + j < pe);
                if (whole) P.gacc[ws.v[j]] = t;
                else atomicAdd(&P.gacc[ws.v[j]], t);
            }
        }
        __syncwarp();
        PROF(PR_EDGE + 4 * MODE + 3);
    }
}

// ------------------------------------------------------------------ edge-stream pass
//
// The scCOOC form (Alg. 2; "less affected by load unbalance"): every stored
// entry k of a format is visited, as the pair (owner own_arr[k], other end idx[k]), with two
// 16-byte loads per lane for kLaneItems consecutive entries -- the whole edge array streams at
// HBM rate with no owner window, and level filters decide which entries contribute:
//   PUSH (CSR, owner u): u on level d-1 and x on level {-1, d}  -> sigma(x) += sigma(u), claims
//   PULL (CSC, owner w): w undiscovered                    -> acc(w) += sigma(x)
//   BWD  (CSR, owner u): u on level L                       -> acc(u) += delta_u(x) of parity L+1
// (an undiscovered vertex's in-neighbours are on level d-1 or undiscovered with sigma = 0; a
// level-L vertex's out-neighbours are on levels <= L+1, and only level L+1 holds delta_u of
// parity L+1 -- so no per-entry level test is needed on the target side)
// With owners sorted (CSC/CSR order) a lane's entries form owner runs, reduced in registers and
// joined across lanes by one segmented scan; only the warp chunk's first and last owners can
// continue into a neighbouring chunk and use an atomic.  Unsorted owners (the BWD / PUSH of a
// directed COO^T graph, whose only format is column-major) use one atomic per contribution.
constexpr int kStages = 3;  // TMA stages per warp (2 chunks in flight while one is processed)

// a lane's kLaneItems consecutive int32 of a stage, as 16-byte shared-memory loads
__device__ __forceinline__ void load_lane_items(const int4 *src, int (&dst)[kLaneItems]) {
#pragma unroll
    for (int q = 0; q < kLaneItems / 4; ++q) {
        const int4 a = src[q];
        dst[4 * q] = a.x;
        dst[4 * q + 1] = a.y;
        dst[4 * q + 2] = a.z;
        dst[4 * q + 3] = a.w;
    }
}

struct StreamStage {
    int32_t own[kWT];
    int32_t idx[kWT];
};
static_assert(sizeof(StreamStage) * kStages + 8 * kStages <= sizeof(WarpSmem), "stream stages fit the warp slice");

template <int MODE>
__device__ __forceinline__ void stream_pass(const Params &P, WarpSmem &ws, const int32_t *__restrict__ own_arr,
                                            const int32_t *__restrict__ idx, bool sorted, int d, int64_t gwarp,
                                            int64_t nwarps, const ListOut &out, const ListOut &out_in) {
    const int lane = threadIdx.x & 31;
    const int64_t m = P.m;
    const uint64_t pol = policy_evict_first();
    const int owner_level = (MODE == MODE_PUSH) ? d - 1 : (MODE == MODE_PULL ? -1 : d);
    // this warp's chunks: gwarp, gwarp + nwarps, ...; the warp slice of smem becomes kStages
    // stages of (owners, other ends), filled by lane 0 with two bulk copies per chunk
    StreamStage *stage = reinterpret_cast<StreamStage *>(&ws);
    uint64_t *bar = reinterpret_cast<uint64_t *>(reinterpret_cast<unsigned char *>(&ws) + sizeof(StreamStage) * kStages);
    const int64_t nchunks = ceil_div(m, kWT);
    const int64_t mine = gwarp < nchunks ? (nchunks - 1 - gwarp) / nwarps + 1 : 0;
    if (mine == 0) return;
    PROF_START();
    __syncwarp();  // every lane is done with the previous contents of the warp slice
    auto issue = [&](int64_t j) {  // lane 0 only
        const int st = (int)(j % kStages);
        const int64_t base = (gwarp + j * nwarps) * kWT;
        const unsigned bytes = (unsigned)((min((int64_t)kWT, m - base) * 4 + 15) & ~15);
        mbar_arrive_expect_tx(&bar[st], 2 * bytes);
        bulk_g2s(stage[st].own, own_arr + base, bytes, &bar[st], pol);
        bulk_g2s(stage[st].idx, idx + base, bytes, &bar[st], pol);
    };
    auto wait_stage = [&](int64_t j) {
        const unsigned long long t0 = globaltimer_ns();
        while (!mbar_try_wait(&bar[j % kStages], (unsigned)((j / kStages) & 1)))
            if (globaltimer_ns() - t0 > kWatchdogNs) __trap();
    };
    // owner filter data of a chunk, loaded one chunk ahead: the depth of every owner run's owner
    // (one load per run; entries repeating the previous owner get kSame)
    constexpr int kSame = -7;
    int od[kLaneItems];
    auto prefetch = [&](int64_t j, int (&odv)[kLaneItems]) {
        const int st = (int)(j % kStages);
        const int64_t kb = (gwarp + j * nwarps) * kWT + lane * kLaneItems;
        const int4 *so = reinterpret_cast<const int4 *>(stage[st].own + lane * kLaneItems);
        int oo[kLaneItems];
        load_lane_items(so, oo);
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            const bool ok = kb + i < m;
            odv[i] = !ok ? -3 : ((i > 0 && oo[i] == oo[i - 1]) ? kSame : P.depth[oo[i]]);
        }
    };
    if (lane == 0) {
        for (int st = 0; st < kStages; ++st) mbar_init(&bar[st], 1);
        fence_mbar_init();
        fence_proxy_async();
        for (int64_t j = 0; j < min((int64_t)kStages, mine); ++j) issue(j);
    }
    __syncwarp();
    wait_stage(0);
    prefetch(0, od);
    for (int64_t j = 0; j < mine; ++j) {
        const int st = (int)(j % kStages);
        const int64_t base = (gwarp + j * nwarps) * kWT;
        const int64_t k0 = base + lane * kLaneItems;
        int o[kLaneItems], x[kLaneItems];
        {
            const int4 *so = reinterpret_cast<const int4 *>(stage[st].own + lane * kLaneItems);
            const int4 *sx = reinterpret_cast<const int4 *>(stage[st].idx + lane * kLaneItems);
            load_lane_items(so, o);
            load_lane_items(sx, x);
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                if (k0 + i >= m) o[i] = -1;
                TBC_CHECK(o[i] < 0 || (o[i] < P.n && x[i] >= 0 && x[i] < P.n), "stream mode %d k %lld o %d x %d",
                          MODE, (long long)(k0 + i), o[i], x[i]);
            }
        }
        int od_n[kLaneItems];
        if (j + 1 < mine) {
            wait_stage(j + 1);
            prefetch(j + 1, od_n);
        }
        __syncwarp();  // stage st fully read: refill it with chunk j + kStages
        if (lane == 0 && j + kStages < mine) {
            fence_proxy_async();  // order our generic reads of the stage before the async refill
            issue(j + kStages);
        }
        // owner filter (from the prefetched owner depths)
        bool act[kLaneItems];
        double osig[kLaneItems];
        {
            int dep = -3;
            double last_sig = 0.0;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                if (od[i] != kSame) {
                    dep = od[i];
                    if (MODE == MODE_PUSH && dep == owner_level) last_sig = P.sigma[o[i]];
                }
                act[i] = o[i] >= 0 && dep == owner_level;
                osig[i] = last_sig;
            }
        }
        if (MODE == MODE_PUSH) {
            int dxs[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) dxs[i] = act[i] ? P.depth[x[i]] : -2;
            double olds[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                olds[i] = 1.0;
                if (dxs[i] == -1 || dxs[i] == d) olds[i] = atomicAdd(&P.sigma[x[i]], osig[i]);
            }
            bool claim[kLaneItems];
            uint32_t cdg[kLaneItems];
            uint32_t cbg[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                claim[i] = olds[i] == 0.0;
                cdg[i] = 0;
                cbg[i] = 0;
                if (claim[i]) {
                    P.depth[x[i]] = d;
                    P.du[x[i]] = 0.0;
                    if (P.out_ptr) adj_span(P.out_ptr, x[i], cdg[i], cbg[i]);
                }
            }
            warp_append(claim, x, cdg, cbg, out, P.ebits);
            if (out_in.ctr) {
#pragma unroll
                for (int i = 0; i < kLaneItems; ++i)
                    if (claim[i]) adj_span(P.in_ptr, x[i], cdg[i], cbg[i]);
                warp_append(claim, x, cdg, cbg, out_in, P.ebits);
            }
        } else {
            double vals[kLaneItems];
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                if (MODE == MODE_PULL) {
                    vals[i] = act[i] ? P.sigma[x[i]] : 0.0;  // sigma is the masked frontier (see edge_pass)
                } else {
                    const double u = act[i] ? P.du[x[i]] : 0.0;  // parity-signed delta_u selects level L+1
                    const double want = ((d + 1) & 1) ? -u : u;
                    vals[i] = want > 0.0 ? want : 0.0;
                }
            }
            if (!sorted) {
#pragma unroll
                for (int i = 0; i < kLaneItems; ++i)
                    if (vals[i] != 0.0) atomicAdd(&P.gacc[o[i]], vals[i]);
            } else {
            // owner runs of this lane (inactive owners contribute zeros)
            int head_o = o[0], tail_o = o[0];
            double head_sum = 0.0, run = 0.0;
            bool single = true;
            const int first_o = __shfl_sync(FULL, o[0], 0);
            int last_valid = -1;
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i) {
                if (o[i] < 0) continue;
                last_valid = o[i];
                if (o[i] != tail_o) {
                    if (single) head_sum = run;
                    else if (run != 0.0) P.gacc[tail_o] = run;  // interior run: a whole owner
                    single = false;
                    run = 0.0;
                    tail_o = o[i];
                }
                run += vals[i];
            }
            // the chunk's last owner: the last valid entry of the highest lane that has one
            const unsigned vm = __ballot_sync(FULL, last_valid >= 0);
            const int last_o = vm ? __shfl_sync(FULL, last_valid, 31 - __clz(vm)) : -1;
            const int prev_tail = __shfl_up_sync(FULL, tail_o, 1);
            bool flag = !(single && lane > 0 && prev_tail == tail_o && tail_o >= 0);
            double S = run;
#pragma unroll
            for (int k = 1; k < 32; k <<= 1) {
                const double s_up = __shfl_up_sync(FULL, S, k);
                const bool f_up = __shfl_up_sync(FULL, flag, k);
                if (lane >= k && !flag) {
                    S += s_up;
                    flag = f_up;
                }
            }
            const double S_prev = __shfl_up_sync(FULL, S, 1);
            const int next_head = __shfl_down_sync(FULL, head_o, 1);
            if (!single && head_o >= 0) {
                const double t = head_sum + ((lane > 0 && prev_tail == head_o) ? S_prev : 0.0);
                if (t != 0.0) {
                    if (head_o == first_o) atomicAdd(&P.gacc[head_o], t);
                    else P.gacc[head_o] = t;
                }
            }
            if (tail_o >= 0 && (lane == 31 || next_head != tail_o) && S != 0.0) {
                if (tail_o == first_o || tail_o == last_o) atomicAdd(&P.gacc[tail_o], S);
                else P.gacc[tail_o] = S;
            }
            }
        }
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) od[i] = od_n[i];
    }
    __syncwarp();
    if (lane == 0)
        for (int st = 0; st < kStages; ++st) mbar_inval(&bar[st]);
    __syncwarp();
    PROF(PR_STREAM + MODE);
}

// ------------------------------------------------------------------ owner passes

// PULL owner pass over the candidate list: the mask of Alg.1 l.20-25 / Alg.3 l.12-13.
// Discovered (sum > 0) -> depth = d, sigma = sum, appended to the level list; otherwise the
// candidate survives into the next candidate list.  Chunks of kWT owners per warp.
__device__ __forceinline__ void pull_owner_pass(const Params &P, const int32_t *cv, int64_t N, int d,
                                                int64_t gwarp, int64_t nwarps, const ListOut &lvl_out,
                                                const ListOut &ilvl_out, const ListOut &cand_out) {
    const int lane = threadIdx.x & 31;
    for (int64_t base = gwarp * kWT; base < N; base += nwarps * kWT) {
        int32_t vv[kLaneItems];
        double tot[kLaneItems];
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            const int64_t p = base + i * 32 + lane;
            vv[i] = p < N ? (cv ? cv[p] : (int32_t)p) : -1;
            // static first pull (cv == nullptr): every undiscovered vertex with in-edges
            if (!cv && vv[i] >= 0 && (P.depth[vv[i]] != -1 || P.deg2[vv[i]].y == 0)) vv[i] = -1;
        }
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            TBC_CHECK(vv[i] < P.n, "pull owner v %d", vv[i]);
            tot[i] = vv[i] >= 0 ? P.gacc[vv[i]] : 0.0;
        }
        bool take[kLaneItems];
        uint32_t dg[kLaneItems];
        uint32_t bg[kLaneItems];
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            take[i] = vv[i] >= 0 && tot[i] > 0.0;
            dg[i] = 0;
            bg[i] = 0;
            if (take[i]) {
                const int32_t v = vv[i];
                P.gacc[v] = 0.0;
                P.depth[v] = d;
                P.sigma[v] = tot[i];
                P.du[v] = 0.0;
                if (P.out_ptr) adj_span(P.out_ptr, v, dg[i], bg[i]);
            }
        }
        warp_append(take, vv, dg, bg, lvl_out, P.ebits);
        if (ilvl_out.ctr) {
#pragma unroll
            for (int i = 0; i < kLaneItems; ++i)
                if (take[i]) adj_span(P.in_ptr, vv[i], dg[i], bg[i]);
            warp_append(take, vv, dg, bg, ilvl_out, P.ebits);
        }
        // survivors: next candidate list, keyed by in-degree
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            take[i] = vv[i] >= 0 && !(tot[i] > 0.0);
            if (take[i]) adj_span(P.in_ptr, vv[i], dg[i], bg[i]);
        }
        warp_append(take, vv, dg, bg, cand_out, P.ebits);
    }
}

// Candidate scan before a pull that follows push levels: every undiscovered vertex with
// in-edges (labels [0, n_scan) -- degree-sorted labels put the isolated vertices last) is
// appended to the candidate list, keyed by in-degree, so the pull pass costs the candidates'
// in-edges instead of all m (Alg.3 examines every column; the mask of l.20 makes
// the discovered columns' work void).
__device__ __forceinline__ void cand_scan_pass(const Params &P, int64_t gwarp, int64_t nwarps,
                                               const ListOut &cand_out) {
    const int lane = threadIdx.x & 31;
    const int64_t N = P.n_scan;
    for (int64_t base = gwarp * kWT; base < N; base += nwarps * kWT) {
        bool take[kLaneItems];
        int32_t vv[kLaneItems];
        uint32_t dg[kLaneItems];
        uint32_t bg[kLaneItems];
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            const int64_t v = base + i * 32 + lane;
            vv[i] = (int32_t)v;
            take[i] = v < N && P.depth[v] == -1;
        }
#pragma unroll
        for (int i = 0; i < kLaneItems; ++i) {
            dg[i] = 0;
            bg[i] = 0;
            if (take[i]) {
                adj_span(P.in_ptr, vv[i], dg[i], bg[i]);
                take[i] = dg[i] > 0;
            }
        }
        warp_append(take, vv, dg, bg, cand_out, P.ebits);
    }
}

// BWD owner pass over level L: Alg.1 l.38-39 (delta = sigma * A delta_u), l.45 with the 1/2
// of P:180, then l.35 (delta_u for the level above), and the reset of the vertex.
__device__ __forceinline__ void bwd_owner_pass(const Params &P, const int32_t *lv, int64_t N, int L, int64_t gtid,
                                               int64_t nthreads) {
    constexpr int U = 4;
    for (int64_t base = gtid; base < N; base += U * nthreads) {
        int32_t v[U], vb[U];
        double acc[U], sg[U], b[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t p = base + u * nthreads;
            v[u] = p < N ? lv[p] : -1;
            TBC_CHECK(v[u] < P.n && (p >= N || v[u] >= 0), "bwd owner v %d p %lld N %lld", v[u], (long long)p,
                      (long long)N);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (v[u] >= 0) {
                acc[u] = P.gacc[v[u]];
                sg[u] = P.sigma[v[u]];
                vb[u] = P.inv ? P.inv[v[u]] : v[u];
                b[u] = P.bc[vb[u]];
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (v[u] < 0) continue;
            const double delta = sg[u] * acc[u];
            if (acc[u] != 0.0) {
                P.gacc[v[u]] = 0.0;
                P.bc[vb[u]] = b[u] + delta * P.bc_scale;
            }
            const double dun = (1.0 + delta) / sg[u];
            P.du[v[u]] = (L & 1) ? -dun : dun;
            P.sigma[v[u]] = 0.0;
            P.depth[v[u]] = -1;
        }
    }
}

// ------------------------------------------------------------------ trace

// per-level timeline of one traced source (TBC_OPT_TRACE): {t_ns, kind, level, N, E, a, b, 0}
enum { TR_INIT = 0, TR_SCAN = 1, TR_PUSH = 2, TR_PULL = 3, TR_BWD = 4, TR_OWNER = 5 };

__device__ __forceinline__ void trace(const Params &P, bool on, int kind, int64_t level, int64_t N, int64_t E,
                                      int64_t a, int64_t b) {
    if (!on || (int)blockIdx.x != P.cta_base || threadIdx.x != 0) return;
    const unsigned long long i = P.gctr->trace_n;
    if ((int64_t)i >= P.trace_cap) return;
    int64_t *t = P.trace + 8 * i;
    t[0] = (int64_t)globaltimer_ns(); t[1] = kind; t[2] = level; t[3] = N; t[4] = E; t[5] = a; t[6] = b; t[7] = 0;
    P.gctr->trace_n = i + 1;
}

// ------------------------------------------------------------------ the persistent kernel

// the launch: one Params per SM partition (workspace pointers, CTA range), plus the shared
// counters (full-grid barrier, trace) and the caller's bc for the final partition reduction
constexpr int kMaxParts = 8;
struct ParamSet {
    Params p[kMaxParts];
    int nparts, cta_per_part;
    Ctrs *gctr;
    double *bc_out;
};

__global__ void __launch_bounds__(kBlock, 1) k_bc(const __grid_constant__ ParamSet S) {
    extern __shared__ __align__(16) unsigned char dyn_smem[];
    WarpSmem &ws = reinterpret_cast<WarpSmem *>(dyn_smem)[threadIdx.x >> 5];
    // SM partition of this CTA: partition `part` runs sources part, part + nparts, ... on its
    // own workspace with its own (partition-local) grid barrier
    const int part = (int)blockIdx.x / S.cta_per_part;
    const Params &P = S.p[part];
    const int lcta = (int)blockIdx.x - P.cta_base;
    const unsigned ncta = (unsigned)S.cta_per_part;
    const int64_t nwarps = (int64_t)ncta * kWarpsPerBlock;
    const int64_t gwarp = (int64_t)lcta * kWarpsPerBlock + (threadIdx.x >> 5);
    const int tid = threadIdx.x;
    const bool cta0 = lcta == 0;
    const int64_t nthreads = (int64_t)ncta * kBlock;
    const int64_t gtid = (int64_t)lcta * kBlock + tid;
    Ctrs *C = P.ctr;
    unsigned gen_all = (tid == 0) ? ld_acquire(&S.gctr->bar_gen) : 0u;
#ifdef TBC_PROF
    for (int i = tid; i < kWarpsPerBlock * PR_SLOTS; i += kBlock) (&tbc_sprof[0][0])[i] = 0;
    __syncthreads();
    const unsigned long long t_kernel0 = clock64();
#endif
    // barrier generation: only thread 0 uses it (the first barrier cannot complete before
    // every CTA has read the current value, so reading it here is race-free)
    unsigned gen = (tid == 0) ? ld_acquire(&C->bar_gen) : 0u;
    const unsigned long long emask = (1ull << P.ebits) - 1ull;
    int32_t prev_s = -1;

    for (int64_t si = part; si < P.k; si += S.nparts) {
        const int32_t s_caller = P.sources[si];
        if (s_caller < 0 || s_caller >= P.n) {
            if (cta0 && tid == 0) atomicAdd(&C->bad_sources, 1ull);
            continue;
        }
        const int32_t s = P.perm ? P.perm[s_caller] : s_caller;
        const bool tr = (si == P.trace_src);
        // ---------------- init (Alg.1 l.7-10, l.15-18): depth(s)=0, sigma(s)=1, frontier={s}
        const int64_t dego = P.deg2[s].x;
        const int64_t degi = P.deg2[s].y;
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
                P.list_beg[0] = P.out_ptr ? (uint32_t)P.out_ptr[s] : 0u;
                C->list = (1ull << P.ebits) | (unsigned long long)dego;
                if (P.in_list) {
                    P.ilist_v[0] = s;
                    P.ilist_pre[0] = 0;
                    P.ilist_beg[0] = (uint32_t)P.in_ptr[s];
                    C->ilist = (1ull << P.ebits) | (unsigned long long)degi;
                }
                C->cand[0] = 0;
                C->cand[1] = 0;
                if (tr) P.gctr->trace_n = 0;
            }
            for (int64_t i = tid; i <= dego / kWT; i += kBlock) P.tiles[i] = 0;
            if (P.in_list)
                for (int64_t i = tid; i <= degi / kWT; i += kBlock) P.itiles[i] = 0;
        }
        prev_s = s;
        grid_sync(C, gen, ncta);
        trace(P, tr, TR_INIT, 0, 1, dego, s, 0);

        // level d-1 (frontier)
        Level cur{0, 1, 0, dego, 0, 0, P.in_list ? degi : dego, 0};
        int d = 1;
        bool cand_valid = false;
        int cb = 0;
        int64_t candN = 0, candE = 0;
        int64_t fwd_edges = 0, pulls = 0, scans = 0;
        // stream-pass arrays: (owner, other end) of every stored entry in the format each mode
        // walks; a directed COO^T graph has only the column-major pairs (unsorted rows)
        const bool coot_dir = P.coot && P.directed;
        const int32_t *push_own = coot_dir ? P.in_idx : P.out_row;
        const int32_t *push_idx = coot_dir ? P.in_col : P.out_idx;
        for (;;) {
            const int64_t ntiles_f = ceil_div(cur.N + cur.E, kWT);
            const int64_t ntiles_i = ceil_div(cur.N + cur.IE, kWT);
            Level nxt{cur.p0 + cur.N, 0, cur.e0 + cur.E, 0, cur.tbase + ntiles_f,
                      cur.ie0 + cur.IE, 0, cur.itbase + ntiles_i};
            // ---- per-level choice: modelled cost of
            //      0 push over the frontier list, 1 push over all entries, 2 pull over the
            //      survivors of the previous pull, 3 pull over all entries, 4 candidate scan +
            //      pull over the candidates' in-edges.  Pull needs d >= 2.
            const double mE = (double)P.m;
            // candidates of a scan: undiscovered vertices with in-edges and their in-edges
            const double scanE = (double)max((int64_t)0, P.m - nxt.ie0);
            const double scanN = (double)max((int64_t)0, P.n_in - nxt.p0);
            double cost[5] = {(double)cur.E * (P.c_list + P.c_atom), mE * P.c_stream + (double)cur.E * P.c_atom,
                              cand_valid ? (double)candE * P.c_list + (double)candN * P.c_vert : 1e300,
                              mE * P.c_stream + (double)P.n * P.c_vert,
                              cand_valid ? 1e300
                                         : (double)P.n_scan * P.c_scan + scanE * P.c_list + scanN * P.c_vert};
            if (d < 2 || P.dir_mode == 1) cost[2] = cost[3] = cost[4] = 1e300;  // push only
            if (d >= 2 && P.dir_mode == 2) cost[0] = cost[1] = 1e300;             // pull whenever possible
            if (P.fmt_mode == 1 && !P.coot) cost[1] = cost[3] = 1e300;            // list passes only
            if (P.fmt_mode == 2 || P.coot) cost[0] = cost[2] = cost[4] = 1e300;   // edge streams only
            int choice = 0;
            for (int c = 1; c < 5; ++c)
                if (cost[c] < cost[choice]) choice = c;
            const bool pull = choice >= 2;
            const ListOut lo{&C->list, P.list_v, P.list_pre, P.list_beg, P.tiles + nxt.tbase, nxt.p0, nxt.e0};
            const ListOut li = P.in_list ? ListOut{&C->ilist, P.ilist_v, P.ilist_pre, P.ilist_beg,
                                                   P.itiles + nxt.itbase, nxt.p0, nxt.ie0}
                                         : ListOut{nullptr, nullptr, nullptr, nullptr, nullptr, 0, 0};
            if (pull) {
                const bool stream = choice == 3;
                if (choice == 4) {
                    // candidate list cb is empty here (reset by the push level before its barrier)
                    const ListOut sc{&C->cand[cb], P.cand_v[cb], P.cand_pre[cb], P.cand_beg[cb], P.cand_tiles[cb], 0, 0};
                    {
                        PROF_START();
                        cand_scan_pass(P, gwarp, nwarps, sc);
                        PROF(PR_SCAN);
                    }
                    grid_sync(C, gen, ncta);
                    const unsigned long long cv = ld_volatile_u64(&C->snap[2 + cb]);
                    candN = (int64_t)(cv >> P.ebits);
                    candE = (int64_t)(cv & emask);
                    ++scans;
                    trace(P, tr, TR_SCAN, d, candN, candE, 0, 0);
                }
                const ListOut co{&C->cand[cb ^ 1], P.cand_v[cb ^ 1], P.cand_pre[cb ^ 1], P.cand_beg[cb ^ 1],
                                 P.cand_tiles[cb ^ 1], 0, 0};
                if (stream) {
                    stream_pass<MODE_PULL>(P, ws, P.in_col, P.in_idx, true, d, gwarp, nwarps, lo, li);
                    candN = P.n;
                    candE = P.m;
                    ++scans;
                } else {
                    edge_pass<MODE_PULL>(P, ws, P.cand_v[cb], P.cand_pre[cb], P.cand_beg[cb], P.cand_tiles[cb], candN,
                                         candE, 0, P.in_ptr, P.in_idx, d, gwarp, nwarps, lo, li);
                }
                grid_sync(C, gen, ncta);
                trace(P, tr, TR_PULL, d, candN, candE, stream, 0);
                // owner pass: the survivors of a stream pull are all undiscovered vertices
                {
                    PROF_START();
                    pull_owner_pass(P, stream ? nullptr : P.cand_v[cb], candN, d, gwarp, nwarps, lo, li, co);
                    PROF(PR_PULL_OWNER);
                }
                fwd_edges += candE;
                ++pulls;
                cand_valid = !P.coot;
            } else {
                if (choice == 1)
                    stream_pass<MODE_PUSH>(P, ws, push_own, push_idx, !coot_dir, d, gwarp, nwarps, lo, li);
                else
                    edge_pass<MODE_PUSH>(P, ws, P.list_v + cur.p0, P.list_pre + cur.p0, P.list_beg + cur.p0,
                                         P.tiles + cur.tbase, cur.N, cur.E, cur.e0, P.out_ptr, P.out_idx, d, gwarp,
                                         nwarps, lo, li);
                fwd_edges += choice == 1 ? P.m : cur.E;
                if (cta0 && tid == 0) {
                    C->cand[0] = 0;  // candidate lists are stale after a push level
                    C->cand[1] = 0;
                }
                cand_valid = false;
            }
            grid_sync(C, gen, ncta);
            {
                const unsigned long long lv = ld_volatile_u64(&C->snap[0]);
                nxt.N = (int64_t)(lv >> P.ebits) - nxt.p0;
                nxt.E = (int64_t)(lv & emask) - nxt.e0;
                const unsigned long long il = ld_volatile_u64(&C->snap[P.in_list ? 1 : 0]);
                nxt.IE = (int64_t)(il & emask) - nxt.ie0;
            }
            trace(P, tr, pull ? TR_OWNER : TR_PUSH, d, nxt.N, nxt.E, choice, pull ? candE : cur.E);
            if (pull) {
                const unsigned long long cv = ld_volatile_u64(&C->snap[2 + (cb ^ 1)]);
                candN = (int64_t)(cv >> P.ebits);
                candE = (int64_t)(cv & emask);
                if (cta0 && tid == 0) C->cand[cb] = 0;  // consumed; next append target after cb flips
                cb ^= 1;
            }
            if (cta0 && tid == 0) {
                int64_t *l = P.lvl + kLvlWords * (int64_t)d;
                l[0] = nxt.p0; l[1] = nxt.N; l[2] = nxt.e0; l[3] = nxt.E; l[4] = nxt.tbase;
                l[5] = nxt.ie0; l[6] = nxt.IE; l[7] = nxt.itbase;
            }
            if (nxt.N == 0) break;
            if (d > P.n + 1) __trap();  // impossible for a correct BFS: fail loudly, never spin
            cur = nxt;
            ++d;
        }
        const int D = d - 1;  // height of the BFS tree (levels 0..D non-empty)
        if (cta0 && tid == 0) {
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

        // ---------------- backward (Alg.1 l.29-47): L = D (owner pass only: delta = 0) .. 1
        // Each level L < D is one of: pull over the out-edges of level L (list or stream), or
        // push from level L+1 over its in-edges (the transposed product with atomics), by cost.
        int64_t bwd_edges = 0;
        Level up = cur;  // level L+1 while processing level L
        for (int L = D; L >= 1; --L) {
            Level lv;
            if (L == D) {
                lv = cur;
            } else {
                const int64_t *l = P.lvl + kLvlWords * (int64_t)L;
                lv = Level{l[0], l[1], l[2], l[3], l[4], l[5], l[6], l[7]};
                const ListOut none{nullptr, nullptr, nullptr, nullptr, nullptr, 0, 0};
                double bcost[3] = {(double)lv.E * P.c_list, (double)P.m * P.c_stream,
                                   (double)up.IE * (P.c_list + P.c_bpush)};
                if (P.coot || P.fmt_mode == 2) bcost[0] = bcost[2] = 1e300;
                if (P.fmt_mode == 1 && !P.coot) bcost[1] = 1e300;
                if (P.bwd_mode == 1) bcost[2] = 1e300;
                if (P.bwd_mode == 2 && bcost[2] < 1e300) bcost[0] = bcost[1] = 1e300;
                int bsel = 0;
                for (int c = 1; c < 3; ++c)
                    if (bcost[c] < bcost[bsel]) bsel = c;
                if (bsel == 1) {
                    stream_pass<MODE_BWD>(P, ws, push_own, push_idx, !coot_dir, L, gwarp, nwarps, none, none);
                    bwd_edges += P.m;
                } else if (bsel == 0) {
                    edge_pass<MODE_BWD>(P, ws, P.list_v + lv.p0, P.list_pre + lv.p0, P.list_beg + lv.p0,
                                        P.tiles + lv.tbase, lv.N, lv.E, lv.e0, P.out_ptr, P.out_idx, L, gwarp, nwarps,
                                        none, none);
                    bwd_edges += lv.E;
                } else {
                    const int32_t *iv = P.in_list ? P.ilist_v : P.list_v;
                    const uint32_t *ip = P.in_list ? P.ilist_pre : P.list_pre;
                    const uint32_t *ib = P.in_list ? P.ilist_beg : P.list_beg;
                    const int32_t *it = P.in_list ? P.itiles + up.itbase : P.tiles + up.tbase;
                    edge_pass<MODE_BPUSH>(P, ws, iv + up.p0, ip + up.p0, ib + up.p0, it, up.N, up.IE, up.ie0,
                                          P.in_ptr, P.in_idx, L, gwarp, nwarps, none, none);
                    bwd_edges += up.IE;
                }
                grid_sync(C, gen, ncta);
                trace(P, tr, TR_BWD, L, lv.N, lv.E, bsel, 0);
            }
            {
                PROF_START();
                bwd_owner_pass(P, P.list_v + lv.p0, lv.N, L, gtid, nthreads);
                PROF(PR_BWD_OWNER);
            }
            grid_sync(C, gen, ncta);
            trace(P, tr, TR_OWNER, L, lv.N, lv.E, 1, 0);
            up = lv;
        }
        if (cta0 && tid == 0) C->st_bwd_edges += bwd_edges;
    }
    // leave the workspace all-unvisited for the next call (bfs_only keeps it for the caller)
    if (!P.bfs_only && cta0 && tid == 0 && prev_s >= 0) {
        P.depth[prev_s] = -1;
        P.sigma[prev_s] = 0.0;
    }
#ifdef TBC_PROF
    if ((tid & 31) == 0) {
        unsigned long long busy = 0;
        for (int r = 0; r < PR_OTHER; ++r) busy += tbc_sprof[tid >> 5][r];
        tbc_sprof[tid >> 5][PR_OTHER] = clock64() - t_kernel0 - busy;  // the rest: control, init, idle
        for (int r = 0; r < PR_SLOTS; ++r) atomicAdd(&S.gctr->prof[r], tbc_sprof[tid >> 5][r]);
    }
#endif
    if (S.nparts > 1 && !P.bfs_only) {
        // every partition done: bc_out += the partitions' partial bc in partition order
        // (deterministic), and the partials return to zero for the next call
        grid_sync(S.gctr, gen_all, gridDim.x);
        const int64_t nt = (int64_t)gridDim.x * kBlock;
        for (int64_t v = (int64_t)blockIdx.x * kBlock + tid; v < P.n; v += nt) {
            double sum = 0.0;
            for (int q = 0; q < S.nparts; ++q) {
                double *bq = S.p[q].bc;
                sum += bq[v];
                bq[v] = 0.0;
            }
            if (sum != 0.0) S.bc_out[v] += sum;
        }
    }
}

}  // namespace

// ------------------------------------------------------------------ host side

// n_scan = 1 + the largest vertex with in-degree > 0; n_in = how many vertices have one
__global__ void k_in_range(int64_t n, const int2 *__restrict__ deg2, unsigned long long *out) {
    const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const bool has = v < n && deg2[v].y > 0;
    const unsigned m = __ballot_sync(FULL, has);
    if (has) atomicMax(&out[0], (unsigned long long)(v + 1));
    if (m && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&out[1], (unsigned long long)__popc(m));
}

tbc_status engine_workspaces(tbc_graph *g, int count) {
    const int64_t n = g->n, m = g->m;
    cudaStream_t s = g->stream;
    cudaError_t e = cudaSuccess;
    auto alloc = [&](auto **p, size_t cnt) -> cudaError_t {
        size_t bytes = sizeof(**p) * (cnt > 0 ? cnt : 1);
        cudaError_t r = cudaMalloc((void **)p, bytes);
        if (r == cudaSuccess) {
            g->device_bytes += bytes;
            g->ws_bytes += bytes;
        }
        return r;
    };
    const int64_t list_tiles = (n + m) / kWT + n + 2 + kListPad;
    const int64_t cand_tiles = (n + m) / kWT + 2 + kListPad;
    for (int i = g->ws_count; i < count; ++i) {
        Workspace &w = g->ws[i];
        g->ws_count = i + 1;  // engine_free releases whatever of it was allocated
        if ((e = alloc(&w.depth, n)) || (e = alloc(&w.sigma, n)) || (e = alloc(&w.du, n)) ||
            (e = alloc(&w.gacc, n)) || (e = alloc(&w.list_v, n + kListPad)) || (e = alloc(&w.list_pre, n + kListPad)) ||
            (e = alloc(&w.list_beg, n + kListPad)) || (e = alloc(&w.tiles, list_tiles)) ||
            (e = alloc(&w.lvl, kLvlWords * (n + 2))) || (e = alloc(&w.ctr, 1)))
            return cuda_error(e, "workspace cudaMalloc");
        if (g->directed && g->engine == TBC_ENGINE_CSC) {
            if ((e = alloc(&w.ilist_v, n + kListPad)) || (e = alloc(&w.ilist_pre, n + kListPad)) ||
                (e = alloc(&w.ilist_beg, n + kListPad)) || (e = alloc(&w.itiles, list_tiles)))
                return cuda_error(e, "workspace cudaMalloc");
        }
        for (int b = 0; b < 2; ++b)
            if ((e = alloc(&w.cand_v[b], n + kListPad)) || (e = alloc(&w.cand_pre[b], n + kListPad)) ||
                (e = alloc(&w.cand_beg[b], n + kListPad)) || (e = alloc(&w.cand_tiles[b], cand_tiles)))
                return cuda_error(e, "workspace cudaMalloc");
        if ((e = alloc(&w.bc_part, n))) return cuda_error(e, "workspace cudaMalloc");
        if ((e = cudaMemsetAsync(w.depth, 0xff, sizeof(int32_t) * n, s)) ||
            (e = cudaMemsetAsync(w.sigma, 0, sizeof(double) * n, s)) ||
            (e = cudaMemsetAsync(w.du, 0, sizeof(double) * n, s)) ||
            (e = cudaMemsetAsync(w.gacc, 0, sizeof(double) * n, s)) ||
            (e = cudaMemsetAsync(w.bc_part, 0, sizeof(double) * n, s)) ||
            (e = cudaMemsetAsync(w.ctr, 0, sizeof(Ctrs), s)) || (e = cudaStreamSynchronize(s)))
            return cuda_error(e, "workspace init");
    }
    return TBC_OK;
}

void engine_free(tbc_graph *g) {
    for (int i = 0; i < g->ws_count; ++i) {
        Workspace &w = g->ws[i];
        cudaFree(w.depth);
        cudaFree(w.sigma);
        cudaFree(w.du);
        cudaFree(w.gacc);
        cudaFree(w.list_v);
        cudaFree(w.list_pre);
        cudaFree(w.list_beg);
        cudaFree(w.tiles);
        cudaFree(w.ilist_v);
        cudaFree(w.ilist_pre);
        cudaFree(w.ilist_beg);
        cudaFree(w.itiles);
        for (int b = 0; b < 2; ++b) {
            cudaFree(w.cand_v[b]);
            cudaFree(w.cand_pre[b]);
            cudaFree(w.cand_beg[b]);
            cudaFree(w.cand_tiles[b]);
        }
        cudaFree(w.lvl);
        cudaFree(w.ctr);
        cudaFree(w.bc_part);
        w = Workspace{};
    }
    g->ws_count = 0;
    g->device_bytes -= g->ws_bytes;
    g->ws_bytes = 0;
    batch_free(g);
    single_free(g);
    cudaFree(g->gctr);
    cudaFree(g->trace);
    g->gctr = nullptr;
    g->trace = nullptr;
}

tbc_status engine_setup(tbc_graph *g) {
    const int64_t n = g->n, m = g->m;
    cudaStream_t s = g->stream;
    cudaError_t e;
    // packed counters: high bits count (<= n), low bits edge sum (<= m)
    int cbits = 1;
    while ((1ll << cbits) <= n) ++cbits;
    g->ebits = 64 - cbits;
    if (g->ebits < 63 && (m >> g->ebits) != 0)
        return set_error(TBC_ERR_UNSUPPORTED, "nnz %lld too large for n %lld", (long long)m, (long long)n);
    if (m >= (1ll << 32))  // warp_append sums degrees of distinct vertices in 32 bits
        return set_error(TBC_ERR_UNSUPPORTED, "nnz %lld >= 2^32", (long long)m);
    if ((e = cudaMalloc(&g->gctr, sizeof(Ctrs))) || (e = cudaMalloc(&g->trace, sizeof(int64_t) * 8 * kTraceCap)))
        return cuda_error(e, "workspace cudaMalloc");
    g->device_bytes += sizeof(Ctrs) + sizeof(int64_t) * 8 * kTraceCap;
    if ((e = cudaMemsetAsync(g->gctr, 0, sizeof(Ctrs), s))) return cuda_error(e, "workspace init");
    {  // vertices that can have in-edges: [0, n_scan); count of in-degree > 0 (scan cost model)
        unsigned long long *d_cnt = nullptr;
        if ((e = cudaMalloc(&d_cnt, 2 * sizeof(unsigned long long))) ||
            (e = cudaMemsetAsync(d_cnt, 0, 2 * sizeof(unsigned long long), s)))
            return cuda_error(e, "scan range");
        k_in_range<<<(int)((n + 255) / 256), 256, 0, s>>>(n, g->deg2, d_cnt);
        unsigned long long h[2] = {0, 0};
        e = cudaMemcpyAsync(h, d_cnt, sizeof h, cudaMemcpyDeviceToHost, s);
        if (!e) e = cudaStreamSynchronize(s);
        cudaFree(d_cnt);
        if (e) return cuda_error(e, "scan range");
        g->n_scan = (int64_t)h[0];
        g->n_in = (int64_t)h[1];
    }
    if (g->engine == TBC_ENGINE_CSC && g->directed && !g->out_idx) {
        g->batch = 1;  // one format: the batched engine only (no per-source workspace)
        return TBC_OK;
    }
    tbc_status st = engine_workspaces(g, 1);
    if (st != TBC_OK) return st;
    int per_sm = 0, sms = 0;
    if ((e = cudaFuncSetAttribute(k_bc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes)) ||
        (e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_bc, kBlock, kSmemBytes)) ||
        (e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device)))
        return cuda_error(e, "occupancy query");
    if (per_sm < 1) return set_error(TBC_ERR_CUDA, "k_bc cannot be resident (occupancy 0)");
    g->grid = per_sm * sms;
    return TBC_OK;
}

// auto (TBC_OPT_BATCH = -1): the first call with sources probes the graph's level width once
// (single_probe); graphs whose levels average fewer than TBC_OPT_NARROW_WIDTH vertices (road
// networks, lattices, small graphs) run the narrow-level engine, the others the batched engine
tbc_status engine_choose(tbc_graph *g, const int32_t *d_sources, int64_t k, cudaStream_t stream, int *mode) {
    if (g->engine != TBC_ENGINE_CSC) {
        *mode = g->last_mode = 0;
        return TBC_OK;
    }
    if (g->batch >= 0 || (g->directed && !g->out_idx)) {  // forced, or one format (batched only)
        if (g->directed && !g->out_idx && g->batch != 1)
            return set_error(TBC_ERR_UNSUPPORTED, "one-format graphs run the batched engine only (TBC_OPT_BATCH = 1)");
        *mode = g->last_mode = g->batch;
        return TBC_OK;
    }
    if (g->narrow < 0 && k > 0) {
        double width = 0.0;
        tbc_status st = single_probe(g, d_sources, stream, &width);
        if (st != TBC_OK) return st;
        g->narrow = width < g->narrow_width ? 1 : 0;
        g->probe_width = width;
        if (!g->narrow) single_free(g);  // the probe's slot
    }
    *mode = g->last_mode = g->narrow == 1 ? 2 : 1;
    return TBC_OK;
}

tbc_status engine_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                      int bfs_only) {
    // bc calls of the CSC engine: batched (tbc_batch.cu) or narrow-level (tbc_single.cu) engine, or
    // this file's per-source engine (TBC_OPT_BATCH, auto by default: engine_choose)
    if (!bfs_only && g->engine == TBC_ENGINE_CSC) {
        int mode = 0;
        tbc_status st = engine_choose(g, d_sources, k, stream, &mode);
        if (st != TBC_OK) return st;
        if (mode == 1) return batch_run(g, d_sources, k, d_bc, stream);
        if (mode == 2) return single_run(g, d_sources, k, d_bc, stream);
    }
    // SM partitions: never more than the sources (a partition without sources only waits)
    int np = g->nparts;
    if (bfs_only || k < 1) np = 1;
    if (np > k) np = (int)k;
    if (np > g->grid) np = g->grid;
    if (np < 1) np = 1;
    tbc_status st = engine_workspaces(g, np);
    if (st != TBC_OK) return st;
    static_assert(sizeof(ParamSet) <= 32000, "kernel parameter space");
    ParamSet S{};
    S.nparts = np;
    S.cta_per_part = g->grid / np;
    S.gctr = g->gctr;
    S.bc_out = d_bc;
    for (int q = 0; q < np; ++q) {
        const Workspace &w = g->ws[q];
        Params &P = S.p[q];
        P.n = g->n;
        P.m = g->m;
        P.in_ptr = g->in_ptr;
        P.in_idx = g->in_idx;
        P.out_ptr = g->out_ptr;
        P.out_idx = g->out_idx;
        P.deg2 = g->deg2;
        P.depth = w.depth;
        P.sigma = w.sigma;
        P.du = w.du;
        P.gacc = w.gacc;
        P.list_v = w.list_v;
        P.list_pre = w.list_pre;
        P.list_beg = w.list_beg;
        P.directed = g->directed;
        P.coot = g->engine == TBC_ENGINE_COOT;
        P.in_col = g->in_col;
        P.out_row = g->out_row;
        P.fmt_mode = g->fmt_mode;
        P.c_list = g->c_list;
        P.c_stream = g->c_stream;
        P.c_atom = g->c_atom;
        P.c_vert = g->c_vert;
        P.tiles = w.tiles;
        P.in_list = w.ilist_v != nullptr;
        P.ilist_v = P.in_list ? w.ilist_v : w.list_v;
        P.ilist_pre = P.in_list ? w.ilist_pre : w.list_pre;
        P.ilist_beg = P.in_list ? w.ilist_beg : w.list_beg;
        P.itiles = P.in_list ? w.itiles : w.tiles;
        P.n_scan = g->n_scan;
        P.n_in = g->n_in;
        P.c_scan = g->c_scan;
        P.c_bpush = g->c_bpush;
        P.bwd_mode = g->bwd_mode;
        for (int b = 0; b < 2; ++b) {
            P.cand_v[b] = w.cand_v[b];
            P.cand_pre[b] = w.cand_pre[b];
            P.cand_beg[b] = w.cand_beg[b];
            P.cand_tiles[b] = w.cand_tiles[b];
        }
        P.lvl = w.lvl;
        P.ctr = w.ctr;
        P.gctr = g->gctr;
        P.cta_base = q * S.cta_per_part;
        P.bc = np > 1 ? w.bc_part : d_bc;
        P.perm = g->perm;
        P.inv = g->inv;
        P.sources = d_sources;
        P.k = k;
        P.bc_scale = g->directed ? 1.0 : 0.5;
        P.ebits = g->ebits;
        P.bfs_only = bfs_only;
        P.dir_mode = g->dir_mode;
        P.trace = g->trace;
        P.trace_cap = g->trace ? kTraceCap : 0;
        P.trace_src = g->trace_src;
    }
    void *args[] = {&S};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_bc, dim3(S.cta_per_part * np), dim3(kBlock), args,
                                                kSmemBytes, stream);
    if (e != cudaSuccess) return cuda_error(e, "cudaLaunchCooperativeKernel(k_bc)");
    return TBC_OK;
}

}  // namespace tbc
