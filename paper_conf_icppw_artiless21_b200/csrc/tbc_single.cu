// tbc_single.cu -- the narrow-level engine: Algorithm 1 of PAPER.md for ONE source per
// CTA, many sources side by side (one per resident CTA), every level separated by a CTA barrier
// (__syncthreads) instead of a grid barrier.
//
// Why: on high-diameter graphs (road networks, lattices: thousands of levels of a
// few thousand vertices) the grid-wide engines pay a grid barrier and several dependent memory round
// trips per level for a level that only a handful of SMs' worth of threads can use; the paper's own
// runs on such graphs are its slowest (luxembourg-osm, d = 1035: 5 MTEPs).  Here a level of
// w vertices costs ceil(w / 512) rounds of a few dependent loads inside one SM, and 148+ sources
// progress concurrently, so the whole GPU streams memory while each source walks its levels.
//
// Per source (Alg.1 with R1-R5 of DESIGN.md):
//   forward level d -> d+1 (l.19-27): every frontier vertex u (BFS order list, level offsets lvl)
//     pushes sigma(u) along its out-edges: depth(w) is claimed with atomicCAS(-1 -> d+1) (the
//     claimer appends w to the order list) and sigma(w) += sigma(u) (fp64 atomic) iff depth(w) = d+1
//     -- the masked SpMV f_t = A^T f restricted to the unvisited vertices (l.19-25).
//   backward level L = D..1 (l.29-47): every v on level L pulls acc = sum of delta_u(w) over its
//     out-edges with depth(w) = L+1 (A delta_u, R1), adds scale * sigma(v) * acc to bc (l.39, l.45,
//     1/2 if undirected P:180) and overwrites sigma(v) with delta_u(v) = 1/sigma(v) + acc (l.35):
//     in place, because a vertex has one level and its sigma is read only by its own update.
//   level L+2 is reset (depth -1, sigma 0) during level L, levels 0..2 at the end: a CTA's arrays
//   are all-unvisited between sources, with no O(n) clear.
// A vertex's whole per-source state is one 32-byte record (one DRAM sector): {sigma / delta_u,
// depth, the slot's partial bc}; every step touches one sector per vertex.  The partial bc of a
// slot accumulates over its sources with plain read-modify-writes (a slot belongs to one CTA) and
// k_bcs_reduce adds the slots into the caller's bc after the kernel.
// Out-degrees above kHeavy are deferred to a per-level shared-memory queue and run by a whole warp.
#include <cstdio>

#include "tbc_internal.cuh"
#include "tbc_device.cuh"

namespace tbc {
namespace {

constexpr unsigned FULL = 0xffffffffu;
#ifndef TBC_SBLOCK
#define TBC_SBLOCK 1024
#endif
constexpr int kSB = TBC_SBLOCK;     // threads per CTA
constexpr int kSWarps = kSB / 32;
constexpr int kHeavy = 32;          // out-degree above which a whole warp handles the vertex
constexpr int kLight = 4;
#ifndef TBC_DIRECT_CAS
#define TBC_DIRECT_CAS 0            // 1: claim low-degree targets with the CAS alone (no depth pre-load)
#endif           // out-degree up to which a vertex's edge loads are issued together
constexpr int kHeavyCap = 2048;     // heavy vertices queued per level (overflow: handled by one thread)

struct SParams {
    int64_t n;
    const int64_t *__restrict__ out_ptr;  // CSR of A (== the CSC when undirected)
    const int32_t *__restrict__ out_idx;
    VRec *rec;        // [slots][n]: sigma / delta_u (0 between sources), depth (-1 between sources), bc
    int32_t *order;   // [slots][n], BFS order, levels concatenated
    int32_t *lvl;     // [slots][n + 2], level offsets into order
    Ctrs *ctr;
    double *bc;       // caller labels, accumulated (fp64 atomics: the CTAs share it)
    const int32_t *sources;  // caller labels
    const int32_t *__restrict__ perm;  // caller -> internal label (nullptr: identity)
    const int32_t *__restrict__ inv;   // internal -> caller label
    int64_t k;
    double bc_scale;
    int32_t *bfs_depth;  // tbc_bfs_batch: forward only, export [source index][caller label]
    double *bfs_sigma;   // sigma, or its mantissa when bfs_sexp is set
    int32_t *bfs_sexp;   // tbc_bfs_batch_ext: binary exponent of sigma
    const int64_t *__restrict__ in_ptr;   // CSC (in-edges): the extended-range sigma pull
    const int32_t *__restrict__ in_idx;
    int sigma_mode;      // TBC_OPT_SIGMA: 0 fp64 with extended-range re-run on overflow, 1 extended
    int fwd_only;        // TBC_OPT_STAGE = 1: forward stage only (measurement), bc untouched
    int64_t probe_cap;   // > 0: probe run (one source, forward only, stop after ~probe_cap vertices)
    int64_t *probe_out;  // {levels completed, vertices discovered}
};

// ---- extended-range numbers (NEXT-2): value = f * 2^e with f = 0 or 0.5 <= |f| < 1.  sigma and
// delta_u of a source on a mesh leave the fp64 range (sigma = C(i+j, i) ~ 2^8190 from a corner of a
// 4096^2 mesh; delta_u = (1 + delta) / sigma ~ 2^-8190), while delta = sigma * acc and bc stay in
// range.  Integer sums below 2^53 stay exact (aligned adds of integers), as in fp64.
struct Xr {
    double f;
    int e;
};

__device__ __forceinline__ Xr xr_norm(double f, int e) {
    int k = 0;
    const double m = frexp(f, &k);
    return Xr{m, f == 0.0 ? 0 : e + k};
}

__device__ __forceinline__ Xr xr_add(Xr a, Xr b) {
    if (a.f == 0.0) return b;
    if (b.f == 0.0) return a;
    if (a.e < b.e) {
        const Xr t = a;
        a = b;
        b = t;
    }
    const int d = a.e - b.e;
    if (d > 1100) return a;  // b is below a's last mantissa bit
    return xr_norm(a.f + ldexp(b.f, -d), a.e);
}

__device__ __forceinline__ Xr xr_mul(Xr a, Xr b) { return xr_norm(a.f * b.f, a.e + b.e); }
__device__ __forceinline__ Xr xr_inv(Xr a) { return xr_norm(1.0 / a.f, -a.e); }
__device__ __forceinline__ Xr xr_shfl_xor(Xr a, int o) {
    return Xr{__shfl_xor_sync(FULL, a.f, o), __shfl_xor_sync(FULL, a.e, o)};
}
__device__ __forceinline__ Xr rec_xr(const VRec *r) {  // one 16-byte load: {sd, depth, sexp}
    const double2 q = __ldcg(reinterpret_cast<const double2 *>(r));
    return Xr{q.x, __double2hiint(q.y)};
}

// relax the out-edge u -> w of frontier level d: claim w for level d+1 (the claimer appends it), and
// in fp64 mode add sigma(u) (Alg.1 l.19-25 as a push); the extended mode sums sigma in a pull
template <bool XR>
__device__ __forceinline__ void relax(VRec *rec, int32_t *order, int32_t w, int d, double su, int *cnt, int end) {
    int dw = __ldcg(&rec[w].depth);
    if (dw == -1) {
        dw = atomicCAS(&rec[w].depth, -1, d + 1);
        if (dw == -1) {
            order[end + atomicAdd(cnt, 1)] = w;
            dw = d + 1;
        }
    }
    if (!XR && dw == d + 1) atomicAdd(&rec[w].sd, su);
}

// delta_u(w) if w is on level L+1, else 0 (one 16-byte load: sd and depth share it); in the
// extended-range sigma pull the same test selects the in-neighbours on level d (L = d - 1)
__device__ __forceinline__ double child(const VRec *rec, int32_t w, int L) {
    const double2 r = __ldcg(reinterpret_cast<const double2 *>(rec + w));
    return __double2loint(r.y) == L + 1 ? r.x : 0.0;
}
__device__ __forceinline__ Xr child_xr(const VRec *rec, int32_t w, int L) {
    const double2 r = __ldcg(reinterpret_cast<const double2 *>(rec + w));
    return __double2loint(r.y) == L + 1 ? Xr{r.x, __double2hiint(r.y)} : Xr{0.0, 0};
}

// Alg.1 l.35-45 for v with acc = sum of delta_u over its level-(L+1) out-neighbours
__device__ __forceinline__ void finish(const SParams &P, VRec *rec, int32_t v, double acc) {
    const double sv = __ldcg(&rec[v].sd);
    const double delta = sv * acc;
    if (delta != 0.0) rec[v].bc += delta * P.bc_scale;
    rec[v].sd = 1.0 / sv + acc;
}
__device__ __forceinline__ void finish_xr(const SParams &P, VRec *rec, int32_t v, Xr acc) {
    const Xr sv = rec_xr(rec + v);
    const Xr dl = xr_mul(sv, acc);
    const double delta = ldexp(dl.f, dl.e);  // delta_s(v) <= n: in range
    if (delta != 0.0) rec[v].bc += delta * P.bc_scale;
    const Xr du = xr_add(xr_inv(sv), acc);
    rec[v].sd = du.f;
    rec[v].sexp = du.e;
}

__device__ __forceinline__ void reset_level(VRec *rec, const int32_t *order, int b0, int b1) {
    for (int i = b0 + (int)threadIdx.x; i < b1; i += kSB) {
        const int32_t x = order[i];
        *reinterpret_cast<int4 *>(rec + x) = make_int4(0, 0, -1, 0);  // sd = 0, depth = -1, sexp = 0
    }
}

struct SShared {
    int cnt[2], hcnt[2];
    int pcnt;  // extended range: heavy vertices of the level's sigma pull
    int ovf;  // fp64 mode: a sigma left the fp64 range (the source is re-run in extended range)
    int32_t heavy[kHeavyCap];
    unsigned long long edges[2];
};

// One source on one CTA (Alg.1 l.7-47).  XR = false: fp64 sigma / delta_u; returns false (nothing
// accumulated, state reset) if a sigma overflowed, so that the caller re-runs the source with XR.
template <bool XR>
__device__ bool bcs_source(const SParams &P, SShared &sh, int64_t si, int32_t s, VRec *rec, int32_t *order,
                           int32_t *lvl) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t n = P.n;
    if (tid == 0) {  // level 0 (Alg.1 l.15-18)
        rec[s].depth = 0;
        rec[s].sd = XR ? 0.5 : 1.0;  // 1 = 0.5 * 2^1
        rec[s].sexp = XR ? 1 : 0;
        order[0] = s;
        lvl[0] = 0;
        lvl[1] = 1;
        sh.cnt[0] = sh.cnt[1] = 0;
        sh.hcnt[0] = sh.hcnt[1] = 0;
        sh.edges[0] = sh.edges[1] = 0;
        sh.ovf = 0;
    }
    __syncthreads();
    // ---------------- forward (Alg.1 l.11-28)
    int d = 0, beg = 0, end = 1;
    unsigned long long my_edges = 0;
    bool probe_stop = false;
    for (;;) {
        const int par = d & 1;
        // two frontier vertices per thread and iteration; low-degree ones (<= kLight out-edges: lattices,
        // road networks) issue all their edge loads, then all depth loads, together
        for (int i = beg + tid; i < end; i += 2 * kSB) {
            if (P.probe_cap > 0 && end + *(volatile int *)&sh.cnt[par] > P.probe_cap) break;
            int32_t uu[2];
            int64_t b0[2], b1[2];
            double su[2];
            bool lt[2];
            uu[0] = order[i];
            uu[1] = i + kSB < end ? order[i + kSB] : -1;
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                b0[t] = b1[t] = 0;
                su[t] = 0.0;
                if (uu[t] >= 0) {
                    b0[t] = P.out_ptr[uu[t]];
                    b1[t] = P.out_ptr[uu[t] + 1];
                    su[t] = XR ? 0.0 : __ldcg(&rec[uu[t]].sd);
                }
            }
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                lt[t] = false;
                if (uu[t] < 0) continue;
                my_edges += (unsigned long long)(b1[t] - b0[t]);
                if (!XR && !(su[t] <= 1.7976931348623157e308)) sh.ovf = 1;  // inf: out of the fp64 range
                if (b1[t] - b0[t] > kHeavy) {
                    const int h = atomicAdd(&sh.hcnt[par], 1);
                    if (h < kHeavyCap) {
                        sh.heavy[h] = uu[t];
                        uu[t] = -1;
                        continue;
                    }
                }
                lt[t] = b1[t] - b0[t] <= kLight;
            }
            int32_t w[2 * kLight];
            int dw[2 * kLight];
#pragma unroll
            for (int q = 0; q < 2 * kLight; ++q) {
                const int t = q / kLight;
                const int64_t e = b0[t] + q % kLight;
                w[q] = (lt[t] && e < b1[t]) ? P.out_idx[e] : -1;
            }
#pragma unroll
            for (int q = 0; q < 2 * kLight; ++q)
                dw[q] = w[q] < 0 ? -2 : TBC_DIRECT_CAS ? atomicCAS(&rec[w[q]].depth, -1, d + 1) : __ldcg(&rec[w[q]].depth);
#pragma unroll
            for (int q = 0; q < 2 * kLight; ++q) {
                if (dw[q] == -1) {
                    if (!TBC_DIRECT_CAS) dw[q] = atomicCAS(&rec[w[q]].depth, -1, d + 1);
                    if (dw[q] == -1) {
                        order[end + atomicAdd(&sh.cnt[par], 1)] = w[q];
                        dw[q] = d + 1;
                    }
                }
                if (!XR && dw[q] == d + 1) atomicAdd(&rec[w[q]].sd, su[q / kLight]);
            }
#pragma unroll
            for (int t = 0; t < 2; ++t)
                if (uu[t] >= 0 && !lt[t])
                    for (int64_t e = b0[t]; e < b1[t]; ++e)
                        relax<XR>(rec, order, P.out_idx[e], d, su[t], &sh.cnt[par], end);
        }
        __syncthreads();
        if (tid == 0) {  // counters of level d+2 (their level-d readers are past the barrier)
            sh.cnt[par ^ 1] = 0;
            sh.hcnt[par ^ 1] = 0;
            sh.pcnt = 0;
        }
        const int nh = min(sh.hcnt[par], kHeavyCap);
        for (int h = warp; h < nh; h += kSWarps) {
            const int32_t u = sh.heavy[h];
            const double su = XR ? 0.0 : __ldcg(&rec[u].sd);
            const int64_t e1 = P.out_ptr[u + 1];
            for (int64_t e = P.out_ptr[u] + lane; e < e1; e += 32)
                relax<XR>(rec, order, P.out_idx[e], d, su, &sh.cnt[par], end);
        }
        __syncthreads();
        const int nn = sh.cnt[par];
        if (P.probe_cap > 0 && end + nn > P.probe_cap) {
            probe_stop = true;
            end += nn;  // every claimed vertex is in the list (reset below)
            break;
        }
        if (nn == 0) break;
        if (XR) {
            // sigma(w) = sum of sigma(u) over the in-neighbours u on level d (Alg.1 l.19 as a pull,
            // extended-range adds); in-degrees above kHeavy by a warp with a shuffle reduction
            for (int i = end + tid; i < end + nn; i += kSB) {
                const int32_t w = order[i];
                const int64_t e0 = P.in_ptr[w], e1 = P.in_ptr[w + 1];
                if (e1 - e0 > kHeavy) {
                    const int h = atomicAdd(&sh.pcnt, 1);
                    if (h < kHeavyCap) {
                        sh.heavy[h] = w;
                        continue;
                    }
                }
                Xr sg{0.0, 0};
                for (int64_t e = e0; e < e1; ++e) sg = xr_add(sg, child_xr(rec, P.in_idx[e], d - 1));  // depth d
                rec[w].sd = sg.f;
                rec[w].sexp = sg.e;
            }
            __syncthreads();
            const int nh2 = min(sh.pcnt, kHeavyCap);
            for (int h = warp; h < nh2; h += kSWarps) {
                const int32_t w = sh.heavy[h];
                const int64_t e1 = P.in_ptr[w + 1];
                Xr sg{0.0, 0};
                for (int64_t e = P.in_ptr[w] + lane; e < e1; e += 32) sg = xr_add(sg, child_xr(rec, P.in_idx[e], d - 1));
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) sg = xr_add(sg, xr_shfl_xor(sg, o));
                if (lane == 0) {
                    rec[w].sd = sg.f;
                    rec[w].sexp = sg.e;
                }
            }
            __syncthreads();
        }
        beg = end;
        end += nn;
        ++d;
        if (tid == 0) lvl[d + 1] = end;
    }
    const int D = d;  // deepest non-empty level
    atomicAdd(&sh.edges[0], my_edges);
    if (tid == 0) sh.hcnt[0] = sh.hcnt[1] = 0;  // their forward readers are past the last barrier
    __syncthreads();
    if (P.probe_cap > 0) {  // probe: report, reset every listed vertex, done
        if (tid == 0) {
            P.probe_out[0] = D + 1;  // levels whose expansion ran
            P.probe_out[1] = end;    // vertices discovered
            P.probe_out[2] = probe_stop ? 0 : 1;
        }
        reset_level(rec, order, 0, end);
        __syncthreads();
        return true;
    }
    if (!XR && sh.ovf) {  // a sigma overflowed fp64: drop this run (nothing accumulated yet)
        reset_level(rec, order, 0, end);
        if (tid == 0) sh.edges[0] = 0;
        __syncthreads();
        return false;
    }
    if (tid == 0) {
        atomicAdd((unsigned long long *)&P.ctr->st_sources, 1ull);
        atomicAdd((unsigned long long *)&P.ctr->st_reached, (unsigned long long)end);
        atomicAdd((unsigned long long *)&P.ctr->st_reached_edges, sh.edges[0]);
        atomicAdd((unsigned long long *)&P.ctr->st_fwd_edges, sh.edges[0]);
        atomicAdd((unsigned long long *)&P.ctr->st_levels, (unsigned long long)(D + 2));
        atomicMax((unsigned long long *)&P.ctr->st_max_depth, (unsigned long long)D);
        if (XR) atomicAdd((unsigned long long *)&P.ctr->st_xr_sources, 1ull);
    }
    if (P.bfs_depth || P.fwd_only) {  // tbc_bfs_batch: export depth / sigma; or forward only
        for (int L = 0; L <= D && P.bfs_depth; ++L) {
            const int b0 = lvl[L], b1 = lvl[L + 1];
            for (int i = b0 + tid; i < b1; i += kSB) {
                const int32_t x = order[i];
                const int64_t o = si * n + (P.inv ? P.inv[x] : x);
                P.bfs_depth[o] = L;
                const Xr sg = XR ? rec_xr(rec + x) : xr_norm(__ldcg(&rec[x].sd), 0);
                if (P.bfs_sexp) {  // mantissa and exponent (any range)
                    P.bfs_sigma[o] = sg.f;
                    P.bfs_sexp[o] = sg.e;
                } else {
                    P.bfs_sigma[o] = ldexp(sg.f, sg.e);
                }
            }
        }
        __syncthreads();
        reset_level(rec, order, 0, end);
        if (tid == 0) sh.edges[0] = 0;
        __syncthreads();
        return true;
    }
    // ---------------- backward, L = D..1 (Alg.1 l.29-47)
    unsigned long long my_bwd = 0;
    for (int L = D; L >= 1; --L) {
        const int par = L & 1;
        const int b0 = lvl[L], b1 = lvl[L + 1];
        for (int i = b0 + tid; i < b1; i += 2 * kSB) {
            int32_t vv[2];
            int64_t c0[2], c1[2];
            bool lt[2];
            vv[0] = order[i];
            vv[1] = i + kSB < b1 ? order[i + kSB] : -1;
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                c0[t] = c1[t] = 0;
                lt[t] = false;
                if (vv[t] < 0) continue;
                c0[t] = P.out_ptr[vv[t]];
                c1[t] = P.out_ptr[vv[t] + 1];
                my_bwd += (unsigned long long)(c1[t] - c0[t]);
                if (c1[t] - c0[t] > kHeavy) {
                    const int h = atomicAdd(&sh.hcnt[par], 1);
                    if (h < kHeavyCap) {
                        sh.heavy[h] = vv[t];
                        vv[t] = -1;
                        continue;
                    }
                }
                lt[t] = !XR && c1[t] - c0[t] <= kLight;
            }
            if (!XR) {  // low-degree owners: every child load of both in flight together
                int32_t w[2 * kLight];
                double c[2 * kLight];
#pragma unroll
                for (int q = 0; q < 2 * kLight; ++q) {
                    const int t = q / kLight;
                    const int64_t e = c0[t] + q % kLight;
                    w[q] = (lt[t] && e < c1[t]) ? P.out_idx[e] : -1;
                }
#pragma unroll
                for (int q = 0; q < 2 * kLight; ++q) c[q] = w[q] >= 0 ? child(rec, w[q], L) : 0.0;
#pragma unroll
                for (int t = 0; t < 2; ++t) {
                    if (!lt[t]) continue;
                    double acc = 0.0;
#pragma unroll
                    for (int q = 0; q < kLight; ++q) acc += c[t * kLight + q];
                    finish(P, rec, vv[t], acc);
                }
            }
#pragma unroll
            for (int t = 0; t < 2; ++t) {
                if (vv[t] < 0 || lt[t]) continue;
                if (XR) {
                    Xr acc{0.0, 0};
                    for (int64_t e = c0[t]; e < c1[t]; ++e) acc = xr_add(acc, child_xr(rec, P.out_idx[e], L));
                    finish_xr(P, rec, vv[t], acc);
                } else {
                    double acc = 0.0;
                    for (int64_t e = c0[t]; e < c1[t]; ++e) acc += child(rec, P.out_idx[e], L);
                    finish(P, rec, vv[t], acc);
                }
            }
        }
        if (L + 2 <= D) reset_level(rec, order, lvl[L + 2], lvl[L + 3]);
        __syncthreads();
        if (tid == 0) sh.hcnt[par ^ 1] = 0;
        const int nh = min(sh.hcnt[par], kHeavyCap);
        for (int h = warp; h < nh; h += kSWarps) {
            const int32_t v = sh.heavy[h];
            const int64_t e1 = P.out_ptr[v + 1];
            if (XR) {
                Xr acc{0.0, 0};
                for (int64_t e = P.out_ptr[v] + lane; e < e1; e += 32) acc = xr_add(acc, child_xr(rec, P.out_idx[e], L));
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) acc = xr_add(acc, xr_shfl_xor(acc, o));
                if (lane == 0) finish_xr(P, rec, v, acc);
            } else {
                double acc = 0.0;
                for (int64_t e = P.out_ptr[v] + lane; e < e1; e += 32) acc += child(rec, P.out_idx[e], L);
#pragma unroll
                for (int o = 16; o >= 1; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
                if (lane == 0) finish(P, rec, v, acc);
            }
        }
        __syncthreads();
    }
    reset_level(rec, order, 0, lvl[min(D, 2) + 1]);
    atomicAdd(&sh.edges[1], my_bwd);
    __syncthreads();
    if (tid == 0) {
        atomicAdd((unsigned long long *)&P.ctr->st_bwd_edges, sh.edges[1]);
        sh.edges[0] = sh.edges[1] = 0;
        sh.hcnt[0] = sh.hcnt[1] = 0;
    }
    __syncthreads();
    return true;
}

__global__ void __launch_bounds__(kSB) k_bcs(const __grid_constant__ SParams P) {
    const int64_t n = P.n;
    const int64_t slot = blockIdx.x;
    VRec *rec = P.rec + slot * n;
    int32_t *order = P.order + slot * n;
    int32_t *lvl = P.lvl + slot * (n + 2);
    __shared__ SShared sh;
    for (int64_t si = blockIdx.x; si < P.k; si += gridDim.x) {
        int32_t s = P.sources[si];
        if (s < 0 || s >= n) {  // skipped and counted (tbc_bc_device does not validate on the host)
            if (threadIdx.x == 0) atomicAdd(&P.ctr->bad_sources, 1ull);
            continue;
        }
        if (P.perm) s = P.perm[s];
        // fp64 first; a source whose sigma leaves the fp64 range runs again in extended range
        if (P.sigma_mode == 1 || !bcs_source<false>(P, sh, si, s, rec, order, lvl))
            bcs_source<true>(P, sh, si, s, rec, order, lvl);
        if (P.probe_cap > 0) return;
    }
}

// bc(v) += sum over the used slots of their partial bc(v); the partials return to 0
__global__ void k_bcs_reduce(int64_t n, int64_t slots, VRec *rec, double *bc, const int32_t *__restrict__ inv) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        double sum = 0.0;
        for (int64_t q = 0; q < slots; ++q) {
            double *p = &rec[q * n + v].bc;
            sum += *p;
            *p = 0.0;
        }
        if (sum != 0.0) bc[inv ? inv[v] : v] += sum;
    }
}

__global__ void k_rec_init(int64_t count, VRec *rec) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x)
        rec[i] = VRec{0.0, -1, 0, 0.0, 0.0};  // sd, depth, sexp, bc, pad
}

}  // namespace

// ------------------------------------------------------------------ host side

static int64_t single_slot_bytes(const tbc_graph *g) { return (int64_t)sizeof(VRec) * g->n + 8 * g->n + 8; }

void single_free(tbc_graph *g) {
    SingleWorkspace &w = g->sws;
    cudaFree(w.rec);
    cudaFree(w.order);
    cudaFree(w.lvl);
    cudaFree(w.ctr);
    cudaFree(w.probe_out);
    g->device_bytes -= w.bytes;
    w = SingleWorkspace{};
}

// one slot (a CTA's arrays) per concurrently running source: as many as the GPU keeps resident,
// within 60 % of the free memory (at least one); sized once per graph.  probe_only: one slot (the
// level-width probe must not take the memory the batched engine may need)
static tbc_status single_alloc(tbc_graph *g, bool probe_only = false) {
    SingleWorkspace &w = g->sws;
    if (w.slots > 1 || (w.slots == 1 && probe_only)) return TBC_OK;
    if (w.slots) single_free(g);  // the probe's single slot: grow to the full set
    cudaError_t e = cudaSuccess;
    int per_sm = 0, sms = 0;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_bcs, kSB, 0)) ||
        (e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device)))
        return cuda_error(e, "k_bcs occupancy query");
    if (per_sm < 1) return set_error(TBC_ERR_CUDA, "k_bcs cannot be resident");
    size_t fr = 0, tot = 0;
    if ((e = cudaMemGetInfo(&fr, &tot))) return cuda_error(e, "cudaMemGetInfo");
    // one source per SM by default: a source's level then gets 1024 threads, and 148 wavefronts keep
    // their neighbours' records in L2 between consecutive levels (A/B on the 4096^2 road lattice:
    // 8.85 GTEPS vs 7.92 at two per SM and 7.39 with 512-thread CTAs)
    int64_t slots = probe_only ? 1 : (int64_t)sms;
    if (!probe_only && g->narrow_slots > 0 && slots > g->narrow_slots) slots = g->narrow_slots;
    const int64_t fit = (int64_t)(0.6 * (double)fr / (double)single_slot_bytes(g));
    if (slots > fit) slots = fit;
    if (slots < 1) slots = 1;
    const int64_t n = g->n;
    auto alloc = [&](auto **p, size_t cnt) -> cudaError_t {
        const size_t bytes = sizeof(**p) * (cnt > 0 ? cnt : 1);
        cudaError_t r = cudaMalloc((void **)p, bytes);
        if (r == cudaSuccess) {
            w.bytes += bytes;
            g->device_bytes += bytes;
        }
        return r;
    };
    if ((e = alloc(&w.rec, slots * n)) || (e = alloc(&w.order, slots * n)) ||
        (e = alloc(&w.lvl, slots * (n + 2))) || (e = alloc(&w.ctr, 1)) || (e = alloc(&w.probe_out, 4))) {
        single_free(g);
        return cuda_error(e, "narrow-level engine workspace cudaMalloc");
    }
    cudaStream_t s = g->stream;
    k_rec_init<<<148 * 8, 256, 0, s>>>(slots * n, w.rec);
    if ((e = cudaGetLastError()) || (e = cudaMemsetAsync(w.ctr, 0, sizeof(Ctrs), s)) || (e = cudaStreamSynchronize(s))) {
        single_free(g);
        return cuda_error(e, "narrow-level engine workspace init");
    }
    w.slots = (int)slots;
    return TBC_OK;
}

static SParams single_params(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc) {
    const SingleWorkspace &w = g->sws;
    SParams P{};
    P.n = g->n;
    P.out_ptr = g->out_ptr;
    P.out_idx = g->out_idx;
    P.rec = w.rec;
    P.order = w.order;
    P.lvl = w.lvl;
    P.ctr = w.ctr;
    P.bc = d_bc;
    P.sources = d_sources;
    P.perm = g->perm;
    P.inv = g->inv;
    P.k = k;
    P.bc_scale = g->directed ? 1.0 : 0.5;
    P.probe_out = w.probe_out;
    P.in_ptr = g->in_ptr;
    P.in_idx = g->in_idx;
    P.sigma_mode = g->sigma_mode;
    return P;
}

tbc_status single_run(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, cudaStream_t stream,
                      int32_t *bfs_depth, double *bfs_sigma, int32_t *bfs_sexp) {
    if (!g->out_ptr) return set_error(TBC_ERR_UNSUPPORTED, "narrow-level engine needs the out-edge format");
    tbc_status st = single_alloc(g);
    if (st != TBC_OK) return st;
    SParams P = single_params(g, d_sources, k, d_bc);
    P.bfs_depth = bfs_depth;
    P.bfs_sigma = bfs_sigma;
    P.bfs_sexp = bfs_sexp;
    P.fwd_only = g->stage == 1;
    const int grid = (int)(k < g->sws.slots ? k : g->sws.slots);
    if (grid < 1) return TBC_OK;
    k_bcs<<<grid, kSB, 0, stream>>>(P);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_bcs launch");
    if (!bfs_depth && !P.fwd_only) {
        k_bcs_reduce<<<148 * 8, 256, 0, stream>>>(g->n, grid, g->sws.rec, d_bc, g->inv);
        if ((e = cudaGetLastError()) != cudaSuccess) return cuda_error(e, "k_bcs_reduce launch");
    }
    return TBC_OK;
}

// Level-width probe (auto engine choice): a forward BFS from the call's first source
// by one CTA, stopped once it has discovered kProbeCap vertices; returns the average number of
// vertices per level seen so far (a narrow, deep graph stays far below the threshold long before
// the cap; a scale-free graph crosses the cap within 2-3 levels).  Synchronises the stream.
tbc_status single_probe(tbc_graph *g, const int32_t *d_sources, cudaStream_t stream, double *width) {
    constexpr int64_t kProbeCap = 1 << 16;
    tbc_status st = single_alloc(g, true);
    if (st != TBC_OK) return st;
    SParams P = single_params(g, d_sources, 1, nullptr);
    P.probe_cap = kProbeCap;
    cudaError_t e = cudaMemsetAsync(g->sws.probe_out, 0, 4 * sizeof(int64_t), stream);
    if (e) return cuda_error(e, "level-width probe");
    k_bcs<<<1, kSB, 0, stream>>>(P);
    int64_t h[4] = {0, 0, 0, 0};
    e = cudaGetLastError();
    if (!e) e = cudaMemcpyAsync(h, g->sws.probe_out, sizeof h, cudaMemcpyDeviceToHost, stream);
    if (!e) e = cudaStreamSynchronize(stream);
    if (e) return cuda_error(e, "level-width probe");
    *width = (double)h[1] / (double)(h[0] > 0 ? h[0] : 1);
    return TBC_OK;
}

}  // namespace tbc
