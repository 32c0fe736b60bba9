// tbc_api.cu -- the extern "C" boundary of libturbobc: graph creation (device-side
// canonicalisation of the CSC / COOC input of P:95-97), the tbc_bc / tbc_bfs drivers,
// options, statistics and error reporting.  Declarations and contracts: include/tbc.h.
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstddef>
#include <cstring>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include "tbc_internal.cuh"

namespace tbc {

static thread_local char g_err[512] = "";

tbc_status set_error(tbc_status s, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof g_err, fmt, ap);
    va_end(ap);
    return s;
}

tbc_status cuda_error(cudaError_t e, const char *what) {
    if (e == cudaErrorMemoryAllocation)
        return set_error(TBC_ERR_OOM, "%s: %s", what, cudaGetErrorString(e));
    return set_error(TBC_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

}  // namespace tbc

using namespace tbc;

#define TBC_CUDA(call)                                             \
    do {                                                           \
        cudaError_t e_ = (call);                                   \
        if (e_ != cudaSuccess) { st = cuda_error(e_, #call); goto fail; } \
    } while (0)

namespace {

// ----------------------------------------------------------------- canonicalisation kernels

// key = (column << 32) | row for every stored entry of the caller's CSC (column-major order)
__global__ void k_csc_to_keys(int64_t n, int64_t nnz, const int64_t *__restrict__ col_ptr,
                              const int32_t *__restrict__ row, unsigned long long *keys) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz;
         i += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = n;  // largest c with col_ptr[c] <= i
        while (hi - lo > 1) {
            int64_t mid = (lo + hi) >> 1;
            if (col_ptr[mid] <= i) lo = mid; else hi = mid;
        }
        keys[i] = ((unsigned long long)lo << 32) | (unsigned)row[i];
    }
}

// key = (dst << 32) | src for an edge list src -> dst (A(src,dst) = 1, column dst)
__global__ void k_coo_to_keys(int64_t nnz, const int32_t *__restrict__ src,
                              const int32_t *__restrict__ dst, unsigned long long *keys) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz;
         i += (int64_t)gridDim.x * blockDim.x)
        keys[i] = ((unsigned long long)(unsigned)dst[i] << 32) | (unsigned)src[i];
}

// split sorted unique keys into (major ptr, minor idx); ptr[v] = first key with major >= v
__global__ void k_keys_to_ptr(int64_t n, int64_t m, const unsigned long long *__restrict__ keys,
                              int64_t *ptr, int32_t *idx, int32_t *major_out) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += stride) {
        idx[i] = (int32_t)(keys[i] & 0xffffffffull);
        if (major_out) major_out[i] = (int32_t)(keys[i] >> 32);
    }
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n; v += stride) {
        int64_t lo = 0, hi = m;  // lower_bound of major v
        unsigned long long key = (unsigned long long)v << 32;
        while (lo < hi) {
            int64_t mid = (lo + hi) >> 1;
            if (keys[mid] < key) lo = mid + 1; else hi = mid;
        }
        ptr[v] = lo;
    }
}

__global__ void k_transpose_keys(int64_t m, const unsigned long long *__restrict__ in,
                                 unsigned long long *out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
         i += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long k = in[i];
        out[i] = (k << 32) | (k >> 32);
    }
}

__global__ void k_count_mismatch(int64_t m, const unsigned long long *__restrict__ a,
                                 const unsigned long long *__restrict__ b, unsigned long long *bad) {
    unsigned long long local = 0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
         i += (int64_t)gridDim.x * blockDim.x)
        local += (a[i] != b[i]);
    if (local) atomicAdd(bad, local);
}

// degree-descending relabelling: endpoint counts of the raw entries
__global__ void k_endpoint_count(int64_t nnz, const unsigned long long *__restrict__ keys, int32_t *deg) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long k = keys[i];
        atomicAdd(&deg[(int64_t)(k >> 32)], 1);
        atomicAdd(&deg[(int64_t)(k & 0xffffffffull)], 1);
    }
}

__global__ void k_iota(int64_t n, int32_t *a) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        a[i] = (int32_t)i;
}

__global__ void k_invert(int64_t n, const int32_t *__restrict__ inv, int32_t *perm) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        perm[inv[i]] = (int32_t)i;
}

__global__ void k_relabel(int64_t nnz, unsigned long long *keys, const int32_t *__restrict__ perm) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long k = keys[i];
        keys[i] = ((unsigned long long)(unsigned)perm[(int64_t)(k >> 32)] << 32) |
                  (unsigned)perm[(int64_t)(k & 0xffffffffull)];
    }
}

__global__ void k_unpermute_bfs(int64_t n, const int32_t *__restrict__ perm, const int32_t *__restrict__ depth,
                                const double *__restrict__ sigma, int32_t *depth_out, double *sigma_out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        depth_out[v] = depth[perm[v]];
        sigma_out[v] = sigma[perm[v]];
    }
}

__global__ void k_deg2(int64_t n, const int64_t *__restrict__ out_ptr,
                       const int64_t *__restrict__ in_ptr, int2 *deg2) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x)
        deg2[v] = make_int2((int)(out_ptr[v + 1] - out_ptr[v]), (int)(in_ptr[v + 1] - in_ptr[v]));
}

// out-degrees from the rows of the CSC (one-format COO^T directed graphs have no CSR):
// zero them, then count every stored row
__global__ void k_out_degree(int64_t n, int64_t m, const int32_t *__restrict__ rows, int2 *deg2) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        deg2[v].x = 0;
}

__global__ void k_count_rows(int64_t m, const int32_t *__restrict__ rows, int2 *deg2) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&deg2[rows[i]].x, 1);
}

constexpr int64_t kPad = 16;  // entries of slack after every edge array (TMA bulk copies round up)

inline int grid_for(int64_t work) {
    int64_t b = (work + 255) / 256;
    if (b < 1) b = 1;
    if (b > 148 * 16) b = 148 * 16;
    return (int)b;
}

template <class T>
cudaError_t dmalloc(tbc_graph *g, T **p, size_t count) {
    size_t bytes = sizeof(T) * (count > 0 ? count : 1);
    cudaError_t e = cudaMalloc((void **)p, bytes);
    if (e == cudaSuccess) g->device_bytes += bytes;
    return e;
}

void free_graph(tbc_graph *g) {
    if (!g) return;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(g->device);
    if (g->out_ptr != g->in_ptr) cudaFree(g->out_ptr);
    if (g->out_idx != g->in_idx) cudaFree(g->out_idx);
    cudaFree(g->in_ptr);
    cudaFree(g->in_idx);
    cudaFree(g->deg2);
    cudaFree(g->perm);
    cudaFree(g->inv);
    cudaFree(g->in_col);
    if (g->out_row != g->in_col) cudaFree(g->out_row);
    engine_free(g);
    if (g->h_bovf) cudaFreeHost(g->h_bovf);
    cudaFree(g->bfs_depth);
    cudaFree(g->bfs_sigma);
    cudaFree(g->bfs_sexp);
    cudaFree(g->bc_tmp);
    cudaFree(g->src_tmp);
    if (g->stream) cudaStreamDestroy(g->stream);
    cudaSetDevice(cur);
    delete g;
}

// Canonicalise entries given as keys (column << 32 | row) into the graph's CSC (+CSR/COO^T).
// Consumes d_keys (device, nnz entries).  Runs on g->stream.
tbc_status build_from_keys(tbc_graph *g, unsigned long long *d_keys, int64_t nnz) {
    tbc_status st = TBC_OK;
    // strict single format (NEXT-4): a directed graph keeps the CSC alone (no CSR, no
    // owner arrays); undirected graphs are one format anyway (the CSC is its own transpose)
    const bool one_format = (g->flags & TBC_FLAG_ONE_FORMAT) && g->directed;
    cudaStream_t s = g->stream;
    unsigned long long *alt = nullptr, *tkeys = nullptr, *d_bad = nullptr;
    int64_t *d_num = nullptr;
    void *temp = nullptr;
    size_t temp_bytes = 0, need = 0;
    int64_t m = 0;
    unsigned long long bad = 0;
    int end_bit = 32;
    while ((1ll << (end_bit - 32)) < g->n) ++end_bit;
    if (end_bit > 64) end_bit = 64;

    TBC_CUDA(cudaMalloc(&alt, sizeof(unsigned long long) * (nnz > 0 ? nnz : 1)));
    TBC_CUDA(cudaMalloc(&d_num, sizeof(int64_t)));
    if (!(g->flags & TBC_FLAG_NO_REORDER) && nnz > 0) {
        // vertex ids by decreasing degree: hubs get small ids, so the gathers of sigma / delta_u
        // that dominate the traversal hit a compact, cache-resident head of the arrays
        int32_t *deg = nullptr, *deg_s = nullptr, *ids = nullptr;
        void *rtemp = nullptr;
        size_t rbytes = 0;
        cudaError_t e1 = cudaMalloc(&deg, sizeof(int32_t) * g->n);
        if (!e1) e1 = cudaMalloc(&deg_s, sizeof(int32_t) * g->n);
        if (!e1) e1 = cudaMalloc(&ids, sizeof(int32_t) * g->n);
        if (!e1) e1 = dmalloc(g, &g->inv, g->n);
        if (!e1) e1 = dmalloc(g, &g->perm, g->n);
        if (!e1) e1 = cudaMemsetAsync(deg, 0, sizeof(int32_t) * g->n, s);
        if (!e1) {
            k_endpoint_count<<<grid_for(nnz), 256, 0, s>>>(nnz, d_keys, deg);
            k_iota<<<grid_for(g->n), 256, 0, s>>>(g->n, ids);
            e1 = cub::DeviceRadixSort::SortPairsDescending(nullptr, rbytes, deg, deg_s, ids, g->inv, g->n, 0, 32, s);
        }
        if (!e1) e1 = cudaMalloc(&rtemp, rbytes);
        if (!e1) e1 = cub::DeviceRadixSort::SortPairsDescending(rtemp, rbytes, deg, deg_s, ids, g->inv, g->n, 0, 32, s);
        // only degree-skewed graphs are relabelled (max endpoint count > 16 x the mean): on flat
        // degree distributions (lattices, road networks, ER) the caller's labels keep whatever
        // locality they have, which the sort by degree would scatter
        int32_t dmax = 0;
        if (!e1) e1 = cudaMemcpyAsync(&dmax, deg_s, sizeof dmax, cudaMemcpyDeviceToHost, s);
        if (!e1) e1 = cudaStreamSynchronize(s);
        const bool skewed = (double)dmax > 16.0 * 2.0 * (double)nnz / (double)g->n;
        if (!e1 && skewed) {
            k_invert<<<grid_for(g->n), 256, 0, s>>>(g->n, g->inv, g->perm);
            k_relabel<<<grid_for(nnz), 256, 0, s>>>(nnz, d_keys, g->perm);
            e1 = cudaStreamSynchronize(s);
        }
        if (!e1 && !skewed) {
            cudaFree(g->inv);
            cudaFree(g->perm);
            g->inv = g->perm = nullptr;
            g->device_bytes -= 2 * sizeof(int32_t) * g->n;
        }
        cudaFree(deg);
        cudaFree(deg_s);
        cudaFree(ids);
        cudaFree(rtemp);
        if (e1) {
            st = cuda_error(e1, "relabel");
            goto fail;
        }
    }
    TBC_CUDA(cudaMalloc(&d_bad, sizeof(unsigned long long)));
    if (nnz > 0) {
        TBC_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, need, d_keys, alt, nnz, 0, end_bit, s));
        temp_bytes = need;
        TBC_CUDA(cub::DeviceSelect::Unique(nullptr, need, alt, d_keys, d_num, nnz, s));
        if (need > temp_bytes) temp_bytes = need;
        TBC_CUDA(cudaMalloc(&temp, temp_bytes));
        TBC_CUDA(cub::DeviceRadixSort::SortKeys(temp, temp_bytes, d_keys, alt, nnz, 0, end_bit, s));
        TBC_CUDA(cub::DeviceSelect::Unique(temp, temp_bytes, alt, d_keys, d_num, nnz, s));
        TBC_CUDA(cudaMemcpyAsync(&m, d_num, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        TBC_CUDA(cudaStreamSynchronize(s));
    }
    g->m = m;
    // CSC of A (in-neighbours)
    TBC_CUDA(dmalloc(g, &g->in_ptr, g->n + 1));
    TBC_CUDA(dmalloc(g, &g->in_idx, m + kPad));  // +pad: 16-byte bulk copies of the last chunk
    if (!one_format)  // column (owner) of every CSC entry: the COOC col_A, for edge streams
        TBC_CUDA(dmalloc(g, &g->in_col, m + kPad));
    k_keys_to_ptr<<<grid_for(m > g->n ? m : g->n + 1), 256, 0, s>>>(g->n, m, d_keys, g->in_ptr,
                                                                   g->in_idx, g->in_col);
    TBC_CUDA(cudaGetLastError());
    if (!g->directed || (g->engine == TBC_ENGINE_CSC && !one_format)) {
        // transpose (row << 32 | col), sorted: the CSR of A; compared to the CSC when undirected
        tkeys = alt;  // reuse: alt is free after Unique
        alt = nullptr;
        if (m > 0) {
            TBC_CUDA(cudaMalloc(&alt, sizeof(unsigned long long) * m));
            k_transpose_keys<<<grid_for(m), 256, 0, s>>>(m, d_keys, alt);
            TBC_CUDA(cudaGetLastError());
            need = 0;
            TBC_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, need, alt, tkeys, m, 0, end_bit, s));
            if (need > temp_bytes) {
                cudaFree(temp);
                temp = nullptr;
                temp_bytes = need;
                TBC_CUDA(cudaMalloc(&temp, temp_bytes));
            }
            TBC_CUDA(cub::DeviceRadixSort::SortKeys(temp, temp_bytes, alt, tkeys, m, 0, end_bit, s));
        }
        if (!g->directed) {
            if (!(g->flags & TBC_FLAG_NO_VALIDATE) && m > 0) {
                TBC_CUDA(cudaMemsetAsync(d_bad, 0, sizeof(unsigned long long), s));
                k_count_mismatch<<<grid_for(m), 256, 0, s>>>(m, d_keys, tkeys, d_bad);
                TBC_CUDA(cudaGetLastError());
                TBC_CUDA(cudaMemcpyAsync(&bad, d_bad, sizeof bad, cudaMemcpyDeviceToHost, s));
                TBC_CUDA(cudaStreamSynchronize(s));
                if (bad) {
                    st = set_error(TBC_ERR_INVALID,
                                   "directed=0 but the pattern is not symmetric (%llu mismatches)", bad);
                    goto fail;
                }
            }
            g->out_ptr = g->in_ptr;
            g->out_idx = g->in_idx;
            g->out_row = g->in_col;
        } else {
            TBC_CUDA(dmalloc(g, &g->out_ptr, g->n + 1));
            TBC_CUDA(dmalloc(g, &g->out_idx, m + kPad));
            TBC_CUDA(dmalloc(g, &g->out_row, m + kPad));
            k_keys_to_ptr<<<grid_for(m > g->n ? m : g->n + 1), 256, 0, s>>>(g->n, m, tkeys, g->out_ptr,
                                                                           g->out_idx, g->out_row);
            TBC_CUDA(cudaGetLastError());
        }
    } else {
        g->out_ptr = nullptr;  // COO^T or TBC_FLAG_ONE_FORMAT directed: one format only
        g->out_idx = nullptr;
        g->out_row = nullptr;
    }
    TBC_CUDA(dmalloc(g, &g->deg2, g->n));
    if (g->out_ptr) {
        k_deg2<<<grid_for(g->n), 256, 0, s>>>(g->n, g->out_ptr, g->in_ptr, g->deg2);
    } else {
        k_deg2<<<grid_for(g->n), 256, 0, s>>>(g->n, g->in_ptr, g->in_ptr, g->deg2);
        TBC_CUDA(cudaGetLastError());
        k_out_degree<<<grid_for(g->n), 256, 0, s>>>(g->n, m, g->in_idx, g->deg2);
        TBC_CUDA(cudaGetLastError());
        if (m > 0) k_count_rows<<<grid_for(m), 256, 0, s>>>(m, g->in_idx, g->deg2);
    }
    TBC_CUDA(cudaGetLastError());
    TBC_CUDA(cudaStreamSynchronize(s));
fail:
    cudaFree(alt);
    if (tkeys) cudaFree(tkeys);
    cudaFree(temp);
    cudaFree(d_num);
    cudaFree(d_bad);
    return st;
}

tbc_status create_common(int64_t n, int directed, int engine, unsigned flags, int device,
                         tbc_graph **gout) {
    if (n <= 0 || n >= (1ll << 31)) return set_error(TBC_ERR_INVALID, "n=%lld out of [1, 2^31)", (long long)n);
    if (engine != TBC_ENGINE_CSC && engine != TBC_ENGINE_COOT)
        return set_error(TBC_ERR_INVALID, "unknown engine %d", engine);
    if ((flags & TBC_FLAG_ONE_FORMAT) && engine != TBC_ENGINE_CSC)
        return set_error(TBC_ERR_UNSUPPORTED, "TBC_FLAG_ONE_FORMAT applies to TBC_ENGINE_CSC (COO^T is one format already)");
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess) return cuda_error(e, "cudaGetDeviceCount");
    if (device < 0 || device >= ndev) return set_error(TBC_ERR_INVALID, "device %d of %d", device, ndev);
    e = cudaSetDevice(device);
    if (e != cudaSuccess) return cuda_error(e, "cudaSetDevice");
    tbc_graph *g = new tbc_graph();
    g->device = device;
    g->n = n;
    g->directed = directed ? 1 : 0;
    g->engine = engine;
    g->flags = flags;
    e = cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking);
    if (e != cudaSuccess) {
        delete g;
        return cuda_error(e, "cudaStreamCreate");
    }
    *gout = g;
    return TBC_OK;
}

}  // namespace

extern "C" {

const char *tbc_status_string(tbc_status s) {
    switch (s) {
        case TBC_OK: return "TBC_OK";
        case TBC_ERR_INVALID: return "TBC_ERR_INVALID";
        case TBC_ERR_OOM: return "TBC_ERR_OOM";
        case TBC_ERR_CUDA: return "TBC_ERR_CUDA";
        case TBC_ERR_UNSUPPORTED: return "TBC_ERR_UNSUPPORTED";
    }
    return "TBC_ERR_UNKNOWN";
}

const char *tbc_last_error(void) { return g_err; }

tbc_status tbc_graph_create_csc(int64_t n, int64_t nnz, const int64_t *col_ptr, const int32_t *row_idx,
                                int directed, int engine, unsigned flags, int device, tbc_graph **out) {
    g_err[0] = 0;
    if (!out) return set_error(TBC_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (nnz < 0) return set_error(TBC_ERR_INVALID, "nnz < 0");
    if (!col_ptr || (nnz > 0 && !row_idx)) return set_error(TBC_ERR_INVALID, "NULL array");
    if (n > 0 && n < (1ll << 31) && !(flags & TBC_FLAG_NO_VALIDATE)) {
        if (col_ptr[0] != 0) return set_error(TBC_ERR_INVALID, "col_ptr[0] = %lld != 0", (long long)col_ptr[0]);
        if (col_ptr[n] != nnz) return set_error(TBC_ERR_INVALID, "col_ptr[n] != nnz");
        for (int64_t v = 0; v < n; ++v)
            if (col_ptr[v + 1] < col_ptr[v]) return set_error(TBC_ERR_INVALID, "col_ptr not monotone at %lld", (long long)v);
        for (int64_t i = 0; i < nnz; ++i)
            if (row_idx[i] < 0 || row_idx[i] >= n)
                return set_error(TBC_ERR_INVALID, "row_idx[%lld] = %d out of range", (long long)i, row_idx[i]);
    }
    tbc_graph *g = nullptr;
    tbc_status st = create_common(n, directed, engine, flags, device, &g);
    if (st != TBC_OK) return st;
    int64_t *d_cp = nullptr;
    int32_t *d_row = nullptr;
    unsigned long long *keys = nullptr;
    TBC_CUDA(cudaMalloc(&d_cp, sizeof(int64_t) * (n + 1)));
    TBC_CUDA(cudaMalloc(&d_row, sizeof(int32_t) * (nnz > 0 ? nnz : 1)));
    TBC_CUDA(cudaMalloc(&keys, sizeof(unsigned long long) * (nnz > 0 ? nnz : 1)));
    TBC_CUDA(cudaMemcpyAsync(d_cp, col_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, g->stream));
    if (nnz > 0) {
        TBC_CUDA(cudaMemcpyAsync(d_row, row_idx, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, g->stream));
        k_csc_to_keys<<<grid_for(nnz), 256, 0, g->stream>>>(n, nnz, d_cp, d_row, keys);
        TBC_CUDA(cudaGetLastError());
    }
    TBC_CUDA(cudaStreamSynchronize(g->stream));
    cudaFree(d_cp);
    d_cp = nullptr;
    cudaFree(d_row);
    d_row = nullptr;
    st = build_from_keys(g, keys, nnz);
    if (st != TBC_OK) goto fail;
    cudaFree(keys);
    keys = nullptr;
    st = engine_setup(g);
    if (st != TBC_OK) goto fail;
    *out = g;
    return TBC_OK;
fail:
    cudaFree(d_cp);
    cudaFree(d_row);
    cudaFree(keys);
    free_graph(g);
    return st;
}

tbc_status tbc_graph_create_coo(int64_t n, int64_t nnz, const int32_t *src, const int32_t *dst,
                                int directed, int engine, unsigned flags, int device, tbc_graph **out) {
    g_err[0] = 0;
    if (!out) return set_error(TBC_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (nnz < 0) return set_error(TBC_ERR_INVALID, "nnz < 0");
    if (nnz > 0 && (!src || !dst)) return set_error(TBC_ERR_INVALID, "NULL array");
    if (n > 0 && n < (1ll << 31) && !(flags & TBC_FLAG_NO_VALIDATE)) {
        for (int64_t i = 0; i < nnz; ++i)
            if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n)
                return set_error(TBC_ERR_INVALID, "edge %lld (%d -> %d) out of range", (long long)i, src[i], dst[i]);
    }
    tbc_graph *g = nullptr;
    tbc_status st = create_common(n, directed, engine, flags, device, &g);
    if (st != TBC_OK) return st;
    int32_t *d_s = nullptr, *d_d = nullptr;
    unsigned long long *keys = nullptr;
    TBC_CUDA(cudaMalloc(&d_s, sizeof(int32_t) * (nnz > 0 ? nnz : 1)));
    TBC_CUDA(cudaMalloc(&d_d, sizeof(int32_t) * (nnz > 0 ? nnz : 1)));
    TBC_CUDA(cudaMalloc(&keys, sizeof(unsigned long long) * (nnz > 0 ? nnz : 1)));
    if (nnz > 0) {
        TBC_CUDA(cudaMemcpyAsync(d_s, src, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, g->stream));
        TBC_CUDA(cudaMemcpyAsync(d_d, dst, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, g->stream));
        k_coo_to_keys<<<grid_for(nnz), 256, 0, g->stream>>>(nnz, d_s, d_d, keys);
        TBC_CUDA(cudaGetLastError());
    }
    TBC_CUDA(cudaStreamSynchronize(g->stream));
    cudaFree(d_s);
    d_s = nullptr;
    cudaFree(d_d);
    d_d = nullptr;
    st = build_from_keys(g, keys, nnz);
    if (st != TBC_OK) goto fail;
    cudaFree(keys);
    keys = nullptr;
    st = engine_setup(g);
    if (st != TBC_OK) goto fail;
    *out = g;
    return TBC_OK;
fail:
    cudaFree(d_s);
    cudaFree(d_d);
    cudaFree(keys);
    free_graph(g);
    return st;
}

tbc_status tbc_destroy(tbc_graph *g) {
    g_err[0] = 0;
    if (!g) return TBC_OK;
    free_graph(g);
    return TBC_OK;
}

tbc_status tbc_graph_info(const tbc_graph *g, int64_t *n, int64_t *nnz, int *directed, size_t *device_bytes) {
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (n) *n = g->n;
    if (nnz) *nnz = g->m;
    if (directed) *directed = g->directed;
    if (device_bytes) *device_bytes = g->device_bytes;
    return TBC_OK;
}

tbc_status tbc_graph_set_option(tbc_graph *g, int key, double value) {
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (key == TBC_OPT_DIRECTION) {
        int v = (int)value;
        if (v < 0 || v > 2 || (double)v != value) return set_error(TBC_ERR_INVALID, "direction %g", value);
        g->dir_mode = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_TRACE) {
        if (value < -1 || (double)(int64_t)value != value) return set_error(TBC_ERR_INVALID, "trace %g", value);
        g->trace_src = (int64_t)value;
        return TBC_OK;
    }
    if (key == TBC_OPT_FORMAT) {
        int v = (int)value;
        if (v < 0 || v > 2 || (double)v != value) return set_error(TBC_ERR_INVALID, "format %g", value);
        g->fmt_mode = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_PARTITIONS) {
        int v = (int)value;
        if (v < 1 || v > kMaxPartitions || (double)v != value)
            return set_error(TBC_ERR_INVALID, "partitions %g not in [1, %d]", value, kMaxPartitions);
        g->nparts = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_BWD_DIRECTION) {
        int v = (int)value;
        if (v < 0 || v > 2 || (double)v != value) return set_error(TBC_ERR_INVALID, "bwd direction %g", value);
        g->bwd_mode = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH) {
        int v = (int)value;
        if (v < -1 || v > 2 || (double)v != value) return set_error(TBC_ERR_INVALID, "engine %g not in [-1, 2]", value);
        if (g->engine == TBC_ENGINE_CSC && g->directed && !g->out_idx && v != 1)
            return set_error(TBC_ERR_UNSUPPORTED, "one-format graphs run the batched engine only");
        g->batch = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_NARROW_SLOTS) {
        int v = (int)value;
        if (v < 0 || (double)v != value) return set_error(TBC_ERR_INVALID, "narrow slots %g", value);
        g->narrow_slots = v;
        if (g->sws.slots > 1) single_free(g);  // re-sized at the next call
        return TBC_OK;
    }
    if (key == TBC_OPT_SIGMA) {
        int v = (int)value;
        if (v < 0 || v > 1 || (double)v != value) return set_error(TBC_ERR_INVALID, "sigma mode %g not 0 or 1", value);
        g->sigma_mode = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_STAGE) {
        int v = (int)value;
        if (v < 0 || v > 1 || (double)v != value) return set_error(TBC_ERR_INVALID, "stage %g not 0 or 1", value);
        g->stage = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_INPLACE) {
        int v = (int)value;
        if (v < -1 || v > 1 || (double)v != value) return set_error(TBC_ERR_INVALID, "batch in-place mode %g", value);
        g->binplace = v;
        g->binplace_eff = -1;
        for (int q = 0; q < kMaxPartitions; ++q) batch_free_one(g, q);  // reallocated at the next call
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_LIST) {
        int v = (int)value;
        if (v < 1 || v > 64 || (double)v != value) return set_error(TBC_ERR_INVALID, "batch list factor %g not in [1, 64]", value);
        g->blist_factor = v;
        for (int q = 0; q < kMaxPartitions; ++q) batch_free_one(g, q);  // resized at the next call
        return TBC_OK;
    }
    if (key == TBC_OPT_NARROW_WIDTH) {
        if (!(value >= 0)) return set_error(TBC_ERR_INVALID, "narrow width %g", value);
        g->narrow_width = value;
        g->narrow = -1;  // decide again at the next call
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_WIDTH) {
        if (value != 0 && value != 32 && value != 64)
            return set_error(TBC_ERR_INVALID, "batch width %g not 0 (auto), 32 or 64", value);
        g->batch_width = (int)value;
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_PARTS) {
        int v = (int)value;
        if (v < 0 || v > kMaxPartitions || (double)v != value)
            return set_error(TBC_ERR_INVALID, "batch partitions %g not in [0 (auto), %d]", value, kMaxPartitions);
        g->batch_parts = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_ORDER) {
        int v = (int)value;
        if (v < 0 || v > 1 || (double)v != value) return set_error(TBC_ERR_INVALID, "batch order %g", value);
        g->batch_order = v;
        return TBC_OK;
    }
    if (key == TBC_OPT_BATCH_PULL) {
        if (!(value >= 0)) return set_error(TBC_ERR_INVALID, "batch pull ratio %g", value);
        g->batch_pull = value;
        return TBC_OK;
    }
    if (key >= TBC_OPT_COST_LIST && key <= TBC_OPT_COST_BPUSH) {
        if (!(value >= 0)) return set_error(TBC_ERR_INVALID, "cost %g", value);
        double *c[] = {&g->c_list, &g->c_stream, &g->c_atom, &g->c_vert, &g->c_scan, &g->c_bpush};
        *c[key - TBC_OPT_COST_LIST] = value;
        return TBC_OK;
    }
    return set_error(TBC_ERR_INVALID, "unknown option %d", key);
}

tbc_status tbc_bc_device(tbc_graph *g, const int32_t *d_sources, int64_t k, double *d_bc, void *cuda_stream) {
    g_err[0] = 0;
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (k < 0) return set_error(TBC_ERR_INVALID, "k < 0");
    if (k > 0 && (!d_sources || !d_bc)) return set_error(TBC_ERR_INVALID, "NULL device pointer");
    if (k == 0) return TBC_OK;
    cudaError_t e = cudaSetDevice(g->device);
    if (e != cudaSuccess) return cuda_error(e, "cudaSetDevice");
    return engine_run(g, d_sources, k, d_bc, (cudaStream_t)cuda_stream, 0);
}

tbc_status tbc_bc(tbc_graph *g, const int32_t *sources, int64_t k, double *bc_out) {
    g_err[0] = 0;
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (k < 0) return set_error(TBC_ERR_INVALID, "k < 0");
    if (!bc_out || (k > 0 && !sources)) return set_error(TBC_ERR_INVALID, "NULL pointer");
    for (int64_t i = 0; i < k; ++i)
        if (sources[i] < 0 || sources[i] >= g->n)
            return set_error(TBC_ERR_INVALID, "sources[%lld] = %d out of range", (long long)i, sources[i]);
    tbc_status st = TBC_OK;
    TBC_CUDA(cudaSetDevice(g->device));
    if (!g->bc_tmp) TBC_CUDA(dmalloc(g, &g->bc_tmp, g->n));
    if (k > g->src_cap) {
        cudaFree(g->src_tmp);
        g->src_tmp = nullptr;
        g->src_cap = 0;
        TBC_CUDA(cudaMalloc(&g->src_tmp, sizeof(int32_t) * k));
        g->src_cap = k;
    }
    TBC_CUDA(cudaMemsetAsync(g->bc_tmp, 0, sizeof(double) * g->n, g->stream));
    if (k > 0) {
        TBC_CUDA(cudaMemcpyAsync(g->src_tmp, sources, sizeof(int32_t) * k, cudaMemcpyHostToDevice, g->stream));
        st = engine_run(g, g->src_tmp, k, g->bc_tmp, g->stream, 0);
        if (st != TBC_OK) return st;
    }
    TBC_CUDA(cudaMemcpyAsync(bc_out, g->bc_tmp, sizeof(double) * g->n, cudaMemcpyDeviceToHost, g->stream));
    TBC_CUDA(cudaStreamSynchronize(g->stream));
    return TBC_OK;
fail:
    return st;
}

tbc_status tbc_bfs(tbc_graph *g, int32_t source, int32_t *depth_out, double *sigma_out) {
    g_err[0] = 0;
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (source < 0 || source >= g->n) return set_error(TBC_ERR_INVALID, "source %d out of range", source);
    tbc_status st = TBC_OK;
    TBC_CUDA(cudaSetDevice(g->device));
    if (g->ws_count == 0) {  // one-format graphs carry no per-source engine: the batched forward stage
        std::vector<int32_t> d(depth_out ? 0 : g->n);
        std::vector<double> sg(sigma_out ? 0 : g->n);
        return tbc_bfs_batch(g, &source, 1, depth_out ? depth_out : d.data(), sigma_out ? sigma_out : sg.data());
    }
    if (g->src_cap < 1) {
        TBC_CUDA(cudaMalloc(&g->src_tmp, sizeof(int32_t)));
        g->src_cap = 1;
    }
    TBC_CUDA(cudaMemcpyAsync(g->src_tmp, &source, sizeof(int32_t), cudaMemcpyHostToDevice, g->stream));
    st = engine_run(g, g->src_tmp, 1, nullptr, g->stream, 1);
    if (st != TBC_OK) return st;
    {
        const Workspace &w = g->ws[0];  // a forward-only run uses partition 0
        const int32_t *dsrc = w.depth;
        const double *ssrc = w.sigma;
        if (g->perm) {  // back to the caller's labels (list_v / bc_tmp are free scratch here)
            if (!g->bc_tmp) TBC_CUDA(dmalloc(g, &g->bc_tmp, g->n));
            k_unpermute_bfs<<<grid_for(g->n), 256, 0, g->stream>>>(g->n, g->perm, w.depth, w.sigma, w.list_v,
                                                                   g->bc_tmp);
            TBC_CUDA(cudaGetLastError());
            dsrc = w.list_v;
            ssrc = g->bc_tmp;
        }
        if (depth_out)
            TBC_CUDA(cudaMemcpyAsync(depth_out, dsrc, sizeof(int32_t) * g->n, cudaMemcpyDeviceToHost, g->stream));
        if (sigma_out)
            TBC_CUDA(cudaMemcpyAsync(sigma_out, ssrc, sizeof(double) * g->n, cudaMemcpyDeviceToHost, g->stream));
    }
    // forward-only runs leave depth/sigma set: restore the all-unvisited workspace invariant
    TBC_CUDA(cudaMemsetAsync(g->ws[0].depth, 0xff, sizeof(int32_t) * g->n, g->stream));
    TBC_CUDA(cudaMemsetAsync(g->ws[0].sigma, 0, sizeof(double) * g->n, g->stream));
    TBC_CUDA(cudaStreamSynchronize(g->stream));
    return TBC_OK;
fail:
    return st;
}

static tbc_status bfs_batch_impl(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out,
                                 double *sigma_out, int32_t *sexp_out);

tbc_status tbc_bfs_batch(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out, double *sigma_out) {
    g_err[0] = 0;
    return bfs_batch_impl(g, sources, k, depth_out, sigma_out, nullptr);
}

tbc_status tbc_bfs_batch_ext(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out,
                             double *sigma_mant_out, int32_t *sigma_exp_out) {
    g_err[0] = 0;
    if (k > 0 && !sigma_exp_out) return set_error(TBC_ERR_INVALID, "NULL pointer");
    return bfs_batch_impl(g, sources, k, depth_out, sigma_mant_out, sigma_exp_out);
}

static tbc_status bfs_batch_impl(tbc_graph *g, const int32_t *sources, int64_t k, int32_t *depth_out,
                                 double *sigma_out, int32_t *sexp_out) {
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    if (k < 0) return set_error(TBC_ERR_INVALID, "k < 0");
    if (k > 0 && (!sources || !depth_out || !sigma_out)) return set_error(TBC_ERR_INVALID, "NULL pointer");
    if (g->engine != TBC_ENGINE_CSC) return set_error(TBC_ERR_UNSUPPORTED, "tbc_bfs_batch: CSC engine only");
    if (g->batch == 0 && g->ws_count > 0)
        return set_error(TBC_ERR_UNSUPPORTED, "tbc_bfs_batch: per-source engine selected (use tbc_bfs)");
    for (int64_t i = 0; i < k; ++i)
        if (sources[i] < 0 || sources[i] >= g->n)
            return set_error(TBC_ERR_INVALID, "sources[%lld] = %d out of range", (long long)i, sources[i]);
    if (k == 0) return TBC_OK;
    if (k > (int64_t)((1ull << 62) / (uint64_t)g->n)) return set_error(TBC_ERR_INVALID, "k * n overflows");
    tbc_status st = TBC_OK;
    const int64_t kn = k * g->n;
    TBC_CUDA(cudaSetDevice(g->device));
    if (kn > g->bfs_cap || (sexp_out && !g->bfs_sexp)) {
        cudaFree(g->bfs_depth);
        cudaFree(g->bfs_sigma);
        cudaFree(g->bfs_sexp);
        g->bfs_depth = nullptr;
        g->bfs_sigma = nullptr;
        g->bfs_sexp = nullptr;
        g->bfs_cap = 0;
        TBC_CUDA(cudaMalloc(&g->bfs_depth, sizeof(int32_t) * kn));
        TBC_CUDA(cudaMalloc(&g->bfs_sigma, sizeof(double) * kn));
        if (sexp_out) TBC_CUDA(cudaMalloc(&g->bfs_sexp, sizeof(int32_t) * kn));
        g->bfs_cap = kn;
    }
    if (k > g->src_cap) {
        cudaFree(g->src_tmp);
        g->src_tmp = nullptr;
        g->src_cap = 0;
        TBC_CUDA(cudaMalloc(&g->src_tmp, sizeof(int32_t) * k));
        g->src_cap = k;
    }
    TBC_CUDA(cudaMemsetAsync(g->bfs_depth, 0xff, sizeof(int32_t) * kn, g->stream));
    TBC_CUDA(cudaMemsetAsync(g->bfs_sigma, 0, sizeof(double) * kn, g->stream));
    TBC_CUDA(cudaMemcpyAsync(g->src_tmp, sources, sizeof(int32_t) * k, cudaMemcpyHostToDevice, g->stream));
    {
        int mode = 1;
        st = engine_choose(g, g->src_tmp, k, g->stream, &mode);
        if (st != TBC_OK) return st;
        st = mode == 2 ? single_run(g, g->src_tmp, k, nullptr, g->stream, g->bfs_depth, g->bfs_sigma,
                                    sexp_out ? g->bfs_sexp : nullptr)
                       : batch_run(g, g->src_tmp, k, nullptr, g->stream, g->bfs_depth, g->bfs_sigma);
        if (st != TBC_OK) return st;
        TBC_CUDA(cudaMemcpyAsync(depth_out, g->bfs_depth, sizeof(int32_t) * kn, cudaMemcpyDeviceToHost, g->stream));
        TBC_CUDA(cudaMemcpyAsync(sigma_out, g->bfs_sigma, sizeof(double) * kn, cudaMemcpyDeviceToHost, g->stream));
        if (sexp_out && mode == 2)
            TBC_CUDA(cudaMemcpyAsync(sexp_out, g->bfs_sexp, sizeof(int32_t) * kn, cudaMemcpyDeviceToHost, g->stream));
        TBC_CUDA(cudaStreamSynchronize(g->stream));
        if (sexp_out && mode != 2)  // fp64 engines: split the (finite) sigma into mantissa and exponent
            for (int64_t i = 0; i < kn; ++i) {
                int e = 0;
                sigma_out[i] = frexp(sigma_out[i], &e);
                sexp_out[i] = e;
            }
    }
    return TBC_OK;
fail:
    return st;
}

tbc_status tbc_stats_get(tbc_graph *g, tbc_stats *out) {
    if (!g || !out) return set_error(TBC_ERR_INVALID, "NULL pointer");
    tbc_status st = TBC_OK;
    Ctrs c;
    TBC_CUDA(cudaSetDevice(g->device));
    TBC_CUDA(cudaDeviceSynchronize());
    *out = tbc_stats{};
    out->batch_width = g->last_width;
    out->batch_parts = g->last_parts;
    out->engine = g->last_mode;
    out->probe_width = (int64_t)g->probe_width;
    for (int q = 0; q < kMaxPartitions; ++q) out->workspace_bytes += (int64_t)g->bws[q].bytes;
    out->workspace_bytes += (int64_t)g->ws_bytes + (int64_t)g->sws.bytes;
    for (int i = 0; i < g->ws_count + kMaxPartitions + 2; ++i) {  // per-source, batched, narrow-level, retired
        Ctrs *src = i < g->ws_count ? g->ws[i].ctr
                    : i < g->ws_count + kMaxPartitions ? g->bws[i - g->ws_count].ctr
                    : i == g->ws_count + kMaxPartitions ? g->sws.ctr : nullptr;
        if (i == g->ws_count + kMaxPartitions + 1) c = g->retired;
        else if (!src) continue;
        else TBC_CUDA(cudaMemcpy(&c, src, sizeof c, cudaMemcpyDeviceToHost));
        out->bad_sources += (int64_t)c.bad_sources;
        if (c.st_list_peak > out->list_peak) out->list_peak = c.st_list_peak;
        out->list_overflows += c.st_overflows;
        out->xr_sources += c.st_xr_sources;
        out->sources += c.st_sources;
        out->reached += c.st_reached;
        out->reached_edges += c.st_reached_edges;
        out->fwd_edges += c.st_fwd_edges;
        out->bwd_edges += c.st_bwd_edges;
        out->levels += c.st_levels;
        out->pull_levels += c.st_pull_levels;
        out->scans += c.st_scans;
        if (c.st_max_depth > out->max_depth) out->max_depth = c.st_max_depth;
    }
    return TBC_OK;
fail:
    return st;
}

tbc_status tbc_trace_get(tbc_graph *g, int64_t *out, int64_t cap, int64_t *count) {
    if (!g || !count || (cap > 0 && !out)) return set_error(TBC_ERR_INVALID, "NULL pointer");
    tbc_status st = TBC_OK;
    Ctrs c;
    int64_t nrec = 0;
    TBC_CUDA(cudaSetDevice(g->device));
    TBC_CUDA(cudaDeviceSynchronize());
    TBC_CUDA(cudaMemcpy(&c, g->gctr, sizeof c, cudaMemcpyDeviceToHost));
    nrec = (int64_t)c.trace_n;
    if (nrec > kTraceCap) nrec = kTraceCap;
    *count = nrec;
    if (cap > 0 && nrec > 0)
        TBC_CUDA(cudaMemcpy(out, g->trace, sizeof(int64_t) * 8 * (nrec < cap ? nrec : cap), cudaMemcpyDeviceToHost));
    return TBC_OK;
fail:
    return st;
}

tbc_status tbc_profile_get(tbc_graph *g, uint64_t *out, int64_t cap, int64_t *count) {
    if (!g || !count || (cap > 0 && !out)) return set_error(TBC_ERR_INVALID, "NULL pointer");
#ifndef TBC_PROF
    *count = 0;
    return set_error(TBC_ERR_UNSUPPORTED, "library built without TBC_PROF");
#else
    tbc_status st = TBC_OK;
    Ctrs c;
    TBC_CUDA(cudaSetDevice(g->device));
    TBC_CUDA(cudaDeviceSynchronize());
    TBC_CUDA(cudaMemcpy(&c, g->gctr, sizeof c, cudaMemcpyDeviceToHost));
    *count = 32;
    for (int64_t i = 0; i < cap && i < 32; ++i) out[i] = c.prof[i];
    TBC_CUDA(cudaMemset(g->gctr->prof, 0, sizeof c.prof));
    return TBC_OK;
fail:
    return st;
#endif
}

static constexpr size_t kStatBytes = offsetof(Ctrs, st_xr_sources) + sizeof(long long) - offsetof(Ctrs, st_sources);

tbc_status tbc_stats_reset(tbc_graph *g) {
    if (!g) return set_error(TBC_ERR_INVALID, "graph is NULL");
    tbc_status st = TBC_OK;
    TBC_CUDA(cudaSetDevice(g->device));
    TBC_CUDA(cudaDeviceSynchronize());
    for (int i = 0; i < g->ws_count + kMaxPartitions + 1; ++i) {
        Ctrs *c = i < g->ws_count ? g->ws[i].ctr
                  : i < g->ws_count + kMaxPartitions ? g->bws[i - g->ws_count].ctr : g->sws.ctr;
        if (!c) continue;
        TBC_CUDA(cudaMemset(&c->st_sources, 0, kStatBytes));  // st_sources .. st_xr_sources
        TBC_CUDA(cudaMemset(&c->bad_sources, 0, sizeof(unsigned long long)));
    }
    g->retired = Ctrs{};
    return TBC_OK;
fail:
    return st;
}

}  // extern "C"
