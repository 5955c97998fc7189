/*
 * kcgen_device.cu -- device implementation of the synthetic graph generator
 * (see kcgen.h).  Same counter-based draws as kcgen_host.c (kcgen_rng.h), so
 * the CSR is byte-identical; the work is a generate -> radix sort (CUB) ->
 * unique -> row-boundary pipeline.  Input infrastructure, not the hot path.
 */
#include "../include/kcgen.h"
#include "kcgen_rng.h"

#include <cub/cub.cuh>
#include <cuda_runtime.h>

namespace {

struct GenArgs {
    kcg_params p;
    uint64_t n;
    kcg_perm perm;
    const double *cdf;
    int vb;
    int64_t v_begin, v_end;
};

__device__ __forceinline__ void dev_edge(const GenArgs &g, uint64_t i, uint64_t *u, uint64_t *v)
{
    if (g.p.kind == KCG_RMAT)
        kcg_rmat_edge(g.p.seed, i, g.p.scale, g.p.a, g.p.b, g.p.c, u, v);
    else if (g.p.kind == KCG_ER)
        kcg_er_edge(g.p.seed, i, g.n, u, v);
    else
        kcg_chunglu_edge(g.p.seed, i, g.cdf, g.n, u, v);
    if (g.p.permute) {
        *u = kcg_perm_apply(&g.perm, *u);
        *v = kcg_perm_apply(&g.perm, *v);
    }
}

/* emit the (up to two) in-range arcs of each edge; keys = (src << vb) | dst.
 * keys == nullptr: count only. */
__global__ void k_gen_keys(GenArgs g, uint64_t *keys, unsigned long long *cursor)
{
    const unsigned lane = threadIdx.x & 31;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t M = (uint64_t)g.p.num_edges;
    for (uint64_t base = (uint64_t)blockIdx.x * blockDim.x; base < M; base += stride) {
        uint64_t i = base + threadIdx.x;
        uint64_t u = 0, v = 0;
        int e0 = 0, e1 = 0;
        if (i < M) {
            dev_edge(g, i, &u, &v);
            if (u != v) {
                e0 = ((int64_t)u >= g.v_begin && (int64_t)u < g.v_end);
                e1 = ((int64_t)v >= g.v_begin && (int64_t)v < g.v_end);
            }
        }
        int mine = e0 + e1;
        /* warp-aggregated reservation */
        unsigned active = __activemask();
        int incl = mine;
        for (int o = 1; o < 32; o <<= 1) {
            int t = __shfl_up_sync(active, incl, o);
            if ((int)lane >= o) incl += t;
        }
        int tot = __shfl_sync(active, incl, 31);
        unsigned long long b = 0;
        if (lane == 31 && tot) b = atomicAdd(cursor, (unsigned long long)tot);
        b = __shfl_sync(active, b, 31);
        if (keys) {
            unsigned long long at = b + (unsigned long long)(incl - mine);
            if (e0) keys[at++] = (u << g.vb) | v;
            if (e1) keys[at] = (v << g.vb) | u;
        }
    }
}

__global__ void k_rows(const uint64_t *keys, int64_t m, int vb, int64_t v_begin, int64_t nl,
                       int64_t *rowptr, int32_t *colidx)
{
    const uint64_t mask = (1ULL << vb) - 1;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (int64_t)gridDim.x * blockDim.x) {
        uint64_t k = keys[i];
        colidx[i] = (int32_t)(k & mask);
        int64_t s = (int64_t)(k >> vb) - v_begin;
        int64_t sp = (i == 0) ? -1 : (int64_t)(keys[i - 1] >> vb) - v_begin;
        for (int64_t v = sp + 1; v <= s; v++) rowptr[v] = i;
        if (i == m - 1)
            for (int64_t v = s + 1; v <= nl; v++) rowptr[v] = m;
    }
}

__global__ void k_fill(int64_t *rowptr, int64_t cnt, int64_t val)
{
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt;
         i += (int64_t)gridDim.x * blockDim.x)
        rowptr[i] = val;
}

} // namespace

#define CK(x)                                                                                      \
    do {                                                                                           \
        if ((x) != cudaSuccess) { rc = KCG_ECUDA; goto done; }                                     \
    } while (0)

extern "C" int64_t kcg_device_generate(const kcg_params *p, int64_t v_begin, int64_t v_end,
                                       int64_t *rowptr, int32_t *colidx, int64_t colidx_cap,
                                       void *stream_)
{
    cudaStream_t st = (cudaStream_t)stream_;
    int64_t n = kcg_num_vertices(p);
    if (n < 0 || p->num_edges < 0 || v_begin < 0 || v_end > n || v_begin > v_end ||
        (colidx && !rowptr))
        return KCG_EINVAL;
    int64_t rc = 0;
    GenArgs g;
    g.p = *p;
    g.n = (uint64_t)n;
    g.perm = kcg_perm_make((uint64_t)n, p->seed);
    g.cdf = nullptr;
    g.vb = 0;
    while (((int64_t)1 << g.vb) < n) g.vb++;
    if (g.vb == 0) g.vb = 1;
    g.v_begin = v_begin;
    g.v_end = v_end;

    double *h_cdf = nullptr, *d_cdf = nullptr;
    unsigned long long *d_cursor = nullptr;
    int64_t *d_nsel = nullptr;
    uint64_t *k0 = nullptr, *k1 = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0, tb2 = 0;
    unsigned long long cnt = 0;
    int64_t m = 0;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = sms * 8, block = 256;

    if (p->kind == KCG_CHUNGLU) {
        h_cdf = (double *)malloc(sizeof(double) * (size_t)n);
        if (!h_cdf) return KCG_ENOMEM;
        kcg_build_cdf(p, h_cdf);
        CK(cudaMallocAsync((void **)&d_cdf, sizeof(double) * (size_t)n, st));
        CK(cudaMemcpyAsync(d_cdf, h_cdf, sizeof(double) * (size_t)n, cudaMemcpyHostToDevice, st));
        g.cdf = d_cdf;
    }
    CK(cudaMallocAsync((void **)&d_cursor, sizeof(unsigned long long), st));
    CK(cudaMallocAsync((void **)&d_nsel, sizeof(int64_t), st));
    /* pass 1: count in-range arcs */
    CK(cudaMemsetAsync(d_cursor, 0, sizeof(unsigned long long), st));
    k_gen_keys<<<grid, block, 0, st>>>(g, nullptr, d_cursor);
    CK(cudaGetLastError());
    CK(cudaMemcpyAsync(&cnt, d_cursor, sizeof(cnt), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (cnt > 0) {
        CK(cudaMallocAsync((void **)&k0, sizeof(uint64_t) * cnt, st));
        CK(cudaMallocAsync((void **)&k1, sizeof(uint64_t) * cnt, st));
        CK(cudaMemsetAsync(d_cursor, 0, sizeof(unsigned long long), st));
        k_gen_keys<<<grid, block, 0, st>>>(g, k0, d_cursor);
        CK(cudaGetLastError());
        CK(cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, k0, k1, (int64_t)cnt, 0, 2 * g.vb, st));
        CK(cub::DeviceSelect::Unique(nullptr, tb2, k1, k0, d_nsel, (int64_t)cnt, st));
        if (tb2 > tmp_bytes) tmp_bytes = tb2;
        CK(cudaMallocAsync(&tmp, tmp_bytes, st));
        tb2 = tmp_bytes;
        CK(cub::DeviceRadixSort::SortKeys(tmp, tb2, k0, k1, (int64_t)cnt, 0, 2 * g.vb, st));
        tb2 = tmp_bytes;
        CK(cub::DeviceSelect::Unique(tmp, tb2, k1, k0, d_nsel, (int64_t)cnt, st));
        CK(cudaMemcpyAsync(&m, d_nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
    }
    if (colidx) {
        if (m > colidx_cap) { rc = KCG_ECAP; goto done; }
        int64_t nloc = v_end - v_begin;
        if (m == 0) {
            k_fill<<<grid, block, 0, st>>>(rowptr, nloc + 1, 0);
        } else {
            k_rows<<<grid, block, 0, st>>>(k0, m, g.vb, v_begin, nloc, rowptr, colidx);
        }
        CK(cudaGetLastError());
    }
    rc = m;
done:
    if (tmp) cudaFreeAsync(tmp, st);
    if (k0) cudaFreeAsync(k0, st);
    if (k1) cudaFreeAsync(k1, st);
    if (d_cursor) cudaFreeAsync(d_cursor, st);
    if (d_nsel) cudaFreeAsync(d_nsel, st);
    if (d_cdf) cudaFreeAsync(d_cdf, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && rc >= 0) rc = KCG_ECUDA;
    free(h_cdf);
    return rc;
}
