// kcore_extract.cu -- k-shell / k-core outputs of a decomposition
// (include/kcore.h "Outputs").
//
//   kcore_kshell         the k-shell {v : core(v) == k}        (Sec. II-A)
//   kcore_kcore_mask     the k-core  {v : core(v) >= k}        (the k-cores
//                        are nested, so the k-core is exactly the vertices whose
//                        core number is at least k)
//   kcore_kcore_subgraph the induced k-core subgraph, renumbered in increasing id
//                        (k-cores as the pre-processing step of dense-
//                        subgraph mining)
//
// All three are order-preserving stream compactions over core_out: a tile
// count pass, one single-block scan of the tile counts, and an emit pass that
// places each tile's survivors with warp ballots -- coalesced int4-friendly
// reads of core[] and no global atomics.  The subgraph adds a warp-per-vertex
// degree pass, the same scan over the kept rows, and a warp-per-vertex fill.
#include "kcore.h"

#include <cstdint>
#include <cuda_runtime.h>

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kT = 256;                  // threads per block
constexpr int kItems = 16;               // elements per thread per tile
constexpr int kTile = kT * kItems;       // 4096 vertices per tile

enum { SEL_SHELL = 0, SEL_CORE = 1 };

__device__ __forceinline__ bool sel(int mode, int32_t c, int32_t k) { return mode == SEL_SHELL ? c == k : c >= k; }

__device__ __forceinline__ unsigned lanemask_lt()
{
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Block-wide exclusive scan of one int64 per thread (kT threads); total out.
__device__ __forceinline__ int64_t block_scan(int64_t x, int64_t *wsum, int64_t &total)
{
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int64_t t = __shfl_up_sync(kFull, inc, o);
        if (lane >= o) inc += t;
    }
    if (lane == 31) wsum[w] = inc;
    __syncthreads();
    if (w == 0) {
        int64_t s = lane < kT / 32 ? wsum[lane] : 0;
        int64_t si = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t t = __shfl_up_sync(kFull, si, o);
            if (lane >= o) si += t;
        }
        if (lane < kT / 32) wsum[lane] = si - s;
        if (lane == kT / 32 - 1) wsum[kT / 32] = si;
    }
    __syncthreads();
    const int64_t r = wsum[w] + inc - x;
    total = wsum[kT / 32];
    __syncthreads();
    return r;
}

// pass 1: survivors per tile
__global__ void __launch_bounds__(kT) k_tile_count(const int32_t *core, int64_t n, int32_t k, int mode,
                                                   int64_t *tile_cnt)
{
    __shared__ int64_t wsum[kT / 32 + 1];
    const int64_t base = (int64_t)blockIdx.x * kTile;
    int64_t c = 0;
#pragma unroll 4
    for (int j = 0; j < kItems; j++) {
        const int64_t i = base + (int64_t)j * kT + threadIdx.x;
        if (i < n && sel(mode, __ldg(core + i), k)) c++;
    }
    int64_t tot;
    block_scan(c, wsum, tot);
    if (threadIdx.x == 0) tile_cnt[blockIdx.x] = tot;
}

// exclusive scan of `cnt` in place (one block, any length); total to *total
__global__ void __launch_bounds__(kT) k_scan_i64(int64_t *cnt, int64_t len, int64_t *total)
{
    __shared__ int64_t wsum[kT / 32 + 1];
    int64_t carry = 0;
    for (int64_t b = 0; b < len; b += kT) {
        const int64_t i = b + threadIdx.x;
        const int64_t x = i < len ? cnt[i] : 0;
        int64_t tot;
        const int64_t ex = block_scan(x, wsum, tot);
        if (i < len) cnt[i] = carry + ex;
        carry += tot;
    }
    if (threadIdx.x == 0) *total = carry;
}

// pass 2: emit survivors of each tile in increasing id (list and/or mask)
__global__ void __launch_bounds__(kT) k_tile_emit(const int32_t *core, int64_t n, int32_t k, int mode,
                                                  const int64_t *tile_off, int32_t *list, uint8_t *mask,
                                                  int32_t *newid)
{
    __shared__ int64_t wsum[kT / 32 + 1];
    const int64_t base = (int64_t)blockIdx.x * kTile;
    int64_t off = tile_off[blockIdx.x];
    for (int j = 0; j < kItems; j++) {
        const int64_t i = base + (int64_t)j * kT + threadIdx.x;
        const bool s = i < n && sel(mode, __ldg(core + i), k);
        if (mask && i < n) mask[i] = s ? 1 : 0;
        int64_t tot;
        const int64_t ex = block_scan(s ? 1 : 0, wsum, tot);
        if (s && list) list[off + ex] = (int32_t)i;
        if (newid && i < n) newid[i] = s ? (int32_t)(off + ex) : -1;
        off += tot;
    }
}

// subgraph pass A: kept neighbours of each kept vertex (warp per vertex)
__global__ void k_sub_degree(const int64_t *rowptr, const int32_t *colidx, const int32_t *core, int32_t k,
                             const int32_t *vmap, int64_t nk, int64_t *sub_deg)
{
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < nk; i += nw) {
        const int32_t v = vmap[i];
        const int64_t b = rowptr[v], e = rowptr[v + 1];
        int64_t c = 0;
        for (int64_t x = b + lane; x < e; x += 32) c += __ldg(core + colidx[x]) >= k;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(kFull, c, o);
        if (lane == 0) sub_deg[i] = c;
    }
}

// subgraph pass B: write each kept row, order preserved (newid is monotone)
__global__ void k_sub_fill(const int64_t *rowptr, const int32_t *colidx, const int32_t *core, int32_t k,
                           const int32_t *vmap, const int32_t *newid, int64_t nk, const int64_t *sub_rowptr,
                           int32_t *sub_colidx)
{
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < nk; i += nw) {
        const int32_t v = vmap[i];
        const int64_t b = rowptr[v], e = rowptr[v + 1];
        int64_t o = sub_rowptr[i];
        for (int64_t x0 = b; x0 < e; x0 += 32) {
            const int64_t x = x0 + lane;
            int32_t u = -1;
            bool keep = false;
            if (x < e) {
                u = colidx[x];
                keep = __ldg(core + u) >= k;
            }
            const unsigned bal = __ballot_sync(kFull, keep);
            if (keep) sub_colidx[o + __popc(bal & lanemask_lt())] = newid[u];
            o += __popc(bal);
        }
    }
}

int map_err(cudaError_t e) { return e == cudaErrorMemoryAllocation ? KCORE_ENOMEM : KCORE_ECUDA; }

// Order-preserving selection of core[] (shell or core); outputs optional.
int select_vertices(const int32_t *core, int64_t n, int32_t k, int mode, int32_t *list, uint8_t *mask,
                    int32_t *newid, int64_t *count, cudaStream_t st)
{
    const int64_t tiles = (n + kTile - 1) / kTile;
    int64_t *d = nullptr;  // tile counts / offsets + total
    int64_t h_total = 0;
    cudaError_t e = cudaMallocAsync((void **)&d, sizeof(int64_t) * (size_t)(tiles + 1), st);
    if (e != cudaSuccess) return map_err(e);
    k_tile_count<<<(unsigned)tiles, kT, 0, st>>>(core, n, k, mode, d);
    k_scan_i64<<<1, kT, 0, st>>>(d, tiles, d + tiles);
    if (list || mask || newid) k_tile_emit<<<(unsigned)tiles, kT, 0, st>>>(core, n, k, mode, d, list, mask, newid);
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemcpyAsync(&h_total, d + tiles, sizeof(int64_t), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFreeAsync(d, st);
    if (e != cudaSuccess) return map_err(e);
    if (count) *count = h_total;
    return KCORE_OK;
}

} // namespace

extern "C" int kcore_kshell(const int32_t *core, int64_t n, int32_t k, int32_t *vertices_out, int64_t *count_out,
                            void *stream)
{
    if (n < 0 || n >= ((int64_t)1 << 31) || (n > 0 && !core)) return KCORE_EINVAL;
    if (n == 0) {
        if (count_out) *count_out = 0;
        return KCORE_OK;
    }
    return select_vertices(core, n, k, SEL_SHELL, vertices_out, nullptr, nullptr, count_out, (cudaStream_t)stream);
}

extern "C" int kcore_kcore_mask(const int32_t *core, int64_t n, int32_t k, uint8_t *mask_out, int64_t *count_out,
                                void *stream)
{
    if (n < 0 || n >= ((int64_t)1 << 31) || (n > 0 && (!core || !mask_out))) return KCORE_EINVAL;
    if (n == 0) {
        if (count_out) *count_out = 0;
        return KCORE_OK;
    }
    return select_vertices(core, n, k, SEL_CORE, nullptr, mask_out, nullptr, count_out, (cudaStream_t)stream);
}

extern "C" int kcore_kcore_subgraph(const int64_t *rowptr, const int32_t *colidx, const int32_t *core, int64_t n,
                                    int64_t m, int32_t k, int64_t *nk_out, int64_t *mk_out, int64_t *sub_rowptr,
                                    int32_t *sub_colidx, int32_t *vmap_out, void *stream)
{
    if (n < 0 || n >= ((int64_t)1 << 31) || m < 0 || !nk_out || !mk_out) return KCORE_EINVAL;
    if (n > 0 && (!rowptr || !core)) return KCORE_EINVAL;
    if (m > 0 && !colidx) return KCORE_EINVAL;
    const bool fill = sub_rowptr != nullptr;
    if (fill && !vmap_out) return KCORE_EINVAL;
    if (n == 0) {
        *nk_out = *mk_out = 0;
        if (fill) return cudaMemsetAsync(sub_rowptr, 0, sizeof(int64_t), (cudaStream_t)stream) == cudaSuccess
                             ? KCORE_OK : KCORE_ECUDA;
        return KCORE_OK;
    }
    cudaStream_t st = (cudaStream_t)stream;
    int32_t *vmap = nullptr, *newid = nullptr;
    int64_t *deg = nullptr;
    int64_t nk = 0, mk = 0;
    int rc = KCORE_OK;
    cudaError_t e = cudaMallocAsync((void **)&newid, sizeof(int32_t) * (size_t)n, st);
    if (e == cudaSuccess && !fill) e = cudaMallocAsync((void **)&vmap, sizeof(int32_t) * (size_t)n, st);
    if (e != cudaSuccess) { rc = map_err(e); goto done; }
    rc = select_vertices(core, n, k, SEL_CORE, fill ? vmap_out : vmap, nullptr, newid, &nk, st);
    if (rc) goto done;
    if (nk > 0) {
        // row degrees of G[k-core] into sub_rowptr[0..nk) (or scratch), exclusive scan -> row offsets
        int64_t *dg = sub_rowptr;
        if (!fill) {
            e = cudaMallocAsync((void **)&deg, sizeof(int64_t) * (size_t)(nk + 1), st);
            if (e != cudaSuccess) { rc = map_err(e); goto done; }
            dg = deg;
        }
        const int32_t *vm = fill ? vmap_out : vmap;
        const unsigned blocks = (unsigned)std::min<int64_t>((nk + 7) / 8, 148 * 16);
        k_sub_degree<<<blocks, 256, 0, st>>>(rowptr, colidx, core, k, vm, nk, dg);
        k_scan_i64<<<1, kT, 0, st>>>(dg, nk, dg + nk);
        if (fill) k_sub_fill<<<blocks, 256, 0, st>>>(rowptr, colidx, core, k, vm, newid, nk, dg, sub_colidx);
        e = cudaGetLastError();
        if (e == cudaSuccess) e = cudaMemcpyAsync(&mk, dg + nk, sizeof(int64_t), cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) { rc = map_err(e); goto done; }
    } else if (fill) {
        e = cudaMemsetAsync(sub_rowptr, 0, sizeof(int64_t), st);
        if (e != cudaSuccess) { rc = map_err(e); goto done; }
    }
    *nk_out = nk;
    *mk_out = mk;
done:
    if (newid) cudaFreeAsync(newid, st);
    if (vmap) cudaFreeAsync(vmap, st);
    if (deg) cudaFreeAsync(deg, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && rc == KCORE_OK) rc = KCORE_ECUDA;
    return rc;
}
