// ubench_arcs.cu -- development microbenchmark (not product): per-arc costs of
// the peel's primitives on a real CSR (R-MAT target skew), one full pass over
// every arc, grid-stride, 8 arcs per thread in flight.
//   mode 0  read colidx only (streaming bandwidth)
//   mode 1  RED     atomicSub(&deg[u], 1)            (no return)
//   mode 2  ATOM    old = atomicSub(&deg[u], 1)      (return consumed)
//   mode 3  LDG     ld.cg deg[u]                     (scattered read)
//   mode 4  LDG bitmap word bits[u>>5] then RED if the bit is clear
//   mode 5  LDG bitmap word then ATOM if clear
//   mode 6  shared-memory probe of a 64 KB table (Bloom-like LDS) + count
//   mode 7  RED on u & mask (working set `mask+1` ints)
//   mode 8  ATOM on u & mask
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC
//        tools/ubench_arcs.cu -o tools/libubench_arcs.so
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(512) k_arcs(const int32_t *__restrict__ colidx, int64_t m, int32_t *deg,
                                              const uint32_t *bits, uint32_t mask, unsigned long long *sink)
{
    extern __shared__ uint32_t tab[];
    if (MODE == 6) {
        for (int i = threadIdx.x; i < 16384; i += blockDim.x) tab[i] = (uint32_t)i * 2654435761u;
        __syncthreads();
    }
    const int64_t n8 = m / 8;
    const int4 *c4 = reinterpret_cast<const int4 *>(colidx);
    unsigned long long acc = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n8; i += (int64_t)gridDim.x * blockDim.x) {
        int4 a, b;
        asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(a.x), "=r"(a.y), "=r"(a.z), "=r"(a.w) : "l"(c4 + 2 * i));
        asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(b.x), "=r"(b.y), "=r"(b.z), "=r"(b.w) : "l"(c4 + 2 * i + 1));
        const int32_t u[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
        if (MODE == 0) {
#pragma unroll
            for (int r = 0; r < 8; r++) acc += (unsigned)u[r];
        } else if (MODE == 1) {
#pragma unroll
            for (int r = 0; r < 8; r++) atomicSub(deg + u[r], 1);
        } else if (MODE == 2) {
            int o[8];
#pragma unroll
            for (int r = 0; r < 8; r++) o[r] = atomicSub(deg + u[r], 1);
#pragma unroll
            for (int r = 0; r < 8; r++) acc += (o[r] == 7);
        } else if (MODE == 3) {
            int o[8];
#pragma unroll
            for (int r = 0; r < 8; r++) o[r] = __ldcg(deg + u[r]);
#pragma unroll
            for (int r = 0; r < 8; r++) acc += (o[r] == 7);
        } else if (MODE == 4 || MODE == 5) {
            uint32_t w[8];
#pragma unroll
            for (int r = 0; r < 8; r++) w[r] = __ldcg(bits + (u[r] >> 5));
            int o[8];
#pragma unroll
            for (int r = 0; r < 8; r++) {
                o[r] = 0;
                if (!((w[r] >> (u[r] & 31)) & 1u)) {
                    if (MODE == 4) atomicSub(deg + u[r], 1);
                    else o[r] = atomicSub(deg + u[r], 1);
                }
            }
#pragma unroll
            for (int r = 0; r < 8; r++) acc += (o[r] == 7);
        } else if (MODE == 6) {
#pragma unroll
            for (int r = 0; r < 8; r++) {
                const uint32_t h = ((uint32_t)u[r] * 0x9E3779B1u) >> 18;
                acc += (tab[h] >> (u[r] & 31)) & 1u;
            }
        } else if (MODE == 7) {
#pragma unroll
            for (int r = 0; r < 8; r++) atomicSub(deg + (u[r] & mask), 1);
        } else if (MODE == 8) {
            int o[8];
#pragma unroll
            for (int r = 0; r < 8; r++) o[r] = atomicSub(deg + (u[r] & mask), 1);
#pragma unroll
            for (int r = 0; r < 8; r++) acc += (o[r] == 7);
        }
    }
    if (acc == 0x123456789ULL) sink[0] = acc;
}

extern "C" float ubench_arcs(int mode, const int32_t *colidx, int64_t m, int32_t *deg, const uint32_t *bits,
                             uint32_t mask, int blocks_per_sm, int threads)
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long *sink;
    cudaMalloc(&sink, 8);
    const int grid = sms * blocks_per_sm;
    const size_t sh = mode == 6 ? 65536 : 0;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 3; rep++) {
        cudaEventRecord(e0);
        switch (mode) {
        case 0: k_arcs<0><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 1: k_arcs<1><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 2: k_arcs<2><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 3: k_arcs<3><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 4: k_arcs<4><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 5: k_arcs<5><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 6:
            cudaFuncSetAttribute(k_arcs<6>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
            k_arcs<6><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink);
            break;
        case 7: k_arcs<7><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        case 8: k_arcs<8><<<grid, threads, sh>>>(colidx, m, deg, bits, mask, sink); break;
        default: return -1.f;
        }
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    cudaFree(sink);
    if (cudaGetLastError() != cudaSuccess) return -2.f;
    return best;
}
