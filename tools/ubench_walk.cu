// ubench_walk.cu -- per-SM throughput of the arc walk (development aid):
// warps walk 256-arc chunks of a random colidx, loading deg[u] (ld.cg) and
// optionally atomicSub'ing it, with U arcs per lane in flight.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_walk tools/ubench_walk.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); return 1;} } while (0)

__device__ __forceinline__ int ld_stream(const int *p) { int v; asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p)); return v; }

template <int U, int MODE>
__global__ void k_walk(const int *colidx, int *deg, long long chunks_per_warp, int K, int *sink)
{
    const int lane = threadIdx.x & 31;
    const long long gw = (long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    int acc = 0;
    for (long long c = 0; c < chunks_per_warp; c++) {
        const long long base = (gw * chunks_per_warp + c) * 256;
        for (int a = 0; a < 256; a += 32 * U) {
            int u[U];
#pragma unroll
            for (int r = 0; r < U; r++) u[r] = ld_stream(colidx + base + a + r * 32 + lane);
            if (MODE == 2) { for (int r = 0; r < U; r++) acc += u[r]; continue; }
            int d[U];
#pragma unroll
            for (int r = 0; r < U; r++) d[r] = __ldcg(deg + u[r]);
            if (MODE == 3) {  // red.sub without return, no deg read
#pragma unroll
                for (int r = 0; r < U; r++) atomicSub(deg + u[r], 1);
                continue;
            }
            if (MODE == 4) {  // atomicSub with return, no deg read
#pragma unroll
                for (int r = 0; r < U; r++) acc += atomicSub(deg + u[r], 1);
                continue;
            }
            if (MODE == 1) {
#pragma unroll
                for (int r = 0; r < U; r++) if (d[r] > K) acc += atomicSub(deg + u[r], 1);
            } else {
#pragma unroll
                for (int r = 0; r < U; r++) acc += d[r];
            }
        }
    }
    if (acc == 0x7fffffff) sink[0] = acc;
}

template <int U, int MODE>
float run(const int *ci, int *deg, int grid, int block, long long cpw, int K, int *sink)
{
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    k_walk<U, MODE><<<grid, block>>>(ci, deg, cpw, K, sink);
    cudaEventRecord(e0);
    k_walk<U, MODE><<<grid, block>>>(ci, deg, cpw, K, sink);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main()
{
    const long long M = 1LL << 27;   // arcs
    const int N = 1 << 22;           // vertices (16 MB deg: L2 resident)
    int *ci, *deg, *sink;
    CK(cudaMalloc(&ci, M * 4)); CK(cudaMalloc(&deg, (size_t)N * 4)); CK(cudaMalloc(&sink, 4));
    std::vector<int> h(M);
    uint64_t x = 88172645463325252ULL;
    for (long long i = 0; i < M; i++) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; h[i] = (int)(x % N); }
    CK(cudaMemcpy(ci, h.data(), M * 4, cudaMemcpyHostToDevice));
    std::vector<int> hd(N, 1 << 30);
    CK(cudaMemcpy(deg, hd.data(), (size_t)N * 4, cudaMemcpyHostToDevice));
    const int block = 768, warps = block / 32;
    for (int hot : {1 << 22, 1 << 16, 1 << 12}) {
        std::vector<int> hh(M);
        for (long long i = 0; i < M; i++) hh[i] = h[i] % hot;
        CK(cudaMemcpy(ci, hh.data(), M * 4, cudaMemcpyHostToDevice));
        const int grid = 148; const long long cpw = 32;
        const double arcs = (double)grid * warps * cpw * 256;
        float t;
        t = run<4, 0>(ci, deg, grid, block, cpw, 0, sink); printf("hot %8d  ld only      : %8.1f G arcs/s\n", hot, arcs / (t * 1e6));
        t = run<4, 1>(ci, deg, grid, block, cpw, 0, sink); printf("hot %8d  ld + atom    : %8.1f G arcs/s\n", hot, arcs / (t * 1e6));
        t = run<4, 4>(ci, deg, grid, block, cpw, 0, sink); printf("hot %8d  atom (ret)   : %8.1f G arcs/s\n", hot, arcs / (t * 1e6));
        t = run<4, 3>(ci, deg, grid, block, cpw, 0, sink); printf("hot %8d  red (no ret) : %8.1f G arcs/s\n", hot, arcs / (t * 1e6));
    }
    CK(cudaMemcpy(ci, h.data(), M * 4, cudaMemcpyHostToDevice));
    for (int grid : {1, 8, 148}) {
        const long long cpw = (grid == 148) ? 32 : 64;
        const double arcs = (double)grid * warps * cpw * 256;
        float t;
        t = run<4, 2>(ci, deg, grid, block, cpw, 0, sink); printf("grid %3d colidx only U4   : %8.1f arcs/us/SM\n", grid, arcs / (t * 1e3) / grid);
        t = run<4, 0>(ci, deg, grid, block, cpw, 0, sink); printf("grid %3d +deg ld   U4     : %8.1f arcs/us/SM\n", grid, arcs / (t * 1e3) / grid);
        t = run<8, 0>(ci, deg, grid, block, cpw, 0, sink); printf("grid %3d +deg ld   U8     : %8.1f arcs/us/SM\n", grid, arcs / (t * 1e3) / grid);
        t = run<4, 1>(ci, deg, grid, block, cpw, 0, sink); printf("grid %3d +atomic   U4     : %8.1f arcs/us/SM\n", grid, arcs / (t * 1e3) / grid);
        t = run<8, 1>(ci, deg, grid, block, cpw, 0, sink); printf("grid %3d +atomic   U8     : %8.1f arcs/us/SM\n", grid, arcs / (t * 1e3) / grid);
    }
    return 0;
}
