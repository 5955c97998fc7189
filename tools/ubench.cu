// ubench.cu -- B200 microbenchmarks for the primitives the k-core path is
// built from (development aid; results summarised in DESIGN.md).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench tools/ubench.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <string>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t *p) { uint32_t v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ void st_release(uint32_t *p, uint32_t v) { asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory"); }
__device__ __forceinline__ uint32_t atom_add_release(uint32_t *p, uint32_t v) { uint32_t o; asm volatile("atom.release.gpu.global.add.u32 %0, [%1], %2;" : "=r"(o) : "l"(p), "r"(v) : "memory"); return o; }
__device__ __forceinline__ uint64_t gtimer() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

// pointer chase: latency of dependent loads
__global__ void k_chase(const int *next, int steps, int start, long long *out_cycles, int *sink)
{
    int p = start;
    long long t0 = clock64();
    for (int i = 0; i < steps; i++) p = __ldcg(next + p);
    long long t1 = clock64();
    out_cycles[0] = t1 - t0;
    sink[0] = p;
}

__global__ void k_atomic_chase(int *arr, int steps, long long *out_cycles)
{
    int p = 0;
    long long t0 = clock64();
    for (int i = 0; i < steps; i++) p = atomicAdd(arr + (p & 1023) * 64, 0) + i;
    long long t1 = clock64();
    out_cycles[0] = t1 - t0;
    arr[5] = p;
}

__global__ void k_fence_cost(long long *out, int iters, int *buf)
{
    long long t0 = clock64();
    for (int i = 0; i < iters; i++) { buf[threadIdx.x] = i; __threadfence(); }
    long long t1 = clock64();
    if (threadIdx.x == 0) out[0] = (t1 - t0) / iters;
}

// scattered ops throughput over an array of `len` ints
template <int MODE>
__global__ void k_scatter(int *arr, uint32_t mask, long long per_thread, int *sink)
{
    uint32_t x = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u + 12345u;
    int acc = 0;
    for (long long i = 0; i < per_thread; i += 4) {
        uint32_t a0 = (x = x * 1664525u + 1013904223u) & mask;
        uint32_t a1 = (x = x * 1664525u + 1013904223u) & mask;
        uint32_t a2 = (x = x * 1664525u + 1013904223u) & mask;
        uint32_t a3 = (x = x * 1664525u + 1013904223u) & mask;
        if (MODE == 0) { acc += __ldcg(arr + a0) + __ldcg(arr + a1) + __ldcg(arr + a2) + __ldcg(arr + a3); }
        else if (MODE == 1) { acc += atomicSub(arr + a0, 1) + atomicSub(arr + a1, 1) + atomicSub(arr + a2, 1) + atomicSub(arr + a3, 1); }
        else if (MODE == 2) { atomicSub(arr + a0, 1); atomicSub(arr + a1, 1); atomicSub(arr + a2, 1); atomicSub(arr + a3, 1); }
        else if (MODE == 3) { acc += __ldg(arr + a0) + __ldg(arr + a1) + __ldg(arr + a2) + __ldg(arr + a3); }
    }
    if (acc == 0x7fffffff) sink[0] = acc;
}

__global__ void k_stream(const int4 *a, long long n4, int *sink)
{
    int acc = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x) {
        int4 v = __ldcs(a + i);
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (acc == 0x7fffffff) sink[0] = acc;
}

struct Bar { uint32_t count; uint32_t pad[31]; uint32_t gen; uint32_t pad2[31]; };

__global__ void k_barriers(Bar *b, int iters, uint64_t *t_out)
{
    uint64_t t0 = gtimer();
    for (int it = 0; it < iters; it++) {
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t gen = ld_acquire(&b->gen);
            __threadfence();
            uint32_t t = atom_add_release(&b->count, 1u);
            if (t + 1 == gridDim.x * (gen + 1)) {
                __threadfence();
                st_release(&b->gen, gen + 1);
            } else {
                while (ld_acquire(&b->gen) == gen) {}
            }
        }
        __syncthreads();
    }
    uint64_t t1 = gtimer();
    if (blockIdx.x == 0 && threadIdx.x == 0) t_out[0] = t1 - t0;
}

// barrier without the __threadfence calls (release/acquire only)
__global__ void k_barriers_nofence(Bar *b, int iters, uint64_t *t_out)
{
    uint64_t t0 = gtimer();
    for (int it = 0; it < iters; it++) {
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t gen = ld_acquire(&b->gen);
            uint32_t t = atom_add_release(&b->count, 1u);
            if (t + 1 == gridDim.x * (gen + 1)) {
                st_release(&b->gen, gen + 1);
            } else {
                while (ld_acquire(&b->gen) == gen) {}
            }
        }
        __syncthreads();
    }
    uint64_t t1 = gtimer();
    if (blockIdx.x == 0 && threadIdx.x == 0) t_out[0] = t1 - t0;
}

__global__ void k_syncthreads(int iters, uint64_t *t_out, long long *c_out)
{
    uint64_t t0 = gtimer();
    long long c0 = clock64();
    for (int it = 0; it < iters; it++) __syncthreads();
    long long c1 = clock64();
    uint64_t t1 = gtimer();
    if (threadIdx.x == 0) { t_out[0] = t1 - t0; c_out[0] = c1 - c0; }
}

__global__ void k_clock_rate(uint64_t *t, long long *c, int spin)
{
    uint64_t t0 = gtimer(); long long c0 = clock64();
    volatile int x = 0;
    for (int i = 0; i < spin; i++) x = x + 1;
    uint64_t t1 = gtimer(); long long c1 = clock64();
    t[0] = t1 - t0; c[0] = c1 - c0;
}

__global__ void k_contend(unsigned long long *ctr, int iters, int spread, unsigned long long *sink)
{
    // one lane per warp does `iters` returning atomics on one of `spread` addresses (128 B apart)
    if ((threadIdx.x & 31) != 0) return;
    const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    unsigned long long acc = 0;
    unsigned long long *p = ctr + (size_t)(w % spread) * 16;
    for (int i = 0; i < iters; i++) acc += atomicAdd(p, 64ULL);
    if (acc == 12345) sink[0] = acc;
}

int hotset()
{
    int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    int *d, *sink;
    CK(cudaMalloc(&d, 64 << 20)); CK(cudaMemset(d, 0, 64 << 20)); CK(cudaMalloc(&sink, 64));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int bits : {24, 20, 17, 14, 12}) {
        const uint32_t mask = (1u << bits) - 1;
        for (int mode = 0; mode < 3; mode++) {
            const int grid = sms * 4, block = 256;
            const long long per = 2048;
            for (int rep = 0; rep < 2; rep++) {
                cudaEventRecord(e0);
                if (mode == 0) k_scatter<0><<<grid, block>>>(d, mask, per, sink);
                if (mode == 1) k_scatter<1><<<grid, block>>>(d, mask, per, sink);
                if (mode == 2) k_scatter<2><<<grid, block>>>(d, mask, per, sink);
                cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
            }
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            const double ops = (double)grid * block * per;
            printf("%s over %8u addresses: %.1f Gops/s\n", mode == 0 ? "ld.cg      " : (mode == 1 ? "atomic ret " : "atomic nort"),
                   mask + 1, ops / ms / 1e6);
        }
    }
    return 0;
}

int contention()
{
    int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    unsigned long long *ctr, *sink;
    CK(cudaMalloc(&ctr, 16 * 8 * 4096)); CK(cudaMalloc(&sink, 64));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int spread : {1, 8, 148, 4096}) {
        for (int wpb : {1, 24}) {
            CK(cudaMemset(ctr, 0, 16 * 8 * 4096));
            const int iters = 200;
            for (int rep = 0; rep < 2; rep++) {
                cudaEventRecord(e0);
                k_contend<<<sms, 32 * wpb>>>(ctr, iters, spread, sink);
                cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
            }
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            const double ops = (double)sms * wpb * iters;
            printf("returning atomicAdd, %4d addresses, %5d warps: %.1f Mops/s, %.0f ns per op per warp\n", spread,
                   sms * wpb, ops / ms / 1e3, ms * 1e6 / iters);
        }
    }
    return 0;
}

// dependent-load latency vs footprint (TLB reach): 4000 hops, each to a
// random 128-B line of a buffer of the given size (device-side init)
__global__ void k_tlb_init(int *buf, size_t lines, uint64_t seed)
{
    // buf[line*32] = next line index*32 of a random cycle: use an LCG walk
    // over lines with a multiplier coprime to lines (full period for odd step)
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    if (i >= lines) return;
    const size_t a = 2862933555777941757ull % lines | 1;  // odd, coprime to 2^k
    buf[i * 32] = (int)(((i * a + 12345) % lines));       // line index
}
__global__ void k_tlb_chase(const int *buf, int steps, long long *out, int *sink, size_t start)
{
    size_t p = start;
    long long t0 = clock64();
    for (int i = 0; i < steps; i++) p = (size_t)__ldcg(buf + p * 32);
    long long t1 = clock64();
    out[0] = t1 - t0;
    sink[0] = (int)p;
}
static int tlb()
{
    long long *d_c; int *sink;
    CK(cudaMalloc(&d_c, 64)); CK(cudaMalloc(&sink, 64));
    for (size_t mb : {16, 64, 256, 1024, 2048, 4096, 8192}) {
        size_t bytes = mb << 20, lines = bytes / 128;
        int *d; CK(cudaMalloc(&d, bytes));
        k_tlb_init<<<(unsigned)((lines + 255) / 256), 256>>>(d, lines, 1);
        CK(cudaDeviceSynchronize());
        long long hc = 0;
        for (int rep = 0; rep < 2; rep++) {
            k_tlb_chase<<<1, 1>>>(d, 4000, d_c, sink, (lines / 3) * rep + 7);
            CK(cudaDeviceSynchronize());
        }
        CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
        printf("dependent ld.cg over %5zu MB (random lines): %.0f cycles/hop\n", mb, hc / 4000.0);
        CK(cudaFree(d));
    }
    return 0;
}

int main(int argc, char **argv)
{
    if (argc > 1 && std::string(argv[1]) == "tlb") return tlb();
    if (argc > 1 && std::string(argv[1]) == "contention") return contention();
    if (argc > 1 && std::string(argv[1]) == "hotset") return hotset();
    int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    int l2; CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, 0));
    printf("SMs=%d L2=%d MB\n", sms, l2 >> 20);
    long long *d_c; uint64_t *d_t; int *sink;
    CK(cudaMalloc(&d_c, 64)); CK(cudaMalloc(&d_t, 64)); CK(cudaMalloc(&sink, 64));
    long long hc; uint64_t ht;

    // clock rate while busy
    k_clock_rate<<<1, 1>>>(d_t, d_c, 20000000); CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(&ht, d_t, 8, cudaMemcpyDeviceToHost)); CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
    double ghz = (double)hc / (double)ht;
    printf("single-thread SM clock while spinning: %.3f GHz\n", ghz);

    // latency: pointer chase on L2-resident (16 MB) and HBM (2 GB) arrays
    for (size_t bytes : {(size_t)16 << 20, (size_t)2 << 30}) {
        size_t n = bytes / 4;
        std::vector<int> h(n);
        // random cyclic permutation with 128B stride granularity
        size_t lines = n / 32;
        std::vector<int> perm(lines);
        for (size_t i = 0; i < lines; i++) perm[i] = (int)i;
        uint64_t s = 88172645463325252ull;
        for (size_t i = lines - 1; i > 0; i--) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; size_t j = s % (i + 1); std::swap(perm[i], perm[j]); }
        for (size_t i = 0; i < lines; i++) h[(size_t)perm[i] * 32] = perm[(i + 1) % lines] * 32;
        int *d; CK(cudaMalloc(&d, bytes)); CK(cudaMemcpy(d, h.data(), bytes, cudaMemcpyHostToDevice));
        k_chase<<<1, 1>>>(d, 20000, perm[0] * 32, d_c, sink); CK(cudaDeviceSynchronize());
        k_chase<<<1, 1>>>(d, 20000, perm[0] * 32, d_c, sink); CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
        printf("dependent load latency over %zu MB: %.0f cycles (%.0f ns)\n", bytes >> 20, hc / 20000.0, hc / 20000.0 / ghz);
        CK(cudaFree(d));
    }
    {
        int *d; CK(cudaMalloc(&d, 1 << 20)); CK(cudaMemset(d, 0, 1 << 20));
        k_atomic_chase<<<1, 1>>>(d, 10000, d_c); CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
        printf("dependent atomicAdd latency: %.0f cycles (%.0f ns)\n", hc / 10000.0, hc / 10000.0 / ghz);
        int *buf; CK(cudaMalloc(&buf, 4096));
        k_fence_cost<<<1, 32>>>(d_c, 10000, buf); CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
        printf("store + __threadfence: %lld cycles\n", hc);
        CK(cudaFree(d));
    }
    // throughput: scattered ops on 64 MB array (L2-resident) and 1 GB (HBM)
    for (size_t bytes : {(size_t)64 << 20, (size_t)1 << 30}) {
        int *d; CK(cudaMalloc(&d, bytes)); CK(cudaMemset(d, 0, bytes));
        uint32_t mask = (uint32_t)(bytes / 4 - 1);
        cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
        const char *names[] = {"ld.cg scattered", "atomicSub(ret) scattered", "atomicSub(noret) scattered", "ld.nc scattered"};
        for (int mode = 0; mode < 4; mode++) {
            for (int bps : {4, 8}) {
                int grid = sms * bps, block = 256;
                long long per = 4096;
                for (int rep = 0; rep < 2; rep++) {
                    cudaEventRecord(e0);
                    if (mode == 0) k_scatter<0><<<grid, block>>>(d, mask, per, sink);
                    if (mode == 1) k_scatter<1><<<grid, block>>>(d, mask, per, sink);
                    if (mode == 2) k_scatter<2><<<grid, block>>>(d, mask, per, sink);
                    if (mode == 3) k_scatter<3><<<grid, block>>>(d, mask, per, sink);
                    cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
                }
                float ms; cudaEventElapsedTime(&ms, e0, e1);
                double ops = (double)grid * block * per;
                printf("%-28s %5zu MB  grid=%d: %.1f Gops/s (%.2f ops/clk/SM at %.2f GHz)\n", names[mode], bytes >> 20, grid,
                       ops / ms / 1e6, ops / (ms * 1e-3) / (ghz * 1e9) / sms, ghz);
            }
        }
        CK(cudaFree(d));
    }
    // streaming read bandwidth
    {
        size_t bytes = (size_t)4 << 30;
        int4 *d; CK(cudaMalloc(&d, bytes)); CK(cudaMemset(d, 1, bytes));
        cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
        for (int rep = 0; rep < 3; rep++) {
            cudaEventRecord(e0);
            k_stream<<<sms * 8, 512>>>(d, bytes / 16, sink);
            cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
        }
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        printf("streaming int4 read: %.0f GB/s\n", bytes / ms / 1e6);
        CK(cudaFree(d));
    }
    // grid barrier cost
    {
        Bar *b; CK(cudaMalloc(&b, sizeof(Bar)));
        for (int bps : {1, 2, 4}) {
            for (int nof = 0; nof < 2; nof++) {
                CK(cudaMemset(b, 0, sizeof(Bar)));
                int grid = sms * bps, iters = 2000;
                void *args[] = {&b, &iters, &d_t};
                CK(cudaLaunchCooperativeKernel(nof ? (void *)k_barriers_nofence : (void *)k_barriers, grid, 256, args, 0, 0));
                CK(cudaDeviceSynchronize());
                CK(cudaMemcpy(&ht, d_t, 8, cudaMemcpyDeviceToHost));
                printf("grid barrier (%s) grid=%d: %.2f us\n", nof ? "no fences" : "with fences", grid, ht / 1e3 / iters);
            }
        }
        k_syncthreads<<<1, 512>>>(10000, d_t, d_c); CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(&ht, d_t, 8, cudaMemcpyDeviceToHost)); CK(cudaMemcpy(&hc, d_c, 8, cudaMemcpyDeviceToHost));
        printf("__syncthreads (512 thr): %.1f ns, %.1f cycles\n", ht / 1e4, hc / 1e4);
    }
    return 0;
}
