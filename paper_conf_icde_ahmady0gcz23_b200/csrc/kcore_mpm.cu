// kcore_mpm.cu -- MPM h-index iteration on sm_100a.
//
// The paper's second algorithm family (Fig. 2; its GPU form
// is Medusa-MPM): every vertex starts from a(v) = deg(v) and
// repeatedly replaces a(v) by the h-index of its neighbours' estimates,
// max{h : |{u in N(v) : a(u) >= h}| >= h}, until nothing changes; then
// a(v) = core(v).  We run the bulk-synchronous (Jacobi) form of P:L388 --
// iteration t reads only the iterate t-1 -- so every iterate, not only the
// fixpoint, is defined independently of scheduling and is compared bit-exactly
// with the oracle (oracle_mpm).
//
// One persistent cooperative kernel per call (no host round trip per
// iteration), with exact SUPPORT COUNTERS: cnt(v) = |{u in N(v) : a(u) >= a(v)}|.
// v keeps its estimate at the next iteration iff cnt(v) >= a(v), so the next
// active set is exactly the set of vertices that WILL change -- hubs are no
// longer re-read whenever a neighbour moves.  Per iteration t:
//   A1  warps take the active vertices with <= 128 arcs: the neighbours'
//       capped estimates a_{t-1} stay in registers; a ballot-count binary
//       search gives h = max{h : N(h) >= h} and N(h); bigger vertices are
//       deferred to a list.
//   A2  CTAs take the big vertices: one counting pass decides "unchanged"
//       (t = 1 only; later every active vertex changes), else a 1024-bin
//       histogram over [lo, hi] (per-warp sub-histograms in shared memory) and
//       a warp suffix search shrink the range 1024x per pass.
//       Every computed vertex stores cnt(v) = N_{t-1}(h); a changed one also
//       stores a_new(v) = h and the stamp cstamp(v) = t.
//   B   every changed x tells each neighbour u whose support it withdraws:
//       if a_{t-1}(x) >= a_t(u) > a_t(x) then cnt(u) -= 1; the decrement that
//       takes cnt(u) from a_t(u) to a_t(u)-1 activates u for t+1 (exactly
//       once).  After B, cnt(u) = |{x : a_t(x) >= a_t(u)}| for every u.
//   C   commit a_t(x) for the changed vertices.
// Estimates never increase (a_{t+1} <= a_t, induction on the monotone
// h-index), so h is searched in [0, min(a_t(v), deg(v))] only.
#include "kcore.h"

#include <algorithm>
#include <cooperative_groups.h>
#include <cstdint>
#include <cuda_runtime.h>

namespace cg = cooperative_groups;

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kB = 512;                 // threads per CTA
constexpr int kW = kB / 32;
constexpr int kSmall = 128;             // arcs held in registers by one warp (4 per lane)
constexpr int kBins = 1024;

struct MState {
    unsigned long long act_len[2];      // active list lengths, by iteration parity
    unsigned long long chg_len[2];      // changed vertices with <= kSmall arcs
    unsigned long long big_len[2];      // big active vertices
    unsigned long long cbig_len[2];     // changed vertices with > kSmall arcs
    unsigned long long iters;           // iterations that changed something
    unsigned long long processed;       // sum of active-set sizes (statistics)
    unsigned long long arcs;            // arcs gathered (statistics)
};

struct MArgs {
    const int64_t *rowptr;
    const int32_t *colidx;
    int32_t *a;        // current iterate (= a_out)
    int32_t *a_new;    // next values of the changed vertices
    int32_t *cnt;      // support counters
    int32_t *cstamp;   // iteration at which a vertex last changed
    int32_t *act[2];   // active lists
    int32_t *chg;      // changed vertices of this iteration (small)
    int32_t *cbig;     // changed vertices of this iteration (big)
    int32_t *big;      // big active vertices of this iteration
    MState *S;
    int64_t n;
    int64_t max_iters;  // < 0: until convergence
};

struct MSmem {
    int32_t hist[kW][kBins];
    int32_t tot[kBins];
    int64_t wsum[kW + 1];
    int32_t bcast[4];
};

__device__ __forceinline__ unsigned lanemask_lt()
{
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// warp-aggregated append of `v` where `p` to list[*len]
__device__ __forceinline__ void warp_append(bool p, int32_t v, int32_t *list, unsigned long long *len)
{
    const unsigned b = __ballot_sync(kFull, p);
    if (!b) return;
    const int lane = threadIdx.x & 31, lead = __ffs(b) - 1;
    unsigned long long base = 0;
    if (lane == lead) base = atomicAdd(len, (unsigned long long)__popc(b));
    base = __shfl_sync(kFull, base, lead);
    if (p) list[base + __popc(b & lanemask_lt())] = v;
}

// B: x changed at iteration t from ax = a_{t-1}(x) to hx = a_t(x); withdraw
// its support from the neighbours u with ax >= a_t(u) > hx (warp, arcs
// [b0+lane0, e) step `step`).  The decrement that takes cnt(u) from a_t(u) to
// a_t(u)-1 activates u for iteration t+1.
__device__ __forceinline__ void notify(const MArgs &A, int64_t b0, int64_t e, int64_t step, int t, int32_t ax,
                                       int32_t hx)
{
    const int t1 = t + 1;
    for (int64_t x0 = b0; x0 < e; x0 += step) {
        const int64_t x = x0 + (threadIdx.x & 31);
        bool p = false;
        int32_t u = 0;
        if (x < e) {
            u = __ldg(A.colidx + x);
            const int32_t au = __ldcg(A.cstamp + u) == t ? __ldcg(A.a_new + u) : __ldcg(A.a + u);
            if (ax >= au && au > hx) p = atomicSub(A.cnt + u, 1) == au;
        }
        warp_append(p, u, A.act[t1 & 1], &A.S->act_len[t1 & 1]);
    }
}

// A1: one warp, vertex v with d <= kSmall arcs
__device__ __forceinline__ void small_vertex(const MArgs &A, int32_t v, int64_t b, int64_t d, int t)
{
    const int lane = threadIdx.x & 31;
    const int32_t c = __ldcg(A.a + v);  // committed by another SM last iteration: L2, not L1
    int32_t x[kSmall / 32];
#pragma unroll
    for (int r = 0; r < kSmall / 32; r++) {
        const int64_t i = r * 32 + lane;
        x[r] = i < d ? min(__ldcg(A.a + __ldg(A.colidx + b + i)), c) : -1;
    }
    int lo = 0, hi = (int)min((int64_t)c, d), nlo = (int)d;  // nlo = N(lo)
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        int cnt = 0;
#pragma unroll
        for (int r = 0; r < kSmall / 32; r++) cnt += __popc(__ballot_sync(kFull, x[r] >= mid));
        if (cnt >= mid) { lo = mid; nlo = cnt; } else hi = mid - 1;
    }
    const bool ch = lo != c;
    if (lane == 0) {
        A.cnt[v] = nlo;
        if (ch) { A.a_new[v] = lo; A.cstamp[v] = t; }
    }
    warp_append(ch && lane == 0, v, A.chg, &A.S->chg_len[t & 1]);
}

// h = max{h <= min(c, d) : N(h) >= h} over the capped estimates x[] (R
// registers per lane) by a ballot-count binary search; also N(h).
template <int R>
__device__ __forceinline__ void hsearch(const int32_t (&x)[R], int32_t c, int64_t d, int &lo, int &nlo)
{
    int hi = (int)min((int64_t)c, d);
    lo = 0;
    nlo = (int)d;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        int cnt = 0;
#pragma unroll
        for (int r = 0; r < R; r++) cnt += __popc(__ballot_sync(kFull, x[r] >= mid));
        if (cnt >= mid) { lo = mid; nlo = cnt; } else hi = mid - 1;
    }
}

// A1 for two vertices of <= 64 arcs at once: both gathers in flight together
// (the small path is bound by the latency of the estimate gathers).
__device__ __forceinline__ void small_pair(const MArgs &A, int32_t v0, int64_t b0, int64_t d0, int32_t v1,
                                           int64_t b1, int64_t d1, int t)
{
    const int lane = threadIdx.x & 31;
    const int32_t c0 = __ldcg(A.a + v0), c1 = __ldcg(A.a + v1);
    int32_t x0[2], x1[2];
#pragma unroll
    for (int r = 0; r < 2; r++) {
        const int64_t i = r * 32 + lane;
        x0[r] = i < d0 ? __ldcg(A.a + __ldg(A.colidx + b0 + i)) : -1;
        x1[r] = i < d1 ? __ldcg(A.a + __ldg(A.colidx + b1 + i)) : -1;
    }
#pragma unroll
    for (int r = 0; r < 2; r++) { x0[r] = min(x0[r], c0); x1[r] = min(x1[r], c1); }
    int h0, n0, h1, n1;
    hsearch(x0, c0, d0, h0, n0);
    hsearch(x1, c1, d1, h1, n1);
    const bool ch0 = h0 != c0, ch1 = h1 != c1;
    if (lane == 0) {
        A.cnt[v0] = n0;
        if (ch0) { A.a_new[v0] = h0; A.cstamp[v0] = t; }
        A.cnt[v1] = n1;
        if (ch1) { A.a_new[v1] = h1; A.cstamp[v1] = t; }
    }
    warp_append(ch0 && lane == 0, v0, A.chg, &A.S->chg_len[t & 1]);
    warp_append(ch1 && lane == 0, v1, A.chg, &A.S->chg_len[t & 1]);
}

// A2: the whole CTA, vertex v with d > kSmall arcs
__device__ void big_vertex(const MArgs &A, MSmem &sm, int32_t v, int t)  // t: iteration
{
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t b = __ldg(A.rowptr + v), e = __ldg(A.rowptr + v + 1), d = e - b;
    const int32_t c = __ldcg(A.a + v);
    int64_t lo = 0, hi = min((int64_t)c, d);  // h in [lo, hi]; |{x >= lo}| >= lo holds
    int32_t nlo = (int32_t)d;                  // N(lo)
    if (t > 1) {
        hi = hi - 1;  // an active vertex always drops (its support fell below a(v))
    } else {
        // most active big vertices keep their estimate: one counting pass
        // decides N(hi) >= hi without building a histogram
        int64_t cnt = 0;
        for (int64_t x0 = b + threadIdx.x; x0 < e; x0 += kB) cnt += __ldcg(A.a + __ldg(A.colidx + x0)) >= hi;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
        if (lane == 0) sm.wsum[w] = cnt;
        __syncthreads();
        if (threadIdx.x == 0) {
            int64_t s = 0;
            for (int q = 0; q < kW; q++) s += sm.wsum[q];
            sm.bcast[0] = s >= hi ? 1 : 0;
            sm.bcast[1] = (int32_t)s;
        }
        __syncthreads();
        if (sm.bcast[0]) { lo = hi; nlo = sm.bcast[1]; }
        else hi = hi - 1;
        __syncthreads();
    }
    while (lo < hi) {
        const int64_t span = hi - lo + 1;
        const int64_t wd = (span + kBins - 1) / kBins;  // bin width
        for (int i = threadIdx.x; i < kW * kBins; i += kB) (&sm.hist[0][0])[i] = 0;
        __syncthreads();
        int64_t above = 0;  // x > hi
        for (int64_t x0 = b + threadIdx.x; x0 < e; x0 += kB) {
            const int64_t xv = min((int64_t)__ldcg(A.a + __ldg(A.colidx + x0)), (int64_t)c);
            if (xv > hi) above++;
            else if (xv >= lo) atomicAdd(&sm.hist[w][(int)((xv - lo) / wd)], 1);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) above += __shfl_xor_sync(kFull, above, o);
        if (lane == 0) sm.wsum[w] = above;
        __syncthreads();
        for (int i = threadIdx.x; i < kBins; i += kB) {
            int32_t s = 0;
#pragma unroll
            for (int q = 0; q < kW; q++) s += sm.hist[q][i];
            sm.tot[i] = s;
        }
        if (threadIdx.x == 0) {
            int64_t ab = 0;
            for (int q = 0; q < kW; q++) ab += sm.wsum[q];
            sm.wsum[kW] = ab;
        }
        __syncthreads();
        // N(lo + j*wd) = above + sum_{j' >= j} tot[j'] ; find the largest j with N >= lo + j*wd
        // (monotone predicate; j = 0 always holds).  Suffix sums by one warp, 32 bins per lane.
        if (w == 0) {
            const int per = kBins / 32;
            int64_t part = 0;
            for (int q = 0; q < per; q++) part += sm.tot[lane * per + q];
            // exclusive suffix over lanes: sum of parts of lanes > lane
            int64_t inc = part;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int64_t tt = __shfl_down_sync(kFull, inc, o);
                if (lane + o < 32) inc += tt;
            }
            int64_t suf = sm.wsum[kW] + inc - part;  // N at the end of this lane's chunk
            int best = -1;
            for (int q = per - 1; q >= 0; q--) {
                const int j = lane * per + q;
                suf += sm.tot[j];
                const int64_t hj = lo + (int64_t)j * wd;
                if (hj <= hi && suf >= hj && best < 0) best = j;  // largest j in this chunk
            }
            // the overall largest j: the highest lane with a hit holds it
            const unsigned bl = __ballot_sync(kFull, best >= 0);
            const int src = 31 - __clz(bl);
            const int jb = __shfl_sync(kFull, best, src);
            // N at the chosen bin start: recompute the suffix there
            int64_t nb = 0;
            if (lane == src) {
                int64_t sf = sm.wsum[kW] + inc - part;
                for (int q = per - 1; q >= 0; q--) {
                    sf += sm.tot[lane * per + q];
                    if (lane * per + q == jb) { nb = sf; break; }
                }
            }
            nb = __shfl_sync(kFull, nb, src);
            if (lane == 0) { sm.bcast[0] = jb; sm.bcast[1] = (int32_t)nb; }
        }
        __syncthreads();
        const int jb = sm.bcast[0];
        nlo = sm.bcast[1];
        const int64_t nlo = lo + (int64_t)jb * wd;
        hi = min(hi, nlo + wd - 1);
        lo = nlo;
        __syncthreads();
    }
    const int32_t h = (int32_t)lo;
    if (threadIdx.x == 0) {
        A.cnt[v] = nlo;
        if (h != c) {
            A.a_new[v] = h;
            A.cstamp[v] = t;
            A.cbig[atomicAdd(&A.S->cbig_len[t & 1], 1ULL)] = v;
        }
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kB, 1) k_mpm(const __grid_constant__ MArgs A)
{
    extern __shared__ __align__(16) unsigned char smraw[];
    MSmem &sm = *reinterpret_cast<MSmem *>(smraw);
    cg::grid_group grid = cg::this_grid();
    MState *S = A.S;
    const int lane = threadIdx.x & 31;
    const int64_t gw = (int64_t)blockIdx.x * kW + (threadIdx.x >> 5);
    const int64_t nw = (int64_t)gridDim.x * kW;
    unsigned long long processed = 0, arcs = 0;
    for (int t = 1;; t++) {
        if (A.max_iters >= 0 && t > A.max_iters) break;
        // (counters of parity t were reset in phase C of iteration t-1 / by k_mpm_init)
        const int64_t len = (t == 1) ? A.n : (int64_t)__ldcg(&S->act_len[t & 1]);
        const int32_t *act = A.act[t & 1];
        // A1: small vertices by warps, big ones deferred
        for (int64_t i = gw; i < len; i += 2 * nw) {  // entries i and i + nw
            const int64_t j = i + nw;
            const int32_t v0 = (t == 1) ? (int32_t)i : __ldcg(act + i);
            const int32_t v1 = j < len ? ((t == 1) ? (int32_t)j : __ldcg(act + j)) : -1;
            const int64_t b0 = __ldg(A.rowptr + v0), d0 = __ldg(A.rowptr + v0 + 1) - b0;
            int64_t b1 = 0, d1 = 0;
            if (v1 >= 0) { b1 = __ldg(A.rowptr + v1); d1 = __ldg(A.rowptr + v1 + 1) - b1; }
            if (lane == 0) {
                if (d0 > kSmall) A.big[atomicAdd(&S->big_len[t & 1], 1ULL)] = v0;
                if (d1 > kSmall) A.big[atomicAdd(&S->big_len[t & 1], 1ULL)] = v1;
            }
            const bool s0 = d0 > 0 && d0 <= kSmall, s1 = v1 >= 0 && d1 > 0 && d1 <= kSmall;
            if (s0 && s1 && d0 <= 64 && d1 <= 64) {
                small_pair(A, v0, b0, d0, v1, b1, d1, t);
            } else {
                if (s0) small_vertex(A, v0, b0, d0, t);
                if (s1) small_vertex(A, v1, b1, d1, t);
            }
            if (lane == 0) { processed += 1 + (v1 >= 0); arcs += d0 + d1; }
        }
        grid.sync();
        // A2: big vertices by whole CTAs
        const int64_t nbig = (int64_t)__ldcg(&S->big_len[t & 1]);
        for (int64_t i = blockIdx.x; i < nbig; i += gridDim.x) big_vertex(A, sm, __ldcg(A.big + i), t);
        grid.sync();
        const int64_t nchg = (int64_t)__ldcg(&S->chg_len[t & 1]);
        const int64_t ncbig = (int64_t)__ldcg(&S->cbig_len[t & 1]);
        if (nchg + ncbig == 0) break;
        // B: changed vertices withdraw their support (small ones by warps, big ones by CTAs)
        for (int64_t i = gw; i < nchg; i += nw) {
            const int32_t x = __ldcg(A.chg + i);
            const int64_t b = __ldg(A.rowptr + x), e = __ldg(A.rowptr + x + 1);
            notify(A, b, e, 32, t, __ldcg(A.a + x), __ldcg(A.a_new + x));
            if (lane == 0) arcs += e - b;
        }
        for (int64_t i = blockIdx.x; i < ncbig; i += gridDim.x) {
            const int32_t x = __ldcg(A.cbig + i);
            const int64_t b = __ldg(A.rowptr + x), e = __ldg(A.rowptr + x + 1);
            notify(A, b + (int64_t)(threadIdx.x >> 5) * 32, e, (int64_t)kB, t, __ldcg(A.a + x), __ldcg(A.a_new + x));
            if (threadIdx.x == 0) arcs += e - b;
        }
        grid.sync();
        // C: commit (Jacobi: every read of iterate t-1 happened before the syncs);
        // reset the counters iteration t+1 will fill (their last readers are done)
        for (int64_t i = (int64_t)blockIdx.x * kB + threadIdx.x; i < nchg + ncbig; i += (int64_t)gridDim.x * kB) {
            const int32_t x = i < nchg ? __ldcg(A.chg + i) : __ldcg(A.cbig + (i - nchg));
            A.a[x] = __ldcg(A.a_new + x);
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            S->iters = (unsigned long long)t;
            S->act_len[t & 1] = 0;  // input of iteration t: read at its start
            S->chg_len[(t + 1) & 1] = 0;
            S->big_len[(t + 1) & 1] = 0;
            S->cbig_len[(t + 1) & 1] = 0;
        }
        grid.sync();
    }
    if (lane == 0 && processed) {
        atomicAdd(&S->processed, processed);
        atomicAdd(&S->arcs, arcs);
    }
}

__global__ void k_mpm_init(const int64_t *rowptr, int64_t n, int32_t *a, int32_t *cstamp, MState *S)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        a[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
        cstamp[v] = 0;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        S->act_len[0] = S->act_len[1] = 0;
        S->chg_len[0] = S->chg_len[1] = 0;
        S->big_len[0] = S->big_len[1] = 0;
        S->cbig_len[0] = S->cbig_len[1] = 0;
        S->iters = S->processed = S->arcs = 0;
    }
}

size_t al(size_t x) { return (x + 255) & ~(size_t)255; }

} // namespace

extern "C" int kcore_mpm(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m, int32_t *a_out,
                         int64_t max_iters, int64_t *iters_out, void *stream, kcore_stats *stats)
{
    if (n < 0 || n >= ((int64_t)1 << 31) || m < 0 || (n > 0 && (!rowptr || !a_out)) || (m > 0 && !colidx))
        return KCORE_EINVAL;
    if (stats) *stats = kcore_stats{};
    if (iters_out) *iters_out = 0;
    if (n == 0) return KCORE_OK;
    cudaStream_t st = (cudaStream_t)stream;
    int dev = 0, sms = 0, major = 0, occ = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return KCORE_ECUDA;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    if (major != 10) return KCORE_EUNSUPPORTED;
    const size_t smem = sizeof(MSmem);
    if (cudaFuncSetAttribute(k_mpm, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
        return KCORE_ECUDA;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mpm, kB, smem) != cudaSuccess || occ < 1)
        return KCORE_EUNSUPPORTED;
    const int grid = sms * occ;
    const size_t nn = (size_t)n;
    const size_t bytes = al(sizeof(MState)) + 8 * al(sizeof(int32_t) * nn);
    char *ws = nullptr;
    int rc = KCORE_OK;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    MState hS{};
    cudaError_t e = cudaMallocAsync((void **)&ws, bytes, st);
    if (e != cudaSuccess) return e == cudaErrorMemoryAllocation ? KCORE_ENOMEM : KCORE_ECUDA;
    MArgs A;
    {
        char *p = ws;
        A.S = (MState *)p; p += al(sizeof(MState));
        A.a_new = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.cnt = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.cstamp = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.act[0] = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.act[1] = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.chg = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.cbig = (int32_t *)p; p += al(sizeof(int32_t) * nn);
        A.big = (int32_t *)p;
    }
    A.rowptr = rowptr;
    A.colidx = colidx;
    A.a = a_out;
    A.n = n;
    A.max_iters = max_iters;
    void *args[] = {&A};
    if (stats) {
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0, st);
    }
    k_mpm_init<<<std::min<int64_t>((n + 255) / 256, (int64_t)sms * 8), 256, 0, st>>>(rowptr, n, a_out, A.cstamp, A.S);
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaLaunchCooperativeKernel((const void *)k_mpm, dim3(grid), dim3(kB), args, smem, st);
    if (e == cudaSuccess && stats) e = cudaEventRecord(e1, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&hS, A.S, sizeof(MState), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
        rc = e == cudaErrorMemoryAllocation ? KCORE_ENOMEM : KCORE_ECUDA;
    } else {
        if (iters_out) *iters_out = (int64_t)hS.iters;
        if (stats) {
            float ms = 0.f;
            cudaEventElapsedTime(&ms, e0, e1);
            stats->levels = (int64_t)hS.iters;
            stats->phases = (int64_t)hS.iters;
            stats->barriers = 4 * (int64_t)hS.iters + 2;
            stats->scanned = (int64_t)hS.processed;
            stats->arcs_walked = (int64_t)hS.arcs;
            stats->grid_blocks = grid;
            stats->block_threads = kB;
            stats->kernel_ms = ms;
            stats->launches = 2;  // k_mpm_init, k_mpm
        }
    }
    cudaFreeAsync(ws, st);
    cudaStreamSynchronize(st);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    return rc;
}
