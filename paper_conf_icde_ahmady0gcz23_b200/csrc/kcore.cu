// kcore.cu -- C ABI of the single-GPU hot path (include/kcore.h).
//
// kcore_decompose_ex: validate arguments, carve the workspace, initialise the
// device State, then launch ONE persistent cooperative kernel (k_persistent)
// that runs deg init, every level scan, every peel sub-round and the level
// control on the device (see kc_kernels.cuh).  The ablation KCORE_ALGO_HOSTLOOP
// drives the same phase code from the host like the paper's Alg. 1
// (P:L187-208): one launch per phase and a device->host read-back after each.
#include "kcore.h"
#include "kc_kernels.cuh"

#include <cstdio>
#include <cstring>
#include <algorithm>
#include <mutex>

using namespace kc;

// L2 property of the window's lines beyond hitRatio (the set-aside is smaller
// than the window on some parts)
#ifndef KC_MISS_PROP
#define KC_MISS_PROP cudaAccessPropertyNormal
#endif


namespace {

constexpr int kMaxDev = 64;

struct DevInfo {
    int sms = 0;
    int occ = 0;  // resident CTAs of k_persistent per SM
    int major = 0, minor = 0;
    int persist_max = 0, window_max = 0;  // cudaDevAttrMaxPersistingL2CacheSize / AccessPolicyMaxWindowSize
    bool init = false;
};

DevInfo g_dev[kMaxDev];
std::mutex g_mu;

int dev_info(DevInfo &out)
{
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return KCORE_ECUDA;
    if (dev < 0 || dev >= kMaxDev) return KCORE_ECUDA;
    std::lock_guard<std::mutex> lk(g_mu);
    DevInfo &d = g_dev[dev];
    if (!d.init) {
        if (cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
            return KCORE_ECUDA;
        cudaDeviceGetAttribute(&d.major, cudaDevAttrComputeCapabilityMajor, dev);
        cudaDeviceGetAttribute(&d.minor, cudaDevAttrComputeCapabilityMinor, dev);
        if (d.major != 10) return KCORE_EUNSUPPORTED;
        cudaDeviceGetAttribute(&d.persist_max, cudaDevAttrMaxPersistingL2CacheSize, dev);
        cudaDeviceGetAttribute(&d.window_max, cudaDevAttrMaxAccessPolicyWindowSize, dev);
        const int smem = (int)sizeof(Smem);
        if (cudaFuncSetAttribute(k_persistent, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess ||
            cudaFuncSetAttribute(k_phase, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess)
            return KCORE_ECUDA;
        int occ = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_persistent, kBlock, smem) != cudaSuccess)
            return KCORE_ECUDA;
        d.occ = occ;
        d.init = true;
    }
    out = d;
    return KCORE_OK;
}

size_t al(size_t x) { return (x + 255) & ~(size_t)255; }

struct Carve {
    State *S;
    int32_t *order;
    uint32_t *claimed;
    int32_t *gq_v;
    int64_t *gq_beg, *gq_arc;
    int32_t *alive0, *alive1;
    int32_t *near0, *near1;
    int32_t *seg0, *seg1;
    int32_t *deg;
};

constexpr int kMaxSeg = 16384;  // one alive-list segment per warp of the persistent grid

size_t carve(void *base, int64_t n, Carve *c)
{
    size_t off = 0;
    auto take = [&](size_t bytes) {
        char *p = base ? (char *)base + off : nullptr;
        off += al(bytes);
        return p;
    };
    Carve t;
    const size_t nn = (size_t)(n > 0 ? n : 1);
    t.S = (State *)take(sizeof(State));
    t.order = (int32_t *)take(sizeof(int32_t) * nn);
    t.gq_v = (int32_t *)take(sizeof(int32_t) * nn);
    t.gq_beg = (int64_t *)take(sizeof(int64_t) * nn);
    t.gq_arc = (int64_t *)take(sizeof(int64_t) * (nn + 1));
    // segments of ceil(n/grid) + 32 entries (the identity scan's slices are 32-aligned)
    t.alive0 = (int32_t *)take(sizeof(int32_t) * (nn + 33 * (size_t)kMaxSeg));
    t.alive1 = (int32_t *)take(sizeof(int32_t) * (nn + 33 * (size_t)kMaxSeg));
    // near lists: 2n entries -- a vertex appears at most twice per epoch (the
    // build's scan may collect it after a walk already appended its theta+1 ->
    // theta crossing; near scans copy both entries, their claims dedup)
    t.near0 = (int32_t *)take(sizeof(int32_t) * 2 * nn);
    t.near1 = (int32_t *)take(sizeof(int32_t) * 2 * nn);
    t.seg0 = (int32_t *)take(sizeof(int32_t) * kMaxSeg);
    t.seg1 = (int32_t *)take(sizeof(int32_t) * kMaxSeg);
    // claim bits and working degrees adjacent: one L2 access-policy window
    t.claimed = (uint32_t *)take(sizeof(uint32_t) * ((nn + 31) / 32));
    t.deg = (int32_t *)take(sizeof(int32_t) * nn);
    if (c) *c = t;
    return off;
}

int check_args(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
               const int32_t *core_out)
{
    if (n < 0 || n >= ((int64_t)1 << 31)) return KCORE_EINVAL;
    if (m < 0 || m >= ((int64_t)1 << kArcBits)) return KCORE_EINVAL;
    if (n > 0 && (!rowptr || !core_out)) return KCORE_EINVAL;
    if (m > 0 && !colidx) return KCORE_EINVAL;
    if (n == 0 && m != 0) return KCORE_EINVAL;
    return KCORE_OK;
}

// Single-CTA ("solo") phases are opt-in: measured on B200 they lose to grid
// phases + a barrier on every config (C1 6.2 -> 2.5 ms, C3 58.7 -> 34.5 ms).
int default_solo_arcs() { return 0; }
int default_solo_scan() { return 0; }

} // namespace

#define KC_CUDA(x)                                                                                 \
    do {                                                                                           \
        cudaError_t e_ = (x);                                                                      \
        if (e_ != cudaSuccess) {                                                                   \
            rc = (e_ == cudaErrorMemoryAllocation) ? KCORE_ENOMEM : KCORE_ECUDA;                   \
            goto done;                                                                             \
        }                                                                                          \
    } while (0)

extern "C" size_t kcore_workspace_size(int64_t n, int64_t m)
{
    (void)m;
    if (n < 0) return 0;
    return carve(nullptr, n, nullptr);
}

extern "C" const char *kcore_strerror(int status)
{
    switch (status) {
    case KCORE_OK: return "KCORE_OK";
    case KCORE_EINVAL: return "KCORE_EINVAL: invalid argument";
    case KCORE_ENOMEM: return "KCORE_ENOMEM: allocation failed";
    case KCORE_ECUDA: return "KCORE_ECUDA: CUDA error";
    case KCORE_ENCCL: return "KCORE_ENCCL: NCCL error";
    case KCORE_EGRAPH: return "KCORE_EGRAPH: CSR violates the preconditions";
    case KCORE_EUNSUPPORTED: return "KCORE_EUNSUPPORTED: device is not sm_100";
    default: return "KCORE: unknown status";
    }
}

#ifdef KC_PROBE
extern "C" int64_t kcore_probe_read(int64_t *host, int64_t cap)
{
    // per-CTA regions; unused records have tag 0 (cleared after each read)
    const size_t bytes = (size_t)(1 << 22) * 4 * sizeof(int64_t);
    if (cap < (int64_t)(1 << 22)) return -1;
    cudaMemcpyFromSymbol(host, kc::g_probe, bytes);
    void *dp = nullptr;
    cudaGetSymbolAddress(&dp, kc::g_probe);
    cudaMemset(dp, 0, bytes);
    return (int64_t)(1 << 22);
}
#endif

extern "C" const char *kcore_version(void) { return "kcore-b200 0.1 (sm_100a persistent peel)"; }

extern "C" int kcore_decompose_ex(const int64_t *rowptr, const int32_t *colidx, int64_t n,
                                  int64_t m, int32_t *core_out, void *stream_,
                                  const kcore_options *opt, kcore_stats *stats)
{
    int rc = check_args(rowptr, colidx, n, m, core_out);
    if (rc) return rc;
    if (stats) memset(stats, 0, sizeof(*stats));
    if (n == 0) return KCORE_OK;
    cudaStream_t st = (cudaStream_t)stream_;
    DevInfo di;
    rc = dev_info(di);
    if (rc) return rc;

    const int algo = opt ? opt->algo : KCORE_ALGO_PERSISTENT;
    if (algo != KCORE_ALGO_PERSISTENT && algo != KCORE_ALGO_HOSTLOOP) return KCORE_EINVAL;
    int bps = (opt && opt->blocks_per_sm > 0) ? opt->blocks_per_sm : di.occ;
    if (bps > di.occ) bps = di.occ;
    if (bps < 1) return KCORE_EUNSUPPORTED;
    const int grid = di.sms * bps;
    if (grid > kMaxSeg) return KCORE_EUNSUPPORTED;
    int solo = default_solo_arcs(), solo_scan = default_solo_scan();
    if (opt && opt->solo_arcs > 0) solo = opt->solo_arcs;
    if (opt && opt->solo_arcs < 0) solo = 0;
    if (opt && opt->solo_scan > 0) solo_scan = opt->solo_scan;
    if (opt && opt->solo_scan < 0) solo_scan = 0;
    if (algo == KCORE_ALGO_HOSTLOOP) solo = solo_scan = 0;
    int64_t *trace = opt ? opt->trace_out : nullptr;
    const int64_t trace_cap = (opt && opt->trace_out) ? opt->trace_cap : 0;
    const int bloom = (opt && (opt->flags & KCORE_FLAG_NO_BLOOM)) ? 0 : 1;
    const int red = ((opt && (opt->flags & KCORE_FLAG_NO_RED)) ? 0 : 1) |
                    ((opt && (opt->flags & KCORE_FLAG_NO_NEAR)) ? 0 : 2);
    const size_t smem = sizeof(Smem);

    const size_t need = carve(nullptr, n, nullptr);
    void *ws = nullptr;
    bool own_ws = false;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    int32_t *d_phase = nullptr;
    int64_t l2_lines = 0;
    int64_t hl_launches = 0;
    const char *l2_base = nullptr;
    State hS;
    size_t prev_limit = 0;
    bool limit_raised = false;
    Carve cv;
    KArgs A;
    if (opt && opt->workspace) {
        if (opt->workspace_bytes < need) return KCORE_EINVAL;
        ws = opt->workspace;
    } else {
        KC_CUDA(cudaMallocAsync(&ws, need, st));
        own_ws = true;
    }
    carve(ws, n, &cv);
    A.rowptr = rowptr;
    A.colidx = colidx;
    A.deg = cv.deg;
    A.core = core_out;
    A.order = (opt && opt->order_out) ? cv.order : nullptr;  // record the peel order only on request
    A.claimed = cv.claimed;
    A.gq_v = cv.gq_v;
    A.gq_beg = cv.gq_beg;
    A.gq_arc = cv.gq_arc;
    A.alive[0] = cv.alive0;
    A.alive[1] = cv.alive1;
    A.near[0] = cv.near0;
    A.near[1] = cv.near1;
    A.seg_len[0] = cv.seg0;
    A.seg_len[1] = cv.seg1;
    A.nseg = grid;
    A.seg_R = (n + A.nseg - 1) / A.nseg + 32;  // room for a 32-aligned identity slice
    A.S = cv.S;
    A.n = n;

    if (stats) {
        KC_CUDA(cudaEventCreate(&ev0));
        KC_CUDA(cudaEventCreate(&ev1));
    }
    k_init_state<<<1, 32, 0, st>>>(cv.S, n, solo, solo_scan, bloom, red, opt ? opt->near_min_alive : 0,
                                   opt ? opt->near_window : 0, trace,
                                   trace ? opt->trace_cta_out : nullptr, trace_cap);
    KC_CUDA(cudaGetLastError());
    if (stats) KC_CUDA(cudaEventRecord(ev0, st));
    if (algo == KCORE_ALGO_PERSISTENT) {
        const bool persist = !(opt && (opt->flags & KCORE_FLAG_NO_L2_PERSIST)) && di.persist_max > 0 &&
                             di.window_max > 0;
        if (persist) {
            // persisting L2 window over the scattered working set (claim bits +
            // working degrees): the adjacency stream of the heavy levels must not
            // evict it.  The set-aside is raised to the
            // window size (device limit, never lowered) and the lines are handed
            // back to normal priority by k_l2_release after the kernel.
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(grid);
            cfg.blockDim = dim3(kBlock);
            cfg.dynamicSmemBytes = smem;
            cfg.stream = st;
            cudaLaunchAttribute at[2];
            at[0].id = cudaLaunchAttributeCooperative;
            at[0].val.cooperative = 1;
            const size_t wbytes = std::min((size_t)((char *)(cv.deg + n) - (char *)cv.claimed), (size_t)di.window_max);
            size_t lim = 0;
            cudaDeviceGetLimit(&lim, cudaLimitPersistingL2CacheSize);
            const size_t want = std::min(wbytes, (size_t)di.persist_max);
            if (lim < want) {
                prev_limit = lim;
                limit_raised = true;
                KC_CUDA(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want));
                KC_CUDA(cudaDeviceGetLimit(&lim, cudaLimitPersistingL2CacheSize));
            }
            if (lim * 4 < wbytes) {
                // no usable set-aside (e.g. a profiler pinned the limit at 0): a window
                // with hitRatio ~ 0 would mark deg streaming -- launch without one
                void *args[] = {&A};
                KC_CUDA(cudaLaunchCooperativeKernel((const void *)k_persistent, dim3(grid), dim3(kBlock), args,
                                                    smem, st));
                goto launched;
            }
            at[1].id = cudaLaunchAttributeAccessPolicyWindow;
            at[1].val.accessPolicyWindow.base_ptr = cv.claimed;
            at[1].val.accessPolicyWindow.num_bytes = wbytes;
            at[1].val.accessPolicyWindow.hitRatio = (float)std::min(1.0, (double)lim / (double)wbytes);
            at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
            at[1].val.accessPolicyWindow.missProp = KC_MISS_PROP;
            cfg.attrs = at;
            cfg.numAttrs = 2;
            KC_CUDA(cudaLaunchKernelEx(&cfg, k_persistent, A));
            l2_lines = (int64_t)(wbytes / 128);
            l2_base = (const char *)cv.claimed;
        } else {
            void *args[] = {&A};
            KC_CUDA(cudaLaunchCooperativeKernel((const void *)k_persistent, dim3(grid), dim3(kBlock), args,
                                                smem, st));
        }
    } else {
        KC_CUDA(cudaMallocAsync((void **)&d_phase, sizeof(int32_t), st));
        int32_t ph = PH_INIT;
        int guard = 0;
        hl_launches = 1;  // k_init_state
        while (ph != PH_DONE) {
            k_phase<<<grid, kBlock, smem, st>>>(A);
            k_leader<<<1, 1, 0, st>>>(A, d_phase);
            hl_launches += 2;
            KC_CUDA(cudaGetLastError());
            KC_CUDA(cudaMemcpyAsync(&ph, d_phase, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
            KC_CUDA(cudaStreamSynchronize(st));
            if (++guard > (1 << 28)) { rc = KCORE_ECUDA; goto done; }
        }
    }
launched:
    if (stats) KC_CUDA(cudaEventRecord(ev1, st));
    if (l2_lines > 0) {
        k_l2_release<<<std::min<int64_t>((l2_lines + 255) / 256, 4 * di.sms), 256, 0, st>>>(l2_base, l2_lines);
        KC_CUDA(cudaGetLastError());
    }
    if (opt && opt->order_out)
        KC_CUDA(cudaMemcpyAsync(opt->order_out, cv.order, sizeof(int32_t) * (size_t)n,
                                cudaMemcpyDeviceToDevice, st));
    if (stats) {
        KC_CUDA(cudaMemcpyAsync(&hS, cv.S, sizeof(State), cudaMemcpyDeviceToHost, st));
        KC_CUDA(cudaStreamSynchronize(st));
        // the call has completed: hand the L2 set-aside back (a stream-ordered
        // restore does not exist; asynchronous calls leave the raised limit --
        // include/kcore.h, KCORE_FLAG_NO_L2_PERSIST)
        if (limit_raised) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, prev_limit);
        limit_raised = false;
        float ms = 0.f;
        cudaEventElapsedTime(&ms, ev0, ev1);
        const Ctrl &c = hS.pub;
        stats->levels = c.st_levels;
        stats->phases = c.st_phases;
        stats->solo_phases = c.st_solo;
        stats->barriers = c.st_bar;
        stats->scanned = c.st_scanned;
        stats->near_scans = c.st_near;
        stats->arcs_walked = (int64_t)hS.arcs_walked;
        stats->compactions = c.st_compact;
        stats->hub_arcs = c.st_hubarcs;
        stats->kmax = c.st_kmax;
        stats->grid_blocks = algo == KCORE_ALGO_PERSISTENT ? grid : grid;
        stats->block_threads = kBlock;
        stats->trace_len = (int32_t)hS.trace_n;
        stats->kernel_ms = ms;
        stats->launches = algo == KCORE_ALGO_PERSISTENT ? 2 + (l2_lines > 0 ? 1 : 0) : hl_launches;
    }
done:
    if (d_phase) cudaFreeAsync(d_phase, st);
    if (own_ws && ws) cudaFreeAsync(ws, st);
    if (ev0) cudaEventDestroy(ev0);
    if (ev1) cudaEventDestroy(ev1);
    return rc;
}

extern "C" int kcore_decompose(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                               int32_t *core_out, void *stream)
{
    return kcore_decompose_ex(rowptr, colidx, n, m, core_out, stream, nullptr, nullptr);
}

namespace {
// The host entry point moves gigabytes per call through stream-ordered
// allocations; by default the pool returns freed memory to the driver at every
// synchronisation, so each call would re-map its buffers.  Keep what the pool
// holds (cudaMemPoolAttrReleaseThreshold on the device's default pool, set
// once; torch's caching allocator does not use this pool).
void keep_pool_warm()
{
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDev) return;
    static bool done[kMaxDev] = {};
    std::lock_guard<std::mutex> lk(g_mu);
    if (done[dev]) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    done[dev] = true;
}
} // namespace

extern "C" int kcore_decompose_host(const int64_t *rowptr_h, const int32_t *colidx_h, int64_t n,
                                    int64_t m, int32_t *core_h, void *stream_,
                                    const kcore_options *opt, kcore_stats *stats)
{
    int rc = check_args(rowptr_h, colidx_h, n, m, core_h);
    if (rc) return rc;
    if (n == 0) {
        if (stats) memset(stats, 0, sizeof(*stats));
        return KCORE_OK;
    }
    cudaStream_t st = (cudaStream_t)stream_;
    int64_t *d_rp = nullptr;
    int32_t *d_ci = nullptr, *d_core = nullptr;
    keep_pool_warm();
    KC_CUDA(cudaMallocAsync((void **)&d_rp, sizeof(int64_t) * (size_t)(n + 1), st));
    KC_CUDA(cudaMallocAsync((void **)&d_ci, sizeof(int32_t) * (size_t)(m > 0 ? m : 1), st));
    KC_CUDA(cudaMallocAsync((void **)&d_core, sizeof(int32_t) * (size_t)n, st));
    KC_CUDA(cudaMemcpyAsync(d_rp, rowptr_h, sizeof(int64_t) * (size_t)(n + 1), cudaMemcpyHostToDevice, st));
    if (m > 0)
        KC_CUDA(cudaMemcpyAsync(d_ci, colidx_h, sizeof(int32_t) * (size_t)m, cudaMemcpyHostToDevice, st));
    {
        kcore_stats local;  // the host path synchronises anyway: stats make the call restore the L2 limit
        rc = kcore_decompose_ex(d_rp, d_ci, n, m, d_core, st, opt, stats ? stats : &local);
    }
    if (rc) goto done;
    KC_CUDA(cudaMemcpyAsync(core_h, d_core, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToHost, st));
    KC_CUDA(cudaStreamSynchronize(st));
done:
    if (d_rp) cudaFreeAsync(d_rp, st);
    if (d_ci) cudaFreeAsync(d_ci, st);
    if (d_core) cudaFreeAsync(d_core, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && rc == KCORE_OK) rc = KCORE_ECUDA;
    return rc;
}

// ------------------------------------------------------------ validation
namespace {
__global__ void k_validate(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                           int *flag)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (tid == 0 && (rowptr[0] != 0 || rowptr[n] != m)) atomicOr(flag, 1);
    for (int64_t v = tid; v < n; v += stride) {
        const int64_t b = rowptr[v], e = rowptr[v + 1];
        if (e < b || b < 0 || e > m) { atomicOr(flag, 1); continue; }
        int32_t prev = -1;
        for (int64_t x = b; x < e; x++) {
            const int32_t u = colidx[x];
            if (u < 0 || u >= n) { atomicOr(flag, 2); break; }
            if (u == v) { atomicOr(flag, 4); break; }
            if (u <= prev) { atomicOr(flag, 8); break; }
            prev = u;
            // symmetric: v must appear in N(u)
            int64_t lo = rowptr[u], hi = rowptr[u + 1];
            if (lo < 0 || hi > m || hi < lo) { atomicOr(flag, 1); break; }
            while (lo < hi) {
                const int64_t mid = lo + (hi - lo) / 2;
                if (colidx[mid] < (int32_t)v) lo = mid + 1; else hi = mid;
            }
            if (lo >= rowptr[u + 1] || colidx[lo] != (int32_t)v) { atomicOr(flag, 16); break; }
        }
    }
}
} // namespace

extern "C" int kcore_validate_csr(const int64_t *rowptr, const int32_t *colidx, int64_t n,
                                  int64_t m, void *stream_)
{
    int rc = check_args(rowptr, colidx, n, m, (const int32_t *)rowptr);
    if (rc) return rc;
    if (n == 0) return KCORE_OK;
    cudaStream_t st = (cudaStream_t)stream_;
    int *d_flag = nullptr, h_flag = 0;
    KC_CUDA(cudaMallocAsync((void **)&d_flag, sizeof(int), st));
    KC_CUDA(cudaMemsetAsync(d_flag, 0, sizeof(int), st));
    k_validate<<<1184, 256, 0, st>>>(rowptr, colidx, n, m, d_flag);
    KC_CUDA(cudaGetLastError());
    KC_CUDA(cudaMemcpyAsync(&h_flag, d_flag, sizeof(int), cudaMemcpyDeviceToHost, st));
    KC_CUDA(cudaStreamSynchronize(st));
    rc = h_flag ? KCORE_EGRAPH : KCORE_OK;
done:
    if (d_flag) cudaFreeAsync(d_flag, st);
    cudaStreamSynchronize(st);
    return rc;
}
