// kcore_mg.cu -- multi-GPU k-core decomposition (include/kcore.h).
//
// 1-D vertex-range ownership (north star; the paper's multi-GPU future work,
// P:L587, with decrements routed to OWNER GPUs instead of a master GPU).
// Rank r owns vertices [vb_r, ve_r) and their CSR rows (global neighbour
// ids) and deg/core for them.  Per level k:
//   scan      owned vertices with deg == k -> frontier F          (Alg. 2)
//   sub-round for every arc (v,u) of F (Alg. 3 l.19-24):
//               u owned  -> filter, atomicSub, append on k+1, restore on <= k
//               u remote -> packed into the send run of owner(u)
//             exchange: counts, then payload (NCCL send/recv over NVLink)
//             apply the received decrements with the same rule
//             all-reduce(min) of {-(F' non-empty), min next degree}
//   level end k <- max(k+1, global min); done when no vertex is alive
// The scan finishes before the level's first peel (stream order), so no
// claim bits are needed: the k+1 -> k transition of each vertex is seen by
// exactly one atomicSub whether it came from a local or a
// received decrement.
//
// The driver is written once against a Transport: NCCL (one rank per
// process) or a device-memory loopback (P virtual ranks on this GPU, used to
// test the protocol on a single GPU).  Host-driven: two stream syncs per
// sub-round (send counts, then the all-reduced control words).
#include "kcore.h"
#include "kcore_mgd.h"

#include <climits>
#include <cstdint>
#include <cstring>
#include <nccl.h>
#include <vector>

#include <cuda_runtime.h>

namespace {

constexpr int kMaxRanks = 64;
constexpr int kMgBlock = 256;

struct Owners {
    int64_t start[kMaxRanks + 1];  // rank r owns [start[r], start[r+1])
    int32_t nranks;
    int32_t pad;
};

__device__ __forceinline__ int owner_of(const Owners &o, int64_t u)
{
    int lo = 0, hi = o.nranks - 1;
    while (lo < hi) {  // largest r with start[r] <= u
        const int mid = (lo + hi + 1) >> 1;
        if (o.start[mid] <= u) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// per-rank device control block (one D2H per step)
struct MgCtl {
    unsigned long long fcount;       // next frontier size
    int32_t min_next;                // lower bound on the next level's degree
    int32_t pad;
    unsigned long long send[kMaxRanks];   // remote decrements per destination
    unsigned long long cursor[kMaxRanks]; // fill cursors
};

struct RankView {
    const int64_t *rp;   // local rowptr, rp[0] may be non-zero (virtual ranks)
    int64_t rp0;         // rp[0] (host copy)
    const int32_t *ci;   // colidx at arc rp0
    int32_t *deg;        // == core_out for the owned range
    int64_t vb, nl;
    int32_t *F, *Fn;     // frontiers (local indices)
    int32_t *sendbuf;    // packed remote targets (global ids)
    int32_t *recvbuf;
    int64_t recv_cap;
    MgCtl *ctl;
};

__global__ void k_mg_init(RankView R, int32_t *min_out)
{
    int lmin = INT_MAX;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < R.nl;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t d = (int32_t)(R.rp[i + 1] - R.rp[i]);
        R.deg[i] = d;
        lmin = min(lmin, d);
    }
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(0xffffffffu, lmin, o));
    if ((threadIdx.x & 31) == 0 && lmin != INT_MAX) atomicMin(min_out, lmin);
}

__device__ __forceinline__ void append_frontier(RankView &R, bool hit, int32_t i)
{
    const unsigned b = __ballot_sync(0xffffffffu, hit);
    if (!b) return;
    const int lane = threadIdx.x & 31, lead = __ffs(b) - 1;
    unsigned long long base = 0;
    if (lane == lead) base = atomicAdd(&R.ctl->fcount, (unsigned long long)__popc(b));
    base = __shfl_sync(0xffffffffu, base, lead);
    if (hit) {
        unsigned below;
        asm("mov.u32 %0, %%lanemask_lt;" : "=r"(below));
        R.Fn[base + __popc(b & below)] = i;
    }
}

// Alg. 2: owned vertices with deg == k -> Fn; min over deg > k.
__global__ void k_mg_scan(RankView R, int k)
{
    int lmin = INT_MAX;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < R.nl; base += stride) {
        const int64_t i = base + threadIdx.x;
        bool hit = false;
        if (i < R.nl) {
            const int d = R.deg[i];
            hit = (d == k);
            if (d > k) lmin = min(lmin, d);
        }
        append_frontier(R, hit, (int32_t)i);
    }
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(0xffffffffu, lmin, o));
    if ((threadIdx.x & 31) == 0 && lmin != INT_MAX) atomicMin(&R.ctl->min_next, lmin);
}

// decrement an OWNED vertex (local index i) with the clamp rule of Alg. 3
__device__ __forceinline__ bool decrement(RankView &R, int64_t i, int k, int &lmin)
{
    if (R.deg[i] <= k) return false;  // P:L324 filter (stale reads are harmless)
    const int old = atomicSub(R.deg + i, 1);
    if (old == k + 1) return true;
    if (old <= k) atomicAdd(R.deg + i, 1);  // restore (Fig. 6)
    else lmin = min(lmin, old - 1);
    return false;
}

// Frontier vertices with more than kBig arcs are walked by a whole CTA
// (BIG=true launch), the rest by one warp each (BIG=false launch).
constexpr int64_t kBig = 4096;

template <bool BIG>
__device__ __forceinline__ bool mg_unit(const RankView &R, int64_t f, int64_t &a0, int64_t &a1)
{
    const int32_t v = R.F[f];
    a0 = R.rp[v] - R.rp0;
    a1 = R.rp[v + 1] - R.rp0;
    return BIG ? (a1 - a0 > kBig) : (a1 - a0 <= kBig);
}

// pass 1: remote decrements per destination (shared-memory histogram)
template <bool BIG>
__global__ void k_mg_count(RankView R, Owners O, int64_t fcnt, int32_t self)
{
    __shared__ unsigned long long hist[kMaxRanks];
    for (int d = threadIdx.x; d < O.nranks; d += blockDim.x) hist[d] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int64_t unit = BIG ? blockIdx.x : (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int64_t units = BIG ? gridDim.x : (((int64_t)gridDim.x * blockDim.x) >> 5);
    const int64_t first = BIG ? wib * 32 : 0, step = BIG ? blockDim.x : 32;
    const int64_t lo_own = O.start[self], hi_own = O.start[self + 1];
    for (int64_t f = unit; f < fcnt; f += units) {
        int64_t a0, a1;
        if (!mg_unit<BIG>(R, f, a0, a1)) continue;
        for (int64_t a = a0 + first + lane; a < a1; a += step) {
            const int64_t u = R.ci[a];
            if (u < lo_own || u >= hi_own) atomicAdd(&hist[owner_of(O, u)], 1ULL);
        }
    }
    __syncthreads();
    for (int d = threadIdx.x; d < O.nranks; d += blockDim.x)
        if (hist[d]) atomicAdd(&R.ctl->send[d], hist[d]);
}

// pass 2: apply owned decrements, pack remote ones at off[d] + cursor
struct Offs { unsigned long long off[kMaxRanks]; };

template <bool BIG>
__global__ void k_mg_fill(RankView R, Owners O, Offs S, int64_t fcnt, int32_t self, int k)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int64_t unit = BIG ? blockIdx.x : (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int64_t units = BIG ? gridDim.x : (((int64_t)gridDim.x * blockDim.x) >> 5);
    const int64_t first = BIG ? wib * 32 : 0, step = BIG ? blockDim.x : 32;
    const int64_t lo_own = O.start[self], hi_own = O.start[self + 1];
    int lmin = INT_MAX;
    for (int64_t f = unit; f < fcnt; f += units) {
        int64_t a0, a1;
        if (!mg_unit<BIG>(R, f, a0, a1)) continue;
        for (int64_t ab = a0 + first; ab < a1; ab += step) {
            const int64_t a = ab + lane;
            int64_t u = -1;
            if (a < a1) u = R.ci[a];
            const bool own = u >= 0 && u >= lo_own && u < hi_own;
            const bool hit = own && decrement(R, u - lo_own, k, lmin);
            append_frontier(R, hit, (int32_t)(u - lo_own));
            const int dest = (u >= 0 && !own) ? owner_of(O, u) : -1;
            // warp-aggregated packing per destination
            unsigned pend = __ballot_sync(0xffffffffu, dest >= 0);
            while (pend) {
                const int dl = __ffs(pend) - 1;
                const int dd = __shfl_sync(0xffffffffu, dest, dl);
                const unsigned grp = __ballot_sync(0xffffffffu, dest == dd);
                unsigned long long base = 0;
                if (lane == dl) base = atomicAdd(&R.ctl->cursor[dd], (unsigned long long)__popc(grp));
                base = __shfl_sync(0xffffffffu, base, dl);
                if (dest == dd) {
                    unsigned below;
                    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(below));
                    R.sendbuf[S.off[dd] + base + __popc(grp & below)] = (int32_t)u;
                }
                pend &= ~grp;
            }
        }
    }
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(0xffffffffu, lmin, o));
    if (lane == 0 && lmin != INT_MAX) atomicMin(&R.ctl->min_next, lmin);
}

// received decrements (global ids of owned vertices)
__global__ void k_mg_apply(RankView R, int64_t cnt, int64_t vb, int k)
{
    int lmin = INT_MAX;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < cnt; base += stride) {
        const int64_t x = base + threadIdx.x;
        bool hit = false;
        int64_t i = 0;
        if (x < cnt) {
            i = (int64_t)R.recvbuf[x] - vb;
            hit = decrement(R, i, k, lmin);
        }
        append_frontier(R, hit, (int32_t)i);
    }
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(0xffffffffu, lmin, o));
    if ((threadIdx.x & 31) == 0 && lmin != INT_MAX) atomicMin(&R.ctl->min_next, lmin);
}

__global__ void k_mg_reset(MgCtl *c, int nranks)
{
    if (threadIdx.x == 0) { c->fcount = 0; c->min_next = INT_MAX; }
    for (int d = threadIdx.x; d < nranks; d += blockDim.x) { c->send[d] = 0; c->cursor[d] = 0; }
}

// --------------------------------------------------------------- transports
struct Transport {
    virtual ~Transport() {}
    // counts[s][d] over the local ranks -> recv counts rc[s][d] (from global rank d)
    virtual int exchange_counts(const std::vector<std::vector<unsigned long long>> &send,
                                std::vector<std::vector<unsigned long long>> &recv) = 0;
    // payload: rank s sends sendbuf[soff[s][d] .. + send[s][d]) to d; receives into recvbuf at roff
    virtual int exchange_payload(std::vector<RankView> &R, const std::vector<std::vector<unsigned long long>> &send,
                                 const std::vector<std::vector<unsigned long long>> &soff,
                                 const std::vector<std::vector<unsigned long long>> &recv,
                                 const std::vector<std::vector<unsigned long long>> &roff) = 0;
    // element-wise min of two ints over all ranks
    virtual int allreduce_min2(int32_t v[2]) = 0;
};

struct LoopbackTransport : Transport {
    int P;
    cudaStream_t st;
    LoopbackTransport(int p, cudaStream_t s) : P(p), st(s) {}
    int exchange_counts(const std::vector<std::vector<unsigned long long>> &send,
                        std::vector<std::vector<unsigned long long>> &recv) override
    {
        for (int d = 0; d < P; d++)
            for (int s = 0; s < P; s++) recv[d][s] = send[s][d];
        return KCORE_OK;
    }
    int exchange_payload(std::vector<RankView> &R, const std::vector<std::vector<unsigned long long>> &send,
                         const std::vector<std::vector<unsigned long long>> &soff,
                         const std::vector<std::vector<unsigned long long>> &,
                         const std::vector<std::vector<unsigned long long>> &roff) override
    {
        for (int s = 0; s < P; s++)
            for (int d = 0; d < P; d++) {
                if (!send[s][d]) continue;
                if (cudaMemcpyAsync(R[d].recvbuf + roff[d][s], R[s].sendbuf + soff[s][d],
                                    sizeof(int32_t) * send[s][d], cudaMemcpyDeviceToDevice, st) != cudaSuccess)
                    return KCORE_ECUDA;
            }
        return KCORE_OK;
    }
    int allreduce_min2(int32_t v[2]) override { (void)v; return KCORE_OK; }  // already global
};

struct NcclTransport : Transport {
    ncclComm_t comm;
    int P, rank;
    cudaStream_t st;
    unsigned long long *d_cnt = nullptr;  // [2][P]
    int32_t *d_red = nullptr;
    bool ok = false;  // both scratch buffers allocated
    NcclTransport(ncclComm_t c, int p, int r, cudaStream_t s) : comm(c), P(p), rank(r), st(s)
    {
        ok = cudaMallocAsync((void **)&d_cnt, sizeof(unsigned long long) * 2 * P, st) == cudaSuccess &&
             cudaMallocAsync((void **)&d_red, sizeof(int32_t) * 2, st) == cudaSuccess;
    }
    ~NcclTransport()
    {
        if (d_cnt) cudaFreeAsync(d_cnt, st);
        if (d_red) cudaFreeAsync(d_red, st);
    }
    int exchange_counts(const std::vector<std::vector<unsigned long long>> &send,
                        std::vector<std::vector<unsigned long long>> &recv) override
    {
        if (cudaMemcpyAsync(d_cnt, send[0].data(), sizeof(unsigned long long) * P, cudaMemcpyHostToDevice, st))
            return KCORE_ECUDA;
        if (ncclGroupStart() != ncclSuccess) return KCORE_ENCCL;
        for (int d = 0; d < P; d++) {
            if (ncclSend(d_cnt + d, 1, ncclUint64, d, comm, st) != ncclSuccess) return KCORE_ENCCL;
            if (ncclRecv(d_cnt + P + d, 1, ncclUint64, d, comm, st) != ncclSuccess) return KCORE_ENCCL;
        }
        if (ncclGroupEnd() != ncclSuccess) return KCORE_ENCCL;
        if (cudaMemcpyAsync(recv[0].data(), d_cnt + P, sizeof(unsigned long long) * P, cudaMemcpyDeviceToHost, st))
            return KCORE_ECUDA;
        return cudaStreamSynchronize(st) == cudaSuccess ? KCORE_OK : KCORE_ECUDA;
    }
    int exchange_payload(std::vector<RankView> &R, const std::vector<std::vector<unsigned long long>> &send,
                         const std::vector<std::vector<unsigned long long>> &soff,
                         const std::vector<std::vector<unsigned long long>> &recv,
                         const std::vector<std::vector<unsigned long long>> &roff) override
    {
        if (ncclGroupStart() != ncclSuccess) return KCORE_ENCCL;
        for (int d = 0; d < P; d++) {
            if (d == rank) continue;
            if (send[0][d] && ncclSend(R[0].sendbuf + soff[0][d], send[0][d], ncclInt32, d, comm, st) != ncclSuccess)
                return KCORE_ENCCL;
            if (recv[0][d] && ncclRecv(R[0].recvbuf + roff[0][d], recv[0][d], ncclInt32, d, comm, st) != ncclSuccess)
                return KCORE_ENCCL;
        }
        return ncclGroupEnd() == ncclSuccess ? KCORE_OK : KCORE_ENCCL;
    }
    int allreduce_min2(int32_t v[2]) override
    {
        if (cudaMemcpyAsync(d_red, v, sizeof(int32_t) * 2, cudaMemcpyHostToDevice, st)) return KCORE_ECUDA;
        if (ncclAllReduce(d_red, d_red, 2, ncclInt32, ncclMin, comm, st) != ncclSuccess) return KCORE_ENCCL;
        if (cudaMemcpyAsync(v, d_red, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, st)) return KCORE_ECUDA;
        return cudaStreamSynchronize(st) == cudaSuccess ? KCORE_OK : KCORE_ECUDA;
    }
};

#define MG_CK(x)                                                                                   \
    do {                                                                                           \
        cudaError_t e_ = (x);                                                                      \
        if (e_ != cudaSuccess) return e_ == cudaErrorMemoryAllocation ? KCORE_ENOMEM : KCORE_ECUDA; \
    } while (0)
#define MG_RC(x)                                                                                   \
    do {                                                                                           \
        int r_ = (x);                                                                              \
        if (r_) return r_;                                                                         \
    } while (0)

int grid_for(int64_t work)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t g = (work + kMgBlock - 1) / kMgBlock;
    if (g > (int64_t)sms * 8) g = (int64_t)sms * 8;
    return (int)(g < 1 ? 1 : g);
}

// The protocol over the local ranks R (global ranks self0 .. self0+L-1).
int mg_drive(std::vector<RankView> &R, const Owners &O, int self0, Transport &T, cudaStream_t st,
             kcore_stats *stats)
{
    const int L = (int)R.size(), P = O.nranks;
    std::vector<MgCtl> hc(L);
    std::vector<std::vector<unsigned long long>> send(L, std::vector<unsigned long long>(P)),
        recv(L, std::vector<unsigned long long>(P)), soff(L, std::vector<unsigned long long>(P + 1)),
        roff(L, std::vector<unsigned long long>(P + 1));
    std::vector<int64_t> fcnt(L, 0);
    int64_t levels = 0, subrounds = 0, exchanged = 0, launches = 0;
    int kmax = 0;

    // deg init and the first k
    int32_t mins[2] = {0, INT_MAX};
    for (int r = 0; r < L; r++) {
        k_mg_reset<<<1, 64, 0, st>>>(R[r].ctl, P);
        if (R[r].nl) k_mg_init<<<grid_for(R[r].nl), kMgBlock, 0, st>>>(R[r], &R[r].ctl->min_next);
        launches += 1 + (R[r].nl ? 1 : 0);
        MG_CK(cudaGetLastError());
        MG_CK(cudaMemcpyAsync(&hc[r], R[r].ctl, sizeof(MgCtl), cudaMemcpyDeviceToHost, st));
    }
    MG_CK(cudaStreamSynchronize(st));
    for (int r = 0; r < L; r++) mins[1] = hc[r].min_next < mins[1] ? hc[r].min_next : mins[1];
    MG_RC(T.allreduce_min2(mins));
    if (mins[1] == INT_MAX) {  // no vertex anywhere
        if (stats) memset(stats, 0, sizeof(*stats));
        return KCORE_OK;
    }
    int k = mins[1];
    while (true) {
        // ---- level scan
        int lvl_min = INT_MAX;
        int64_t lvl_removed = 0;
        for (int r = 0; r < L; r++) {
            k_mg_reset<<<1, 64, 0, st>>>(R[r].ctl, P);
            if (R[r].nl) k_mg_scan<<<grid_for(R[r].nl), kMgBlock, 0, st>>>(R[r], k);
            launches += 1 + (R[r].nl ? 1 : 0);
            MG_CK(cudaGetLastError());
            MG_CK(cudaMemcpyAsync(&hc[r], R[r].ctl, sizeof(MgCtl), cudaMemcpyDeviceToHost, st));
        }
        MG_CK(cudaStreamSynchronize(st));
        for (int r = 0; r < L; r++) {
            fcnt[r] = (int64_t)hc[r].fcount;
            lvl_min = hc[r].min_next < lvl_min ? hc[r].min_next : lvl_min;
            std::swap(R[r].F, R[r].Fn);
        }
        // ---- peel sub-rounds
        while (true) {
            int32_t ctl2[2] = {0, INT_MAX};
            for (int r = 0; r < L; r++) if (fcnt[r]) ctl2[0] = -1;
            MG_RC(T.allreduce_min2(ctl2));
            if (ctl2[0] == 0) break;  // every frontier is empty: level done
            subrounds++;
            for (int r = 0; r < L; r++) lvl_removed += fcnt[r];
            // pass 1: counts
            for (int r = 0; r < L; r++) {
                k_mg_reset<<<1, 64, 0, st>>>(R[r].ctl, P);
                if (fcnt[r]) {
                    k_mg_count<false><<<grid_for(fcnt[r] * 32), kMgBlock, 0, st>>>(R[r], O, fcnt[r], self0 + r);
                    k_mg_count<true><<<grid_for(fcnt[r] * kMgBlock), kMgBlock, 0, st>>>(R[r], O, fcnt[r], self0 + r);
                    launches += 2;
                }
                launches++;
                MG_CK(cudaGetLastError());
                MG_CK(cudaMemcpyAsync(&hc[r], R[r].ctl, sizeof(MgCtl), cudaMemcpyDeviceToHost, st));
            }
            MG_CK(cudaStreamSynchronize(st));
            for (int r = 0; r < L; r++) {
                soff[r][0] = 0;
                for (int d = 0; d < P; d++) {
                    send[r][d] = hc[r].send[d];
                    soff[r][d + 1] = soff[r][d] + send[r][d];
                }
            }
            MG_RC(T.exchange_counts(send, recv));
            for (int r = 0; r < L; r++) {
                roff[r][0] = 0;
                for (int d = 0; d < P; d++) roff[r][d + 1] = roff[r][d] + recv[r][d];
                const int64_t need = (int64_t)roff[r][P];
                if (need > R[r].recv_cap) {
                    if (R[r].recvbuf) MG_CK(cudaFreeAsync(R[r].recvbuf, st));
                    R[r].recv_cap = need + need / 2 + 1024;
                    MG_CK(cudaMallocAsync((void **)&R[r].recvbuf, sizeof(int32_t) * R[r].recv_cap, st));
                }
                exchanged += (int64_t)soff[r][P];
            }
            // pass 2: owned decrements + packing
            for (int r = 0; r < L; r++) {
                Offs S;
                for (int d = 0; d < P; d++) S.off[d] = soff[r][d];
                if (fcnt[r]) {
                    k_mg_fill<false><<<grid_for(fcnt[r] * 32), kMgBlock, 0, st>>>(R[r], O, S, fcnt[r], self0 + r, k);
                    k_mg_fill<true><<<grid_for(fcnt[r] * kMgBlock), kMgBlock, 0, st>>>(R[r], O, S, fcnt[r], self0 + r, k);
                    launches += 2;
                }
                MG_CK(cudaGetLastError());
            }
            MG_RC(T.exchange_payload(R, send, soff, recv, roff));
            for (int r = 0; r < L; r++) {
                const int64_t cnt = (int64_t)roff[r][P];
                if (cnt) {
                    k_mg_apply<<<grid_for(cnt), kMgBlock, 0, st>>>(R[r], cnt, O.start[self0 + r], k);
                    launches++;
                }
                MG_CK(cudaGetLastError());
                MG_CK(cudaMemcpyAsync(&hc[r], R[r].ctl, sizeof(MgCtl), cudaMemcpyDeviceToHost, st));
            }
            MG_CK(cudaStreamSynchronize(st));
            for (int r = 0; r < L; r++) {
                fcnt[r] = (int64_t)hc[r].fcount;
                lvl_min = hc[r].min_next < lvl_min ? hc[r].min_next : lvl_min;
                std::swap(R[r].F, R[r].Fn);
            }
        }
        // ---- level end: k <- max(k+1, global min); done when nothing is alive
        int32_t m2[2] = {lvl_removed ? -1 : 0, lvl_min};
        MG_RC(T.allreduce_min2(m2));
        if (m2[0] < 0) { levels++; kmax = k; }
        if (m2[1] == INT_MAX) break;
        k = m2[1] > k + 1 ? m2[1] : k + 1;
    }
    if (stats) {
        memset(stats, 0, sizeof(*stats));
        stats->levels = levels;
        stats->phases = subrounds;
        stats->kmax = kmax;
        stats->hub_arcs = exchanged;  // remote decrements sent by the local ranks
        stats->launches = launches;
    }
    return KCORE_OK;
}

int alloc_rank(RankView &v, int64_t nl, int64_t m_local, int nranks, cudaStream_t st)
{
    const size_t nn = (size_t)(nl > 0 ? nl : 1);
    MG_CK(cudaMallocAsync((void **)&v.F, sizeof(int32_t) * nn, st));
    MG_CK(cudaMallocAsync((void **)&v.Fn, sizeof(int32_t) * nn, st));
    MG_CK(cudaMallocAsync((void **)&v.sendbuf, sizeof(int32_t) * (size_t)(m_local > 0 ? m_local : 1), st));
    MG_CK(cudaMallocAsync((void **)&v.ctl, sizeof(MgCtl), st));
    v.recvbuf = nullptr;
    v.recv_cap = 0;
    (void)nranks;
    return KCORE_OK;
}

void free_rank(RankView &v, cudaStream_t st)
{
    if (v.F) cudaFreeAsync(v.F, st);
    if (v.Fn) cudaFreeAsync(v.Fn, st);
    if (v.sendbuf) cudaFreeAsync(v.sendbuf, st);
    if (v.recvbuf) cudaFreeAsync(v.recvbuf, st);
    if (v.ctl) cudaFreeAsync(v.ctl, st);
    v.F = v.Fn = v.sendbuf = v.recvbuf = nullptr;
    v.ctl = nullptr;
}

} // namespace

extern "C" int kcore_nccl_unique_id(void *id_out)
{
    if (!id_out) return KCORE_EINVAL;
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) return KCORE_ENCCL;
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    memcpy(id_out, &id, sizeof(id));
    return KCORE_OK;
}

extern "C" int kcore_nccl_comm_init(void **comm_out, int32_t nranks, const void *id_in, int32_t rank)
{
    if (!comm_out || !id_in || nranks < 1 || rank < 0 || rank >= nranks) return KCORE_EINVAL;
    ncclUniqueId id;
    memcpy(&id, id_in, sizeof(id));
    ncclComm_t c = nullptr;
    if (ncclCommInitRank(&c, nranks, id, rank) != ncclSuccess) return KCORE_ENCCL;
    *comm_out = (void *)c;
    return KCORE_OK;
}

extern "C" int kcore_nccl_comm_destroy(void *comm)
{
    if (!comm) return KCORE_EINVAL;
    return ncclCommDestroy((ncclComm_t)comm) == ncclSuccess ? KCORE_OK : KCORE_ENCCL;
}

static int mg_hostloop_nccl(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global,
                            int64_t v_begin, int64_t v_end, int64_t m_local, int32_t *core_out_local,
                            void *stream_, void *nccl_comm, kcore_stats *stats);
static int mg_hostloop_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                               int32_t nranks, int32_t *core_out, void *stream_, kcore_stats *stats);

extern "C" int kcore_decompose_mg(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global,
                                  int64_t v_begin, int64_t v_end, int64_t m_local, int32_t *core_out_local,
                                  void *stream_, void *nccl_comm, kcore_stats *stats)
{
    return mg_hostloop_nccl(rowptr_local, colidx_local, n_global, v_begin, v_end, m_local, core_out_local, stream_,
                            nccl_comm, stats);
}

extern "C" int kcore_decompose_mg_ex(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global,
                                     int64_t v_begin, int64_t v_end, int64_t m_local, int32_t *core_out_local,
                                     void *stream_, void *nccl_comm, int32_t mg_algo, kcore_stats *stats)
{
    if (mg_algo == KCORE_MG_DEVICE)
        return mgd_nccl(rowptr_local, colidx_local, n_global, v_begin, v_end, m_local, core_out_local, stream_,
                        nccl_comm, stats);
    if (mg_algo == KCORE_MG_HOSTLOOP)
        return mg_hostloop_nccl(rowptr_local, colidx_local, n_global, v_begin, v_end, m_local, core_out_local,
                                stream_, nccl_comm, stats);
    return KCORE_EINVAL;
}

extern "C" int kcore_decompose_mg_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                                          int32_t nranks, int32_t *core_out, void *stream_, kcore_stats *stats)
{
    return mgd_virtual(rowptr, colidx, n, m, nranks, core_out, stream_, stats);
}

extern "C" int kcore_decompose_mg_virtual_ex(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                                             int32_t nranks, int32_t *core_out, void *stream_, int32_t mg_algo,
                                             kcore_stats *stats)
{
    if (mg_algo == KCORE_MG_DEVICE) return mgd_virtual(rowptr, colidx, n, m, nranks, core_out, stream_, stats);
    if (mg_algo == KCORE_MG_HOSTLOOP)
        return mg_hostloop_virtual(rowptr, colidx, n, m, nranks, core_out, stream_, stats);
    return KCORE_EINVAL;
}

static int mg_hostloop_nccl(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global,
                            int64_t v_begin, int64_t v_end, int64_t m_local, int32_t *core_out_local,
                            void *stream_, void *nccl_comm, kcore_stats *stats)
{
    if (!nccl_comm || n_global < 0 || n_global >= ((int64_t)1 << 31) || v_begin < 0 || v_end < v_begin ||
        v_end > n_global || m_local < 0)
        return KCORE_EINVAL;
    const int64_t nl = v_end - v_begin;
    if (nl > 0 && (!rowptr_local || !core_out_local)) return KCORE_EINVAL;
    if (m_local > 0 && !colidx_local) return KCORE_EINVAL;
    cudaStream_t st = (cudaStream_t)stream_;
    ncclComm_t comm = (ncclComm_t)nccl_comm;
    int P = 0, rank = 0;
    if (ncclCommCount(comm, &P) != ncclSuccess || ncclCommUserRank(comm, &rank) != ncclSuccess) return KCORE_ENCCL;
    if (P > kMaxRanks) return KCORE_EUNSUPPORTED;
    NcclTransport T(comm, P, rank, st);
    // owner table: every rank contributes its v_begin (ranges tile [0, n) in rank order).
    // The validity of every rank's range (and of its scratch) is all-reduced, so
    // all ranks return the same status together -- none is left waiting in a
    // collective of the protocol.
    Owners O;
    memset(&O, 0, sizeof(O));
    O.nranks = P;
    {
        int64_t *d_vb = nullptr;
        MG_CK(cudaMallocAsync((void **)&d_vb, sizeof(int64_t) * (P + 1), st));
        MG_CK(cudaMemcpyAsync(d_vb + rank, &v_begin, sizeof(int64_t), cudaMemcpyHostToDevice, st));
        if (ncclAllGather(d_vb + rank, d_vb, 1, ncclInt64, comm, st) != ncclSuccess) return KCORE_ENCCL;
        MG_CK(cudaMemcpyAsync(O.start, d_vb, sizeof(int64_t) * P, cudaMemcpyDeviceToHost, st));
        MG_CK(cudaFreeAsync(d_vb, st));
        MG_CK(cudaStreamSynchronize(st));
        O.start[P] = n_global;
        const bool mine_ok = T.ok && O.start[rank] == v_begin && (rank + 1 >= P || O.start[rank + 1] == v_end) &&
                             (rank + 1 != P || v_end == n_global) && O.start[0] == 0;
        int32_t flag[2] = {mine_ok ? 0 : -1, INT_MAX};
        MG_RC(T.allreduce_min2(flag));  // min over ranks: -1 if any rank is invalid
        if (flag[0] < 0) return T.ok ? KCORE_EINVAL : KCORE_ENOMEM;
    }
    std::vector<RankView> R(1);
    RankView &v = R[0];
    memset(&v, 0, sizeof(v));
    v.rp = rowptr_local;
    v.rp0 = 0;
    if (nl > 0) MG_CK(cudaMemcpyAsync(&v.rp0, rowptr_local, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    MG_CK(cudaStreamSynchronize(st));
    v.ci = colidx_local;
    v.deg = core_out_local;
    v.vb = v_begin;
    v.nl = nl;
    int rc = alloc_rank(v, nl, m_local, P, st);
    if (!rc) rc = mg_drive(R, O, rank, T, st, stats);
    free_rank(v, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && !rc) rc = KCORE_ECUDA;
    return rc;
}

static int mg_hostloop_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                               int32_t nranks, int32_t *core_out, void *stream_, kcore_stats *stats)
{
    if (n < 0 || n >= ((int64_t)1 << 31) || m < 0 || nranks < 1 || nranks > kMaxRanks) return KCORE_EINVAL;
    if (n > 0 && (!rowptr || !core_out)) return KCORE_EINVAL;
    if (m > 0 && !colidx) return KCORE_EINVAL;
    if (stats) memset(stats, 0, sizeof(*stats));
    if (n == 0) return KCORE_OK;
    cudaStream_t st = (cudaStream_t)stream_;
    Owners O;
    memset(&O, 0, sizeof(O));
    O.nranks = nranks;
    for (int r = 0; r <= nranks; r++) O.start[r] = (n * r) / nranks;
    std::vector<int64_t> hrp(nranks + 1);
    for (int r = 0; r <= nranks; r++)
        MG_CK(cudaMemcpyAsync(&hrp[r], rowptr + O.start[r], sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    MG_CK(cudaStreamSynchronize(st));
    std::vector<RankView> R(nranks);
    int rc = KCORE_OK;
    for (int r = 0; r < nranks && !rc; r++) {
        RankView &v = R[r];
        memset(&v, 0, sizeof(v));
        v.rp = rowptr + O.start[r];
        v.rp0 = hrp[r];
        v.ci = colidx + hrp[r];
        v.deg = core_out + O.start[r];
        v.vb = O.start[r];
        v.nl = O.start[r + 1] - O.start[r];
        rc = alloc_rank(v, v.nl, hrp[r + 1] - hrp[r], nranks, st);
    }
    LoopbackTransport T(nranks, st);
    if (!rc) rc = mg_drive(R, O, 0, T, st, stats);
    for (auto &v : R) free_rank(v, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && !rc) rc = KCORE_ECUDA;
    return rc;
}
