// kc_kernels.cuh -- sm_100a kernels of the k-core hot path.
//
// One call = one persistent cooperative kernel (k_persistent) that runs the
// whole decomposition as a device-resident state machine:
//
//   INIT   deg[v] = rowptr[v+1]-rowptr[v] into core_out, min-degree reduce    (Alg.1 l.1)
//   SCAN   level k: frontier <- {v alive : deg[v] == k}; fused min{deg > k};   (Alg.2)
//          optional alive-list compaction (reading R6 / Q14)
//   PEEL   sub-round over frontier slots [s,e): for every arc (v,u):          (Alg.3 l.12-24)
//          if deg[u] > k: old = atomicSub(&deg[u],1);
//             old == k+1 -> append u (it reached k: next sub-round)
//             old <= k   -> atomicAdd(&deg[u],1)  (restore, Fig. 6)
//             else       -> min_next = min(min_next, old-1)   (level skip, reading R5)
//   SOLO   a small peel sub-round sequence run by ONE CTA with __syncthreads
//          instead of grid barriers (latency path for tiny frontiers)
//   level end: k <- max(k+1, min_next)  (Alg.1 l.9 does k+1; reading R5)
//
// Phases are separated by a grid barrier whose last arriver ("leader") runs
// the level/sub-round control logic (Alg.1 l.5-9 and Alg.3 l.5) on the device
// and publishes the next phase, so there is no host round-trip at all.
//
// The frontier queue is one array order[n] (every vertex is appended exactly
// once in the whole run, so it cannot overflow -- cf. the paper's per-block
// buf[i] and ring buffers) plus qarc[n]: the exclusive prefix
// of the appended vertices' degrees.  A packed 64-bit tail (count<<33 | arcs)
// reserves slots and their arc range with one atomic, so a peel sub-round can
// split its ARCS evenly over all warps (hub vertices are shared by many warps;
// no degree buckets needed).
#pragma once

#include "kc_common.cuh"
#include <climits>

namespace kc {

constexpr int kBlock = 512;
constexpr int kWarps = kBlock / 32;
constexpr int kScanItems = 4;
constexpr int kScanTile = kBlock * kScanItems;
constexpr int kStageCap = 256;  // per-warp append stage (>= 32 * kUnroll)
constexpr int kUnroll = 4;      // arcs per lane in flight per peel batch
constexpr int kBatch = 32 * kUnroll;

enum : int32_t { PH_INIT = 0, PH_SCAN = 1, PH_PEEL = 2, PH_SOLO = 3, PH_DONE = 4 };

struct Ctl {
    int32_t phase, k, level, compact;
    int32_t src_sel, dst_sel, solo_block, pad;
    int64_t src_len;
    int64_t s, e, as, ae;  // PEEL/SOLO: slots [s,e), arcs [as,ae)
};

struct alignas(128) State {
    unsigned long long qtail;      // packed (count << 33) | arcs
    unsigned long long alive_out;  // compaction output length
    int32_t min_next;              // atomicMin target for the level skip
    uint32_t bar_count;            // grid barrier arrivals (monotone)
    uint32_t bar_gen;              // grid barrier generation
    int32_t nblocks;
    Ctl ctl[2];                    // published by the leader, indexed by gen & 1
    // leader-private bookkeeping
    int64_t n;
    int64_t lvl_cnt0, lvl_arc0;    // queue tail when the current level's scan began
    int64_t alive_len;
    int32_t alive_sel;             // -1: no alive list yet (scan the identity)
    int32_t solo_arcs;             // peel phases with <= this many arcs go SOLO
    int64_t solo_e, solo_ae;       // progress reported by a SOLO phase
    int64_t solo_sub;              // sub-rounds run by the SOLO phase
    // statistics
    int64_t st_levels, st_subrounds, st_solo_subrounds, st_barriers, st_scanned, st_arcs,
        st_compactions;
    int32_t st_kmax;
    int32_t error;
};

struct KArgs {
    const int64_t *rowptr;
    const int32_t *colidx;
    int32_t *deg;  // == core_out
    int32_t *order;
    int64_t *qarc;
    int32_t *alive[2];
    State *S;
    int64_t n;
};

struct Smem {
    int32_t sv[kWarps][kStageCap];
    int32_t sd[kWarps][kStageCap];
    unsigned long long scan_q[kWarps];
    uint32_t scan_k[kWarps];
    unsigned long long tot_q, base_q;
    unsigned long long tot_k, base_k;
    int32_t red_min[kWarps];
    Ctl ctl;
    uint32_t gen;
    int32_t solo_go;
};

// ---------------------------------------------------------------- helpers
__device__ __forceinline__ int warp_min(int v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(kFull, v, o));
    return v;
}

__device__ __forceinline__ int64_t warp_sum64(int64_t v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

// CTA-wide min, then one atomicMin per CTA
__device__ __forceinline__ void block_min_atomic(Smem &sm, int v, int32_t *target)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    v = warp_min(v);
    if (lane == 0) sm.red_min[wib] = v;
    __syncthreads();
    if (wib == 0) {
        int x = lane < kWarps ? sm.red_min[lane] : INT_MAX;
        x = warp_min(x);
        if (lane == 0 && x != INT_MAX) atomicMin(target, x);
    }
    __syncthreads();
}

// ----------------------------------------------------------- frontier queue
// Per-warp append stage in shared memory; flushed with ONE packed atomic.
__device__ __noinline__ void warp_flush(const KArgs &A, Smem &sm, int wib, int &scnt)
{
    const int lane = threadIdx.x & 31;
    if (scnt == 0) return;
    __syncwarp();
    int64_t tot = 0;
    for (int x = lane; x < scnt; x += 32) tot += sm.sd[wib][x];
    tot = warp_sum64(tot);
    unsigned long long base = 0;
    if (lane == 0)
        base = atomicAdd(&A.S->qtail, ((unsigned long long)scnt << kArcBits) | (unsigned long long)tot);
    base = __shfl_sync(kFull, base, 0);
    const int64_t bc = (int64_t)(base >> kArcBits);
    int64_t carry = (int64_t)(base & kArcMask);
    for (int x0 = 0; x0 < scnt; x0 += 32) {
        const int x = x0 + lane;
        const int64_t d = (x < scnt) ? (int64_t)sm.sd[wib][x] : 0;
        int64_t incl = d;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int64_t t = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += t;
        }
        if (x < scnt) {
            A.order[bc + x] = sm.sv[wib][x];
            A.qarc[bc + x] = carry + incl - d;
        }
        carry += __shfl_sync(kFull, incl, 31);
    }
    __syncwarp();
    scnt = 0;
}

// Ballot compaction (Fig. 8(c)) of this warp's hits into its stage.
__device__ __forceinline__ void warp_append(const KArgs &A, Smem &sm, int wib, int &scnt, bool hit,
                                            int32_t u, int32_t du)
{
    const unsigned b = __ballot_sync(kFull, hit);
    if (b == 0) return;
    const int c = __popc(b);
    if (scnt + c > kStageCap) warp_flush(A, sm, wib, scnt);
    if (hit) {
        const int pos = scnt + __popc(b & lanemask_lt());
        sm.sv[wib][pos] = u;
        sm.sd[wib][pos] = du;
    }
    scnt += c;
    __syncwarp();
}

// ------------------------------------------------------------------ INIT
__device__ void phase_init(const KArgs &A, Smem &sm)
{
    int lmin = INT_MAX;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < A.n; v += stride) {
        const int32_t d = (int32_t)(ld_ro_i64(A.rowptr + v + 1) - ld_ro_i64(A.rowptr + v));
        A.deg[v] = d;
        lmin = min(lmin, d);
    }
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// ------------------------------------------------------------------ SCAN
// Block-wide exclusive scan of (packed frontier count|arcs, kept count).
__device__ __forceinline__ void block_scan2(Smem &sm, unsigned long long q, uint32_t kk,
                                            unsigned long long &q_ex, uint32_t &k_ex)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned long long qi = q;
    uint32_t ki = kk;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned long long t = __shfl_up_sync(kFull, qi, o);
        uint32_t t2 = __shfl_up_sync(kFull, ki, o);
        if (lane >= o) { qi += t; ki += t2; }
    }
    if (lane == 31) { sm.scan_q[wib] = qi; sm.scan_k[wib] = ki; }
    __syncthreads();
    if (wib == 0) {
        unsigned long long wq = lane < kWarps ? sm.scan_q[lane] : 0ULL;
        uint32_t wk = lane < kWarps ? sm.scan_k[lane] : 0u;
        unsigned long long iq = wq;
        uint32_t ik = wk;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long t = __shfl_up_sync(kFull, iq, o);
            uint32_t t2 = __shfl_up_sync(kFull, ik, o);
            if (lane >= o) { iq += t; ik += t2; }
        }
        if (lane < kWarps) { sm.scan_q[lane] = iq - wq; sm.scan_k[lane] = ik - wk; }
        if (lane == kWarps - 1) { sm.tot_q = iq; sm.tot_k = ik; }
    }
    __syncthreads();
    q_ex = sm.scan_q[wib] + (qi - q);
    k_ex = sm.scan_k[wib] + (ki - kk);
}

__device__ void phase_scan(const KArgs &A, const Ctl &c, Smem &sm)
{
    const int k = c.k;
    const int32_t *src = c.src_sel < 0 ? nullptr : A.alive[c.src_sel];
    int32_t *dst = c.compact ? A.alive[c.dst_sel] : nullptr;
    const int64_t len = c.src_len;
    const int64_t ntiles = (len + kScanTile - 1) / kScanTile;
    int lmin = INT_MAX;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
        int32_t vv[kScanItems], dd[kScanItems], fd[kScanItems];
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            const int64_t idx = t * kScanTile + (int64_t)j * kBlock + threadIdx.x;
            vv[j] = -1;
            if (idx < len) vv[j] = src ? ld_cg_i32(src + idx) : (int32_t)idx;
        }
#pragma unroll
        for (int j = 0; j < kScanItems; j++) dd[j] = vv[j] >= 0 ? ld_cg_i32(A.deg + vv[j]) : -1;
        unsigned long long q = 0;
        uint32_t keep = 0, fmask = 0, kmask = 0;
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            fd[j] = 0;
            if (vv[j] < 0) continue;
            if (dd[j] == k) {
                fmask |= 1u << j;
                fd[j] = (int32_t)(ld_ro_i64(A.rowptr + vv[j] + 1) - ld_ro_i64(A.rowptr + vv[j]));
                q += kCntOne | (unsigned long long)fd[j];
            } else if (dd[j] > k) {
                lmin = min(lmin, dd[j]);
                if (dst) { kmask |= 1u << j; keep++; }
            }
        }
        unsigned long long q_ex;
        uint32_t k_ex;
        block_scan2(sm, q, keep, q_ex, k_ex);
        if (threadIdx.x == 0) {
            sm.base_q = sm.tot_q ? atomicAdd(&A.S->qtail, sm.tot_q) : 0ULL;
            sm.base_k = sm.tot_k ? atomicAdd(&A.S->alive_out, sm.tot_k) : 0ULL;
        }
        __syncthreads();
        int64_t slot = (int64_t)((sm.base_q + q_ex) >> kArcBits);
        int64_t arc = (int64_t)(((sm.base_q & kArcMask) + (q_ex & kArcMask)));
        int64_t kpos = (int64_t)(sm.base_k + k_ex);
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            if (fmask & (1u << j)) {
                A.order[slot] = vv[j];
                A.qarc[slot] = arc;
                slot++;
                arc += fd[j];
            }
            if (kmask & (1u << j)) dst[kpos++] = vv[j];
        }
    }
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// ------------------------------------------------------------------ PEEL
// Largest slot i in [s,e) with qarc[i] <= a (warp-cooperative 32-ary search).
__device__ __forceinline__ int64_t find_slot(const int64_t *qarc, int64_t s, int64_t e, int64_t a)
{
    const int lane = threadIdx.x & 31;
    int64_t lo = s, hi = e;
    while (hi - lo > 32) {
        const int64_t step = (hi - lo + 31) / 32;
        const int64_t p = lo + lane * step;
        const bool ok = (p < hi) && (ld_cg_i64(qarc + p) <= a);
        const unsigned b = __ballot_sync(kFull, ok);
        const int L = 31 - __clz(b);
        lo = lo + L * step;
        hi = min(hi, lo + step);
    }
    const int64_t p = lo + lane;
    const bool ok = (p < hi) && (ld_cg_i64(qarc + p) <= a);
    const unsigned b = __ballot_sync(kFull, ok);
    return lo + (31 - __clz(b));
}

// Walk arcs [a0,a1) of the frontier [s,e) (arc range [as,ae)) with one warp.
__device__ __forceinline__ void peel_range(const KArgs &A, Smem &sm, const int k, int64_t s,
                                           int64_t e, int64_t ae, int64_t a0, int64_t a1,
                                           int &scnt, int &lmin)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int64_t i = find_slot(A.qarc, s, e, a0);
    int64_t a = a0;
    while (a < a1) {
        // window: slots i .. i+31, one per lane
        const int64_t j = i + lane;
        int64_t wq = LLONG_MAX, nxt;
        if (j < e) wq = ld_cg_i64(A.qarc + j);
        nxt = __shfl_down_sync(kFull, wq, 1);
        if (lane == 31) nxt = (j + 1 < e) ? ld_cg_i64(A.qarc + j + 1) : ae;
        if (j + 1 >= e) nxt = ae;
        int64_t wbeg = 0;
        if (j < e && nxt > wq && nxt > a && wq < a1) {
            const int32_t v = ld_cg_i32(A.order + j);
            wbeg = ld_ro_i64(A.rowptr + v);
        }
        const int64_t limit = min(a1, __shfl_sync(kFull, nxt, 31));
        while (a < limit) {
            int32_t u[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                const int64_t my = a + r * 32 + lane;
                u[r] = -1;
                // slot of arc `my`: highest lane whose window start is <= my
                int pos = 0;
#pragma unroll
                for (int bstep = 16; bstep >= 1; bstep >>= 1) {
                    const int64_t q = __shfl_sync(kFull, wq, pos + bstep);
                    if (q <= my) pos += bstep;
                }
                const int64_t beg = __shfl_sync(kFull, wbeg, pos);
                const int64_t base = __shfl_sync(kFull, wq, pos);
                if (my < limit) u[r] = ld_stream_i32(A.colidx + beg + (my - base));
            }
            int32_t d[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) d[r] = u[r] >= 0 ? ld_cg_i32(A.deg + u[r]) : -1;
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                bool hit = false;
                int32_t du = 0;
                if (d[r] > k) {
                    const int old = atomicSub(A.deg + u[r], 1);
                    if (old == k + 1) {
                        hit = true;
                        du = (int32_t)(ld_ro_i64(A.rowptr + u[r] + 1) - ld_ro_i64(A.rowptr + u[r]));
                    } else if (old <= k) {
                        atomicAdd(A.deg + u[r], 1);
                    } else {
                        lmin = min(lmin, old - 1);
                    }
                }
                warp_append(A, sm, wib, scnt, hit, u[r], du);
            }
            a += kBatch;
        }
        a = limit;
        i += 32;
    }
}

__device__ void phase_peel(const KArgs &A, const Ctl &c, Smem &sm)
{
    const int wib = threadIdx.x >> 5;
    const int64_t gw = (int64_t)blockIdx.x * kWarps + wib;
    const int64_t W = (int64_t)gridDim.x * kWarps;
    const int64_t T = c.ae - c.as;
    int64_t C = (T + W - 1) / W;
    C = ((C + kBatch - 1) / kBatch) * kBatch;
    int scnt = 0, lmin = INT_MAX;
    const int64_t a0 = c.as + gw * C;
    if (a0 < c.ae) peel_range(A, sm, c.k, c.s, c.e, c.ae, a0, min(a0 + C, c.ae), scnt, lmin);
    warp_flush(A, sm, wib, scnt);
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// SOLO: this CTA alone runs sub-rounds starting at [s,e) until the frontier
// is empty or grows past the solo threshold; reports progress in the State.
__device__ void phase_solo(const KArgs &A, const Ctl &c, Smem &sm)
{
    const int wib = threadIdx.x >> 5;
    int64_t s = c.s, e = c.e, as = c.as, ae = c.ae, sub = 0;
    int lmin = INT_MAX;
    while (true) {
        const int64_t T = ae - as;
        int64_t C = (T + kWarps - 1) / kWarps;
        C = ((C + kBatch - 1) / kBatch) * kBatch;
        int scnt = 0;
        const int64_t a0 = as + (int64_t)wib * C;
        if (a0 < ae) peel_range(A, sm, c.k, s, e, ae, a0, min(a0 + C, ae), scnt, lmin);
        warp_flush(A, sm, wib, scnt);
        sub++;
        __threadfence();
        __syncthreads();
        if (threadIdx.x == 0) sm.base_q = ld_relaxed_u64(&A.S->qtail);
        __syncthreads();
        const unsigned long long qt = sm.base_q;
        const int64_t cnt = (int64_t)(qt >> kArcBits), arcs = (int64_t)(qt & kArcMask);
        __syncthreads();
        s = e; as = ae; e = cnt; ae = arcs;
        if (e == s || ae == as || (ae - as) > (int64_t)A.S->solo_arcs) break;
    }
    block_min_atomic(sm, lmin, &A.S->min_next);
    if (threadIdx.x == 0) {
        volatile State *S = A.S;
        S->solo_e = s;   // first slot NOT yet peeled
        S->solo_ae = as;
        S->solo_sub = sub;
    }
}

// ---------------------------------------------------------------- control
// Runs on ONE thread (the last CTA to arrive at a barrier) while every other
// CTA waits: reads the counters and publishes the next phase in ctl[(gen+1)&1].
__device__ __noinline__ void leader_step(const KArgs &A, uint32_t gen)
{
    volatile State *S = A.S;
    Ctl cur;
    {
        volatile Ctl *pc = &S->ctl[gen & 1];
        cur.phase = pc->phase; cur.k = pc->k; cur.level = pc->level; cur.compact = pc->compact;
        cur.src_sel = pc->src_sel; cur.dst_sel = pc->dst_sel; cur.solo_block = pc->solo_block;
        cur.pad = 0; cur.src_len = pc->src_len;
        cur.s = pc->s; cur.e = pc->e; cur.as = pc->as; cur.ae = pc->ae;
    }
    Ctl nx = cur;
    const unsigned long long qt = ld_relaxed_u64(&A.S->qtail);
    const int64_t cnt = (int64_t)(qt >> kArcBits), arcs = (int64_t)(qt & kArcMask);
    const int64_t n = S->n;
    S->st_barriers = S->st_barriers + 1;

    bool level_end = false;
    int64_t ps = 0, pe = 0, pas = 0, pae = 0;  // next peel frontier, if any
    bool peel = false;
    switch (cur.phase) {
    case PH_INIT: {
        const int k0 = ld_relaxed_i32(&A.S->min_next);
        S->min_next = INT_MAX;
        nx.level = -1;
        nx.k = (k0 == INT_MAX) ? 0 : k0;
        break;
    }
    case PH_SCAN: {
        if (cur.compact) {
            S->alive_sel = cur.dst_sel;
            S->alive_len = (int64_t)ld_relaxed_u64(&A.S->alive_out);
            S->st_compactions = S->st_compactions + 1;
        }
        S->st_scanned = S->st_scanned + cur.src_len;
        const int64_t c0 = S->lvl_cnt0, a0 = S->lvl_arc0;
        if (arcs > a0) { peel = true; ps = c0; pe = cnt; pas = a0; pae = arcs; }
        else level_end = true;
        break;
    }
    case PH_PEEL: {
        S->st_subrounds = S->st_subrounds + 1;
        S->st_arcs = S->st_arcs + (cur.ae - cur.as);
        if (cnt > cur.e && arcs > cur.ae) { peel = true; ps = cur.e; pe = cnt; pas = cur.ae; pae = arcs; }
        else level_end = true;
        break;
    }
    case PH_SOLO: {
        S->st_subrounds = S->st_subrounds + S->solo_sub;
        S->st_solo_subrounds = S->st_solo_subrounds + S->solo_sub;
        S->st_arcs = S->st_arcs + (S->solo_ae - cur.as);
        const int64_t se = S->solo_e, sae = S->solo_ae;
        if (cnt > se && arcs > sae) { peel = true; ps = se; pe = cnt; pas = sae; pae = arcs; }
        else level_end = true;
        break;
    }
    default: break;
    }

    int next_k = nx.k;
    bool start_scan = (cur.phase == PH_INIT);
    if (level_end) {
        S->st_levels = S->st_levels + 1;
        S->st_kmax = cur.k;
        if (cnt >= n) {
            nx.phase = PH_DONE;
        } else {
            const int mn = ld_relaxed_i32(&A.S->min_next);
            S->min_next = INT_MAX;
            next_k = max(cur.k + 1, mn);
            start_scan = true;
        }
    }
    if (peel) {
        const bool solo = S->solo_arcs > 0 && (pae - pas) <= (int64_t)S->solo_arcs;
        nx.phase = solo ? PH_SOLO : PH_PEEL;
        nx.solo_block = -1;
        nx.s = ps; nx.e = pe; nx.as = pas; nx.ae = pae;
    } else if (start_scan) {
        const int64_t live = n - cnt;
        const int src_sel = S->alive_sel;
        const int64_t src_len = src_sel < 0 ? n : S->alive_len;
        const bool compact = src_sel < 0 ? (live * 4 < n) : (live * 2 < src_len);
        nx.phase = PH_SCAN;
        nx.k = next_k;
        nx.level = nx.level + 1;
        nx.src_sel = src_sel;
        nx.src_len = src_len;
        nx.compact = compact ? 1 : 0;
        nx.dst_sel = src_sel < 0 ? 0 : 1 - src_sel;
        if (compact) S->alive_out = 0;
        S->lvl_cnt0 = cnt;
        S->lvl_arc0 = arcs;
    }
    volatile Ctl *pn = &S->ctl[(gen + 1) & 1];
    pn->phase = nx.phase; pn->k = nx.k; pn->level = nx.level; pn->compact = nx.compact;
    pn->src_sel = nx.src_sel; pn->dst_sel = nx.dst_sel; pn->solo_block = nx.solo_block;
    pn->src_len = nx.src_len; pn->s = nx.s; pn->e = nx.e; pn->as = nx.as; pn->ae = nx.ae;
}

// Grid barrier; the last arriver runs leader_step before releasing.  Copies
// the published Ctl into shared memory.  Returns whether this CTA was leader.
__device__ __forceinline__ bool grid_sync(const KArgs &A, Smem &sm)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        State *S = A.S;
        const uint32_t gen = ld_acquire_u32(&S->bar_gen);
        __threadfence();
        const uint32_t t = atom_add_release_u32(&S->bar_count, 1u);
        const bool last = (t + 1u) == (uint32_t)gridDim.x * (gen + 1u);
        if (last) {
            __threadfence();
            leader_step(A, gen);
            __threadfence();
            st_release_u32(&S->bar_gen, gen + 1u);
        } else {
            while (ld_acquire_u32(&S->bar_gen) == gen) {
            }
        }
        volatile Ctl *pc = &S->ctl[(gen + 1u) & 1u];
        sm.ctl.phase = pc->phase; sm.ctl.k = pc->k; sm.ctl.level = pc->level;
        sm.ctl.compact = pc->compact; sm.ctl.src_sel = pc->src_sel; sm.ctl.dst_sel = pc->dst_sel;
        sm.ctl.solo_block = pc->solo_block; sm.ctl.src_len = pc->src_len;
        sm.ctl.s = pc->s; sm.ctl.e = pc->e; sm.ctl.as = pc->as; sm.ctl.ae = pc->ae;
        sm.gen = gen + 1u;
        sm.solo_go = last;
    }
    __syncthreads();
    return sm.solo_go != 0;
}

__global__ void __launch_bounds__(kBlock, 2) k_persistent(KArgs A)
{
    __shared__ Smem sm;
    phase_init(A, sm);
    bool leader = grid_sync(A, sm);
    while (true) {
        const Ctl c = sm.ctl;
        if (c.phase == PH_DONE) break;
        if (c.phase == PH_SCAN) phase_scan(A, c, sm);
        else if (c.phase == PH_PEEL) phase_peel(A, c, sm);
        else if (c.phase == PH_SOLO) { if (leader) phase_solo(A, c, sm); }
        leader = grid_sync(A, sm);
    }
}

// -------------------------------------------- host-driven ablation kernels
// (KCORE_ALGO_HOSTLOOP: paper Alg. 1 structure, one launch per phase plus a
// host read-back of the phase.)
__global__ void __launch_bounds__(kBlock, 2) k_phase(KArgs A)
{
    __shared__ Smem sm;
    if (threadIdx.x == 0) {
        volatile State *S = A.S;
        volatile Ctl *pc = &S->ctl[S->bar_gen & 1u];
        sm.ctl.phase = pc->phase; sm.ctl.k = pc->k; sm.ctl.level = pc->level;
        sm.ctl.compact = pc->compact; sm.ctl.src_sel = pc->src_sel; sm.ctl.dst_sel = pc->dst_sel;
        sm.ctl.solo_block = pc->solo_block; sm.ctl.src_len = pc->src_len;
        sm.ctl.s = pc->s; sm.ctl.e = pc->e; sm.ctl.as = pc->as; sm.ctl.ae = pc->ae;
    }
    __syncthreads();
    const Ctl c = sm.ctl;
    if (c.phase == PH_INIT) phase_init(A, sm);
    else if (c.phase == PH_SCAN) phase_scan(A, c, sm);
    else if (c.phase == PH_PEEL) phase_peel(A, c, sm);
    else if (c.phase == PH_SOLO) { if (blockIdx.x == 0) phase_solo(A, c, sm); }
}

__global__ void k_leader(KArgs A, int32_t *phase_out)
{
    State *S = A.S;
    const uint32_t gen = S->bar_gen;
    leader_step(A, gen);
    S->bar_gen = gen + 1u;
    *phase_out = S->ctl[(gen + 1u) & 1u].phase;
}

__global__ void k_init_state(State *S, int64_t n, int32_t solo_arcs, int32_t nblocks)
{
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        State z = {};
        z.min_next = INT_MAX;
        z.nblocks = nblocks;
        z.ctl[0].phase = PH_INIT;
        z.ctl[1].phase = PH_INIT;
        z.n = n;
        z.alive_sel = -1;
        z.solo_arcs = solo_arcs;
        *S = z;
    }
}

} // namespace kc
