// kc_kernels.cuh -- sm_100a kernels of the k-core hot path.
//
// One call = one persistent cooperative kernel (k_persistent) that runs the
// whole decomposition as a device-resident state machine:
//
//   INIT   deg[v] = rowptr[v+1]-rowptr[v] into core_out, min-degree reduce    (Alg.1 l.1)
//   SCAN   level k: frontier <- {v alive : deg[v] == k}; fused min{deg > k};   (Alg.2)
//          optional alive-list compaction (reading R6)
//   PEEL   sub-round over frontier slots [s,e): for every arc (v,u):          (Alg.3 l.12-24)
//          if deg[u] > k: old = atomicSub(&deg[u],1);
//             old == k+1 -> append u (it reached k: next sub-round)
//             old <= k   -> atomicAdd(&deg[u],1)  (restore, Fig. 6)
//             else       -> min_next = min(min_next, old-1)   (level skip, reading R5)
//   level end: k <- max(k+1, min_next)  (Alg.1 l.9 does k+1; reading R5)
//
// Control.  Every CTA keeps an identical copy of the control state (Ctrl) in
// shared memory.  A phase ends with a grid barrier whose last arriver takes a
// SNAPSHOT of the three counters (queue tail, compaction length, min) and
// resets them; every CTA then advances its Ctrl with the same pure function
// advance(Ctrl, Snap).  No host round-trip, no serial "leader" logic.
// Phases whose work is tiny (a few thousand arcs, or a short alive list) are
// marked `solo`: CTA 0 runs them -- and every following tiny phase, across
// sub-rounds and levels -- alone with __syncthreads instead of grid barriers,
// then publishes its Ctrl; the other CTAs wait at one barrier.
//
// Frontier queue: one array order[n] (every vertex is appended exactly once in
// the whole run, so it cannot overflow -- cf. the paper's per-block buf[i] and
// ring buffers) plus qarc[n], the exclusive prefix of the
// appended vertices' degrees.  A packed 64-bit tail (count<<33 | arcs)
// reserves slots and their arc range with one atomic, so a peel sub-round
// splits its ARCS evenly over all warps (hubs are shared by many warps; no
// degree buckets needed).
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
constexpr int kTraceFields = 8;

enum : int32_t { PH_INIT = 0, PH_SCAN = 1, PH_PEEL = 2, PH_DONE = 3 };

// Control state; replicated in every CTA, advanced by advance().
struct Ctrl {
    int32_t phase, solo, k, level_min;
    int32_t compact, src_sel, dst_sel, alive_sel;
    int64_t src_len, alive_len;
    int64_t s, e, as, ae;         // PEEL: slots [s,e), arcs [as,ae)
    int64_t lvl_cnt0, lvl_arc0;   // queue tail when the level's scan began
    int64_t st_levels, st_sub, st_solo_sub, st_bar, st_scanned, st_arcs, st_compact;
    int32_t st_kmax, st_pad;
};

struct Snap {
    unsigned long long qtail, alive_out;
    int32_t min;
    int32_t pad;
};

struct Params {
    int64_t n;
    int32_t solo_arcs;  // PEEL phases with <= this many arcs run solo
    int32_t solo_scan;  // SCAN phases over <= this many entries run solo
};

struct State {
    alignas(128) unsigned long long qtail;      // packed (count << 33) | arcs
    alignas(128) unsigned long long alive_out;  // compaction output length
    alignas(128) int32_t min_next;              // atomicMin target
    alignas(128) uint32_t bar_count;            // grid barrier arrivals (monotone)
    alignas(128) uint32_t bar_gen;              // grid barrier generation
    Snap snap[2];                               // counters at barrier gen, by gen & 1
    alignas(128) Ctrl pub;                      // Ctrl published by CTA 0 after a solo run
    alignas(128) Params prm;
    int64_t *trace;                             // optional [trace_cap][kTraceFields]
    int64_t trace_cap;
    unsigned long long trace_n;
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
    Ctrl ctrl;
    Snap snap;
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

__device__ __forceinline__ unsigned long long globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
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

__device__ void phase_scan(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk)
{
    const int k = c.k;
    const int32_t *src = c.src_sel < 0 ? nullptr : A.alive[c.src_sel];
    int32_t *dst = c.compact ? A.alive[c.dst_sel] : nullptr;
    const int64_t len = c.src_len;
    const int64_t ntiles = (len + kScanTile - 1) / kScanTile;
    int lmin = INT_MAX;
    for (int64_t t = bid; t < ntiles; t += nblk) {
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

// Walk arcs [a0,a1) of the frontier [s,e) (arc range [.,ae)) with one warp.
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

__device__ void phase_peel(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk)
{
    const int wib = threadIdx.x >> 5;
    const int64_t gw = (int64_t)bid * kWarps + wib;
    const int64_t W = (int64_t)nblk * kWarps;
    const int64_t T = c.ae - c.as;
    int64_t C = (T + W - 1) / W;
    C = ((C + kBatch - 1) / kBatch) * kBatch;
    int scnt = 0, lmin = INT_MAX;
    const int64_t a0 = c.as + gw * C;
    if (a0 < c.ae) peel_range(A, sm, c.k, c.s, c.e, c.ae, a0, min(a0 + C, c.ae), scnt, lmin);
    warp_flush(A, sm, wib, scnt);
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// ---------------------------------------------------------------- control
// The pure transition function (Alg.1 l.5-9, Alg.3 l.5 and the level skip).
// Every CTA applies it to identical inputs, so all copies stay identical.
__device__ __noinline__ void advance(Ctrl &c, const Snap &sn, const Params &p)
{
    const int64_t cnt = (int64_t)(sn.qtail >> kArcBits), arcs = (int64_t)(sn.qtail & kArcMask);
    c.level_min = min(c.level_min, sn.min);
    bool level_end = false, peel = false;
    int64_t ps = 0, pe = 0, pas = 0, pae = 0;
    int next_k = 0;
    if (c.phase == PH_INIT) {
        next_k = (c.level_min == INT_MAX) ? 0 : c.level_min;
        c.level_min = INT_MAX;
    } else if (c.phase == PH_SCAN) {
        c.st_scanned += c.src_len;
        if (c.compact) {
            c.alive_sel = c.dst_sel;
            c.alive_len = (int64_t)sn.alive_out;
            c.st_compact++;
        }
        if (arcs > c.lvl_arc0) { peel = true; ps = c.lvl_cnt0; pe = cnt; pas = c.lvl_arc0; pae = arcs; }
        else level_end = true;
    } else if (c.phase == PH_PEEL) {
        c.st_sub++;
        if (c.solo) c.st_solo_sub++;
        c.st_arcs += c.ae - c.as;
        if (cnt > c.e && arcs > c.ae) { peel = true; ps = c.e; pe = cnt; pas = c.ae; pae = arcs; }
        else level_end = true;
    }
    bool scan = (c.phase == PH_INIT);
    if (level_end) {
        if (cnt > c.lvl_cnt0) { c.st_levels++; c.st_kmax = c.k; }
        if (cnt >= p.n) {
            c.phase = PH_DONE;
            c.solo = 0;
        } else {
            next_k = max(c.k + 1, c.level_min);
            c.level_min = INT_MAX;
            scan = true;
        }
    }
    if (peel) {
        c.phase = PH_PEEL;
        c.solo = (pae - pas) <= (int64_t)p.solo_arcs;
        c.s = ps; c.e = pe; c.as = pas; c.ae = pae;
    } else if (scan) {
        const int64_t live = p.n - cnt;
        const int64_t src_len = c.alive_sel < 0 ? p.n : c.alive_len;
        const bool compact = c.alive_sel < 0 ? (live * 4 < p.n) : (live * 2 < src_len);
        c.phase = PH_SCAN;
        c.k = next_k;
        c.src_sel = c.alive_sel;
        c.src_len = src_len;
        c.compact = compact ? 1 : 0;
        c.dst_sel = c.alive_sel < 0 ? 0 : 1 - c.alive_sel;
        c.solo = src_len <= (int64_t)p.solo_scan;
        c.lvl_cnt0 = cnt;
        c.lvl_arc0 = arcs;
    }
}

// Snapshot + reset of the counters (caller guarantees nobody else touches them).
__device__ __forceinline__ Snap take_snapshot(State *S)
{
    Snap sn;
    sn.qtail = ld_relaxed_u64(&S->qtail);
    sn.alive_out = ld_relaxed_u64(&S->alive_out);
    sn.min = ld_relaxed_i32(&S->min_next);
    sn.pad = 0;
    S->alive_out = 0ULL;
    S->min_next = INT_MAX;
    return sn;
}

__device__ __forceinline__ void trace_rec(State *S, const Ctrl &c, const Snap &sn, int grid)
{
    if (!S->trace) return;
    const unsigned long long i = S->trace_n;
    if ((int64_t)i >= S->trace_cap) return;
    int64_t *r = S->trace + i * kTraceFields;
    r[0] = (int64_t)globaltimer();
    r[1] = (int64_t)clock64();
    r[2] = ((int64_t)c.phase << 8) | ((int64_t)c.solo << 4) | grid;  // phase that ENDED
    r[3] = c.k;
    r[4] = c.phase == PH_SCAN ? c.src_len : (c.e - c.s);
    r[5] = c.phase == PH_PEEL ? (c.ae - c.as) : 0;
    r[6] = (int64_t)(sn.qtail >> kArcBits);
    r[7] = 0;
    S->trace_n = i + 1;
}

// Grid barrier; the last arriver snapshots+resets the counters.  Leaves the
// snapshot in sm.snap (thread 0 only is guaranteed to see it before the final
// __syncthreads; all threads after).
__device__ __forceinline__ void grid_barrier(const KArgs &A, Smem &sm)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        State *S = A.S;
        const uint32_t gen = ld_acquire_u32(&S->bar_gen);
        __threadfence();
        const uint32_t t = atom_add_release_u32(&S->bar_count, 1u);
        Snap sn;
        if ((t + 1u) == (uint32_t)gridDim.x * (gen + 1u)) {
            __threadfence();
            sn = take_snapshot(S);
            S->snap[(gen + 1u) & 1u] = sn;
            st_release_u32(&S->bar_gen, gen + 1u);
        } else {
            while (ld_acquire_u32(&S->bar_gen) == gen) {
            }
            const Snap *ps = &S->snap[(gen + 1u) & 1u];
            sn.qtail = ld_relaxed_u64(&ps->qtail);
            sn.alive_out = ld_relaxed_u64(&ps->alive_out);
            sn.min = ld_relaxed_i32(&ps->min);
            sn.pad = 0;
        }
        sm.snap = sn;
    }
    __syncthreads();
}

__device__ __forceinline__ void run_phase(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk)
{
    if (c.phase == PH_SCAN) phase_scan(A, c, sm, bid, nblk);
    else if (c.phase == PH_PEEL) phase_peel(A, c, sm, bid, nblk);
}

// CTA 0 alone: run consecutive solo phases with CTA-local synchronisation.
__device__ void solo_run(const KArgs &A, Smem &sm, const Params &p)
{
    State *S = A.S;
    while (true) {
        const Ctrl c = sm.ctrl;
        run_phase(A, c, sm, 0, 1);  // ends with __syncthreads (block_min_atomic)
        if (threadIdx.x == 0) {
            __threadfence();
            const Snap sn = take_snapshot(S);
            trace_rec(S, sm.ctrl, sn, 0);
            advance(sm.ctrl, sn, p);
        }
        __syncthreads();
        if (sm.ctrl.phase == PH_DONE || !sm.ctrl.solo) break;
    }
    if (threadIdx.x == 0) {
        S->pub = sm.ctrl;
        __threadfence();
    }
}

__global__ void __launch_bounds__(kBlock, 2) k_persistent(KArgs A)
{
    __shared__ Smem sm;
    State *S = A.S;
    const Params p = S->prm;
    if (threadIdx.x == 0) {
        Ctrl z = {};
        z.phase = PH_INIT;
        z.level_min = INT_MAX;
        z.alive_sel = -1;
        z.src_sel = -1;
        sm.ctrl = z;
    }
    phase_init(A, sm);
    grid_barrier(A, sm);
    if (threadIdx.x == 0) advance(sm.ctrl, sm.snap, p);
    __syncthreads();
    while (true) {
        if (sm.ctrl.phase == PH_DONE) break;
        if (sm.ctrl.solo) {
            if (blockIdx.x == 0) solo_run(A, sm, p);
            grid_barrier(A, sm);
            if (threadIdx.x == 0) {
                const Ctrl *pc = &S->pub;
                Ctrl c;
                // plain loads are safe: written before CTA 0's release-arrive,
                // read after this CTA's acquire; bypass L1 with ld.cg
                const int4 *src = reinterpret_cast<const int4 *>(pc);
                int4 *dst = reinterpret_cast<int4 *>(&c);
#pragma unroll
                for (int w = 0; w < (int)(sizeof(Ctrl) / sizeof(int4)); w++) dst[w] = __ldcg(src + w);
                c.st_bar++;
                sm.ctrl = c;
            }
        } else {
            const Ctrl c = sm.ctrl;
            run_phase(A, c, sm, blockIdx.x, gridDim.x);
            grid_barrier(A, sm);
            if (threadIdx.x == 0) {
                if (blockIdx.x == 0) trace_rec(S, sm.ctrl, sm.snap, 1);
                sm.ctrl.st_bar++;
                advance(sm.ctrl, sm.snap, p);
            }
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) S->pub = sm.ctrl;  // final statistics
}

// -------------------------------------------- host-driven ablation kernels
// (KCORE_ALGO_HOSTLOOP: the paper's Alg. 1 structure -- one launch per phase
// and a host read-back of the phase after each.  No solo phases.)
__global__ void __launch_bounds__(kBlock, 2) k_phase(KArgs A)
{
    __shared__ Smem sm;
    if (threadIdx.x == 0) sm.ctrl = A.S->pub;
    __syncthreads();
    const Ctrl c = sm.ctrl;
    if (c.phase == PH_INIT) phase_init(A, sm);
    else run_phase(A, c, sm, blockIdx.x, gridDim.x);
}

__global__ void k_leader(KArgs A, int32_t *phase_out)
{
    State *S = A.S;
    const Params p = S->prm;
    Ctrl c = S->pub;
    const Snap sn = take_snapshot(S);
    trace_rec(S, c, sn, 1);
    c.st_bar++;
    advance(c, sn, p);
    S->pub = c;
    *phase_out = c.phase;
}

__global__ void k_init_state(State *S, int64_t n, int32_t solo_arcs, int32_t solo_scan,
                             int64_t *trace, int64_t trace_cap)
{
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        S->qtail = 0ULL;
        S->alive_out = 0ULL;
        S->min_next = INT_MAX;
        S->bar_count = 0u;
        S->bar_gen = 0u;
        Ctrl z = {};
        z.phase = PH_INIT;
        z.level_min = INT_MAX;
        z.alive_sel = -1;
        z.src_sel = -1;
        S->pub = z;
        S->prm.n = n;
        S->prm.solo_arcs = solo_arcs;
        S->prm.solo_scan = solo_scan;
        S->trace = trace;
        S->trace_cap = trace ? trace_cap : 0;
        S->trace_n = 0ULL;
    }
}

} // namespace kc
