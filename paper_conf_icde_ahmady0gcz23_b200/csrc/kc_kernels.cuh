// kc_kernels.cuh -- sm_100a kernels of the k-core hot path (v5).
//
// One call = one persistent cooperative kernel (k_persistent), one CTA per SM,
// running the whole decomposition as a device-resident state machine.  Per
// level k (Alg. 1's round) there is ONE grid phase and one grid
// barrier:
//
//   scan   every CTA scans its segment of the alive list (Alg. 2):
//          deg[v] == k -> v is in the k-shell: claim it, append it to the
//                         CTA's LOCAL frontier (shared memory) or, if it is
//                         big or the frontier is full, to the global POOL;
//          deg[v] >  k -> running min for the level skip; alive-list compaction.
//   drain  the CTA drains its local frontier breadth-first with CTA-local
//          sub-rounds (__syncthreads only) -- the paper's block-local BFS of
//          Alg. 3.  For every arc (v,u) (Alg. 3 l.19-24):
//            if deg[u] > k: old = atomicSub(&deg[u],1)
//               old == k+1 -> u reached k: claim, append to the next local
//                             frontier (or the pool)
//               old <= k   -> atomicAdd(&deg[u],1)  (restore, Fig. 6)
//               else       -> min_next = min(min_next, old-1)          (level skip)
//   pool   vertices too big for a CTA-local sub-round, or overflowing it, go
//          to a global pool (one packed atomic reserves entries and their
//          range in the pool's ARC space).  A CTA with no local work claims a
//          range of pool arcs (CAS, never past the reserved arcs) and walks it
//          with all its warps, arc-balanced (hubs are shared by many CTAs),
//          then drains the local frontier that produced -- asynchronous work
//          sharing, no sub-round barrier.  The level ends when every CTA has
//          finished its scan and the pool's done arcs equal its reserved arcs.
//   level end: k <- max(k+1, min_next)  (Alg. 1 l.9 does k+1; reading R5)
//
// Scans and drains of one level run concurrently in different CTAs, so a
// vertex can be seen with deg == k by a scan and reached (old == k+1) by a
// peel; a claim bit per vertex (atomicOr) makes removal exactly-once
// (reading R9).
//
// Control: every CTA keeps an identical copy of the control state in shared
// memory; a phase ends with a grid barrier whose last arriver snapshots and
// resets the counters, and every CTA applies the same pure advance().  Levels
// over a short alive list run `solo` on CTA 0 with CTA-local sync only.
//
// Filter: a CTA that walks many arcs in a level whose alive list is short
// builds a Bloom filter of that list in shared memory; arcs whose target is
// definitely not alive skip the scattered deg[] read.
#pragma once

#include "kc_common.cuh"
#include <climits>

namespace kc {

constexpr int kBlock = 768;
constexpr int kWarps = kBlock / 32;
constexpr int kScanItems = 8;        // alive-list entries per lane per warp step
constexpr int kLCap = kBlock;        // local frontier capacity (one entry per thread in the prefix)
constexpr int kSub = 8192;           // arc budget of one CTA-local sub-round
constexpr int kPStage = 64;          // per-warp pool stage (vertices)
constexpr int kClaimMin = 4096;      // pool ARCS claimed at a time: backlog / (2 grid),
constexpr int kClaimMax = 1 << 19;   //   clamped to [kClaimMin, kClaimMax]
constexpr int kMaxLocalRounds = 4;   // then the local frontier goes back to the pool
constexpr int kSoloBail = 16384;     // a solo level with more pending pool arcs goes grid-wide
constexpr int kBloomBits = 1 << 20;  // 128 KB
constexpr int kBloomWords = kBloomBits / 32;
constexpr int kBloomMaxA = 1 << 18;  // build only for alive lists up to this length
constexpr int kUnroll = 4;           // arcs per lane in flight per batch (handle_hits assumes 4)
constexpr int kBatch = 32 * kUnroll;
constexpr int kTraceFields = 8;

enum : int32_t { PH_INIT = 0, PH_LEVEL = 1, PH_DONE = 3 };

struct Ctrl {
    int32_t phase, solo, k, level_min;
    int32_t compact, src_sel, dst_sel, alive_sel;
    int32_t src_single, alive_single;  // 1: the list is one contiguous run in segment 0
    int32_t cont;                      // 1: the level's scan is done, only the pool is left
    int32_t pad1;
    int64_t src_len, alive_len;
    int64_t scan_target;               // scans_done value that ends the current level
    int64_t ord_lvl0;                  // removed count when the level began
    int64_t level;                     // level index (for the Bloom cache)
    int64_t st_levels, st_phases, st_solo, st_bar, st_scanned, st_compact, st_pool;
    int32_t st_kmax, st_pad;
    int64_t alive_carry;               // compaction output already counted (solo bail-out)
};

static_assert(sizeof(Ctrl) % 16 == 0, "Ctrl is copied as int4");

struct Snap {
    unsigned long long ord;        // removed vertices
    unsigned long long alive_out;  // compaction output length
    unsigned long long pool;       // pool entries so far
    int32_t min;
    int32_t pad;
};

struct Params {
    int64_t n;
    int32_t solo_arcs;  // unused (kept for the options ABI)
    int32_t solo_scan;  // levels over <= this many alive entries run solo
    int32_t bloom;      // 0 disables the Bloom filter
    int32_t pad;
};

struct State {
    alignas(128) unsigned long long ord_tail;   // removed vertices (order slots if recorded)
    alignas(128) unsigned long long alive_out;  // compaction output length
    alignas(128) int32_t min_next;              // atomicMin target
    alignas(128) unsigned long long pool_tail;  // packed (entries << 33) | arcs reserved
    alignas(128) unsigned long long pool_claim; // pool arcs claimed
    alignas(128) unsigned long long pool_done;  // pool arcs fully processed
    alignas(128) unsigned long long scans_done; // CTA scans finished (monotone)
    alignas(128) uint32_t bar_count;            // grid barrier arrivals (monotone)
    alignas(128) uint32_t bar_gen;              // grid barrier generation
    Snap snap[2];                               // counters at barrier gen, by gen & 1
    alignas(128) unsigned long long arcs_walked;
    alignas(128) Ctrl pub;                      // Ctrl published by CTA 0 after a solo run
    alignas(128) Params prm;
    int64_t *trace;                             // optional [trace_cap][kTraceFields]
    int64_t *trace_cta;                         // optional [trace_cap][grid][4]
    int64_t trace_cap;
    unsigned long long trace_n;
};

struct KArgs {
    const int64_t *rowptr;
    const int32_t *colidx;
    int32_t *deg;         // == core_out
    int32_t *order;       // removal order, or nullptr when not requested
    uint32_t *claimed;    // claim bit per vertex
    int32_t *pool_v;      // pool entry j: vertex,
    int64_t *pool_beg;    //   its first arc in colidx,
    int64_t *pool_P;      //   its first arc in the pool's arc space (prefix),
    int32_t *pool_len;    //   its arcs (0 = not yet published; zeroed at init)
    int64_t pool_cap;
    int32_t *alive[2];    // alive lists, one segment per CTA
    int32_t *seg_len[2];  // entries of segment b in alive[x]: seg_len[x][b]
    int64_t seg_R;        // segment region size: segment b lives at [b*R, b*R + len)
    int32_t nseg;         // = persistent grid size
    int32_t pad;
    State *S;
    int64_t n;
};

struct Smem {
    int32_t lv[2][kLCap];
    int32_t ld[2][kLCap];
    int64_t lb[2][kLCap];
    int64_t lpre[kLCap + 1];
    int32_t lcnt[2];
    int32_t larc[2];
    int32_t removed;     // vertices removed by this CTA this phase (order not recorded)
    int32_t kcur;        // scan: compaction cursor
    int32_t pv[kWarps][kPStage];
    int32_t pd[kWarps][kPStage];
    int64_t pb[kWarps][kPStage];
    unsigned long long scan_q[kWarps];
    unsigned long long tot_q;
    int32_t red_min[kWarps];
    int64_t c0, c1;      // claimed pool arcs
    int64_t cnt;         // pool entries reserved when they were claimed
    int64_t backlog;     // unclaimed pool arcs per CTA when they were claimed
    int32_t done, pad3;
    int64_t lvl_arcs;    // arcs this CTA walked in the current level
    int64_t bloom_level;
    int32_t bloom_on;
    int32_t pad4;
    Ctrl ctrl;
    Snap snap;
    uint32_t bloom[kBloomWords];
};

// ---------------------------------------------------------------- helpers
__device__ __forceinline__ int warp_min(int v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(kFull, v, o));
    return v;
}

__device__ __forceinline__ unsigned long long globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ int32_t ld_acquire_i32(const int32_t *p)
{
    int32_t v;
    asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t bloom_h1(uint32_t v) { return (v * 0x9E3779B1u) >> 12; }
__device__ __forceinline__ uint32_t bloom_h2(uint32_t v) { return ((v ^ (v >> 15)) * 0x85EBCA6Bu) >> 12; }

__device__ __forceinline__ bool bloom_maybe(const Smem &sm, uint32_t v)
{
    const uint32_t a = bloom_h1(v), b = bloom_h2(v);
    return ((sm.bloom[a >> 5] >> (a & 31)) & (sm.bloom[b >> 5] >> (b & 31)) & 1u) != 0;
}

// Per-CTA timestamps of the current phase (trace mode only), indexed by the
// number of grid barriers passed: 0 start, 1 end of own scan, 2 end of own
// drain, 3 barrier arrival (after the pool loop).
__device__ __forceinline__ void cta_time(const KArgs &A, const Ctrl &c, int slot)
{
    if (threadIdx.x != 0 || c.solo) return;
    State *S = A.S;
    if (!S->trace_cta || c.st_bar >= S->trace_cap) return;
    S->trace_cta[(c.st_bar * gridDim.x + blockIdx.x) * 4 + slot] = (int64_t)globaltimer();
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

// Block-wide exclusive scan of one u64 per thread; total in sm.tot_q.
__device__ __forceinline__ unsigned long long block_excl_scan(Smem &sm, unsigned long long q)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned long long qi = q;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned long long t = __shfl_up_sync(kFull, qi, o);
        if (lane >= o) qi += t;
    }
    if (lane == 31) sm.scan_q[wib] = qi;
    __syncthreads();
    if (wib == 0) {
        const unsigned long long wq = lane < kWarps ? sm.scan_q[lane] : 0ULL;
        unsigned long long iq = wq;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long t = __shfl_up_sync(kFull, iq, o);
            if (lane >= o) iq += t;
        }
        if (lane < kWarps) sm.scan_q[lane] = iq - wq;
        if (lane == kWarps - 1) sm.tot_q = iq;
    }
    __syncthreads();
    return sm.scan_q[wib] + (qi - q);
}

__device__ __forceinline__ bool claim(const KArgs &A, int32_t v)
{
    const uint32_t bit = 1u << (v & 31);
    return (atomicOr(A.claimed + (v >> 5), bit) & bit) == 0u;
}

// ------------------------------------------------------------- the pool
// Flush this warp's pool stage: one packed atomic reserves the entries and
// their range in the pool's arc space; entries are published by writing their
// length last, after a fence (consumers spin until it is non-zero).
__device__ __noinline__ void pool_flush(const KArgs &A, Smem &sm, int wib, int &pcnt)
{
    const int lane = threadIdx.x & 31;
    if (pcnt == 0) return;
    __syncwarp();
    int64_t dd[2], pre[2];
    int64_t carry = 0;
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int x = h * 32 + lane;
        dd[h] = x < pcnt ? (int64_t)sm.pd[wib][x] : 0;
        int64_t incl = dd[h];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t t = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += t;
        }
        pre[h] = carry + incl - dd[h];
        carry += __shfl_sync(kFull, incl, 31);
    }
    unsigned long long base = 0;
    if (lane == 0)
        base = atomicAdd(&A.S->pool_tail, ((unsigned long long)pcnt << kArcBits) | (unsigned long long)carry);
    base = __shfl_sync(kFull, base, 0);
    const int64_t bc = (int64_t)(base >> kArcBits), ba = (int64_t)(base & kArcMask);
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int x = h * 32 + lane;
        if (x < pcnt) {
            A.pool_v[bc + x] = sm.pv[wib][x];
            A.pool_beg[bc + x] = sm.pb[wib][x];
            A.pool_P[bc + x] = ba + pre[h];
        }
    }
    __threadfence();
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const int x = h * 32 + lane;
        if (x < pcnt) A.pool_len[bc + x] = (int32_t)dd[h];
    }
    __syncwarp();
    pcnt = 0;
}

// Route claimed vertices (one per lane where `won`): record the removal
// (order slot if requested -- a vertex is claimed only after every vertex
// whose processing made it reach k was claimed, so claim-time slots form a
// valid peel order, the I4 certificate -- else a count), then send each to
// the local next frontier `nx` if it fits the sub-round's arc budget, else
// to the pool.  Zero-degree vertices are only recorded.
__device__ __noinline__ void route_won(const KArgs &A, Smem &sm, int wib, bool won, int32_t v,
                                          int32_t dv, int64_t bv, int nx, int &pcnt)
{
    const int lane = threadIdx.x & 31;
    const unsigned b = __ballot_sync(kFull, won);
    if (b == 0) return;
    {
        const int lead = __ffs(b) - 1;
        if (A.order) {
            unsigned long long base = 0;
            if (lane == lead) base = atomicAdd(&A.S->ord_tail, (unsigned long long)__popc(b));
            base = __shfl_sync(kFull, base, lead);
            if (won) A.order[base + __popc(b & lanemask_lt())] = v;
        } else if (lane == lead) {
            atomicAdd(&sm.removed, __popc(b));
        }
    }
    const bool cand = won && dv > 0 && dv <= kSub;
    const unsigned bc = __ballot_sync(kFull, cand);
    bool wantl = false;
    int lbase = 0;
    if (bc) {
        int sumd = cand ? dv : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sumd += __shfl_xor_sync(kFull, sumd, o);
        const int lead = __ffs(bc) - 1;
        int ok = 0;
        if (lane == lead) {
            const int oa = atomicAdd(&sm.larc[nx], sumd);
            if (oa + sumd <= kSub) { ok = 1; lbase = atomicAdd(&sm.lcnt[nx], __popc(bc)); }
        }
        ok = __shfl_sync(kFull, ok, lead);
        lbase = __shfl_sync(kFull, lbase, lead);
        wantl = cand && ok;
    }
    bool top = won && dv > 0 && !wantl;
    if (wantl) {
        const int pos = lbase + __popc(bc & lanemask_lt());
        if (pos < kLCap) {
            sm.lv[nx][pos] = v;
            sm.ld[nx][pos] = dv;
            sm.lb[nx][pos] = bv;
        } else {
            top = true;
        }
    }
    const unsigned bg = __ballot_sync(kFull, top);
    if (bg) {
        const int c = __popc(bg);
        if (pcnt + c > kPStage) pool_flush(A, sm, wib, pcnt);
        if (top) {
            const int pos = pcnt + __popc(bg & lanemask_lt());
            sm.pv[wib][pos] = v;
            sm.pd[wib][pos] = dv;
            sm.pb[wib][pos] = bv;
        }
        pcnt += c;
    }
    __syncwarp();
}

// --------------------------------------------------------- arc walking
// Hits of one batch (u reached k): claim, fetch row bounds, prefetch the
// row's first line for the next hop, route.  Out of line: rare path.
__device__ __noinline__ void handle_hits(const KArgs &A, Smem &sm, int nx, int u0, int u1, int u2, int u3,
                                         unsigned hm, int &pcnt)
{
    const int wib = threadIdx.x >> 5;
    const int uu[4] = {u0, u1, u2, u3};
    bool won[4];
#pragma unroll
    for (int r = 0; r < 4; r++) won[r] = ((hm >> r) & 1u) && claim(A, uu[r]);
    int64_t b0[4], b1[4];
#pragma unroll
    for (int r = 0; r < 4; r++) {
        b0[r] = won[r] ? ld_ro_i64(A.rowptr + uu[r]) : 0;
        b1[r] = won[r] ? ld_ro_i64(A.rowptr + uu[r] + 1) : 0;
    }
#pragma unroll
    for (int r = 0; r < 4; r++) {
        if (won[r] && b1[r] > b0[r]) asm volatile("prefetch.global.L2 [%0];" ::"l"(A.colidx + b0[r]));
        route_won(A, sm, wib, won[r], uu[r], (int32_t)(b1[r] - b0[r]), b0[r], nx, pcnt);
    }
}

// Walk arcs [a0,a1) of the local frontier `cur` (entries [0,e), arc prefix
// lpre[], row begins lb[cur][]; the last entry ends at arc ae) with one warp.
// Each lane holds one entry of a 32-entry window; an arc finds its entry with
// a 5-step shuffle search on 32-bit offsets relative to the current batch.
__device__ __forceinline__ void walk(const KArgs &A, Smem &sm, const int k, const int cur, const int nx,
                                     int64_t e, int64_t ae, int64_t a0, int64_t a1, bool use_bloom,
                                     int &lmin, int &pcnt)
{
    const int lane = threadIdx.x & 31;
    int64_t lo = 0, hi = e;  // first entry: largest i with lpre[i] <= a0 (32-ary search)
    while (true) {
        const int64_t step = hi - lo > 32 ? (hi - lo + 31) / 32 : 1;
        const int64_t p = lo + lane * step;
        const bool ok = (p < hi) && sm.lpre[p] <= a0;
        const unsigned b = __ballot_sync(kFull, ok);
        lo = lo + (31 - __clz(b)) * step;
        if (step == 1) break;
        hi = min(hi, lo + step);
    }
    int64_t i = lo;
    int64_t a = a0;
    while (a < a1) {
        const int64_t j = i + lane;
        int64_t wq = LLONG_MAX, wbeg = 0;
        if (j < e) {
            wq = sm.lpre[j];
            wbeg = sm.lb[cur][j];
        }
        int64_t nxt = __shfl_down_sync(kFull, wq, 1);
        if (j + 1 >= e) nxt = ae;
        else if (lane == 31) nxt = sm.lpre[j + 1];
        const int64_t limit = min(a1, __shfl_sync(kFull, nxt, 31));
        const int64_t bmq = wbeg - wq;  // colidx index of arc x in this entry = bmq + x
        while (a < limit) {
            const int64_t rq = wq - a;
            const int32_t q32 = rq < -1 ? -1 : (rq > 0x7fffffff ? 0x7fffffff : (int32_t)rq);
            const int32_t lim = (int32_t)min((int64_t)kBatch, limit - a);
            int32_t u[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                const int32_t my = r * 32 + lane;
                int pos = 0;
#pragma unroll
                for (int bs = 16; bs >= 1; bs >>= 1) {
                    const int32_t q = __shfl_sync(kFull, q32, pos + bs);
                    if (q <= my) pos += bs;
                }
                const int64_t off = __shfl_sync(kFull, bmq, pos);
                u[r] = (my < lim) ? ld_stream_i32(A.colidx + off + a + my) : -1;
            }
            if (use_bloom) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if (u[r] >= 0 && !bloom_maybe(sm, (uint32_t)u[r])) u[r] = -1;
            }
            int32_t d[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) d[r] = u[r] >= 0 ? ld_cg_i32(A.deg + u[r]) : -1;
            int old[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) old[r] = d[r] > k ? atomicSub(A.deg + u[r], 1) : INT_MIN;
            unsigned hm = 0;
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                if (old[r] == k + 1) hm |= 1u << r;
                else if (old[r] != INT_MIN && old[r] <= k) atomicAdd(A.deg + u[r], 1);
                else if (old[r] > k + 1) lmin = min(lmin, old[r] - 1);
            }
            if (__any_sync(kFull, hm != 0)) handle_hits(A, sm, nx, u[0], u[1], u[2], u[3], hm, pcnt);
            a += kBatch;
        }
        a = limit;
        i += 32;
    }
}

// Pool entry j (spinning until it is published): arc-space start, length, row begin.
__device__ __forceinline__ int32_t pool_entry(const KArgs &A, int64_t j, int64_t &P, int64_t &beg)
{
    int32_t len;
    while ((len = ld_acquire_i32(A.pool_len + j)) == 0) {
    }
    P = ld_cg_i64(A.pool_P + j);
    beg = ld_cg_i64(A.pool_beg + j);
    return len;
}

// Walk pool arcs [a0,a1) with one warp (entries [0,cnt) are reserved; every
// arc below a1 belongs to one of them).  Same window scheme as walk().
__device__ __forceinline__ void walk_pool(const KArgs &A, Smem &sm, const int k, const int nx, int64_t cnt,
                                          int64_t a0, int64_t a1, bool use_bloom, int &lmin, int &pcnt)
{
    const int lane = threadIdx.x & 31;
    int64_t lo = 0, hi = cnt;  // first entry: largest j with P(j) <= a0
    while (true) {
        const int64_t step = hi - lo > 32 ? (hi - lo + 31) / 32 : 1;
        const int64_t p = lo + lane * step;
        bool ok = false;
        if (p < hi) {
            int64_t P, beg;
            pool_entry(A, p, P, beg);
            ok = P <= a0;
        }
        const unsigned b = __ballot_sync(kFull, ok);
        lo = lo + (31 - __clz(b)) * step;
        if (step == 1) break;
        hi = min(hi, lo + step);
    }
    int64_t i = lo;
    int64_t a = a0;
    while (a < a1) {
        const int64_t j = i + lane;
        int64_t wq = LLONG_MAX, wbeg = 0, wend = LLONG_MAX;
        if (j < cnt) {
            const int32_t len = pool_entry(A, j, wq, wbeg);
            wend = wq + len;
        }
        const int last = (int)min((int64_t)31, cnt - 1 - i);
        const int64_t limit = min(a1, __shfl_sync(kFull, wend, last));
        const int64_t bmq = wbeg - wq;
        while (a < limit) {
            const int64_t rq = wq - a;
            const int32_t q32 = rq < -1 ? -1 : (rq > 0x7fffffff ? 0x7fffffff : (int32_t)rq);
            const int32_t lim = (int32_t)min((int64_t)kBatch, limit - a);
            int32_t u[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                const int32_t my = r * 32 + lane;
                int pos = 0;
#pragma unroll
                for (int bs = 16; bs >= 1; bs >>= 1) {
                    const int32_t q = __shfl_sync(kFull, q32, pos + bs);
                    if (q <= my) pos += bs;
                }
                const int64_t off = __shfl_sync(kFull, bmq, pos);
                u[r] = (my < lim) ? ld_stream_i32(A.colidx + off + a + my) : -1;
            }
            if (use_bloom) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if (u[r] >= 0 && !bloom_maybe(sm, (uint32_t)u[r])) u[r] = -1;
            }
            int32_t d[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) d[r] = u[r] >= 0 ? ld_cg_i32(A.deg + u[r]) : -1;
            int old[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) old[r] = d[r] > k ? atomicSub(A.deg + u[r], 1) : INT_MIN;
            unsigned hm = 0;
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                if (old[r] == k + 1) hm |= 1u << r;
                else if (old[r] != INT_MIN && old[r] <= k) atomicAdd(A.deg + u[r], 1);
                else if (old[r] > k + 1) lmin = min(lmin, old[r] - 1);
            }
            if (__any_sync(kFull, hm != 0)) handle_hits(A, sm, nx, u[0], u[1], u[2], u[3], hm, pcnt);
            a += kBatch;
        }
        a = limit;
        i += 32;
    }
}

// Bloom filter of the alive list at level start (built once per level).
__device__ void bloom_build(const KArgs &A, const Ctrl &c, Smem &sm)
{
    for (int w = threadIdx.x; w < kBloomWords; w += kBlock) sm.bloom[w] = 0u;
    __syncthreads();
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    if (c.src_single) {  // one contiguous run: every thread strides it
        const int32_t *src = A.alive[c.src_sel];
        for (int64_t i = threadIdx.x; i < c.src_len; i += kBlock) {
            const uint32_t v = (uint32_t)ld_cg_i32(src + i);
            const uint32_t h1 = bloom_h1(v), h2 = bloom_h2(v);
            atomicOr(&sm.bloom[h1 >> 5], 1u << (h1 & 31));
            atomicOr(&sm.bloom[h2 >> 5], 1u << (h2 & 31));
        }
    } else {  // per-CTA segments: one warp per segment
        for (int b = wib; b < A.nseg; b += kWarps) {
            const int32_t *src = A.alive[c.src_sel] + (int64_t)b * A.seg_R;
            const int64_t len = ld_cg_i32(A.seg_len[c.src_sel] + b);
            for (int64_t i = lane; i < len; i += 32) {
                const uint32_t v = (uint32_t)ld_cg_i32(src + i);
                const uint32_t h1 = bloom_h1(v), h2 = bloom_h2(v);
                atomicOr(&sm.bloom[h1 >> 5], 1u << (h1 & 31));
                atomicOr(&sm.bloom[h2 >> 5], 1u << (h2 & 31));
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) { sm.bloom_level = c.level; sm.bloom_on = 1; }
    __syncthreads();
}

// Decide (CTA-uniform) whether the arcs this CTA walks this level pay for a filter.
__device__ __forceinline__ bool want_bloom(const KArgs &A, const Ctrl &c, Smem &sm, int64_t more)
{
    if (!A.S->prm.bloom || c.src_sel < 0 || c.src_len > kBloomMaxA) return false;
    if (sm.bloom_on && sm.bloom_level == c.level) return true;
    if (sm.lvl_arcs + more < 4 * c.src_len + 65536) return false;
    bloom_build(A, c, sm);
    return true;
}

// Drain this CTA's local frontier (list `cur`) breadth-first with CTA-local
// sub-rounds.  Returns the number of arcs walked.
__device__ int64_t local_drain(const KArgs &A, const Ctrl &c, Smem &sm, int cur, int &lmin, int &pcnt)
{
    const int wib = threadIdx.x >> 5;
    int64_t walked = 0;
    for (int round = 0;; round++) {
        __syncthreads();
        const int L = min(sm.lcnt[cur], kLCap);
        if (L == 0) break;
        if (round == kMaxLocalRounds) {
            // a long local chain: hand the frontier back to the pool so idle
            // CTAs share it (each warp pushes a slice through its stage)
            for (int x0 = wib * 32; x0 < L; x0 += kWarps * 32) {
                const int x = x0 + (threadIdx.x & 31);
                const bool has = x < L;
                const unsigned bg = __ballot_sync(kFull, has);
                if (pcnt + __popc(bg) > kPStage) pool_flush(A, sm, wib, pcnt);
                if (has) {
                    const int pos = pcnt + __popc(bg & lanemask_lt());
                    sm.pv[wib][pos] = sm.lv[cur][x];
                    sm.pd[wib][pos] = sm.ld[cur][x];
                    sm.pb[wib][pos] = sm.lb[cur][x];
                }
                pcnt += __popc(bg);
                __syncwarp();
            }
            __syncthreads();
            if (threadIdx.x == 0) { sm.lcnt[cur] = 0; sm.larc[cur] = 0; }
            __syncthreads();
            break;
        }
        const int64_t dv = threadIdx.x < L ? (int64_t)sm.ld[cur][threadIdx.x] : 0;
        const unsigned long long ex = block_excl_scan(sm, (unsigned long long)dv);
        if (threadIdx.x < L) sm.lpre[threadIdx.x] = (int64_t)ex;
        const int64_t T = (int64_t)sm.tot_q;
        const int nx = cur ^ 1;
        if (threadIdx.x == 0) { sm.lpre[L] = T; sm.lcnt[nx] = 0; sm.larc[nx] = 0; }
        __syncthreads();
        const bool bl = want_bloom(A, c, sm, T);
        int64_t C = (T + kWarps - 1) / kWarps;
        C = ((C + kBatch - 1) / kBatch) * kBatch;
        const int64_t a0 = (int64_t)wib * C;
        if (a0 < T) walk(A, sm, c.k, cur, nx, L, T, a0, min(a0 + C, T), bl, lmin, pcnt);
        walked += T;
        __syncthreads();
        if (threadIdx.x == 0) { sm.lcnt[cur] = 0; sm.larc[cur] = 0; sm.lvl_arcs += T; }
        cur = nx;
    }
    return walked;
}

// ------------------------------------------------------------------ INIT
__device__ void phase_init(const KArgs &A, Smem &sm)
{
    int lmin = INT_MAX;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t v = tid; v < A.n; v += stride) {
        const int32_t d = (int32_t)(ld_ro_i64(A.rowptr + v + 1) - ld_ro_i64(A.rowptr + v));
        A.deg[v] = d;
        lmin = min(lmin, d);
    }
    for (int64_t w = tid; w < (A.n + 31) / 32; w += stride) A.claimed[w] = 0u;
    for (int64_t w = tid; w < A.pool_cap; w += stride) A.pool_len[w] = 0;
    if (threadIdx.x == 0) {
        sm.bloom_on = 0; sm.bloom_level = -1;
        sm.lcnt[0] = sm.lcnt[1] = 0; sm.larc[0] = sm.larc[1] = 0;
    }
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// ------------------------------------------------------------------ LEVEL
// Scan entries [lo,hi) of list `src` (nullptr: the identity) with every warp
// of this CTA (Alg. 2): eight entries per lane in flight; deg == k -> claim +
// route; deg > k -> min and ballot compaction (Fig. 8(c)) into dst[0..) with a
// shared-memory cursor.  No block sync, no global atomics.
__device__ void scan_range(const KArgs &A, const Ctrl &c, Smem &sm, const int32_t *src, int64_t lo,
                           int64_t hi, int32_t *dst, int &lmin, int &pcnt)
{
    const int k = c.k;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    constexpr int CH = 32 * kScanItems;
    for (int64_t off = lo + (int64_t)wib * CH; off < hi; off += (int64_t)kWarps * CH) {
        int32_t vv[kScanItems], dd[kScanItems];
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            const int64_t idx = off + j * 32 + lane;
            vv[j] = -1;
            if (idx < hi) vv[j] = src ? ld_cg_i32(src + idx) : (int32_t)idx;
        }
#pragma unroll
        for (int j = 0; j < kScanItems; j++) dd[j] = vv[j] >= 0 ? ld_cg_i32(A.deg + vv[j]) : -1;
        unsigned wm = 0, km = 0;
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            // at k = 0 the frontier is the isolated vertices: nothing can race for them
            if (dd[j] == k) { if (k == 0 || claim(A, vv[j])) wm |= 1u << j; }
            else if (dd[j] > k) { lmin = min(lmin, dd[j]); km |= 1u << j; }
        }
        if (dst) {
            const int mine = __popc(km);
            int incl = mine;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += t;
            }
            const int tot = __shfl_sync(kFull, incl, 31);
            int pos = 0;
            if (lane == 31 && tot) pos = atomicAdd(&sm.kcur, tot);
            pos = __shfl_sync(kFull, pos, 31) + incl - mine;
#pragma unroll
            for (int j = 0; j < kScanItems; j++)
                if ((km >> j) & 1u) dst[pos++] = vv[j];
        }
        if (__any_sync(kFull, wm != 0)) {
            int64_t b0[kScanItems];
            int32_t du[kScanItems];
#pragma unroll
            for (int j = 0; j < kScanItems; j++) {
                b0[j] = 0; du[j] = 0;
                if (((wm >> j) & 1u) && k > 0) {  // at k = 0 every claimed vertex is isolated
                    b0[j] = ld_ro_i64(A.rowptr + vv[j]);
                    du[j] = (int32_t)(ld_ro_i64(A.rowptr + vv[j] + 1) - b0[j]);
                }
            }
#pragma unroll
            for (int j = 0; j < kScanItems; j++) {
                if (du[j] > 0) asm volatile("prefetch.global.L2 [%0];" ::"l"(A.colidx + b0[j]));
                route_won(A, sm, wib, (wm >> j) & 1u, vv[j], du[j], b0[j], 0, pcnt);
            }
        }
    }
}

// Source layout: identity (src_sel < 0), one contiguous run (src_single) or
// per-CTA segments.  Grid mode: CTA b scans its share and compacts into its
// own segment b.  Solo mode: CTA 0 scans everything into one run (segment 0).
__device__ void level_scan(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk, int &lmin,
                           int &pcnt)
{
    const bool solo = (nblk == 1);
    const int32_t *srcb = c.src_sel < 0 ? nullptr : A.alive[c.src_sel];
    int32_t *dstb = c.compact ? A.alive[c.dst_sel] : nullptr;
    const int dseg = solo ? 0 : bid;
    if (threadIdx.x == 0) sm.kcur = 0;
    __syncthreads();
    int32_t *dst = dstb ? dstb + (int64_t)dseg * A.seg_R : nullptr;
    if (c.src_sel < 0 || c.src_single) {
        const int64_t L = c.src_len;
        const int64_t lo = solo ? 0 : (L * bid) / nblk, hi = solo ? L : (L * (bid + 1)) / nblk;
        scan_range(A, c, sm, srcb, lo, hi, dst, lmin, pcnt);
    } else if (!solo) {
        const int64_t len = ld_cg_i32(A.seg_len[c.src_sel] + bid);
        scan_range(A, c, sm, srcb + (int64_t)bid * A.seg_R, 0, len, dst, lmin, pcnt);
    } else {
        for (int b = 0; b < A.nseg; b++) {
            const int64_t len = ld_cg_i32(A.seg_len[c.src_sel] + b);
            if (len) scan_range(A, c, sm, srcb + (int64_t)b * A.seg_R, 0, len, dst, lmin, pcnt);
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && dstb) {
        A.seg_len[c.dst_sel][dseg] = sm.kcur;
        if (sm.kcur) atomicAdd(&A.S->alive_out, (unsigned long long)sm.kcur);
    }
}

// One level (Alg. 1 round k): scan, drain the local frontier, then share the
// pool until every CTA has scanned and every pool entry is processed.
// c.cont: the scan was done by a solo CTA that bailed out; only the pool is
// left.  A solo CTA (nblk == 1) bails out when its pool backlog is large and
// returns true (the grid then finishes the level).
__device__ bool phase_level(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk)
{
    const int wib = threadIdx.x >> 5;
    State *S = A.S;
    int lmin = INT_MAX, pcnt = 0;
    int64_t walked = 0;
    cta_time(A, c, 0);
    if (threadIdx.x == 0) {
        sm.lcnt[0] = sm.lcnt[1] = 0; sm.larc[0] = sm.larc[1] = 0;
        sm.removed = 0; sm.lvl_arcs = 0;
    }
    __syncthreads();
    if (!c.cont) {
        level_scan(A, c, sm, bid, nblk, lmin, pcnt);
        cta_time(A, c, 1);
        walked = local_drain(A, c, sm, 0, lmin, pcnt);
        pool_flush(A, sm, wib, pcnt);
        __syncthreads();
    }
    cta_time(A, c, 2);
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(&S->scans_done, 1ULL);
        sm.done = 0;
        if (nblk == 1) {
            const unsigned long long pend = (ld_acquire_u64(&S->pool_tail) & kArcMask) - ld_acquire_u64(&S->pool_done);
            if (pend > (unsigned long long)kSoloBail) sm.done = 2;
        }
    }
    __syncthreads();
    const bool bail = sm.done == 2;
    // pool loop: claim, copy into the local frontier, drain, report
    bool bailed = bail;
    while (!bailed) {
        if (threadIdx.x == 0) {
            int64_t c0 = -1, c1 = -1;
            int done = 0;
            const unsigned long long tp = ld_acquire_u64(&S->pool_tail);
            const unsigned long long tcnt = tp >> kArcBits, tarc = tp & kArcMask;
            unsigned long long cl = ld_acquire_u64(&S->pool_claim);
            if (nblk == 1 && tarc - cl > (unsigned long long)kSoloBail) { cl = tarc; done = 2; }
            while (cl < tarc) {
                unsigned long long J = (tarc - cl) / (2ULL * (unsigned long long)nblk);
                J = J < (unsigned long long)kClaimMin ? (unsigned long long)kClaimMin
                                                      : (J > (unsigned long long)kClaimMax ? (unsigned long long)kClaimMax : J);
                const unsigned long long want = min(cl + J, tarc);
                const unsigned long long got = atomicCAS(&S->pool_claim, cl, want);
                if (got == cl) { c0 = (int64_t)cl; c1 = (int64_t)want; break; }
                cl = got;
            }
            if (c0 < 0 && done == 0) {
                const unsigned long long dn = ld_acquire_u64(&S->pool_done);
                const unsigned long long sd = ld_acquire_u64(&S->scans_done);
                const unsigned long long t2 = ld_acquire_u64(&S->pool_tail) & kArcMask;
                if (sd >= (unsigned long long)c.scan_target && dn == t2) done = 1;
                else __nanosleep(64);
            }
            sm.c0 = c0;
            sm.c1 = c1;
            sm.cnt = (int64_t)tcnt;
            sm.backlog = (int64_t)(tarc - (c0 < 0 ? tarc : (unsigned long long)c0)) / nblk;
            sm.done = done;
        }
        __syncthreads();
        if (sm.done == 2) { bailed = true; break; }
        if (sm.done) break;
        const int64_t c0 = sm.c0, c1 = sm.c1;
        if (c0 < 0) continue;
        // arc-balanced walk of the claimed pool arcs; hits go to local list 0
        {
            const int64_t T = c1 - c0;
            const bool bl = want_bloom(A, c, sm, max(T, sm.backlog));
            int64_t C = (T + kWarps - 1) / kWarps;
            C = ((C + kBatch - 1) / kBatch) * kBatch;
            const int64_t w0 = c0 + (int64_t)wib * C;
            if (w0 < c1) walk_pool(A, sm, c.k, 0, sm.cnt, w0, min(w0 + C, c1), bl, lmin, pcnt);
            walked += T;
            __syncthreads();
            if (threadIdx.x == 0) sm.lvl_arcs += T;
        }
        walked += local_drain(A, c, sm, 0, lmin, pcnt);  // starts with __syncthreads
        pool_flush(A, sm, wib, pcnt);
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            atomicAdd(&S->pool_done, (unsigned long long)(c1 - c0));
        }
    }
    if (threadIdx.x == 0) {
        if (walked) atomicAdd(&S->arcs_walked, (unsigned long long)walked);
        if (sm.removed) atomicAdd(&S->ord_tail, (unsigned long long)sm.removed);
    }
    block_min_atomic(sm, lmin, &S->min_next);
    return bailed;
}

// ---------------------------------------------------------------- control
// The pure transition function (Alg. 1 l.5-9 and the level skip).  Every CTA
// applies it to identical inputs, so all copies stay identical.
__device__ __noinline__ void advance(Ctrl &c, const Snap &sn, const Params &p, int nblk)
{
    const int64_t removed = (int64_t)sn.ord;
    c.level_min = min(c.level_min, sn.min);
    int next_k = 0;
    if (c.phase == PH_INIT) {
        next_k = (c.level_min == INT_MAX) ? 0 : c.level_min;
        c.level_min = INT_MAX;
        c.level = -1;
    } else {  // a LEVEL phase ended: the level is complete
        c.st_phases++;
        if (c.solo) c.st_solo++;
        c.st_scanned += c.src_len;
        c.st_pool = (int64_t)sn.pool;
        if (c.compact) {
            c.alive_sel = c.dst_sel;
            c.alive_len = (int64_t)sn.alive_out + c.alive_carry;
            c.alive_single = c.solo || c.cont;  // a solo scan compacts into one run
            c.st_compact++;
        }
        if (removed > c.ord_lvl0) { c.st_levels++; c.st_kmax = c.k; }
        if (removed >= p.n) {
            c.phase = PH_DONE;
            c.solo = 0;
            return;
        }
        next_k = max(c.k + 1, c.level_min);
        c.level_min = INT_MAX;
    }
    const int64_t live = p.n - removed;
    const int64_t src_len = c.alive_sel < 0 ? p.n : c.alive_len;
    c.phase = PH_LEVEL;
    c.cont = 0;
    c.alive_carry = 0;
    c.k = next_k;
    c.level++;
    c.src_sel = c.alive_sel;
    c.src_single = c.alive_single;
    c.src_len = src_len;
    c.compact = (live * 8 < src_len * 7) ? 1 : 0;  // >= 1/8 of the scan source is dead
    c.dst_sel = c.alive_sel < 0 ? 0 : 1 - c.alive_sel;
    c.solo = src_len <= (int64_t)p.solo_scan;
    // a solo scan of a segmented list gathers it into one run for next time
    if (c.solo && c.alive_sel >= 0 && !c.alive_single) c.compact = 1;
    c.scan_target += c.solo ? 1 : nblk;
    c.ord_lvl0 = removed;
}

// Snapshot + reset of the counters (caller guarantees nobody else touches them).
__device__ __forceinline__ Snap take_snapshot(State *S)
{
    Snap sn;
    sn.ord = ld_relaxed_u64(&S->ord_tail);
    sn.alive_out = ld_relaxed_u64(&S->alive_out);
    sn.pool = ld_relaxed_u64(&S->pool_tail) & kArcMask;
    sn.min = ld_relaxed_i32(&S->min_next);
    sn.pad = 0;
    S->alive_out = 0ULL;
    S->min_next = INT_MAX;
    return sn;
}

__device__ __forceinline__ void trace_rec(State *S, const Ctrl &c, const Snap &sn, int grid, int64_t arcs)
{
    if (!S->trace) return;
    const unsigned long long i = S->trace_n;
    if ((int64_t)i >= S->trace_cap) return;
    int64_t *r = S->trace + i * kTraceFields;
    r[0] = (int64_t)globaltimer();
    r[1] = (int64_t)clock64();
    r[2] = ((int64_t)c.phase << 8) | ((int64_t)c.solo << 4) | grid;  // phase that ENDED
    r[3] = c.k;
    r[4] = c.src_len;
    r[5] = arcs;                  // arcs walked so far (cumulative)
    r[6] = (int64_t)sn.ord;
    r[7] = c.st_bar;
    S->trace_n = i + 1;
}

// Grid barrier; the last arriver snapshots+resets the counters.
__device__ __forceinline__ void grid_barrier(const KArgs &A, Smem &sm)
{
    __syncthreads();
    cta_time(A, sm.ctrl, 3);
    if (threadIdx.x == 0) {
        State *S = A.S;
        const uint32_t gen = ld_acquire_u32(&S->bar_gen);
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
            sn.ord = ld_relaxed_u64(&ps->ord);
            sn.alive_out = ld_relaxed_u64(&ps->alive_out);
            sn.pool = ld_relaxed_u64(&ps->pool);
            sn.min = ld_relaxed_i32(&ps->min);
            sn.pad = 0;
        }
        sm.snap = sn;
    }
    __syncthreads();
}

// CTA 0 alone: run consecutive solo levels with CTA-local synchronisation.
__device__ void solo_run(const KArgs &A, Smem &sm, const Params &p)
{
    State *S = A.S;
    while (true) {
        const Ctrl c = sm.ctrl;
        const bool bail = phase_level(A, c, sm, 0, 1);  // ends with __syncthreads
        if (bail) {  // the level's pool is too big for one CTA: the grid finishes it
            if (threadIdx.x == 0) {
                // fold this partial level's counters into the control state: the
                // barrier that follows resets them before the grid continues
                __threadfence();
                const Snap sn = take_snapshot(S);
                sm.ctrl.level_min = min(sm.ctrl.level_min, sn.min);
                sm.ctrl.alive_carry = (int64_t)sn.alive_out;
                sm.ctrl.cont = 1;
                sm.ctrl.solo = 0;
                sm.ctrl.scan_target += gridDim.x;
            }
            __syncthreads();
            break;
        }
        if (threadIdx.x == 0) {
            __threadfence();
            const Snap sn = take_snapshot(S);
            trace_rec(S, sm.ctrl, sn, 0, (int64_t)ld_relaxed_u64(&S->arcs_walked));
            advance(sm.ctrl, sn, p, (int)gridDim.x);
        }
        __syncthreads();
        if (sm.ctrl.phase == PH_DONE || !sm.ctrl.solo) break;
    }
    if (threadIdx.x == 0) {
        S->pub = sm.ctrl;
        __threadfence();
    }
}

__device__ __forceinline__ void init_ctrl(Ctrl &z)
{
    z = Ctrl{};
    z.phase = PH_INIT;
    z.level_min = INT_MAX;
    z.alive_sel = -1;
    z.src_sel = -1;
}

__global__ void __launch_bounds__(kBlock, 1) k_persistent(KArgs A)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    State *S = A.S;
    const Params p = S->prm;
    if (threadIdx.x == 0) init_ctrl(sm.ctrl);
    phase_init(A, sm);
    grid_barrier(A, sm);
    if (threadIdx.x == 0) advance(sm.ctrl, sm.snap, p, (int)gridDim.x);
    __syncthreads();
    while (true) {
        if (sm.ctrl.phase == PH_DONE) break;
        if (sm.ctrl.solo) {
            if (blockIdx.x == 0) solo_run(A, sm, p);
            grid_barrier(A, sm);
            if (threadIdx.x == 0) {
                Ctrl c;
                const int4 *src = reinterpret_cast<const int4 *>(&S->pub);
                int4 *dst = reinterpret_cast<int4 *>(&c);
#pragma unroll
                for (int w = 0; w < (int)(sizeof(Ctrl) / sizeof(int4)); w++) dst[w] = __ldcg(src + w);
                c.st_bar++;
                sm.ctrl = c;
            }
        } else {
            const Ctrl c = sm.ctrl;
            phase_level(A, c, sm, blockIdx.x, gridDim.x);
            grid_barrier(A, sm);
            if (threadIdx.x == 0) {
                if (blockIdx.x == 0) trace_rec(S, sm.ctrl, sm.snap, 1, (int64_t)ld_relaxed_u64(&S->arcs_walked));
                sm.ctrl.st_bar++;
                advance(sm.ctrl, sm.snap, p, (int)gridDim.x);
            }
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) S->pub = sm.ctrl;  // final statistics
}

// -------------------------------------------- host-driven ablation kernels
// (KCORE_ALGO_HOSTLOOP: the paper's Alg. 1 structure -- one launch per level
// and a host read-back of the phase after each.  No solo levels.
// Launched cooperatively: the pool loop waits on other CTAs of the launch.)
__global__ void __launch_bounds__(kBlock, 1) k_phase(KArgs A)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    if (threadIdx.x == 0) {
        sm.ctrl = A.S->pub;
        sm.bloom_on = 0;
        sm.bloom_level = -1;
    }
    __syncthreads();
    const Ctrl c = sm.ctrl;
    if (c.phase == PH_INIT) phase_init(A, sm);
    else if (c.phase == PH_LEVEL) phase_level(A, c, sm, blockIdx.x, gridDim.x);
}

__global__ void k_leader(KArgs A, int32_t *phase_out, int32_t nblk)
{
    State *S = A.S;
    const Params p = S->prm;
    Ctrl c = S->pub;
    const Snap sn = take_snapshot(S);
    trace_rec(S, c, sn, 1, (int64_t)S->arcs_walked);
    c.st_bar++;
    advance(c, sn, p, nblk);
    S->pub = c;
    *phase_out = c.phase;
}

__global__ void k_init_state(State *S, int64_t n, int32_t solo_arcs, int32_t solo_scan, int32_t bloom,
                             int64_t *trace, int64_t *trace_cta, int64_t trace_cap)
{
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        S->ord_tail = 0ULL;
        S->alive_out = 0ULL;
        S->min_next = INT_MAX;
        S->pool_tail = 0ULL;
        S->pool_claim = 0ULL;
        S->pool_done = 0ULL;
        S->scans_done = 0ULL;
        S->bar_count = 0u;
        S->bar_gen = 0u;
        S->arcs_walked = 0ULL;
        Ctrl z;
        init_ctrl(z);
        S->pub = z;
        S->prm.n = n;
        S->prm.solo_arcs = solo_arcs;
        S->prm.solo_scan = solo_scan;
        S->prm.bloom = bloom;
        S->trace = trace;
        S->trace_cta = trace_cta;
        S->trace_cap = trace ? trace_cap : 0;
        S->trace_n = 0ULL;
    }
}

} // namespace kc
