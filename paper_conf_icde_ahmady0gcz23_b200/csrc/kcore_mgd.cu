// kcore_mgd.cu -- device-initiated multi-GPU peel (the paper's
// multi-GPU future work): ONE persistent kernel per rank, no host
// round trip per level or sub-round.
//
// 1-D vertex-range ownership as in kcore_mg.cu: rank r owns [vb_r, vb_{r+1})
// and the CSR rows of those vertices (global neighbour ids).  Every rank
// exposes one symmetric WINDOW (same layout on every rank):
//     ctl   barrier counter/generation, level-min accumulator, pushed count
//           (only rank 0's copy is used: the global control block)
//     tail  inbox append cursors [2]
//     deg   working degrees of the owned vertices (clamp-free, DESIGN R10)
//     inbox [2][nl_max]  owned vertices to walk in the next sub-round
// and reaches every other rank's window through a peer table: NCCL 2.28
// symmetric memory (ncclMemAlloc + ncclCommWindowRegister, peer addresses
// from ncclGetPeerPointer over NVLink/NVSwitch) or -- to test the protocol on
// the single GPU this project runs on -- P slices of one allocation
// ("virtual ranks", one cooperative kernel whose CTAs are split into P rank
// groups; a rank group touches another rank's data only through the peer
// table, exactly as a remote GPU would).
//
// Per level k (Alg. 1 round), bulk-synchronous with a device-side
// barrier over every CTA of every rank:
//   SCAN   each rank scans its own alive list (Alg. 2): deg <= k -> removed
//          (deg += 2^30), core = k, pushed into its own inbox; deg > k -> min
//          and compaction.  No walk runs during a scan, so no claim bits.
//   barrier
//   SUB-ROUNDS while anything was pushed: every rank walks the rows of its
//          inbox (Alg. 3 l.12-24) and decrements each target IN ITS OWNER'S
//          WINDOW (remote atomicSub through the peer table); the unique
//          decrement that sees old == k+1 marks the target removed
//          (remote red +2^30) and appends it to the owner's next inbox
//          (remote append); old > k+1 feeds the level-skip minimum.
//          barrier
//   level end: k <- max(k+1, global min) (reading R5), done when every vertex
//          is removed.
// deg >= 2^29 means removed: a removed vertex's word stays above 2^29 under
// any number of later decrements (at most its degree < 2^29), so walkers
// simply ignore it.  The last arriver of each barrier snapshots the global
// counters and resets the per-rank cursors; every CTA then applies the same
// transition.
#include "kcore.h"
#include "kcore_mgd.h"

#include <climits>
#include <cstdint>
#include <cstring>
#include <vector>

#include <cuda_runtime.h>
#include <nccl.h>
#if NCCL_VERSION_CODE >= 22800
#include <nccl_device.h>
#define KC_HAVE_NCCL_WINDOWS 1
#else
#define KC_HAVE_NCCL_WINDOWS 0
#endif

namespace mgd {

constexpr int kMaxR = 64;        // ranks (peer table)
constexpr int kMaxPL = 16;       // ranks in one launch (virtual ranks)
constexpr int kBlk = 512;
constexpr int kWarps = kBlk / 32;
constexpr int32_t kRemoved = 1 << 30;  // added to deg when a vertex is removed
constexpr int32_t kDead = 1 << 29;     // deg >= kDead: removed
constexpr int kChunk = 256;            // chunk queue granularity (arcs)
static_assert(kChunk <= 256, "chunk length - 1 is stored in 8 bits");
constexpr int kNearW = 16;             // near window W (DESIGN R15): levels k..k+W scan only the near list
constexpr int64_t kNearMin = 1 << 17;  // alive vertices (all ranks) from which a FULL scan builds one
constexpr int kSmall = 64;             // longer rows are walked through the chunk queue
constexpr unsigned kFull = 0xffffffffu;

struct Ctl {  // rank 0's copy is the global control block
    alignas(128) unsigned int bar_count;
    alignas(128) unsigned int bar_gen;
    alignas(128) int min_next;
    alignas(128) unsigned long long pushed;  // vertices removed so far (scan + crossings + isolated)
    alignas(128) unsigned long long arcs;
    alignas(128) int snap_min;
    unsigned long long snap_pushed;
    unsigned long long snap_prev;  // pushed at the previous barrier
    int snap_par;
    alignas(128) int abort;        // watchdog: a CTA waited past the deadline (every CTA leaves)
};

struct RankLocal {
    const int64_t *rp;     // local rowptr (rp[0] = rp0)
    int64_t rp0;
    const int32_t *ci;     // colidx of the owned rows (index rp[i] - rp0)
    int32_t *core;         // core_out of the owned range
    int32_t *alive[2];     // per-CTA segments [G][seg_cap] of owned local ids
    int32_t *seglen[2];    // [G]
    int64_t seg_cap;
    unsigned long long *chunk;  // long-row chunks: (epoch << 44) | ((len-1) << 36) | begin, one atomic word
    int64_t chunk_cap;
    unsigned long long *lctl;  // rank-local cursors: [0] item pop [1] items done [2] chunk tail [3] chunk pop
    int64_t nl;
};

struct Args {
    int PL;      // ranks in this launch (virtual: P, NCCL: 1)
    int P;       // ranks in total
    int G;       // CTAs per rank
    int rank0;   // global rank of the launch's first rank
    int sys;     // 1: peers are other GPUs (system-scope atomics and fences)
    int pad;
    int64_t n;
    int64_t vb[kMaxR + 1];
    char *peer[kMaxR];  // window base of every rank (virtual; NCCL: peer_dev)
    char *const *peer_dev;
    int64_t off_tail, off_deg, off_in0, off_in1, in_cap;
    int64_t off_near0, off_near1;  // near lists [2][nl_max] (their tails follow the inbox tails)
    int64_t *stats;     // [0] levels [1] sub-rounds [2] barriers [3] kmax [4] arcs
    int64_t timeout_ns; // watchdog: a wait longer than this aborts the call (KCORE_ECUDA), 0 = none
    int64_t *trace;     // optional [trace_cap][8]: {globaltimer, phase (0 init 1 scan 2 peel), k, pushed,
                        //  block 0's peel: items done, chunks done, end}
    int64_t trace_cap;
    RankLocal R[kMaxPL];
};

struct Smem {
    char *peer[kMaxR];
    int64_t vb[kMaxR + 1];
    int red_min[kWarps];
    int kcur;
    unsigned long long snap_pushed, snap_prev;
    int snap_min, snap_par;
    float inv_n;  // P / n
    unsigned long long deadline;  // globaltimer deadline of the watchdog
    int aborted;
    int th1;      // theta + 1 of the running near epoch (INT_MIN: none): walks append theta+1 -> theta crossings
    int near_cur; // near[near_cur] is the list the next near scan reads (and walks append to)
};

// ------------------------------------------------------------ scoped atomics
__device__ __forceinline__ int atom_sub(int32_t *p, bool sys)
{
    return sys ? atomicSub_system(p, 1) : atomicSub(p, 1);
}
__device__ __forceinline__ void red_add(int32_t *p, int32_t v, bool sys)
{
    if (sys) atomicAdd_system(p, v);
    else atomicAdd(p, v);
}
__device__ __forceinline__ unsigned long long atom_add64(unsigned long long *p, unsigned long long v, bool sys)
{
    return sys ? atomicAdd_system(p, v) : atomicAdd(p, v);
}
__device__ __forceinline__ void atom_min(int *p, int v, bool sys)
{
    if (sys) atomicMin_system(p, v);
    else atomicMin(p, v);
}
__device__ __forceinline__ void fence(bool sys)
{
    if (sys) __threadfence_system();
    else __threadfence();
}
__device__ __forceinline__ unsigned ld_volatile_u32(const unsigned *p) { return *(const volatile unsigned *)p; }

__device__ __forceinline__ int owner_of(const Smem &sm, int P, int64_t n, int32_t u)
{
    if (P == 1) return 0;
    int r = min(P - 1, (int)((float)u * sm.inv_n));  // estimate, corrected below
    while (r > 0 && u < sm.vb[r]) r--;
    while (r + 1 < P && u >= sm.vb[r + 1]) r++;
    return r;
}

__device__ __forceinline__ Ctl *gctl(const Smem &sm) { return (Ctl *)sm.peer[0]; }
__device__ __forceinline__ int32_t *deg_of(const Args &A, const Smem &sm, int r) { return (int32_t *)(sm.peer[r] + A.off_deg); }
__device__ __forceinline__ int32_t *inbox_of(const Args &A, const Smem &sm, int r, int which)
{
    return (int32_t *)(sm.peer[r] + (which ? A.off_in1 : A.off_in0));
}
__device__ __forceinline__ unsigned long long *tail_of(const Args &A, const Smem &sm, int r, int which)
{
    return (unsigned long long *)(sm.peer[r] + A.off_tail) + which;
}
__device__ __forceinline__ int32_t *near_of(const Args &A, const Smem &sm, int r, int which)
{
    return (int32_t *)(sm.peer[r] + (which ? A.off_near1 : A.off_near0));
}
__device__ __forceinline__ unsigned long long *ntail_of(const Args &A, const Smem &sm, int r, int which)
{
    return (unsigned long long *)(sm.peer[r] + A.off_tail) + 2 + which;
}

// Device barrier over every CTA of every rank, two-level: the CTAs of a rank
// arrive on a rank-local counter; the rank's last arriver resets the rank's
// cursors (and the consumed inbox tail `reset_par` when >= 0) and arrives on
// rank 0's global counter (P arrivals); the global last arriver snapshots the
// counters and releases the generation; each rank's last arriver copies the
// snapshot into rank-local memory and releases its own CTAs.  mode 0 (INIT):
// always take the level minimum; mode 1: take it (and end the level) only if
// nothing was pushed since the previous barrier.
enum : int { L_POP = 0, L_DONE = 1, L_CTAIL = 2, L_CPOP = 3, L_BAR = 4, L_GEN = 5, L_SPUSH = 6, L_SPREV = 7,
             L_SMIN = 8, L_ABORT = 9 };

// Watchdog of every wait (the multi-GPU protocol has not run on several GPUs
// yet): past the deadline, or once any CTA gave up, the waiter leaves, the
// kernel returns and the host reports KCORE_ECUDA instead of hanging.
__device__ __noinline__ bool watchdog(const Args &A, Smem &sm)
{
    if (A.timeout_ns <= 0) return false;
    Ctl *c = (Ctl *)sm.peer[0];
    if (*(volatile int *)&c->abort) return true;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t > sm.deadline) {
        *(volatile int *)&c->abort = 1;
        return true;
    }
    return false;
}

// deadline check at a barrier's entry (no memory traffic: the local deadline only)
__device__ __forceinline__ bool past_deadline(const Args &A, const Smem &sm)
{
    if (A.timeout_ns <= 0) return false;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t > sm.deadline;
}

// Virtual ranks (one launch holds every rank): a single-level barrier over all
// P*G CTAs; the last arriver resets every rank's cursors itself.
__device__ void gbar_flat(const Args &A, Smem &sm, int reset_par, int mode, int near_reset)
{
    __syncthreads();
    if (threadIdx.x == 0 && past_deadline(A, sm)) {  // leave without arriving: every waiter times out too
        *(volatile int *)&gctl(sm)->abort = 1;
        sm.aborted = 1;
    }
    if (threadIdx.x == 0 && !sm.aborted) {
        Ctl *c = gctl(sm);
        const unsigned gen = ld_volatile_u32(&c->bar_gen);
        __threadfence();
        const unsigned t = atomicAdd(&c->bar_count, 1u);
        if (t == (unsigned)(A.P * A.G - 1)) {
            __threadfence();
            const unsigned long long pushed = *(volatile unsigned long long *)&c->pushed;
            c->snap_prev = c->snap_pushed;
            c->snap_pushed = pushed;
            if (mode == 0 || pushed == c->snap_prev) {
                c->snap_min = *(volatile int *)&c->min_next;
                c->min_next = INT_MAX;
            }
            for (int r = 0; r < A.PL; r++) {
                unsigned long long *lc = A.R[r].lctl;
                lc[L_POP] = lc[L_DONE] = lc[L_CTAIL] = lc[L_CPOP] = 0ULL;
                if (reset_par >= 0) *tail_of(A, sm, A.rank0 + r, reset_par) = 0ULL;
                if (near_reset >= 0) *ntail_of(A, sm, A.rank0 + r, near_reset) = 0ULL;
            }
            c->bar_count = 0u;
            __threadfence();
            *(volatile unsigned *)&c->bar_gen = gen + 1u;
        } else {
            for (unsigned it = 1; ld_volatile_u32(&c->bar_gen) == gen; it++) {
                if ((it & 1023u) == 0u && watchdog(A, sm)) { sm.aborted = 1; break; }
            }
            __threadfence();
        }
        sm.snap_pushed = *(volatile unsigned long long *)&c->snap_pushed;
        sm.snap_prev = *(volatile unsigned long long *)&c->snap_prev;
        sm.snap_min = *(volatile int *)&c->snap_min;
    }
    __syncthreads();
}

__device__ void gbar(const Args &A, Smem &sm, int rl, int reset_par, int mode, int near_reset = -1)
{
    if (A.PL == A.P) {
        gbar_flat(A, sm, reset_par, mode, near_reset);
        return;
    }
    __syncthreads();
    if (threadIdx.x == 0 && past_deadline(A, sm)) {
        *(volatile int *)&gctl(sm)->abort = 1;
        sm.aborted = 1;
    }
    if (threadIdx.x == 0 && !sm.aborted) {
        const bool sys = A.sys;
        unsigned long long *lc = A.R[rl].lctl;
        const unsigned long long lgen = *(volatile unsigned long long *)&lc[L_GEN];
        __threadfence();
        fence(sys);
        const unsigned long long lt = atomicAdd(&lc[L_BAR], 1ULL);
        if (lt == (unsigned long long)(A.G - 1)) {  // the rank's last arriver
            lc[L_BAR] = 0ULL;
            lc[L_POP] = lc[L_DONE] = lc[L_CTAIL] = lc[L_CPOP] = 0ULL;
            if (reset_par >= 0) *tail_of(A, sm, A.rank0 + rl, reset_par) = 0ULL;
            if (near_reset >= 0) *ntail_of(A, sm, A.rank0 + rl, near_reset) = 0ULL;
            Ctl *c = gctl(sm);
            const unsigned gen = ld_volatile_u32(&c->bar_gen);
            fence(sys);
            const unsigned t = sys ? atomicAdd_system(&c->bar_count, 1u) : atomicAdd(&c->bar_count, 1u);
            if (t == (unsigned)(A.P - 1)) {  // the global last arriver
                fence(sys);
                const unsigned long long pushed = *(volatile unsigned long long *)&c->pushed;
                c->snap_prev = c->snap_pushed;
                c->snap_pushed = pushed;
                if (mode == 0 || pushed == c->snap_prev) {  // nothing pushed: the level is over
                    c->snap_min = *(volatile int *)&c->min_next;
                    c->min_next = INT_MAX;
                }
                c->bar_count = 0u;
                fence(sys);
                *(volatile unsigned *)&c->bar_gen = gen + 1u;
            } else {
                for (unsigned it = 1; ld_volatile_u32(&c->bar_gen) == gen; it++) {
                    if ((it & 1023u) == 0u && watchdog(A, sm)) { sm.aborted = 1; break; }
                }
                fence(sys);
            }
            lc[L_SPUSH] = *(volatile unsigned long long *)&c->snap_pushed;
            lc[L_SPREV] = *(volatile unsigned long long *)&c->snap_prev;
            lc[L_SMIN] = (unsigned long long)(uint32_t)*(volatile int *)&c->snap_min;
            __threadfence();
            *(volatile unsigned long long *)&lc[L_GEN] = lgen + 1ULL;
        } else {
            for (unsigned it = 1; *(volatile unsigned long long *)&lc[L_GEN] == lgen; it++) {
                if ((it & 1023u) == 0u && watchdog(A, sm)) { sm.aborted = 1; break; }
            }
            __threadfence();
        }
        sm.snap_pushed = *(volatile unsigned long long *)&lc[L_SPUSH];
        sm.snap_prev = *(volatile unsigned long long *)&lc[L_SPREV];
        sm.snap_min = (int)(uint32_t)*(volatile unsigned long long *)&lc[L_SMIN];
    }
    __syncthreads();
}

// warp-aggregated count of pushes into the global pushed counter
__device__ __forceinline__ void count_pushed(const Args &A, const Smem &sm, unsigned cnt)
{
    const unsigned tot = __reduce_add_sync(kFull, cnt);
    if ((threadIdx.x & 31) == 0 && tot) atom_add64(&gctl(sm)->pushed, (unsigned long long)tot, A.sys);
}

// ---------------------------------------------------------------- INIT
__device__ void phase_init(const Args &A, Smem &sm, int rl, int b)
{
    const RankLocal &R = A.R[rl];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int32_t *deg = deg_of(A, sm, A.rank0 + rl);
    const int64_t lo = R.nl * b / A.G, hi = R.nl * (b + 1) / A.G;
    int32_t *dst = R.alive[0] + (int64_t)b * R.seg_cap;
    if (threadIdx.x == 0) sm.kcur = 0;
    __syncthreads();
    int lmin = INT_MAX;
    unsigned iso = 0;
    for (int64_t base = lo; base < hi; base += kBlk) {
        const int64_t i = base + threadIdx.x;
        int32_t d = -1;
        if (i < hi) {
            d = (int32_t)(R.rp[i + 1] - R.rp[i]);
            deg[i] = d > 0 ? d : kRemoved;
            if (d == 0) { R.core[i] = 0; iso++; }
            else lmin = min(lmin, d);
        }
        const bool keep = d > 0;
        const unsigned bal = __ballot_sync(kFull, keep);
        int pos = 0;
        if (lane == 0 && bal) pos = atomicAdd(&sm.kcur, __popc(bal));
        pos = __shfl_sync(kFull, pos, 0);
        if (keep) dst[pos + __popc(bal & ((1u << lane) - 1u))] = (int32_t)i;
    }
    count_pushed(A, sm, iso);
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(kFull, lmin, o));
    if (lane == 0) sm.red_min[wib] = lmin;
    __syncthreads();
    if (threadIdx.x == 0) {
        int m = INT_MAX;
        for (int w = 0; w < kWarps; w++) m = min(m, sm.red_min[w]);
        if (m != INT_MAX) atom_min(&gctl(sm)->min_next, m, A.sys);
        R.seglen[0][b] = sm.kcur;
    }
    __syncthreads();
}

// ---------------------------------------------------------------- SCAN (Alg. 2)
// mode 0: FULL scan of the alive segments; 1: FULL scan that also builds the
// next near list (k < deg <= theta into near[near_cur ^ 1]); 2: near scan (the
// rank's near[near_cur] split over its CTAs, survivors into near[near_cur ^ 1]).
__device__ void phase_scan(const Args &A, Smem &sm, int rl, int b, int k, int sel, int par, int mode, int theta)
{
    const RankLocal &R = A.R[rl];
    const int me = A.rank0 + rl;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    int32_t *deg = deg_of(A, sm, me);
    int32_t *inbox = inbox_of(A, sm, me, par);
    unsigned long long *tail = tail_of(A, sm, me, par);
    const int32_t *src;
    int32_t *dst = nullptr;
    int64_t lo = 0, hi;
    if (mode == 2) {
        const int64_t L = (int64_t)*(volatile unsigned long long *)ntail_of(A, sm, me, sm.near_cur);
        src = near_of(A, sm, me, sm.near_cur);
        lo = L * b / A.G;
        hi = L * (b + 1) / A.G;
    } else {
        src = R.alive[sel] + (int64_t)b * R.seg_cap;
        dst = R.alive[sel ^ 1] + (int64_t)b * R.seg_cap;
        hi = R.seglen[sel][b];
    }
    int32_t *ndst = mode ? near_of(A, sm, me, sm.near_cur ^ 1) : nullptr;
    unsigned long long *ntail = mode ? ntail_of(A, sm, me, sm.near_cur ^ 1) : nullptr;
    if (threadIdx.x == 0) sm.kcur = 0;
    __syncthreads();
    int lmin = INT_MAX;
    unsigned pushed = 0;
    for (int64_t base = lo; base < hi; base += kBlk) {
        const int64_t i = base + threadIdx.x;
        int32_t v = -1, d = kDead;
        if (i < hi) { v = src[i]; d = deg[v]; }
        const bool fr = d <= k;               // alive (< kDead) and in the k-shell
        const bool keep = d > k && d < kDead;
        if (keep) lmin = min(lmin, d);
        if (mode) {  // near list: k < deg <= theta
            const bool nk = keep && d <= theta;
            const unsigned bn = __ballot_sync(kFull, nk);
            if (bn) {
                unsigned long long p2 = 0;
                if (lane == 0) p2 = atomicAdd(ntail, (unsigned long long)__popc(bn));
                p2 = __shfl_sync(kFull, p2, 0);
                if (nk) ndst[p2 + __popc(bn & ((1u << lane) - 1u))] = v;
            }
        }
        if (fr) { deg[v] = d + kRemoved; R.core[v] = k; }
        // frontier -> own inbox (local append), survivors -> compacted segment
        const unsigned bf = __ballot_sync(kFull, fr);
        if (bf) {
            unsigned long long p0 = 0;
            if (lane == 0) p0 = atomicAdd(tail, (unsigned long long)__popc(bf));
            p0 = __shfl_sync(kFull, p0, 0);
            if (fr) inbox[p0 + __popc(bf & ((1u << lane) - 1u))] = v;
            pushed += lane == 0 ? __popc(bf) : 0;
        }
        const unsigned bk = __ballot_sync(kFull, keep && dst != nullptr);
        if (bk) {
            int p1 = 0;
            if (lane == 0) p1 = atomicAdd(&sm.kcur, __popc(bk));
            p1 = __shfl_sync(kFull, p1, 0);
            if (keep) dst[p1 + __popc(bk & ((1u << lane) - 1u))] = v;
        }
    }
    count_pushed(A, sm, pushed);
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(kFull, lmin, o));
    if (lane == 0) sm.red_min[wib] = lmin;
    __syncthreads();
    if (threadIdx.x == 0) {
        int m = INT_MAX;
        for (int w = 0; w < kWarps; w++) m = min(m, sm.red_min[w]);
        if (m != INT_MAX) atom_min(&gctl(sm)->min_next, m, A.sys);
        if (mode != 2) R.seglen[sel ^ 1][b] = sm.kcur;
    }
    __syncthreads();
}

// Decrements (Alg. 3 l.19-24) of up to 4 targets per lane in their owners'
// windows: all four atomics are issued before any result is used (one round
// trip per batch, not four); the crossing k+1 -> k is seen once per target:
// mark it removed and append it to the owner's next inbox.
__device__ __forceinline__ unsigned dec_targets4(const Args &A, const Smem &sm, const int32_t (&u)[4], int k, int par,
                                                 int &lmin)
{
    int32_t *p[4];
    int o[4];
    int32_t lu[4];
#pragma unroll
    for (int r = 0; r < 4; r++) {
        o[r] = u[r] >= 0 ? owner_of(sm, A.P, A.n, u[r]) : 0;
        lu[r] = u[r] >= 0 ? (int32_t)(u[r] - sm.vb[o[r]]) : 0;
        p[r] = deg_of(A, sm, o[r]) + lu[r];
    }
    int old[4];
#pragma unroll
    for (int r = 0; r < 4; r++) old[r] = u[r] >= 0 ? atom_sub(p[r], A.sys) : INT_MIN;
    unsigned hits = 0;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        if (old[r] == k + 1) {
            red_add(p[r], kRemoved, A.sys);  // removed: later decrements are ignored
            const unsigned long long pos = atom_add64(tail_of(A, sm, o[r], par ^ 1), 1ULL, A.sys);
            inbox_of(A, sm, o[r], par ^ 1)[pos] = lu[r];
            hits++;
        } else if (old[r] > k + 1 && old[r] < kDead) {
            lmin = min(lmin, old[r] - 1);
            if (old[r] == sm.th1) {  // theta+1 -> theta: the target joins its owner's near list
                const unsigned long long pos = atom_add64(ntail_of(A, sm, o[r], sm.near_cur), 1ULL, A.sys);
                near_of(A, sm, o[r], sm.near_cur)[pos] = lu[r];
            }
        }
    }
    return hits;
}

// Walk arcs [a, e) of one owned row with the whole warp; the next batch's
// colidx loads are in flight while this batch's atomics complete.
__device__ __forceinline__ void walk_arcs(const Args &A, Smem &sm, const RankLocal &R, int64_t a, int64_t e, int k,
                                          int par, int &lmin, unsigned long long &walked, unsigned &pushed)
{
    const int lane = threadIdx.x & 31;
    walked += (unsigned long long)(e - a);
    int32_t un[4];
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const int64_t x = a + r * 32 + lane;
        un[r] = x < e ? __ldg(R.ci + x) : -1;
    }
    for (; a < e; a += 128) {
        int32_t u[4];
#pragma unroll
        for (int r = 0; r < 4; r++) u[r] = un[r];
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const int64_t x = a + 128 + r * 32 + lane;
            un[r] = x < e ? __ldg(R.ci + x) : -1;
        }
        pushed += dec_targets4(A, sm, u, k, par, lmin);
    }
}

// Walk the rows of up to 32 items at once (one per lane: row begin b, length
// d, exclusive prefix pre over the lanes, total T): 128 arcs per step, each
// arc finds its row with a 5-step shuffle search -- short rows fill the lanes.
__device__ __forceinline__ void walk_rows32(const Args &A, Smem &sm, const RankLocal &R, int64_t b, int32_t pre,
                                            int32_t T, int k, int par, int &lmin, unsigned long long &walked,
                                            unsigned &pushed)
{
    const int lane = threadIdx.x & 31;
    walked += (unsigned long long)T;
    for (int32_t a = 0; a < T; a += 128) {
        int32_t u[4];
#pragma unroll
        for (int r = 0; r < 4; r++) {
            const int32_t x = a + r * 32 + lane;
            int pos = 0;
#pragma unroll
            for (int bs = 16; bs >= 1; bs >>= 1) {
                const int32_t q = __shfl_sync(kFull, pre, pos + bs);
                if (q <= x) pos += bs;
            }
            const int64_t rb = __shfl_sync(kFull, b, pos);
            const int32_t rq = __shfl_sync(kFull, pre, pos);
            u[r] = x < T ? __ldg(R.ci + rb + (x - rq)) : -1;
        }
        pushed += dec_targets4(A, sm, u, k, par, lmin);
    }
}

// ---------------------------------------------------------------- sub-round
// The rank's warps pop 32 inbox items at a time and walk the short rows
// (<= kSmall arcs) together; longer rows are cut into chunks of <= kChunk arcs
// that every warp of the rank walks once the items are exhausted.
__device__ __forceinline__ void peel_mark(const Args &A, int64_t rec, int slot)
{
    if (A.trace && blockIdx.x == 0 && (threadIdx.x & 31) == 0 && rec < A.trace_cap) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        atomicMax((unsigned long long *)(A.trace + 8 * rec + slot), t);
    }
}

__device__ void phase_peel(const Args &A, Smem &sm, int rl, int k, int par, int epoch, int64_t rec)
{
    const RankLocal &R = A.R[rl];
    const int me = A.rank0 + rl;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int32_t *inbox = inbox_of(A, sm, me, par);
    const int64_t size = (int64_t)*(volatile unsigned long long *)tail_of(A, sm, me, par);
    unsigned long long *lc = R.lctl;
    int lmin = INT_MAX;
    unsigned long long walked = 0;
    unsigned pushed = 0;  // counted into the global pushed counter once, at the end
    while (true) {  // items, 32 per pop
        int64_t i0 = 0;
        if (lane == 0) i0 = (int64_t)atomicAdd(&lc[0], 32ULL);
        i0 = __shfl_sync(kFull, i0, 0);
        if (i0 >= size) break;
        const int64_t idx = i0 + lane;
        int64_t b = 0, e = 0;
        if (idx < size) {
            const int32_t v = inbox[idx];
            R.core[v] = k;
            b = R.rp[v] - R.rp0;
            e = R.rp[v + 1] - R.rp0;
        }
        // rows longer than kSmall go through the chunk queue (every warp of the rank shares them)
        const int64_t dl = e - b;
        const bool big = dl > kSmall;
        // publish every chunk of the warp's long rows at once: one reservation,
        // all lanes writing, one fence, then the tags
        const int32_t nch = big ? (int32_t)((dl + kChunk - 1) / kChunk) : 0;
        int32_t cincl = nch;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int32_t t = __shfl_up_sync(kFull, cincl, o);
            if (lane >= o) cincl += t;
        }
        const int32_t ctot = __shfl_sync(kFull, cincl, 31);
        if (ctot > 0) {
            unsigned long long c0 = 0;
            if (lane == 0) c0 = atomicAdd(&lc[2], (unsigned long long)ctot);
            c0 = __shfl_sync(kFull, c0, 0);
            const int32_t cpre = cincl - nch;
            for (int32_t q0 = 0; q0 < ctot; q0 += 32) {
                const int32_t q = q0 + lane;
                int pos = 0;
#pragma unroll
                for (int bs = 16; bs >= 1; bs >>= 1) {
                    const int32_t x = __shfl_sync(kFull, cpre, pos + bs);
                    if (x <= q) pos += bs;
                }
                const int64_t bj = __shfl_sync(kFull, b, pos), ej = __shfl_sync(kFull, e, pos);
                const int32_t qj = q - __shfl_sync(kFull, cpre, pos);
                if (q < ctot) {  // descriptor and publication are one atomic word: no fence
                    const int64_t cb = bj + (int64_t)qj * kChunk;
                    const int len = (int)min((int64_t)kChunk, ej - cb);
                    atomicExch(&R.chunk[c0 + q], ((unsigned long long)epoch << 44) |
                                                     ((unsigned long long)(len - 1) << 36) | (unsigned long long)cb);
                }
            }
        }
        __syncwarp();
        if (lane == 0) atomicAdd(&lc[1], (unsigned long long)min((int64_t)32, size - i0));  // chunks published
        const int32_t d = big ? 0 : (int32_t)dl;
        int32_t incl = d;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int32_t t = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += t;
        }
        const int32_t T = __shfl_sync(kFull, incl, 31);
        if (T > 0) walk_rows32(A, sm, R, b, incl - d, T, k, par, lmin, walked, pushed);
    }
    peel_mark(A, rec, 4);
    while (true) {  // chunks of long rows
        unsigned long long w = 0ULL;
        bool done = false;
        if (lane == 0) {
            const int64_t c = (int64_t)atomicAdd(&lc[3], 1ULL);
            unsigned spins = 0;
            while (true) {
                const unsigned long long tail = *(volatile unsigned long long *)&lc[2];
                if ((unsigned long long)c < tail) {
                    bool gone = false;
                    for (unsigned it = 1; ((w = atomicAdd(&R.chunk[c], 0ULL)) >> 44) != (unsigned long long)epoch; it++) {
                        __nanosleep(20);
                        if ((it & 1023u) == 0u && watchdog(A, sm)) { gone = true; break; }
                    }
                    if (gone) { sm.aborted = 1; done = true; }
                    break;
                }
                if (*(volatile unsigned long long *)&lc[1] >= (unsigned long long)size &&
                    *(volatile unsigned long long *)&lc[2] <= (unsigned long long)c) {
                    done = true;
                    break;
                }
                __nanosleep(64);  // back off: idle warps must not slow the working ones down
                if ((++spins & 255u) == 0u && watchdog(A, sm)) { sm.aborted = 1; done = true; break; }
            }
        }
        done = __shfl_sync(kFull, done, 0);
        if (done) break;
        w = __shfl_sync(kFull, w, 0);
        const int64_t cb = (int64_t)(w & ((1ULL << 36) - 1ULL));
        const int len = (int)((w >> 36) & 255ULL) + 1;
        walk_arcs(A, sm, R, cb, cb + len, k, par, lmin, walked, pushed);
    }
    peel_mark(A, rec, 5);
    count_pushed(A, sm, pushed);  // before the barrier reads the counter
    if (A.trace && (threadIdx.x & 31) == 0 && rec < A.trace_cap && walked) {  // latest end of any walking warp
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        atomicMax((unsigned long long *)(A.trace + 8 * rec + 7), t);
    }
    for (int o = 16; o > 0; o >>= 1) lmin = min(lmin, __shfl_xor_sync(kFull, lmin, o));
    if (lane == 0) sm.red_min[wib] = lmin;
    if (lane == 0 && walked) atom_add64(&gctl(sm)->arcs, walked, A.sys);
    __syncthreads();
    if (threadIdx.x == 0) {
        int m = INT_MAX;
        for (int w = 0; w < kWarps; w++) m = min(m, sm.red_min[w]);
        if (m != INT_MAX) atom_min(&gctl(sm)->min_next, m, A.sys);
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kBlk, 1) k_mgd(const __grid_constant__ Args A)
{
    __shared__ Smem sm;
    const int rl = blockIdx.x / A.G, b = blockIdx.x % A.G;
    if (threadIdx.x < kMaxR) sm.peer[threadIdx.x] = A.peer_dev ? A.peer_dev[threadIdx.x] : A.peer[threadIdx.x];
    if (threadIdx.x <= kMaxR) sm.vb[threadIdx.x] = A.vb[threadIdx.x];
    if (threadIdx.x == 0) {
        sm.inv_n = (float)A.P / (float)(A.n > 0 ? A.n : 1);
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        sm.deadline = t + (unsigned long long)A.timeout_ns;
        sm.aborted = 0;
    }
    __syncthreads();
    auto tr = [&](int64_t i, int ph, int k) {
        if (A.trace && blockIdx.x == 0 && threadIdx.x == 0 && i < A.trace_cap) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            int64_t *r = A.trace + 8 * i;
            r[0] = (int64_t)t; r[1] = ph; r[2] = k; r[3] = (int64_t)sm.snap_pushed;
        }
    };
    tr(0, -1, 0);
    phase_init(A, sm, rl, b);
    gbar(A, sm, rl, -1, 0);
    if (sm.aborted) { if (threadIdx.x == 0) A.R[rl].lctl[L_ABORT] = 1ULL; return; }
    tr(1, 0, 0);
    int k = -1, sel = 0, par = 0, epoch = 1;
    int64_t levels = sm.snap_pushed > 0 ? 1 : 0;  // the 0-shell (isolated vertices, removed at INIT)
    int64_t subrounds = 0, barriers = 1, kmax = 0, near_scans = 0;
    bool near_on = false;
    int theta = 0;
    if (threadIdx.x == 0) { sm.th1 = INT_MIN; sm.near_cur = 0; }
    __syncthreads();
    while (true) {
        if (sm.snap_pushed >= (unsigned long long)A.n) break;  // every vertex removed
        // level skip (R5); inside a near epoch every vertex outside the list has deg > theta
        k = near_on ? max(k + 1, min(sm.snap_min, theta + 1)) : max(k + 1, sm.snap_min);
        const unsigned long long before = sm.snap_pushed;
        int mode, near_reset = -1;
        if (near_on && k <= theta) {
            mode = 2;  // near scan: consumes near[cur]
            near_reset = sm.near_cur;
            near_scans++;
        } else {
            near_on = (int64_t)(A.n - (int64_t)sm.snap_pushed) >= kNearMin;  // uniform decision
            theta = near_on ? (int)min((int64_t)INT_MAX - 2, (int64_t)k + kNearW) : 0;
            mode = near_on ? 1 : 0;
            if (near_on) near_reset = sm.near_cur;  // the previous epoch's list is dropped
        }
        phase_scan(A, sm, rl, b, k, sel, par, mode, theta);
        if (mode != 2) sel ^= 1;
        gbar(A, sm, rl, -1, 1, near_reset);
        if (sm.aborted) { if (threadIdx.x == 0) A.R[rl].lctl[L_ABORT] = 1ULL; return; }
        if (threadIdx.x == 0) {
            if (mode) sm.near_cur ^= 1;  // the list this scan wrote is current; walks append to it
            sm.th1 = near_on ? theta + 1 : INT_MIN;
        }
        __syncthreads();
        barriers++;
        tr(barriers, 1, k);
        while (sm.snap_pushed != sm.snap_prev) {  // something was pushed: walk it
            phase_peel(A, sm, rl, k, par, 1 + (epoch++ % 0xfffff), barriers + 1);  // 20-bit epochs, never 0
            peel_mark(A, barriers + 1, 6);
            gbar(A, sm, rl, par, 1);  // the consumed inbox tail is reset by the rank's last arriver
            if (sm.aborted) { if (threadIdx.x == 0) A.R[rl].lctl[L_ABORT] = 1ULL; return; }
            par ^= 1;
            subrounds++;
            barriers++;
            tr(barriers, 2, k);
        }
        if (sm.snap_pushed > before) { levels++; kmax = k; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0 && A.stats) {
        A.stats[0] = levels;
        A.stats[1] = subrounds;
        A.stats[2] = barriers;
        A.stats[3] = kmax;
        A.stats[4] = (int64_t)*(volatile unsigned long long *)&gctl(sm)->arcs;
        A.stats[5] = near_scans;
    }
}

#if KC_HAVE_NCCL_WINDOWS
__global__ void k_mgd_peers(ncclWindow_t win, int P, char **out)
{
    const int p = threadIdx.x;
    if (p < P) out[p] = (char *)ncclGetPeerPointer(win, 0, p);
}
#endif

__global__ void k_mgd_ctl_init(char *base)
{
    Ctl *c = (Ctl *)base;
    if (threadIdx.x == 0) {
        memset(c, 0, sizeof(Ctl));
        c->min_next = INT_MAX;
        c->snap_min = INT_MAX;
    }
}

} // namespace mgd

namespace {

#define MGD_CK(x)                                                                      \
    do {                                                                               \
        cudaError_t e_ = (x);                                                          \
        if (e_ != cudaSuccess) {                                                       \
            rc = (e_ == cudaErrorMemoryAllocation) ? KCORE_ENOMEM : KCORE_ECUDA;       \
            goto out;                                                                  \
        }                                                                              \
    } while (0)

size_t al256(size_t x) { return (x + 255) & ~(size_t)255; }

struct Layout {
    int64_t off_tail, off_deg, off_in0, off_in1, off_near0, off_near1, in_cap;
    size_t bytes;
};

Layout window_layout(int64_t nl_max)
{
    Layout L;
    const int64_t nn = nl_max > 0 ? nl_max : 1;
    size_t off = al256(sizeof(mgd::Ctl));
    L.off_tail = (int64_t)off;
    off += 256;
    L.off_deg = (int64_t)off;
    off += al256(sizeof(int32_t) * (size_t)nn);
    L.off_in0 = (int64_t)off;
    off += al256(sizeof(int32_t) * (size_t)nn);
    L.off_in1 = (int64_t)off;
    off += al256(sizeof(int32_t) * (size_t)nn);
    L.off_near0 = (int64_t)off;
    off += al256(sizeof(int32_t) * (size_t)nn);
    L.off_near1 = (int64_t)off;
    off += al256(sizeof(int32_t) * (size_t)nn);
    L.in_cap = nn;
    L.bytes = off;
    return L;
}

// rank-local scratch (alive segments, chunk queue, cursors)
struct LocalScratch {
    void *mem = nullptr;
};

int setup_local(mgd::RankLocal &R, int G, int64_t m_local, cudaStream_t st, void **mem_out)
{
    int rc = KCORE_OK;
    const int64_t nl = R.nl;
    const int64_t seg_cap = (nl + G - 1) / G + 1;
    const int64_t chunk_cap = m_local / mgd::kChunk + (nl > 0 ? nl : 1) + 1;
    size_t off = 0;
    const size_t o_alive0 = off; off += al256(sizeof(int32_t) * (size_t)(seg_cap * G));
    const size_t o_alive1 = off; off += al256(sizeof(int32_t) * (size_t)(seg_cap * G));
    const size_t o_seg0 = off; off += al256(sizeof(int32_t) * (size_t)G);
    const size_t o_seg1 = off; off += al256(sizeof(int32_t) * (size_t)G);
    const size_t o_cb = off; off += al256(sizeof(unsigned long long) * (size_t)chunk_cap);
    const size_t o_lc = off; off += 256;
    char *m = nullptr;
    MGD_CK(cudaMallocAsync((void **)&m, off, st));
    MGD_CK(cudaMemsetAsync(m + o_cb, 0, sizeof(unsigned long long) * (size_t)chunk_cap, st));
    MGD_CK(cudaMemsetAsync(m + o_lc, 0, 256, st));  // rank-local cursors and barrier words
    R.alive[0] = (int32_t *)(m + o_alive0);
    R.alive[1] = (int32_t *)(m + o_alive1);
    R.seglen[0] = (int32_t *)(m + o_seg0);
    R.seglen[1] = (int32_t *)(m + o_seg1);
    R.seg_cap = seg_cap;
    R.chunk = (unsigned long long *)(m + o_cb);
    R.chunk_cap = chunk_cap;
    R.lctl = (unsigned long long *)(m + o_lc);
    *mem_out = m;
out:
    return rc;
}

int launch(mgd::Args &A, cudaStream_t st, kcore_stats *stats, int64_t *d_stats, int64_t launches,
           int64_t timeout_ns)
{
    int rc = KCORE_OK;
    // watchdog: no wait of the protocol may exceed a minute (tests may shorten it)
    A.timeout_ns = timeout_ns > 0 ? timeout_ns : (int64_t)60 * 1000000000LL;
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    int64_t hs[8] = {0};
    A.stats = d_stats;
    if (stats) {
        MGD_CK(cudaEventCreate(&e0));
        MGD_CK(cudaEventCreate(&e1));
        MGD_CK(cudaEventRecord(e0, st));
    }
    {
        void *args[] = {&A};
        MGD_CK(cudaLaunchCooperativeKernel((const void *)mgd::k_mgd, dim3(A.PL * A.G), dim3(mgd::kBlk), args, 0, st));
    }
    if (stats) {
        MGD_CK(cudaEventRecord(e1, st));
        MGD_CK(cudaMemcpyAsync(hs, d_stats, sizeof(hs), cudaMemcpyDeviceToHost, st));
        MGD_CK(cudaStreamSynchronize(st));
        float ms = 0.f;
        cudaEventElapsedTime(&ms, e0, e1);
        memset(stats, 0, sizeof(*stats));
        stats->levels = hs[0];
        stats->phases = hs[1];  // sub-rounds
        stats->barriers = hs[2];
        stats->kmax = (int32_t)hs[3];
        stats->arcs_walked = hs[4];
        stats->near_scans = hs[5];
        stats->grid_blocks = A.PL * A.G;
        stats->block_threads = mgd::kBlk;
        stats->kernel_ms = ms;
        stats->launches = launches;
    }
    {  // a CTA that hit the watchdog marked its rank: report an error, do not hang
        unsigned long long ab = 0;
        for (int r = 0; r < A.PL && !rc; r++) {
            MGD_CK(cudaMemcpyAsync(&ab, A.R[r].lctl + mgd::L_ABORT, sizeof(ab), cudaMemcpyDeviceToHost, st));
            MGD_CK(cudaStreamSynchronize(st));
            if (ab) rc = KCORE_ECUDA;
        }
        if (rc) goto out;
    }
out:
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    return rc;
}

} // namespace

static int64_t g_timeout_ns = 0;    // kcore_test_mgd_timeout: watchdog override (tests), 0 = default
static int64_t *g_trace = nullptr;  // kcore_test_mgd_trace: phase trace of the next call (dev aid)
static int64_t g_trace_cap = 0;

extern "C" int kcore_test_mgd_timeout(int64_t ns)
{
    g_timeout_ns = ns > 0 ? ns : 0;
    return KCORE_OK;
}

extern "C" int kcore_test_mgd_trace(int64_t *trace, int64_t cap)
{
    g_trace = trace;
    g_trace_cap = trace ? cap : 0;
    return KCORE_OK;
}

// P virtual ranks on this GPU: one window slab cut into P slices, one
// cooperative kernel with P rank groups of G CTAs.
int mgd_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                                 int32_t nranks, int32_t *core_out, void *stream_, kcore_stats *stats)
{
    using namespace mgd;
    if (n < 0 || n >= ((int64_t)1 << 31) || m < 0 || nranks < 1 || nranks > kMaxPL) return KCORE_EINVAL;
    if (n > 0 && (!rowptr || !core_out)) return KCORE_EINVAL;
    if (m > 0 && !colidx) return KCORE_EINVAL;
    if (stats) memset(stats, 0, sizeof(*stats));
    if (n == 0) return KCORE_OK;
    cudaStream_t st = (cudaStream_t)stream_;
    int rc = KCORE_OK;
    int dev = 0, sms = 0, occ = 0;
    char *slab = nullptr;
    int64_t *d_stats = nullptr;
    std::vector<void *> locals(nranks, nullptr);
    std::vector<int64_t> hrp(nranks + 1);
    Args *A = new Args();
    memset(A, 0, sizeof(Args));
    MGD_CK(cudaGetDevice(&dev));
    MGD_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    MGD_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mgd, kBlk, 0));
    if (occ < 1) { rc = KCORE_EUNSUPPORTED; goto out; }
    A->PL = A->P = nranks;
    A->G = sms * occ / nranks;
    if (A->G < 1) { rc = KCORE_EUNSUPPORTED; goto out; }
    A->rank0 = 0;
    A->sys = 0;
    A->n = n;
    for (int r = 0; r <= nranks; r++) A->vb[r] = (n * r) / nranks;
    for (int r = 0; r <= nranks; r++)
        MGD_CK(cudaMemcpyAsync(&hrp[r], rowptr + A->vb[r], sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    MGD_CK(cudaStreamSynchronize(st));
    {
        int64_t nl_max = 0;
        for (int r = 0; r < nranks; r++) nl_max = std::max<int64_t>(nl_max, A->vb[r + 1] - A->vb[r]);
        const Layout L = window_layout(nl_max);
        A->off_tail = L.off_tail; A->off_deg = L.off_deg; A->off_in0 = L.off_in0; A->off_in1 = L.off_in1;
        A->off_near0 = L.off_near0; A->off_near1 = L.off_near1;
        A->in_cap = L.in_cap;
        MGD_CK(cudaMallocAsync((void **)&slab, L.bytes * nranks, st));
        MGD_CK(cudaMemsetAsync(slab, 0, L.bytes * nranks, st));
        for (int r = 0; r < nranks; r++) A->peer[r] = slab + L.bytes * r;
        k_mgd_ctl_init<<<1, 32, 0, st>>>(slab);
        MGD_CK(cudaGetLastError());
    }
    for (int r = 0; r < nranks && !rc; r++) {
        RankLocal &R = A->R[r];
        R.rp = rowptr + A->vb[r];
        R.rp0 = hrp[r];
        R.ci = colidx + hrp[r];
        R.core = core_out + A->vb[r];
        R.nl = A->vb[r + 1] - A->vb[r];
        rc = setup_local(R, A->G, hrp[r + 1] - hrp[r], st, &locals[r]);
    }
    if (rc) goto out;
    MGD_CK(cudaMallocAsync((void **)&d_stats, sizeof(int64_t) * 8, st));
    A->trace = g_trace;
    A->trace_cap = g_trace_cap;
    rc = launch(*A, st, stats, d_stats, 2, g_timeout_ns);
out:
    for (void *p : locals) if (p) cudaFreeAsync(p, st);
    if (slab) cudaFreeAsync(slab, st);
    if (d_stats) cudaFreeAsync(d_stats, st);
    if (cudaStreamSynchronize(st) != cudaSuccess && !rc) rc = KCORE_ECUDA;
    delete A;
    return rc;
}

// One rank per process over NCCL symmetric memory (ncclMemAlloc +
// ncclCommWindowRegister; peers reached through ncclGetPeerPointer over
// NVLink).  Collective: every rank calls it.  Build-gated on NCCL >= 2.28.
int mgd_nccl(const int64_t *rowptr_local, const int32_t *colidx_local, int64_t n_global,
                              int64_t v_begin, int64_t v_end, int64_t m_local, int32_t *core_out_local,
                              void *stream_, void *nccl_comm, kcore_stats *stats)
{
#if !KC_HAVE_NCCL_WINDOWS
    (void)rowptr_local; (void)colidx_local; (void)n_global; (void)v_begin; (void)v_end; (void)m_local;
    (void)core_out_local; (void)stream_; (void)nccl_comm; (void)stats;
    return KCORE_EUNSUPPORTED;
#else
    using namespace mgd;
    if (!nccl_comm || n_global < 0 || n_global >= ((int64_t)1 << 31) || v_begin < 0 || v_end < v_begin ||
        v_end > n_global || m_local < 0)
        return KCORE_EINVAL;
    const int64_t nl = v_end - v_begin;
    if (nl > 0 && (!rowptr_local || !core_out_local)) return KCORE_EINVAL;
    if (m_local > 0 && !colidx_local) return KCORE_EINVAL;
    if (stats) memset(stats, 0, sizeof(*stats));
    cudaStream_t st = (cudaStream_t)stream_;
    ncclComm_t comm = (ncclComm_t)nccl_comm;
    int rc = KCORE_OK;
    int P = 0, rank = 0, dev = 0, sms = 0, occ = 0, ok_all = 0;
    void *win_mem = nullptr, *local_mem = nullptr;
    ncclWindow_t win = nullptr;
    int64_t *d_vb = nullptr, *d_stats = nullptr;
    int32_t *d_ok = nullptr;
    char **d_peer = nullptr;
    Args *A = new Args();
    memset(A, 0, sizeof(Args));
    if (ncclCommCount(comm, &P) != ncclSuccess || ncclCommUserRank(comm, &rank) != ncclSuccess) {
        rc = KCORE_ENCCL;
        goto out;
    }
    if (P > kMaxR) { rc = KCORE_EUNSUPPORTED; goto out; }
    MGD_CK(cudaGetDevice(&dev));
    MGD_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    MGD_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_mgd, kBlk, 0));
    // owner table (all-gather of v_begin) and a collective validity check:
    // every rank returns the same status (no rank left waiting in a barrier)
    MGD_CK(cudaMallocAsync((void **)&d_vb, sizeof(int64_t) * (P + 1), st));
    MGD_CK(cudaMallocAsync((void **)&d_ok, sizeof(int32_t), st));
    MGD_CK(cudaMemcpyAsync(d_vb + rank, &v_begin, sizeof(int64_t), cudaMemcpyHostToDevice, st));
    if (ncclAllGather(d_vb + rank, d_vb, 1, ncclInt64, comm, st) != ncclSuccess) { rc = KCORE_ENCCL; goto out; }
    MGD_CK(cudaMemcpyAsync(A->vb, d_vb, sizeof(int64_t) * P, cudaMemcpyDeviceToHost, st));
    MGD_CK(cudaStreamSynchronize(st));
    A->vb[P] = n_global;
    {
        int32_t mine = (A->vb[rank] == v_begin && A->vb[rank + 1] == v_end && A->vb[0] == 0 && occ >= 1) ? 1 : 0;
        MGD_CK(cudaMemcpyAsync(d_ok, &mine, sizeof(int32_t), cudaMemcpyHostToDevice, st));
        if (ncclAllReduce(d_ok, d_ok, 1, ncclInt32, ncclMin, comm, st) != ncclSuccess) { rc = KCORE_ENCCL; goto out; }
        MGD_CK(cudaMemcpyAsync(&ok_all, d_ok, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        MGD_CK(cudaStreamSynchronize(st));
        if (!ok_all) { rc = KCORE_EINVAL; goto out; }
    }
    {
        int64_t nl_max = 0;
        for (int r = 0; r < P; r++) nl_max = std::max<int64_t>(nl_max, A->vb[r + 1] - A->vb[r]);
        const Layout L = window_layout(nl_max);
        A->off_tail = L.off_tail; A->off_deg = L.off_deg; A->off_in0 = L.off_in0; A->off_in1 = L.off_in1;
        A->off_near0 = L.off_near0; A->off_near1 = L.off_near1;
        A->in_cap = L.in_cap;
        if (ncclMemAlloc(&win_mem, L.bytes) != ncclSuccess) { rc = KCORE_ENCCL; goto out; }
        MGD_CK(cudaMemsetAsync(win_mem, 0, L.bytes, st));
        if (rank == 0) k_mgd_ctl_init<<<1, 32, 0, st>>>((char *)win_mem);
        MGD_CK(cudaStreamSynchronize(st));
        if (ncclCommWindowRegister(comm, win_mem, L.bytes, &win, 0) != ncclSuccess) { rc = KCORE_ENCCL; goto out; }
        MGD_CK(cudaMallocAsync((void **)&d_peer, sizeof(char *) * kMaxR, st));
        MGD_CK(cudaMemsetAsync(d_peer, 0, sizeof(char *) * kMaxR, st));
        k_mgd_peers<<<1, kMaxR, 0, st>>>(win, P, d_peer);
        MGD_CK(cudaGetLastError());
        // every window is initialised before any rank's kernel starts
        if (ncclAllReduce(d_ok, d_ok, 1, ncclInt32, ncclMin, comm, st) != ncclSuccess) { rc = KCORE_ENCCL; goto out; }
        MGD_CK(cudaStreamSynchronize(st));
    }
    A->PL = 1;
    A->P = P;
    A->G = sms * occ;
    A->rank0 = rank;
    A->sys = 1;
    A->n = n_global;
    A->peer_dev = d_peer;
    {
        RankLocal &R = A->R[0];
        R.rp = rowptr_local;
        R.rp0 = 0;
        if (nl > 0) MGD_CK(cudaMemcpyAsync(&R.rp0, rowptr_local, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        MGD_CK(cudaStreamSynchronize(st));
        R.ci = colidx_local;
        R.core = core_out_local;
        R.nl = nl;
        rc = setup_local(R, A->G, m_local, st, &local_mem);
        if (rc) goto out;
    }
    MGD_CK(cudaMallocAsync((void **)&d_stats, sizeof(int64_t) * 8, st));
    rc = launch(*A, st, stats, d_stats, 3, g_timeout_ns);
out:
    if (cudaStreamSynchronize(st) != cudaSuccess && !rc) rc = KCORE_ECUDA;
    if (win) ncclCommWindowDeregister(comm, win);
    if (win_mem) ncclMemFree(win_mem);
    if (local_mem) cudaFree(local_mem);
    if (d_vb) cudaFree(d_vb);
    if (d_ok) cudaFree(d_ok);
    if (d_peer) cudaFree(d_peer);
    if (d_stats) cudaFree(d_stats);
    delete A;
    return rc;
#endif
}
