// kc_kernels.cuh -- sm_100a kernels of the k-core hot path (v3).
//
// One call = one persistent cooperative kernel (k_persistent), one CTA per SM,
// running the whole decomposition as a device-resident state machine.  Per
// level k (Alg. 1's round) there is ONE grid phase:
//
//   LEVEL(k)  every CTA scans its tiles of the alive list (Alg. 2):
//             deg[v] == k  -> v is in the k-shell: claim it, append it to the
//                             CTA's LOCAL frontier (shared memory);
//             deg[v] >  k  -> running min for the level skip, optional
//                             alive-list compaction;
//             then drains its local frontier breadth-first with CTA-local
//             sub-rounds (__syncthreads only) -- the paper's block-local BFS
//             of Alg. 3.  For every arc (v,u) (Alg. 3 l.19-24)
//             whose target passes the alive filter:
//               old = atomicSub(&deg[u],1)
//                  old == k+1 -> u reached k: claim it, core[u] = k, append it
//                                to the next local frontier
//                  old >  k+1 -> min_next = min(min_next, old-1)    (level skip)
//             deg is a private working array (reading R10): removed
//             targets take garbage decrements, so no restore (Fig. 6) is needed.
//   HUB       vertices too big for one CTA (> kHub arcs) or overflowing a
//             local frontier go to a global queue; a HUB phase splits that
//             queue's ARCS evenly over every warp of the grid, then drains
//             the resulting local frontiers the same way.
//   level end k <- max(k+1, min_next)  (Alg. 1 l.9 does k+1; reading R5)
//
// Scan and drain run concurrently in different CTAs, so a vertex can be seen
// with deg == k by a scan and reached (old == k+1) by a peel in the same
// level; a claim bit per vertex (atomicOr) makes removal exactly-once
// (reading R9).
//
// Control: every CTA keeps an identical copy of the control state in shared
// memory; a phase ends with a grid barrier whose last arriver snapshots and
// resets the counters, and every CTA applies the same pure advance().  Phases
// over a short alive list / few arcs run `solo` on CTA 0 with CTA-local sync.
//
// Filter: when a CTA has many arcs to walk and the alive list at level start
// is short, it builds a Bloom filter of that list in shared memory; arcs whose
// target is definitely not alive (removed at an earlier level) then skip the
// scattered deg[] read entirely (the read is the throughput limiter, see
// DESIGN.md "Measured primitives").
#pragma once

#include "kc_common.cuh"
#include <climits>

namespace kc {

#ifndef KC_BLOCK
#define KC_BLOCK 512
#endif
constexpr int kBlock = KC_BLOCK;
constexpr int kWarps = kBlock / 32;
#ifndef KC_SCAN_ITEMS
#define KC_SCAN_ITEMS 4
#endif
constexpr int kScanItems = KC_SCAN_ITEMS;        // alive-list entries per lane per warp step
constexpr int kLCap = kBlock;        // local frontier capacity (entries; one per thread in the prefix scan)
constexpr int kQCap = 1024;          // async drain: chunk queue capacity (chunks of <= 128 arcs)
constexpr int kAsyncNx = 2;          // route target "async chunk queue" (lists 0/1 are the sub-round lists)
// CTA-local routing budgets (arcs): a claimed vertex with more arcs than
// kHub, or one that would push the next local sub-round past kSub or the
// CTA's phase total past kPhase, goes to the global queue (HUB phase) instead
// of the CTA's own frontier (tuned on B200: DESIGN.md §8).
#ifndef KC_HUB
#define KC_HUB 8192
#endif
#ifndef KC_SUB
#define KC_SUB 32768
#endif
#ifndef KC_PHASE
#define KC_PHASE 65536
#endif
constexpr int kHub = KC_HUB, kSub = KC_SUB, kPhase = KC_PHASE;
#ifndef KC_GSTAGE
#define KC_GSTAGE 64
#endif
constexpr int kGStage = KC_GSTAGE;          // per-warp global-queue stage (any size; flushed 32 at a time)
#ifndef KC_BLOOM_LOG2
#define KC_BLOOM_LOG2 19
#endif
constexpr int kBloomBits = 1 << KC_BLOOM_LOG2;  // 64 KB: shared memory is taken from L1 (2^20 bits: C4 +5 %)
constexpr int kBloomWords = kBloomBits / 32;
#ifndef KC_BLOOM_MAXA
#define KC_BLOOM_MAXA (1 << 18)
#endif
constexpr int kBloomMaxA = KC_BLOOM_MAXA;  // build only for alive lists up to this length
constexpr int kUnroll = 4;  // arcs per lane in flight per batch (handle_hits assumes 4)
constexpr int kBatch = 32 * kUnroll;
constexpr int kTraceFields = 8;
// With the alive-set filter on (most removed targets never reach L2), walks
// may skip the deg pre-read and decrement every target that passes it: one
// scattered atomic instead of a read followed by an atomic on the same line.
// Removed targets then take garbage decrements -- harmless, their core was
// written when they were claimed (deg is a private working array).
#ifndef KC_ROUTE4
#define KC_ROUTE4 1
#endif
#ifndef KC_CF_HUB
#define KC_CF_HUB 0
#endif
#ifndef KC_CF_LOCAL
#define KC_CF_LOCAL 0
#endif
#ifndef KC_CF_LOCAL_MIN
#define KC_CF_LOCAL_MIN 0
#endif
#ifndef KC_HITS_INLINE
#define KC_HITS_INLINE 1
#endif
#ifndef KC_ROUTE4_INLINE
#define KC_ROUTE4_INLINE 1
#endif
#ifndef KC_SCAN_PIPE
#define KC_SCAN_PIPE 1
#endif
#ifndef KC_COMPACT_D
#define KC_COMPACT_D 32 // compact the alive list once >= 1/KC_COMPACT_D of it is dead
#endif
#ifndef KC_ASYNC
#define KC_ASYNC 2  // 1: CTA-local drain as an asynchronous chunk queue (no sub-round barriers);
                    // 2: per CTA and phase, async when the frontier's rows are long
#endif
#ifndef KC_ASYNC_MINAVG
#define KC_ASYNC_MINAVG 64  // KC_ASYNC 2: async when the local frontier averages >= this many arcs per vertex
#endif
#ifndef KC_FASTSUB
#define KC_FASTSUB 1
#endif
#ifndef KC_AO_HUB
#define KC_AO_HUB 1
#endif
#ifndef KC_AO_LOCAL
#define KC_AO_LOCAL 1
#endif
#ifndef KC_AO_ALWAYS
#define KC_AO_ALWAYS 1
#endif
// Heavy HUB phases with non-returning decrements (walk_red) followed by a
// rescan of the alive list at the same k: used when the phase walks at least
// KC_RED_MIN arcs and the alive set is at most 1/KC_RED_RATIO of them (the
// rescan then costs far less than the returns it saves).  0 disables.
#ifndef KC_RED_MIN
#define KC_RED_MIN (1 << 21)
#endif
#ifndef KC_RED_RATIO
#define KC_RED_RATIO 4
#endif
#ifndef KC_RED_UNROLL
#define KC_RED_UNROLL 8
#endif
// Near list: a FULL level scan over an alive list of at
// least KC_NEAR_MIN_A entries also collects every alive vertex with
// k < deg <= theta = k + W into a near list, and walks append a vertex when its
// decrement crosses theta+1 -> theta.  Levels k' <= theta then scan only the
// near list: every alive vertex of degree <= theta is in it, so the frontier
// (deg <= k') and the level-skip bound min(near min, walk min, theta+1) are
// exact.  W adapts per epoch (KC_NEAR_W initial).  0 disables.
#ifndef KC_NEAR_MIN_A
#define KC_NEAR_MIN_A (1 << 17)
#endif
#ifndef KC_NEAR_W
#define KC_NEAR_W 16
#endif
#ifndef KC_WALK_FAST
#define KC_WALK_FAST 1  // walk<>: a batch inside one row skips the per-arc entry search
#endif
#ifndef KC_HIT_BF
#define KC_HIT_BF 1  // decrement outcomes (hit mask, level-skip min) without per-arc branches
#endif
#ifndef KC_PRED_ATOM
#define KC_PRED_ATOM 1
#endif
#ifndef KC_BLOOM_BF
#define KC_BLOOM_BF 1  // Bloom probes without per-arc branches (C3 -0.9 %)
#endif
#ifndef KC_BLOOM_MULT
#define KC_BLOOM_MULT 1  // ... and only when it walks >= KC_BLOOM_MULT x the list's length
#endif
#ifndef KC_BLOOM_GATE
#define KC_BLOOM_GATE 1  // build the alive-set filter only when the CTA walks >= 1/KC_BLOOM_GATE of the list's length
#endif
#ifndef KC_TRACE
#define KC_TRACE 0  // 1: per-phase / per-CTA trace support (lib/libkcore_trace.so; the checks cost ~2-3 %)
#endif
#ifndef KC_SCAN_EC
#define KC_SCAN_EC 0  // 1 (ablation): level-scan compaction with block scans (Fig. 9) instead of warp ballots
#endif
#ifndef KC_NO_SMBUF
#define KC_NO_SMBUF 0  // 1 (ablation): no shared-memory frontier -- every claimed vertex goes to the global queue
#endif
#ifndef KC_NEAR
#define KC_NEAR 1  // 0: compile the near list out (walks never test for theta crossings)
#endif
#ifndef KC_ROUTE_FAST
#define KC_ROUTE_FAST 1  // route_won4: a single claimed vertex per warp takes a short path (C3 -1.5 %, C4 -1 %)
#endif
#ifndef KC_PUSH_PAR
#define KC_PUSH_PAR 1  // async-queue chunks of claimed rows are published by all 32 lanes
#endif
#ifndef KC_SPIN_LD
#define KC_SPIN_LD 0  // (measured: no gain) 1: idle warps of the async drain wait on their slot with plain loads
#endif
#ifndef KC_SPIN_NAP
#define KC_SPIN_NAP 0  // ns of __nanosleep between those polls
#endif
enum : int32_t { PH_INIT = 0, PH_LEVEL = 1, PH_HUB = 2, PH_DONE = 3 };

struct Ctrl {
    int32_t phase, solo, k, level_min;
    int32_t compact, src_sel, dst_sel, alive_sel;
    int32_t src_single, alive_single;  // 1: the list is one contiguous run in segment 0
    int32_t red;                       // HUB phase walks with non-returning decrements (then a rescan)
    int32_t near_app;                  // walks append theta+1 -> theta crossings to near[near_app] (-1: off)
    int64_t arcs_lvl0;                 // arcs walked when the level began
    int64_t st_near;                   // near-list level scans
    int64_t src_len, alive_len;
    int64_t s, e, as, ae;          // HUB: global-queue slots [s,e), arcs [as,ae)
    int64_t gq_cnt, gq_arc;        // global queue consumed so far
    int64_t ord_lvl0;              // order tail when the level began
    int64_t level;                 // level index (for the Bloom cache)
    int64_t st_levels, st_phases, st_solo, st_bar, st_scanned, st_compact, st_hubarcs;
    int32_t st_kmax, st_pad;
    // near-list state (KC_NEAR_MIN_A)
    int32_t near_on;     // an epoch is active: every alive vertex with deg <= theta is in near[near_cur]
    int32_t theta;
    int32_t near_cur;    // buffer holding the list the next near scan reads
    int32_t near_scan;   // this LEVEL phase scans near[near_cur] (compacting into near[near_cur ^ 1])
    int32_t near_build;  // this FULL LEVEL phase also collects k < deg <= theta into near[near_cur ^ 1]
    int32_t near_reset;  // buffer whose tail the barrier after this phase resets (-1: none)
    int32_t near_w;      // window W of the next epoch
    int32_t near_lv;     // near levels in the current epoch
    int64_t near_len;    // entries of near[near_cur] when this phase began
    int64_t near_first;  // near-list length at the epoch's first near scan
};

static_assert(sizeof(Ctrl) % 16 == 0, "Ctrl is copied as int4");

struct Snap {
    unsigned long long arcs;       // arcs walked so far
    unsigned long long gq;         // packed global-queue tail
    unsigned long long ord;        // order tail (= removed vertices)
    unsigned long long alive_out;  // compaction output length
    unsigned long long near[2];    // near-list tails
    int32_t min;
    int32_t pad;
};

struct Params {
    int64_t n;
    int32_t solo_arcs;  // HUB phases with <= this many arcs run solo
    int32_t solo_scan;  // LEVEL phases over <= this many entries run solo
    int32_t bloom;      // 0 disables the Bloom filter
    int16_t red;        // 0 disables non-returning heavy HUB walks (KC_RED_MIN)
    int16_t near;       // 0 disables the near list (KC_NEAR_MIN_A)
    int32_t near_min;   // alive-list length from which a FULL scan builds a near list
    int32_t near_w;     // initial near window W
};

struct State {
    alignas(128) unsigned long long gq_tail;    // packed (count << 33) | arcs
    alignas(128) unsigned long long ord_tail;   // vertices written to order[]
    alignas(128) unsigned long long alive_out;  // compaction output length
    alignas(128) int32_t min_next;              // atomicMin target
    alignas(128) uint32_t bar_count;            // grid barrier arrivals (monotone)
    alignas(128) uint32_t bar_gen;              // grid barrier generation
    Snap snap[2];                               // counters at barrier gen, by gen & 1
    alignas(128) unsigned long long arcs_walked;
    alignas(128) unsigned long long near_tail[2];  // near-list append cursors (one line)
    alignas(128) uint32_t scan_done;            // CTAs whose level scan of this phase is complete
    alignas(128) Ctrl pub;                      // Ctrl published by CTA 0 after a solo run
    alignas(128) Params prm;
    int64_t *trace;                             // optional [trace_cap][kTraceFields]
    int64_t *trace_cta;                         // optional [trace_cap][grid][8]
    int64_t trace_cap;
    unsigned long long trace_n;
};

struct KArgs {
    const int64_t *rowptr;
    const int32_t *colidx;
    int32_t *deg;       // working degrees (workspace): only decrease, garbage once removed
    int32_t *core;      // core_out: written once per vertex, when it is claimed at level k
    int32_t *order;     // removal order (all vertices)
    uint32_t *claimed;  // claim bit per vertex
    int32_t *gq_v;      // global queue: vertex, row begin, arc prefix
    int64_t *gq_beg;
    int64_t *gq_arc;
    int32_t *alive[2];  // alive lists, partitioned into nseg per-CTA segments
    int32_t *near[2];   // near lists (contiguous runs, global cursors S->near_tail)
    int32_t *seg_len[2];  // entries of segment b in alive[x]: seg_len[x][b]
    int64_t seg_R;        // segment region size: segment b lives at [b*R, b*R + len)
    int32_t nseg;         // = persistent grid size
    State *S;
    int64_t n;
};

struct Smem {
    union {
        struct {  // sub-round lists (synchronous drain)
            int32_t lv[2][kLCap];
            int32_t ld[2][kLCap];
            int64_t lb[2][kLCap];
            int64_t lpre[kLCap + 1];
        };
    };
    // Chunk queue of the asynchronous drain (KC_ASYNC): slot = one 64-bit word
    // published and consumed with shared-memory atomics -- colidx begin in bits
    // [0,34), chunk length - 1 in bits [34,41), bit 63 = valid; 0 = empty.  A
    // popper takes the word with atomicExch(slot, 0), so every slot is empty
    // again when the drain ends (qpend == 0 => every pushed chunk was popped).
    // Outside the union: the synchronous sub-round lists overwrite the union.
    unsigned long long qword[kQCap];
    int32_t lcnt[2];
    int32_t larc[2];
    int32_t lphase;      // local arcs accepted this phase
    int32_t removed;     // vertices removed by this CTA this phase (order not recorded)
    int32_t pad_fit;
    int32_t kcur;        // scan: compaction cursor within the current segment
    int32_t seg_cache[2];     // length of this CTA's own segment in alive[x], as it last wrote it
    int32_t seg_cache_ok[2];  // (persistent kernel only; a k_phase launch starts without it)
    int32_t bud_hub, bud_sub, bud_phase, bud_pad;  // routing budgets of this phase
    unsigned long long scan_q2[kWarps];
    unsigned long long tot_q2, base_g, base_w;
    int32_t gv[kWarps][kGStage];
    int32_t gd[kWarps][kGStage];
    int64_t gb[kWarps][kGStage];
    unsigned long long scan_q[kWarps];
    unsigned long long tot_q, base_o, base_k;
    int32_t red_min[kWarps];
    int64_t bloom_level;  // alive-list length the filter was built from
    int32_t bloom_on;
    Ctrl ctrl;
    Snap snap;
    int32_t qhead, qtail, qpend;
    int32_t near_th1;  // theta + 1 while walks feed a near list, else INT_MIN (set per phase)
    int32_t bloom_en;  // Params::bloom (kept in shared memory: no global load per phase)
    int32_t nclaim;    // 1: a level scan may still be running somewhere -- hits must claim (see handle_hits)
    int32_t spec;      // walks load the row bounds of every decremented target with its atomic (KC_SPEC)
    int64_t *tr_cta;   // per-CTA trace (kcore_options.trace_cta_out) or nullptr, and its capacity
    int64_t tr_cap;
    unsigned long long qwalked;
    uint32_t bloom[kBloomWords];
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

#ifdef KC_PROBE
// Development probe (variant builds only): {cta, tag, globaltimer, value}.
__device__ unsigned long long g_probe_n;
__device__ int64_t g_probe[(1 << 22) * 4];
#ifndef KC_PROBE_KMIN
#define KC_PROBE_KMIN 0
#endif
__shared__ int s_probe_k;
__shared__ unsigned s_probe_n;
constexpr int kProbePerCta = (1 << 22) / 160;
__device__ __forceinline__ void probe(int tag, int64_t val)
{
    if (*(volatile int *)&s_probe_k < KC_PROBE_KMIN) return;
    const int64_t t = (int64_t)globaltimer();
    const unsigned i = atomicAdd(&s_probe_n, 1u);
    if (i >= (unsigned)kProbePerCta) return;
    int64_t *r = g_probe + ((int64_t)blockIdx.x * kProbePerCta + i) * 4;
    r[0] = blockIdx.x; r[1] = tag; r[2] = t; r[3] = val;
}
#define PROBE(tag, val) probe(tag, val)
#ifdef KC_PROBE_W
#define PROBE_W(tag, val) probe(tag, val)
#else
#define PROBE_W(tag, val) ((void)0)
#endif
#else
#define PROBE_W(tag, val) ((void)0)
#define PROBE(tag, val) ((void)0)
#endif

__device__ __forceinline__ uint32_t bloom_h1(uint32_t v) { return (v * 0x9E3779B1u) >> (32 - KC_BLOOM_LOG2); }
__device__ __forceinline__ uint32_t bloom_h2(uint32_t v) { return ((v ^ (v >> 15)) * 0x85EBCA6Bu) >> (32 - KC_BLOOM_LOG2); }

__device__ __forceinline__ bool bloom_maybe(const Smem &sm, uint32_t v)
{
    const uint32_t a = bloom_h1(v), b = bloom_h2(v);
    return ((sm.bloom[a >> 5] >> (a & 31)) & (sm.bloom[b >> 5] >> (b & 31)) & 1u) != 0;
}

// Per-CTA timestamps of the current phase (trace mode only): slot 0 phase
// start, 1 end of scan / queue walk, 2 end of local drain, 3 barrier arrival.
// Indexed by the number of grid barriers passed (identical in every CTA).
// (the trace pointers are read from shared memory: a global load here would
// stall thread 0, and with it the CTA's next barrier, on every phase)
__device__ __forceinline__ void cta_time(const KArgs &A, const Smem &sm, int slot)
{
    const Ctrl &c = sm.ctrl;
    if (!KC_TRACE || threadIdx.x != 0 || c.solo || !sm.tr_cta || c.st_bar >= sm.tr_cap) return;
    sm.tr_cta[(c.st_bar * gridDim.x + blockIdx.x) * 8 + slot] = (int64_t)globaltimer();
}

// Per-CTA counters of the current phase (trace mode only): slot 4 local
// sub-rounds, 5 arcs walked, 6 vertices removed, 7 largest sub-round (arcs).
__device__ __forceinline__ void cta_count(const KArgs &A, const Smem &sm, int slot, int64_t val)
{
    const Ctrl &c = sm.ctrl;
    if (!KC_TRACE || threadIdx.x != 0 || c.solo || !sm.tr_cta || c.st_bar >= sm.tr_cap) return;
    sm.tr_cta[(c.st_bar * gridDim.x + blockIdx.x) * 8 + slot] = val;
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

// Block-wide exclusive scans of two u64 per thread; totals in tot_q / tot_q2.
__device__ __forceinline__ void block_excl_scan2(Smem &sm, unsigned long long q, unsigned long long r,
                                                 unsigned long long &qe, unsigned long long &re)
{
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    unsigned long long qi = q, ri = r;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long t = __shfl_up_sync(kFull, qi, o);
        const unsigned long long t2 = __shfl_up_sync(kFull, ri, o);
        if (lane >= o) { qi += t; ri += t2; }
    }
    if (lane == 31) { sm.scan_q[wib] = qi; sm.scan_q2[wib] = ri; }
    __syncthreads();
    if (wib == 0) {
        const unsigned long long wq = lane < kWarps ? sm.scan_q[lane] : 0ULL;
        const unsigned long long wr = lane < kWarps ? sm.scan_q2[lane] : 0ULL;
        unsigned long long iq = wq, ir = wr;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long t = __shfl_up_sync(kFull, iq, o);
            const unsigned long long t2 = __shfl_up_sync(kFull, ir, o);
            if (lane >= o) { iq += t; ir += t2; }
        }
        if (lane < kWarps) { sm.scan_q[lane] = iq - wq; sm.scan_q2[lane] = ir - wr; }
        if (lane == kWarps - 1) { sm.tot_q = iq; sm.tot_q2 = ir; }
    }
    __syncthreads();
    qe = sm.scan_q[wib] + (qi - q);
    re = sm.scan_q2[wib] + (ri - r);
}

// async chunk-queue words (Smem::qword)
__device__ __forceinline__ unsigned long long qword_pack(int64_t beg, int len)
{
    return (1ULL << 63) | ((unsigned long long)(len - 1) << 34) | (unsigned long long)beg;
}

// ------------------------------------------------------------ warp stages
// Global queue: one packed atomic reserves slots and their arc range.
#ifndef KC_GQF_INLINE
#define KC_GQF_INLINE 0  // the global-queue flush is a rare path: out of line keeps the kernel small
#endif
#if KC_GQF_INLINE
__device__ __forceinline__
#else
__device__ __noinline__
#endif
void gq_flush_(const KArgs &A, Smem &sm, int wib, int gcnt)
{
    const int lane = threadIdx.x & 31;
    if (gcnt == 0) return;
    __syncwarp();
    int64_t tot = 0;
    for (int x = lane; x < gcnt; x += 32) tot += sm.gd[wib][x];
    tot = warp_sum64(tot);
    unsigned long long base = 0;
    if (lane == 0)
        base = atomicAdd(&A.S->gq_tail, ((unsigned long long)gcnt << kArcBits) | (unsigned long long)tot);
    base = __shfl_sync(kFull, base, 0);
    const int64_t bc = (int64_t)(base >> kArcBits);
    int64_t carry = (int64_t)(base & kArcMask);
    for (int x0 = 0; x0 < gcnt; x0 += 32) {
        const int x = x0 + lane;
        const int64_t d = x < gcnt ? (int64_t)sm.gd[wib][x] : 0;
        int64_t incl = d;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t t = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += t;
        }
        if (x < gcnt) {
            A.gq_v[bc + x] = sm.gv[wib][x];
            A.gq_beg[bc + x] = sm.gb[wib][x];
            A.gq_arc[bc + x] = carry + incl - d;
        }
        carry += __shfl_sync(kFull, incl, 31);
    }
    __syncwarp();
}

// (gcnt passed by value: a reference across the out-of-line call kept the
// stage count in local memory on every routing path)
__device__ __forceinline__ void gq_flush(const KArgs &A, Smem &sm, int wib, int &gcnt)
{
    if (gcnt) gq_flush_(A, sm, wib, gcnt);
    gcnt = 0;
}

// Route claimed vertices (one per lane where `won`): reserve their slots in
// the removal order right away (a vertex is claimed only after every vertex
// whose processing made it reach k was claimed, so claim-time slots form a
// valid peel order -- the I4 certificate), then send each to the local next
// frontier `nx` if it is small and fits the sub-round's arc budget, else to
// the global queue.  Zero-degree vertices are only recorded.
__device__ __noinline__ void route_won(const KArgs &A, Smem &sm, int wib, bool won, int32_t v,
                                          int32_t dv, int64_t bv, int nx, int &gcnt)
{
    const int lane = threadIdx.x & 31;
    const unsigned b = __ballot_sync(kFull, won);
    if (b == 0) return;
    {
        const int lead = __ffs(b) - 1;
        if (A.order) {  // peel order requested: slots in claim order
            unsigned long long base = 0;
            if (lane == lead) base = atomicAdd(&A.S->ord_tail, (unsigned long long)__popc(b));
            base = __shfl_sync(kFull, base, lead);
            if (won) A.order[base + __popc(b & lanemask_lt())] = v;
        } else if (lane == lead) {
            atomicAdd(&sm.removed, __popc(b));
        }
    }
    const bool cand = !KC_NO_SMBUF && won && dv > 0 && dv <= sm.bud_hub && nx >= 0;  // nx < 0: no local list
    const unsigned bc = __ballot_sync(kFull, cand);
    bool wantl = false;
    int lbase = 0;
    if (bc) {
        int sumd = cand ? dv : 0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sumd += __shfl_xor_sync(kFull, sumd, o);
        const int lead = __ffs(bc) - 1;
        int oa = 0;
        int ok = 0;
        if (lane == lead) {
            oa = atomicAdd(&sm.larc[nx], sumd);
            if (oa + sumd <= sm.bud_sub) {
                const int op = atomicAdd(&sm.lphase, sumd);
                if (op + sumd <= sm.bud_phase) { ok = 1; lbase = atomicAdd(&sm.lcnt[nx], __popc(bc)); }
            }
        }
        ok = __shfl_sync(kFull, ok, lead);
        lbase = __shfl_sync(kFull, lbase, lead);
        wantl = cand && ok;
    }
    bool tog = won && dv > 0 && !wantl;
    if (wantl) {
        const int pos = lbase + __popc(bc & lanemask_lt());
        if (pos < kLCap) {
            sm.lv[nx][pos] = v;
            sm.ld[nx][pos] = dv;
            sm.lb[nx][pos] = bv;
        } else {
            tog = true;
        }
    }
    const unsigned bg = __ballot_sync(kFull, tog);
    if (bg) {
        const int c = __popc(bg);
        if (gcnt + c > kGStage) gq_flush(A, sm, wib, gcnt);
        if (tog) {
            const int pos = gcnt + __popc(bg & lanemask_lt());
            sm.gv[wib][pos] = v;
            sm.gd[wib][pos] = dv;
            sm.gb[wib][pos] = bv;
        }
        gcnt += c;
    }
    __syncwarp();
}

// route_won for four candidates per lane (one batch of a walk or a scan step):
// the same decisions as four route_won calls, with ONE order/removed update,
// ONE budget reservation and one local-list reservation for the whole warp
// (the shared-memory atomics are a dependent chain on the hit path).
#if KC_ROUTE4_INLINE
__device__ __forceinline__
#else
__device__ __noinline__
#endif
void route_won4(const KArgs &A, Smem &sm, int wib, unsigned wm, int32_t v0, int32_t v1,
                                        int32_t v2, int32_t v3, int32_t d0, int32_t d1, int32_t d2, int32_t d3,
                                        int64_t b0, int64_t b1, int64_t b2, int64_t b3, int nx, int &gcnt)
{
    const int lane = threadIdx.x & 31;
#if KC_ROUTE_FAST
    if (KC_ASYNC && nx == kAsyncNx) {
        // fast path: ONE vertex claimed by the whole warp (the usual hit of a
        // light walk) -- no prefix sums, one reservation chain, its chunks
        // published by all lanes
        const unsigned anyl = __ballot_sync(kFull, wm != 0u);
        const int L = __ffs(anyl) - 1;
        const unsigned wmL = __shfl_sync(kFull, wm, L & 31);
        if (anyl != 0u && (anyl & (anyl - 1u)) == 0u && (wmL & (wmL - 1u)) == 0u) {
            const int r = __ffs(wmL) - 1;
            const int32_t v = __shfl_sync(kFull, r == 0 ? v0 : r == 1 ? v1 : r == 2 ? v2 : v3, L);
            const int32_t d = __shfl_sync(kFull, r == 0 ? d0 : r == 1 ? d1 : r == 2 ? d2 : d3, L);
            const int64_t b = __shfl_sync(kFull, r == 0 ? b0 : r == 1 ? b1 : r == 2 ? b2 : b3, L);
            if (lane == 0) {
                if (A.order) A.order[atomicAdd(&A.S->ord_tail, 1ULL)] = v;
                else atomicAdd(&sm.removed, 1);
            }
            if (d > 0) {
                const int nc = (d + kBatch - 1) / kBatch;
                int ok = 0, base = 0;
                if (lane == 0 && !KC_NO_SMBUF && d <= sm.bud_hub && atomicAdd(&sm.lphase, d) + d <= sm.bud_phase) {
                    int t = *(volatile int *)&sm.qtail;
                    while (t + nc <= kQCap) {
                        const int o2 = atomicCAS(&sm.qtail, t, t + nc);
                        if (o2 == t) { ok = 1; base = t; break; }
                        t = o2;
                    }
                    if (ok) atomicAdd(&sm.qpend, nc);  // before any chunk is visible
                }
                ok = __shfl_sync(kFull, ok, 0);
                if (ok) {
                    base = __shfl_sync(kFull, base, 0);
                    for (int q = lane; q < nc; q += 32)
                        atomicExch(&sm.qword[base + q], qword_pack(b + (int64_t)q * kBatch, min(kBatch, d - q * kBatch)));
                } else {
                    if (gcnt + 1 > kGStage) gq_flush(A, sm, wib, gcnt);
                    if (lane == 0) { sm.gv[wib][gcnt] = v; sm.gd[wib][gcnt] = d; sm.gb[wib][gcnt] = b; }
                    gcnt += 1;
                }
            }
            __syncwarp();
            return;
        }
    }
#endif
    const unsigned lt = lanemask_lt();
    const int32_t vv[4] = {v0, v1, v2, v3};
    const int32_t dd[4] = {d0, d1, d2, d3};
    const int64_t bb[4] = {b0, b1, b2, b3};
    unsigned bal[4];
    int off[4], pre[4], tot = 0;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        pre[r] = ballot_excl((wm >> r) & 1u, bal[r]);  // Fig. 8(c)
        off[r] = tot;
        tot += __popc(bal[r]);
    }
    if (tot == 0) return;
    if (A.order) {  // peel order requested: slots in claim order
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&A.S->ord_tail, (unsigned long long)tot);
        base = __shfl_sync(kFull, base, 0);
#pragma unroll
        for (int r = 0; r < 4; r++)
            if ((wm >> r) & 1u) A.order[base + off[r] + pre[r]] = vv[r];
    } else if (lane == 0) {
        atomicAdd(&sm.removed, tot);
    }
    if (lane == 0) PROBE_W(15, threadIdx.x >> 5);
    unsigned cm = 0;
#pragma unroll
    for (int r = 0; r < 4; r++)
        if (!KC_NO_SMBUF && ((wm >> r) & 1u) && dd[r] > 0 && dd[r] <= sm.bud_hub && nx >= 0) cm |= 1u << r;
    unsigned cb[4];
    int coff[4], ctot = 0, sumd = 0;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        cb[r] = __ballot_sync(kFull, (cm >> r) & 1u);
        coff[r] = ctot;
        ctot += __popc(cb[r]);
        if ((cm >> r) & 1u) sumd += dd[r];
    }
    unsigned lm = 0;  // candidates that go to the local list
    int lbase = 0;
    if (KC_ASYNC && nx == kAsyncNx && ctot) {
        // chunks of <= 128 arcs per candidate into the CTA's async queue
        int nc[4], mine = 0;
#pragma unroll
        for (int r = 0; r < 4; r++) {
            nc[r] = ((cm >> r) & 1u) ? (dd[r] + kBatch - 1) / kBatch : 0;
            mine += nc[r];
        }
        int incl = mine;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += t;
        }
        const int tot = __shfl_sync(kFull, incl, 31);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sumd += __shfl_xor_sync(kFull, sumd, o);
        int ok = 0, base = 0;
        if (lane == 0) {
            const int op = atomicAdd(&sm.lphase, sumd);
            if (op + sumd <= sm.bud_phase) {
                int t = atomicAdd(&sm.qtail, 0);
                while (t + tot <= kQCap) {
                    const int o2 = atomicCAS(&sm.qtail, t, t + tot);
                    if (o2 == t) { ok = 1; base = t; break; }
                    t = o2;
                }
                if (ok) atomicAdd(&sm.qpend, tot);  // before any chunk is visible
            }
        }
        ok = __shfl_sync(kFull, ok, 0);
        base = __shfl_sync(kFull, base, 0);
        if (lane == 0) PROBE_W(16, threadIdx.x >> 5);
        if (ok) {
#if KC_PUSH_PAR
            // publish the chunks with every lane: a hub row is dozens of chunks,
            // one lane writing them in sequence stalls the hop by ~1 us
            int p0[4];
            p0[0] = base + incl - mine;
#pragma unroll
            for (int r = 1; r < 4; r++) p0[r] = p0[r - 1] + nc[r - 1];
            unsigned any = __ballot_sync(kFull, mine > 0);
            while (any) {
                const int L = __ffs(any) - 1;
                any &= any - 1;
#pragma unroll
                for (int r = 0; r < 4; r++) {
                    const int ncr = __shfl_sync(kFull, nc[r], L);
                    if (ncr == 0) continue;
                    const int64_t b = __shfl_sync(kFull, bb[r], L);
                    const int d = __shfl_sync(kFull, dd[r], L);
                    const int ps = __shfl_sync(kFull, p0[r], L);
                    for (int q = lane; q < ncr; q += 32)
                        atomicExch(&sm.qword[ps + q], qword_pack(b + (int64_t)q * kBatch, min(kBatch, d - q * kBatch)));
                }
            }
#else
            int pos = base + incl - mine;
#pragma unroll
            for (int r = 0; r < 4; r++) {
                for (int q = 0; q < nc[r]; q++, pos++)
                    atomicExch(&sm.qword[pos], qword_pack(bb[r] + (int64_t)q * kBatch, min(kBatch, dd[r] - q * kBatch)));
            }
#endif
            lm |= cm;
        }
        if (lane == 0) PROBE_W(17, threadIdx.x >> 5);
    } else if (ctot) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sumd += __shfl_xor_sync(kFull, sumd, o);
        int ok = 0;
        if (lane == 0) {
            const int oa = atomicAdd(&sm.larc[nx], sumd);
            if (oa + sumd <= sm.bud_sub) {
                const int op = atomicAdd(&sm.lphase, sumd);
                if (op + sumd <= sm.bud_phase) { ok = 1; lbase = atomicAdd(&sm.lcnt[nx], ctot); }
            }
        }
        ok = __shfl_sync(kFull, ok, 0);
        lbase = __shfl_sync(kFull, lbase, 0);
        if (ok) {
#pragma unroll
            for (int r = 0; r < 4; r++) {
                if ((cm >> r) & 1u) {
                    const int pos = lbase + coff[r] + __popc(cb[r] & lt);
                    if (pos < kLCap) {
                        sm.lv[nx][pos] = vv[r];
                        sm.ld[nx][pos] = dd[r];
                        sm.lb[nx][pos] = bb[r];
                        lm |= 1u << r;
                    }
                }
            }
        }
    }
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const bool tog = ((wm >> r) & 1u) && dd[r] > 0 && !((lm >> r) & 1u);
        const unsigned bg = __ballot_sync(kFull, tog);
        if (bg) {
            const int c = __popc(bg);
            if (gcnt + c > kGStage) gq_flush(A, sm, wib, gcnt);
            if (tog) {
                const int pos = gcnt + __popc(bg & lt);
                sm.gv[wib][pos] = vv[r];
                sm.gd[wib][pos] = dd[r];
                sm.gb[wib][pos] = bb[r];
            }
            gcnt += c;
        }
    }
    __syncwarp();
}

__device__ __forceinline__ uint64_t deg_policy()
{
#if KC_DEG_EVICT_LAST
    return l2_evict_last_policy();
#else
    return 0;
#endif
}

__device__ __forceinline__ bool claim(const KArgs &A, int32_t v)
{
    const uint32_t bit = 1u << (v & 31);
    return (atom_or_claim(A.claimed + (v >> 5), bit, deg_policy()) & bit) == 0u;
}

// theta+1 of the running near epoch (INT_MIN: no near list), re-read from
// shared memory at each use so it never holds a register across the walk loop
__device__ __forceinline__ int near_th1(const Smem &sm)
{
    if (!KC_NEAR) return INT_MIN;
    return *(const volatile int32_t *)&sm.near_th1;
}

// One theta+1 -> theta crossing joins the near list: a lane-level append (each
// vertex crosses once per epoch, so these are rare; no warp-collective code in
// the walk's hot loop).
__device__ __forceinline__ void near_push(const KArgs &A, const Smem &sm, int32_t u)
{
    const int app = *(const volatile int32_t *)&sm.ctrl.near_app;
    const unsigned long long pos = atomicAdd(&A.S->near_tail[app], 1ULL);
    A.near[app][pos] = u;
}

// old = atomicSub(p, 1) if go, else INT_MIN -- as ONE predicated atomic
// (KC_PRED_ATOM; the ternary compiles to a branch + reconvergence per arc)
__device__ __forceinline__ int atom_dec_if(bool go, int32_t *p, uint64_t pol)
{
#if KC_PRED_ATOM && !KC_DEG_EVICT_LAST
    (void)pol;
    int old = INT_MIN;
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q atom.global.add.s32 %0, [%1], -1;\n\t}"
                 : "+r"(old) : "l"(p), "r"((unsigned)go) : "memory");
    return old;
#else
    return go ? atom_dec_deg(p, pol) : INT_MIN;
#endif
}

// Near list: targets whose decrement crossed theta+1 -> theta (cm bit r set for
// u[r]) join near[near_app] -- one warp-aggregated append.  Each vertex crosses
// once per epoch (degrees only decrease), so the list stays within n.
// --------------------------------------------------------- arc walking
// Hits of one batch (u reached k): claim, fetch row bounds, prefetch the
// row's first line for the next hop, route.  Out of line: rare path.
#ifndef KC_NOCLAIM
#define KC_NOCLAIM 0  // (C1/C3/C4 ~1 % faster without: the per-batch flag read costs more) 1: hits skip the claim atomic once every level scan of the phase is known complete
#endif
#ifndef KC_SPEC
#define KC_SPEC 0  // (measured slower: extra scattered loads) filtered (light) walks load the row bounds of each decremented target with its atomic
#endif
// Hits of one batch (u reached k: old == k+1 from its decrement).  `nc`
// (read before the batch's decrements): some CTA's level scan of this phase
// may still be running.  Only a scan can race a hit -- it may read deg[u] <= k
// after the decrement that took u from k+1 to k -- so while nc, the claim bit
// decides (atomicOr, reading R9).  Once every scan of the phase has finished
// before the decrement was issued (scan_done == grid observed, acquire chain:
// scanner deg read -> red.release -> this CTA's fence -> nclaim store
// (release.cta) -> walker's acquire.cta load -> its decrement), nothing can
// race: old == k+1 is seen exactly once, so the hit is owned without a round
// trip and the claim bit is set fire-and-forget (later scans test it).  HUB
// phases run no scan at all.  With SPEC the row bounds were loaded together
// with the decrements (pb0/pb1), so a claim-free hit costs no round trip here.
template <bool SPEC>
#if KC_HITS_INLINE
__device__ __forceinline__
#else
__device__ __noinline__
#endif
void handle_hits(const KArgs &A, Smem &sm, int k, int nx, int u0, int u1, int u2, int u3,
                                         unsigned hm, int &gcnt, bool nc, const int64_t *pb0 = nullptr,
                                         const int64_t *pb1 = nullptr)
{
    const int lane = threadIdx.x & 31;
    const int wib = threadIdx.x >> 5;
    const int uu[4] = {u0, u1, u2, u3};
    // row bounds and claims issued together (independent round trips)
    int64_t b0[4], b1[4];
#pragma unroll
    for (int r = 0; r < 4; r++) {
        const bool h = (hm >> r) & 1u;
        if (SPEC) {
            b0[r] = h ? pb0[r] : 0;
            b1[r] = h ? pb1[r] : 0;
        } else {
            b0[r] = h ? ld_ro_i64(A.rowptr + uu[r]) : 0;
            b1[r] = h ? ld_ro_i64(A.rowptr + uu[r] + 1) : 0;
        }
    }
    bool won[4];
    if (KC_NOCLAIM && !nc) {
#pragma unroll
        for (int r = 0; r < 4; r++) {
            won[r] = (hm >> r) & 1u;
            if (won[r]) red_or_u32(A.claimed + (uu[r] >> 5), 1u << (uu[r] & 31));
        }
    } else {
        const unsigned hb = __ballot_sync(kFull, hm != 0);
        const int lead = __ffs(hb) - 1;
        uint32_t sd = 0;
        if (KC_NOCLAIM && lane == lead) sd = ld_relaxed_u32(&A.S->scan_done);  // in flight with the claims
#pragma unroll
        for (int r = 0; r < 4; r++) won[r] = ((hm >> r) & 1u) && claim(A, uu[r]);
        if (KC_NOCLAIM && lane == lead && sd >= gridDim.x) {
            fence_acq_rel_gpu();
            st_release_cta_shared(&sm.nclaim, 0);
        }
    }
#ifdef KC_PROBE_W
    {
        int64_t dep = 0;
#pragma unroll
        for (int r = 0; r < 4; r++) dep += b0[r] + b1[r] + (won[r] ? 1 : 0);
        dep = __reduce_add_sync(kFull, (unsigned)(dep & 0xffff));
        if ((threadIdx.x & 31) == 0) PROBE_W(14, (threadIdx.x >> 5) | ((dep & 0xff) << 8));
    }
#endif
#pragma unroll
    for (int r = 0; r < 4; r++)
        if (won[r]) A.core[uu[r]] = k;
#if KC_ROUTE4
    unsigned wm = 0;
#pragma unroll
    for (int r = 0; r < 4; r++) {
        if (won[r] && b1[r] > b0[r]) prefetch_row(A.colidx, b0[r], b1[r]);
        if (won[r]) wm |= 1u << r;
    }
    route_won4(A, sm, wib, wm, uu[0], uu[1], uu[2], uu[3], (int32_t)(b1[0] - b0[0]), (int32_t)(b1[1] - b0[1]),
               (int32_t)(b1[2] - b0[2]), (int32_t)(b1[3] - b0[3]), b0[0], b0[1], b0[2], b0[3], nx, gcnt);
#else
#pragma unroll
    for (int r = 0; r < 4; r++) {
        if (won[r] && b1[r] > b0[r]) prefetch_row(A.colidx, b0[r], b1[r]);
        route_won(A, sm, wib, won[r], uu[r], (int32_t)(b1[r] - b0[r]), b0[r], nx, gcnt);
    }
#endif
}

// Walk arcs [a0,a1) of a frontier whose entries are i = [s,e) with arc
// prefix P(i) and row begin B(i); the last entry ends at arc ae.  LOCAL=true:
// entries live in this CTA's shared-memory list `cur`; else in the global
// queue.  Hits are routed into local list `nx`.  Each lane holds one entry
// of a 32-entry window; an arc finds its entry with a 5-step shuffle search
// on 32-bit offsets relative to the current batch.
template <bool LOCAL>
__device__ __forceinline__ void walk(const KArgs &A, Smem &sm, const int k, const int cur, const int nx,
                                     int64_t s, int64_t e, int64_t ae, int64_t a0, int64_t a1,
                                     bool use_bloom, bool atom_only, int &lmin, int &gcnt, bool claim_filter = false)
{
    const int lane = threadIdx.x & 31;
    const uint64_t pol = deg_policy();
    // first entry: largest i in [s,e) with P(i) <= a0 (32-ary search)
    int64_t lo = s, hi = e;
    while (true) {
        const int64_t step = hi - lo > 32 ? (hi - lo + 31) / 32 : 1;
        const int64_t p = lo + lane * step;
        bool ok = false;
        if (p < hi) ok = (LOCAL ? sm.lpre[p] : ld_cg_i64(A.gq_arc + p)) <= a0;
        const unsigned b = __ballot_sync(kFull, ok);
        const int L = 31 - __clz(b);
        lo = lo + L * step;
        if (step == 1) break;
        hi = min(hi, lo + step);
    }
    int64_t i = lo;
    int64_t a = a0;
    if (lane == 0) PROBE_W(10, threadIdx.x >> 5);
    while (a < a1) {
        const int64_t j = i + lane;
        int64_t wq = LLONG_MAX, wbeg = 0;
        if (j < e) {
            wq = LOCAL ? sm.lpre[j] : ld_cg_i64(A.gq_arc + j);
            wbeg = LOCAL ? sm.lb[cur][j] : ld_cg_i64(A.gq_beg + j);
        }
        int64_t nxt = __shfl_down_sync(kFull, wq, 1);
        if (j + 1 >= e) nxt = ae;
        else if (lane == 31) nxt = LOCAL ? sm.lpre[j + 1] : ld_cg_i64(A.gq_arc + j + 1);
        const int64_t limit = min(a1, __shfl_sync(kFull, nxt, 31));
        const int64_t bmq = wbeg - wq;  // colidx index of arc x in this entry = bmq + x
        // colidx targets of the batch at arc ab (window search relative to ab)
        auto gather = [&](int64_t ab, int32_t *out) {
            const int64_t rq = wq - ab;
            const int32_t q32 = rq < -1 ? -1 : (rq > 0x7fffffff ? 0x7fffffff : (int32_t)rq);
            const int32_t lim = (int32_t)min((int64_t)kBatch, limit - ab);
#if KC_WALK_FAST
            // fast path: the whole batch lies in one entry (a long row) -- no search
            const unsigned le = __ballot_sync(kFull, q32 <= 0);
            const int first = le ? 31 - __clz(le) : 0;
            const int32_t qn = __shfl_sync(kFull, q32, min(first + 1, 31));
            if (first == 31 || qn >= kBatch) {
                const int64_t off = __shfl_sync(kFull, bmq, first) + ab;
#pragma unroll
                for (int r = 0; r < kUnroll; r++) {
                    const int32_t my = r * 32 + lane;
                    out[r] = (my < lim) ? ld_stream_i32(A.colidx + off + my) : -1;
                }
                return;
            }
#endif
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
                out[r] = (my < lim) ? ld_stream_i32(A.colidx + off + ab + my) : -1;
            }
        };
        // software pipeline: the next batch's colidx loads (HBM) are in flight
        // while this batch's deg loads and atomics (L2) complete
        int32_t un[kUnroll];
        if (a < limit) gather(a, un);
        while (a < limit) {
            int32_t u[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) u[r] = un[r];
            const int64_t an = a + kBatch;
            if (an < limit) gather(an, un);
            if (use_bloom) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    {
#if KC_BLOOM_BF
                    // branch-free: both probes for every lane (a -1 id probes harmlessly)
                    const bool keep = bloom_maybe(sm, (uint32_t)u[r]);
                    u[r] = keep ? u[r] : -1;
#else
                    if (u[r] >= 0 && !bloom_maybe(sm, (uint32_t)u[r])) u[r] = -1;
#endif
                }
            }
            if (claim_filter) {
                // exact dead-target filter: the claim bitmap (2 MB at C4, L1/L2
                // resident) -- a set bit is final, a stale clear bit only costs
                // the atomic we would have issued anyway
                uint32_t cw[kUnroll];
#pragma unroll
                for (int r = 0; r < kUnroll; r++) cw[r] = u[r] >= 0 ? A.claimed[u[r] >> 5] : 0u;
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if (u[r] >= 0 && ((cw[r] >> (u[r] & 31)) & 1u)) u[r] = -1;
            }
            if (lane == 0) PROBE_W(13, (threadIdx.x >> 5) | ((int64_t)u[0] << 16));
            int32_t d[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++)
                d[r] = u[r] < 0 ? -1 : (atom_only ? INT_MAX : ld_deg(A.deg + u[r], pol));
            const bool nc = !KC_NOCLAIM || __shfl_sync(kFull, ld_acquire_cta_shared(&sm.nclaim), 0) != 0;  // warp-uniform
            int old[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) old[r] = atom_dec_if(d[r] > k, A.deg + u[r], pol);
            unsigned hm = 0, nm = 0;
            const int th1 = near_th1(sm);
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
#if KC_HIT_BF
                // branch-free outcome; theta crossings (rare) pushed after the loop
                hm |= (old[r] == k + 1 ? 1u : 0u) << r;
                lmin = min(lmin, old[r] > k + 1 ? old[r] - 1 : INT_MAX);
                nm |= (old[r] > k + 1 && old[r] == th1 ? 1u : 0u) << r;
#else
                if (old[r] == k + 1) hm |= 1u << r;
                else if (old[r] > k + 1) { lmin = min(lmin, old[r] - 1); if (old[r] == th1) near_push(A, sm, u[r]); }
#endif
            }
#if KC_HIT_BF
            if (nm) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if ((nm >> r) & 1u) near_push(A, sm, u[r]);
            }
#endif
            const unsigned hb = __ballot_sync(kFull, hm != 0);
            if (lane == 0) PROBE_W(11, (threadIdx.x >> 5) | ((int64_t)__popc(hb) << 8) | ((int64_t)old[0] << 16));
            if (hb) {
                handle_hits<false>(A, sm, k, nx, u[0], u[1], u[2], u[3], hm, gcnt, nc);
            }
            if (lane == 0) PROBE_W(12, threadIdx.x >> 5);
            a = an;
        }
        a = limit;
        i += 32;
    }
}

// Heavy HUB walk with NON-returning decrements (Ctrl::red): arcs [a0,a1) of
// global-queue entries [s,e) (arc prefix gq_arc, row begin gq_beg; the last
// entry ends at arc ae).  Every target that passes the alive filter takes
// `red.global.add -1` (Alg. 3 l.21 without its return value); nothing is
// claimed here.  The phase that follows is a rescan -- a LEVEL phase at the
// same k -- which claims every alive vertex this walk took to <= k (the scan
// test deg <= k, reading R10), so each removal stays exactly-once and the
// level-skip bound stays a lower bound (the rescan's min covers every target
// decremented here).  With no return to wait for, a warp keeps
// 32 x KC_RED_UNROLL arcs of colidx in flight and the next batch's loads are
// issued before this batch's decrements.
__device__ __forceinline__ void red_dec(int32_t *p)
{
    asm volatile("red.global.add.s32 [%0], -1;" ::"l"(p) : "memory");
}

__device__ void walk_red(const KArgs &A, Smem &sm, int64_t s, int64_t e, int64_t ae, int64_t a0, int64_t a1,
                         bool use_bloom)
{
    constexpr int U = KC_RED_UNROLL;
    constexpr int RB = 32 * U;
    const int lane = threadIdx.x & 31;
    int64_t lo = s, hi = e;
    while (true) {  // first entry: largest i in [s,e) with P(i) <= a0 (32-ary search)
        const int64_t step = hi - lo > 32 ? (hi - lo + 31) / 32 : 1;
        const int64_t p = lo + lane * step;
        bool ok = false;
        if (p < hi) ok = ld_cg_i64(A.gq_arc + p) <= a0;
        const unsigned b = __ballot_sync(kFull, ok);
        lo = lo + (31 - __clz(b)) * step;
        if (step == 1) break;
        hi = min(hi, lo + step);
    }
    int64_t i = lo, a = a0;
    while (a < a1) {
        const int64_t j = i + lane;
        int64_t wq = LLONG_MAX, wbeg = 0;
        if (j < e) { wq = ld_cg_i64(A.gq_arc + j); wbeg = ld_cg_i64(A.gq_beg + j); }
        int64_t nxt = __shfl_down_sync(kFull, wq, 1);
        if (j + 1 >= e) nxt = ae;
        else if (lane == 31) nxt = ld_cg_i64(A.gq_arc + j + 1);
        const int64_t limit = min(a1, __shfl_sync(kFull, nxt, 31));
        const int64_t bmq = wbeg - wq;
        auto gather = [&](int64_t ab, int32_t *out) {
            const int64_t rq = wq - ab;
            const int32_t q32 = rq < -1 ? -1 : (rq > 0x7fffffff ? 0x7fffffff : (int32_t)rq);
            const int32_t lim = (int32_t)min((int64_t)RB, limit - ab);
            // fast path: the whole batch lies in one entry (long rows: the usual case)
            const unsigned le = __ballot_sync(kFull, q32 <= 0);
            const int first = le ? 31 - __clz(le) : 0;
            const int32_t qn = __shfl_sync(kFull, q32, min(first + 1, 31));
            if (first == 31 || qn >= RB) {
                const int64_t off = __shfl_sync(kFull, bmq, first) + ab;
#pragma unroll
                for (int r = 0; r < U; r++) {
                    const int32_t my = r * 32 + lane;
                    out[r] = (my < lim) ? ld_stream_i32(A.colidx + off + my) : -1;
                }
            } else {
#pragma unroll
                for (int r = 0; r < U; r++) {
                    const int32_t my = r * 32 + lane;
                    int pos = 0;
#pragma unroll
                    for (int bs = 16; bs >= 1; bs >>= 1) {
                        const int32_t q = __shfl_sync(kFull, q32, pos + bs);
                        if (q <= my) pos += bs;
                    }
                    const int64_t off = __shfl_sync(kFull, bmq, pos);
                    out[r] = (my < lim) ? ld_stream_i32(A.colidx + off + ab + my) : -1;
                }
            }
        };
        int32_t un[U];
        if (a < limit) gather(a, un);
        while (a < limit) {
            int32_t u[U];
#pragma unroll
            for (int r = 0; r < U; r++) u[r] = un[r];
            const int64_t an = a + RB;
            if (an < limit) gather(an, un);
#pragma unroll
            for (int r = 0; r < U; r++) {
#if KC_PRED_ATOM
                // branch-free: the filter result predicates the red
                const bool go = u[r] >= 0 && (!use_bloom || bloom_maybe(sm, (uint32_t)u[r]));
                asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %1, 0;\n\t@q red.global.add.s32 [%0], -1;\n\t}"
                             ::"l"(A.deg + u[r]), "r"((unsigned)go) : "memory");
#else
                if (u[r] >= 0 && (!use_bloom || bloom_maybe(sm, (uint32_t)u[r]))) red_dec(A.deg + u[r]);
#endif
            }
            a = an;
        }
        a = limit;
        i += 32;
    }
}

// Drain this CTA's local frontier (list `cur`) breadth-first with CTA-local
// sub-rounds.  Returns the number of arcs walked.
__device__ int64_t local_drain(const KArgs &A, Smem &sm, const int k, int cur, bool use_bloom, bool atom_only,
                               int &lmin, int &gcnt, int64_t *subs = nullptr, int64_t *tmax = nullptr)
{
    const int wib = threadIdx.x >> 5;
    int64_t walked = 0;
    while (true) {
        __syncthreads();
        const int L = min(sm.lcnt[cur], kLCap);
        if (threadIdx.x == 0) PROBE(1, L);
        if (L == 0) break;
        // arc prefix of the list
        const int nx = cur ^ 1;
        int64_t T;
        if (KC_FASTSUB && L <= 32) {  // one warp: no block-wide scan
            if (threadIdx.x < 32) {
                const int lane = threadIdx.x;
                const int64_t dv = lane < L ? (int64_t)sm.ld[cur][lane] : 0;
                int64_t incl = dv;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int64_t t = __shfl_up_sync(kFull, incl, o);
                    if (lane >= o) incl += t;
                }
                if (lane < L) sm.lpre[lane] = incl - dv;
                if (lane == 31) { sm.lpre[L] = incl; sm.tot_q = (unsigned long long)incl; sm.lcnt[nx] = 0; sm.larc[nx] = 0; }
            }
            __syncthreads();
            T = (int64_t)sm.tot_q;
        } else {
            const int64_t dv = threadIdx.x < L ? (int64_t)sm.ld[cur][threadIdx.x] : 0;
            const unsigned long long ex = block_excl_scan(sm, (unsigned long long)dv);
            if (threadIdx.x < L) sm.lpre[threadIdx.x] = (int64_t)ex;
            T = (int64_t)sm.tot_q;
            if (threadIdx.x == 0) { sm.lpre[L] = T; sm.lcnt[nx] = 0; sm.larc[nx] = 0; }
            __syncthreads();
        }
        if (threadIdx.x == 0) PROBE(2, T);
        int64_t C = (T + kWarps - 1) / kWarps;
        C = ((C + kBatch - 1) / kBatch) * kBatch;
        const int64_t a0 = (int64_t)wib * C;
        if (a0 < T)
            walk<true>(A, sm, k, cur, nx, 0, L, T, a0, min(a0 + C, T), use_bloom, atom_only, lmin, gcnt,
                       KC_CF_LOCAL && T >= KC_CF_LOCAL_MIN);
        walked += T;
        if (subs) { *subs += 1; *tmax = max(*tmax, T); }
        if (threadIdx.x == 0) PROBE(3, sm.lcnt[nx]);
        if (!KC_FASTSUB) {
            __syncthreads();
            if (threadIdx.x == 0) { sm.lcnt[cur] = 0; sm.larc[cur] = 0; }
        }
        // (KC_FASTSUB: the loop-top barrier orders the walk before the next
        // read of lcnt; list `cur` is reset when it next becomes `nx`)
        cur = nx;
    }
    return walked;
}

// Asynchronous CTA-local drain (KC_ASYNC; the PKC idea of P:L63 -- no
// sub-level synchronisation -- at CTA scope): the frontier lives in a
// shared-memory queue of chunks (<= 128 arcs of one row); each warp pops a
// chunk, walks it, and pushes the chunks of the vertices it claimed.
// qpend counts pushed-but-unfinished chunks; the drain ends when it is 0.
__device__ int64_t local_drain_async(const KArgs &A, Smem &sm, const int k, bool use_bloom, bool atom_only,
                                     int &lmin, int &gcnt)
{
    const int lane = threadIdx.x & 31;
    const uint64_t pol = deg_policy();
    const bool spec = sm.spec != 0;
    int64_t walked = 0;
    while (true) {
        unsigned long long w = 0ULL;
        int src = 3;  // 1: a chunk, 3: the drain is over
        if (lane == 0) {
            // blocking ticket: the warp owns slot idx and takes it when published
            const int idx = atomicAdd(&sm.qhead, 1);
            if (idx < kQCap) {
#if KC_SPIN_LD
                // wait with plain loads (and a nap): spinning shared-memory
                // atomics would queue ahead of the working warps' queue updates
                while (true) {
                    if (*(volatile unsigned long long *)&sm.qword[idx] != 0ULL) {
                        w = atomicExch(&sm.qword[idx], 0ULL);  // the slot is this warp's ticket
                        break;
                    }
                    if (*(volatile int *)&sm.qpend == 0) break;
                    if (KC_SPIN_NAP > 0) __nanosleep(KC_SPIN_NAP);
                }
#else
                while ((w = atomicExch(&sm.qword[idx], 0ULL)) == 0ULL) {
                    if (atomicAdd(&sm.qpend, 0) == 0) break;
                }
#endif
                if (w) src = 1;
            }
        }
        w = __shfl_sync(kFull, w, 0);
        src = __shfl_sync(kFull, src, 0);
        if (src == 3) break;
        if (lane == 0) PROBE_W(20, (threadIdx.x >> 5) | (src << 8));
        const int64_t beg = (int64_t)(w & ((1ULL << 34) - 1ULL));
        const int len = (int)((w >> 34) & 127ULL) + 1;
        int32_t u[kUnroll];
#pragma unroll
        for (int r = 0; r < kUnroll; r++) {
            const int my = r * 32 + lane;
            u[r] = my < len ? ld_stream_i32(A.colidx + beg + my) : -1;
        }
        if (use_bloom) {
#pragma unroll
            for (int r = 0; r < kUnroll; r++)
                {
#if KC_BLOOM_BF
                    // branch-free: both probes for every lane (a -1 id probes harmlessly)
                    const bool keep = bloom_maybe(sm, (uint32_t)u[r]);
                    u[r] = keep ? u[r] : -1;
#else
                    if (u[r] >= 0 && !bloom_maybe(sm, (uint32_t)u[r])) u[r] = -1;
#endif
                }
        }
#ifdef KC_PROBE_W
        {
            const unsigned all = __ballot_sync(kFull, (u[0] ^ u[1] ^ u[2] ^ u[3]) == 7);
            if (lane == 0) PROBE_W(21, (threadIdx.x >> 5) | ((int64_t)(all & 1u) << 16));
        }
#endif
        const bool nc = !KC_NOCLAIM || __shfl_sync(kFull, ld_acquire_cta_shared(&sm.nclaim), 0) != 0;  // warp-uniform
        int old[kUnroll];
        if (KC_SPEC && spec) {
            // light walk: the row bounds of every decremented target travel with
            // its atomic, so a hit is routed one round trip sooner
            int64_t sb0[kUnroll], sb1[kUnroll];
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                const bool go = u[r] >= 0;
                sb0[r] = go ? ld_ro_i64(A.rowptr + u[r]) : 0;
                sb1[r] = go ? ld_ro_i64(A.rowptr + u[r] + 1) : 0;
                old[r] = go ? atom_dec_deg(A.deg + u[r], pol) : INT_MIN;
            }
            unsigned hm = 0, nm = 0;
            const int th1 = near_th1(sm);
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
#if KC_HIT_BF
                // branch-free outcome; theta crossings (rare) pushed after the loop
                hm |= (old[r] == k + 1 ? 1u : 0u) << r;
                lmin = min(lmin, old[r] > k + 1 ? old[r] - 1 : INT_MAX);
                nm |= (old[r] > k + 1 && old[r] == th1 ? 1u : 0u) << r;
#else
                if (old[r] == k + 1) hm |= 1u << r;
                else if (old[r] > k + 1) { lmin = min(lmin, old[r] - 1); if (old[r] == th1) near_push(A, sm, u[r]); }
#endif
            }
#if KC_HIT_BF
            if (nm) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if ((nm >> r) & 1u) near_push(A, sm, u[r]);
            }
#endif
            if (__any_sync(kFull, hm != 0))
                handle_hits<true>(A, sm, k, kAsyncNx, u[0], u[1], u[2], u[3], hm, gcnt, nc, sb0, sb1);
        } else {
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
                const int32_t d = u[r] < 0 ? -1 : (atom_only ? INT_MAX : ld_deg(A.deg + u[r], pol));
                old[r] = atom_dec_if(d > k, A.deg + u[r], pol);
            }
            unsigned hm = 0, nm = 0;
            const int th1 = near_th1(sm);
#pragma unroll
            for (int r = 0; r < kUnroll; r++) {
#if KC_HIT_BF
                // branch-free outcome; theta crossings (rare) pushed after the loop
                hm |= (old[r] == k + 1 ? 1u : 0u) << r;
                lmin = min(lmin, old[r] > k + 1 ? old[r] - 1 : INT_MAX);
                nm |= (old[r] > k + 1 && old[r] == th1 ? 1u : 0u) << r;
#else
                if (old[r] == k + 1) hm |= 1u << r;
                else if (old[r] > k + 1) { lmin = min(lmin, old[r] - 1); if (old[r] == th1) near_push(A, sm, u[r]); }
#endif
            }
#if KC_HIT_BF
            if (nm) {
#pragma unroll
                for (int r = 0; r < kUnroll; r++)
                    if ((nm >> r) & 1u) near_push(A, sm, u[r]);
            }
#endif
#ifdef KC_PROBE_W
            {
                const unsigned hbp = __ballot_sync(kFull, hm != 0);
                if (lane == 0) PROBE_W(22, (threadIdx.x >> 5) | ((int64_t)__popc(hbp) << 8) | ((int64_t)old[0] << 16));
            }
#endif
            if (__any_sync(kFull, hm != 0))
                handle_hits<false>(A, sm, k, kAsyncNx, u[0], u[1], u[2], u[3], hm, gcnt, nc);
        }
        if (lane == 0) PROBE_W(23, threadIdx.x >> 5);
        walked += len;
        __syncwarp();
        if (lane == 0) atomicSub(&sm.qpend, 1);
    }
    if (lane == 0 && walked) atomicAdd(&sm.qwalked, (unsigned long long)walked);
    __syncthreads();
    return (int64_t)sm.qwalked;
}

// The CTA's drain of its local frontier (list 0 or, KC_ASYNC 1, the chunk
// queue).  KC_ASYNC 2 picks per CTA and phase: long rows (a chain of hubs-to-
// be) drain asynchronously, many short rows keep the packed sub-rounds.
__device__ int64_t drain(const KArgs &A, Smem &sm, const int k, bool use_bloom, bool atom_only, int &lmin,
                         int &gcnt, int64_t *subs, int64_t *tmax)
{
    if (KC_ASYNC == 1) return local_drain_async(A, sm, k, use_bloom, atom_only, lmin, gcnt);
    if (KC_ASYNC == 2) {
        __syncthreads();
        const int L = min(sm.lcnt[0], kLCap);
        int32_t v = 0, d = 0;
        int64_t b = 0;
        if ((int)threadIdx.x < L) { v = sm.lv[0][threadIdx.x]; d = sm.ld[0][threadIdx.x]; b = sm.lb[0][threadIdx.x]; }
        const int nc = (int)threadIdx.x < L ? (d + kBatch - 1) / kBatch : 0;
        unsigned long long tq, tr;
        block_excl_scan2(sm, (unsigned long long)nc, (unsigned long long)d, tq, tr);
        const int64_t chunks = (int64_t)sm.tot_q, arcs = (int64_t)sm.tot_q2;
        if (L > 0 && arcs >= (int64_t)KC_ASYNC_MINAVG * L && chunks <= kQCap) {
            __syncthreads();  // everyone holds its list entry: the queue may overwrite the lists
            for (int q = 0; q < nc; q++) sm.qword[(int)tq + q] = qword_pack(b + (int64_t)q * kBatch, min(kBatch, d - q * kBatch));
            (void)v;
            if (threadIdx.x == 0) { sm.qtail = (int)chunks; sm.qpend = (int)chunks; sm.qhead = 0; }
            __syncthreads();
            return local_drain_async(A, sm, k, use_bloom, atom_only, lmin, gcnt);
        }
    }
    return local_drain(A, sm, k, 0, use_bloom, atom_only, lmin, gcnt, subs, tmax);
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
    if (threadIdx.x == 0) { sm.bloom_level = c.src_len; sm.bloom_on = 1; }
    __syncthreads();
}

// Decide (CTA-uniform) whether this phase's walks use the filter.  The alive
// set only shrinks, so a filter built at an earlier level stays a valid
// superset test; it is rebuilt once the alive list has halved since (fewer
// false positives).  Dead targets then cost a shared-memory probe instead of
// a scattered L2/HBM request -- the per-SM request rate is what bounds a
// cascade walked by one CTA.
__device__ __forceinline__ bool want_bloom(const KArgs &A, const Ctrl &c, Smem &sm, int64_t arcs)
{
    if (!sm.bloom_en) return false;
    const bool have = sm.bloom_on != 0;
    if (have && c.src_len * 2 > sm.bloom_level) return true;
    if (c.src_sel < 0 || c.src_len > kBloomMaxA) return have;
    // building costs one pass over the alive list per CTA: only for a walk
    // of comparable size (CTA-uniform: arcs is this CTA's pending walk)
    if (KC_BLOOM_GATE > 0 && arcs * KC_BLOOM_GATE < c.src_len * KC_BLOOM_MULT) return have;
    bloom_build(A, c, sm);
    return true;
}

// ------------------------------------------------------------------ INIT
__device__ void phase_init(const KArgs &A, Smem &sm)
{
    int lmin = INT_MAX;
    unsigned niso = 0;
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (threadIdx.x == 0) sm.removed = 0;
    for (int i = threadIdx.x; i < kQCap; i += kBlock) sm.qword[i] = 0ULL;

    __syncthreads();
    // The 0-shell is the isolated vertices: nothing can reach them, so
    // they are removed here -- claim bit set, core 0, counted as removed -- and
    // the first level is the smallest positive degree (no full scan at k = 0).
    // A warp covers 32 consecutive, aligned ids (one claim-bit word).
    static_assert(kBlock % 32 == 0, "warps cover aligned 32-vertex words");
    for (int64_t v0 = tid - lane; v0 < A.n; v0 += stride) {
        const int64_t v = v0 + lane;
        int32_t d = -1;
        if (v < A.n) {
            d = (int32_t)(ld_ro_i64(A.rowptr + v + 1) - ld_ro_i64(A.rowptr + v));
            A.deg[v] = d;
            if (d > 0) lmin = min(lmin, d);
            else A.core[v] = 0;
        }
        const unsigned iso = __ballot_sync(kFull, d == 0);
        if (lane == 0) A.claimed[v0 >> 5] = iso;
        if (iso && A.order) {  // peel order requested: the 0-shell comes first
            unsigned long long base = 0;
            if (lane == 0) base = atomicAdd(&A.S->ord_tail, (unsigned long long)__popc(iso));
            base = __shfl_sync(kFull, base, 0);
            if (d == 0) A.order[base + __popc(iso & lanemask_lt())] = (int32_t)v;
        } else if (iso && lane == 0) {
            niso += __popc(iso);
        }
    }
    if (lane == 0 && niso) atomicAdd(&sm.removed, (int)niso);
    if (threadIdx.x == 0) {
        sm.bloom_on = 0; sm.bloom_level = -1; sm.lcnt[0] = sm.lcnt[1] = 0; sm.larc[0] = sm.larc[1] = 0;
        sm.seg_cache_ok[0] = sm.seg_cache_ok[1] = 0;
    }
    block_min_atomic(sm, lmin, &A.S->min_next);  // (ends with __syncthreads)
    if (threadIdx.x == 0 && sm.removed) atomicAdd(&A.S->ord_tail, (unsigned long long)sm.removed);
}

// ------------------------------------------------------------------ LEVEL
// Scan entries [lo,hi) of list `src` (nullptr: the identity, ids lo..hi-1)
// with every warp of this CTA (Alg. 2): kScanItems entries per lane in flight;
// deg == k -> claim + route (local frontier or global queue); deg > k ->
// min for the level skip and, when compacting, ballot compaction (Fig. 8(c))
// into dst[0..) with a shared-memory cursor.  No block sync, no global atomics.
template <bool IDENT>
__device__ void scan_range(const KArgs &A, const Ctrl &c, Smem &sm, const int32_t *src, int64_t lo,
                           int64_t hi, int32_t *dst, int &lmin, int &gcnt, int32_t *ndst = nullptr,
                           unsigned long long *ntail = nullptr)
{
    const int k = c.k;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const uint64_t pol = deg_policy();
    constexpr int CH = 32 * kScanItems;
    // software pipeline: the next chunk's alive entries are loaded while this
    // chunk's degrees are in flight
    int32_t vn[kScanItems];
    auto load_chunk = [&](int64_t o) {
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            const int64_t idx = o + j * 32 + lane;
            vn[j] = -1;
            if (idx < hi) vn[j] = src ? ld_cg_i32(src + idx) : (int32_t)idx;
        }
    };
    load_chunk(lo + (int64_t)wib * CH);
#if KC_SCAN_EC
    // (ablation: block-level compaction needs every warp in every step)
    for (int64_t base = lo; base < hi; base += (int64_t)kWarps * CH) {
        const int64_t off = base + (int64_t)wib * CH;
#else
    for (int64_t off = lo + (int64_t)wib * CH; off < hi; off += (int64_t)kWarps * CH) {
#endif
        int32_t vv[kScanItems], dd[kScanItems];
        if (!KC_SCAN_PIPE && off != lo + (int64_t)wib * CH) load_chunk(off);
#pragma unroll
        for (int j = 0; j < kScanItems; j++) vv[j] = vn[j];
#pragma unroll
        for (int j = 0; j < kScanItems; j++) dd[j] = vv[j] >= 0 ? ld_deg(A.deg + vv[j], pol) : -1;
        if (KC_SCAN_PIPE) load_chunk(off + (int64_t)kWarps * CH);
        unsigned wm = 0, km = 0;
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            // deg <= k: v is in the k-shell.  Every alive vertex has deg >= k at
            // level start; atomic-only walks may already have taken a
            // not-yet-scanned k-shell vertex below k (its crossing to k+1 was
            // before this level, so no peel claims it).  Removed vertices left
            // in a lazily compacted list fail the claim.  At k = 0 the frontier
            // is the isolated vertices: nothing walks, nothing races.
#if KC_HIT_BF
            // branch-free (an empty slot has vv = dd = -1)
            const bool live = vv[j] >= 0, shell = live && dd[j] <= k;
            wm |= (shell ? 1u : 0u) << j;
            km |= (live && !shell ? 1u : 0u) << j;
            lmin = min(lmin, live && !shell ? dd[j] : INT_MAX);
#else
            if (vv[j] < 0) continue;
            if (dd[j] <= k) wm |= 1u << j;
            else { lmin = min(lmin, dd[j]); km |= 1u << j; }
#endif
        }
        // row bounds of every candidate, in flight together with its claim
        // (at k = 0 every candidate is isolated)
        int64_t b0[kScanItems], e0[kScanItems];
#pragma unroll
        for (int j = 0; j < kScanItems; j++) {
            const bool cand = ((wm >> j) & 1u) && k > 0;
            b0[j] = cand ? ld_ro_i64(A.rowptr + vv[j]) : 0;
            e0[j] = cand ? ld_ro_i64(A.rowptr + vv[j] + 1) : 0;
        }
        if (!IDENT && k > 0) {
#pragma unroll
            for (int j = 0; j < kScanItems; j++)
                if (((wm >> j) & 1u) && !claim(A, vv[j])) wm &= ~(1u << j);
        }
        if (IDENT && k > 0) {
            // identity scan (ids lo..hi-1, the first level): the 32 lanes of item j
            // hold 32 consecutive ids starting at a multiple of 32 (lo is aligned),
            // i.e. ONE claim-bit word -- one atomicOr for the warp instead of 32
            // serialised ones on the same address
#pragma unroll
            for (int j = 0; j < kScanItems; j++) {
                const unsigned bits = __ballot_sync(kFull, (wm >> j) & 1u);
                if (!bits) continue;
                uint32_t old = 0u;
                if (lane == 0) old = atom_or_claim(A.claimed + ((uint32_t)(vv[j] - lane) >> 5), bits, pol);
                old = __shfl_sync(kFull, old, 0);
                if ((old >> lane) & 1u) wm &= ~(1u << j);
            }
        }
        if (ndst) {  // near list: k < deg <= theta (a near scan's compaction, or a build)
            unsigned nm = 0;
#pragma unroll
            for (int j = 0; j < kScanItems; j++)
                if (((km >> j) & 1u) && dd[j] <= c.theta) nm |= 1u << j;
            const int mine = __popc(nm);
            int incl = mine;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += t;
            }
            const int tot = __shfl_sync(kFull, incl, 31);
            if (tot) {
                unsigned long long pos = 0;
                if (lane == 31) pos = atomicAdd(ntail, (unsigned long long)tot);
                pos = __shfl_sync(kFull, pos, 31) + (unsigned long long)(incl - mine);
#pragma unroll
                for (int j = 0; j < kScanItems; j++)
                    if ((nm >> j) & 1u) ndst[pos++] = vv[j];
            }
        }
#if KC_SCAN_EC
        if (dst) {  // the paper's block-level compaction (Fig. 9): two-stage block scan
            const unsigned long long ex = block_excl_scan(sm, (unsigned long long)__popc(km));
            int pos = sm.kcur + (int)ex;
#pragma unroll
            for (int j = 0; j < kScanItems; j++)
                if ((km >> j) & 1u) dst[pos++] = vv[j];
            __syncthreads();
            if (threadIdx.x == 0) sm.kcur += (int)sm.tot_q;
        }
        if (false) {
#else
        if (dst) {
#endif
            int mine = __popc(km), incl = mine;
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
#pragma unroll
        for (int j = 0; j < kScanItems; j++)
            if ((wm >> j) & 1u) A.core[vv[j]] = k;
        if (__any_sync(kFull, wm != 0)) {
            int32_t du[kScanItems];
#pragma unroll
            for (int j = 0; j < kScanItems; j++) du[j] = ((wm >> j) & 1u) ? (int32_t)(e0[j] - b0[j]) : 0;
#pragma unroll
            for (int j = 0; j < kScanItems; j++)
                if (du[j] > 0) prefetch_row(A.colidx, b0[j], b0[j] + du[j]);
            if constexpr (KC_ROUTE4 && kScanItems == 4) {
                route_won4(A, sm, wib, wm, vv[0], vv[1], vv[2], vv[3], du[0], du[1], du[2], du[3], b0[0], b0[1],
                           b0[2], b0[3], KC_ASYNC == 1 ? kAsyncNx : 0, gcnt);
            } else {
#pragma unroll
                for (int j = 0; j < kScanItems; j++) route_won(A, sm, wib, (wm >> j) & 1u, vv[j], du[j], b0[j], 0, gcnt);
            }
        }
    }
}

// Source layout: identity (src_sel < 0), one contiguous run (src_single) or
// per-CTA segments.  Grid mode: CTA b scans its share and compacts into its
// own segment b.  Solo mode: CTA 0 scans everything and compacts into one
// contiguous run (segment 0).
__device__ void level_scan(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk, int &lmin,
                           int &gcnt)
{
    const bool solo = (nblk == 1);
    int32_t *ndst = nullptr;
    unsigned long long *ntail = nullptr;
    if (c.near_scan || c.near_build) {
        ndst = A.near[c.near_cur ^ 1];
        ntail = &A.S->near_tail[c.near_cur ^ 1];
    }
    const int32_t *srcb = c.src_sel < 0 ? nullptr : A.alive[c.src_sel];
    int32_t *dstb = c.compact ? A.alive[c.dst_sel] : nullptr;  // (a near scan never compacts the alive list)
    const int dseg = solo ? 0 : bid;
    if (threadIdx.x == 0) sm.kcur = 0;
    __syncthreads();
    int32_t *dst = dstb ? dstb + (int64_t)dseg * A.seg_R : nullptr;
    if (!c.near_scan && c.src_sel < 0) {
        // the identity: 32-aligned slices (one claim-bit word per warp item)
        const int64_t L = c.src_len;
        const int64_t W = (L + 31) / 32;
        const int64_t lo = solo ? 0 : 32 * ((W * bid) / nblk), hi = solo ? L : min(L, 32 * ((W * (bid + 1)) / nblk));
        scan_range<true>(A, c, sm, nullptr, lo, hi, dst, lmin, gcnt, ndst, ntail);
    } else {
        // one call site for every list layout (each inlined copy of scan_range
        // grows the kernel): the near list or a contiguous alive list -- an even
        // slice per CTA; per-CTA segments -- this CTA's own, or all of them (solo)
        const bool segs = !c.near_scan && !c.src_single;
        const int nit = (segs && solo) ? A.nseg : 1;
        for (int it = 0; it < nit; it++) {
            const int32_t *src;
            int64_t lo, hi;
            if (!segs) {
                src = c.near_scan ? A.near[c.near_cur] : srcb;
                const int64_t L = c.near_scan ? c.near_len : c.src_len;
                lo = solo ? 0 : (L * bid) / nblk;
                hi = solo ? L : (L * (bid + 1)) / nblk;
            } else if (!solo) {
                // this CTA wrote its own segment's length at the last compaction
                src = srcb + (int64_t)bid * A.seg_R;
                lo = 0;
                hi = sm.seg_cache_ok[c.src_sel] ? sm.seg_cache[c.src_sel] : ld_cg_i32(A.seg_len[c.src_sel] + bid);
            } else {
                src = srcb + (int64_t)it * A.seg_R;
                lo = 0;
                hi = ld_cg_i32(A.seg_len[c.src_sel] + it);
            }
            scan_range<false>(A, c, sm, src, lo, hi, dst, lmin, gcnt, ndst, ntail);
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && dstb) {
        A.seg_len[c.dst_sel][dseg] = sm.kcur;
        sm.seg_cache[c.dst_sel] = sm.kcur;
        sm.seg_cache_ok[c.dst_sel] = solo ? 0 : 1;
        if (sm.kcur) atomicAdd(&A.S->alive_out, (unsigned long long)sm.kcur);
    }
}

// One phase.  LEVEL (Alg. 1 round k): scan this CTA's segment(s), then drain
// the local frontier breadth-first.  HUB: walk this CTA's even share of the
// global queue's arcs (non-returning when c.red), then drain what it claimed.
// LEVEL and HUB share ONE drain call site (each inlined copy of the drain
// machinery grows the kernel; measured: a larger kernel runs slower).
__device__ void run_phase(const KArgs &A, const Ctrl &c, Smem &sm, int bid, int nblk)
{
    const int wib = threadIdx.x >> 5;
    const bool hub = c.phase == PH_HUB;
    int lmin = INT_MAX, gcnt = 0;
    cta_time(A, sm, 0);
#ifdef KC_PROBE
    if (threadIdx.x == 0) s_probe_k = c.k;
#endif
    if (threadIdx.x == 0) PROBE(30, c.k * 4 + c.phase);
    if (threadIdx.x == 0) {
        sm.lcnt[0] = sm.lcnt[1] = 0; sm.larc[0] = sm.larc[1] = 0;
        sm.lphase = 0; sm.removed = 0;
        sm.bud_hub = kHub;
        sm.bud_sub = kSub;
        sm.bud_phase = kPhase;
        sm.qhead = 0; sm.qtail = 0; sm.qpend = 0; sm.qwalked = 0ULL;
        sm.near_th1 = c.near_app >= 0 ? c.theta + 1 : INT_MIN;
        sm.nclaim = hub ? 0 : 1;  // a HUB phase runs no scan: nothing races its hits
    }
    __syncthreads();
    // HUB: this CTA's share of the queue's arcs
    const int64_t gw = (int64_t)bid * kWarps + wib;
    const int64_t W = (int64_t)nblk * kWarps;
    int64_t C = (c.ae - c.as + W - 1) / W;
    C = ((C + kBatch - 1) / kBatch) * kBatch;
    const int64_t cta_arcs =
        hub ? min(c.ae, c.as + (int64_t)(bid + 1) * kWarps * C) - min(c.ae, c.as + (int64_t)bid * kWarps * C) : 0;
    if (!hub) {
        level_scan(A, c, sm, bid, nblk, lmin, gcnt);
        __syncthreads();
        cta_time(A, sm, 1);
        if (threadIdx.x == 0) PROBE(40, 0);
    }
    const bool bl = want_bloom(A, c, sm, hub ? cta_arcs : (int64_t)sm.larc[0]);
    const bool ao = (bl || KC_AO_ALWAYS) && (hub ? KC_AO_HUB : KC_AO_LOCAL);
    if (threadIdx.x == 0) {
        // (LEVEL) this CTA's scan is complete (its deg reads happen-before the release)
        if (!hub && nblk == 1) sm.nclaim = 0;  // solo: the only scan was ours
        else if (!hub && KC_NOCLAIM) red_release_add_u32(&A.S->scan_done, 1u);
        sm.spec = (bl && ao) ? 1 : 0;
    }
    int64_t walked = cta_arcs;
    if (hub) {
        __syncthreads();
        const int64_t a0 = c.as + gw * C;
        if (c.red) {  // non-returning walk; the next phase rescans (advance())
            if (a0 < c.ae) walk_red(A, sm, c.s, c.e, c.ae, a0, min(a0 + C, c.ae), bl);
            __syncthreads();
            cta_time(A, sm, 1);
            cta_time(A, sm, 2);
            cta_count(A, sm, 5, cta_arcs);
            if (threadIdx.x == 0 && cta_arcs > 0) atomicAdd(&A.S->arcs_walked, (unsigned long long)cta_arcs);
            return;
        }
        if (a0 < c.ae)
            walk<false>(A, sm, c.k, 0, KC_ASYNC == 1 ? kAsyncNx : 0, c.s, c.e, c.ae, a0, min(a0 + C, c.ae), bl, ao,
                        lmin, gcnt, KC_CF_HUB);
        __syncthreads();
        cta_time(A, sm, 1);
    }
    // (drain() begins with __syncthreads)
    int64_t subs = 0, tmax = 0;
    walked += drain(A, sm, c.k, bl, ao && KC_AO_LOCAL, lmin, gcnt, &subs, &tmax);
    if (threadIdx.x == 0) PROBE(41, 0);
    cta_time(A, sm, 2);
    gq_flush(A, sm, wib, gcnt);
    __syncthreads();
    if (threadIdx.x == 0) PROBE(42, 0);
    cta_count(A, sm, 4, subs); cta_count(A, sm, 5, walked); cta_count(A, sm, 6, sm.removed); cta_count(A, sm, 7, tmax);
    if (threadIdx.x == 0) {
        const unsigned long long wk = (unsigned long long)walked;
        if (wk) atomicAdd(&A.S->arcs_walked, wk);
        if (sm.removed) atomicAdd(&A.S->ord_tail, (unsigned long long)sm.removed);
    }
    block_min_atomic(sm, lmin, &A.S->min_next);
}

// ---------------------------------------------------------------- control
// The pure transition function (Alg. 1 l.5-9 and the level skip).  Every CTA
// applies it to identical inputs, so all copies stay identical.
// A FULL level scan (the alive list) at c.k.  With the near list enabled and
// a long alive list it also collects the next epoch's near list.
__device__ __forceinline__ void setup_full(Ctrl &c, const Params &p, int64_t removed)
{
    const int64_t live = p.n - removed;
    const int64_t src_len = c.alive_sel < 0 ? p.n : c.alive_len;
    c.phase = PH_LEVEL;
    c.src_sel = c.alive_sel;
    c.src_single = c.alive_single;
    c.src_len = src_len;
    c.compact = (live * KC_COMPACT_D < src_len * (KC_COMPACT_D - 1)) ? 1 : 0;  // >= 1/D of the source is dead
    c.dst_sel = c.alive_sel < 0 ? 0 : 1 - c.alive_sel;
    c.solo = src_len <= (int64_t)p.solo_scan;
    // a solo scan of a segmented list gathers it into one run for next time
    if (c.solo && c.alive_sel >= 0 && !c.alive_single) c.compact = 1;
    c.near_scan = 0;
    if (KC_NEAR && p.near && !c.solo && src_len >= (int64_t)p.near_min && c.near_w > 0) {
        c.near_build = 1;
        c.near_on = 1;
        c.theta = (int32_t)min((int64_t)INT_MAX - 2, (int64_t)c.k + c.near_w);
        c.near_app = c.near_cur ^ 1;  // scan and walks of this phase fill the other buffer
        c.near_reset = c.near_cur;    // the previous epoch's list is dropped at this barrier
        c.near_lv = 0;
        c.near_first = 0;
    } else {
        c.near_build = 0;
        c.near_on = 0;
        c.near_app = -1;
        c.near_reset = -1;
    }
}

// A near level scan at c.k <= theta: reads near[near_cur], compacts into the other buffer.
__device__ __forceinline__ void setup_near(Ctrl &c, const Snap &sn, const Params &p)
{
    c.phase = PH_LEVEL;
    c.near_scan = 1;
    c.near_build = 0;
    c.near_len = (int64_t)sn.near[c.near_cur];
    // the alive list stays as it is (not scanned, not compacted); the Bloom
    // filter logic keeps reading its length from src_len
    c.src_sel = c.alive_sel;
    c.src_single = c.alive_single;
    c.src_len = c.alive_sel < 0 ? p.n : c.alive_len;
    c.compact = 0;
    c.solo = 0;  // (solo near levels on CTA 0 measured 3-15 % slower: one SM's atomic rate)
    c.near_app = c.near_cur ^ 1;
    c.near_reset = c.near_cur;
    if (c.near_lv == 0) c.near_first = c.near_len;
    c.near_lv++;
    c.st_near++;
}

// The pure transition function (Alg. 1 l.5-9 and the level skip).  Every CTA
// applies it to identical inputs, so all copies stay identical.
#ifndef KC_ADV_REG
#define KC_ADV_REG 1  // advance() on a register copy of the control state (not field by field in shared memory)
#endif
#if KC_ADV_REG
__device__ __forceinline__
#else
__device__ __noinline__
#endif
void advance(Ctrl &c, const Snap &sn, const Params &p)
{
    const int64_t gcnt = (int64_t)(sn.gq >> kArcBits), garc = (int64_t)(sn.gq & kArcMask);
    const int64_t removed = (int64_t)sn.ord;
    c.level_min = min(c.level_min, sn.min);
    int next_k = 0;
    if (c.phase == PH_INIT) {
        if (removed > 0) { c.st_levels = 1; c.st_kmax = 0; }  // the 0-shell, removed by INIT
        if (removed >= p.n) {  // nothing but isolated vertices
            c.phase = PH_DONE;
            return;
        }
        next_k = c.level_min;  // smallest positive degree
        c.level_min = INT_MAX;
        c.level = -1;
    } else {
        c.st_phases++;
        if (c.solo) c.st_solo++;
        if (c.phase == PH_LEVEL) {
            c.st_scanned += c.near_scan ? c.near_len : c.src_len;
            if (c.compact) {
                c.alive_sel = c.dst_sel;
                c.alive_len = (int64_t)sn.alive_out;
                c.alive_single = c.solo;  // a solo scan compacts into one run
                c.st_compact++;
            }
            if (c.near_scan || c.near_build) c.near_cur ^= 1;  // the list this phase wrote is current
            c.near_scan = 0;
            c.near_build = 0;
        } else {
            c.st_hubarcs += c.ae - c.as;
        }
        c.near_reset = -1;
        if (removed >= p.n) {  // every vertex claimed: the rest of the level changes nothing
            if (removed > c.ord_lvl0) { c.st_levels++; c.st_kmax = c.k; }
            c.phase = PH_DONE;
            c.solo = 0;
            c.red = 0;
            return;
        }
        if (c.phase == PH_HUB && c.red) {
            // after a non-returning walk: rescan the alive list at the SAME k
            // (same level; its claims and min complete what the walk started).
            // The walk appended no theta crossings, so a near epoch restarts here.
            c.red = 0;
            setup_full(c, p, removed);
            return;
        }
        if (gcnt > c.gq_cnt) {  // hub / overflow vertices pending: HUB phase
            c.phase = PH_HUB;
            c.s = c.gq_cnt; c.e = gcnt; c.as = c.gq_arc; c.ae = garc;
            c.gq_cnt = gcnt; c.gq_arc = garc;
            c.solo = (c.ae - c.as) <= (int64_t)p.solo_arcs;
            const int64_t live = p.n - removed;
            c.red = (KC_RED_MIN > 0 && !c.solo && p.red && c.ae - c.as >= (int64_t)KC_RED_MIN &&
                     live * KC_RED_RATIO <= c.ae - c.as) ? 1 : 0;
            c.near_app = c.near_on ? c.near_cur : -1;
            return;
        }
        // level end
        if (removed > c.ord_lvl0) { c.st_levels++; c.st_kmax = c.k; }
        next_k = max(c.k + 1, c.level_min);
        if (c.near_on) {
            // vertices outside the near list have degree > theta
            next_k = max(c.k + 1, min(c.level_min, c.theta + 1));
        }
        c.level_min = INT_MAX;
    }
    // new level at next_k
    c.k = next_k;
    c.level++;
    c.ord_lvl0 = removed;
    c.arcs_lvl0 = (int64_t)sn.arcs;
    if (c.near_on && next_k <= c.theta) {
        setup_near(c, sn, p);
        return;
    }
    if (c.near_on) {  // epoch over: adapt the window to the list it produced
        const int64_t A = c.alive_sel < 0 ? p.n : c.alive_len;
        if (c.near_lv > 0 && c.near_first * 4 > A) c.near_w = max(1, c.near_w / 2);
        else if (c.near_first * 32 < A) c.near_w = min(1 << 14, c.near_w * 2);
    }
    setup_full(c, p, removed);
}

// Snapshot + reset of the counters (caller guarantees nobody else touches them).
__device__ __forceinline__ Snap take_snapshot(State *S, unsigned grid, int near_reset)
{
    Snap sn;
    sn.arcs = ld_relaxed_u64(&S->arcs_walked);
    sn.gq = ld_relaxed_u64(&S->gq_tail);
    sn.ord = ld_relaxed_u64(&S->ord_tail);
    sn.alive_out = ld_relaxed_u64(&S->alive_out);
    sn.near[0] = ld_relaxed_u64(&S->near_tail[0]);
    sn.near[1] = ld_relaxed_u64(&S->near_tail[1]);
    sn.min = ld_relaxed_i32(&S->min_next);
    sn.pad = 0;
    S->alive_out = 0ULL;
    S->min_next = INT_MAX;
    S->scan_done = 0u;
    // the list this phase consumed (a near scan's source / the previous list of
    // a build) is empty from now on; nobody appends to it until it is a scan's
    // destination again
    if (near_reset >= 0) S->near_tail[near_reset] = 0ULL;
    return sn;
}

__device__ __forceinline__ void trace_rec(State *S, const Ctrl &c, const Snap &sn, int grid)
{
    if (!KC_TRACE || !S->trace) return;
    const unsigned long long i = S->trace_n;
    if ((int64_t)i >= S->trace_cap) return;
    int64_t *r = S->trace + i * kTraceFields;
    r[0] = (int64_t)globaltimer();
    r[1] = (int64_t)clock64();
    r[2] = ((int64_t)c.phase << 8) | ((int64_t)c.solo << 4) | grid;  // phase that ENDED
    r[3] = c.k;
    r[4] = c.phase == PH_LEVEL ? c.src_len : (c.e - c.s);
    r[5] = c.phase == PH_HUB ? (c.ae - c.as) : 0;
    r[6] = (int64_t)sn.ord;
    r[7] = c.st_bar;
    S->trace_n = i + 1;
}

// Grid barrier; the last arriver snapshots+resets the counters.
//

__device__ __forceinline__ void grid_barrier(const KArgs &A, Smem &sm)
{
    __syncthreads();
    cta_time(A, sm, 3);
    if (threadIdx.x == 0) {
        State *S = A.S;
        PROBE(33, 0);
        // bar_count is monotone and every barrier adds gridDim.x, so the
        // generation follows from the ticket: one round trip to arrive.  The
        // acq_rel RMW chain on bar_count orders every CTA's counter updates
        // before the last arriver's snapshot (no separate fence).
        const uint32_t t = atom_add_acq_rel_u32(&S->bar_count, 1u);
        const uint32_t gen = t / (uint32_t)gridDim.x;
        PROBE(35, t);
        Snap sn;
        if ((t + 1u) == (uint32_t)gridDim.x * (gen + 1u)) {
            sn = take_snapshot(S, gridDim.x, sm.ctrl.near_reset);
            S->snap[(gen + 1u) & 1u] = sn;
            st_release_u32(&S->bar_gen, gen + 1u);
        } else {
            while (ld_acquire_u32(&S->bar_gen) == gen) {
            }
            PROBE(34, 0);
            const Snap *ps = &S->snap[(gen + 1u) & 1u];
            sn.arcs = ld_relaxed_u64(&ps->arcs);
            sn.gq = ld_relaxed_u64(&ps->gq);
            sn.ord = ld_relaxed_u64(&ps->ord);
            sn.alive_out = ld_relaxed_u64(&ps->alive_out);
            sn.near[0] = ld_relaxed_u64(&ps->near[0]);
            sn.near[1] = ld_relaxed_u64(&ps->near[1]);
            sn.min = ld_relaxed_i32(&ps->min);
            sn.pad = 0;
        }
        sm.snap = sn;
    }
    __syncthreads();
}


__device__ __forceinline__ void init_ctrl(Ctrl &z)
{
    z = Ctrl{};
    z.phase = PH_INIT;
    z.level_min = INT_MAX;
    z.alive_sel = -1;
    z.src_sel = -1;
    z.near_app = -1;
    z.near_reset = -1;
    z.near_w = 0;  // set from Params by the caller
}

__global__ void __launch_bounds__(kBlock, 1) k_persistent(const __grid_constant__ KArgs A)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    State *S = A.S;
    const Params p = S->prm;
    if (threadIdx.x == 0) {
        init_ctrl(sm.ctrl);
        sm.ctrl.near_w = p.near_w;
        sm.tr_cta = S->trace_cta;
        sm.tr_cap = S->trace_cap;
        sm.bloom_en = p.bloom;
    }
#ifdef KC_PROBE
    if (threadIdx.x == 0) { s_probe_n = 0u; s_probe_k = 0; }
    __syncthreads();
#endif
    phase_init(A, sm);
    grid_barrier(A, sm);
    if (threadIdx.x == 0) advance(sm.ctrl, sm.snap, p);
    __syncthreads();
    while (true) {
        if (sm.ctrl.phase == PH_DONE) break;
        // ONE call site of the phase code (a second one -- e.g. a separate solo
        // loop -- duplicates every inlined phase function: measured, the larger
        // kernel runs slower even where the copy is never executed)
        const bool solo = sm.ctrl.solo != 0;
        if (threadIdx.x == 0 && !solo) PROBE(38, 0);
        if (!solo || blockIdx.x == 0) run_phase(A, sm.ctrl, sm, solo ? 0 : blockIdx.x, solo ? 1 : gridDim.x);
        if (solo) {
            // CTA 0 alone, CTA-local synchronisation: consecutive solo phases
            // run without a grid barrier; the others wait at the next one
            if (blockIdx.x == 0) {
                if (threadIdx.x == 0) {
                    __threadfence();
                    const Snap sn = take_snapshot(S, 1u, sm.ctrl.near_reset);
                    trace_rec(S, sm.ctrl, sn, 0);
                    advance(sm.ctrl, sn, p);
                }
                __syncthreads();
                if (sm.ctrl.phase != PH_DONE && sm.ctrl.solo) continue;
                if (threadIdx.x == 0) {
                    S->pub = sm.ctrl;
                    __threadfence();
                }
            }
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
            grid_barrier(A, sm);
            if (threadIdx.x == 0) {
                PROBE(36, 0);
                if (blockIdx.x == 0) trace_rec(S, sm.ctrl, sm.snap, 1);
                sm.ctrl.st_bar++;
#if KC_ADV_REG
                Ctrl cc = sm.ctrl;
                const Snap sn = sm.snap;
                advance(cc, sn, p);
                sm.ctrl = cc;
#else
                advance(sm.ctrl, sm.snap, p);
#endif
                PROBE(37, 0);
            }
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) S->pub = sm.ctrl;  // final statistics
}

// -------------------------------------------- host-driven ablation kernels
// (KCORE_ALGO_HOSTLOOP: the paper's Alg. 1 structure -- one launch per phase
// and a host read-back of the phase after each.  No solo phases.)
__global__ void __launch_bounds__(kBlock, 1) k_phase(const __grid_constant__ KArgs A)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem &sm = *reinterpret_cast<Smem *>(smem_raw);
    if (threadIdx.x == 0) {
        sm.ctrl = A.S->pub;
        sm.tr_cta = A.S->trace_cta;
        sm.tr_cap = A.S->trace_cap;
        sm.bloom_en = A.S->prm.bloom;
        sm.bloom_on = 0;
        sm.bloom_level = -1;
        sm.seg_cache_ok[0] = sm.seg_cache_ok[1] = 0;
    }
    for (int i = threadIdx.x; i < kQCap; i += kBlock) sm.qword[i] = 0ULL;
    __syncthreads();
    const Ctrl &c = sm.ctrl;
    if (c.phase == PH_INIT) phase_init(A, sm);
    else run_phase(A, c, sm, blockIdx.x, gridDim.x);
}

__global__ void k_leader(const __grid_constant__ KArgs A, int32_t *phase_out)
{
    State *S = A.S;
    const Params p = S->prm;
    Ctrl c = S->pub;
    const Snap sn = take_snapshot(S, gridDim.x, c.near_reset);
    trace_rec(S, c, sn, 1);
    c.st_bar++;
    advance(c, sn, p);
    S->pub = c;
    *phase_out = c.phase;
}

// Hand the persisting L2 window of a call back to normal eviction priority
// (stream-ordered, after k_persistent), so later kernels get the whole L2.
__global__ void k_l2_release(const char *base, int64_t lines)
{
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < lines; i += (int64_t)gridDim.x * blockDim.x)
        asm volatile("applypriority.global.L2::evict_normal [%0], 128;" ::"l"(base + i * 128) : "memory");
}

__global__ void k_init_state(State *S, int64_t n, int32_t solo_arcs, int32_t solo_scan, int32_t bloom, int32_t red,
                             int32_t near_min, int32_t near_w,
                             int64_t *trace, int64_t *trace_cta, int64_t trace_cap)
{
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        S->gq_tail = 0ULL;
        S->ord_tail = 0ULL;
        S->alive_out = 0ULL;
        S->min_next = INT_MAX;
        S->bar_count = 0u;
        S->bar_gen = 0u;
        S->arcs_walked = 0ULL;
        S->near_tail[0] = S->near_tail[1] = 0ULL;
        S->scan_done = 0u;
        Ctrl z;
        init_ctrl(z);
        z.near_w = near_w > 0 ? near_w : KC_NEAR_W;
        S->pub = z;
        S->prm.n = n;
        S->prm.solo_arcs = solo_arcs;
        S->prm.solo_scan = solo_scan;
        S->prm.bloom = bloom;
        S->prm.red = (int16_t)(red & 1);
        S->prm.near = (int16_t)((red >> 1) & 1);
        S->prm.near_min = near_min > 0 ? near_min : KC_NEAR_MIN_A;
        S->prm.near_w = near_w > 0 ? near_w : KC_NEAR_W;
        S->trace = trace;
        S->trace_cta = trace_cta;
        S->trace_cap = trace ? trace_cap : 0;
        S->trace_n = 0ULL;
    }
}

} // namespace kc
