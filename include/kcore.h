/*
 * kcore.h -- C ABI of the B200-native k-core decomposition library
 *            (paper_conf_icde_ahmady0gcz23_b200/lib/libkcore.so).
 *
 * Problem (Sec. I; Sec. II-A): given an undirected
 * simple graph G=(V,E), compute core(v) for every v, where the k-core is the
 * largest induced subgraph of minimum degree >= k and core(v) is the largest
 * k whose k-core contains v.  Input is CSR with dense vertex ids (P:L151-159,
 * Sec. IV "Graph Organization in GPU"); output is core(v) for all v
 * (Alg. 1 Input/Output).
 *
 * Method: level-synchronous degree-based peeling (the two-phase scan/loop
 * framework of PKC/ParK that the paper follows, Alg. 1-3
 * P:L187-298), re-designed for sm_100a as ONE persistent cooperative kernel
 * per call: deg init (Alg. 1 l.1), level scan (Alg. 2) fused with the
 * min-degree reduction for level skipping, peel sub-rounds (Alg. 3 l.12-24:
 * atomicSub returning the old value, append on old == k+1), with
 * no host round-trip between levels or sub-rounds.  The degrees are a private
 * working array, so the restore of Fig. 6 is not needed: core(v)
 * is written once, when v is claimed (reading R10).
 *
 * Conventions shared by every entry point
 *  - n      : |V|, 0 <= n < 2^31 (vertex ids are int32).
 *  - m      : number of ARCS = 2|E| = rowptr[n] (NOT |E|; reading R3),
 *             0 <= m < 2^33.
 *  - rowptr : int64[n+1], rowptr[0] = 0, non-decreasing, rowptr[n] = m.
 *  - colidx : int32[m]; row v lists N(v) strictly increasing (no duplicates),
 *             no self-loops, and the arc set is symmetric (directed
 *             inputs are made undirected by ignoring direction, reading R2).
 *             These preconditions are NOT checked on the fast path; call
 *             kcore_validate_csr() (tests/debug) to check them.
 *  - core_out: int32[n] output.  core_out[v] is written once, when v is
 *             removed at level k (the removal level is the core
 *             number); the working degrees live in the workspace.
 *  - Ownership: the caller owns all inputs/outputs; inputs are never
 *             modified; the library never frees caller memory.  Scratch
 *             (kcore_workspace_size bytes) is either caller-provided via
 *             kcore_options.workspace or allocated stream-ordered
 *             (cudaMallocAsync on `stream`) and freed before return.
 *  - Streams: device entry points are stream-ordered; results are valid once
 *             `stream` completes (no host synchronisation unless stats are
 *             requested).  `stream` is a cudaStream_t (0 = legacy default).
 *  - Errors : every function returns a kcore_status.  Argument errors are
 *             reported before any launch and leave outputs untouched.
 */
#ifndef KCORE_H
#define KCORE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    KCORE_OK = 0,
    KCORE_EINVAL = -1,      /* bad argument (null pointer, n or m out of range)     */
    KCORE_ENOMEM = -2,      /* device or host allocation failed                     */
    KCORE_ECUDA = -3,       /* CUDA launch / runtime error                          */
    KCORE_ENCCL = -4,       /* NCCL error (multi-GPU entry points)                  */
    KCORE_EGRAPH = -5,      /* only from kcore_validate_csr: input violates the CSR */
                            /* preconditions above                                  */
    KCORE_EUNSUPPORTED = -6 /* device cannot run the kernel (e.g. not sm_100)       */
} kcore_status;

/* kcore_options.flags */
#define KCORE_FLAG_NO_BLOOM 1   /* disable the shared-memory alive-set filter (ablation) */
#define KCORE_FLAG_NO_L2_PERSIST 2 /* do not pin the working degrees in L2 (ablation).  By    */
                                /* default the call launches with a persisting L2 access- */
                                /* policy window over its claim bits + working degrees,   */
                                /* raising cudaLimitPersistingL2CacheSize (device-wide)   */
                                /* to the window size if it is smaller, and returns the   */
                                /* lines to normal priority after the kernel.  A call that */
                                /* synchronises (stats != NULL, kcore_decompose_host)     */
                                /* restores the previous limit before returning; an       */
                                /* asynchronous call leaves it raised.                    */
#define KCORE_FLAG_NO_RED 4     /* ablation: heavy HUB phases keep returning atomicSub     */
                                /* (default: phases walking >= 2^21 arcs over an alive set */
                                /* <= 1/8 of them use non-returning red.global.add and a   */
                                /* rescan of the alive list at the same k)      */
#define KCORE_FLAG_NO_NEAR 8    /* ablation: every level scans the whole alive list       */
                                /* (default: long alive lists hand the next levels a near */
                                /* list of the vertices with degree <= k + W)  */

/* Algorithms selectable through kcore_options.algo. */
#define KCORE_ALGO_PERSISTENT 0 /* default: one persistent kernel, device-resident loop */
#define KCORE_ALGO_HOSTLOOP 1   /* ablation: paper Alg. 1 style host-driven loop of      */
                                /* scan/peel launches (host round-trip per sub-round)   */

typedef struct {
    int32_t algo;            /* KCORE_ALGO_*                                           */
    int32_t blocks_per_sm;   /* 0 = auto (occupancy); persistent grid = SMs x this     */
    int32_t solo_arcs;       /* > 0: HUB phases with <= this many arcs run on ONE CTA   */
                             /* with CTA-local sync (no grid barrier); 0/-1 = off      */
                             /* (default: off, slower on B200 -- DESIGN.md)            */
    int32_t solo_scan;       /* > 0: levels over <= this many alive entries run on one */
                             /* CTA; 0/-1 = off (default off)                           */
    int32_t *order_out;      /* optional DEVICE int32[n]: peel order (concatenated      */
                             /* frontiers; a degeneracy order)          */
    void *workspace;         /* optional DEVICE scratch of >= kcore_workspace_size()    */
    size_t workspace_bytes;
    int64_t *trace_out;      /* optional DEVICE int64[trace_cap][8] (trace build only:   */
                             /* lib/libkcore_trace.so; ignored by libkcore.so): one    */
                             /* record per                                              */
                             /* phase {globaltimer ns, clock64, phase<<8|solo<<4|grid,  */
                             /* k, frontier or scan length, arcs, queue count, 0}       */
    int64_t trace_cap;       /* records available at trace_out (records written are     */
                             /* reported in kcore_stats.trace_len)                      */
    int32_t flags;           /* KCORE_FLAG_* bits                                        */
    int32_t reserved1;
    int64_t *trace_cta_out;  /* optional DEVICE int64[trace_cap][grid][8]: per phase and */
                             /* CTA, globaltimer at {phase start, end of scan or queue  */
                             /* walk, end of local drain, barrier arrival, local sub-  */
                             /* rounds, arcs walked, vertices removed, largest sub-     */
                             /* round in arcs}                                          */
    int32_t near_min_alive;  /* > 0: alive-list length from which level scans build a   */
                             /* near list (default 2^17; tuning / tests)                 */
    int32_t near_window;     /* > 0: initial near window W (default 16; tuning / tests)  */
} kcore_options;

/* Run statistics (filled when a non-NULL pointer is passed; this makes the
 * call synchronise `stream`). */
typedef struct {
    int64_t levels;        /* distinct core values peeled (non-empty levels)          */
    int64_t phases;        /* LEVEL + HUB phases executed (grid-wide or single-CTA)   */
    int64_t solo_phases;   /* of which ran on a single CTA                             */
    int64_t barriers;      /* grid barriers executed                                   */
    int64_t scanned;       /* sum over levels of scanned entries (Sigma A_l)           */
    int64_t arcs_walked;   /* arcs walked by the peel (= m for a full run)            */
    int64_t compactions;   /* alive-list rewrites                                      */
    int64_t hub_arcs;      /* arcs walked in grid-wide (global queue) HUB phases       */
    int32_t kmax;          /* largest core number                                     */
    int32_t grid_blocks;   /* persistent grid size                                     */
    int32_t block_threads;
    int32_t trace_len;     /* trace records written (see kcore_options.trace_out)    */
    double kernel_ms;      /* device time of the decomposition kernel(s) (CUDA events) */
    int64_t launches;      /* kernels this call launched                              */
    int64_t near_scans;    /* level scans that read the near list instead of the     */
                           /* whole alive list (included in `scanned`)               */
    int64_t reserved[1];
} kcore_stats;

/* Core decomposition on one GPU (north-star signature).  All array pointers
 * are DEVICE pointers.  Equivalent to kcore_decompose_ex(..., NULL, NULL). */
int kcore_decompose(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                    int32_t *core_out, void *stream);

/* Same, with options (may be NULL) and statistics (may be NULL). */
int kcore_decompose_ex(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                       int32_t *core_out, void *stream, const kcore_options *opt,
                       kcore_stats *stats);

/* End-to-end variant on HOST buffers: copies rowptr/colidx host->device,
 * decomposes, copies core_out device->host, and synchronises `stream` before
 * returning.  Host buffers should be pinned for full PCIe bandwidth.
 * Device memory for the graph and scratch is allocated stream-ordered and
 * freed before return.  The first call sets the release threshold of the
 * device's default memory pool to "never" (device-wide, cudaMallocAsync users
 * only), so repeated calls reuse the pool's pages instead of re-mapping
 * gigabytes each time. */
int kcore_decompose_host(const int64_t *rowptr_host, const int32_t *colidx_host, int64_t n,
                         int64_t m, int32_t *core_out_host, void *stream,
                         const kcore_options *opt, kcore_stats *stats);

/* Scratch bytes needed by kcore_decompose_ex for a graph with n vertices and
 * m arcs (about 36 n bytes + 4 KiB). */
size_t kcore_workspace_size(int64_t n, int64_t m);

/* Check the CSR preconditions on the device (DEVICE pointers): rowptr[0]==0,
 * monotone, rowptr[n]==m, ids in range, no self-loops, rows strictly
 * increasing, symmetric.  Returns KCORE_OK, KCORE_EGRAPH, or an error.
 * Synchronises `stream`. */
int kcore_validate_csr(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m,
                       void *stream);

/* Human-readable name of a status code (static string). */
const char *kcore_strerror(int status);

/* Library version string. */
const char *kcore_version(void);

/* ---------------------------------------------------------------------------
 * Outputs derived from a decomposition.  `core` is a
 * DEVICE int32[n] core array (e.g. kcore_decompose's core_out).  All three
 * synchronise `stream` (they return host counts).  Vertex lists are in
 * increasing vertex id.
 * ------------------------------------------------------------------------- */

/* The k-shell {v : core(v) == k} (Sec. II-A).  vertices_out: DEVICE
 * int32 with room for the shell (NULL: count only).  *count_out (HOST) = its
 * size. */
int kcore_kshell(const int32_t *core, int64_t n, int32_t k, int32_t *vertices_out, int64_t *count_out,
                 void *stream);

/* Membership mask of the k-core {v : core(v) >= k} (the k-cores are
 * nested).  mask_out: DEVICE uint8[n] (1 = in the k-core).  *count_out
 * (HOST, may be NULL) = k-core size. */
int kcore_kcore_mask(const int32_t *core, int64_t n, int32_t k, uint8_t *mask_out, int64_t *count_out,
                     void *stream);

/* The k-core as an induced subgraph (k-core as the pre-processing of
 * dense-subgraph mining), vertices renumbered in increasing original id.
 * Two calls: with sub_rowptr == NULL only *nk_out / *mk_out (HOST) are
 * computed; then with DEVICE buffers sub_rowptr int64[nk+1], sub_colidx
 * int32[mk], vmap_out int32[nk] (vmap_out[new] = original id), which are
 * filled (rows sorted, symmetric, like the input). */
int kcore_kcore_subgraph(const int64_t *rowptr, const int32_t *colidx, const int32_t *core, int64_t n,
                         int64_t m, int32_t k, int64_t *nk_out, int64_t *mk_out, int64_t *sub_rowptr,
                         int32_t *sub_colidx, int32_t *vmap_out, void *stream);

/* ---------------------------------------------------------------------------
 * MPM: the paper's h-index algorithm family (P:L27,
 * P:L65-69, Fig. 2) in the bulk-synchronous form of Medusa-MPM:
 *   a_0(v) = deg(v);  a_t(v) = max{h : |{u in N(v) : a_{t-1}(u) >= h}| >= h}
 * until an iteration changes nothing (then a = core) or `max_iters`
 * iterations have run (max_iters < 0: no limit).  DEVICE rowptr/colidx/a_out
 * (int32[n], the last iterate).  *iters_out (HOST, may be NULL) = iterations
 * that changed at least one value.  One persistent cooperative kernel with
 * exact support counters (only vertices that will change are recomputed);
 * scratch (about 32 n bytes) is allocated stream-ordered.  Synchronises
 * `stream`.  stats (may be NULL): levels = phases = iterations, scanned =
 * sum of active-set sizes, arcs_walked = arcs gathered, kernel_ms. */
int kcore_mpm(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t m, int32_t *a_out,
              int64_t max_iters, int64_t *iters_out, void *stream, kcore_stats *stats);

/* ---------------------------------------------------------------------------
 * Multi-GPU: 1D vertex-range ownership (north star; the paper's multi-GPU
 * future work, with owner routing instead of a master GPU).
 * Rank r owns vertices [v_begin, v_end) and stores their rows:
 *   rowptr_local int64[v_end-v_begin+1] (local offsets, rowptr_local[0]=0),
 *   colidx_local int32[m_local] with GLOBAL neighbour ids,
 *   core_out_local int32[v_end-v_begin].
 * Ranges must tile [0, n_global) in rank order (rank 0 starts at 0).
 * Per peel sub-round every rank peels its owned frontier, applies local
 * decrements in place and routes remote ones to their owners with one NCCL
 * all-to-all; an all-reduce of {frontier non-empty, min next degree} ends
 * sub-rounds and levels.  Host-driven: synchronises `stream` once per
 * sub-round.  All ranks must call collectively.
 * ------------------------------------------------------------------------- */
int kcore_decompose_mg(const int64_t *rowptr_local, const int32_t *colidx_local,
                       int64_t n_global, int64_t v_begin, int64_t v_end, int64_t m_local,
                       int32_t *core_out_local, void *stream, void *nccl_comm,
                       kcore_stats *stats);

/* The multi-GPU protocol with `nranks` VIRTUAL ranks (1..16) on the current
 * device: the device-initiated kernel (KCORE_MG_DEVICE) with every rank's
 * window a slice of one allocation; _ex with KCORE_MG_HOSTLOOP runs the
 * host-driven protocol with a device-memory loopback transport instead of
 * NCCL (same kernels, same driver, same routing).  Takes the GLOBAL CSR (DEVICE pointers), partitions
 * it into equal vertex ranges internally and writes the global core_out.  For
 * testing the multi-GPU protocol on one GPU.  Synchronises `stream`. */
int kcore_decompose_mg_virtual(const int64_t *rowptr, const int32_t *colidx, int64_t n,
                               int64_t m, int32_t nranks, int32_t *core_out, void *stream,
                               kcore_stats *stats);

/* Multi-GPU protocol selection (kcore_decompose_mg_ex / _virtual_ex):
 *  KCORE_MG_DEVICE    device-initiated: ONE persistent
 *                     kernel per rank; decrements and frontier appends go
 *                     straight into the owner's memory (NCCL 2.28 symmetric
 *                     windows over NVLink; slices of one allocation for
 *                     virtual ranks); a device-side barrier per sub-round;
 *                     no host round trip.  Default of kcore_decompose_mg_virtual.
 *  KCORE_MG_HOSTLOOP  host-driven: grouped ncclSend/Recv of packed decrements
 *                     and an all-reduce per sub-round.  Default of
 *                     kcore_decompose_mg (the device path has not run on more
 *                     than one GPU yet). */
#define KCORE_MG_DEVICE 0
#define KCORE_MG_HOSTLOOP 1

int kcore_decompose_mg_ex(const int64_t *rowptr_local, const int32_t *colidx_local,
                          int64_t n_global, int64_t v_begin, int64_t v_end, int64_t m_local,
                          int32_t *core_out_local, void *stream, void *nccl_comm,
                          int32_t mg_algo, kcore_stats *stats);

int kcore_decompose_mg_virtual_ex(const int64_t *rowptr, const int32_t *colidx, int64_t n,
                                  int64_t m, int32_t nranks, int32_t *core_out, void *stream,
                                  int32_t mg_algo, kcore_stats *stats);

/* NCCL plumbing for callers without their own communicator (the Python
 * binding uses these; the unique id is exchanged over torch.distributed).
 * kcore_nccl_unique_id writes 128 bytes.  The comm handle is an ncclComm_t. */
int kcore_nccl_unique_id(void *id_out_128);
int kcore_nccl_comm_init(void **comm_out, int32_t nranks, const void *id_128, int32_t rank);
int kcore_nccl_comm_destroy(void *comm);

#ifdef __cplusplus
}
#endif
#endif /* KCORE_H */
