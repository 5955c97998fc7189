/*
 * kcgen.h -- C ABI of the synthetic graph generator (input infrastructure).
 *
 * The paper's inputs are 20 real SNAP/LAW/KONECT graphs (Table I,
 * P:L400-423), undirected "by ignoring the edge direction" with
 * dense vertex ids.  No dataset is available offline, so every
 * workload is a seeded synthetic graph of the same shape (BASELINE.json
 * configs; recipe in DESIGN.md "Input recipe").  The generator holds no
 * k-core arithmetic; it feeds both the CUDA path and the CPU oracle.
 *
 * Output format (both host and device): a simple undirected graph in CSR
 * restricted to source vertices [v_begin, v_end):
 *   rowptr[v_end - v_begin + 1]  int64, rowptr[0] = 0 (local offsets)
 *   colidx[rowptr[last]]         int32 GLOBAL neighbour ids, strictly
 *                                increasing within a row (sorted, no dups),
 *                                no self-loops; the full graph is symmetric.
 * Host and device produce byte-identical arrays for the same params.
 *
 * Errors: negative return values (KCG_EINVAL -1, KCG_ENOMEM -2, KCG_ECUDA -3,
 * KCG_ECAP -4 = colidx capacity too small).
 */
#ifndef KCGEN_H
#define KCGEN_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define KCG_OK 0
#define KCG_EINVAL -1
#define KCG_ENOMEM -2
#define KCG_ECUDA -3
#define KCG_ECAP -4

typedef struct {
    int32_t kind;       /* 1 = R-MAT, 2 = Erdos-Renyi G(n,M), 3 = Chung-Lu */
    int32_t scale;      /* R-MAT: n = 2^scale (ignored otherwise)          */
    int64_t n;          /* ER / Chung-Lu: number of vertices               */
    int64_t num_edges;  /* M: generated (undirected) edge draws            */
    double a, b, c;     /* R-MAT quadrant probabilities (d = 1-a-b-c)      */
    double gamma;       /* Chung-Lu exponent; w_i = (i+1)^(-1/(gamma-1))   */
    uint64_t seed;
    int32_t permute;    /* 1: relabel vertices by a seeded Feistel bijection */
    int32_t reserved;
} kcg_params;

/* number of vertices of the generated graph */
int64_t kcg_num_vertices(const kcg_params *p);

/* Chung-Lu cumulative weights cdf[n] (double, cdf[n-1] == 1.0).  Computed on
 * the host only, so host and device draw from identical tables. */
int kcg_build_cdf(const kcg_params *p, double *cdf_out);

/* endpoints (after permutation) of generated edge i; cdf may be NULL unless
 * kind == Chung-Lu.  For tests. */
int kcg_edge(const kcg_params *p, const double *cdf, int64_t i, int64_t *u, int64_t *v);

/* Host generator.  Writes rowptr[v_end-v_begin+1] and up to colidx_cap arcs.
 * Returns the number of arcs written, or a negative error. */
int64_t kcg_host_generate(const kcg_params *p, int64_t v_begin, int64_t v_end,
                          int64_t *rowptr, int32_t *colidx, int64_t colidx_cap);

/* Device generator (all pointers are DEVICE pointers; stream is a
 * cudaStream_t).  If colidx == NULL only the arc count is computed and
 * returned.  Synchronises `stream` before returning.  Scratch is allocated
 * internally and freed before return. */
int64_t kcg_device_generate(const kcg_params *p, int64_t v_begin, int64_t v_end,
                            int64_t *rowptr, int32_t *colidx, int64_t colidx_cap,
                            void *stream);

#ifdef __cplusplus
}
#endif
#endif
