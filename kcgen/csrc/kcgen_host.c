/*
 * kcgen_host.c -- host implementation of the synthetic graph generator
 * (see kcgen.h).  Plain C; used for small graphs and the CPU tests, and for
 * the Chung-Lu weight table shared with the device generator.
 */
#include "../include/kcgen.h"
#include "kcgen_rng.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

int64_t kcg_num_vertices(const kcg_params *p)
{
    if (!p) return KCG_EINVAL;
    if (p->kind == KCG_RMAT) {
        if (p->scale < 1 || p->scale > 31) return KCG_EINVAL;
        return (int64_t)1 << p->scale;
    }
    if (p->kind == KCG_ER || p->kind == KCG_CHUNGLU) {
        if (p->n < 1 || p->n > 0x7fffffffLL) return KCG_EINVAL;
        return p->n;
    }
    return KCG_EINVAL;
}

int kcg_build_cdf(const kcg_params *p, double *cdf)
{
    if (!p || p->kind != KCG_CHUNGLU || !cdf || p->gamma <= 1.0) return KCG_EINVAL;
    int64_t n = p->n;
    double ex = -1.0 / (p->gamma - 1.0);
    double tot = 0.0;
    for (int64_t i = 0; i < n; i++) {
        tot += pow((double)(i + 1), ex);
        cdf[i] = tot;
    }
    for (int64_t i = 0; i < n; i++) cdf[i] /= tot;
    cdf[n - 1] = 1.0;
    return KCG_OK;
}

/* raw endpoints (before permutation) */
static void raw_edge(const kcg_params *p, const double *cdf, uint64_t n, uint64_t i,
                     uint64_t *u, uint64_t *v)
{
    if (p->kind == KCG_RMAT)
        kcg_rmat_edge(p->seed, i, p->scale, p->a, p->b, p->c, u, v);
    else if (p->kind == KCG_ER)
        kcg_er_edge(p->seed, i, n, u, v);
    else
        kcg_chunglu_edge(p->seed, i, cdf, n, u, v);
}

int kcg_edge(const kcg_params *p, const double *cdf, int64_t i, int64_t *u, int64_t *v)
{
    int64_t n = kcg_num_vertices(p);
    if (n < 0 || i < 0 || i >= p->num_edges) return KCG_EINVAL;
    if (p->kind == KCG_CHUNGLU && !cdf) return KCG_EINVAL;
    uint64_t a, b;
    raw_edge(p, cdf, (uint64_t)n, (uint64_t)i, &a, &b);
    if (p->permute) {
        kcg_perm pm = kcg_perm_make((uint64_t)n, p->seed);
        a = kcg_perm_apply(&pm, a);
        b = kcg_perm_apply(&pm, b);
    }
    *u = (int64_t)a;
    *v = (int64_t)b;
    return KCG_OK;
}

/* LSD radix sort of 64-bit keys on the low `bits` bits, 16-bit digits */
static int radix_sort_u64(uint64_t *keys, int64_t cnt, int bits)
{
    if (cnt <= 1) return KCG_OK;
    uint64_t *tmp = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)cnt);
    int64_t *hist = (int64_t *)malloc(sizeof(int64_t) * 65536);
    if (!tmp || !hist) { free(tmp); free(hist); return KCG_ENOMEM; }
    uint64_t *src = keys, *dst = tmp;
    for (int shift = 0; shift < bits; shift += 16) {
        memset(hist, 0, sizeof(int64_t) * 65536);
        for (int64_t i = 0; i < cnt; i++) hist[(src[i] >> shift) & 0xffff]++;
        int64_t s = 0;
        for (int d = 0; d < 65536; d++) { int64_t c = hist[d]; hist[d] = s; s += c; }
        for (int64_t i = 0; i < cnt; i++) dst[hist[(src[i] >> shift) & 0xffff]++] = src[i];
        uint64_t *t = src; src = dst; dst = t;
    }
    if (src != keys) memcpy(keys, src, sizeof(uint64_t) * (size_t)cnt);
    free(tmp); free(hist);
    return KCG_OK;
}

int64_t kcg_host_generate(const kcg_params *p, int64_t v_begin, int64_t v_end,
                          int64_t *rowptr, int32_t *colidx, int64_t colidx_cap)
{
    int64_t n = kcg_num_vertices(p);
    if (n < 0 || p->num_edges < 0 || v_begin < 0 || v_end > n || v_begin > v_end || !rowptr)
        return KCG_EINVAL;
    double *cdf = NULL;
    if (p->kind == KCG_CHUNGLU) {
        cdf = (double *)malloc(sizeof(double) * (size_t)n);
        if (!cdf) return KCG_ENOMEM;
        kcg_build_cdf(p, cdf);
    }
    int vb = 0;
    while (((int64_t)1 << vb) < n) vb++;
    if (vb == 0) vb = 1;
    int64_t cap = 2 * p->num_edges;
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(cap > 0 ? cap : 1));
    if (!keys) { free(cdf); return KCG_ENOMEM; }
    kcg_perm pm = kcg_perm_make((uint64_t)n, p->seed);
    int64_t cnt = 0;
    for (int64_t i = 0; i < p->num_edges; i++) {
        uint64_t u, v;
        raw_edge(p, cdf, (uint64_t)n, (uint64_t)i, &u, &v);
        if (p->permute) { u = kcg_perm_apply(&pm, u); v = kcg_perm_apply(&pm, v); }
        if (u == v) continue; /* drop self-loops (reading R2) */
        if ((int64_t)u >= v_begin && (int64_t)u < v_end) keys[cnt++] = (u << vb) | v;
        if ((int64_t)v >= v_begin && (int64_t)v < v_end) keys[cnt++] = (v << vb) | u;
    }
    free(cdf);
    int rc = radix_sort_u64(keys, cnt, 2 * vb);
    if (rc) { free(keys); return rc; }
    /* unique */
    int64_t m = 0;
    for (int64_t i = 0; i < cnt; i++)
        if (i == 0 || keys[i] != keys[i - 1]) keys[m++] = keys[i];
    if (colidx && m > colidx_cap) { free(keys); return KCG_ECAP; }
    int64_t nl = v_end - v_begin;
    memset(rowptr, 0, sizeof(int64_t) * (size_t)(nl + 1));
    uint64_t mask = ((uint64_t)1 << vb) - 1;
    for (int64_t i = 0; i < m; i++) {
        int64_t src = (int64_t)(keys[i] >> vb) - v_begin;
        rowptr[src + 1]++;
        if (colidx) colidx[i] = (int32_t)(keys[i] & mask);
    }
    for (int64_t v = 0; v < nl; v++) rowptr[v + 1] += rowptr[v];
    free(keys);
    return m;
}
