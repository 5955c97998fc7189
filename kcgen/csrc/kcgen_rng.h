/*
 * kcgen_rng.h -- counter-based RNG, vertex permutation and per-edge endpoint
 * draws for the synthetic graph generators (R-MAT, Erdos-Renyi, Chung-Lu).
 *
 * This header belongs to the INPUT-GENERATOR module (kcgen/).  It holds no
 * k-core arithmetic.  It is compiled into both the host generator
 * (kcgen_host.c, used for small graphs and by the CPU tests) and the device
 * generator (kcgen_device.cu, used for the full-size configs), so the two
 * produce byte-identical CSRs for the same (kind, params, seed).
 *
 * The paper evaluates on 20 real graphs (Table I); none
 * are available offline, so the configs in BASELINE.json are synthetic graphs
 * of the same shape.  Recipes: DESIGN.md "Input recipe".
 */
#ifndef KCGEN_RNG_H
#define KCGEN_RNG_H

#include <stdint.h>

#ifdef __CUDACC__
#define KCG_HD __host__ __device__ __forceinline__
#else
#define KCG_HD static inline
#endif

#define KCG_GOLDEN 0x9e3779b97f4a7c15ULL

/* splitmix64 finaliser */
KCG_HD uint64_t kcg_mix64(uint64_t z)
{
    z += KCG_GOLDEN;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

/* Draw j of item i in stream `stream` under `seed`: a pure function, so any
 * host or device thread can regenerate any edge independently. */
KCG_HD uint64_t kcg_rand(uint64_t seed, uint64_t stream, uint64_t i, uint64_t j)
{
    uint64_t key = kcg_mix64(seed * 0xd1b54a32d192ed03ULL + stream);
    return kcg_mix64(kcg_mix64(key ^ (i * 0xa0761d6478bd642fULL)) + j * KCG_GOLDEN);
}

/* uniform double in [0,1) with 53 random bits (exact on host and device) */
KCG_HD double kcg_u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

/* ---- vertex permutation: 4-round Feistel on an even number of bits with
 *      cycle-walking into [0,n).  A bijection of [0,n) keyed by the seed. ---- */
typedef struct {
    uint64_t n;
    uint32_t half;   /* bits per Feistel half */
    uint64_t mask;   /* (1<<half)-1 */
    uint64_t key;
} kcg_perm;

KCG_HD kcg_perm kcg_perm_make(uint64_t n, uint64_t seed)
{
    kcg_perm p;
    uint32_t bits = 0;
    while (bits < 64 && (1ULL << bits) < n) bits++;
    if (bits < 2) bits = 2;
    if (bits & 1) bits++;
    p.n = n;
    p.half = bits / 2;
    p.mask = (1ULL << p.half) - 1ULL;
    p.key = kcg_mix64(seed ^ 0x5851f42d4c957f2dULL);
    return p;
}

KCG_HD uint64_t kcg_feistel(const kcg_perm *p, uint64_t x)
{
    uint64_t L = (x >> p->half) & p->mask, R = x & p->mask;
    for (uint32_t r = 0; r < 4; r++) {
        uint64_t F = kcg_mix64(R ^ (p->key + (uint64_t)r * KCG_GOLDEN)) & p->mask;
        uint64_t t = L ^ F;
        L = R;
        R = t;
    }
    return (L << p->half) | R;
}

KCG_HD uint64_t kcg_perm_apply(const kcg_perm *p, uint64_t x)
{
    do { x = kcg_feistel(p, x); } while (x >= p->n);
    return x;
}

/* ---- generator kinds ---- */
enum { KCG_RMAT = 1, KCG_ER = 2, KCG_CHUNGLU = 3 };

/* R-MAT (Graph500 style, no per-level noise): for each of `scale` bits draw x
 * and pick a quadrant with probabilities (a, b, c, 1-a-b-c). */
KCG_HD void kcg_rmat_edge(uint64_t seed, uint64_t i, int scale, double a, double b, double c,
                          uint64_t *u_out, uint64_t *v_out)
{
    uint64_t u = 0, v = 0;
    double ab = a + b, abc = a + b + c;
    for (int j = 0; j < scale; j++) {
        double x = kcg_u01(kcg_rand(seed, KCG_RMAT, i, (uint64_t)j));
        uint64_t ub, vb;
        if (x < a) { ub = 0; vb = 0; }
        else if (x < ab) { ub = 0; vb = 1; }
        else if (x < abc) { ub = 1; vb = 0; }
        else { ub = 1; vb = 1; }
        u |= ub << j;
        v |= vb << j;
    }
    *u_out = u;
    *v_out = v;
}

/* Erdos-Renyi G(n, M) with M i.i.d. uniform endpoint pairs. */
KCG_HD void kcg_er_edge(uint64_t seed, uint64_t i, uint64_t n, uint64_t *u_out, uint64_t *v_out)
{
    uint64_t u = (uint64_t)(kcg_u01(kcg_rand(seed, KCG_ER, i, 0)) * (double)n);
    uint64_t v = (uint64_t)(kcg_u01(kcg_rand(seed, KCG_ER, i, 1)) * (double)n);
    if (u >= n) u = n - 1;
    if (v >= n) v = n - 1;
    *u_out = u;
    *v_out = v;
}

/* Chung-Lu: endpoint = smallest index t with cdf[t] > x (cdf[n-1] == 1). */
KCG_HD uint64_t kcg_cdf_search(const double *cdf, uint64_t n, double x)
{
    uint64_t lo = 0, hi = n - 1;
    while (lo < hi) {
        uint64_t mid = lo + (hi - lo) / 2;
        if (cdf[mid] > x) hi = mid; else lo = mid + 1;
    }
    return lo;
}

KCG_HD void kcg_chunglu_edge(uint64_t seed, uint64_t i, const double *cdf, uint64_t n,
                             uint64_t *u_out, uint64_t *v_out)
{
    *u_out = kcg_cdf_search(cdf, n, kcg_u01(kcg_rand(seed, KCG_CHUNGLU, i, 0)));
    *v_out = kcg_cdf_search(cdf, n, kcg_u01(kcg_rand(seed, KCG_CHUNGLU, i, 1)));
}

#endif
