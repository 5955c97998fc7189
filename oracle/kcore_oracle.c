/*
 * kcore_oracle.c -- CPU ORACLE for k-core decomposition.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_icde_ahmady0gcz23_b200/csrc); neither includes the other.
 *
 * Citations are to /root/reference/PAPER.md lines ("P:Lnnn") and to the
 * section / algorithm they fall in.
 *
 *  - core number definition: P:L15 (Sec. I: "the k-core of a graph G=(V,E)
 *    is the largest induced subgraph with minimum degree k")
 *    (Sec. II-A: k-shell, k_max, rounds k = 0,1,2,...).
 *  - BZ serial peeling [30]: P:L25 ("removes the vertex with the smallest
 *    degree from G each time"), P:L51, P:L59 ("four carefully selected
 *    arrays").  The bin-sort listing follows Batagelj & Zaversnik [30]
 *    (restated in SURVEY.md Appendix D); there is no blocking or reordering.
 *  - h-index operator of MPM: P:L65-69 (Sec. II-A, Fig. 2).
 *
 * Input convention for every function: a simple undirected graph in CSR,
 * rowptr int64[n+1] (rowptr[0]=0), colidx int32[rowptr[n]] (each undirected
 * edge stored as two arcs).  All functions are single-threaded.
 *
 * Pins (tests/test_oracle.py): paper worked examples (Fig.1/Fig.2
 * reconstruction, Fig.6 bowtie), closed forms (K_n, C_n, trees, K_{a,b},
 * Petersen, hypercube, grid, wheel, windmill), exhaustive agreement of the
 * three independent algorithms below on every labelled graph with n<=7,
 * networkx.core_number on random graphs.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_OK 0
#define OR_ENOMEM -2
#define OR_EINVAL -1

/* ------------------------------------------------------------------------ */
/* (1) BZ [30]: O(n+m) bin-sort peeling.  SURVEY.md Appendix D.              */
/*     core_out[v] = core(v); vert_out (optional) = the removal order, which */
/*     is a degeneracy (peel) order.                                          */
/* ------------------------------------------------------------------------ */
int oracle_bz_core(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                   int32_t *core_out, int32_t *vert_out)
{
    if (n < 0) return OR_EINVAL;
    if (n == 0) return OR_OK;
    int32_t *deg = core_out; /* deg becomes core in place */
    int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    int32_t *vert = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int64_t md = 0;
    for (int64_t v = 0; v < n; v++) {
        deg[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
        if (deg[v] > md) md = deg[v];
    }
    int64_t *bin = (int64_t *)calloc((size_t)md + 1, sizeof(int64_t));
    if (!pos || !vert || !bin) { free(pos); free(vert); free(bin); return OR_ENOMEM; }
    /* counting sort of vertices by degree */
    for (int64_t v = 0; v < n; v++) bin[deg[v]]++;
    int64_t start = 0;
    for (int64_t d = 0; d <= md; d++) {
        int64_t num = bin[d];
        bin[d] = start;
        start += num;
    }
    for (int64_t v = 0; v < n; v++) {
        pos[v] = bin[deg[v]];
        vert[pos[v]] = (int32_t)v;
        bin[deg[v]]++;
    }
    for (int64_t d = md; d >= 1; d--) bin[d] = bin[d - 1];
    bin[0] = 0;
    /* main loop: process vertices in non-decreasing current degree */
    for (int64_t i = 0; i < n; i++) {
        int32_t v = vert[i];
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
            int32_t u = colidx[e];
            if (deg[u] > deg[v]) {
                int32_t du = deg[u];
                int64_t pu = pos[u];
                int64_t pw = bin[du];
                int32_t w = vert[pw];
                if (u != w) {
                    pos[u] = pw; vert[pu] = w;
                    pos[w] = pu; vert[pw] = u;
                }
                bin[du]++;
                deg[u]--;
            }
        }
    }
    if (vert_out) memcpy(vert_out, vert, sizeof(int32_t) * (size_t)n);
    free(pos); free(vert); free(bin);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* (2) Definition by repeated deletion: for k = 0,1,2,...     */
/*     start from S = V and delete every v in S with deg_S(v) < k until no   */
/*     such vertex is left; what remains is the k-core.  core(v) = largest k */
/*     whose k-core contains v.  Recomputed from V for every k (no reuse).   */
/*     O(kmax * n * (n+m)) -- small graphs only.                             */
/* ------------------------------------------------------------------------ */
int oracle_core_by_deletion(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                            int32_t *core_out)
{
    if (n < 0) return OR_EINVAL;
    if (n == 0) return OR_OK;
    char *in_s = (char *)malloc((size_t)n);
    if (!in_s) return OR_ENOMEM;
    for (int64_t v = 0; v < n; v++) core_out[v] = 0;
    for (int64_t k = 1;; k++) {
        for (int64_t v = 0; v < n; v++) in_s[v] = 1;
        int changed = 1;
        while (changed) {
            changed = 0;
            for (int64_t v = 0; v < n; v++) {
                if (!in_s[v]) continue;
                int64_t d = 0;
                for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) d += in_s[colidx[e]];
                if (d < k) { in_s[v] = 0; changed = 1; }
            }
        }
        int64_t left = 0;
        for (int64_t v = 0; v < n; v++)
            if (in_s[v]) { core_out[v] = (int32_t)k; left++; }
        if (left == 0) break;
    }
    free(in_s);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* (3) Smallest-last removal (Matula-Beck, P:L91 ref [58]; the BZ idea of    */
/*     P:L25 without the bin data structure): repeatedly delete a vertex of  */
/*     minimum current degree d; cur = max(cur, d); core(v) = cur.  O(n^2).  */
/* ------------------------------------------------------------------------ */
int oracle_core_smallest_last(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                              int32_t *core_out)
{
    if (n < 0) return OR_EINVAL;
    if (n == 0) return OR_OK;
    int64_t *d = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    char *gone = (char *)calloc((size_t)n, 1);
    if (!d || !gone) { free(d); free(gone); return OR_ENOMEM; }
    for (int64_t v = 0; v < n; v++) d[v] = rowptr[v + 1] - rowptr[v];
    int64_t cur = 0;
    for (int64_t it = 0; it < n; it++) {
        int64_t best = -1;
        for (int64_t v = 0; v < n; v++)
            if (!gone[v] && (best < 0 || d[v] < d[best])) best = v;
        if (d[best] > cur) cur = d[best];
        core_out[best] = (int32_t)cur;
        gone[best] = 1;
        for (int64_t e = rowptr[best]; e < rowptr[best + 1]; e++) {
            int32_t u = colidx[e];
            if (!gone[u]) d[u]--;
        }
    }
    free(d); free(gone);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* (4) Literal subset definition for tiny graphs (n <= 20), adjacency given  */
/*     as bitmasks adj[v]: core(v) = max over vertex subsets S containing v  */
/*     of min_{w in S} |N(w) & S|.  (If S has min degree >= k then S lies in */
/*     the k-core, the largest such subgraph.)                        */
/* ------------------------------------------------------------------------ */
static int popc32(uint32_t x) { int c = 0; while (x) { x &= x - 1; c++; } return c; }

void oracle_core_subsets_mask(int n, const uint32_t *adj, int32_t *core_out)
{
    for (int v = 0; v < n; v++) core_out[v] = 0;
    uint32_t full = (n == 32) ? 0xffffffffu : ((1u << n) - 1u);
    for (uint32_t s = 1; s <= full && s != 0; s++) {
        int mind = 1 << 30;
        for (int w = 0; w < n; w++)
            if (s & (1u << w)) {
                int dw = popc32(adj[w] & s);
                if (dw < mind) mind = dw;
            }
        for (int v = 0; v < n; v++)
            if ((s & (1u << v)) && mind > core_out[v]) core_out[v] = mind;
        if (s == full) break;
    }
}

/* Exhaustive agreement over every labelled simple graph on n vertices
 * (n <= 7: 2^21 graphs).  Runs BZ, repeated deletion, smallest-last and the
 * subset definition on each and returns the number of graphs where any two
 * disagree (0 expected).  *graphs_out = number of graphs examined. */
int64_t oracle_exhaustive_check(int n, int64_t *graphs_out)
{
    if (n < 1 || n > 7) return -1;
    int npairs = n * (n - 1) / 2;
    int pu[21], pv[21], p = 0;
    for (int a = 0; a < n; a++)
        for (int b = a + 1; b < n; b++) { pu[p] = a; pv[p] = b; p++; }
    int64_t rowptr[8];
    int32_t colidx[42];
    int32_t c1[7], c2[7], c3[7], c4[7];
    uint32_t adj[7];
    int64_t bad = 0, count = 0;
    for (uint32_t g = 0; g < (1u << npairs); g++) {
        for (int v = 0; v < n; v++) adj[v] = 0;
        for (int q = 0; q < npairs; q++)
            if (g & (1u << q)) { adj[pu[q]] |= 1u << pv[q]; adj[pv[q]] |= 1u << pu[q]; }
        int64_t e = 0;
        for (int v = 0; v < n; v++) {
            rowptr[v] = e;
            for (int w = 0; w < n; w++)
                if (adj[v] & (1u << w)) colidx[e++] = w;
        }
        rowptr[n] = e;
        oracle_bz_core(n, rowptr, colidx, c1, NULL);
        oracle_core_by_deletion(n, rowptr, colidx, c2);
        oracle_core_smallest_last(n, rowptr, colidx, c3);
        oracle_core_subsets_mask(n, adj, c4);
        for (int v = 0; v < n; v++)
            if (c1[v] != c2[v] || c1[v] != c3[v] || c1[v] != c4[v]) { bad++; break; }
        count++;
    }
    if (graphs_out) *graphs_out = count;
    return bad;
}

/* ------------------------------------------------------------------------ */
/* (5) h-index operator of MPM (Fig. 2): sort the multiset in      */
/*     non-increasing order and return max{ i : A[i] >= i } (1-based).       */
/* ------------------------------------------------------------------------ */
static int cmp_desc_i32(const void *a, const void *b)
{
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x < y) - (x > y);
}

int32_t oracle_hindex(const int32_t *vals, int64_t cnt)
{
    if (cnt <= 0) return 0;
    int32_t *s = (int32_t *)malloc(sizeof(int32_t) * (size_t)cnt);
    if (!s) return -1;
    memcpy(s, vals, sizeof(int32_t) * (size_t)cnt);
    qsort(s, (size_t)cnt, sizeof(int32_t), cmp_desc_i32);
    int32_t h = 0;
    for (int64_t i = 1; i <= cnt; i++)
        if (s[i - 1] >= i) h = (int32_t)i;
    free(s);
    return h;
}

/* ------------------------------------------------------------------------ */
/* (6) Invariants of a claimed core array.  Returns a  */
/*     bitmask of VIOLATED invariants (0 = all hold):                        */
/*      bit0 I1: 0 <= core(v) <= deg(v)                                       */
/*      bit1 I2: |{u in N(v): core(u) >= core(v)}| >= core(v)               */
/*      bit2 I3: for every k, G[{v: core(v) >= k}] has min degree >= k        */
/*      bit3 I5: core(v) == h-index{core(u) : u in N(v)}   (P:L65-69 limit)   */
/*      bit4 I6: k_max-core non-empty with min degree >= k_max        */
/* ------------------------------------------------------------------------ */
int oracle_check_invariants(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                            const int32_t *core)
{
    int bad = 0;
    int32_t kmax = 0;
    for (int64_t v = 0; v < n; v++) {
        int64_t dv = rowptr[v + 1] - rowptr[v];
        if (core[v] < 0 || core[v] > dv) bad |= 1;
        if (core[v] > kmax) kmax = core[v];
    }
    if (bad & 1) return bad; /* later checks index by core values */
    /* I2 */
    for (int64_t v = 0; v < n; v++) {
        int64_t c = 0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
            if (core[colidx[e]] >= core[v]) c++;
        if (c < core[v]) { bad |= 2; break; }
    }
    /* I3: each vertex v with core(v) >= k needs >= k neighbours with core >= k,
     * for every k in 1..core(v); the binding constraint is k = core(v) only if
     * counts are monotone, so check every k explicitly via a histogram. */
    {
        int64_t *cnt = (int64_t *)calloc((size_t)kmax + 2, sizeof(int64_t));
        if (!cnt) return -2;
        for (int64_t v = 0; v < n && !(bad & 4); v++) {
            int32_t cv = core[v];
            if (cv == 0) continue;
            memset(cnt, 0, sizeof(int64_t) * ((size_t)kmax + 2));
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
                int32_t cu = core[colidx[e]];
                cnt[cu < cv ? cu : cv]++;
            }
            /* number of neighbours with core >= k, for k = cv down to 1 */
            int64_t ge = 0;
            for (int32_t k = cv; k >= 1; k--) {
                ge += cnt[k];
                if (ge < k) { bad |= 4; break; }
            }
        }
        free(cnt);
    }
    /* I5 */
    {
        int64_t maxdeg = 0;
        for (int64_t v = 0; v < n; v++)
            if (rowptr[v + 1] - rowptr[v] > maxdeg) maxdeg = rowptr[v + 1] - rowptr[v];
        int32_t *buf = (int32_t *)malloc(sizeof(int32_t) * ((size_t)maxdeg + 1));
        if (!buf) return -2;
        for (int64_t v = 0; v < n; v++) {
            int64_t d = 0;
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) buf[d++] = core[colidx[e]];
            if (oracle_hindex(buf, d) != core[v]) { bad |= 8; break; }
        }
        free(buf);
    }
    /* I6 */
    if (n > 0 && kmax > 0) {
        int64_t members = 0;
        for (int64_t v = 0; v < n; v++) {
            if (core[v] != kmax) continue;
            members++;
            int64_t c = 0;
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
                if (core[colidx[e]] >= kmax) c++;
            if (c < kmax) bad |= 16;
        }
        if (members == 0) bad |= 16;
    }
    return bad;
}

/* ------------------------------------------------------------------------ */
/* (7) Peel-order certificate I4 (upper bound): given a */
/*     permutation `order` of V, core must be non-decreasing along order and */
/*     every v must have <= core(v) neighbours later in the order.  Together */
/*     with I2 this certifies exactness.  Returns 0 if the certificate holds,*/
/*     1 not a permutation, 2 not non-decreasing, 4 too many later nbrs.    */
/* ------------------------------------------------------------------------ */
int oracle_check_certificate(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                             const int32_t *core, const int32_t *order)
{
    int64_t *rank = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!rank) return -2;
    for (int64_t v = 0; v < n; v++) rank[v] = -1;
    for (int64_t i = 0; i < n; i++) {
        int32_t v = order[i];
        if (v < 0 || v >= n || rank[v] != -1) { free(rank); return 1; }
        rank[v] = i;
    }
    int bad = 0;
    for (int64_t i = 1; i < n; i++)
        if (core[order[i]] < core[order[i - 1]]) { bad |= 2; break; }
    for (int64_t v = 0; v < n; v++) {
        int64_t later = 0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
            if (rank[colidx[e]] > rank[v]) later++;
        if (later > core[v]) { bad |= 4; break; }
    }
    free(rank);
    return bad;
}

/* ------------------------------------------------------------------------ */
/* (8) CSR validator for the inputs both sides consume:     */
/*     0 ok; 1 rowptr; 2 id range; 3 self-loop; 4 unsorted/duplicate;       */
/*     5 asymmetric.                                                          */
/* ------------------------------------------------------------------------ */
static int has_arc(const int64_t *rowptr, const int32_t *colidx, int32_t u, int32_t v)
{
    int64_t lo = rowptr[u], hi = rowptr[u + 1];
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (colidx[mid] < v) lo = mid + 1; else hi = mid;
    }
    return lo < rowptr[u + 1] && colidx[lo] == v;
}

int oracle_validate_csr(int64_t n, int64_t arcs, const int64_t *rowptr, const int32_t *colidx)
{
    if (n < 0 || rowptr[0] != 0 || rowptr[n] != arcs) return 1;
    for (int64_t v = 0; v < n; v++)
        if (rowptr[v + 1] < rowptr[v]) return 1;
    for (int64_t v = 0; v < n; v++)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
            int32_t u = colidx[e];
            if (u < 0 || u >= n) return 2;
            if (u == v) return 3;
            if (e > rowptr[v] && colidx[e - 1] >= u) return 4;
        }
    for (int64_t v = 0; v < n; v++)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++)
            if (!has_arc(rowptr, colidx, colidx[e], (int32_t)v)) return 5;
    return 0;
}

/* ------------------------------------------------------------------------ */
/* (8) The k-core itself ("the largest induced subgraph with minimum  */
/*     degree k"), by its definition: start from S = V and delete vertices   */
/*     with fewer than k neighbours in S until none is left (a queue makes   */
/*     each deletion O(deg)).  in_core[v] = 1 iff v is in the k-core.        */
/*     Uses no core numbers.                                                  */
/* ------------------------------------------------------------------------ */
int oracle_kcore_members(int64_t n, const int64_t *rowptr, const int32_t *colidx, int64_t k,
                         uint8_t *in_core)
{
    if (n < 0) return OR_EINVAL;
    if (n == 0) return OR_OK;
    int64_t *d = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    int32_t *q = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    if (!d || !q) { free(d); free(q); return OR_ENOMEM; }
    int64_t qh = 0, qt = 0;
    for (int64_t v = 0; v < n; v++) {
        in_core[v] = 1;
        d[v] = rowptr[v + 1] - rowptr[v];
        if (d[v] < k) { in_core[v] = 0; q[qt++] = (int32_t)v; }
    }
    while (qh < qt) {
        int32_t v = q[qh++];
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
            int32_t u = colidx[e];
            if (!in_core[u]) continue;
            if (--d[u] < k) { in_core[u] = 0; q[qt++] = u; }
        }
    }
    free(d); free(q);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* (9) Induced subgraph G[S] for S = {v : keep[v]}, vertices renumbered in   */
/*     increasing original id (vmap[new] = old), rows sorted.  Call with     */
/*     rp_out == NULL to get the sizes only.                                  */
/* ------------------------------------------------------------------------ */
int oracle_induced_csr(int64_t n, const int64_t *rowptr, const int32_t *colidx, const uint8_t *keep,
                       int64_t *nk, int64_t *mk, int64_t *rp_out, int32_t *ci_out, int32_t *vmap_out)
{
    if (n < 0) return OR_EINVAL;
    int32_t *newid = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    if (!newid) return OR_ENOMEM;
    int64_t cnt = 0, arcs = 0;
    for (int64_t v = 0; v < n; v++) newid[v] = keep[v] ? (int32_t)cnt++ : -1;
    if (rp_out) rp_out[0] = 0;
    for (int64_t v = 0; v < n; v++) {
        if (!keep[v]) continue;
        if (vmap_out) vmap_out[newid[v]] = (int32_t)v;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) {
            int32_t u = colidx[e];
            if (!keep[u]) continue;
            if (ci_out) ci_out[arcs] = newid[u];
            arcs++;
        }
        if (rp_out) rp_out[newid[v] + 1] = arcs;
    }
    *nk = cnt;
    *mk = arcs;
    free(newid);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* (10) MPM [63] as the paper describes it (Fig. 2) in the        */
/*      bulk-synchronous form of Medusa-MPM (every vertex reads its  */
/*      neighbours' estimates of the previous iteration; a global flag says  */
/*      whether another iteration is needed):                                 */
/*        a_0(v) = deg(v);                                                    */
/*        a_{t+1}(v) = h-index of the multiset {a_t(u) : (u,v) in E}          */
/*      using oracle_hindex (sort non-increasing, max i with A[i] >= i).      */
/*      Runs until an iteration changes nothing or `max_iters` iterations    */
/*      have run (max_iters < 0: no limit).  a_out = the last iterate;       */
/*      *iters_out = number of iterations that changed at least one value.   */
/*      At convergence a = core.                                      */
/* ------------------------------------------------------------------------ */
int oracle_mpm(int64_t n, const int64_t *rowptr, const int32_t *colidx, int64_t max_iters,
               int32_t *a_out, int64_t *iters_out)
{
    if (n < 0) return OR_EINVAL;
    *iters_out = 0;
    if (n == 0) return OR_OK;
    int64_t md = 0;
    for (int64_t v = 0; v < n; v++)
        if (rowptr[v + 1] - rowptr[v] > md) md = rowptr[v + 1] - rowptr[v];
    int32_t *prev = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *vals = (int32_t *)malloc(sizeof(int32_t) * (size_t)(md > 0 ? md : 1));
    if (!prev || !vals) { free(prev); free(vals); return OR_ENOMEM; }
    for (int64_t v = 0; v < n; v++) a_out[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
    int64_t it = 0;
    while (max_iters < 0 || it < max_iters) {
        memcpy(prev, a_out, sizeof(int32_t) * (size_t)n);
        int changed = 0;
        for (int64_t v = 0; v < n; v++) {
            int64_t c = 0;
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; e++) vals[c++] = prev[colidx[e]];
            int32_t h = oracle_hindex(vals, c);
            if (h < 0) { free(prev); free(vals); return OR_ENOMEM; }
            if (h != prev[v]) changed = 1;
            a_out[v] = h;
        }
        if (!changed) break;
        it++;
    }
    *iters_out = it;
    free(prev); free(vals);
    return OR_OK;
}
