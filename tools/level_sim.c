/* level_sim.c -- analysis tool (not product, not oracle): simulate the
 * level-synchronous peel with BFS sub-rounds on a CSR and print per-level
 * statistics that decide kernel design (where arcs are walked, how many of
 * them point at alive / claimed / dead targets, alive-set sizes).
 *
 * Usage from Python: tools/level_sim.py (loads the CSR via kcgen, calls
 * level_sim() through ctypes and writes a JSON summary).
 *
 * Per level k (record of 12 int64):
 *  0 k, 1 alive at level start, 2 alive arcs at level start (sum of current
 *  degrees), 3 scan frontier size, 4 sub-rounds, 5 vertices peeled,
 *  6 arcs walked (full rows of peeled vertices), 7 arcs to targets alive and
 *  unclaimed when walked (useful decrements), 8 arcs to targets claimed in
 *  this level (incl. same sub-round), 9 arcs to targets removed in earlier
 *  levels, 10 max frontier of a sub-round, 11 arcs in the largest sub-round.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

int64_t level_sim(const int64_t *rowptr, const int32_t *colidx, int64_t n, int64_t *rec, int64_t rec_cap, int64_t *near)
{
    int32_t *deg = malloc(sizeof(int32_t) * n);
    int32_t *lvl = malloc(sizeof(int32_t) * n); /* -1 alive, else level claimed */
    int32_t *fr = malloc(sizeof(int32_t) * n);
    int32_t *nf = malloc(sizeof(int32_t) * n);
    int32_t *alive = malloc(sizeof(int32_t) * n);
    if (!deg || !lvl || !fr || !nf || !alive) return -1;
    int64_t na = 0, alive_arcs = 0;
    for (int64_t v = 0; v < n; v++) {
        deg[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
        lvl[v] = -1;
        alive[na++] = (int32_t)v;
        alive_arcs += deg[v];
    }
    int64_t nrec = 0, removed = 0;
    int32_t k = 0;
    while (removed < n) {
        int64_t r[12] = {0};
        r[0] = k;
        /* compact alive, find frontier */
        int64_t w = 0, nfr = 0, mn = INT32_MAX;
        for (int64_t i = 0; i < na; i++) {
            int32_t v = alive[i];
            if (lvl[v] >= 0) continue;
            alive[w++] = v;
        }
        na = w;
        r[1] = na;
        int64_t aa = 0;
        for (int64_t i = 0; i < na; i++) aa += deg[alive[i]];
        r[2] = aa;
        for (int64_t i = 0; i < na; i++) {
            int32_t v = alive[i];
            if (deg[v] <= k) { lvl[v] = k; fr[nfr++] = v; }
        }
        r[3] = nfr;
        if (near && nrec < rec_cap) { /* alive with deg <= k+8, k+32, k+128, 2k+2 at level start */
            int64_t *q = near + 4 * nrec; q[0] = q[1] = q[2] = q[3] = 0;
            for (int64_t i = 0; i < na; i++) {
                int32_t d = deg[alive[i]];
                q[0] += d <= k + 8; q[1] += d <= k + 32; q[2] += d <= k + 128; q[3] += d <= 2 * k + 2;
            }
        }
        while (nfr > 0) {
            r[4]++;
            r[5] += nfr;
            int64_t sub_arcs = 0, nn = 0;
            for (int64_t i = 0; i < nfr; i++) {
                int32_t v = fr[i];
                for (int64_t a = rowptr[v]; a < rowptr[v + 1]; a++) {
                    int32_t u = colidx[a];
                    sub_arcs++;
                    if (lvl[u] < 0) {
                        r[7]++;
                        if (--deg[u] == k) { lvl[u] = k; nf[nn++] = u; }
                        else if (deg[u] < mn) mn = deg[u];
                    } else if (lvl[u] == k) r[8]++;
                    else r[9]++;
                }
            }
            r[6] += sub_arcs;
            if (nfr > r[10]) r[10] = nfr;
            if (sub_arcs > r[11]) r[11] = sub_arcs;
            memcpy(fr, nf, sizeof(int32_t) * nn);
            nfr = nn;
        }
        removed += r[5];
        if (r[5] > 0 && nrec < rec_cap) { memcpy(rec + 12 * nrec, r, sizeof r); nrec++; }
        /* next level: min remaining degree */
        int32_t nk = INT32_MAX;
        for (int64_t i = 0; i < na; i++) {
            int32_t v = alive[i];
            if (lvl[v] < 0 && deg[v] < nk) nk = deg[v];
        }
        if (nk == INT32_MAX) break;
        k = nk > k + 1 ? nk : k + 1;
    }
    free(deg); free(lvl); free(fr); free(nf); free(alive);
    return nrec;
}
