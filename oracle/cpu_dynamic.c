/*
 * oracle/cpu_dynamic.c -- CPU COMPARISON BASELINE, TEST/BENCH INFRASTRUCTURE.
 *
 * The dynamic sequential CPU algorithm the paper compares against (Green et
 * al., restated as Alg. 2; Table II's "CPU" column,
 * P:444), single-threaded, generalised to Case 3 as in
 * SURVEY.md Sec. 8(a).  It is NOT the oracle (the oracle is the naive rule,
 * oracle/__init__.py); it is pinned against the oracle in tests/test_oracle.py
 * and timed by bench.py as `cpu_dynamic`.  It shares no code with the CUDA
 * path; the initial state comes from oracle_brandes (brandes.c).
 *
 * Per root s and insertion (u, v) (adjacency already holding the edge):
 *   Case 1  d[u] == d[v] (both unreachable included): nothing.
 *   Init    O(n), as in Alg. 2 lines 1-8 / Alg. 3: t[] = untouched,
 *           Delta-delta[] = 0, old d[] = d[], level buckets empty.
 *   Seed    u_high = the closer endpoint; Case 3 lowers d[u_low] to d[u_high]+1.
 *   Down    (Alg. 2 lines 9-20) level by level from u_low: sigma[w] = sum of
 *           sigma[x], x in adj(w), d[x] = d[w]-1, in canonical order (pull: the
 *           push form sigma^[w] += sigma^[v] - sigma[v] of line 17 is not
 *           bit-reproducible above 2^53); neighbours with
 *           d > L+1 are lowered (Case 3), neighbours at L+1 become t = down.
 *   Removal (Case 3) every lowered w with finite old level loses its old
 *           predecessors x not in D: Ddelta[x] -= sigma[x]/sigma_old(w)*(1+delta_old(w)).
 *   Up      (Alg. 2 lines 21-35, Alg. 8) deepest touched level down to 1:
 *           t = down: delta by Eq. (2) pull; BC += new - old; predecessors p
 *           not in D get Ddelta[p] += new - old contribution (old only over an
 *           old, non-new edge: the guard of line 32);
 *           t = up: delta += Ddelta, BC += Ddelta; at level >= 2 push
 *           sigma[p]/sigma[x]*Ddelta[x] to every predecessor p (t[p] = up).
 * Unreachable: d = INT32_MAX, sigma = 0, delta = 0.  fp64, -ffp-contract=off.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define CD_INF INT32_MAX

int oracle_brandes(int32_t n, const int64_t *row_ptr, const int32_t *col, const int32_t *roots,
                   int32_t k, int32_t *d_out, double *sigma_out, double *delta_out, double *bc_out);

enum { T_UNTOUCHED = 0, T_DOWN = 1, T_UP = 2 };

typedef struct {
    int32_t n, k;
    const int64_t *rp;   /* base CSR (copied) */
    const int32_t *col;
    int32_t *xdeg, *xcap; /* inserted neighbours per vertex, insertion order */
    int32_t **xnb;
    int32_t *roots;
    int32_t *d;           /* [k][n] */
    double *sig, *del;    /* [k][n] */
    double *bc;           /* [n] */
    /* per-update scratch, O(n) */
    uint8_t *t;
    int32_t *od;          /* old d */
    double *osig, *odel;  /* old sigma / delta (valid for D) */
    double *dd;           /* Delta-delta */
    int32_t *F, *N, *D;   /* frontiers and the down set */
    int32_t *head, *next; /* up buckets by level */
    int64_t scenarios[3];
} cd_ctx;

static void *xmalloc(size_t b) { return malloc(b ? b : 1); }

/* canonical row of v: base entries, then inserted neighbours in insertion order */
#define FOR_ROW(c, v, y, BODY)                                                      \
    do {                                                                            \
        for (int64_t j_ = (c)->rp[v]; j_ < (c)->rp[(v) + 1]; ++j_) {                \
            int32_t y = (c)->col[j_];                                               \
            BODY                                                                    \
        }                                                                           \
        for (int32_t j_ = 0; j_ < (c)->xdeg[v]; ++j_) {                             \
            int32_t y = (c)->xnb[v][j_];                                            \
            BODY                                                                    \
        }                                                                           \
    } while (0)

void *cd_create(int32_t n, const int64_t *rp, const int32_t *col, const int32_t *roots, int32_t k) {
    cd_ctx *c = (cd_ctx *)calloc(1, sizeof(cd_ctx));
    if (!c) return NULL;
    c->n = n;
    c->k = k;
    int64_t *rpc = (int64_t *)xmalloc(sizeof(int64_t) * (size_t)(n + 1));
    int32_t *colc = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)rp[n]);
    memcpy(rpc, rp, sizeof(int64_t) * (size_t)(n + 1));
    memcpy(colc, col, sizeof(int32_t) * (size_t)rp[n]);
    c->rp = rpc;
    c->col = colc;
    c->xdeg = (int32_t *)calloc((size_t)n + 1, sizeof(int32_t));
    c->xcap = (int32_t *)calloc((size_t)n + 1, sizeof(int32_t));
    c->xnb = (int32_t **)calloc((size_t)n + 1, sizeof(int32_t *));
    c->roots = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)k);
    memcpy(c->roots, roots, sizeof(int32_t) * (size_t)k);
    c->d = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)k * n);
    c->sig = (double *)xmalloc(sizeof(double) * (size_t)k * n);
    c->del = (double *)xmalloc(sizeof(double) * (size_t)k * n);
    c->bc = (double *)xmalloc(sizeof(double) * (size_t)n);
    c->t = (uint8_t *)xmalloc((size_t)n);
    c->od = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)n);
    c->osig = (double *)xmalloc(sizeof(double) * (size_t)n);
    c->odel = (double *)xmalloc(sizeof(double) * (size_t)n);
    c->dd = (double *)xmalloc(sizeof(double) * (size_t)n);
    c->F = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)n);
    c->N = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)n);
    c->D = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)n);
    c->head = (int32_t *)xmalloc(sizeof(int32_t) * ((size_t)n + 1));
    c->next = (int32_t *)xmalloc(sizeof(int32_t) * (size_t)n);
    if (oracle_brandes(n, rp, col, roots, k, c->d, c->sig, c->del, c->bc) != 0) return NULL;
    return c;
}

void cd_destroy(void *h) {
    cd_ctx *c = (cd_ctx *)h;
    if (!c) return;
    for (int32_t v = 0; v < c->n; ++v) free(c->xnb[v]);
    free((void *)c->rp); free((void *)c->col); free(c->xdeg); free(c->xcap); free(c->xnb);
    free(c->roots); free(c->d); free(c->sig); free(c->del); free(c->bc);
    free(c->t); free(c->od); free(c->osig); free(c->odel); free(c->dd);
    free(c->F); free(c->N); free(c->D); free(c->head); free(c->next);
    free(c);
}

static int append_nb(cd_ctx *c, int32_t v, int32_t y) {
    if (c->xdeg[v] == c->xcap[v]) {
        int32_t nc = c->xcap[v] ? 2 * c->xcap[v] : 4;
        int32_t *p = (int32_t *)realloc(c->xnb[v], sizeof(int32_t) * (size_t)nc);
        if (!p) return -1;
        c->xnb[v] = p;
        c->xcap[v] = nc;
    }
    c->xnb[v][c->xdeg[v]++] = y;
    return 0;
}

/* queue x (not in D) for the up phase at its level */
static void touch_up(cd_ctx *c, const int32_t *d, int32_t x) {
    if (c->t[x] != T_UNTOUCHED) return;
    c->t[x] = T_UP;
    c->next[x] = c->head[d[x]];
    c->head[d[x]] = x;
}

static void update_root(cd_ctx *c, int32_t slot, int32_t u, int32_t v) {
    const int32_t n = c->n, s = c->roots[slot];
    int32_t *d = c->d + (size_t)slot * n;
    double *sig = c->sig + (size_t)slot * n, *del = c->del + (size_t)slot * n;
    if (d[u] == d[v]) { c->scenarios[0]++; return; }  /* Case 1 */
    const int32_t uh = d[u] < d[v] ? u : v, ul = d[u] < d[v] ? v : u;
    const int case3 = d[ul] != d[uh] + 1;
    c->scenarios[case3 ? 2 : 1]++;
    /* O(n) initialisation (Alg. 2 lines 1-8) */
    for (int32_t x = 0; x < n; ++x) {
        c->t[x] = T_UNTOUCHED;
        c->dd[x] = 0.0;
        c->od[x] = d[x];
        c->head[x] = -1;
    }
    c->head[n] = -1;
    if (case3) d[ul] = d[uh] + 1;
    /* ---- down phase ---- */
    int32_t nf = 1, nd = 0, L = d[ul];
    c->F[0] = ul;
    c->t[ul] = T_DOWN;
    while (nf > 0) {
        for (int32_t i = 0; i < nf; ++i) {
            const int32_t w = c->F[i];
            c->osig[w] = sig[w];
            c->odel[w] = del[w];
            double acc = 0.0;
            FOR_ROW(c, w, x, { if (d[x] != CD_INF && d[x] == L - 1) acc = acc + sig[x]; });
            sig[w] = acc;
            c->D[nd++] = w;
        }
        int32_t nn = 0;
        for (int32_t i = 0; i < nf; ++i) {
            const int32_t w = c->F[i];
            FOR_ROW(c, w, y, {
                if (d[y] > L + 1) d[y] = L + 1; /* Case 3 pull-up; od[y] keeps the old level */
                if (d[y] == L + 1 && c->t[y] == T_UNTOUCHED) {
                    c->t[y] = T_DOWN;
                    c->N[nn++] = y;
                }
            });
        }
        int32_t *tmp = c->F; c->F = c->N; c->N = tmp;
        nf = nn;
        ++L;
    }
    int32_t lmax = 0;
    for (int32_t i = 0; i < nd; ++i) {
        const int32_t w = c->D[i];
        if (d[w] > lmax) lmax = d[w];
    }
    /* ---- (0) removal pushes: old predecessors of pulled-up vertices ---- */
    for (int32_t i = 0; i < nd; ++i) {
        const int32_t w = c->D[i];
        const int32_t ow = c->od[w];
        if (ow == d[w] || ow == CD_INF) continue;
        FOR_ROW(c, w, x, {
            if (c->t[x] != T_DOWN && d[x] == ow - 1 && !(x == uh && w == ul)) {
                c->dd[x] = c->dd[x] - (sig[x] / c->osig[w]) * (1.0 + c->odel[w]);
                touch_up(c, d, x);
                if (d[x] > lmax) lmax = d[x];
            }
        });
    }
    /* D into the level buckets (after the removal pushes: D is final) */
    for (int32_t i = 0; i < nd; ++i) {
        const int32_t w = c->D[i];
        c->next[w] = c->head[d[w]];
        c->head[d[w]] = w;
    }
    /* ---- up phase, deepest level first ---- */
    for (int32_t l = lmax; l >= 1; --l) {
        for (int32_t x = c->head[l]; x >= 0; x = c->next[x]) {
            if (c->t[x] == T_DOWN) {
                double dn = 0.0;
                FOR_ROW(c, x, y, {
                    if (d[y] != CD_INF && d[y] == l + 1) dn = dn + (sig[x] / sig[y]) * (1.0 + del[y]);
                });
                if (x != s) c->bc[x] = c->bc[x] + (dn - c->odel[x]);
                del[x] = dn;
                const int32_t ox = c->od[x];
                FOR_ROW(c, x, p, {
                    if (d[p] == l - 1 && c->t[p] != T_DOWN) {
                        double nw = (sig[p] / sig[x]) * (1.0 + del[x]);
                        double old = 0.0;
                        if (ox != CD_INF && d[p] == ox - 1 && !(p == uh && x == ul))
                            old = (sig[p] / c->osig[x]) * (1.0 + c->odel[x]);
                        c->dd[p] = c->dd[p] + (nw - old);
                        touch_up(c, d, p);
                    }
                });
            } else {
                const double g = c->dd[x];
                if (x != s) c->bc[x] = c->bc[x] + g;
                del[x] = del[x] + g;
                if (l >= 2 && g != 0.0) {
                    FOR_ROW(c, x, p, {
                        if (d[p] == l - 1 && c->t[p] != T_DOWN) {
                            c->dd[p] = c->dd[p] + (sig[p] / sig[x]) * g;
                            touch_up(c, d, p);
                        }
                    });
                }
            }
        }
    }
    del[s] = 0.0;
}

/* Insert (u, v) into the graph, then update every root (Sec. II-D).
 * Returns 0, or -1 on allocation failure.  No validation: the caller (tests,
 * bench) only passes non-edges. */
int cd_insert(void *h, int32_t u, int32_t v) {
    cd_ctx *c = (cd_ctx *)h;
    if (append_nb(c, u, v) || append_nb(c, v, u)) return -1;
    for (int32_t slot = 0; slot < c->k; ++slot) update_root(c, slot, u, v);
    return 0;
}

/* Same for a subset of root slots [s0, s1) (bench samples; BC is then partial). */
int cd_insert_roots(void *h, int32_t u, int32_t v, int32_t s0, int32_t s1) {
    cd_ctx *c = (cd_ctx *)h;
    if (append_nb(c, u, v) || append_nb(c, v, u)) return -1;
    for (int32_t slot = s0; slot < s1 && slot < c->k; ++slot) update_root(c, slot, u, v);
    return 0;
}

void cd_get(void *h, double *bc, int32_t *d, double *sig, double *del) {
    cd_ctx *c = (cd_ctx *)h;
    const size_t kn = (size_t)c->k * c->n;
    if (bc) memcpy(bc, c->bc, sizeof(double) * (size_t)c->n);
    if (d) memcpy(d, c->d, sizeof(int32_t) * kn);
    if (sig) memcpy(sig, c->sig, sizeof(double) * kn);
    if (del) memcpy(del, c->del, sizeof(double) * kn);
}

void cd_scenarios(void *h, int64_t *out3) {
    cd_ctx *c = (cd_ctx *)h;
    memcpy(out3, c->scenarios, sizeof(c->scenarios));
}
