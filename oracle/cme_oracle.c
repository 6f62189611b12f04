/*
 * cme_oracle.c -- TEST INFRASTRUCTURE ONLY (see cme_oracle.h).
 *
 * A plain, slow, obviously correct CPU implementation of every step of the
 * CME steady-state Jacobi hot path, written from /root/reference/PAPER.md
 * ("P:Lnn") and the readings listed in DESIGN.md section 3.  No blocking,
 * fusion or reordering beyond what those definitions state.  Plain C99 +
 * optional OpenMP (only to time it on many cores; the bits do not change).
 */
#include "cme_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <float.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void oracle_free(void* p) { free(p); }

/* ------------------------------------------------------------------------ */
/* growable arrays                                                            */
/* ------------------------------------------------------------------------ */
static int grow(void** p, int64_t* cap, int64_t need, size_t elem) {
    if (need <= *cap) return 0;
    int64_t nc = *cap ? *cap : 1024;
    while (nc < need) nc *= 2;
    void* q = realloc(*p, (size_t)nc * elem);
    if (!q) return -1;
    *p = q;
    *cap = nc;
    return 0;
}

/* ------------------------------------------------------------------------ */
/* 1. Enumeration (eq. 1-2)                   */
/* ------------------------------------------------------------------------ */

/* C(x, c) by the multiplicative formula; every intermediate is itself a
 * binomial coefficient, so the division is exact.  0 if x < c. */
static uint64_t binom(int64_t x, int c) {
    if (x < c) return 0;
    uint64_t r = 1;
    for (int i = 1; i <= c; i++) r = r * (uint64_t)(x - c + i) / (uint64_t)i;
    return r;
}

/* A_k(x) = r_k * prod_i C(x_i, c_ki)   (eq. 1; index i = species). */
static double propensity(int m, const int32_t* x, const int32_t* ck, double rk) {
    uint64_t prod = 1;
    for (int i = 0; i < m; i++) prod *= binom(x[i], ck[i]);
    return rk * (double)prod;
}

/* Reaction k is enabled at x iff its propensity is > 0, the target x + nu_k is
 * non-negative and it fits the finite buffer w . y <= cap (reading R7). */
static int enabled(int m, const int32_t* x, const int32_t* ck, const int32_t* nuk, double rk,
                   const int32_t* w, int64_t cap, int32_t* y) {
    if (!(propensity(m, x, ck, rk) > 0.0)) return 0;
    int64_t load = 0;
    for (int i = 0; i < m; i++) {
        y[i] = x[i] + nuk[i];
        if (y[i] < 0) return 0;
        load += (int64_t)w[i] * y[i];
    }
    return load <= cap;
}

typedef struct {
    int m;
    int32_t* states; /* n * m */
    int64_t n, cap_states;
    int64_t* slot;   /* hash table of state indices, -1 = empty */
    int64_t tsize;
} statetab;

static uint64_t hash_state(int m, const int32_t* x) {
    uint64_t h = 1469598103934665603ULL;
    for (int i = 0; i < m; i++) {
        h ^= (uint64_t)(uint32_t)x[i];
        h *= 1099511628211ULL;
        h ^= h >> 29;
    }
    return h;
}

static int64_t tab_find(const statetab* t, const int32_t* x) {
    uint64_t mask = (uint64_t)t->tsize - 1, h = hash_state(t->m, x) & mask;
    for (;;) {
        int64_t s = t->slot[h];
        if (s < 0) return -1;
        if (memcmp(t->states + s * t->m, x, sizeof(int32_t) * t->m) == 0) return s;
        h = (h + 1) & mask;
    }
}

static int tab_rehash(statetab* t, int64_t newsize) {
    int64_t* ns = (int64_t*)malloc(sizeof(int64_t) * newsize);
    if (!ns) return -1;
    for (int64_t i = 0; i < newsize; i++) ns[i] = -1;
    uint64_t mask = (uint64_t)newsize - 1;
    for (int64_t s = 0; s < t->n; s++) {
        uint64_t h = hash_state(t->m, t->states + s * t->m) & mask;
        while (ns[h] >= 0) h = (h + 1) & mask;
        ns[h] = s;
    }
    free(t->slot);
    t->slot = ns;
    t->tsize = newsize;
    return 0;
}

static int64_t tab_add(statetab* t, const int32_t* x) {
    if ((t->n + 1) * 2 > t->tsize && tab_rehash(t, t->tsize * 2)) return -1;
    if (grow((void**)&t->states, &t->cap_states, (t->n + 1) * t->m, sizeof(int32_t))) return -1;
    memcpy(t->states + t->n * t->m, x, sizeof(int32_t) * t->m);
    uint64_t mask = (uint64_t)t->tsize - 1, h = hash_state(t->m, x) & mask;
    while (t->slot[h] >= 0) h = (h + 1) & mask;
    t->slot[h] = t->n;
    return t->n++;
}

int oracle_enumerate(int m, const int32_t* x0, int R, const int32_t* reac, const int32_t* change,
                     const double* rates, const int32_t* w, int64_t cap,
                     int64_t* n_out, int64_t* nnz_out, int32_t** states_out,
                     int32_t** row_out, int32_t** col_out, double** rate_out) {
    if (m <= 0 || R <= 0 || !x0 || !reac || !change || !rates || !w) return ORACLE_INVALID_ARG;
    for (int k = 0; k < R; k++) {
        int nz = 0;
        for (int i = 0; i < m; i++) nz |= change[k * m + i] != 0;
        if (!nz || !(rates[k] >= 0.0)) return ORACLE_INVALID_ARG;
    }
    int64_t load0 = 0;
    for (int i = 0; i < m; i++) {
        if (x0[i] < 0) return ORACLE_INVALID_ARG;
        load0 += (int64_t)w[i] * x0[i];
    }
    if (load0 > cap) return ORACLE_INVALID_ARG;

    statetab t = {m, NULL, 0, 0, NULL, 0};
    if (tab_rehash(&t, 1 << 16)) return ORACLE_OOM;
    int32_t* y = (int32_t*)malloc(sizeof(int32_t) * m);
    int64_t* st_node = NULL; int32_t* st_k = NULL; int64_t st_cap = 0, st_cap2 = 0, sp = 0;
    int64_t* tgt = NULL; int64_t tgt_cap = 0;   /* tgt[j*R+k]: target of reaction k at j, -1 = disabled */
    int rc = ORACLE_OOM;
    if (!y || tab_add(&t, x0) < 0) goto fail;
    if (grow((void**)&st_node, &st_cap, 1, sizeof(int64_t)) ||
        grow((void**)&st_k, &st_cap2, 1, sizeof(int32_t)) ||
        grow((void**)&tgt, &tgt_cap, R, sizeof(int64_t))) goto fail;
    for (int k = 0; k < R; k++) tgt[k] = -1;
    st_node[0] = 0; st_k[0] = 0; sp = 1;
    /* recursive DFS preorder with an explicit stack of (state, next reaction):
     * a state is numbered when first reached and explored at once (reading R9).
     * Every (state, reaction) pair is tried exactly once; its target is kept. */
    while (sp > 0) {
        int64_t j = st_node[sp - 1];
        int k = st_k[sp - 1];
        if (k >= R) { sp--; continue; }
        st_k[sp - 1] = k + 1;
        const int32_t* xj = t.states + j * m;
        if (!enabled(m, xj, reac + k * m, change + k * m, rates[k], w, cap, y)) continue;
        int64_t id = tab_find(&t, y);
        if (id >= 0) { tgt[j * R + k] = id; continue; }
        id = tab_add(&t, y);
        if (id < 0) goto fail;
        if (grow((void**)&tgt, &tgt_cap, (id + 1) * R, sizeof(int64_t))) goto fail;
        for (int q = 0; q < R; q++) tgt[id * R + q] = -1;
        tgt[j * R + k] = id;
        if (grow((void**)&st_node, &st_cap, sp + 1, sizeof(int64_t)) ||
            grow((void**)&st_k, &st_cap2, sp + 1, sizeof(int32_t))) goto fail;
        st_node[sp] = id; st_k[sp] = 0; sp++;
    }
    free(st_node); st_node = NULL; free(st_k); st_k = NULL;

    {
        int64_t n0 = t.n;
        uint8_t* alive = (uint8_t*)malloc(n0);
        int64_t* newid = (int64_t*)malloc(sizeof(int64_t) * n0);
        if (!alive || !newid) { free(alive); free(newid); goto fail; }
        for (int64_t j = 0; j < n0; j++) alive[j] = 1;
        /* delete zero-outflow states and the edges into them, to a fixpoint (R8) */
        int changed = 1;
        while (changed) {
            changed = 0;
            for (int64_t j = 0; j < n0; j++) {
                if (!alive[j]) continue;
                int out = 0;
                for (int k = 0; k < R; k++) {
                    int64_t s = tgt[j * R + k];
                    if (s >= 0 && alive[s]) out++;
                }
                if (out == 0) { alive[j] = 0; changed = 1; }
            }
        }
        int64_t n = 0, nnz = 0;
        for (int64_t j = 0; j < n0; j++) newid[j] = alive[j] ? n++ : -1;
        for (int64_t j = 0; j < n0; j++) {
            if (!alive[j]) continue;
            for (int k = 0; k < R; k++) {
                int64_t s = tgt[j * R + k];
                if (s >= 0 && alive[s]) nnz++;
            }
        }
        int32_t* S = (int32_t*)malloc(sizeof(int32_t) * (n ? n : 1) * m);
        int32_t* Ro = (int32_t*)malloc(sizeof(int32_t) * (nnz ? nnz : 1));
        int32_t* Co = (int32_t*)malloc(sizeof(int32_t) * (nnz ? nnz : 1));
        double* Vo = (double*)malloc(sizeof(double) * (nnz ? nnz : 1));
        if (!S || !Ro || !Co || !Vo) {
            free(S); free(Ro); free(Co); free(Vo); free(alive); free(newid);
            goto fail;
        }
        int64_t e = 0;
        for (int64_t j = 0; j < n0; j++) {
            if (!alive[j]) continue;
            const int32_t* xj = t.states + j * m;
            memcpy(S + newid[j] * m, xj, sizeof(int32_t) * m);
            for (int k = 0; k < R; k++) {
                int64_t s = tgt[j * R + k];
                if (s < 0 || !alive[s]) continue;
                Ro[e] = (int32_t)newid[s];
                Co[e] = (int32_t)newid[j];
                Vo[e] = propensity(m, xj, reac + k * m, rates[k]);
                e++;
            }
        }
        free(alive); free(newid);
        *n_out = n; *nnz_out = nnz;
        *states_out = S; *row_out = Ro; *col_out = Co; *rate_out = Vo;
        rc = ORACLE_OK;
    }
fail:
    free(st_node); free(st_k); free(tgt); free(y); free(t.states); free(t.slot);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* 2. Ingest: COO -> CSR + diagonal                                */
/* ------------------------------------------------------------------------ */
int oracle_ingest(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col, const double* rate,
                  int diag_given, int64_t** row_ptr_out, int32_t** col_out, double** val_out,
                  double** diag_out) {
    if (n <= 0 || n > 2147483647LL || nnz < 0 || (nnz > 0 && (!row || !col || !rate)))
        return ORACLE_INVALID_ARG;
    for (int64_t e = 0; e < nnz; e++) {
        if (row[e] < 0 || row[e] >= n || col[e] < 0 || col[e] >= n) return ORACLE_INVALID_ARG;
        if (isnan(rate[e]) || isinf(rate[e])) return ORACLE_INVALID_ARG;
        if (row[e] == col[e]) {
            if (!diag_given) return ORACLE_INVALID_ARG;
            continue;                       /* a given a_ii is negative */
        }
        if (rate[e] < 0.0) return ORACLE_NEGATIVE_RATE;
    }
    /* stable sort by (row, col): counting sort on col, then stable on row */
    int64_t* cnt = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    int64_t* tmp = (int64_t*)malloc(sizeof(int64_t) * (nnz ? nnz : 1));
    int64_t* ord = (int64_t*)malloc(sizeof(int64_t) * (nnz ? nnz : 1));
    double* given = (double*)calloc((size_t)n, sizeof(double));
    if (!cnt || !tmp || !ord || !given) { free(cnt); free(tmp); free(ord); free(given); return ORACLE_OOM; }
    for (int64_t e = 0; e < nnz; e++) cnt[col[e] + 1]++;
    for (int64_t i = 0; i < n; i++) cnt[i + 1] += cnt[i];
    for (int64_t e = 0; e < nnz; e++) tmp[cnt[col[e]]++] = e;
    memset(cnt, 0, sizeof(int64_t) * ((size_t)n + 1));
    for (int64_t e = 0; e < nnz; e++) cnt[row[e] + 1]++;
    for (int64_t i = 0; i < n; i++) cnt[i + 1] += cnt[i];
    for (int64_t q = 0; q < nnz; q++) { int64_t e = tmp[q]; ord[cnt[row[e]]++] = e; }
    free(tmp);
    /* merge duplicates in input order (eq. 2: A = sum_k A_k), drop exact zeros */
    int64_t* rp = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t* cj = (int32_t*)malloc(sizeof(int32_t) * (nnz ? nnz : 1));
    double* vv = (double*)malloc(sizeof(double) * (nnz ? nnz : 1));
    double* d = (double*)malloc(sizeof(double) * n);
    if (!rp || !cj || !vv || !d) {
        free(cnt); free(ord); free(given); free(rp); free(cj); free(vv); free(d);
        return ORACLE_OOM;
    }
    int64_t out = 0;
    int64_t q = 0;
    for (int64_t i = 0; i < n; i++) {
        rp[i] = out;
        while (q < nnz && row[ord[q]] == i) {
            int32_t j = col[ord[q]];
            double s = 0.0;
            while (q < nnz && row[ord[q]] == i && col[ord[q]] == j) { s += rate[ord[q]]; q++; }
            if (j == i) { given[i] += s; continue; }  /* only reachable when diag_given */
            if (s != 0.0) { cj[out] = j; vv[out] = s; out++; }
        }
    }
    rp[n] = out;
    free(cnt); free(ord);
    /* column sums in ascending row order; A(x,x) = -sum_{x'!=x} A(x',x) */
    double* colsum = (double*)calloc((size_t)n, sizeof(double));
    if (!colsum) { free(given); free(rp); free(cj); free(vv); free(d); return ORACLE_OOM; }
    for (int64_t i = 0; i < n; i++)
        for (int64_t p = rp[i]; p < rp[i + 1]; p++) colsum[cj[p]] += vv[p];
    int rc = ORACLE_OK;
    for (int64_t j = 0; j < n && rc == ORACLE_OK; j++) {
        if (colsum[j] == 0.0) { rc = ORACLE_ZERO_OUTFLOW; break; }
        if (!diag_given) {
            d[j] = -colsum[j];
        } else {
            d[j] = given[j];
            if (!(d[j] < 0.0) || fabs(colsum[j] + d[j]) > 64.0 * DBL_EPSILON * fabs(d[j]))
                rc = ORACLE_INVALID_ARG;
        }
    }
    free(colsum); free(given);
    if (rc != ORACLE_OK) { free(rp); free(cj); free(vv); free(d); return rc; }
    *row_ptr_out = rp; *col_out = cj; *val_out = vv; *diag_out = d;
    return ORACLE_OK;
}

/* transpose pattern: for column j the rows i with a_ij != 0, ascending i */
static int transpose_pattern(int64_t n, const int64_t* rp, const int32_t* col, int64_t** cp_out,
                             int32_t** ri_out) {
    int64_t nnz = rp[n];
    int64_t* cp = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t* ri = (int32_t*)malloc(sizeof(int32_t) * (nnz ? nnz : 1));
    int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (n ? n : 1));
    if (!cp || !ri || !pos) { free(cp); free(ri); free(pos); return -1; }
    for (int64_t p = 0; p < nnz; p++) cp[col[p] + 1]++;
    for (int64_t j = 0; j < n; j++) cp[j + 1] += cp[j];
    for (int64_t j = 0; j < n; j++) pos[j] = cp[j];
    for (int64_t i = 0; i < n; i++)
        for (int64_t p = rp[i]; p < rp[i + 1]; p++) ri[pos[col[p]]++] = (int32_t)i;
    free(pos);
    *cp_out = cp; *ri_out = ri;
    return 0;
}

/* ------------------------------------------------------------------------ */
/* 3. Orderings                                                               */
/* ------------------------------------------------------------------------ */
/* DFS preorder of the transition graph j -> i (a_ij != 0), out-neighbours in
 * ascending index, from root, restarting at the smallest unvisited state
 * (reading R11). */
int oracle_order_dfs(int64_t n, const int64_t* row_ptr, const int32_t* col, int64_t root,
                     int32_t* new_to_old) {
    if (n <= 0 || root < 0 || root >= n || !new_to_old) return ORACLE_INVALID_ARG;
    int64_t* cp; int32_t* ri;
    if (transpose_pattern(n, row_ptr, col, &cp, &ri)) return ORACLE_OOM;
    uint8_t* seen = (uint8_t*)calloc((size_t)n, 1);
    int64_t* stn = (int64_t*)malloc(sizeof(int64_t) * n);
    int64_t* stp = (int64_t*)malloc(sizeof(int64_t) * n);
    if (!seen || !stn || !stp) { free(cp); free(ri); free(seen); free(stn); free(stp); return ORACLE_OOM; }
    int64_t next = 0, scan = 0;
    int64_t start = root;
    while (next < n) {
        if (start < 0) {
            while (seen[scan]) scan++;
            start = scan;
        }
        int64_t sp = 0;
        seen[start] = 1; new_to_old[next++] = (int32_t)start;
        stn[sp] = start; stp[sp] = cp[start]; sp++;
        while (sp > 0) {
            int64_t u = stn[sp - 1];
            if (stp[sp - 1] >= cp[u + 1]) { sp--; continue; }
            int64_t v = ri[stp[sp - 1]++];
            if (seen[v]) continue;
            seen[v] = 1; new_to_old[next++] = (int32_t)v;
            stn[sp] = v; stp[sp] = cp[v]; sp++;
        }
        start = -1;
    }
    free(cp); free(ri); free(seen); free(stn); free(stp);
    return ORACLE_OK;
}

/* undirected off-diagonal pattern of A + A^T, neighbour lists ascending */
static int sym_pattern(int64_t n, const int64_t* rp, const int32_t* col, int64_t** sp_out,
                       int32_t** sj_out) {
    int64_t* cp; int32_t* ri;
    if (transpose_pattern(n, rp, col, &cp, &ri)) return -1;
    int64_t* sp = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t* sj = (int32_t*)malloc(sizeof(int32_t) * (2 * rp[n] + 1));
    if (!sp || !sj) { free(cp); free(ri); free(sp); free(sj); return -1; }
    int64_t out = 0;
    for (int64_t i = 0; i < n; i++) {
        sp[i] = out;
        int64_t a = rp[i], ae = rp[i + 1], b = cp[i], be = cp[i + 1];
        int64_t last = -1;
        while (a < ae || b < be) {
            int64_t v;
            if (b >= be || (a < ae && col[a] <= ri[b])) v = col[a++];
            else v = ri[b++];
            if (v == i || v == last) continue;
            sj[out++] = (int32_t)v; last = v;
        }
    }
    sp[n] = out;
    free(cp); free(ri);
    *sp_out = sp; *sj_out = sj;
    return 0;
}

/* BFS from s over unmarked-by-other-components vertices; returns eccentricity,
 * fills lvl (stamped via `mark`) and the last level's vertices in order. */
static int64_t bfs_levels(int64_t s, const int64_t* sp, const int32_t* sj, int64_t* lvl,
                          int64_t* queue, int64_t* qlen_out, int64_t* last_begin) {
    int64_t h = 0, t = 0;
    queue[t++] = s; lvl[s] = 0;
    int64_t ecc = 0;
    while (h < t) {
        int64_t u = queue[h++];
        for (int64_t p = sp[u]; p < sp[u + 1]; p++) {
            int64_t v = sj[p];
            if (lvl[v] >= 0) continue;
            lvl[v] = lvl[u] + 1;
            if (lvl[v] > ecc) ecc = lvl[v];
            queue[t++] = v;
        }
    }
    int64_t lb = t;
    while (lb > 0 && lvl[queue[lb - 1]] == ecc) lb--;
    *qlen_out = t; *last_begin = lb;
    return ecc;
}

/* Reverse Cuthill-McKee with George-Liu pseudo-peripheral start (reading R12). */
int oracle_order_rcm(int64_t n, const int64_t* row_ptr, const int32_t* col, int32_t* new_to_old) {
    if (n <= 0 || !new_to_old) return ORACLE_INVALID_ARG;
    int64_t* sp; int32_t* sj;
    if (sym_pattern(n, row_ptr, col, &sp, &sj)) return ORACLE_OOM;
    int64_t* lvl = (int64_t*)malloc(sizeof(int64_t) * n);
    int64_t* queue = (int64_t*)malloc(sizeof(int64_t) * n);
    uint8_t* done = (uint8_t*)calloc((size_t)n, 1);
    int32_t* order = (int32_t*)malloc(sizeof(int32_t) * n);
    int64_t* nb = (int64_t*)malloc(sizeof(int64_t) * (n + 1));
    if (!lvl || !queue || !done || !order || !nb) {
        free(sp); free(sj); free(lvl); free(queue); free(done); free(order); free(nb);
        return ORACLE_OOM;
    }
    for (int64_t i = 0; i < n; i++) lvl[i] = -1;
    int64_t placed = 0;
    for (int64_t v0 = 0; v0 < n; v0++) {
        if (done[v0]) continue;
        /* the component of v0 (all its vertices are not yet done) */
        int64_t qlen, lb;
        bfs_levels(v0, sp, sj, lvl, queue, &qlen, &lb);
        int64_t best = v0;
        for (int64_t q = 0; q < qlen; q++) {
            int64_t u = queue[q];
            int64_t du = sp[u + 1] - sp[u], db = sp[best + 1] - sp[best];
            if (du < db || (du == db && u < best)) best = u;
        }
        for (int64_t q = 0; q < qlen; q++) lvl[queue[q]] = -1;
        /* pseudo-peripheral search */
        int64_t ecc = bfs_levels(best, sp, sj, lvl, queue, &qlen, &lb);
        for (;;) {
            int64_t cand = -1;
            for (int64_t q = lb; q < qlen; q++) {
                int64_t u = queue[q];
                if (cand < 0) { cand = u; continue; }
                int64_t du = sp[u + 1] - sp[u], dc = sp[cand + 1] - sp[cand];
                if (du < dc || (du == dc && u < cand)) cand = u;
            }
            for (int64_t q = 0; q < qlen; q++) lvl[queue[q]] = -1;
            int64_t e2 = bfs_levels(cand, sp, sj, lvl, queue, &qlen, &lb);
            if (e2 > ecc) { ecc = e2; best = cand; continue; }
            for (int64_t q = 0; q < qlen; q++) lvl[queue[q]] = -1;
            break;
        }
        /* Cuthill-McKee BFS: unvisited neighbours appended by (degree, index) */
        int64_t h = placed, t = placed;
        order[t++] = (int32_t)best; done[best] = 1;
        while (h < t) {
            int64_t u = order[h++];
            int64_t k = 0;
            for (int64_t p = sp[u]; p < sp[u + 1]; p++) {
                int64_t v = sj[p];
                if (done[v]) continue;
                done[v] = 1;
                /* insertion sort by (degree, index) */
                int64_t dv = sp[v + 1] - sp[v];
                int64_t a = k++;
                while (a > 0) {
                    int64_t w2 = nb[a - 1], dw = sp[w2 + 1] - sp[w2];
                    if (dw < dv || (dw == dv && w2 < v)) break;
                    nb[a] = nb[a - 1]; a--;
                }
                nb[a] = v;
            }
            for (int64_t a = 0; a < k; a++) order[t++] = (int32_t)nb[a];
        }
        placed = t;
    }
    for (int64_t r = 0; r < n; r++) new_to_old[r] = order[n - 1 - r];
    free(sp); free(sj); free(lvl); free(queue); free(done); free(order); free(nb);
    return ORACLE_OK;
}

int oracle_permute(int64_t n, const int64_t* row_ptr, const int32_t* col, const double* val,
                   const double* diag, const int32_t* p, int64_t** rp_out, int32_t** col_out,
                   double** val_out, double** diag_out) {
    int64_t nnz = row_ptr[n];
    int32_t* inv = (int32_t*)malloc(sizeof(int32_t) * n);
    int64_t* rp = (int64_t*)malloc(sizeof(int64_t) * (n + 1));
    int32_t* cj = (int32_t*)malloc(sizeof(int32_t) * (nnz ? nnz : 1));
    double* vv = (double*)malloc(sizeof(double) * (nnz ? nnz : 1));
    double* d = (double*)malloc(sizeof(double) * n);
    if (!inv || !rp || !cj || !vv || !d) {
        free(inv); free(rp); free(cj); free(vv); free(d); return ORACLE_OOM;
    }
    for (int64_t i = 0; i < n; i++) inv[i] = -1;
    for (int64_t r = 0; r < n; r++) {
        if (p[r] < 0 || p[r] >= n || inv[p[r]] >= 0) {
            free(inv); free(rp); free(cj); free(vv); free(d); return ORACLE_INVALID_ARG;
        }
        inv[p[r]] = (int32_t)r;
    }
    int64_t out = 0;
    for (int64_t r = 0; r < n; r++) {
        int64_t o = p[r];
        rp[r] = out;
        d[r] = diag[o];
        for (int64_t q = row_ptr[o]; q < row_ptr[o + 1]; q++) {
            int32_t c = inv[col[q]];
            double v = val[q];
            int64_t a = out++;
            while (a > rp[r] && cj[a - 1] > c) { cj[a] = cj[a - 1]; vv[a] = vv[a - 1]; a--; }
            cj[a] = c; vv[a] = v;
        }
    }
    rp[n] = out;
    free(inv);
    *rp_out = rp; *col_out = cj; *val_out = vv; *diag_out = d;
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------ */
/* 4. Directed period (reading R1: chooses the default omega)                 */
/* ------------------------------------------------------------------------ */
static int64_t gcd64(int64_t a, int64_t b) {
    if (a < 0) a = -a;
    if (b < 0) b = -b;
    while (b) { int64_t t = a % b; a = b; b = t; }
    return a;
}

int64_t oracle_period(int64_t n, const int64_t* row_ptr, const int32_t* col, int64_t root) {
    if (n <= 0 || root < 0 || root >= n) return -1;
    int64_t* cp; int32_t* ri;
    if (transpose_pattern(n, row_ptr, col, &cp, &ri)) return -1;
    int64_t* lvl = (int64_t*)malloc(sizeof(int64_t) * n);
    int64_t* queue = (int64_t*)malloc(sizeof(int64_t) * n);
    if (!lvl || !queue) { free(cp); free(ri); free(lvl); free(queue); return -1; }
    for (int64_t i = 0; i < n; i++) lvl[i] = -1;
    int64_t scan = 0, start = root;
    for (;;) {
        if (start < 0) {
            while (scan < n && lvl[scan] >= 0) scan++;
            if (scan >= n) break;
            start = scan;
        }
        int64_t h = 0, t = 0;
        queue[t++] = start; lvl[start] = 0;
        while (h < t) {
            int64_t u = queue[h++];
            for (int64_t p = cp[u]; p < cp[u + 1]; p++) {
                int64_t v = ri[p];
                if (lvl[v] < 0) { lvl[v] = lvl[u] + 1; queue[t++] = v; }
            }
        }
        start = -1;
    }
    int64_t g = 0;
    for (int64_t u = 0; u < n; u++)
        for (int64_t p = cp[u]; p < cp[u + 1]; p++) g = gcd64(g, lvl[u] + 1 - lvl[ri[p]]);
    free(cp); free(ri); free(lvl); free(queue);
    return g;
}

/* ------------------------------------------------------------------------ */
/* 5. Pack: DIAG band + warp-grained sliced ELL + local rearrangement         */
/*    (layout v0 frozen in DESIGN.md section 5)                   */
/* ------------------------------------------------------------------------ */
void oracle_packed_free(oracle_packed* p) {
    if (!p) return;
    free(p->lo); free(p->up); free(p->inv_d); free(p->row_of);
    free(p->slice_off); free(p->slice_w); free(p->val); free(p->col);
    memset(p, 0, sizeof(*p));
}

static double find_entry(const int64_t* rp, const int32_t* col, const double* val, int64_t i,
                         int64_t j) {
    for (int64_t p = rp[i]; p < rp[i + 1]; p++)
        if (col[p] == j) return val[p];
    return 0.0;
}

int oracle_pack(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                const double* diag, int32_t window, int32_t band, int32_t group,
                oracle_packed* out) {
    if (n <= 0 || !out || band < 0 || band > 2 || group < 0) return ORACLE_INVALID_ARG;
    memset(out, 0, sizeof(*out));
    /* band rule: DIA pays off when the +-1 density exceeds 8/12 = 2/3 */
    int64_t cnt = 0;
    for (int64_t i = 0; i < n; i++) {
        if (i >= 1 && find_entry(rp, col, val, i, i - 1) != 0.0) cnt++;
        if (i + 1 < n && find_entry(rp, col, val, i, i + 1) != 0.0) cnt++;
    }
    int64_t den = 2 * n - 2;
    int band_on = band == 1 ? 1 : band == 2 ? 0 : (den > 0 && 3 * cnt >= 2 * den);
    int64_t n_slots = (n + 31) / 32 * 32, n_slices = n_slots / 32;
    out->n = n; out->n_slots = n_slots; out->n_slices = n_slices;
    out->band_on = band_on; out->window = window <= 1 ? 1 : window;
    out->lo = (double*)calloc(n_slots, sizeof(double));
    out->up = (double*)calloc(n_slots, sizeof(double));
    out->inv_d = (double*)calloc(n_slots, sizeof(double));
    out->row_of = (int32_t*)malloc(sizeof(int32_t) * n_slots);
    out->slice_off = (int64_t*)malloc(sizeof(int64_t) * (n_slices + 1));
    out->slice_w = (int32_t*)malloc(sizeof(int32_t) * n_slices);
    int32_t* c = (int32_t*)malloc(sizeof(int32_t) * n);
    if (!out->lo || !out->up || !out->inv_d || !out->row_of || !out->slice_off || !out->slice_w || !c) {
        free(c); oracle_packed_free(out); return ORACLE_OOM;
    }
    /* ELL count per row: off-diagonals minus the ones the band takes */
    for (int64_t i = 0; i < n; i++) {
        int64_t k = rp[i + 1] - rp[i];
        if (band_on) {
            if (i >= 1 && find_entry(rp, col, val, i, i - 1) != 0.0) k--;
            if (i + 1 < n && find_entry(rp, col, val, i, i + 1) != 0.0) k--;
        }
        c[i] = (int32_t)k;
    }
    /* local rearrangement: inside each window the slots take rows in stable
     * order of (-c_i, i) (reading R13) */
    for (int64_t s = 0; s < n_slots; s++) out->row_of[s] = (int32_t)s;
    if (window > 1) {
        for (int64_t w0 = 0; w0 < n; w0 += window) {
            int64_t w1 = w0 + window < n ? w0 + window : n;
            for (int64_t a = w0 + 1; a < w1; a++) {    /* stable insertion sort */
                int32_t r = out->row_of[a];
                int64_t b = a;
                while (b > w0 && c[out->row_of[b - 1]] < c[r]) { out->row_of[b] = out->row_of[b - 1]; b--; }
                out->row_of[b] = r;
            }
        }
    }
    int32_t kmax = 0;
    for (int64_t i = 0; i < n; i++) if (c[i] > kmax) kmax = c[i];
    /* width of a slice = max ELL count of its rows; slices of one
     * group share the group's max (group 8 = 256-row block-sliced ELL [5]);
     * group 0 = one global width (plain ELL) */
    for (int64_t q = 0; q < n_slices; q++) {
        int32_t wq = 0;
        for (int64_t s = q * 32; s < q * 32 + 32; s++)
            if (s < n && c[out->row_of[s]] > wq) wq = c[out->row_of[s]];
        out->slice_w[q] = wq;
    }
    if (group == 0) {
        for (int64_t q = 0; q < n_slices; q++) out->slice_w[q] = kmax;
    } else if (group > 1) {
        for (int64_t g0 = 0; g0 < n_slices; g0 += group) {
            int64_t g1 = g0 + group < n_slices ? g0 + group : n_slices;
            int32_t wg = 0;
            for (int64_t q = g0; q < g1; q++) if (out->slice_w[q] > wg) wg = out->slice_w[q];
            for (int64_t q = g0; q < g1; q++) out->slice_w[q] = wg;
        }
    }
    out->slice_off[0] = 0;
    for (int64_t q = 0; q < n_slices; q++)
        out->slice_off[q + 1] = out->slice_off[q] + 32 * (int64_t)out->slice_w[q];
    int64_t n_ell = out->slice_off[n_slices];
    out->n_ell = n_ell;
    out->val = (double*)malloc(sizeof(double) * (n_ell ? n_ell : 1));
    out->col = (int32_t*)malloc(sizeof(int32_t) * (n_ell ? n_ell : 1));
    if (!out->val || !out->col) { free(c); oracle_packed_free(out); return ORACLE_OOM; }
    for (int64_t s = 0; s < n_slots; s++) {
        int64_t q = s / 32, l = s % 32;
        int64_t base = out->slice_off[q] + l;
        int32_t wq = out->slice_w[q];
        if (s >= n) { /* pad slot: zero row, in-range column */
            for (int32_t t = 0; t < wq; t++) { out->val[base + 32 * t] = 0.0; out->col[base + 32 * t] = (int32_t)(n - 1); }
            continue;
        }
        int64_t r = out->row_of[s];
        out->inv_d[s] = 1.0 / (-diag[r]);
        if (band_on) {
            out->lo[s] = r >= 1 ? find_entry(rp, col, val, r, r - 1) : 0.0;
            out->up[s] = r + 1 < n ? find_entry(rp, col, val, r, r + 1) : 0.0;
        }
        int32_t t = 0;
        for (int64_t p = rp[r]; p < rp[r + 1]; p++) {
            if (band_on && (col[p] == r - 1 || col[p] == r + 1)) continue;
            out->val[base + 32 * t] = val[p];
            out->col[base + 32 * t] = col[p];
            t++;
        }
        for (; t < wq; t++) { out->val[base + 32 * t] = 0.0; out->col[base + 32 * t] = (int32_t)r; }
    }
    free(c);
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------ */
/* 6. Jacobi                                                      */
/* ------------------------------------------------------------------------ */
static int g_threads = 1;

static void step_rows(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                      const double* diag, double omega, const double* x, double* y) {
    /* x_i^(k+1) = (1/a_ii) [ - sum_{j != i} a_ij x_j^(k) ]   (eq. 8),
     * relaxed: y_i = (1 - omega) x_i + omega * that (reading R1). */
#ifdef _OPENMP
#pragma omp parallel for schedule(static) num_threads(g_threads) if (g_threads > 1)
#endif
    for (int64_t i = 0; i < n; i++) {
        double s = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; p++) s += val[p] * x[col[p]];
        y[i] = (1.0 - omega) * x[i] + omega * (s / (-diag[i]));
    }
}

int oracle_jacobi_step(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                       const double* diag, double omega, const double* x, double* y) {
    if (n <= 0 || !x || !y) return ORACLE_INVALID_ARG;
    g_threads = 1;
    step_rows(n, rp, col, val, diag, omega, x, y);
    return ORACLE_OK;
}

#define OBLK 4096
/* fixed 4096-row blocks combined in block order: same bits serial or threaded */
enum { S_Y = 0, S_X, S_D, NSUM };
static void check_sums(int64_t n, const double* x, const double* y, const double* diag,
                       double* sums, double* maxdd, double* maxx) {
    int64_t nb = (n + OBLK - 1) / OBLK;
    double* part = (double*)malloc(sizeof(double) * nb * (NSUM + 2));
#ifdef _OPENMP
#pragma omp parallel for schedule(static) num_threads(g_threads) if (g_threads > 1)
#endif
    for (int64_t b = 0; b < nb; b++) {
        double sy = 0, sx = 0, sd = 0, md = 0, mx = 0;
        int64_t e = (b + 1) * OBLK < n ? (b + 1) * OBLK : n;
        for (int64_t i = b * OBLK; i < e; i++) {
            double df = fabs(y[i] - x[i]);
            sy += y[i]; sx += x[i]; sd += df;
            double rd = fabs(diag[i]) * df;
            if (rd > md) md = rd;
            if (x[i] > mx) mx = x[i];
        }
        double* q = part + b * (NSUM + 2);
        q[0] = sy; q[1] = sx; q[2] = sd; q[3] = md; q[4] = mx;
    }
    sums[0] = sums[1] = sums[2] = 0; *maxdd = 0; *maxx = 0;
    for (int64_t b = 0; b < nb; b++) {
        double* q = part + b * (NSUM + 2);
        sums[0] += q[0]; sums[1] += q[1]; sums[2] += q[2];
        if (q[3] > *maxdd) *maxdd = q[3];
        if (q[4] > *maxx) *maxx = q[4];
    }
    free(part);
}

static double block_sum(int64_t n, const double* x) {
    double t = 0.0;
    for (int64_t b = 0; b * OBLK < n; b++) {
        double s = 0.0;
        int64_t e = (b + 1) * OBLK < n ? (b + 1) * OBLK : n;
        for (int64_t i = b * OBLK; i < e; i++) s += x[i];
        t += s;
    }
    return t;
}

int oracle_jacobi_solve(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                        const double* diag, const double* p0, double omega, double tol,
                        int64_t C, int64_t max_iter, int stop_mode, double stag_tol,
                        int nthreads, double* p_out, int64_t* iters_out, double* delta_out,
                        double* resid_out) {
    if (n <= 0 || !p_out || C <= 0 || max_iter < 0 || !(omega > 0.0 && omega <= 1.0) ||
        stop_mode < 0 || stop_mode > 1 || !(stag_tol >= 0.0))
        return ORACLE_INVALID_ARG;
    g_threads = nthreads < 1 ? 1 : nthreads;
    double* x = (double*)malloc(sizeof(double) * n);
    double* y = (double*)malloc(sizeof(double) * n);
    if (!x || !y) { free(x); free(y); return ORACLE_OOM; }
    /* ||A||_inf: max row sum of |a_ij| including the diagonal.  Each
     * row sum is the same serial sum in every thread count; the max of them
     * does not depend on the order, so the threads only change the time. */
    double normA = 0.0;
#pragma omp parallel for schedule(static) reduction(max : normA) num_threads(g_threads) if (g_threads > 1)
    for (int64_t i = 0; i < n; i++) {
        double s = fabs(diag[i]);
        for (int64_t p = rp[i]; p < rp[i + 1]; p++) s += fabs(val[p]);
        if (s > normA) normA = s;
    }
    if (p0) {
        double s0 = block_sum(n, p0);
        if (!(s0 > 0.0) || isinf(s0)) { free(x); free(y); return ORACLE_INVALID_ARG; }
        for (int64_t i = 0; i < n; i++) {
            if (!(p0[i] >= 0.0)) { free(x); free(y); return ORACLE_INVALID_ARG; }
            x[i] = p0[i] / s0;
        }
    } else {
        for (int64_t i = 0; i < n; i++) x[i] = 1.0 / (double)n;   /* reading R6 */
    }
    int status = ORACLE_NOT_CONVERGED;
    double delta = -1.0, delta_prev = -1.0, resid = -1.0;
    int64_t k = 0;
    while (k < max_iter) {
        step_rows(n, rp, col, val, diag, omega, x, y);
        k++;
        if (k % C == 0 || k == max_iter) {
            double sums[3], maxdd, maxx;
            check_sums(n, x, y, diag, sums, &maxdd, &maxx);
            double s = sums[0];
            delta = sums[2] / sums[1];
            resid = maxdd / (omega * normA * maxx);
            if (!(s > 0.0) || isinf(s) || isnan(delta)) { status = ORACLE_NUMERIC; break; }
            for (int64_t i = 0; i < n; i++) x[i] = y[i] / s;  /* periodic L1 normalisation */
            if (k % C != 0) { status = ORACLE_NOT_CONVERGED; break; }
            double crit = stop_mode == 0 ? delta : resid;
            if (crit <= tol) { status = ORACLE_OK; break; }
            if (stag_tol > 0.0 && k >= 2 * C && fabs(delta - delta_prev) <= stag_tol * delta_prev) {
                status = ORACLE_STAGNATED; break;
            }
            delta_prev = delta;
            if (k == max_iter) { status = ORACLE_NOT_CONVERGED; break; }
        } else {
            double* t = x; x = y; y = t;   /* deferred normalisation (reading R5) */
        }
    }
    if (max_iter == 0) {
        double s = block_sum(n, x);
        for (int64_t i = 0; i < n; i++) x[i] = x[i] / s;
    }
    memcpy(p_out, x, sizeof(double) * n);
    if (iters_out) *iters_out = k;
    if (delta_out) *delta_out = delta;
    if (resid_out) *resid_out = resid;
    free(x); free(y);
    return status;
}

/* ------------------------------------------------------------------------ */
/* 7. Transient landscape by uniformization (P:L277 future work; R22)         */
/* ------------------------------------------------------------------------ */
int oracle_transient(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                     const double* diag, const double* p0, double t, double eps, double* p_out,
                     int64_t* terms_out, double* lambda_out) {
    if (n <= 0 || !p_out || !(t >= 0.0) || !(eps > 0.0 && eps < 1.0)) return ORACLE_INVALID_ARG;
    double lam = 0.0;
    for (int64_t i = 0; i < n; i++) if (-diag[i] > lam) lam = -diag[i];
    double* x = (double*)malloc(sizeof(double) * n);
    double* y = (double*)malloc(sizeof(double) * n);
    if (!x || !y) { free(x); free(y); return ORACLE_OOM; }
    for (int64_t i = 0; i < n; i++) { x[i] = p0 ? p0[i] : (i == 0 ? 1.0 : 0.0); p_out[i] = 0.0; }
    /* Poisson(k; mu = Lambda t) weights (R22): w_k ~ exp(k ln mu - lgamma(k+1))
     * for k <= Kmax = ceil(mu + 10 sqrt(mu) + 40), normalised to sum 1;
     * K = the smallest k with sum_{j>k} w_j <= eps */
    const double mu = lam * t;
    const int64_t kmax = (int64_t)ceil(mu + 10.0 * sqrt(mu) + 40.0);
    double* w = (double*)malloc(sizeof(double) * (kmax + 1));
    if (!w) { free(x); free(y); return ORACLE_OOM; }
    double lmax = -INFINITY;
    for (int64_t k = 0; k <= kmax; k++) {
        w[k] = mu > 0.0 ? (double)k * log(mu) - lgamma((double)k + 1.0) : (k == 0 ? 0.0 : -INFINITY);
        if (w[k] > lmax) lmax = w[k];
    }
    double W = 0.0;
    for (int64_t k = 0; k <= kmax; k++) { w[k] = exp(w[k] - lmax); W += w[k]; }
    for (int64_t k = 0; k <= kmax; k++) w[k] /= W;
    int64_t K = kmax;
    double tail = 0.0;
    while (K > 0 && tail + w[K] <= eps) { tail += w[K]; K--; }
    int64_t k = 0;
    for (;; k++) {
        for (int64_t i = 0; i < n; i++) p_out[i] += w[k] * x[i];
        if (k == K) break;
        /* x <- P x = x + A x / Lambda */
        for (int64_t i = 0; i < n; i++) {
            double s = 0.0;
            for (int64_t p = rp[i]; p < rp[i + 1]; p++) s += val[p] * x[col[p]];
            y[i] = x[i] + (s + diag[i] * x[i]) / lam;
        }
        double* tmp = x; x = y; y = tmp;
    }
    free(w);
    if (terms_out) *terms_out = k + 1;
    if (lambda_out) *lambda_out = lam;
    free(x); free(y);
    return ORACLE_OK;
}

/* ------------------------------------------------------------------------ */
/* 8. Dense LU null-space solve for tiny state spaces (north star)            */
/* ------------------------------------------------------------------------ */
int oracle_lu_steady(int64_t n, const int64_t* rp, const int32_t* col, const double* val,
                     const double* diag, double* p_out) {
    if (n <= 0 || n > 4096 || !p_out) return ORACLE_INVALID_ARG;
    double* A = (double*)calloc((size_t)(n * n), sizeof(double));
    double* b = (double*)calloc((size_t)n, sizeof(double));
    if (!A || !b) { free(A); free(b); return ORACLE_OOM; }
    for (int64_t i = 0; i < n; i++) {
        A[i * n + i] = diag[i];
        for (int64_t p = rp[i]; p < rp[i + 1]; p++) A[i * n + col[p]] = val[p];
    }
    /* AP = 0 is singular: replace the last equation by sum p = 1 */
    for (int64_t j = 0; j < n; j++) A[(n - 1) * n + j] = 1.0;
    b[n - 1] = 1.0;
    for (int64_t k = 0; k < n; k++) {      /* Gaussian elimination, partial pivoting */
        int64_t piv = k;
        for (int64_t i = k + 1; i < n; i++)
            if (fabs(A[i * n + k]) > fabs(A[piv * n + k])) piv = i;
        if (A[piv * n + k] == 0.0) { free(A); free(b); return ORACLE_NUMERIC; }
        if (piv != k) {
            for (int64_t j = 0; j < n; j++) { double t = A[k * n + j]; A[k * n + j] = A[piv * n + j]; A[piv * n + j] = t; }
            double t = b[k]; b[k] = b[piv]; b[piv] = t;
        }
        for (int64_t i = k + 1; i < n; i++) {
            double f = A[i * n + k] / A[k * n + k];
            if (f == 0.0) continue;
            for (int64_t j = k; j < n; j++) A[i * n + j] -= f * A[k * n + j];
            b[i] -= f * b[k];
        }
    }
    for (int64_t i = n - 1; i >= 0; i--) {
        double s = b[i];
        for (int64_t j = i + 1; j < n; j++) s -= A[i * n + j] * p_out[j];
        p_out[i] = s / A[i * n + i];
    }
    free(A); free(b);
    return ORACLE_OK;
}
