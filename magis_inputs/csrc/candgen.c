/*
 * candgen.c -- seeded candidate-schedule generator (INPUT GENERATION ONLY).
 *
 * Produces K candidate schedules for one graph from (seed, global candidate
 * id), so candidates do not depend on how they are sharded over ranks.  It
 * stands in for MAGIS's rule application + re-ordering (§5.2 P:1352-1357,
 * Alg. 2), and holds no evaluation arithmetic.  The CUDA path
 * has its own implementation of exactly this recipe (bit-exact, checked in
 * tests); the two share no code.
 *
 * Recipe (candidate construction):
 *   rnd(stream, i) = mix(mix(mix(seed + G*(stream+1)) ^ k) ^ i), mix = SplitMix64
 *   family f = rnd(FAM,0) % 100 : < pct_random  -> F1 random topo order
 *                                  < +pct_local  -> F2 local move (window)
 *                                  else          -> F3 = F1 + one transposition
 *   dec[r]:  x = rnd(DEC,r) % 10000; x < p_remat (and t_r has inputs) -> 1;
 *            x < p_remat + p_swap -> 2; else 0
 *   F1: Kahn over the base graph, ready node with the smallest
 *       (key(v) = rnd(KEY,v) >> 48, v) first (a 16-bit priority, ties by id:
 *       the device generator compares (key, id) as one u32).
 *   F2: natural order; window length w = 2 + rnd(WIN,0) % (wmax-1) (<= n),
 *       start b = rnd(WIN,1) % (n-w+1); the window re-ordered by the same
 *       keyed Kahn restricted to its induced sub-DAG.
 *   optional nodes, placed into gaps of the base order (gap g = before base[g]):
 *       store_r: g = pos(t_r)+1, prio 0      ("Store as early as possible")
 *       load_r : g = max(q - j, pos(t_r)+1), prio 1
 *       clone_r: g = max(q - j, max_{x in pre(t_r)} pos(x) + 1), prio 1
 *       q = min over U_r of pos(b), j = rnd(SLK,r) % (slack+1)
 *     sorted by (g, prio, r); inactive optional ids follow in ascending order.
 *   F3: swap perm[rnd(TRN,0) % NT] and perm[rnd(TRN,1) % NT] (may be invalid).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define S_FAM 1u
#define S_DEC 2u
#define S_KEY 3u
#define S_WIN 4u
#define S_SLK 5u
#define S_TRN 6u
#define S_VAR 7u

static inline uint64_t mix64(uint64_t x)
{
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

static inline uint64_t rnd(uint64_t seed, uint64_t k, uint32_t stream, uint64_t i)
{
    uint64_t h = mix64(seed + 0x9E3779B97F4A7C15ull * (uint64_t)(stream + 1u));
    h = mix64(h ^ k);
    return mix64(h ^ i);
}

typedef struct {
    int32_t n, R, NT;
    const int64_t *succ_ptr;   /* [n+1] successors of the base graph (deduplicated) */
    const int32_t *succ_idx;
    const int64_t *pred_ptr;   /* [n+1] */
    const int32_t *pred_idx;
    const int32_t *elig;       /* [R] */
    const int64_t *U_ptr;      /* [R+1] */
    const int32_t *U_idx;
    uint64_t seed;
    int32_t pct_random, pct_local;
    int32_t p_remat, p_swap;   /* per 10000 */
    int32_t wmax, slack;
    /* F-Trans variant regions (NEXT-4): dec[R + i] = rnd(VAR, i) % nvar[i];
     * only the ops of the chosen variants (and the ungated ones) are ordered;
     * local moves (F2) become F1; absent ops follow the optional nodes. */
    int32_t F;
    const int32_t *nvar;       /* [F] */
    const int32_t *nreg;       /* [n] region or -1 */
    const uint8_t *nvn;        /* [n] variant */
} gen_cfg;

typedef struct {
    int32_t *indeg;
    uint64_t *heap;
    int32_t *base;
    int32_t *posb;
    int64_t *opt;    /* sort keys of active optional nodes */
    uint8_t *inwin;
    uint8_t *act;    /* present original ops (regions), or NULL */
} gen_ws;

static void heap_push(uint64_t *h, int32_t *n, uint64_t x)
{
    int32_t i = (*n)++;
    while (i > 0) {
        int32_t p = (i - 1) >> 1;
        if (h[p] <= x) break;
        h[i] = h[p]; i = p;
    }
    h[i] = x;
}

static uint64_t heap_pop(uint64_t *h, int32_t *n)
{
    uint64_t top = h[0], x = h[--(*n)];
    int32_t i = 0;
    for (;;) {
        int32_t c = 2 * i + 1;
        if (c >= *n) break;
        if (c + 1 < *n && h[c + 1] < h[c]) c++;
        if (h[c] >= x) break;
        h[i] = h[c]; i = c;
    }
    if (*n > 0) h[i] = x;
    return top;
}

static int cmp_i64(const void *a, const void *b)
{
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

/* keyed Kahn over nodes [lo, hi) of the natural order, restricted to edges
 * inside the range; writes the order into out[0 .. hi-lo). */
static void keyed_kahn(const gen_cfg *c, gen_ws *w, uint64_t k, int32_t lo, int32_t hi, int32_t *out)
{
    int32_t v, nh = 0, m = 0;
    int64_t e;
    for (v = lo; v < hi; v++) {
        int32_t d = 0;
        for (e = c->pred_ptr[v]; e < c->pred_ptr[v + 1]; e++)
            if (c->pred_idx[e] >= lo && (!w->act || w->act[c->pred_idx[e]])) d++;   /* preds < lo are placed */
        w->indeg[v] = d;
    }
    for (v = lo; v < hi; v++)
        if (w->indeg[v] == 0 && (!w->act || w->act[v]))
            heap_push(w->heap, &nh, ((rnd(c->seed, k, S_KEY, (uint64_t)v) >> 48) << 32) | (uint32_t)v);
    while (nh > 0) {
        uint64_t x = heap_pop(w->heap, &nh);
        int32_t u = (int32_t)(x & 0xffffffffu);
        out[m++] = u;
        for (e = c->succ_ptr[u]; e < c->succ_ptr[u + 1]; e++) {
            int32_t s = c->succ_idx[e];
            if (s >= hi || (w->act && !w->act[s])) continue;
            if (--w->indeg[s] == 0)
                heap_push(w->heap, &nh, ((rnd(c->seed, k, S_KEY, (uint64_t)s) >> 48) << 32) | (uint32_t)s);
        }
    }
}

static void gen_one(const gen_cfg *c, gen_ws *w, uint64_t k, int32_t *perm, uint8_t *dec)
{
    const int32_t n = c->n, R = c->R, NT = c->NT;
    uint32_t fam = (uint32_t)(rnd(c->seed, k, S_FAM, 0) % 100u);
    int32_t r, i, nopt = 0, m = 0, oi;
    int64_t e;

    for (r = 0; r < R; r++) {
        uint32_t x = (uint32_t)(rnd(c->seed, k, S_DEC, (uint64_t)r) % 10000u);
        int32_t t = c->elig[r];
        uint8_t d = 0;
        if ((int32_t)x < c->p_remat && c->pred_ptr[t + 1] > c->pred_ptr[t]) d = 1;
        else if ((int32_t)x < c->p_remat + c->p_swap) d = 2;
        dec[r] = d;
    }

    int32_t nb = n;                         /* ops in the base order */
    if (c->F > 0) {
        for (i = 0; i < c->F; i++)
            dec[R + i] = (uint8_t)(rnd(c->seed, k, S_VAR, (uint64_t)i) % (uint64_t)c->nvar[i]);
        nb = 0;
        for (i = 0; i < n; i++) {
            w->act[i] = (uint8_t)(c->nreg[i] < 0 || dec[R + c->nreg[i]] == c->nvn[i]);
            nb += w->act[i];
        }
    }
    if (c->F > 0 || (int32_t)fam < c->pct_random || (int32_t)fam >= c->pct_random + c->pct_local) {
        keyed_kahn(c, w, k, 0, n, w->base);
    } else {
        int32_t len = 2 + (int32_t)(rnd(c->seed, k, S_WIN, 0) % (uint64_t)(c->wmax - 1));
        int32_t b;
        if (len > n) len = n;
        b = (int32_t)(rnd(c->seed, k, S_WIN, 1) % (uint64_t)(n - len + 1));
        for (i = 0; i < n; i++) w->base[i] = i;
        keyed_kahn(c, w, k, b, b + len, w->base + b);
    }
    for (i = 0; i < nb; i++) w->posb[w->base[i]] = i;

    for (r = 0; r < R; r++) {
        int32_t t = c->elig[r], q = INT32_MAX, j, g;
        if (dec[r] == 0) continue;
        for (e = c->U_ptr[r]; e < c->U_ptr[r + 1]; e++)
            if (w->posb[c->U_idx[e]] < q) q = w->posb[c->U_idx[e]];
        j = (int32_t)(rnd(c->seed, k, S_SLK, (uint64_t)r) % (uint64_t)(c->slack + 1));
        if (dec[r] == 2) {
            int32_t gs = w->posb[t] + 1;
            g = q - j; if (g < gs) g = gs;
            w->opt[nopt++] = ((int64_t)gs << 32) | (0 << 30) | r;            /* store */
            w->opt[nopt++] = ((int64_t)g << 32) | (1 << 30) | r;             /* load  */
        } else {
            int32_t lo = 0;
            for (e = c->pred_ptr[t]; e < c->pred_ptr[t + 1]; e++)
                if (w->posb[c->pred_idx[e]] + 1 > lo) lo = w->posb[c->pred_idx[e]] + 1;
            g = q - j; if (g < lo) g = lo;
            w->opt[nopt++] = ((int64_t)g << 32) | (1 << 30) | r;             /* clone */
        }
    }
    qsort(w->opt, (size_t)nopt, sizeof(int64_t), cmp_i64);
    oi = 0;
    for (i = 0; i <= nb; i++) {
        while (oi < nopt && (int32_t)(w->opt[oi] >> 32) == i) {
            int32_t rr = (int32_t)(w->opt[oi] & 0x3fffffff);
            int32_t pr = (int32_t)((w->opt[oi] >> 30) & 3);
            int32_t id;
            if (pr == 0) id = n + 3 * rr + 1;
            else id = (dec[rr] == 2) ? n + 3 * rr + 2 : n + 3 * rr;
            perm[m++] = id;
            oi++;
        }
        if (i < nb) perm[m++] = w->base[i];
    }
    if (c->F > 0)                           /* ops of the variants not chosen: no-ops, ascending */
        for (i = 0; i < n; i++)
            if (!w->act[i]) perm[m++] = i;
    for (r = 0; r < R; r++) {
        if (dec[r] != 1) perm[m++] = n + 3 * r;
        if (dec[r] != 2) { perm[m++] = n + 3 * r + 1; perm[m++] = n + 3 * r + 2; }
    }
    /* inactive ids must be ascending: clone_r < store_r < load_r < clone_{r+1} already */
    if ((int32_t)fam >= c->pct_random + c->pct_local) {
        int32_t a = (int32_t)(rnd(c->seed, k, S_TRN, 0) % (uint64_t)NT);
        int32_t b2 = (int32_t)(rnd(c->seed, k, S_TRN, 1) % (uint64_t)NT);
        int32_t tmp = perm[a]; perm[a] = perm[b2]; perm[b2] = tmp;
    }
    (void)m;
}

typedef struct {
    const gen_cfg *c;
    uint64_t id0;
    int64_t k0, k1;
    int32_t *perms;
    uint8_t *decs;
} job;

static void *worker(void *arg)
{
    job *j = (job *)arg;
    const gen_cfg *c = j->c;
    gen_ws w;
    int64_t k;
    w.indeg = (int32_t *)malloc(sizeof(int32_t) * (c->n + 1));
    w.heap = (uint64_t *)malloc(sizeof(uint64_t) * (c->n + 1));
    w.base = (int32_t *)malloc(sizeof(int32_t) * (c->n + 1));
    w.posb = (int32_t *)malloc(sizeof(int32_t) * (c->n + 1));
    w.opt = (int64_t *)malloc(sizeof(int64_t) * (2 * c->R + 1));
    w.inwin = NULL;
    w.act = c->F > 0 ? (uint8_t *)malloc((size_t)c->n + 1) : NULL;
    for (k = j->k0; k < j->k1; k++)
        gen_one(c, &w, j->id0 + (uint64_t)k, j->perms + k * (int64_t)c->NT,
                j->decs + k * (int64_t)((c->R + c->F) ? c->R + c->F : 1));
    free(w.indeg); free(w.heap); free(w.base); free(w.posb); free(w.opt); free(w.act);
    return NULL;
}

void candgen_regions(int32_t n, int32_t R, const int64_t *succ_ptr, const int32_t *succ_idx,
                     const int64_t *pred_ptr, const int32_t *pred_idx, const int32_t *elig,
                     const int64_t *U_ptr, const int32_t *U_idx, uint64_t seed,
                     int32_t pct_random, int32_t pct_local, int32_t p_remat, int32_t p_swap,
                     int32_t wmax, int32_t slack, uint64_t id0, int64_t K,
                     int32_t *perms, uint8_t *decs, int32_t nthreads,
                     int32_t F, const int32_t *nvar, const int32_t *nreg, const uint8_t *nvn);

/* Generate candidates with global ids id0 .. id0+K-1 into perms (K x NT) and
 * decs (K x max(R,1)).  nthreads >= 1. */
void candgen(int32_t n, int32_t R, const int64_t *succ_ptr, const int32_t *succ_idx,
             const int64_t *pred_ptr, const int32_t *pred_idx, const int32_t *elig,
             const int64_t *U_ptr, const int32_t *U_idx, uint64_t seed,
             int32_t pct_random, int32_t pct_local, int32_t p_remat, int32_t p_swap,
             int32_t wmax, int32_t slack, uint64_t id0, int64_t K,
             int32_t *perms, uint8_t *decs, int32_t nthreads)
{
    candgen_regions(n, R, succ_ptr, succ_idx, pred_ptr, pred_idx, elig, U_ptr, U_idx, seed, pct_random,
                    pct_local, p_remat, p_swap, wmax, slack, id0, K, perms, decs, nthreads, 0, NULL, NULL, NULL);
}

/* As candgen, over a graph with F-Trans variant regions: decs is K x (R + F). */
void candgen_regions(int32_t n, int32_t R, const int64_t *succ_ptr, const int32_t *succ_idx,
                     const int64_t *pred_ptr, const int32_t *pred_idx, const int32_t *elig,
                     const int64_t *U_ptr, const int32_t *U_idx, uint64_t seed,
                     int32_t pct_random, int32_t pct_local, int32_t p_remat, int32_t p_swap,
                     int32_t wmax, int32_t slack, uint64_t id0, int64_t K,
                     int32_t *perms, uint8_t *decs, int32_t nthreads,
                     int32_t F, const int32_t *nvar, const int32_t *nreg, const uint8_t *nvn)
{
    gen_cfg c;
    pthread_t th[256];
    job jobs[256];
    int32_t t;
    c.n = n; c.R = R; c.NT = n + 3 * R;
    c.succ_ptr = succ_ptr; c.succ_idx = succ_idx; c.pred_ptr = pred_ptr; c.pred_idx = pred_idx;
    c.elig = elig; c.U_ptr = U_ptr; c.U_idx = U_idx; c.seed = seed;
    c.pct_random = pct_random; c.pct_local = pct_local; c.p_remat = p_remat; c.p_swap = p_swap;
    c.wmax = wmax < 2 ? 2 : wmax; c.slack = slack < 0 ? 0 : slack;
    c.F = F; c.nvar = nvar; c.nreg = nreg; c.nvn = nvn;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    if (K < nthreads) nthreads = K > 0 ? (int32_t)K : 1;
    for (t = 0; t < nthreads; t++) {
        jobs[t].c = &c; jobs[t].id0 = id0;
        jobs[t].k0 = K * t / nthreads; jobs[t].k1 = K * (t + 1) / nthreads;
        jobs[t].perms = perms; jobs[t].decs = decs;
    }
    if (nthreads == 1) { worker(&jobs[0]); return; }
    for (t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, worker, &jobs[t]);
    for (t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
}

/*
 * Local-move (window) candidates over a base schedule (INPUT GENERATION):
 * candidate k re-orders the base steps [b, b+w) and keeps the base
 * decisions.  w = 2 + rnd(WIN,0) % (wmax-1) (<= NT), b = rnd(WIN,1) % (NT-w+1);
 * the window's nodes are re-ordered by the keyed Kahn (key = rnd(KEY,node))
 * over the window's dependencies under the base decisions (Fig. 8 rules: a
 * late user reads t_r, its clone or its Load by dec[r]; the clone reads
 * pre(t_r); t_r -> Store -> Load).  With probability pct_bad/100 the two
 * ends of the window are swapped afterwards (may be invalid).
 * Outputs: wstart[K], wlen[K], wperm[K x wmax] (unused entries -1).
 */
typedef struct {
    int32_t n, R, NT;
    const int64_t *pred_ptr;  const int32_t *pred_idx;   /* base graph */
    const int32_t *elig;      const int64_t *U_ptr; const int32_t *U_idx;
    const int64_t *lu_ptr;    const int32_t *lu_idx;     /* per original node: r with node in U_r */
    const int32_t *bperm, *bpos; const uint8_t *bdec;
    uint64_t seed; int32_t wmax, pct_bad;
} win_cfg;

static int in_win(const win_cfg *c, int32_t v, int32_t b, int32_t w)
{
    int32_t p = c->bpos[v];
    return p >= b && p < b + w;
}

static void win_one(const win_cfg *c, uint64_t k, int32_t *ws, int32_t *wl, int32_t *wp)
{
    const int32_t n = c->n, NT = c->NT;
    int32_t w = 2 + (int32_t)(rnd(c->seed, k, S_WIN, 0) % (uint64_t)(c->wmax - 1));
    int32_t b, i, j, m = 0;
    uint64_t pre[64], done = 0;
    int64_t e, f;
    if (w > NT) w = NT;
    b = (int32_t)(rnd(c->seed, k, S_WIN, 1) % (uint64_t)(NT - w + 1));
    for (i = 0; i < w; i++) {
        int32_t v = c->bperm[b + i];
        uint64_t msk = 0;
        if (v < n) {
            for (e = c->pred_ptr[v]; e < c->pred_ptr[v + 1]; e++) {
                int32_t u = c->pred_idx[e], moved = 0;
                for (f = c->lu_ptr[v]; f < c->lu_ptr[v + 1]; f++) {
                    int32_t r = c->lu_idx[f];
                    if (c->elig[r] == u && c->bdec[r] != 0) moved = 1;
                }
                if (!moved && in_win(c, u, b, w)) msk |= 1ull << (c->bpos[u] - b);
            }
            for (f = c->lu_ptr[v]; f < c->lu_ptr[v + 1]; f++) {
                int32_t r = c->lu_idx[f], src = -1;
                if (c->bdec[r] == 1) src = n + 3 * r;
                if (c->bdec[r] == 2) src = n + 3 * r + 2;
                if (src >= 0 && in_win(c, src, b, w)) msk |= 1ull << (c->bpos[src] - b);
            }
        } else {
            int32_t r = (v - n) / 3, kd = (v - n) % 3, t = c->elig[r];
            if (kd == 0 && c->bdec[r] == 1) {
                for (e = c->pred_ptr[t]; e < c->pred_ptr[t + 1]; e++)
                    if (in_win(c, c->pred_idx[e], b, w)) msk |= 1ull << (c->bpos[c->pred_idx[e]] - b);
            } else if (kd == 1 && c->bdec[r] == 2) {
                if (in_win(c, t, b, w)) msk |= 1ull << (c->bpos[t] - b);
            } else if (kd == 2 && c->bdec[r] == 2) {
                if (in_win(c, n + 3 * r + 1, b, w)) msk |= 1ull << (c->bpos[n + 3 * r + 1] - b);
            }
        }
        pre[i] = msk;
    }
    /* keyed Kahn over the window: repeatedly take the ready slot with the smallest key */
    for (m = 0; m < w; m++) {
        int32_t best = -1;
        uint64_t bk = 0;
        for (i = 0; i < w; i++) {
            uint64_t key;
            if ((done >> i) & 1ull) continue;
            if ((pre[i] & ~done) != 0) continue;
            key = ((rnd(c->seed, k, S_KEY, (uint64_t)c->bperm[b + i]) >> 32) << 32) | (uint32_t)c->bperm[b + i];
            if (best < 0 || key < bk) { best = i; bk = key; }
        }
        done |= 1ull << best;
        wp[m] = c->bperm[b + best];
    }
    if ((int32_t)(rnd(c->seed, k, S_TRN, 0) % 100u) < c->pct_bad) {
        int32_t t = wp[0]; wp[0] = wp[w - 1]; wp[w - 1] = t;
    }
    for (j = w; j < c->wmax; j++) wp[j] = -1;
    *ws = b;
    *wl = w;
}

void wingen(int32_t n, int32_t R, const int64_t *pred_ptr, const int32_t *pred_idx, const int32_t *elig,
            const int64_t *U_ptr, const int32_t *U_idx, const int64_t *lu_ptr, const int32_t *lu_idx,
            const int32_t *bperm, const int32_t *bpos, const uint8_t *bdec, uint64_t seed, int32_t wmax,
            int32_t pct_bad, uint64_t id0, int64_t K, int32_t *wstart, int32_t *wlen, int32_t *wperm)
{
    win_cfg c;
    int64_t k;
    c.n = n; c.R = R; c.NT = n + 3 * R;
    c.pred_ptr = pred_ptr; c.pred_idx = pred_idx; c.elig = elig; c.U_ptr = U_ptr; c.U_idx = U_idx;
    c.lu_ptr = lu_ptr; c.lu_idx = lu_idx; c.bperm = bperm; c.bpos = bpos; c.bdec = bdec;
    c.seed = seed; c.wmax = wmax < 2 ? 2 : (wmax > 64 ? 64 : wmax); c.pct_bad = pct_bad;
    for (k = 0; k < K; k++)
        win_one(&c, id0 + (uint64_t)k, wstart + k, wlen + k, wperm + k * (int64_t)c.wmax);
}
