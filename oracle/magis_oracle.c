/*
 * magis_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded CPU event simulator of the MAGIS schedule
 * semantics (Chen et al., ASPLOS '24).  It is the correctness oracle for the
 * B200 evaluation path and shares NO code, header, table or helper with it.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  The product path never does.
 *
 * Citations are to /root/reference/PAPER.md lines ("P:a-b") and to the
 * readings listed in DESIGN.md ("reading Pn", numbering from SURVEY.md §8c).
 *
 * What it computes, per candidate (perm over the super-graph, dec per
 * eligible tensor), in the paper's order:
 *   1. permutation / decision check                       (reading P12)
 *   2. active set and transformed edge list (Fig. 8 rules) (reading P5, P6)
 *   3. topological validity over every transformed edge
 *   4. compaction to the active order                       (reading: inactive nodes are no-ops)
 *   5. lifetimes S_j < i <= F_j, F = last reader            (reading P1, P2)
 *   6. event simulation, M_i, M_peak = max_i M_i, first argmax
 *   (+) memory hot-spots and F-Trans heat / score over the dominator tree
 *       (Eq. 3-4; reading H1)       -- orc_hotspots
 *   7. latency: three in-order queues (compute, D2H, H2D)   (reading P7, P8, P9)
 *
 * Super-graph ids: original nodes 0..n-1; for eligible tensor r:
 *   clone_r = n+3r, store_r = n+3r+1, load_r = n+3r+2.
 *
 * Everything is written for clarity, not speed: explicit edge lists, explicit
 * free lists, no scans, no CSR shared with anything.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

typedef struct {
    int32_t n;          /* original nodes */
    int32_t R;          /* eligible tensors */
    int32_t NT;         /* n + 3R */
    int64_t *size;      /* [n] */
    double  *cost;      /* [n] */
    uint8_t *is_output; /* [n] */
    int64_t ne;         /* deduplicated edge count (E is a set; reading P17) */
    int32_t *src, *dst;
    int32_t *elig;      /* [R] t_r */
    int64_t *U_ptr;     /* [R+1] */
    int32_t *U_idx;     /* late users U_r (reading P6) */
    int32_t *r_of;      /* [n] eligible index of a node or -1 */
    uint8_t *has_input; /* [n] node has at least one predecessor */
    double   swap_Bps;  /* swap link bytes/s (reading P7) */
    double   swap_lat;  /* per-transfer latency seconds (reading P7) */
    /* F-Trans variant regions (NEXT-4, reading F1): region i offers
     * nvar[i] variants of one sub-graph; an original node with nreg[v] >= 0
     * exists only in variant nvn[v] of region nreg[v]; the candidate picks
     * the variant in dec[R + i]. */
    int32_t  F;
    int32_t *nvar;      /* [F] */
    int32_t *nreg;      /* [n] region or -1 */
    uint8_t *nvn;       /* [n] variant */
} orc_graph;

static int cmp_pair(const void *a, const void *b)
{
    const int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

void orc_graph_free(orc_graph *g)
{
    if (!g) return;
    free(g->size); free(g->cost); free(g->is_output);
    free(g->src); free(g->dst); free(g->elig); free(g->U_ptr); free(g->U_idx);
    free(g->r_of); free(g->has_input);
    free(g->nvar); free(g->nreg); free(g->nvn);
    free(g);
}

/* Returns NULL on an obviously malformed graph (ids out of range). The oracle
 * does not re-implement the loader's validation; tests feed it valid graphs. */
orc_graph *orc_graph_new(int32_t n, const int64_t *size, const double *cost,
                         const uint8_t *is_output, int64_t n_edges,
                         const int32_t *src, const int32_t *dst, int32_t R,
                         const int32_t *elig, const int64_t *U_ptr,
                         const int32_t *U_idx, double swap_Bps, double swap_lat)
{
    orc_graph *g = (orc_graph *)calloc(1, sizeof(orc_graph));
    int64_t i;
    int64_t *pairs;
    if (!g) return NULL;
    g->n = n; g->R = R; g->NT = n + 3 * R;
    g->swap_Bps = swap_Bps; g->swap_lat = swap_lat;
    g->size = (int64_t *)malloc(sizeof(int64_t) * (n ? n : 1));
    g->cost = (double *)malloc(sizeof(double) * (n ? n : 1));
    g->is_output = (uint8_t *)malloc(n ? n : 1);
    memcpy(g->size, size, sizeof(int64_t) * n);
    memcpy(g->cost, cost, sizeof(double) * n);
    memcpy(g->is_output, is_output, n);
    /* E is a set: sort the (src,dst) pairs and drop repeats. */
    pairs = (int64_t *)malloc(sizeof(int64_t) * (n_edges ? n_edges : 1));
    for (i = 0; i < n_edges; i++) {
        if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) {
            free(pairs); orc_graph_free(g); return NULL;
        }
        pairs[i] = ((int64_t)src[i] << 32) | (uint32_t)dst[i];
    }
    qsort(pairs, (size_t)n_edges, sizeof(int64_t), cmp_pair);
    g->src = (int32_t *)malloc(sizeof(int32_t) * (n_edges ? n_edges : 1));
    g->dst = (int32_t *)malloc(sizeof(int32_t) * (n_edges ? n_edges : 1));
    g->ne = 0;
    for (i = 0; i < n_edges; i++) {
        if (i > 0 && pairs[i] == pairs[i - 1]) continue;
        g->src[g->ne] = (int32_t)(pairs[i] >> 32);
        g->dst[g->ne] = (int32_t)(pairs[i] & 0xffffffff);
        g->ne++;
    }
    free(pairs);
    g->has_input = (uint8_t *)calloc(n ? n : 1, 1);
    for (i = 0; i < g->ne; i++) g->has_input[g->dst[i]] = 1;
    g->elig = (int32_t *)malloc(sizeof(int32_t) * (R ? R : 1));
    g->U_ptr = (int64_t *)malloc(sizeof(int64_t) * (R + 1));
    memcpy(g->elig, elig, sizeof(int32_t) * R);
    memcpy(g->U_ptr, U_ptr, sizeof(int64_t) * (R + 1));
    g->U_idx = (int32_t *)malloc(sizeof(int32_t) * (U_ptr[R] ? U_ptr[R] : 1));
    memcpy(g->U_idx, U_idx, sizeof(int32_t) * U_ptr[R]);
    g->r_of = (int32_t *)malloc(sizeof(int32_t) * (n ? n : 1));
    for (i = 0; i < n; i++) g->r_of[i] = -1;
    for (i = 0; i < R; i++) g->r_of[elig[i]] = (int32_t)i;
    return g;
}

int32_t orc_graph_n_total(const orc_graph *g) { return g->NT; }
int64_t orc_graph_n_edges(const orc_graph *g) { return g->ne; }

/* Is node v one of the late users U_r of eligible tensor r? (reading P6) */
static int in_U(const orc_graph *g, int32_t r, int32_t v)
{
    int64_t k;
    for (k = g->U_ptr[r]; k < g->U_ptr[r + 1]; k++)
        if (g->U_idx[k] == v) return 1;
    return 0;
}

/* Device bytes held by a super-graph node's output (reading P5, P9). */
static int64_t node_bytes(const orc_graph *g, int32_t v)
{
    int32_t r, kind;
    if (v < g->n) return g->size[v];
    r = (v - g->n) / 3; kind = (v - g->n) % 3;
    if (kind == 1) return 0;            /* Store: data lives in external storage */
    return g->size[g->elig[r]];         /* clone A' (= |A|) or Load (= |A|) */
}

/*
 * Active set and transformed edge list of one candidate (Fig. 8,
 * P:1328-1346; readings P5, P6): original nodes are always active; clone_r
 * iff dec[r] = 1; store_r and load_r iff dec[r] = 2.  Re-mat moves the late
 * users U_r to the clone A', which reads the original copies of pre(t_r);
 * swap adds t_r -> Store -> Load and moves U_r to the Load.  active[NT] is
 * zeroed by the caller; *tsrc / *tdst are malloc'ed here.
 */
static void transformed_graph(const orc_graph *g, const uint8_t *dec, uint8_t *active,
                              int32_t **tsrc_out, int32_t **tdst_out, int64_t *nte_out)
{
    const int32_t n = g->n, R = g->R;
    int64_t nte = 0, cap_te, i, k;
    int32_t *tsrc, *tdst;
    for (i = 0; i < n; i++)
        active[i] = (g->F == 0 || g->nreg[i] < 0 || dec[R + g->nreg[i]] == g->nvn[i]) ? 1 : 0;
    for (i = 0; i < R; i++) {
        if (dec[i] == 1) active[n + 3 * i] = 1;
        if (dec[i] == 2) { active[n + 3 * i + 1] = 1; active[n + 3 * i + 2] = 1; }
    }
    cap_te = g->ne + 2 * R + 1;
    for (i = 0; i < R; i++) if (dec[i] == 1) {
        for (k = 0; k < g->ne; k++) if (g->dst[k] == g->elig[i]) cap_te++;
    }
    tsrc = (int32_t *)malloc(sizeof(int32_t) * cap_te);
    tdst = (int32_t *)malloc(sizeof(int32_t) * cap_te);
    for (k = 0; k < g->ne; k++) {
        int32_t u = g->src[k], v = g->dst[k];
        int32_t r = g->r_of[u];
        if (r >= 0 && dec[r] != 0 && in_U(g, r, v)) {
            /* the late user v now reads the clone A' (re-mat) or the Load (swap) */
            tsrc[nte] = (dec[r] == 1) ? (n + 3 * r) : (n + 3 * r + 2);
        } else {
            tsrc[nte] = u;
        }
        tdst[nte] = v;
        nte++;
    }
    for (i = 0; i < R; i++) {
        int32_t t = g->elig[i];
        if (dec[i] == 1) {
            /* A' has A's inputs (Fig. 8(a)(b)); it reads the original copies */
            for (k = 0; k < g->ne; k++) if (g->dst[k] == t) {
                tsrc[nte] = g->src[k]; tdst[nte] = n + 3 * (int32_t)i; nte++;
            }
        } else if (dec[i] == 2) {
            /* A -> Store -> Load -> B (Fig. 8(e)) */
            tsrc[nte] = t;                  tdst[nte] = n + 3 * (int32_t)i + 1; nte++;
            tsrc[nte] = n + 3 * (int32_t)i + 1; tdst[nte] = n + 3 * (int32_t)i + 2; nte++;
        }
    }
    /* the chosen F-Trans variants: an edge exists iff both ends exist (reading F1) */
    if (g->F > 0) {
        int64_t m = 0;
        for (k = 0; k < nte; k++)
            if (active[tsrc[k]] && active[tdst[k]]) { tsrc[m] = tsrc[k]; tdst[m] = tdst[k]; m++; }
        nte = m;
    }
    *tsrc_out = tsrc; *tdst_out = tdst; *nte_out = nte;
}

/* decision check (reading P12, R-noinput; F1: a variant index below nvar). */
static uint8_t check_dec(const orc_graph *g, const uint8_t *dec)
{
    uint8_t status = 0;
    int32_t i;
    for (i = 0; i < g->R; i++) {
        uint8_t d = dec[i];
        if (d > 2) status |= 4;
        /* re-materialization needs A's inputs: a tensor with no
         * inputs cannot be re-computed (reading R-noinput). */
        if (d == 1 && !g->has_input[g->elig[i]]) status |= 4;
    }
    for (i = 0; i < g->F; i++)
        if (dec[g->R + i] >= g->nvar[i]) status |= 4;
    return status;
}

/* Attach F-Trans variant regions (NEXT-4).  Returns 0, or -1 on bad input. */
int orc_graph_set_regions(orc_graph *g, int32_t F, const int32_t *nvar, const int32_t *nreg,
                          const uint8_t *nvn)
{
    int32_t i;
    if (F < 0) return -1;
    free(g->nvar); free(g->nreg); free(g->nvn);
    g->F = F;
    g->nvar = (int32_t *)malloc(sizeof(int32_t) * (F ? F : 1));
    g->nreg = (int32_t *)malloc(sizeof(int32_t) * (g->n ? g->n : 1));
    g->nvn = (uint8_t *)malloc(g->n ? g->n : 1);
    for (i = 0; i < F; i++) g->nvar[i] = nvar[i];
    for (i = 0; i < g->n; i++) {
        g->nreg[i] = F ? nreg[i] : -1;
        g->nvn[i] = F ? nvn[i] : 0;
        if (g->nreg[i] >= F) return -1;
    }
    return 0;
}

int32_t orc_graph_dec_len(const orc_graph *g) { return g->R + g->F; }

/*
 * Evaluate one candidate.
 *   perm[NT]  : the schedule over super-graph ids (step -> node)
 *   dec[R]    : 0 keep, 1 re-materialize, 2 swap (may be NULL when R == 0)
 * Outputs: status bits (bit0 not a permutation, bit1 edge violated,
 * bit2 bad decision), peak bytes (-1 if invalid), latency (+inf if invalid),
 * first compacted step attaining the peak (-1 if invalid).
 */
static void eval_impl(const orc_graph *g, const int32_t *perm, const uint8_t *dec,
                      uint8_t *status_out, int64_t *peak_out, double *lat_out,
                      int64_t *argmax_out, uint8_t *hot_out)
{
    const int32_t n = g->n, NT = g->NT;
    uint8_t status = 0;
    uint8_t *seen = NULL, *active = NULL;
    int32_t *pos = NULL, *step = NULL, *ord = NULL, *last = NULL;
    int32_t *tsrc = NULL, *tdst = NULL;
    int64_t nte = 0, i, k;
    int32_t nact = 0;
    int64_t peak = -1, argmax = -1;
    double latency = INFINITY;

    /* 1. permutation and decision check (reading P12) */
    seen = (uint8_t *)calloc(NT ? NT : 1, 1);
    for (i = 0; i < NT; i++) {
        int32_t p = perm[i];
        if (p < 0 || p >= NT || seen[p]) { status |= 1; continue; }
        seen[p] = 1;
    }
    status |= check_dec(g, dec);
    if (status) goto done;

    /* 2. active set and transformed graph (Fig. 8) */
    active = (uint8_t *)calloc(NT ? NT : 1, 1);
    transformed_graph(g, dec, active, &tsrc, &tdst, &nte);

    /* 3. validity: every dependency must be respected */
    pos = (int32_t *)malloc(sizeof(int32_t) * NT);
    for (i = 0; i < NT; i++) pos[perm[i]] = (int32_t)i;
    for (k = 0; k < nte; k++)
        if (pos[tsrc[k]] >= pos[tdst[k]]) { status |= 2; break; }
    if (status) goto done;

    /* 4. compaction: the active nodes in schedule order */
    ord = (int32_t *)malloc(sizeof(int32_t) * NT);
    step = (int32_t *)malloc(sizeof(int32_t) * NT);
    for (i = 0; i < NT; i++) step[i] = -1;
    for (i = 0; i < NT; i++) {
        int32_t v = perm[i];
        if (active[v]) { step[v] = nact; ord[nact] = v; nact++; }
    }

    /* 5. lifetimes: S_u = step(u); F_u = last reader's step; graph outputs
     * live to the end; tensors without readers die after their own step
     * (P:409-416 with S_j < i <= F_j, reading P1; reading P2). */
    last = (int32_t *)malloc(sizeof(int32_t) * NT);
    for (i = 0; i < NT; i++) last[i] = -1;
    for (k = 0; k < nte; k++) {
        int32_t u = tsrc[k], s = step[tdst[k]];
        if (s > last[u]) last[u] = s;
    }
    for (i = 0; i < NT; i++) {
        if (!active[i]) continue;
        if (i < n && g->is_output[i]) last[i] = nact - 1;
        else if (last[i] < 0) last[i] = step[i];
    }

    /* 6. memory: M_i = sum of |u| over u with S_u <= i <= F_u, walked as an
     * event list: before step i free every u with F_u = i-1, then allocate
     * the output of step i. */
    {
        int32_t *head = (int32_t *)malloc(sizeof(int32_t) * (nact + 1));
        int32_t *next = (int32_t *)malloc(sizeof(int32_t) * NT);
        int64_t cur = 0;
        for (i = 0; i <= nact; i++) head[i] = -1;
        for (i = 0; i < NT; i++) {
            if (!active[i]) continue;
            next[i] = head[last[i]]; head[last[i]] = (int32_t)i;
        }
        int64_t *curve = (int64_t *)malloc(sizeof(int64_t) * (nact ? nact : 1));
        peak = 0; argmax = -1;
        for (i = 0; i < nact; i++) {
            int32_t u;
            if (i > 0)
                for (u = head[i - 1]; u >= 0; u = next[u]) cur -= node_bytes(g, u);
            cur += node_bytes(g, ord[i]);
            curve[i] = cur;
            if (i == 0 || cur > peak) { peak = cur; argmax = i; }  /* first argmax (reading P10) */
        }
        /* memory hot-spots H = union of A_i over the steps with M_i = M_peak,
         * A_i = {u : S_u <= i <= F_u}, by the definition */
        if (hot_out) {
            for (i = 0; i < NT; i++) hot_out[i] = 0;
            for (i = 0; i < nact; i++) {
                if (curve[i] != peak) continue;
                for (k = 0; k < NT; k++)
                    if (active[k] && step[k] <= i && i <= last[k]) hot_out[k] = 1;
            }
        }
        free(head); free(next); free(curve);
    }

    /* 7. latency: compute, D2H (Store) and H2D (Load) are three in-order
     * queues; a compute op waits for the Loads it reads; a Store waits for
     * its producer; a Load waits for its Store (reading P7).
     * Without swaps this is sum(cost) over active compute ops. */
    {
        double Tc = 0.0, Td = 0.0, Th = 0.0;
        double *end = (double *)calloc(NT, sizeof(double));
        /* the (Load, reader) edges of the transformed graph */
        int64_t nlw = 0;
        int32_t *lw_load = (int32_t *)malloc(sizeof(int32_t) * (nte ? nte : 1));
        int32_t *lw_dst = (int32_t *)malloc(sizeof(int32_t) * (nte ? nte : 1));
        for (k = 0; k < nte; k++) {
            int32_t u = tsrc[k];
            if (u >= n && (u - n) % 3 == 2) { lw_load[nlw] = u; lw_dst[nlw] = tdst[k]; nlw++; }
        }
        for (i = 0; i < nact; i++) {
            int32_t v = ord[i];
            int32_t kind = (v < n) ? -1 : (v - n) % 3;
            int32_t r = (v < n) ? -1 : (v - n) / 3;
            if (kind == -1 || kind == 0) {
                double start = Tc;
                double c = (kind == -1) ? g->cost[v] : g->cost[g->elig[r]];
                for (k = 0; k < nlw; k++)
                    if (lw_dst[k] == v && end[lw_load[k]] > start) start = end[lw_load[k]];
                end[v] = start + c;
                Tc = end[v];
            } else if (kind == 1) {
                int32_t t = g->elig[r];
                double start = Td > end[t] ? Td : end[t];
                end[v] = start + g->swap_lat + (double)g->size[t] / g->swap_Bps;
                Td = end[v];
            } else {
                int32_t t = g->elig[r];
                int32_t st = v - 1;
                double start = Th > end[st] ? Th : end[st];
                end[v] = start + g->swap_lat + (double)g->size[t] / g->swap_Bps;
                Th = end[v];
            }
        }
        latency = Tc;
        if (Td > latency) latency = Td;
        if (Th > latency) latency = Th;
        free(end); free(lw_load); free(lw_dst);
    }

done:
    if (status) { peak = -1; latency = INFINITY; argmax = -1; }
    *status_out = status;
    *peak_out = peak;
    *lat_out = latency;
    if (argmax_out) *argmax_out = argmax;
    free(seen); free(active); free(pos); free(step); free(ord); free(last);
    free(tsrc); free(tdst);
}

void orc_eval(const orc_graph *g, const int32_t *perm, const uint8_t *dec,
              uint8_t *status_out, int64_t *peak_out, double *lat_out,
              int64_t *argmax_out)
{
    eval_impl(g, perm, dec, status_out, peak_out, lat_out, argmax_out, NULL);
}

/*
 * Dominators of the original graph G (T = T(G)): u dominates v
 * iff every path from a source (a node without predecessors) to v passes
 * through u.  Plain iterative set intersection over a topological order,
 * Dom(v) = {v} + intersection of Dom(p) over the predecessors p (sources:
 * {v}), as n x n byte matrices.  dom[u * n + v] = 1 iff u dominates v.
 * Returns NULL if G has a cycle.
 */
static uint8_t *dominators(const orc_graph *g)
{
    const int32_t n = g->n;
    int32_t *indeg = (int32_t *)calloc(n ? n : 1, sizeof(int32_t));
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (n ? n : 1));
    uint8_t *dom = (uint8_t *)calloc((size_t)n * n + 1, 1);
    int64_t k;
    int32_t head = 0, tail = 0, i, v, u;
    for (k = 0; k < g->ne; k++) indeg[g->dst[k]]++;
    for (v = 0; v < n; v++) if (indeg[v] == 0) order[tail++] = v;
    while (head < tail) {
        v = order[head++];
        for (k = 0; k < g->ne; k++)
            if (g->src[k] == v && --indeg[g->dst[k]] == 0) order[tail++] = g->dst[k];
    }
    if (tail != n) { free(indeg); free(order); free(dom); return NULL; }
    for (i = 0; i < n; i++) {
        int first = 1;
        v = order[i];
        for (k = 0; k < g->ne; k++) {
            if (g->dst[k] != v) continue;
            u = g->src[k];
            if (first) {
                int32_t w;
                for (w = 0; w < n; w++) dom[(size_t)w * n + v] = dom[(size_t)w * n + u];
                first = 0;
            } else {
                int32_t w;
                for (w = 0; w < n; w++) dom[(size_t)w * n + v] &= dom[(size_t)w * n + u];
            }
        }
        dom[(size_t)v * n + v] = 1;
    }
    free(indeg); free(order);
    return dom;
}

/* Immediate dominator of every node (-1: dominated only by the sources'
 * virtual root).  The strict dominators of v form a chain; idom(v) is the one
 * dominated by all the others.  Returns 0, or -1 on a cycle. */
int orc_idom(const orc_graph *g, int32_t *idom)
{
    const int32_t n = g->n;
    uint8_t *dom = dominators(g);
    int32_t v, u, w;
    if (!dom) return -1;
    for (v = 0; v < n; v++) {
        idom[v] = -1;
        for (u = 0; u < n; u++) {
            int all = 1;
            if (u == v || !dom[(size_t)u * n + v]) continue;
            for (w = 0; w < n && all; w++)
                if (w != v && dom[(size_t)w * n + v] && !dom[(size_t)w * n + u]) all = 0;
            if (all) { idom[v] = u; break; }
        }
    }
    free(dom);
    return 0;
}

/*
 * Memory hot-spots and the F-Trans metrics of one candidate.
 *   H: the tensors live at some step where M_i = M_peak.  Over
 *   the original graph (reading H1): a live clone A' or Load of t_r stands for
 *   t_r; a Store holds no device bytes and does not count.
 *   heat(v) = sum of |w| over w in H and in T.des(v)          (Eq. 3)
 *   score(v) = (1 - 1/nsplit) heat(v) - sum of |u| over u in
 *              G.inps(T.des(v)) minus H                          (Eq. 4)
 *   where T.des(v) = {w : v dominates w} and G.inps(S) = the nodes outside S
 *   with an edge into S.
 * hot[n] u8, heat[n] int64, score[n] double (zeroed if the candidate is
 * invalid).  Returns the status bits; *peak_out as orc_eval.
 */
int orc_hotspots(const orc_graph *g, const int32_t *perm, const uint8_t *dec, int32_t nsplit,
                 uint8_t *hot, int64_t *heat, double *score, int64_t *peak_out)
{
    const int32_t n = g->n, NT = g->NT;
    uint8_t status;
    int64_t peak, k;
    double lat;
    int32_t v, w, r;
    uint8_t *hs = (uint8_t *)calloc(NT ? NT : 1, 1);
    uint8_t *dom, *in_s;
    eval_impl(g, perm, dec, &status, &peak, &lat, NULL, hs);
    *peak_out = peak;
    for (v = 0; v < n; v++) { hot[v] = 0; heat[v] = 0; score[v] = 0.0; }
    if (status) { free(hs); return status; }
    for (v = 0; v < n; v++) hot[v] = hs[v];
    for (r = 0; r < g->R; r++)
        if (hs[n + 3 * r] || hs[n + 3 * r + 2]) hot[g->elig[r]] = 1;
    free(hs);
    dom = dominators(g);
    in_s = (uint8_t *)malloc(n ? n : 1);
    for (v = 0; v < n; v++) {
        int64_t h = 0, inp = 0;
        for (w = 0; w < n; w++)
            if (dom[(size_t)v * n + w] && hot[w]) h += g->size[w];
        /* G.inps(T.des(v)): sources of edges entering T.des(v), each once */
        for (w = 0; w < n; w++) in_s[w] = 0;
        for (k = 0; k < g->ne; k++) {
            int32_t a = g->src[k], b = g->dst[k];
            if (dom[(size_t)v * n + b] && !dom[(size_t)v * n + a]) in_s[a] = 1;
        }
        for (w = 0; w < n; w++)
            if (in_s[w] && !hot[w]) inp += g->size[w];
        heat[v] = h;
        score[v] = (1.0 - 1.0 / (double)nsplit) * (double)h - (double)inp;
    }
    free(dom); free(in_s);
    return status;
}

/* K candidates back to back: perms is K x NT row-major, decs K x R. */
void orc_eval_batch(const orc_graph *g, int64_t K, const int32_t *perms,
                    const uint8_t *decs, uint8_t *status, int64_t *peak,
                    double *lat)
{
    int64_t k;
    for (k = 0; k < K; k++)
        orc_eval(g, perms + k * (int64_t)g->NT,
                 (g->R + g->F) ? decs + k * (int64_t)(g->R + g->F) : NULL,
                 status + k, peak + k, lat + k, NULL);
}

/*
 * Pareto front of (peak, latency) over valid candidates, by the definition
 * (reading P10): a dominates b iff a.peak <= b.peak and
 * a.lat <= b.lat and one is strict; among exact duplicates only the smallest
 * id is kept.  Brute force O(n^2).  Output indices (into the input arrays)
 * sorted by ascending peak.  Returns the front size.
 */
int64_t orc_pareto(int64_t n, const int64_t *peak, const double *lat,
                   const uint8_t *status, const int64_t *id, int64_t *front_idx)
{
    int64_t i, j, nf = 0;
    for (i = 0; i < n; i++) {
        int keep = 1;
        if (status[i]) continue;
        for (j = 0; j < n && keep; j++) {
            if (j == i || status[j]) continue;
            if (peak[j] <= peak[i] && lat[j] <= lat[i] &&
                (peak[j] < peak[i] || lat[j] < lat[i])) keep = 0;
            else if (peak[j] == peak[i] && lat[j] == lat[i] && id[j] < id[i]) keep = 0;
        }
        if (keep) front_idx[nf++] = i;
    }
    /* insertion sort by ascending peak (front peaks are distinct) */
    for (i = 1; i < nf; i++) {
        int64_t x = front_idx[i];
        j = i - 1;
        while (j >= 0 && peak[front_idx[j]] > peak[x]) { front_idx[j + 1] = front_idx[j]; j--; }
        front_idx[j + 1] = x;
    }
    return nf;
}

/*
 * Best candidate under a memory limit M (Alg. 3 BetterThan with delta = 1,
 * P:1689-1692): argmin over valid candidates of the lexicographic key
 * (max(peak, M), lat, peak, id).  The extra "peak" key (reading P10b) makes
 * the best point non-dominated.  Under a latency limit L (the second mode,
 * P:1742-1745): argmin of (max(lat, L), peak, lat, id).  Returns the index
 * or -1 when no candidate is valid.
 */
int64_t orc_best_mem(int64_t n, const int64_t *peak, const double *lat,
                     const uint8_t *status, const int64_t *id, int64_t M)
{
    int64_t i, b = -1;
    for (i = 0; i < n; i++) {
        int64_t a1, b1;
        if (status[i]) continue;
        if (b < 0) { b = i; continue; }
        a1 = peak[i] > M ? peak[i] : M;
        b1 = peak[b] > M ? peak[b] : M;
        if (a1 != b1) { if (a1 < b1) b = i; continue; }
        if (lat[i] != lat[b]) { if (lat[i] < lat[b]) b = i; continue; }
        if (peak[i] != peak[b]) { if (peak[i] < peak[b]) b = i; continue; }
        if (id[i] < id[b]) b = i;
    }
    return b;
}

int64_t orc_best_lat(int64_t n, const int64_t *peak, const double *lat,
                     const uint8_t *status, const int64_t *id, double L)
{
    int64_t i, b = -1;
    for (i = 0; i < n; i++) {
        double a1, b1;
        if (status[i]) continue;
        if (b < 0) { b = i; continue; }
        a1 = lat[i] > L ? lat[i] : L;
        b1 = lat[b] > L ? lat[b] : L;
        if (a1 != b1) { if (a1 < b1) b = i; continue; }
        if (peak[i] != peak[b]) { if (peak[i] < peak[b]) b = i; continue; }
        if (lat[i] != lat[b]) { if (lat[i] < lat[b]) b = i; continue; }
        if (id[i] < id[b]) b = i;
    }
    return b;
}

/* ------------------------------------------------------------------------
 * GraphHash (Alg. 3 lines 3-6; the Weisfeiler-Lehman idea and
 * "(+) means bytes concatenation").  Readings G1-G4:
 *
 *   hash(b), b a byte string of 8m bytes read as little-endian 64-bit words
 *   w_0..w_{m-1}:   h = GAMMA * (m + 1);  h = mix64(h ^ w_i) for i = 0..m-1
 *   mix64 = the SplitMix64 output function, GAMMA = 0x9E3779B97F4A7C15   (G1)
 *
 *   line 5:  x_v = hash( hash(label_v) (+) x_{u_1} (+) ... (+) x_{u_k} )
 *            u_1..u_k = pre(v) in the transformed graph, in ascending order
 *            of x_u (pre(v) is a set; G2)
 *   line 6:  GraphHash(G) = hash( sum_v x_v mod 2^64 )
 *
 * label_v: the caller's 64-bit label of original op v; a clone A' carries
 * label(t_r) (same op, same inputs; G3); Store_r / Load_r carry
 * the tags 0x45524F5453 ("STORE") / 0x44414F4C ("LOAD") (G3).  The graph of
 * a candidate is its transformed graph (Fig. 8) over the active nodes; the
 * schedule does not enter (G4).  Invalid decisions: status bit 2, hash 0.
 * ------------------------------------------------------------------------ */
#define ORC_GAMMA 0x9E3779B97F4A7C15ull
#define ORC_TAG_STORE 0x45524F5453ull
#define ORC_TAG_LOAD 0x44414F4Cull

uint64_t orc_mix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t orc_hash_words(const uint64_t *w, int64_t m)
{
    uint64_t h = ORC_GAMMA * (uint64_t)(m + 1);
    int64_t i;
    for (i = 0; i < m; i++) h = orc_mix64(h ^ w[i]);
    return h;
}

static int cmp_u64(const void *a, const void *b)
{
    const uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return (x > y) - (x < y);
}

/* x_out[NT] (0 for inactive nodes) may be NULL.  Returns the status bits. */
int orc_graph_hash(const orc_graph *g, const uint64_t *label, const uint8_t *dec,
                   uint64_t *x_out, uint64_t *hash_out)
{
    const int32_t n = g->n, NT = g->NT;
    uint8_t *active;
    int32_t *tsrc, *tdst, *indeg, *queue;
    int64_t nte, i, k;
    int32_t qh = 0, qt = 0;
    uint64_t *x, *buf, sum = 0;
    int status = 0;

    status = check_dec(g, dec);
    if (status) {
        if (x_out) for (i = 0; i < NT; i++) x_out[i] = 0;
        *hash_out = 0;
        return status;
    }
    active = (uint8_t *)calloc(NT ? NT : 1, 1);
    transformed_graph(g, dec, active, &tsrc, &tdst, &nte);
    x = (uint64_t *)calloc(NT ? NT : 1, sizeof(uint64_t));
    buf = (uint64_t *)malloc(sizeof(uint64_t) * (nte + 1));
    indeg = (int32_t *)calloc(NT ? NT : 1, sizeof(int32_t));
    queue = (int32_t *)malloc(sizeof(int32_t) * (NT ? NT : 1));
    for (k = 0; k < nte; k++) indeg[tdst[k]]++;
    for (i = 0; i < NT; i++) if (active[i] && indeg[i] == 0) queue[qt++] = (int32_t)i;
    /* line 4: for v in topo-order(G) (Kahn) */
    while (qh < qt) {
        const int32_t v = queue[qh++];
        uint64_t lab;
        int64_t m = 0;
        if (v < n) lab = label[v];
        else {
            const int32_t r = (v - n) / 3, kind = (v - n) % 3;
            lab = kind == 0 ? label[g->elig[r]] : kind == 1 ? ORC_TAG_STORE : ORC_TAG_LOAD;
        }
        /* line 5: hash(v) (+) the x_u of pre(v), ascending */
        buf[m++] = orc_hash_words(&lab, 1);
        for (k = 0; k < nte; k++) if (tdst[k] == v) buf[m++] = x[tsrc[k]];
        qsort(buf + 1, (size_t)(m - 1), sizeof(uint64_t), cmp_u64);
        x[v] = orc_hash_words(buf, m);
        sum += x[v];
        for (k = 0; k < nte; k++) if (tsrc[k] == v && --indeg[tdst[k]] == 0) queue[qt++] = tdst[k];
    }
    /* line 6 */
    *hash_out = orc_hash_words(&sum, 1);
    if (x_out) for (i = 0; i < NT; i++) x_out[i] = x[i];
    free(active); free(tsrc); free(tdst); free(x); free(buf); free(indeg); free(queue);
    return 0;
}

void orc_graph_hash_batch(const orc_graph *g, const uint64_t *label, int64_t K, const uint8_t *decs,
                          uint8_t *status, uint64_t *hash)
{
    int64_t k;
    for (k = 0; k < K; k++)
        status[k] = (uint8_t)orc_graph_hash(g, label, (g->R + g->F) ? decs + k * (int64_t)(g->R + g->F) : NULL,
                                            NULL, hash + k);
}
