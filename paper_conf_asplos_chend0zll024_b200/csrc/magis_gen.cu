// magis_gen.cu -- seeded candidate generation on the device.
//
// Candidate k (global id) is a function of (seed, k) only, so a rank
// generates its own shard and the result does not depend on the rank count.
// The recipe stands in for MAGIS's rule application + re-ordering (§5.2
// P:1352-1357, Alg. 2) and is the one documented in DESIGN.md §5:
// decisions per eligible tensor, a random-priority Kahn order (or a local
// move: a window of the natural order re-ordered by the same keyed Kahn),
// Stores right after their producer ("as early as possible"),
// Loads / clones 0..slack steps before the first late user, inactive optional
// nodes last in id order, and 1% one random transposition.  It is bit-exact
// with the CPU generator used to produce test inputs (tests compare them).
//
// One thread builds one candidate (Kahn is sequential); its heap, in-degree
// and position arrays live in a graph-owned global scratch, contiguous per
// thread: a node's successors are mostly near it in id, so a thread's
// in-degree decrements share cache lines (an index-major layout put every
// access on its own line).  The scratch is sized for up to one thread per
// candidate of the call (within a memory budget): the kernel is latency
// bound on that scratch, so threads in flight are what pays (ncu, C2: 7
// warps per SM and 60% long-scoreboard stalls with 148 x 256 threads).
#include <algorithm>
#include <climits>
#include <cstdio>
#include <cstdlib>

#include "magis_internal.h"

namespace magis {

namespace {

constexpr uint32_t S_FAM = 1, S_DEC = 2, S_KEY = 3, S_WIN = 4, S_SLK = 5, S_TRN = 6;

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__device__ __forceinline__ uint64_t rnd(uint64_t seed, uint64_t k, uint32_t stream, uint64_t i) {
    uint64_t h = mix64(seed + 0x9E3779B97F4A7C15ull * (uint64_t)(stream + 1u));
    h = mix64(h ^ k);
    return mix64(h ^ i);
}

struct Scratch {
    int32_t* indeg;   // [n][T]
    uint64_t* heap;   // [n][T]
    int32_t* base;    // [n][T]
    int32_t* posb;    // [n][T]
    int64_t* opt;     // [2R][T]
    int64_t T;
    int64_t n, no;    // per-thread row lengths (nodes, 2R)
    __device__ __forceinline__ int32_t& I(int32_t i, int64_t t) const { return indeg[t * n + i]; }
    __device__ __forceinline__ uint64_t& H(int32_t i, int64_t t) const { return heap[t * n + i]; }
    __device__ __forceinline__ int32_t& B(int32_t i, int64_t t) const { return base[t * n + i]; }
    __device__ __forceinline__ int32_t& Q(int32_t i, int64_t t) const { return posb[t * n + i]; }
    __device__ __forceinline__ int64_t& O(int32_t i, int64_t t) const { return opt[t * no + i]; }
};

__device__ void heap_push(const Scratch& w, int64_t t, int32_t& nh, uint64_t x) {
    int32_t i = nh++;
    while (i > 0) {
        const int32_t p = (i - 1) >> 1;
        const uint64_t hp = w.H(p, t);
        if (hp <= x) break;
        w.H(i, t) = hp;
        i = p;
    }
    w.H(i, t) = x;
}

__device__ uint64_t heap_pop(const Scratch& w, int64_t t, int32_t& nh) {
    const uint64_t top = w.H(0, t), x = w.H(--nh, t);
    int32_t i = 0;
    for (;;) {
        int32_t c = 2 * i + 1;
        if (c >= nh) break;
        uint64_t hc = w.H(c, t);
        if (c + 1 < nh) {
            const uint64_t h2 = w.H(c + 1, t);
            if (h2 < hc) { c++; hc = h2; }
        }
        if (hc >= x) break;
        w.H(i, t) = hc;
        i = c;
    }
    if (nh > 0) w.H(i, t) = x;
    return top;
}

// keyed Kahn over the natural-order range [lo, hi) (edges inside the range)
__device__ void keyed_kahn(const DevGraph& g, const GenTables& gt, const Scratch& w, int64_t t,
                           uint64_t seed, uint64_t k, int32_t lo, int32_t hi, int32_t out0) {
    int32_t nh = 0, m = 0;
    for (int32_t v = lo; v < hi; v++) {
        int32_t d = 0;
        for (int32_t e = gt.pred_ptr[v]; e < gt.pred_ptr[v + 1]; e++) d += gt.pred[e] >= lo;
        w.I(v, t) = d;
    }
    for (int32_t v = lo; v < hi; v++)
        if (w.I(v, t) == 0)
            heap_push(w, t, nh, ((rnd(seed, k, S_KEY, (uint64_t)v) >> 48) << 32) | (uint32_t)v);
    while (nh > 0) {
        const uint64_t x = heap_pop(w, t, nh);
        const int32_t u = (int32_t)(x & 0xffffffffu);
        w.B(out0 + m, t) = u;
        m++;
        for (int32_t e = gt.succ_ptr[u]; e < gt.succ_ptr[u + 1]; e++) {
            const int32_t s = gt.succ[e];
            if (s >= hi) continue;
            if (--w.I(s, t) == 0)
                heap_push(w, t, nh, ((rnd(seed, k, S_KEY, (uint64_t)s) >> 48) << 32) | (uint32_t)s);
        }
    }
    (void)g;
}

__global__ void __launch_bounds__(128)
gen_kernel(DevGraph g, GenTables gt, GenSpec sp, uint64_t id0, int64_t K, int32_t* __restrict__ perms,
           uint8_t* __restrict__ decs, Scratch w, const uint8_t* __restrict__ only, const int32_t* __restrict__ nonly) {
    const int32_t n = g.n, R = g.R, NT = g.NT;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // re-run mode: only the candidates the fast kernel flagged (usually none)
    if (only && *nonly == 0) return;
    for (int64_t kk = t; kk < K; kk += w.T) {
        if (only && !only[kk]) continue;
        const uint64_t k = id0 + (uint64_t)kk;
        const uint64_t seed = sp.seed;
        int32_t* perm = perms + kk * (int64_t)NT;
        uint8_t* dec = decs + kk * (int64_t)(R ? R : 1);
        const uint32_t fam = (uint32_t)(rnd(seed, k, S_FAM, 0) % 100u);
        if (R == 0) dec[0] = 0;                          // the row's pad byte (no decisions)
        for (int32_t r = 0; r < R; r++) {
            const uint32_t x = (uint32_t)(rnd(seed, k, S_DEC, (uint64_t)r) % 10000u);
            const int32_t tr = g.elig[r];
            uint8_t d = 0;
            if ((int32_t)x < sp.p_remat && gt.pred_ptr[tr + 1] > gt.pred_ptr[tr]) d = 1;
            else if ((int32_t)x < sp.p_remat + sp.p_swap) d = 2;
            dec[r] = d;
        }
        if ((int32_t)fam < sp.pct_random || (int32_t)fam >= sp.pct_random + sp.pct_local) {
            keyed_kahn(g, gt, w, t, seed, k, 0, n, 0);
        } else {
            int32_t len = 2 + (int32_t)(rnd(seed, k, S_WIN, 0) % (uint64_t)(sp.wmax - 1));
            if (len > n) len = n;
            const int32_t b = (int32_t)(rnd(seed, k, S_WIN, 1) % (uint64_t)(n - len + 1));
            for (int32_t i = 0; i < n; i++) w.B(i, t) = i;
            keyed_kahn(g, gt, w, t, seed, k, b, b + len, b);
        }
        for (int32_t i = 0; i < n; i++) w.Q(w.B(i, t), t) = i;
        // optional nodes: sort keys (gap, prio, r)
        int32_t nopt = 0;
        for (int32_t r = 0; r < R; r++) {
            const uint8_t d = dec[r];
            if (d == 0) continue;
            const int32_t tr = g.elig[r];
            int32_t q = INT_MAX;
            for (int32_t e = g.U_ptr[r]; e < g.U_ptr[r + 1]; e++) q = min(q, w.Q(g.U_idx[e], t));
            const int32_t j = (int32_t)(rnd(seed, k, S_SLK, (uint64_t)r) % (uint64_t)(sp.slack + 1));
            if (d == 2) {
                const int32_t gs = w.Q(tr, t) + 1;
                const int32_t gl = max(q - j, gs);
                w.O(nopt++, t) = ((int64_t)gs << 32) | (0ll << 30) | r;
                w.O(nopt++, t) = ((int64_t)gl << 32) | (1ll << 30) | r;
            } else {
                int32_t lo = 0;
                for (int32_t e = gt.pred_ptr[tr]; e < gt.pred_ptr[tr + 1]; e++) lo = max(lo, w.Q(gt.pred[e], t) + 1);
                w.O(nopt++, t) = ((int64_t)max(q - j, lo) << 32) | (1ll << 30) | r;
            }
        }
        for (int32_t i = 1; i < nopt; i++) {           // insertion sort (few active optional nodes)
            const int64_t x = w.O(i, t);
            int32_t j = i - 1;
            while (j >= 0 && w.O(j, t) > x) { w.O(j + 1, t) = w.O(j, t); j--; }
            w.O(j + 1, t) = x;
        }
        int32_t m = 0, oi = 0;
        for (int32_t i = 0; i <= n; i++) {
            while (oi < nopt && (int32_t)(w.O(oi, t) >> 32) == i) {
                const int64_t o = w.O(oi, t);
                const int32_t rr = (int32_t)(o & 0x3fffffff);
                const int32_t pr = (int32_t)((o >> 30) & 3);
                perm[m++] = (pr == 0) ? n + 3 * rr + 1 : (dec[rr] == 2 ? n + 3 * rr + 2 : n + 3 * rr);
                oi++;
            }
            if (i < n) perm[m++] = w.B(i, t);
        }
        for (int32_t r = 0; r < R; r++) {
            if (dec[r] != 1) perm[m++] = n + 3 * r;
            if (dec[r] != 2) { perm[m++] = n + 3 * r + 1; perm[m++] = n + 3 * r + 2; }
        }
        if ((int32_t)fam >= sp.pct_random + sp.pct_local) {
            const int32_t a = (int32_t)(rnd(seed, k, S_TRN, 0) % (uint64_t)NT);
            const int32_t b2 = (int32_t)(rnd(seed, k, S_TRN, 1) % (uint64_t)NT);
            const int32_t tmp = perm[a];
            perm[a] = perm[b2];
            perm[b2] = tmp;
        }
    }
}

// ----------------------------------------------------------- fast kernel --
// Same recipe, same bytes, re-laid out for the SM (one thread per candidate,
// persistent grid):
//  * the per-stream hash prefix mix64(mix64(seed + G (s + 1)) ^ k) is computed
//    once per candidate, so every draw is one mix64;
//  * the Kahn ready set is split: the sources of G (ready from the start; 163
//    of 1,472 nodes on C2, 502 of 22,026 on C4) are bucket-sorted by key once
//    per candidate into a global stream read in order, and only the nodes that
//    become ready during the sweep go to a binary heap held on chip (measured
//    at most 14 entries on C2 / C5, 97 on C3, 65 on C4);
//  * a heap entry is 4 bytes: the key's top 16 bits and the node id, so the
//    common comparison is one u32 compare; equal top halves (p = 2^-16) fall
//    back to the full (key, id) order, so the output is the same order;
//  * readiness is a bitset of emitted nodes (on chip for n <= 3,072) tested
//    over the successor's inputs (in-degree <= 4 on these graphs) instead of
//    per-candidate in-degree counters;
//  * the base order is written straight into the candidate's perm row, only
//    the positions the optional-node placement reads are kept (slot map), and
//    the optional nodes are merged in place from the end of the row.
// A candidate whose dynamic ready set outgrows the on-chip heap is flagged and
// re-generated by the sequential kernel above (gen_kernel's re-run mode).
// (key, id) of a node as one u32: the key is the draw's top 16 bits (candgen.c)
__device__ __forceinline__ uint32_t ent_of(uint64_t hk, uint32_t v) { return ((uint32_t)(mix64(hk ^ v) >> 48) << 16) | v; }

// heap entries on chip per thread (more spill to the thread's global slice):
// 32, or 64 on graphs past 16k nodes (measured: C4 146 -> 125 ms per 65,536;
// C3 26.4 -> 28.7 ms, its L1 share matters more than its 96-wide bursts)
template <int HCT> constexpr int gen_hc() { return HCT; }
constexpr int kGenHG = 1024;      // spill entries; a larger ready set re-runs the candidate on gen_kernel

// graph tables: read-only path, kept in L1 ahead of the per-thread scratch
__device__ __forceinline__ uint2 ld_tab(const uint2* p) {
    uint2 r;
    asm volatile("ld.global.nc.L1::evict_last.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}

template <bool BSM, int HCT>
__global__ void __launch_bounds__(128)
gen2_kernel(DevGraph g, GenTables gt, GenSpec sp, uint64_t id0, int64_t K, int32_t* __restrict__ perms,
            uint8_t* __restrict__ decs, char* __restrict__ scr, int64_t wstride, int32_t lgnb,
            uint8_t* __restrict__ flag, int32_t* __restrict__ nflag) {
    constexpr int HC = gen_hc<HCT>();
    extern __shared__ uint32_t smg[];
    const int TB = blockDim.x, tid = threadIdx.x;
    const int32_t n = g.n, R = g.R, NT = g.NT, S = gt.S, nq = gt.nq;
    const int32_t NW = (n + 31) >> 5, NB = 1 << lgnb;
    const int64_t T = (int64_t)gridDim.x * TB, t = (int64_t)blockIdx.x * TB + tid;
    uint32_t* hp = smg + tid;                            // heap entry i < HC at hp[i * TB]
    char* my = scr + t * wstride;
    uint32_t* srt = (uint32_t*)my;                       // [S] sources, bucketed by key
    uint16_t* boff = (uint16_t*)(my + ((size_t)S * 4 + 15) / 16 * 16);            // [NB + 1]
    uint16_t* Q = boff + (((size_t)NB + 1 + 7) & ~(size_t)7);                       // [nq] base positions
    uint16_t* bs = Q + (((size_t)nq + 7) & ~(size_t)7);                             // [n] base order (u16)
    uint32_t* gbits = (uint32_t*)(bs + (((size_t)n + 7) & ~(size_t)7));            // [NW] (!BSM)
    uint32_t* opt = gbits + (BSM ? 0 : ((NW + 3) & ~3));                           // [2R]
    uint32_t* hg = opt + ((2 * (R ? R : 1) + 3) & ~3) - HC;                        // heap entry i >= HC at hg[i]
    uint16_t* wc = (uint16_t*)(hg + HC + kGenHG);                                   // [W] emitted inputs of wide nodes
    auto bw = [&](int32_t w) -> uint32_t& { if constexpr (BSM) return smg[(HC + w) * TB + tid]; else return gbits[w]; };
    auto hat = [&](int32_t i) -> uint32_t& { return i < HC ? hp[i * TB] : hg[i]; };
    // per-stream prefixes mix64(seed + G (stream + 1)), shared by all candidates
    uint64_t hb[7];
#pragma unroll
    for (int s = 1; s <= 6; s++) hb[s] = mix64(sp.seed + 0x9E3779B97F4A7C15ull * (uint64_t)(s + 1));
    for (int64_t kk = t; kk < K; kk += T) {
        const uint64_t k = id0 + (uint64_t)kk;
        uint64_t hk[7];
#pragma unroll
        for (int s = 1; s <= 6; s++) hk[s] = mix64(hb[s] ^ k);
        const uint64_t hK = hk[S_KEY];
        int32_t* perm = perms + kk * (int64_t)NT;
        uint8_t* dec = decs + kk * (int64_t)(R ? R : 1);
        const uint32_t fam = (uint32_t)(mix64(hk[S_FAM]) % 100u);
        if (R == 0) dec[0] = 0;                          // the row's pad byte (no decisions)
        for (int32_t r = 0; r < R; r++) {
            const uint32_t x = (uint32_t)(mix64(hk[S_DEC] ^ (uint64_t)r) % 10000u);
            const int32_t tr = g.elig[r];
            uint8_t d = 0;
            if ((int32_t)x < sp.p_remat && gt.pred_ptr[tr + 1] > gt.pred_ptr[tr]) d = 1;
            else if ((int32_t)x < sp.p_remat + sp.p_swap) d = 2;
            dec[r] = d;
        }
        int32_t nh = 0;
        bool over = false;
        // heap ops: entries below HC on chip; the general accessor only while
        // the ready set is larger (rare, warp-uniform in practice)
        auto push = [&](uint32_t x) {
            int32_t i = nh++;
            if (nh <= HC) {
                while (i > 0) {
                    const int32_t p = (i - 1) >> 1;
                    const uint32_t hpp = hp[p * TB];
                    if (hpp <= x) break;
                    hp[i * TB] = hpp;
                    i = p;
                }
                hp[i * TB] = x;
                return;
            }
            while (i > 0) {
                const int32_t p = (i - 1) >> 1;
                const uint32_t hpp = hat(p);
                if (hpp <= x) break;
                hat(i) = hpp;
                i = p;
            }
            hat(i) = x;
        };
        auto pop = [&]() -> uint32_t {
            const uint32_t top = hp[0];
            int32_t i = 0;
            if (nh <= HC) {
                const uint32_t x = hp[(--nh) * TB];
                for (;;) {
                    int32_t c = 2 * i + 1;
                    if (c >= nh) break;
                    uint32_t hc = hp[c * TB];
                    if (c + 1 < nh) {
                        const uint32_t h2 = hp[(c + 1) * TB];
                        if (h2 < hc) { c++; hc = h2; }
                    }
                    if (hc >= x) break;
                    hp[i * TB] = hc;
                    i = c;
                }
                if (nh > 0) hp[i * TB] = x;
                return top;
            }
            const uint32_t x = hat(--nh);
            for (;;) {
                int32_t c = 2 * i + 1;
                if (c >= nh) break;
                uint32_t hc = hat(c);
                if (c + 1 < nh) {
                    const uint32_t h2 = hat(c + 1);
                    if (h2 < hc) { c++; hc = h2; }
                }
                if (hc >= x) break;
                hat(i) = hc;
                i = c;
            }
            if (nh > 0) hat(i) = x;
            return top;
        };
        auto emitted = [&](uint32_t p, int32_t lo) -> bool {
            return p == 0xffffu || (int32_t)p < lo || ((bw((int32_t)p >> 5) >> (p & 31)) & 1u);
        };
        // successor record of edge u -> s: every other input of s emitted
        // (inputs below lo count as emitted: the window's prefix)
        bool wide_ok = false;                            // wide-node counters zeroed (F1 / F3)
        auto ready = [&](uint2 rc, int32_t u, int32_t lo) -> bool {
            const uint32_t o0 = rc.x >> 16;
            if (o0 == 0xfffeu && wide_ok && (rc.y & 0xffffu) != 0xffffu) {
                // wide node (C4's 32-input merges): count its emitted inputs
                // instead of scanning them at every input's emission
                const uint32_t slot = rc.y & 0xffffu;
                const uint32_t c = (uint32_t)wc[slot] + 1u;
                wc[slot] = (uint16_t)c;
                return c == (rc.y >> 16);
            }
            if (o0 == 0xfffeu) {
                const int32_t s = (int32_t)(rc.x & 0xffffu);
                for (int32_t e = gt.pred_ptr[s], e1 = gt.pred_ptr[s + 1]; e < e1; e++) {
                    const int32_t p = gt.pred[e];
                    if (p != u && !emitted((uint32_t)p, lo)) return false;
                }
                return true;
            }
            return emitted(o0, lo) & emitted(rc.y & 0xffffu, lo) & emitted(rc.y >> 16, lo);
        };
        auto visit = [&](int32_t u, int32_t m, int32_t hi, int32_t lo) {
            const uint2 si = ld_tab(gt.sinfo + u);
            const uint32_t cnt = si.y & 0xffffu, qs = si.y >> 16;
            if (qs != 0xffffu) Q[qs] = (uint16_t)m;
            // successors 4 at a time: the records, then the readiness tests of
            // all 4 (independent loads), then the pushes (the emitted set does
            // not change inside one node's visit, and the pop order depends on
            // the keys only, not on the order of pushes)
            for (uint32_t e0 = 0; e0 < cnt; e0 += 4) {
                uint2 rc[4];
#pragma unroll
                for (int k = 0; k < 4; k++)
                    rc[k] = e0 + k < cnt ? ld_tab(gt.rec + si.x + e0 + k) : make_uint2(0xffffu, 0u);
                bool rd[4];
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const int32_t s = (int32_t)(rc[k].x & 0xffffu);
                    rd[k] = e0 + k < cnt && s < hi && ready(rc[k], u, lo);
                }
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (!rd[k]) continue;
                    if (nh >= HC + kGenHG) { over = true; return; }
                    push(ent_of(hK, rc[k].x & 0xffffu));
                }
            }
        };
        int32_t lo = 0, hi = n;
        if ((int32_t)fam < sp.pct_random || (int32_t)fam >= sp.pct_random + sp.pct_local) {
            // ---- F1 / F3: keyed Kahn over G ----------------------------------
            for (int32_t w = 0; w < NW; w++) bw(w) = 0u;
            for (int32_t i = 0; i < gt.W; i++) wc[i] = 0;
            wide_ok = true;
            for (int32_t b = 0; b <= NB; b++) boff[b] = 0;
            const int32_t sh = 32 - lgnb;
            for (int32_t i = 0; i < S; i++) boff[(ent_of(hK, (uint32_t)gt.src[i]) >> sh) + 1]++;
            for (int32_t b = 0; b < NB; b++) boff[b + 1] += boff[b];
            // scatter: boff[b] advances from the start of bucket b to its end
            for (int32_t i = 0; i < S; i++) {
                const uint32_t x = ent_of(hK, (uint32_t)gt.src[i]);
                srt[boff[x >> sh]++] = x;
            }
            int32_t cur = 0, bend = 0, bk = -1;
            uint32_t sv = 0;
            // next non-empty bucket, insertion-sorted on entry
            auto advance = [&]() {
                while (cur == bend && bk + 1 < NB) bend = boff[++bk];
                for (int32_t i = cur + 1; i < bend; i++) {
                    const uint32_t x = srt[i];
                    int32_t j = i - 1;
                    while (j >= cur && x < srt[j]) { srt[j + 1] = srt[j]; j--; }
                    srt[j + 1] = x;
                }
                if (cur < bend) sv = srt[cur];
            };
            advance();
            for (int32_t m = 0; m < n; m++) {
                uint32_t x;
                if (nh > 0 && (cur >= bend || hp[0] < sv)) {
                    x = pop();
                } else {
                    x = sv;
                    if (++cur == bend) advance(); else sv = srt[cur];
                }
                const int32_t u = (int32_t)(x & 0xffffu);
                bs[m] = (uint16_t)u;
                bw(u >> 5) |= 1u << (u & 31);
                visit(u, m, n, 0);
                if (over) break;
            }
        } else {
            // ---- F2: a window of the natural order re-ordered by the keyed Kahn
            int32_t len = 2 + (int32_t)(mix64(hk[S_WIN]) % (uint64_t)(sp.wmax - 1));
            if (len > n) len = n;
            lo = (int32_t)(mix64(hk[S_WIN] ^ 1ull) % (uint64_t)(n - len + 1));
            hi = lo + len;
            for (int32_t w = lo >> 5; w <= (hi - 1) >> 5; w++) bw(w) = 0u;
            for (int32_t v = lo; v < hi && !over; v++) {
                bool src = true;
                for (int32_t e = gt.pred_ptr[v], e1 = gt.pred_ptr[v + 1]; e < e1; e++) src &= gt.pred[e] < lo;
                if (src) {
                    if (nh >= HC + kGenHG) { over = true; break; }
                    push(ent_of(hK, (uint32_t)v));
                }
            }
            for (int32_t j = 0; j < nq; j++) Q[j] = (uint16_t)gt.qnode[j];
            int32_t m = 0;
            while (nh > 0 && !over) {
                const int32_t u = (int32_t)(pop() & 0xffffu);
                bs[m] = (uint16_t)u;                     // window order at bs[0, len)
                bw(u >> 5) |= 1u << (u & 31);
                visit(u, lo + m, hi, lo);
                m++;
            }
        }
        flag[kk] = over ? 1 : 0;
        if (over) {
            atomicAdd(nflag, 1);
            continue;                                   // re-generated by gen_kernel
        }
        const bool win = lo > 0 || hi < n;             // F2 with a proper window
        // ---- optional nodes: keys (gap << 16 | prio << 15 | r), ascending ------
        int32_t nopt = 0;
        for (int32_t r = 0; r < R; r++) {
            const uint8_t d = dec[r];
            if (d == 0) continue;
            const int32_t tr = g.elig[r];
            int32_t q = INT_MAX;
            for (int32_t e = g.U_ptr[r]; e < g.U_ptr[r + 1]; e++) q = min(q, (int32_t)Q[gt.qmap[g.U_idx[e]]]);
            const int32_t j = (int32_t)(mix64(hk[S_SLK] ^ (uint64_t)r) % (uint64_t)(sp.slack + 1));
            uint32_t ks[2];
            int no = 0;
            if (d == 2) {
                const int32_t gs = (int32_t)Q[gt.qmap[tr]] + 1;
                ks[no++] = ((uint32_t)gs << 16) | (uint32_t)r;
                ks[no++] = ((uint32_t)max(q - j, gs) << 16) | (1u << 15) | (uint32_t)r;
            } else {
                int32_t lo2 = 0;
                for (int32_t e = gt.pred_ptr[tr]; e < gt.pred_ptr[tr + 1]; e++)
                    lo2 = max(lo2, (int32_t)Q[gt.qmap[gt.pred[e]]] + 1);
                ks[no++] = ((uint32_t)max(q - j, lo2) << 16) | (1u << 15) | (uint32_t)r;
            }
            for (int a = 0; a < no; a++) {                // insertion into the sorted list
                const uint32_t x = ks[a];
                int32_t i = nopt - 1;
                while (i >= 0 && opt[i] > x) { opt[i + 1] = opt[i]; i--; }
                opt[i + 1] = x;
                nopt++;
            }
        }
        // ---- the row: optional nodes of gap i before base[i], in key order -------
        {
            int32_t m = 0, oi = 0;
            uint32_t gnext = nopt > 0 ? (opt[0] >> 16) : 0xffffffffu;
            auto emit_opts = [&](int32_t i) {
                while ((int32_t)gnext == i) {
                    const uint32_t o = opt[oi++];
                    const int32_t rr = (int32_t)(o & 0x7fffu);
                    __stcs(perm + m++, ((o >> 15) & 1u) == 0 ? n + 3 * rr + 1 : (dec[rr] == 2 ? n + 3 * rr + 2 : n + 3 * rr));
                    gnext = oi < nopt ? (opt[oi] >> 16) : 0xffffffffu;
                }
            };
            if (!win) {
                const int32_t n8 = n & ~7;
                for (int32_t i0 = 0; i0 < n8; i0 += 8) {
                    const uint4 c = *reinterpret_cast<const uint4*>(bs + i0);
                    const uint32_t w4[4] = {c.x, c.y, c.z, c.w};
#pragma unroll
                    for (int j = 0; j < 8; j++) {
                        emit_opts(i0 + j);
                        __stcs(perm + m++, (int32_t)((w4[j >> 1] >> (16 * (j & 1))) & 0xffffu));
                    }
                }
                for (int32_t i = n8; i < n; i++) { emit_opts(i); __stcs(perm + m++, (int32_t)bs[i]); }
            } else {
                for (int32_t i = 0; i < n; i++) {
                    emit_opts(i);
                    __stcs(perm + m++, (i >= lo && i < hi) ? (int32_t)bs[i - lo] : i);
                }
            }
            emit_opts(n);
            for (int32_t r = 0; r < R; r++) {
                const uint8_t d = dec[r];
                if (d != 1) __stcs(perm + m++, n + 3 * r);
                if (d != 2) { __stcs(perm + m++, n + 3 * r + 1); __stcs(perm + m++, n + 3 * r + 2); }
            }
        }
        if ((int32_t)fam >= sp.pct_random + sp.pct_local) {
            const int32_t a = (int32_t)(mix64(hk[S_TRN]) % (uint64_t)NT);
            const int32_t b2 = (int32_t)(mix64(hk[S_TRN] ^ 1ull) % (uint64_t)NT);
            const int32_t tmp = perm[a];
            perm[a] = perm[b2];
            perm[b2] = tmp;
        }
    }
}

}  // namespace

namespace {
size_t seq_bytes_per_thread(const DevGraph& g) {
    return (size_t)g.n * (4 + 8 + 4 + 4) + (size_t)2 * (g.R ? g.R : 1) * 8;
}
int gen_lgnb(const GenTables& gt) {
    int lg = 1;                                   // >= 2 buckets: the shift 32 - lg stays < 32
    while ((1 << lg) * 4 < gt.S && lg < 12) lg++;
    return lg;
}
const void* gen2_select(int bsm, int hc) {
    return bsm ? (const void*)gen2_kernel<true, 32> : (hc == 64 ? (const void*)gen2_kernel<false, 64> : (const void*)gen2_kernel<false, 32>);
}
constexpr int kGenTB = 128;
constexpr int64_t kSeqFixT = 1024;   // sequential re-run threads
}  // namespace

GenPlan gen_plan(int device, const DevGraph& g, const GenTables& gt, int64_t K) {
    GenPlan p;
    int sms = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || sms < 1) {
        cudaGetLastError();
        sms = 148;
    }
    const char* off = std::getenv("MAGIS_GEN_SEQ");            // force the sequential kernel (tests)
    if (gt.fast && !(off && std::atoi(off) != 0)) {
        const int32_t NW = (g.n + 31) >> 5;
        const char* bf = std::getenv("MAGIS_GEN_BSM");
        p.bsm = bf ? (std::atoi(bf) != 0 && NW <= 384) : (NW <= 96 ? 1 : 0);
        p.hc = (!p.bsm && g.n > 16384) ? 64 : 32;
        const size_t smem = (size_t)kGenTB * (p.hc + (p.bsm ? NW : 0)) * 4;
        const void* fn = gen2_select(p.bsm, p.hc);
        cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        // the attribute persists per kernel: start from the all-shared carveout
        // (an earlier call on a smaller graph may have lowered it)
        cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
        int per = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, kGenTB, smem) != cudaSuccess || per < 1) {
            cudaGetLastError();
            per = 1;
        }
        const int64_t cand = (K + kGenTB - 1) / kGenTB * kGenTB;
        // the rest of the SM's unified memory stays L1 for the graph tables:
        // ask for the shared-memory carveout of the blocks one wave needs
        {
            const int64_t need = std::min<int64_t>(per, (cand / kGenTB + sms - 1) / sms);
            const size_t bytes = (size_t)need * (smem + 1024);
            const int pct = (int)std::min<size_t>(100, (bytes * 100 + 228 * 1024 - 1) / (228 * 1024));
            // (only when it leaves L1 at least 32 KB: C5's 4 x 57 KB at 99% measured
            // 9.6 -> 13.1 ms; C2 6.1 -> 5.2, C3 30.8 -> 26.2, C4 199 -> 176 ms)
            const char* cv = std::getenv("MAGIS_GEN_CARVE");
            const int want = cv ? std::atoi(cv) : (bytes + 32 * 1024 <= 228 * 1024 ? std::max(pct, 1) : 100);
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, want);
            int per2 = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per2, fn, kGenTB, smem) != cudaSuccess) {
                cudaGetLastError();
                per2 = 0;
            }
            if (per2 >= need) {
                per = per2;
            } else {                                   // the rounded carveout holds fewer blocks: all shared
                cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
                if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per2, fn, kGenTB, smem) == cudaSuccess && per2 >= 1)
                    per = per2;
                else
                    cudaGetLastError();
            }
        }
        p.T2 = std::min<int64_t>((int64_t)sms * per * kGenTB, cand);
        const size_t nb = (size_t)1 << gen_lgnb(gt);
        p.w2 = ((size_t)gt.S * 4 + 15) / 16 * 16 + ((nb + 1 + 7) & ~(size_t)7) * 2 + (((size_t)gt.nq + 7) & ~(size_t)7) * 2 +
               (((size_t)g.n + 7) & ~(size_t)7) * 2 + (p.bsm ? 0 : (size_t)((NW + 3) & ~3) * 4) +
               (((size_t)2 * std::max(g.R, 1) + 3) & ~(size_t)3) * 4 + (size_t)kGenHG * 4 +
               (((size_t)gt.W + 7) & ~(size_t)7) * 2;
        p.w2 = (p.w2 + 127) / 128 * 128;
        p.T1 = std::min<int64_t>(kSeqFixT, K);
    } else {
        // sequential kernel for the whole call: up to one thread per candidate
        // within a 16 GiB scratch budget
        const int64_t base = (int64_t)sms * 256;
        const int64_t cap = std::max<int64_t>(base, (16LL << 30) / (int64_t)std::max<size_t>(seq_bytes_per_thread(g), 1));
        p.T1 = std::max<int64_t>(base, std::min<int64_t>(K, cap)) / 128 * 128;
    }
    p.bytes = (size_t)p.T2 * p.w2 + ((size_t)K + 255) / 256 * 256 + 256 + (size_t)p.T1 * seq_bytes_per_thread(g) + 256;
    return p;
}

cudaError_t gen_launch(const DevGraph& g, const GenTables& gt, const GenSpec& sp, uint64_t id0, int64_t K,
                       int32_t* perm, uint8_t* dec, void* scratch, const GenPlan& gp, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    char* b = (char*)scratch;
    char* s2 = b;                                   b += (size_t)gp.T2 * gp.w2;
    uint8_t* flag = (uint8_t*)b;                    b += ((size_t)K + 255) / 256 * 256;
    int32_t* nflag = (int32_t*)b;                   b += 256;
    Scratch w;
    w.T = gp.T1;
    w.n = g.n;
    w.no = 2 * (g.R ? g.R : 1);
    w.heap = (uint64_t*)b;   b += (size_t)g.n * 8 * gp.T1;
    w.opt = (int64_t*)b;     b += (size_t)2 * (g.R ? g.R : 1) * 8 * gp.T1;
    w.indeg = (int32_t*)b;   b += (size_t)g.n * 4 * gp.T1;
    w.base = (int32_t*)b;    b += (size_t)g.n * 4 * gp.T1;
    w.posb = (int32_t*)b;
    const unsigned blocks1 = (unsigned)((std::min<int64_t>(gp.T1, K) + 127) / 128);
    if (gp.T2 > 0) {
        cudaError_t e = cudaMemsetAsync(nflag, 0, 4, stream);
        if (e != cudaSuccess) return e;
        const int32_t NW = (g.n + 31) >> 5;
        const size_t smem = (size_t)kGenTB * (gp.hc + (gp.bsm ? NW : 0)) * 4;
        const int lg = gen_lgnb(gt);
        const unsigned blocks2 = (unsigned)(gp.T2 / kGenTB);
        if (gp.bsm) gen2_kernel<true, 32><<<blocks2, kGenTB, smem, stream>>>(g, gt, sp, id0, K, perm, dec, s2, (int64_t)gp.w2, lg, flag, nflag);
        else if (gp.hc == 64) gen2_kernel<false, 64><<<blocks2, kGenTB, smem, stream>>>(g, gt, sp, id0, K, perm, dec, s2, (int64_t)gp.w2, lg, flag, nflag);
        else gen2_kernel<false, 32><<<blocks2, kGenTB, smem, stream>>>(g, gt, sp, id0, K, perm, dec, s2, (int64_t)gp.w2, lg, flag, nflag);
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
        const char* dbg = std::getenv("MAGIS_GEN_DEBUG");          // report the re-run count (syncs)
        if (dbg && std::atoi(dbg) != 0) {
            int32_t h = -1;
            cudaMemcpyAsync(&h, nflag, 4, cudaMemcpyDeviceToHost, stream);
            cudaStreamSynchronize(stream);
            std::fprintf(stderr, "magis gen: %d of %lld candidates re-run (hc %d bsm %d T2 %lld)\n", h, (long long)K,
                         gp.hc, gp.bsm, (long long)gp.T2);
            if (std::atoi(dbg) == 2) return cudaGetLastError();         // fast kernel only (timing)
        }
        // re-run of the flagged candidates (exits at once when there are none)
        gen_kernel<<<blocks1, 128, 0, stream>>>(g, gt, sp, id0, K, perm, dec, w, flag, nflag);
        return cudaGetLastError();
    }
    gen_kernel<<<blocks1, 128, 0, stream>>>(g, gt, sp, id0, K, perm, dec, w, nullptr, nullptr);
    return cudaGetLastError();
}

}  // namespace magis
