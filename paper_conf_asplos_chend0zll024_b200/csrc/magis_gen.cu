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
#include <climits>

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
            heap_push(w, t, nh, ((rnd(seed, k, S_KEY, (uint64_t)v) >> 32) << 32) | (uint32_t)v);
    while (nh > 0) {
        const uint64_t x = heap_pop(w, t, nh);
        const int32_t u = (int32_t)(x & 0xffffffffu);
        w.B(out0 + m, t) = u;
        m++;
        for (int32_t e = gt.succ_ptr[u]; e < gt.succ_ptr[u + 1]; e++) {
            const int32_t s = gt.succ[e];
            if (s >= hi) continue;
            if (--w.I(s, t) == 0)
                heap_push(w, t, nh, ((rnd(seed, k, S_KEY, (uint64_t)s) >> 32) << 32) | (uint32_t)s);
        }
    }
    (void)g;
}

__global__ void __launch_bounds__(128)
gen_kernel(DevGraph g, GenTables gt, GenSpec sp, uint64_t id0, int64_t K, int32_t* __restrict__ perms,
           uint8_t* __restrict__ decs, Scratch w) {
    const int32_t n = g.n, R = g.R, NT = g.NT;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t kk = t; kk < K; kk += w.T) {
        const uint64_t k = id0 + (uint64_t)kk;
        const uint64_t seed = sp.seed;
        int32_t* perm = perms + kk * (int64_t)NT;
        uint8_t* dec = decs + kk * (int64_t)(R ? R : 1);
        const uint32_t fam = (uint32_t)(rnd(seed, k, S_FAM, 0) % 100u);
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

}  // namespace

size_t gen_scratch_bytes(const DevGraph& g, int64_t T) {
    return (size_t)T * ((size_t)g.n * (4 + 8 + 4 + 4) + (size_t)2 * (g.R ? g.R : 1) * 8) + 256;
}

int64_t gen_threads(int device, const DevGraph& g, int64_t K) {
    cudaDeviceProp p;
    const int64_t base = (cudaGetDeviceProperties(&p, device) == cudaSuccess ? p.multiProcessorCount : 148) * 256LL;
    // up to one thread per candidate, within a scratch budget of 16 GiB
    const int64_t per = (int64_t)gen_scratch_bytes(g, 1);
    const int64_t cap = std::max<int64_t>(base, (16LL << 30) / std::max<int64_t>(per, 1));
    return std::max<int64_t>(base, std::min<int64_t>(K, cap)) / 128 * 128;
}

cudaError_t gen_launch(const DevGraph& g, const GenTables& gt, const GenSpec& sp, uint64_t id0, int64_t K,
                       int32_t* perm, uint8_t* dec, void* scratch, int64_t T, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    Scratch w;
    char* b = (char*)scratch;
    w.T = T;
    w.n = g.n;
    w.no = 2 * (g.R ? g.R : 1);
    w.heap = (uint64_t*)b;   b += (size_t)g.n * 8 * T;
    w.opt = (int64_t*)b;     b += (size_t)2 * (g.R ? g.R : 1) * 8 * T;
    w.indeg = (int32_t*)b;   b += (size_t)g.n * 4 * T;
    w.base = (int32_t*)b;    b += (size_t)g.n * 4 * T;
    w.posb = (int32_t*)b;
    const int64_t threads = std::min<int64_t>(T, K);
    const unsigned blocks = (unsigned)((threads + 127) / 128);
    // the kernel strides over candidates by w.T; with fewer threads than T the
    // surplus threads see kk >= K and exit
    gen_kernel<<<blocks, 128, 0, stream>>>(g, gt, sp, id0, K, perm, dec, w);
    return cudaGetLastError();
}

}  // namespace magis
