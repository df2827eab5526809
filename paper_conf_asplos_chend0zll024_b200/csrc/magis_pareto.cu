// magis_pareto.cu -- Pareto front of (peak, latency) and the BetterThan-best
// point.
//
// Four asynchronous kernels, no host synchronisation:
//   K1 chunk     : each CTA drops the points of its chunk of 1024 that one of
//                  16 pivots (each warp's minimum by (peak, lat, id) and by
//                  (lat, peak, id)) dominates -- they cannot be on the front --
//                  sorts the survivors by (peak, lat, id) in shared memory
//                  (bitonic, next power of two) and keeps the staircase
//                  (strictly decreasing latency) -- the chunk-local front.
//   K2 filter    : a chunk-front point survives iff no other chunk's front has
//                  a point dominating it (binary search on that staircase; a
//                  warp per point, a lane per other chunk).
//   K3 count     : per-chunk exclusive scan of the survivor flags; counts for
//                  the best-point queries.
//   K4 scatter   : global rank of a survivor = number of survivors with a
//                  smaller peak (binary search per chunk); write front[rank];
//                  the BetterThan-best points are rank lookups on the front.
// The result is independent of chunking (the front of a set is unique given
// the tie rule), so the per-rank fronts merged after an all-gather equal the
// single-GPU front bit for bit.
#include <algorithm>
#include <climits>
#include <cmath>

#include "magis_internal.h"

namespace magis {

constexpr int kCH = 1024;          // points per chunk
constexpr int kPB = 256;           // threads per K1 / K3 block
constexpr int kPer = kCH / kPB;    // 4 points per thread
constexpr int kCHS = kCH + 8;      // + a sentinel point at index kCH (padding of the survivor sort)
constexpr int kSmemChunk = kCHS * 26;  // pk, lt, ix (8 B each) + ord (2 B)

__device__ unsigned long long g_pareto_dummy[3];

struct PWs {
    int64_t* spk;   // [C*CH] staircase peaks
    double* slt;    // [C*CH]
    int64_t* sid;   // [C*CH]
    uint8_t* flag;  // [C*CH]
    int32_t* pref;  // [C*CH]
    int32_t* cnt;   // [C]
    int32_t* tot;   // [C]
    unsigned long long* ctr;   // [3]: cntM, cntL, front size
};

static size_t a256(size_t x) { return (x + 255) / 256 * 256; }

static PWs ws_layout(void* base, int64_t C) {
    PWs w;
    char* b = (char*)base;
    size_t o = 0, S = (size_t)C * kCH;
    w.spk = (int64_t*)(b + o);  o += a256(S * 8);
    w.slt = (double*)(b + o);   o += a256(S * 8);
    w.sid = (int64_t*)(b + o);  o += a256(S * 8);
    w.flag = (uint8_t*)(b + o); o += a256(S);
    w.pref = (int32_t*)(b + o); o += a256(S * 4);
    w.cnt = (int32_t*)(b + o);  o += a256((size_t)C * 4);
    w.tot = (int32_t*)(b + o);  o += a256((size_t)C * 4);
    w.ctr = (unsigned long long*)(b + o);
    return w;
}

int64_t pareto_workspace_size(int64_t n) {
    int64_t C = (n + kCH - 1) / kCH;
    size_t S = (size_t)C * kCH;
    return (int64_t)(a256(S * 8) * 3 + a256(S) + a256(S * 4) + a256((size_t)C * 4) * 2 + 256);
}

__device__ __forceinline__ bool key_less(long long pa, double la, long long ia, long long pb,
                                         double lb, long long ib) {
    if (pa != pb) return pa < pb;
    if (la != lb) return la < lb;
    return ia < ib;
}

__global__ void pareto_init(PWs w, int64_t* front_n, int64_t* best) {
    w.ctr[0] = 0;
    w.ctr[1] = 0;
    w.ctr[2] = 0;
    *front_n = 0;
    if (best) { best[0] = -1; best[1] = -1; }
}

__global__ void __launch_bounds__(kPB)
pareto_chunk(int64_t n, const int64_t* __restrict__ peak, const double* __restrict__ lat,
             const uint8_t* __restrict__ status, const int64_t* __restrict__ id,
             int64_t id_base, PWs w) {
    extern __shared__ __align__(16) char psm[];
    long long* pk = (long long*)psm;
    double* lt = (double*)(psm + kCHS * 8);
    long long* ix = (long long*)(psm + kCHS * 16);
    unsigned short* ord = (unsigned short*)(psm + kCHS * 24);
    __shared__ double wmin[kPB / 32];
    __shared__ int wcnt[kPB / 32 + 1];
    constexpr int kNP = 2 * (kPB / 32);   // pivots
    __shared__ long long vpk[kNP], vix[kNP];
    __shared__ double vlt[kNP];
    const int c = blockIdx.x, tid = threadIdx.x;
    const int64_t base = (int64_t)c * kCH;
    for (int j = tid; j < kCH; j += kPB) {
        const int64_t q = base + j;
        if (q < n && (!status || status[q] == 0) && (!id || id[q] >= 0)) {
            pk[j] = peak[q];
            lt[j] = lat[q];
            ix[j] = id ? id[q] : id_base + q;
        } else {
            pk[j] = LLONG_MAX;
            lt[j] = INFINITY;
            ix[j] = LLONG_MAX;
        }
    }
    if (tid == 0) { pk[kCH] = LLONG_MAX; lt[kCH] = INFINITY; ix[kCH] = LLONG_MAX; }
    __syncthreads();
    const int lane = tid & 31, wid = tid >> 5;
    // pivots: per warp the minimum by (pk, lt, ix) and by (lt, pk, ix)
    {
        long long ap = LLONG_MAX, ai = LLONG_MAX, bp = LLONG_MAX, bi = LLONG_MAX;
        double al = INFINITY, bl = INFINITY;
        for (int q = 0; q < kPer; q++) {
            const int j = tid * kPer + q;
            const long long p = pk[j], i = ix[j];
            const double l = lt[j];
            if (key_less(p, l, i, ap, al, ai)) { ap = p; al = l; ai = i; }
            if (l < bl || (l == bl && (p < bp || (p == bp && i < bi)))) { bp = p; bl = l; bi = i; }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            const long long p1 = __shfl_xor_sync(0xffffffffu, ap, o), i1 = __shfl_xor_sync(0xffffffffu, ai, o);
            const double l1 = __shfl_xor_sync(0xffffffffu, al, o);
            if (key_less(p1, l1, i1, ap, al, ai)) { ap = p1; al = l1; ai = i1; }
            const long long p2 = __shfl_xor_sync(0xffffffffu, bp, o), i2 = __shfl_xor_sync(0xffffffffu, bi, o);
            const double l2 = __shfl_xor_sync(0xffffffffu, bl, o);
            if (l2 < bl || (l2 == bl && (p2 < bp || (p2 == bp && i2 < bi)))) { bp = p2; bl = l2; bi = i2; }
        }
        if (lane == 0) {
            vpk[2 * wid] = ap; vlt[2 * wid] = al; vix[2 * wid] = ai;
            vpk[2 * wid + 1] = bp; vlt[2 * wid + 1] = bl; vix[2 * wid + 1] = bi;
        }
    }
    __syncthreads();
    // survivors: valid and dominated by no pivot (a pivot equal in (pk, lt)
    // with a smaller id also removes it: duplicates keep the smallest id)
    unsigned smask = 0;
    int ns = 0;
    for (int q = 0; q < kPer; q++) {
        const int j = tid * kPer + q;
        const long long p = pk[j], i = ix[j];
        const double l = lt[j];
        bool sv = p != LLONG_MAX;
        for (int v = 0; v < kNP && sv; v++) {
            const long long vp = vpk[v];
            const double vl = vlt[v];
            if (vp <= p && vl <= l && (vp < p || vl < l || vix[v] < i)) sv = false;
        }
        if (sv) { smask |= 1u << q; ns++; }
    }
    {
        int ki = ns;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, ki, o);
            if (lane >= o) ki += y;
        }
        if (lane == 31) wcnt[wid] = ki;
        __syncthreads();
        if (tid == 0) {
            int acc = 0;
            for (int q = 0; q < kPB / 32; q++) { const int t2 = wcnt[q]; wcnt[q] = acc; acc += t2; }
            wcnt[kPB / 32] = acc;
        }
        __syncthreads();
        int r = wcnt[wid] + ki - ns;
        for (int q = 0; q < kPer; q++)
            if (smask & (1u << q)) ord[r++] = (unsigned short)(tid * kPer + q);
    }
    const int m = wcnt[kPB / 32];
    int M = 2;
    while (M < m) M <<= 1;
    for (int j = m + tid; j < kCH; j += kPB) ord[j] = (unsigned short)kCH;   // sentinels sort last
    __syncthreads();
    // bitonic sort of ord[0, M) by (pk, lt, ix)
    for (int size = 2; size <= M; size <<= 1) {
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int t = tid; t < M / 2; t += kPB) {
                const int i = 2 * t - (t & (stride - 1));
                const int j = i + stride;
                const bool asc = ((i & size) == 0);
                const int a = ord[i], b = ord[j];
                const bool lt_ab = key_less(pk[b], lt[b], ix[b], pk[a], lt[a], ix[a]);  // b < a
                if (lt_ab == asc) { ord[i] = (unsigned short)b; ord[j] = (unsigned short)a; }
            }
            __syncthreads();
        }
    }
    // staircase: keep sorted item j iff valid and lat < min lat of all items before it
    double vals[kPer];
    double tmin = INFINITY;
#pragma unroll
    for (int q = 0; q < kPer; q++) {
        vals[q] = lt[ord[tid * kPer + q]];
        tmin = fmin(tmin, vals[q]);
    }
    // exclusive min-scan of tmin over threads
    double inc = tmin;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        double y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc = fmin(inc, y);
    }
    if (lane == 31) wmin[wid] = inc;
    __syncthreads();
    double wex = INFINITY;
    for (int q = 0; q < wid; q++) wex = fmin(wex, wmin[q]);
    double ex = __shfl_up_sync(0xffffffffu, inc, 1);
    if (lane == 0) ex = INFINITY;
    double run = fmin(wex, ex);
    unsigned keepmask = 0;
    int kept = 0;
#pragma unroll
    for (int q = 0; q < kPer; q++) {
        const int j = ord[tid * kPer + q];
        const bool valid = pk[j] != LLONG_MAX;
        if (valid && vals[q] < run) { keepmask |= 1u << q; kept++; }
        run = fmin(run, vals[q]);
    }
    // exclusive scan of kept counts
    int ki = kept;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(0xffffffffu, ki, o);
        if (lane >= o) ki += y;
    }
    if (lane == 31) wcnt[wid] = ki;
    __syncthreads();
    if (tid == 0) {
        int acc = 0;
        for (int q = 0; q < kPB / 32; q++) { int t2 = wcnt[q]; wcnt[q] = acc; acc += t2; }
        wcnt[kPB / 32] = acc;
    }
    __syncthreads();
    int r = wcnt[wid] + ki - kept;
#pragma unroll
    for (int q = 0; q < kPer; q++) {
        if (keepmask & (1u << q)) {
            const int j = ord[tid * kPer + q];
            w.spk[base + r] = pk[j];
            w.slt[base + r] = lt[j];
            w.sid[base + r] = ix[j];
            r++;
        }
    }
    if (tid == 0) w.cnt[c] = wcnt[kPB / 32];
}

// last index j in stair c' with spk[j] <= p (or -1)
__device__ __forceinline__ int last_le(const int64_t* spk, int cnt, long long p) {
    int lo = 0, hi = cnt;   // first index with spk > p
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (spk[mid] <= p) lo = mid + 1; else hi = mid;
    }
    return lo - 1;
}

// first index j with spk[j] >= p (or cnt)
__device__ __forceinline__ int first_ge(const int64_t* spk, int cnt, long long p) {
    int lo = 0, hi = cnt;
    while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (spk[mid] < p) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// one CTA per chunk, one warp per chunk-front point, one lane per other chunk
__global__ void pareto_filter(int64_t C, PWs w) {
    const int64_t c = blockIdx.x;
    const int lane = threadIdx.x & 31, nwarp = blockDim.x >> 5;
    const int cnt = w.cnt[c];
    for (int i = threadIdx.x >> 5; i < cnt; i += nwarp) {
        const int64_t s = c * kCH + i;
        const long long p = w.spk[s];
        const double l = w.slt[s];
        const long long myid = w.sid[s];
        bool dom = false;
        for (int64_t c2 = lane; c2 < C && !dom; c2 += 32) {
            if (c2 == c) continue;
            const int64_t b2 = c2 * kCH;
            const int j = last_le(w.spk + b2, w.cnt[c2], p);
            if (j < 0) continue;
            const double l2 = w.slt[b2 + j];
            const long long p2 = w.spk[b2 + j];
            if (l2 < l) dom = true;
            else if (l2 == l) {
                if (p2 < p) dom = true;
                else if (w.sid[b2 + j] < myid) dom = true;   // exact duplicate: smaller id wins
            }
        }
        dom = __any_sync(0xffffffffu, dom);
        if (lane == 0) w.flag[s] = dom ? 0 : 1;
    }
}

__global__ void __launch_bounds__(kPB)
pareto_count(PWs w, int64_t mem_limit, double lat_limit) {
    __shared__ int wcnt[kPB / 32 + 1];
    const int c = blockIdx.x, tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int64_t base = (int64_t)c * kCH;
    const int cnt = w.cnt[c];
    int f[kPer];
    int kept = 0, cm = 0, cl = 0;
#pragma unroll
    for (int q = 0; q < kPer; q++) {
        const int i = tid * kPer + q;
        f[q] = (i < cnt) ? w.flag[base + i] : 0;
        kept += f[q];
        if (f[q]) {
            if (mem_limit >= 0 && w.spk[base + i] <= mem_limit) cm++;
            if (lat_limit >= 0.0 && w.slt[base + i] > lat_limit) cl++;
        }
    }
    int ki = kept;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(0xffffffffu, ki, o);
        if (lane >= o) ki += y;
    }
    if (lane == 31) wcnt[wid] = ki;
    __syncthreads();
    if (tid == 0) {
        int acc = 0;
        for (int q = 0; q < kPB / 32; q++) { int t2 = wcnt[q]; wcnt[q] = acc; acc += t2; }
        wcnt[kPB / 32] = acc;
    }
    __syncthreads();
    int r = wcnt[wid] + ki - kept;
#pragma unroll
    for (int q = 0; q < kPer; q++) {
        const int i = tid * kPer + q;
        if (i < cnt) w.pref[base + i] = r;
        r += f[q];
    }
    if (tid == 0) {
        w.tot[c] = wcnt[kPB / 32];
        atomicAdd(&w.ctr[2], (unsigned long long)wcnt[kPB / 32]);
    }
    for (int o = 16; o > 0; o >>= 1) {
        cm += __shfl_xor_sync(0xffffffffu, cm, o);
        cl += __shfl_xor_sync(0xffffffffu, cl, o);
    }
    if (lane == 0 && cm) atomicAdd(&w.ctr[0], (unsigned long long)cm);
    if (lane == 0 && cl) atomicAdd(&w.ctr[1], (unsigned long long)cl);
}

// one CTA per chunk, one warp per surviving point, one lane per chunk of the rank sum
__global__ void pareto_scatter(int64_t C, PWs w, int64_t cap, int64_t* front_id,
                               int64_t* front_peak, double* front_lat, int64_t* front_n,
                               int64_t mem_limit, double lat_limit, int64_t* best) {
    const int64_t c = blockIdx.x;
    const int lane = threadIdx.x & 31, nwarp = blockDim.x >> 5;
    const int64_t nf = (int64_t)w.ctr[2];              // total front size (pareto_count)
    if (c == 0 && threadIdx.x == 0) *front_n = nf;
    const int cnt = w.cnt[c];
    for (int i = threadIdx.x >> 5; i < cnt; i += nwarp) {
        const int64_t s = c * kCH + i;
        if (!w.flag[s]) continue;
        const long long p = w.spk[s];
        long long rank = 0;
        for (int64_t c2 = lane; c2 < C; c2 += 32) {
            const int64_t b2 = c2 * kCH;
            const int cnt2 = w.cnt[c2];
            const int j = (c2 == c) ? i : first_ge(w.spk + b2, cnt2, p);
            rank += (j < cnt2) ? w.pref[b2 + j] : w.tot[c2];
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) rank += __shfl_xor_sync(0xffffffffu, rank, o);
        if (lane != 0) continue;
        if (rank < cap) {
            front_id[rank] = w.sid[s];
            front_peak[rank] = p;
            front_lat[rank] = w.slt[s];
        }
        if (best) {
            if (mem_limit >= 0) {
                const int64_t cm = (int64_t)w.ctr[0];
                if (rank == (cm > 0 ? cm - 1 : 0)) best[0] = w.sid[s];
            }
            if (lat_limit >= 0.0) {
                const int64_t cl = (int64_t)w.ctr[1];
                if (rank == (cl < nf ? cl : nf - 1)) best[1] = w.sid[s];
            }
        }
    }
}

// fill front entries [front_n, cap) with padding (id -1, peak -1, lat +inf) so a
// padded front can be all-gathered and merged directly (ids < 0 are ignored).
__global__ void pareto_pad(const unsigned long long* nfp, int64_t cap, int64_t* front_id,
                           int64_t* front_peak, double* front_lat) {
    const int64_t nf = nfp ? (int64_t)*nfp : 0;
    for (int64_t r = nf + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < cap;
         r += (int64_t)gridDim.x * blockDim.x) {
        front_id[r] = -1;
        front_peak[r] = -1;
        front_lat[r] = INFINITY;
    }
}

cudaError_t pareto_launch(int64_t n, const int64_t* peak, const double* lat,
                          const uint8_t* status, const int64_t* id, int64_t id_base,
                          int64_t cap, int64_t* front_id, int64_t* front_peak,
                          double* front_lat, int64_t* front_n, int64_t mem_limit,
                          double lat_limit, int64_t* best, void* ws, cudaStream_t stream) {
    const int64_t C = (n + kCH - 1) / kCH;
    PWs w = ws_layout(ws, C);
    if (n == 0) {
        // no points: front_n = 0, best = -1 (the workspace may be NULL)
        PWs w0{};
        unsigned long long* dp = nullptr;
        cudaError_t e = cudaGetSymbolAddress((void**)&dp, g_pareto_dummy);
        if (e != cudaSuccess) return e;
        w0.ctr = dp;
        pareto_init<<<1, 1, 0, stream>>>(w0, front_n, best);
        if (cap > 0)
            pareto_pad<<<(unsigned)std::min<int64_t>((cap + 255) / 256, 1024), 256, 0, stream>>>(
                nullptr, cap, front_id, front_peak, front_lat);
        return cudaGetLastError();
    }
    {
        cudaError_t e = cudaFuncSetAttribute(pareto_chunk, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             kSmemChunk);
        if (e != cudaSuccess) return e;
    }
    pareto_init<<<1, 1, 0, stream>>>(w, front_n, best);
    pareto_chunk<<<(unsigned)C, kPB, kSmemChunk, stream>>>(n, peak, lat, status, id, id_base, w);
    pareto_filter<<<(unsigned)C, 256, 0, stream>>>(C, w);
    pareto_count<<<(unsigned)C, kPB, 0, stream>>>(w, mem_limit, lat_limit);
    pareto_scatter<<<(unsigned)C, 256, 0, stream>>>(C, w, cap, front_id, front_peak, front_lat, front_n,
                                               mem_limit, lat_limit, best);
    if (cap > 0)
        pareto_pad<<<(unsigned)std::min<int64_t>((cap + 255) / 256, 1024), 256, 0, stream>>>(
            w.ctr + 2, cap, front_id, front_peak, front_lat);
    return cudaGetLastError();
}

}  // namespace magis
