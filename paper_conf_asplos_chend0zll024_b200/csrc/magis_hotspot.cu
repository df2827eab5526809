// magis_hotspot.cu -- memory hot-spots and F-Trans heat / score of candidate
// schedules.
//
//   H: the tensors live at some step where M_i = M_peak.  Over the
//   original graph (reading H1) a live clone A' or Load of t_r stands for
//   t_r; a Store holds no device bytes and does not count.
//   heat(v)  = sum of |w| over w in H and T.des(v)                 Eq. 3
//   score(v) = (1 - 1/nsplit) heat(v) - sum of |u| over the inputs of
//              T.des(v) that are not in H                           Eq. 4
//
// T is the dominator tree of G (built once at graph load).  Two facts make
// this data-parallel:
//  * T.des(v) is the preorder range [tin(v), tout(v)), so heat is a
//    difference of prefix sums of the hot sizes laid out in preorder;
//  * the inputs of T.des(v) are exactly pred(v): for an edge u -> w, every
//    strict dominator of w dominates u or is u, so an edge entering des(v)
//    from outside must end at v itself.
// H itself: with the per-step curve M (a block scan of alloc - free, as in
// a5-a7) and c(i) = number of peak steps before i, tensor u (live on
// [pos(u), last(u)]) is hot iff c(last(u) + 1) > c(pos(u)).
//
// One CTA per candidate (a query on a few selected schedules, not the batch
// hot loop); per-candidate state in a per-CTA global slice.
#include <climits>

#include "magis_internal.h"

namespace magis {

namespace {

constexpr int kHB = 512;
constexpr int kHW = kHB / 32;

struct HsLayout {
    size_t pos, last, A, Fr, M, pc, hs, hp, dec, total;
};

size_t al16(size_t x) { return (x + 15) / 16 * 16; }

HsLayout hs_layout(int32_t NT, int32_t n, int32_t R) {
    HsLayout L{};
    size_t o = 0;
    L.pos = o;  o += al16((size_t)NT * 4);
    L.last = o; o += al16((size_t)NT * 4);
    L.A = o;    o += al16((size_t)NT * 8);
    L.Fr = o;   o += al16((size_t)NT * 8);
    L.M = o;    o += al16((size_t)NT * 8);
    L.pc = o;   o += al16((size_t)(NT + 1) * 4);
    L.hs = o;   o += al16((size_t)NT);
    L.hp = o;   o += al16((size_t)(n + 1) * 8);
    L.dec = o;  o += al16((size_t)(R > 0 ? R : 1));
    L.total = (o + 255) / 256 * 256;
    return L;
}

__device__ __forceinline__ bool gate_ok(int32_t gate, const uint8_t* dec_s) {
    return gate < 0 || dec_s[gate >> 2] == (uint8_t)(gate & 3);
}

// block-wide exclusive scan of one value per thread (+ total)
template <typename T>
__device__ __forceinline__ T bscan(T x, T* red, T& total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    T inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) red[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        const T w = lane < kHW ? red[lane] : T(0);
        T wi = w;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const T y = __shfl_up_sync(0xffffffffu, wi, o);
            if (lane >= o) wi += y;
        }
        if (lane < kHW) red[lane] = wi - w;
        if (lane == kHW - 1) red[kHW] = wi;
    }
    __syncthreads();
    const T ex = red[wid] + inc - x;
    total = red[kHW];
    __syncthreads();
    return ex;
}

__device__ __forceinline__ long long bmax(long long x, long long* red) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x = max(x, __shfl_xor_sync(0xffffffffu, x, o));
    if (lane == 0) red[wid] = x;
    __syncthreads();
    if (wid == 0) {
        long long w = lane < kHW ? red[lane] : LLONG_MIN;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) w = max(w, __shfl_xor_sync(0xffffffffu, w, o));
        if (lane == 0) red[kHW] = w;
    }
    __syncthreads();
    const long long r = red[kHW];
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(kHB)
hotspot_kernel(DevGraph g, int64_t K, const int32_t* __restrict__ perm, const uint8_t* __restrict__ dec,
               double frac, uint8_t* __restrict__ out_status, int64_t* __restrict__ out_peak,
               uint8_t* __restrict__ out_hot, int64_t* __restrict__ out_heat, double* __restrict__ out_score,
               char* __restrict__ ws, HsLayout L) {
    __shared__ long long red_ll[kHW + 1];
    __shared__ int red_i[kHW + 1];
    __shared__ int s_flags;
    char* st = ws + (size_t)blockIdx.x * L.total;
    int32_t* pos = (int32_t*)(st + L.pos);
    int32_t* last = (int32_t*)(st + L.last);
    long long* A = (long long*)(st + L.A);
    long long* Fr = (long long*)(st + L.Fr);
    long long* M = (long long*)(st + L.M);
    int32_t* pc = (int32_t*)(st + L.pc);
    uint8_t* hs = (uint8_t*)(st + L.hs);
    long long* hp = (long long*)(st + L.hp);
    uint8_t* dec_s = (uint8_t*)(st + L.dec);
    const int tid = threadIdx.x;
    const int32_t NT = g.NT, R = g.R, n = g.n;
    const int32_t Lc = (NT + kHB - 1) / kHB;
    const int32_t Ln = (n + kHB - 1) / kHB;

    for (int64_t k = blockIdx.x; k < K; k += gridDim.x) {
        const int32_t* Pk = perm + k * (int64_t)NT;
        uint8_t* hot = out_hot + k * (int64_t)n;
        if (tid == 0) s_flags = 0;
        // ---- decisions, inverse permutation, validity, last use (a2-a4) ------
        int bad = 0;
        for (int32_t r = tid; r < R; r += kHB) {
            const uint8_t d = dec[k * (int64_t)R + r];
            dec_s[r] = d;
            bad |= ((d > 2) | ((d == 1) & !(g.rflag[r] & kRHasInput))) ? MAGIS_ST_BAD_DEC : 0;
        }
        for (int32_t v = tid; v < NT; v += kHB) pos[v] = -1;
        __syncthreads();
        for (int32_t i = tid; i < NT; i += kHB) {
            const int32_t v = Pk[i];
            if ((uint32_t)v < (uint32_t)NT) pos[v] = i; else bad |= MAGIS_ST_NOT_PERM;
        }
        __syncthreads();
        for (int32_t v = tid; v < NT; v += kHB) {
            const int32_t p = pos[v];
            if (p < 0) { bad |= MAGIS_ST_NOT_PERM; continue; }
            if (!gate_ok(g.ngate[v], dec_s)) { last[v] = -1; continue; }   // inactive: no tensor
            int32_t lst = p;
            for (int32_t e = g.cons_ptr[v]; e < g.cons_ptr[v + 1]; e++) {
                const int2 ce = g.cons_ent[e];
                if (!gate_ok(ce.y, dec_s)) continue;
                const int32_t q = pos[ce.x];
                if (q <= p) bad |= MAGIS_ST_EDGE;
                lst = max(lst, q);
            }
            if (g.nflag[v] & kFlagOutput) lst = NT - 1;
            last[v] = lst;
        }
        if (bad) atomicOr(&s_flags, bad);
        __syncthreads();
        int status = s_flags;
        if (status & (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC)) status &= (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC);
        if (status) {
            if (tid == 0) { out_status[k] = (uint8_t)status; out_peak[k] = -1; }
            for (int32_t v = tid; v < n; v += kHB) {
                hot[v] = 0;
                if (out_heat) out_heat[k * (int64_t)n + v] = 0;
                if (out_score) out_score[k * (int64_t)n + v] = 0.0;
            }
            __syncthreads();
            continue;
        }
        // ---- alloc / free per step (a5) ---------------------------------------
        for (int32_t v = tid; v < NT; v += kHB) {
            const int32_t p = pos[v];
            if (last[v] < 0) { A[p] = 0; Fr[p] = 0; continue; }
            const long long sz = g.size[v];
            long long f = (last[v] == p) ? sz : 0;
            for (int32_t e = g.in_ptr[v]; e < g.in_ptr[v + 1]; e++) {
                const int2 ie = g.in_ent[e];
                if (gate_ok(ie.y, dec_s) && last[ie.x] == p) f += g.size[ie.x];
            }
            A[p] = sz;
            Fr[p] = f;
        }
        __syncthreads();
        // ---- curve M_i and the peak (a6-a7) ------------------------------------
        const int32_t lo = tid * Lc, hi = min(lo + Lc, NT);
        long long s = 0;
        for (int32_t i = lo; i < hi; i++) s += A[i] - Fr[i];
        long long tot;
        long long run = bscan<long long>(s, red_ll, tot);
        long long mx = LLONG_MIN;
        for (int32_t i = lo; i < hi; i++) {
            const long long m = run + A[i];
            M[i] = m;
            mx = max(mx, m);
            run = m - Fr[i];
        }
        const long long peak = bmax(mx, red_ll);
        // ---- peak steps: c(i) = number of peak steps before i -------------------
        int cnt = 0;
        for (int32_t i = lo; i < hi; i++) cnt += M[i] == peak;
        int ctot;
        int c0 = bscan<int>(cnt, red_i, ctot);
        for (int32_t i = lo; i < hi; i++) {
            pc[i] = c0;
            c0 += M[i] == peak;
        }
        if (tid == 0) pc[NT] = ctot;
        __syncthreads();
        // ---- H over the super-graph, then over G (reading H1) -------------------
        for (int32_t v = tid; v < NT; v += kHB) {
            const int32_t p = pos[v], l = last[v];
            hs[v] = (l >= 0 && pc[l + 1] > pc[p]) ? 1 : 0;
        }
        __syncthreads();
        for (int32_t v = tid; v < n; v += kHB) {
            uint8_t h = hs[v];
            hot[v] = h;
        }
        __syncthreads();
        for (int32_t r = tid; r < R; r += kHB)
            if (hs[n + 3 * r] | hs[n + 3 * r + 2]) hot[g.elig[r]] = 1;
        __syncthreads();
        if (out_heat || out_score) {
            // ---- heat: hot sizes in dominator-tree preorder, prefix sums -------
            for (int32_t v = tid; v < n; v += kHB) hp[g.dtin[v]] = hot[v] ? (long long)g.size[v] : 0ll;
            __syncthreads();
            const int32_t a = tid * Ln, b = min(a + Ln, n);
            long long hsum = 0;
            for (int32_t i = a; i < b; i++) hsum += hp[i];
            long long htot;
            long long hr = bscan<long long>(hsum, red_ll, htot);
            for (int32_t i = a; i < b; i++) {          // in place: hp[i] = sum before i
                const long long x = hp[i];
                hp[i] = hr;
                hr += x;
            }
            if (tid == 0) hp[n] = htot;
            __syncthreads();
            for (int32_t v = tid; v < n; v += kHB) {
                const long long h = hp[g.dtout[v]] - hp[g.dtin[v]];
                if (out_heat) out_heat[k * (int64_t)n + v] = h;
                if (out_score) {
                    long long inp = 0;                     // inputs of T.des(v) = pred(v)
                    for (int32_t e = g.pred_ptr[v]; e < g.pred_ptr[v + 1]; e++) {
                        const int32_t u = g.pred[e];
                        if (!hot[u]) inp += g.size[u];
                    }
                    out_score[k * (int64_t)n + v] = __dsub_rn(__dmul_rn(frac, (double)h), (double)inp);
                }
            }
        }
        if (tid == 0) { out_status[k] = 0; out_peak[k] = peak; }
        __syncthreads();
    }
}

}  // namespace

size_t hotspot_ws_per_cta(const DevGraph& g) { return hs_layout(g.NT, g.n, g.R).total; }

cudaError_t hotspot_launch(const DevGraph& g, int grid, void* ws, int64_t K, const int32_t* perm, const uint8_t* dec,
                           int32_t nsplit, uint8_t* status, int64_t* peak, uint8_t* hot, int64_t* heat,
                           double* score, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    const HsLayout L = hs_layout(g.NT, g.n, g.R);
    const double frac = 1.0 - 1.0 / (double)nsplit;
    const int gr = (int)std::min<int64_t>(grid, K);
    hotspot_kernel<<<gr, kHB, 0, stream>>>(g, K, perm, dec, frac, status, peak, hot, heat, score,
                                           (char*)ws, L);
    return cudaGetLastError();
}

}  // namespace magis
