// magis_window.cu -- windowed delta evaluation of local-move candidates
// (the incremental-scheduling idea of Alg. 2,
// P:1591-1613, applied to evaluation).
//
// A local move re-orders the w steps [b, b+w) of a base schedule and keeps
// the base decisions.  Outside the window the memory curve is unchanged: for
// i < b no position changes; for i >= b+w every tensor live at i has its
// producer before i and a reader at or after i, and window readers stay
// inside the window (reading P1 lifetimes).  So
//     peak = max(max_{i<b} M_i, max over the re-ordered window, max_{i>=b+w} M_i)
// where the window part starts from the bytes carried into step b and sees
// (a) the window ops' allocations and (b) the frees of exactly the tensors the
// base frees inside the window, each now at the new position of its last
// in-window reader.  The latency re-runs the three-queue sweep (reading P7)
// over the base's swap events with the window's events moved to their new
// steps and compute-cost prefixes.  Cost is O(w + window-incident edges +
// swap events) per candidate instead of O(n_total + E).
//
// magis_base_create evaluates the base once (one CTA; a plain sequential pass
// per step -- it runs once per base) and stores the per-step profile.
#include <climits>
#include <cmath>

#include "magis_internal.h"

namespace magis {

namespace {

__device__ __forceinline__ bool gate_ok(int32_t gate, const uint8_t* dec) {
    return gate < 0 || dec[gate >> 2] == (uint8_t)(gate & 3);
}

// ---------------------------------------------------------------- base ----
// One block: pos / active / last in parallel, then thread 0 walks the steps.
__global__ void base_kernel(DevGraph g, BaseDev b, const int32_t* __restrict__ perm, const uint8_t* __restrict__ dec) {
    const int32_t NT = g.NT, R = g.R, n = g.n;
    __shared__ int st_flags;
    if (threadIdx.x == 0) st_flags = 0;
    for (int32_t r = threadIdx.x; r < R; r += blockDim.x) b.dec[r] = dec[r];
    for (int32_t x = threadIdx.x; x < 3 * R; x += blockDim.x) b.evix[x] = INT_MAX;
    for (int32_t i = threadIdx.x; i < NT; i += blockDim.x) b.pos[i] = -1;
    __syncthreads();
    int bad = 0;
    for (int32_t r = threadIdx.x; r < R; r += blockDim.x) {
        const uint8_t d = dec[r];
        bad |= (d > 2 || (d == 1 && !(g.rflag[r] & kRHasInput))) ? MAGIS_ST_BAD_DEC : 0;
    }
    for (int32_t i = threadIdx.x; i < NT; i += blockDim.x) {
        const int32_t v = perm[i];
        b.perm[i] = v;
        if ((uint32_t)v < (uint32_t)NT) b.pos[v] = i; else bad |= MAGIS_ST_NOT_PERM;
    }
    if (bad) atomicOr(&st_flags, bad);
    __syncthreads();
    bad = 0;
    for (int32_t v = threadIdx.x; v < NT; v += blockDim.x) {
        const int32_t p = b.pos[v];
        if (p < 0) { bad |= MAGIS_ST_NOT_PERM; continue; }
        const bool act = gate_ok(g.ngate[v], b.dec);
        b.active[v] = act ? 1 : 0;
        int32_t lst = p;
        if (act) {
            for (int32_t e = g.cons_ptr[v]; e < g.cons_ptr[v + 1]; e++) {
                const int2 ce = g.cons_ent[e];
                if (!gate_ok(ce.y, b.dec)) continue;
                const int32_t q = b.pos[ce.x];
                if (q <= p) bad |= MAGIS_ST_EDGE;
                lst = max(lst, q);
            }
            if (g.nflag[v] & kFlagOutput) lst = NT;      // never freed
        } else {
            lst = -1;
        }
        b.last[v] = lst;
    }
    if (bad) atomicOr(&st_flags, bad);
    __syncthreads();
    if (threadIdx.x != 0) return;
    int st = st_flags;
    if (st & (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC)) st &= (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC);
    b.hdr->status = st;
    if (st) return;
    // memory walk: carry[i] = bytes live entering step i, M_i = carry[i] + alloc_i
    long long carry = 0, pm = -1;
    double cb = 0.0;
    for (int32_t i = 0; i < NT; i++) {
        const int32_t v = b.perm[i];
        b.carry[i] = carry;
        b.pm[i] = pm;
        b.cb[i] = cb;
        long long a = 0, f = 0;
        if (b.active[v]) {
            a = g.size[v];
            if (b.last[v] == i) f += a;
            for (int32_t e = g.in_ptr[v]; e < g.in_ptr[v + 1]; e++) {
                const int2 ie = g.in_ent[e];
                if (gate_ok(ie.y, b.dec) && b.last[ie.x] == i) f += g.size[ie.x];
            }
            if (g.nflag[v] & kFlagCompute) cb += g.cost[v];
        }
        const long long M = carry + a;
        b.mstep[i] = M;
        pm = max(pm, M);
        carry = M - f;
    }
    b.carry[NT] = carry;
    b.pm[NT] = pm;
    b.cb[NT] = cb;
    long long sm = -1;
    b.sm[NT] = -1;
    for (int32_t i = NT - 1; i >= 0; i--) {
        sm = max(sm, b.mstep[i]);
        b.sm[i] = sm;
    }
    b.hdr->peak = pm;
    b.hdr->ctot = cb;
    // swap events in step order (STALL before PRODUCE at one step)
    int ne = 0;
    for (int32_t i = 0; i < NT; i++) {
        const int32_t v = b.perm[i];
        if (!b.active[v]) continue;
        if (v < n) {
            for (int32_t r = 0; r < R; r++) {
                if (b.dec[r] != 2) continue;
                for (int32_t j = g.U_ptr[r]; j < g.U_ptr[r + 1]; j++)
                    if (g.U_idx[j] == v) b.evk[ne++] = ((unsigned long long)i << 32) | ((unsigned long long)kEvStall << 24) | r;
            }
            for (int32_t r = 0; r < R; r++)
                if (b.dec[r] == 2 && g.elig[r] == v)
                    b.evk[ne++] = ((unsigned long long)i << 32) | ((unsigned long long)kEvProduce << 24) | r;
        } else {
            const int32_t o = v - n, r = o / 3, kd = o % 3;
            if (kd != 0)
                b.evk[ne++] = ((unsigned long long)i << 32) |
                              ((unsigned long long)(kd == 1 ? kEvStore : kEvLoad) << 24) | r;
        }
    }
    b.hdr->nev = ne;
    double base_lat = cb;
    if (ne) {
        double D = 0.0, Td = 0.0, Th = 0.0;
        for (int e = 0; e < ne; e++) {
            // the state before each event and the event writing each end time:
            // a window walk starts from the base's state at the window
            b.snap[3 * e] = D;
            b.snap[3 * e + 1] = Td;
            b.snap[3 * e + 2] = Th;
            const unsigned long long kk = b.evk[e];
            const uint32_t type = (uint32_t)(kk >> 24) & 0xff;
            const int32_t r = (int32_t)(kk & 0xffffff);
            const double c = b.cb[(int32_t)(kk >> 32)];
            double* en = b.endb + 3 * r;
            if (type == kEvStall) D = fmax(D, en[2] - c);
            else if (type == kEvProduce) { en[0] = c + D + g.tcost[r]; b.evix[3 * r] = e; }
            else if (type == kEvStore) { Td = fmax(Td, en[0]) + g.xfer[r]; en[1] = Td; b.evix[3 * r + 1] = e; }
            else { Th = fmax(Th, en[1]) + g.xfer[r]; en[2] = Th; b.evix[3 * r + 2] = e; }
        }
        b.snap[3 * ne] = D;
        b.snap[3 * ne + 1] = Td;
        b.snap[3 * ne + 2] = Th;
        base_lat = fmax(fmax(cb + D, Td), Th);
    }
    b.hdr->latency = base_lat;
}

// ------------------------------------------------------------- windows ----
constexpr int kWMax = 64;
constexpr int kWarpsW = 8;
constexpr int kEvWin = 128;      // swap events inside one window (per warp)

struct WarpScratch {
    int16_t newrel[kWMax];       // new window slot of the node at base step b + rel
    unsigned long long fw[kWMax];    // bytes freed after each new window slot
    unsigned long long evk[kEvWin];
    double evcb[kEvWin];
    double cw[kWMax + 1];        // compute-cost prefix over new window slots
    unsigned int seen[2];
    int nev;
};

__global__ void __launch_bounds__(kWarpsW * 32)
window_kernel(DevGraph g, BaseDev b, int64_t K, const int32_t* __restrict__ wstart,
              const int32_t* __restrict__ wlen, const int32_t* __restrict__ wperm, int32_t wmax,
              uint8_t* __restrict__ out_status, int64_t* __restrict__ out_peak, double* __restrict__ out_lat,
              double* __restrict__ endb_ws) {
    __shared__ WarpScratch wsm[kWarpsW];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    WarpScratch& W = wsm[wid];
    const int32_t NT = g.NT;
    const int64_t gw = (int64_t)blockIdx.x * kWarpsW + wid, nw = (int64_t)gridDim.x * kWarpsW;
    const uint8_t* dec = b.dec;
    for (int64_t k = gw; k < K; k += nw) {
        const int32_t b0 = wstart[k], w = wlen[k];
        int status = b.hdr->status;
        if (status == 0 && (w < 1 || w > kWMax || w > wmax || b0 < 0 || b0 + w > NT)) status = MAGIS_ST_NOT_PERM;
        if (status) {
            if (lane == 0) { out_status[k] = (uint8_t)status; out_peak[k] = -1; out_lat[k] = INFINITY; }
            continue;
        }
        if (lane < 2) W.seen[lane] = 0;
        if (lane == 0) W.nev = 0;
        for (int j = lane; j < kWMax; j += 32) W.fw[j] = 0;
        __syncwarp();
        // 1. the window entries must be a permutation of the base window's nodes
        int bad = 0;
        int32_t vj[2];
        for (int q = 0; q < 2; q++) {
            const int j = lane + 32 * q;
            vj[q] = -1;
            if (j < w) {
                const int32_t v = wperm[k * (int64_t)wmax + j];
                const int32_t bp = ((uint32_t)v < (uint32_t)NT) ? b.pos[v] : -1;
                if (bp < b0 || bp >= b0 + w) { bad = 1; continue; }
                vj[q] = v;
                const int rel = bp - b0;
                const unsigned old = atomicOr(&W.seen[rel >> 5], 1u << (rel & 31));
                if (old & (1u << (rel & 31))) bad = 1;
                W.newrel[rel] = (int16_t)j;
            }
        }
        if (__any_sync(0xffffffffu, bad)) {
            if (lane == 0) { out_status[k] = MAGIS_ST_NOT_PERM; out_peak[k] = -1; out_lat[k] = INFINITY; }
            __syncwarp();
            continue;
        }
        __syncwarp();
        // 2. validity of edges inside the window; 3. allocations and compute costs
        long long a_j[2] = {0, 0};
        double c_j[2] = {0.0, 0.0};
        for (int q = 0; q < 2; q++) {
            const int j = lane + 32 * q;
            if (j >= w) continue;
            const int32_t v = vj[q];
            if (!b.active[v]) continue;
            for (int32_t e = g.in_ptr[v]; e < g.in_ptr[v + 1]; e++) {
                const int2 ie = g.in_ent[e];
                if (!gate_ok(ie.y, dec)) continue;
                const int32_t bp = b.pos[ie.x];
                if (bp >= b0 && bp < b0 + w && W.newrel[bp - b0] >= j) bad = 1;
            }
            a_j[q] = g.size[v];
            if (g.nflag[v] & kFlagCompute) c_j[q] = g.cost[v];
        }
        if (__any_sync(0xffffffffu, bad)) {
            if (lane == 0) { out_status[k] = MAGIS_ST_EDGE; out_peak[k] = -1; out_lat[k] = INFINITY; }
            __syncwarp();
            continue;
        }
        // 4. frees: the tensors the base frees at a window step, now after the
        //    new slot of their last in-window reader (or their own slot)
        for (int q = 0; q < 2; q++) {
            const int rel = lane + 32 * q;
            if (rel >= w) continue;
            const int32_t s = b0 + rel;
            const int32_t x = b.perm[s];
            if (!b.active[x]) continue;
            if (b.last[x] == s)                                     // no reader: freed after its own step
                atomicAdd(&W.fw[W.newrel[rel]], (unsigned long long)g.size[x]);
            for (int32_t e = g.in_ptr[x]; e < g.in_ptr[x + 1]; e++) {
                const int2 ie = g.in_ent[e];
                const int32_t u = ie.x;
                if (!gate_ok(ie.y, dec) || b.last[u] != s) continue;
                int nf = -1;
                for (int32_t f = g.cons_ptr[u]; f < g.cons_ptr[u + 1]; f++) {
                    const int2 ce = g.cons_ent[f];
                    if (!gate_ok(ce.y, dec)) continue;
                    const int32_t bp = b.pos[ce.x];
                    if (bp >= b0 && bp < b0 + w) nf = max(nf, (int)W.newrel[bp - b0]);
                }
                atomicAdd(&W.fw[nf], (unsigned long long)g.size[u]);
            }
        }
        __syncwarp();
        // 5. window memory curve: carry + alloc prefix - free prefix (new order)
        // slots are j = lane and j = lane + 32: (sum, max-prefix) monoid scan of
        // the first 32, then of the second 32 offset by the first half's sum
        const long long d0 = a_j[0] - (long long)(lane < w ? W.fw[lane] : 0);
        const long long d1 = a_j[1] - (long long)(lane + 32 < w ? W.fw[lane + 32] : 0);
        long long inc0 = d0, mx0 = a_j[0];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long ps = __shfl_up_sync(0xffffffffu, inc0, o);
            const long long pm = __shfl_up_sync(0xffffffffu, mx0, o);
            if (lane >= o) { mx0 = max(pm, ps + mx0); inc0 = ps + inc0; }
        }
        const long long tot0 = __shfl_sync(0xffffffffu, inc0, 31);
        long long wmax_l = (lane < w) ? mx0 : LLONG_MIN / 2;
        long long inc1 = d1, mx1 = a_j[1];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const long long ps = __shfl_up_sync(0xffffffffu, inc1, o);
            const long long pm = __shfl_up_sync(0xffffffffu, mx1, o);
            if (lane >= o) { mx1 = max(pm, ps + mx1); inc1 = ps + inc1; }
        }
        if (lane + 32 < w) wmax_l = max(wmax_l, tot0 + mx1);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) wmax_l = max(wmax_l, __shfl_xor_sync(0xffffffffu, wmax_l, o));
        const long long wpk = b.carry[b0] + wmax_l;
        const long long peak = max(max(b.pm[b0], wpk), b.sm[b0 + w]);
        // 6. latency
        double lat = b.hdr->latency;
        if (b.hdr->nev > 0) {
            // compute-cost prefix over the new window slots
            double ci0 = c_j[0], ci1 = c_j[1];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const double p0 = __shfl_up_sync(0xffffffffu, ci0, o);
                const double p1 = __shfl_up_sync(0xffffffffu, ci1, o);
                if (lane >= o) { ci0 += p0; ci1 += p1; }
            }
            const double t0 = __shfl_sync(0xffffffffu, ci0, 31);
            W.cw[lane] = ci0 - c_j[0];
            W.cw[lane + 32] = t0 + ci1 - c_j[1];
            __syncwarp();
            // base events inside the window move to their new steps
            const unsigned long long* ev = b.evk;
            const int ne = b.hdr->nev;
            int e0 = 0, e1 = ne;                // first event at step >= b0, first at step >= b0 + w
            {
                int lo = 0, hi = ne;
                while (lo < hi) { int mid = (lo + hi) >> 1; if ((int32_t)(ev[mid] >> 32) < b0) lo = mid + 1; else hi = mid; }
                e0 = lo;
                lo = e0; hi = ne;
                while (lo < hi) { int mid = (lo + hi) >> 1; if ((int32_t)(ev[mid] >> 32) < b0 + w) lo = mid + 1; else hi = mid; }
                e1 = lo;
            }
            const int nin = e1 - e0;
            const bool buf = nin <= kEvWin;
            // no swap event inside the window: every event keeps its step and
            // its compute-cost prefix (the window holds the same ops), so the
            // walk would repeat the base's arithmetic exactly -- the latency is
            // the base's, bit for bit
            if (nin > 0) {
                if (buf) {
                    for (int q = lane; q < nin; q += 32) {
                        const unsigned long long kk = ev[e0 + q];
                        const int32_t rel = (int32_t)(kk >> 32) - b0;
                        const int32_t ns = W.newrel[rel];
                        W.evk[q] = ((unsigned long long)(b0 + ns) << 32) | (kk & 0xffffffffull);
                        W.evcb[q] = b.cb[b0] + W.cw[ns];
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    if (buf) {
                        // insertion sort of the window's events by (new step, type, r)
                        for (int i = 1; i < nin; i++) {
                            const unsigned long long x = W.evk[i];
                            const double cx = W.evcb[i];
                            int j = i - 1;
                            while (j >= 0 && W.evk[j] > x) { W.evk[j + 1] = W.evk[j]; W.evcb[j + 1] = W.evcb[j]; j--; }
                            W.evk[j + 1] = x;
                            W.evcb[j + 1] = cx;
                        }
                    }
                    // the walk starts at the window from the base's state there:
                    // an end time written before the window is the base's
                    // (read-through via evix), later ones are written by this walk
                    double* en = endb_ws + (size_t)gw * 3 * g.R;
                    double D = b.snap[3 * e0], Td = b.snap[3 * e0 + 1], Th = b.snap[3 * e0 + 2];
                    auto rd = [&](int32_t x) { return b.evix[x] < e0 ? b.endb[x] : en[x]; };
                    unsigned long long prev = 0;
                    bool same = false;                  // the walk rejoined the base: its latency
                    for (int e = e0; e < ne; e++) {
                        if (e == e1) {
                            // past the window: if the state and every end time the
                            // window wrote equal the base's, the rest of the walk
                            // repeats the base's arithmetic exactly
                            same = D == b.snap[3 * e1] && Td == b.snap[3 * e1 + 1] && Th == b.snap[3 * e1 + 2];
                            for (int q = e0; q < e1 && same; q++) {
                                const unsigned long long k0 = ev[q];
                                const uint32_t ty = (uint32_t)(k0 >> 24) & 0xff;
                                if (ty == kEvStall) continue;
                                const int32_t x = 3 * (int32_t)(k0 & 0xffffff) +
                                                  (ty == kEvProduce ? 0 : ty == kEvStore ? 1 : 2);
                                same = en[x] == b.endb[x];
                            }
                            if (same) break;
                        }
                        unsigned long long kk;
                        double c;
                        if (e < e0 || e >= e1) {
                            kk = ev[e];
                            c = b.cb[(int32_t)(kk >> 32)];
                        } else if (buf) {
                            kk = W.evk[e - e0];
                            c = W.evcb[e - e0];
                        } else {
                            // many events in the window: select the next smallest re-keyed event
                            unsigned long long best = ~0ull;
                            for (int q = e0; q < e1; q++) {
                                const unsigned long long k0 = ev[q];
                                const unsigned long long kq =
                                    ((unsigned long long)(b0 + W.newrel[(int32_t)(k0 >> 32) - b0]) << 32) | (k0 & 0xffffffffull);
                                if (kq > prev || (e == e0 && kq >= prev)) best = kq < best ? kq : best;
                            }
                            kk = best;
                            prev = best;
                            c = b.cb[b0] + W.cw[(int32_t)(kk >> 32) - b0];
                        }
                        const uint32_t type = (uint32_t)(kk >> 24) & 0xff;
                        const int32_t r = (int32_t)(kk & 0xffffff);
                        double* er = en + 3 * r;
                        if (type == kEvStall) D = fmax(D, rd(3 * r + 2) - c);
                        else if (type == kEvProduce) er[0] = c + D + g.tcost[r];
                        else if (type == kEvStore) { Td = fmax(Td, rd(3 * r)) + g.xfer[r]; er[1] = Td; }
                        else { Th = fmax(Th, rd(3 * r + 1)) + g.xfer[r]; er[2] = Th; }
                    }
                    W.cw[kWMax] = same ? b.hdr->latency : fmax(fmax(b.hdr->ctot + D, Td), Th);
                }
                __syncwarp();
                lat = W.cw[kWMax];
            }
        }
        if (lane == 0) {
            out_status[k] = 0;
            out_peak[k] = peak;
            out_lat[k] = lat;
        }
        __syncwarp();
    }
}

}  // namespace

size_t base_bytes(const DevGraph& g) {
    const size_t NT = (size_t)g.NT;
    return 256 + NT * 4 * 3 + NT + (NT + 1) * 8 * 4 + NT * 8 + (size_t)(g.R ? g.R : 1) * (1 + 24 + 12) +
           (size_t)(g.max_events + 1) * (8 + 24) + 64 * 8;
}

BaseDev base_layout(const DevGraph& g, void* mem) {
    BaseDev b{};
    char* p = (char*)mem;
    auto take = [&](size_t bytes) { char* q = p; p += (bytes + 15) / 16 * 16; return q; };
    const size_t NT = (size_t)g.NT;
    b.hdr = (BaseHdr*)take(sizeof(BaseHdr));
    b.perm = (int32_t*)take(NT * 4);
    b.pos = (int32_t*)take(NT * 4);
    b.last = (int32_t*)take(NT * 4);
    b.active = (uint8_t*)take(NT);
    b.carry = (long long*)take((NT + 1) * 8);
    b.pm = (long long*)take((NT + 1) * 8);
    b.sm = (long long*)take((NT + 1) * 8);
    b.cb = (double*)take((NT + 1) * 8);
    b.mstep = (long long*)take(NT * 8);
    b.dec = (uint8_t*)take((size_t)(g.R ? g.R : 1));
    b.endb = (double*)take((size_t)(g.R ? g.R : 1) * 24);
    b.evk = (unsigned long long*)take((size_t)(g.max_events + 1) * 8);
    b.snap = (double*)take((size_t)(g.max_events + 1) * 24);
    b.evix = (int32_t*)take((size_t)(g.R ? g.R : 1) * 12);
    return b;
}

cudaError_t base_launch(const DevGraph& g, const BaseDev& b, const int32_t* perm, const uint8_t* dec,
                        cudaStream_t s) {
    base_kernel<<<1, 256, 0, s>>>(g, b, perm, dec);
    return cudaGetLastError();
}

int window_grid(int device) {
    cudaDeviceProp p;
    if (cudaGetDeviceProperties(&p, device) != cudaSuccess) return 148 * 4;
    // as many resident CTAs as registers / shared memory allow: the warps are
    // latency bound (global gathers of the base tables), so occupancy pays
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, window_kernel, kWarpsW * 32, 0) != cudaSuccess || occ < 1) {
        cudaGetLastError();
        occ = 4;
    }
    return p.multiProcessorCount * occ;
}

cudaError_t window_launch(const DevGraph& g, const BaseDev& b, int grid, double* endb_ws, int64_t K,
                          const int32_t* wstart, const int32_t* wlen, const int32_t* wperm, int32_t wmax,
                          uint8_t* st, int64_t* pk, double* lt, cudaStream_t s) {
    if (K <= 0) return cudaSuccess;
    const int64_t need = (K + kWarpsW - 1) / kWarpsW;
    const int gr = (int)std::min<int64_t>(grid, need);
    window_kernel<<<gr, kWarpsW * 32, 0, s>>>(g, b, K, wstart, wlen, wperm, wmax, st, pk, lt, endb_ws);
    return cudaGetLastError();
}

int window_wmax_supported() { return kWMax; }

}  // namespace magis
