// magis_eval.cu -- batched schedule evaluation on sm_100a.
//
// One CTA scores one candidate at a time; the grid is persistent (CTAs stride
// over candidates).  Per candidate, in the paper's order:
//   a2  inverse permutation pos[perm[i]] = i  (perm streamed, coalesced)
//   a3  validity: every active super-graph edge (u,v) has pos[u] < pos[v]
//   a4  last[u] = max pos over active readers (segmented max over the
//       consumer CSR); outputs live to the end; no reader -> own step
//   a5  per step p: A[p] = bytes allocated by the op at p, Fr[p] = bytes
//       freed after p (gather over the op's input CSR: inputs whose last
//       reader is this op, plus its own output if it has no reader)
//   a6/a7 M_i = sum_{k<=i} A[k] - sum_{k<i} Fr[k]; peak = max_i M_i, as a
//       block scan of the (sum, max-prefix) monoid over per-thread chunks
//   a8  latency: base + sum of clone costs (order-invariant, P:406-408,
//       P:1615-1617); with swaps, the three in-order queues (compute, D2H,
//       H2D) as a sorted sweep over the swap events only
// The per-candidate state (pos, last, A, Fr, C, events) lives in shared
// memory (variant 0) or, for graphs too large for 227 KB, in a per-CTA slice
// of global memory (variant 1).  Graph tables are read through the read-only
// path (L1/L2 resident; they are shared by every candidate).
#include <cfloat>
#include <climits>
#include <cmath>

#include "magis_internal.h"

namespace magis {

constexpr int kBlock = 512;
constexpr int kWarps = kBlock / 32;

static size_t al(size_t x) { return (x + 15) / 16 * 16; }

StateLayout state_layout(int32_t NT, int32_t R, int32_t max_events, int32_t Rd) {
    StateLayout L{};
    size_t o = 0;
    L.pos = o;       o += al((size_t)NT * 4);
    L.last = o;      o += al((size_t)NT * 4);
    L.A = o;         o += al((size_t)NT * 8);
    L.Fr = o;        o += al((size_t)NT * 8);
    L.C = o;         o += al((size_t)NT * 8);
    L.evkey_in = o;  o += al((size_t)max_events * 8);
    L.evkey_out = o; o += al((size_t)max_events * 8);
    L.evcb = o;      o += al((size_t)max_events * 8);
    L.endT = o;      o += al((size_t)R * 8);
    L.endS = o;      o += al((size_t)R * 8);
    L.endL = o;      o += al((size_t)R * 8);
    L.dec = o;       o += al((size_t)Rd);
    L.total = o;
    return L;
}

struct Scratch {
    long long red_ll[kWarps + 1];
    double red_d[kWarps + 1];
    double cofs[kBlock];
    int status;
    int nev;
};

__device__ __forceinline__ bool gate_on(int32_t gate, const uint8_t* dec_s) {
    return gate < 0 || dec_s[gate >> 2] == (uint8_t)(gate & 3);
}

// Block-wide exclusive scan (sum) of one value per thread; also returns the total.
template <typename T>
__device__ __forceinline__ T block_excl_scan(T x, T* red, T& total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    T inc = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) red[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        T w = lane < kWarps ? red[lane] : T(0);
        T wi = w;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T y = __shfl_up_sync(0xffffffffu, wi, o);
            if (lane >= o) wi += y;
        }
        if (lane < kWarps) red[lane] = wi - w;
        if (lane == kWarps - 1) red[kWarps] = wi;
    }
    __syncthreads();
    T ex = red[wid] + inc - x;
    total = red[kWarps];
    __syncthreads();
    return ex;
}

__device__ __forceinline__ long long block_max_ll(long long x, long long* red) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x = max(x, __shfl_xor_sync(0xffffffffu, x, o));
    if (lane == 0) red[wid] = x;
    __syncthreads();
    if (wid == 0) {
        long long w = lane < kWarps ? red[lane] : LLONG_MIN;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) w = max(w, __shfl_xor_sync(0xffffffffu, w, o));
        if (lane == 0) red[kWarps] = w;
    }
    __syncthreads();
    long long r = red[kWarps];
    __syncthreads();
    return r;
}

__device__ __forceinline__ double block_sum_d(double x, double* red) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (lane == 0) red[wid] = x;
    __syncthreads();
    if (wid == 0) {
        double w = lane < kWarps ? red[lane] : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) w += __shfl_xor_sync(0xffffffffu, w, o);
        if (lane == 0) red[kWarps] = w;
    }
    __syncthreads();
    double r = red[kWarps];
    __syncthreads();
    return r;
}

template <bool kGlobalState>
__global__ void __launch_bounds__(kBlock)
eval_kernel(DevGraph g, int64_t K, const int32_t* __restrict__ perm,
            const uint8_t* __restrict__ dec, uint8_t* __restrict__ out_status,
            int64_t* __restrict__ out_peak, double* __restrict__ out_lat,
            char* __restrict__ gws, size_t ws_stride, StateLayout L) {
    extern __shared__ __align__(16) char smem_dyn[];
    __shared__ Scratch sc;
    char* st = kGlobalState ? (gws + (size_t)blockIdx.x * ws_stride) : smem_dyn;
    int32_t* pos = (int32_t*)(st + L.pos);
    int32_t* last = (int32_t*)(st + L.last);
    long long* A = (long long*)(st + L.A);
    long long* Fr = (long long*)(st + L.Fr);
    double* C = (double*)(st + L.C);
    unsigned long long* evk = (unsigned long long*)(st + L.evkey_in);
    unsigned long long* evk_s = (unsigned long long*)(st + L.evkey_out);
    double* evcb = (double*)(st + L.evcb);
    double* endT = (double*)(st + L.endT);
    double* endS = (double*)(st + L.endS);
    double* endL = (double*)(st + L.endL);
    uint8_t* dec_s = (uint8_t*)(st + L.dec);

    const int tid = threadIdx.x;
    const int32_t NT = g.NT, R = g.R, n = g.n;
    const int32_t Lc = (NT + kBlock - 1) / kBlock;   // scan chunk per thread

    for (int64_t k = blockIdx.x; k < K; k += gridDim.x) {
        const int32_t* P = perm + k * (int64_t)NT;
        // ---- P0: decisions, reset ------------------------------------------------
        if (tid == 0) { sc.status = 0; sc.nev = 0; }
        int bad_dec = 0, any_sw = 0;
        for (int32_t r = tid; r < g.Rd; r += kBlock) {
            uint8_t d = dec[k * (int64_t)g.Rd + r];
            dec_s[r] = d;
            if (r < R) {
                bad_dec |= (d > 2) | ((d == 1) & !(g.rflag[r] & kRHasInput));
                any_sw |= (d == 2);
            } else {
                bad_dec |= d >= __ldg(g.nvar + (r - R));   // reading F1: a variant of region r - R
            }
        }
        for (int32_t v = tid; v < NT; v += kBlock) pos[v] = -1;
        bad_dec = __syncthreads_or(bad_dec);
        any_sw = __syncthreads_or(any_sw);
        // ---- a2: inverse permutation ------------------------------------------------
        int notperm = 0;
        for (int32_t i = tid; i < NT; i += kBlock) {
            int32_t v = __ldcs(P + i);
            if ((uint32_t)v < (uint32_t)NT) pos[v] = i;
            else notperm = 1;
        }
        notperm = __syncthreads_or(notperm);
        // ---- a3 + a4: validity and last use ----------------------------------------
        int flags = 0;
        for (int32_t v = tid; v < NT; v += kBlock) {
            const int32_t p = pos[v];
            if (p < 0) { flags |= MAGIS_ST_NOT_PERM; continue; }
            if (!gate_on(__ldg(g.ngate + v), dec_s)) { last[v] = p; continue; }
            int32_t lst = p;
            const int32_t e1 = __ldg(g.cons_ptr + v + 1);
            for (int32_t e = __ldg(g.cons_ptr + v); e < e1; e++) {
                const int2 ce = __ldg(g.cons_ent + e);
                if (!gate_on(ce.y, dec_s)) continue;
                const int32_t q = pos[ce.x];
                if (q <= p) flags |= MAGIS_ST_EDGE;
                lst = max(lst, q);
            }
            if (__ldg(g.nflag + v) & kFlagOutput) lst = NT - 1;
            last[v] = lst;
        }
        if (flags) atomicOr(&sc.status, flags);
        __syncthreads();
        int status = sc.status | (notperm ? MAGIS_ST_NOT_PERM : 0) | (bad_dec ? MAGIS_ST_BAD_DEC : 0);
        if (status & (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC)) status &= (MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC);
        if (status) {
            if (tid == 0) {
                out_status[k] = (uint8_t)status;
                out_peak[k] = -1;
                out_lat[k] = __longlong_as_double(0x7ff0000000000000ll);
            }
            __syncthreads();
            continue;
        }
        // ---- a5: per-step alloc / free ------------------------------------------------
        for (int32_t v = tid; v < NT; v += kBlock) {
            const int32_t p = pos[v];
            if (!gate_on(__ldg(g.ngate + v), dec_s)) {
                A[p] = 0;
                Fr[p] = 0;
                if (any_sw) C[p] = 0.0;
                continue;
            }
            const long long sz = __ldg(g.size + v);
            long long f = (last[v] == p) ? sz : 0;
            const int32_t e1 = __ldg(g.in_ptr + v + 1);
            for (int32_t e = __ldg(g.in_ptr + v); e < e1; e++) {
                const int2 ie = __ldg(g.in_ent + e);
                if (gate_on(ie.y, dec_s) && last[ie.x] == p) f += __ldg(g.size + ie.x);
            }
            A[p] = sz;
            Fr[p] = f;
            if (any_sw) C[p] = (__ldg(g.nflag + v) & kFlagCompute) ? __ldg(g.cost + v) : 0.0;
        }
        __syncthreads();
        // ---- a6 + a7: scan of the (sum, max-prefix) monoid -------------------------
        const int32_t lo = tid * Lc, hi = min(lo + Lc, NT);
        long long s = 0, m = LLONG_MIN;
        double cs = 0.0;
        for (int32_t i = lo; i < hi; i++) {
            s += A[i];
            m = max(m, s);
            s -= Fr[i];
            if (any_sw) cs += C[i];
        }
        long long stot;
        const long long off = block_excl_scan<long long>(s, sc.red_ll, stot);
        const long long cand = (m == LLONG_MIN) ? LLONG_MIN : off + m;
        const long long peak = block_max_ll(cand, sc.red_ll);
        // ---- a8: latency -------------------------------------------------------------
        double lat;
        if (!any_sw) {
            double cl = 0.0;
            for (int32_t r = tid; r < R; r += kBlock)
                if (dec_s[r] == 1) cl += __ldg(g.tcost + r);
            for (int32_t i = tid; i < g.F; i += kBlock)              // the chosen F-Trans variants
                cl += __ldg(g.vcost + 4 * i + dec_s[R + i]);
            lat = g.base_cost + block_sum_d(cl, sc.red_d);
        } else {
            double ctot;
            const double cofs = block_excl_scan<double>(cs, sc.red_d, ctot);
            sc.cofs[tid] = cofs;
            // gather swap events
            for (int32_t r = tid; r < R; r += kBlock) {
                if (dec_s[r] != 2) continue;
                const int32_t u0 = __ldg(g.U_ptr + r), u1 = __ldg(g.U_ptr + r + 1);
                const int base = atomicAdd(&sc.nev, 3 + (u1 - u0));
                const unsigned long long rr = (unsigned long long)r;
                evk[base + 0] = ((unsigned long long)pos[__ldg(g.elig + r)] << 32) | (kEvProduce << 24) | rr;
                evk[base + 1] = ((unsigned long long)pos[n + 3 * r + 1] << 32) | (kEvStore << 24) | rr;
                evk[base + 2] = ((unsigned long long)pos[n + 3 * r + 2] << 32) | (kEvLoad << 24) | rr;
                for (int32_t j = u0; j < u1; j++)
                    evk[base + 3 + (j - u0)] =
                        ((unsigned long long)pos[__ldg(g.U_idx + j)] << 32) | (kEvStall << 24) | rr;
            }
            __syncthreads();
            const int nev = sc.nev;
            // rank sort (keys are unique) + compute-prefix before each event's step
            for (int e = tid; e < nev; e += kBlock) {
                const unsigned long long key = evk[e];
                int rank = 0;
                for (int j = 0; j < nev; j++) rank += (evk[j] < key);
                const int32_t stp = (int32_t)(key >> 32);
                const int32_t th = stp / Lc;
                double cb = sc.cofs[th];
                for (int32_t i = th * Lc; i < stp; i++) cb += C[i];
                evk_s[rank] = key;
                evcb[rank] = cb;
            }
            __syncthreads();
            if (tid == 0) {
                double D = 0.0, Td = 0.0, Th = 0.0;
                for (int e = 0; e < nev; e++) {
                    const unsigned long long key = evk_s[e];
                    const uint32_t type = (uint32_t)(key >> 24) & 0xff;
                    const int32_t r = (int32_t)(key & 0xffffff);
                    const double cb = evcb[e];
                    if (type == kEvStall) {
                        D = fmax(D, endL[r] - cb);
                    } else if (type == kEvProduce) {
                        endT[r] = cb + D + __ldg(g.tcost + r);
                    } else if (type == kEvStore) {
                        Td = fmax(Td, endT[r]) + __ldg(g.xfer + r);
                        endS[r] = Td;
                    } else {
                        Th = fmax(Th, endS[r]) + __ldg(g.xfer + r);
                        endL[r] = Th;
                    }
                }
                sc.red_d[kWarps] = fmax(fmax(ctot + D, Td), Th);
            }
            __syncthreads();
            lat = sc.red_d[kWarps];
        }
        if (tid == 0) {
            out_status[k] = 0;
            out_peak[k] = peak;
            out_lat[k] = lat;
        }
        __syncthreads();
    }
}

cudaError_t eval_configure(const DevGraph& g, int device, EvalConfig* cfg) {
    cudaDeviceProp prop;
    cudaError_t e = cudaGetDeviceProperties(&prop, device);
    if (e != cudaSuccess) return e;
    StateLayout L = state_layout(g.NT, g.R, g.max_events, g.Rd);
    cfg->block = kBlock;
    cfg->state_bytes = (L.total + 255) / 256 * 256;
    const size_t smem_cap = (size_t)prop.sharedMemPerBlockOptin - sizeof(Scratch) - 1024;
    int occ = 0;
    if (L.total <= smem_cap) {
        cfg->variant = 0;
        cfg->smem = L.total;
        e = cudaFuncSetAttribute(eval_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)cfg->smem);
        if (e != cudaSuccess) return e;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, eval_kernel<false>, kBlock, cfg->smem);
    } else {
        cfg->variant = 1;
        cfg->smem = 0;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, eval_kernel<true>, kBlock, 0);
    }
    if (e != cudaSuccess) return e;
    if (occ < 1) occ = 1;
    cfg->grid = prop.multiProcessorCount * occ;
    return cudaSuccess;
}

cudaError_t eval_launch(const DevGraph& g, const EvalConfig& cfg, void* gws, int64_t K,
                        const int32_t* perm, const uint8_t* dec, uint8_t* status,
                        int64_t* peak, double* lat, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    StateLayout L = state_layout(g.NT, g.R, g.max_events, g.Rd);
    const int grid = (int)std::min<int64_t>(cfg.grid, K);
    if (cfg.variant == 0) {
        eval_kernel<false><<<grid, kBlock, cfg.smem, stream>>>(g, K, perm, dec, status, peak, lat,
                                                               nullptr, 0, L);
    } else {
        eval_kernel<true><<<grid, kBlock, 0, stream>>>(g, K, perm, dec, status, peak, lat,
                                                       (char*)gws, cfg.state_bytes, L);
    }
    return cudaGetLastError();
}

}  // namespace magis
