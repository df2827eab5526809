// magis_evalb.cu -- "kernel B": one candidate per two-CTA thread-block cluster
// (the north_star's several-CTAs-per-candidate
// path for large graphs).  Same semantics as the packed kernel's tier 2
// (P:402-424 with reading P1; Fig. 8 rules, reading P6; latency, reading P7):
//
//  * both CTAs of the cluster build the whole position array of the
//    candidate in their own shared memory (phase 1, the scatter is local) and
//    resolve the optional nodes (phase 2);
//  * the consumer rows are split: CTA r walks the rows dealt to warps
//    [r 16, r 16 + 16) of the plan and scatters each node's alloc / free into
//    its OWN full-size per-step delta array (D[i] = alloc(i) - free(i - 1));
//  * after a cluster barrier each CTA adds the peer's deltas for its half of
//    the steps with coalesced DSMEM reads, scans that half ((sum, max-prefix)
//    monoid) and emits the half's swap-event steps with their compute-cost
//    prefix;
//  * CTA 0 combines the two halves (peak = max(m0, s0 + m1)), reads CTA 1's
//    flags and events through DSMEM / global memory and walks the three
//    copy queues.
//
// B200 trade-off: phases 0-2 are replicated and the halves meet
// through DSMEM (17-21 B/clk/SM); it is selectable with MAGIS_KERNELB=1 and
// measured against the single-CTA tier 2.
#include <cooperative_groups.h>

#include <climits>
#include <cmath>

#include "magis_internal.h"

namespace cg = cooperative_groups;

namespace magis {

namespace {

constexpr int kB = 512;              // threads per CTA
constexpr int kWB = kB / 32;         // warps per CTA
constexpr uint32_t kKShift = 29, kIdMaskB = (1u << 29) - 1;
constexpr uint32_t kHOut = 2, kHClone = 3, kHNop = 7;
constexpr long long kNegInfB = -(1ll << 62);

struct CtlB {
    int flags;          // MAGIS_ST_NOT_PERM | MAGIS_ST_BAD_DEC of this CTA
    int viol;           // MAGIS_ST_EDGE of this CTA
    int swaps;          // the candidate swaps some tensor
    long long s, m;     // this CTA's (sum, max-prefix) of its half of the steps
    double c;           // compute cost of its half
    int nev;            // event steps in its half
};

__device__ __forceinline__ void monoid(long long& s, long long& m, long long ps, long long pm) {
    // (ps, pm) precedes (s, m)
    m = max(pm, ps + m);
    s = ps + s;
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kB, 1)
evalb_kernel(DevGraph g, Plan2 pl, const char* __restrict__ blob, BLayout lay, int64_t K,
             const int32_t* __restrict__ perm, const uint8_t* __restrict__ dec,
             uint8_t* __restrict__ out_status, int64_t* __restrict__ out_peak, double* __restrict__ out_lat,
             unsigned long long* __restrict__ evk_g, double* __restrict__ evc_g) {
    cg::cluster_group cl = cg::this_cluster();
    const int rank = (int)cl.block_rank();
    extern __shared__ __align__(16) char smb[];
    __shared__ CtlB ctl;
    __shared__ long long ws_s[kWB], ws_m[kWB];
    __shared__ double ws_c[kWB];
    __shared__ int ws_e[kWB];
    __shared__ uint64_t mbar;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int32_t NT = pl.NT, n = pl.n, R = pl.R;
    const int32_t NTX = pl.NTX;
    const int32_t L = lay.L, S = lay.S, S0 = lay.S0;
    const uint32_t Lm = lay.Lm;

    // tables: rows and per-node tables from the global image; the cost classes
    // (tier-2 plans of graphs with <= 256 distinct costs) staged per CTA
    const uint32_t* wtab = (const uint32_t*)(blob + pl.off_wtab);
    const uint2* crow = (const uint2*)(blob + pl.off_crow);
    const uint32_t* chdr = (const uint32_t*)(blob + pl.off_chdr);
    const uint32_t* csize = (const uint32_t*)(blob + pl.off_csize);
    const uint16_t* cent = (const uint16_t*)(blob + pl.off_cent);
    const uint2* ninfo = (const uint2*)(blob + pl.off_ninfo);
    const uint16_t* lul = (const uint16_t*)(blob + pl.off_lul);
    const uint32_t* urow = (const uint32_t*)(blob + pl.off_urow);
    const uint16_t* ubs = (const uint16_t*)(blob + pl.off_ubs);
    const uint16_t* utr = (const uint16_t*)(blob + pl.off_utr);
    const double* cost_g = (const double*)(blob + pl.off_cost);
    const bool ccls = pl.cost_cls != 0;
    const double* cval = (const double*)smb;
    const uint8_t* cidx = (const uint8_t*)(smb + pl.ccls_idx_off);
    if (ccls) {
        const uint32_t bytes = lay.stage;
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&mbar);
        if (tid == 0) {
            asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bar) : "memory");
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
        if (tid == 0) {
            asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
            for (uint32_t o = 0; o < bytes; o += 32768u) {
                const uint32_t nb = min(32768u, bytes - o);
                const uint32_t dst = (uint32_t)__cvta_generic_to_shared(smb + o);
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                    "l"(blob + pl.off_ccls + o), "r"(nb), "r"(bar)
                    : "memory");
            }
        }
        uint32_t done = 0;
        while (!done)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
                         : "=r"(done) : "r"(bar) : "memory");
    }
    uint16_t* pos = (uint16_t*)(smb + lay.pos);          // [NTX + 1], +1 encoded, 0 = absent
    int32_t* D = (int32_t*)(smb + lay.D);                // [Sl] per-step deltas (this CTA's rows)
    uint32_t* marks = (uint32_t*)(smb + lay.marks);      // [nwm] event-step bits
    uint8_t* dec_s = (uint8_t*)(smb + lay.dec);          // [R]
    double* endb = (double*)(smb + lay.end);             // [3R] (CTA 0's walk)
    for (int i = tid; i <= NTX; i += kB) pos[i] = 0;
    for (int i = tid; i < lay.Sl; i += kB) D[i] = 0;
    for (int i = tid; i < lay.nwm; i += kB) marks[i] = 0;
    if (tid == 0) { ctl.flags = 0; ctl.viol = 0; ctl.swaps = 0; }
    __syncthreads();
    cl.sync();

    const int64_t ncl = gridDim.x / 2, cid = blockIdx.x / 2;
    const int peer = rank ^ 1;
    int32_t* Dp = cl.map_shared_rank(D, peer);
    CtlB* ctlp = cl.map_shared_rank(&ctl, peer);
    for (int64_t k = cid; k < K; k += ncl) {
        const int32_t* pk = perm + k * (int64_t)NT;
        // ---- phase 0: decisions (bad values, re-mat of an input-less tensor)
        {
            int bad = 0, sw = 0;
            for (int r = tid; r < R; r += kB) {
                const uint8_t d = dec[k * (int64_t)R + r];
                dec_s[r] = d;
                sw |= d == 2;
                bad |= (d > 2) | ((d == 1) & !(__ldg(g.rflag + r) & kRHasInput));
            }
            // ---- phase 1: inverse permutation (the whole schedule, local)
            for (int32_t i = tid; i < NT; i += kB) {
                const uint32_t v = (uint32_t)__ldcs(pk + i);
                if (v < (uint32_t)NT) pos[v] = (uint16_t)(i + 1);
                else bad |= 2;
            }
            bad = __reduce_or_sync(0xffffffffu, bad);
            sw = __reduce_or_sync(0xffffffffu, sw);
            if (lane == 0) {
                if (bad & 1) atomicOr(&ctl.flags, MAGIS_ST_BAD_DEC);
                if (bad & 2) atomicOr(&ctl.flags, MAGIS_ST_NOT_PERM);
                if (sw) atomicOr(&ctl.swaps, 1);
            }
        }
        __syncthreads();
        // ---- phase 2: optional nodes, virtual late-user slots, event steps
        for (int r = tid; r < R; r += kB) {
            const uint32_t ur = urow[r];
            const uint32_t u0 = ur & 0xffffu, u1 = u0 + (ur >> 16);
            const uint8_t d = dec_s[r];
#pragma unroll
            for (int o = 0; o < 3; o++) {
                const int32_t id = n + 3 * r + o;
                const uint32_t p = pos[id];
                if (p == 0) { atomicOr(&ctl.flags, MAGIS_ST_NOT_PERM); continue; }
                const bool act = (o == 0) ? (d == 1) : (d == 2);
                if (!act) pos[id] = 0;
                else if (o > 0) atomicOr(marks + ((p - 1) >> 5), 1u << ((p - 1) & 31));
            }
            if (d == 2) {
                const uint32_t pt = pos[utr[r]];
                if (pt) atomicOr(marks + ((pt - 1) >> 5), 1u << ((pt - 1) & 31));
            }
            for (uint32_t j = u0; j < u1; j++) {
                const uint32_t pb = pos[ubs[j]];
                pos[NT + j] = (d == 0) ? (uint16_t)pb : (uint16_t)0;
                if (d == 2 && pb) atomicOr(marks + ((pb - 1) >> 5), 1u << ((pb - 1) & 31));
            }
        }
        __syncthreads();
        // ---- phase 3: this CTA's share of the consumer rows
        {
            int nperm = 0, viol = 0;
            const int vw = rank * kWB + warp;
            const uint32_t r0 = wtab[vw * 4 + 0], r1 = wtab[vw * 4 + 1];
            for (uint32_t r = r0; r < r1; r++) {
                const uint2 rw = crow[r];
                const uint32_t h = chdr[r * 32 + lane];
                const uint32_t A = csize[r * 32 + lane];
                const uint32_t kind = h >> kKShift, id = h & kIdMaskB;
                const uint32_t p = pos[id];
                uint32_t lst = p, mn = 0xffffu;
                const uint16_t* ent = cent + rw.x + lane;
                for (uint32_t j = 0; j < rw.y; j++) {
                    const uint32_t q = pos[ent[j * 32]];
                    mn = min(mn, (q - 1u) & 0xffffu);
                    lst = max(lst, q);
                }
                if (kind == kHNop) continue;
                if (kind < kHClone && p == 0) nperm = 1;
                if (mn < p) viol = 1;
                if (p == 0 || A == 0) continue;
                const uint32_t st = p - 1;
                atomicAdd(&D[st + __umulhi(st, Lm)], (int32_t)A);          // alloc at the own step
                if (kind != kHOut && lst < (uint32_t)NT)                     // freed after the last reader
                    atomicAdd(&D[lst + __umulhi(lst, Lm)], -(int32_t)A);
            }
            nperm = __reduce_or_sync(0xffffffffu, nperm);
            viol = __reduce_or_sync(0xffffffffu, viol);
            if (lane == 0) {
                if (nperm) atomicOr(&ctl.flags, MAGIS_ST_NOT_PERM);
                if (viol) atomicOr(&ctl.viol, MAGIS_ST_EDGE);
            }
        }
        cl.sync();    // both CTAs' deltas and flags complete
        const int st_all = [&] {
            const int f = ctl.flags | ctlp->flags;
            return f ? f : (ctl.viol | ctlp->viol);
        }();
        const bool swp = ctl.swaps != 0;
        const int c0 = rank * S0, c1 = min(S, c0 + S0);        // this CTA's chunks
        if (st_all == 0) {
            // ---- phase 4: add the peer's deltas of this half (coalesced DSMEM reads)
            for (int i = c0 * (L + 1) + tid; i < c1 * (L + 1); i += kB) D[i] += Dp[i];
            __syncthreads();
            // ---- phase 5: scan of the half; cost prefix and event steps
            const int c = c0 + tid;
            const int32_t lo = c * L, nst = (c < c1) ? max(0, min(L, NT - lo)) : 0;
            long long s1 = 0, m1 = kNegInfB;
            double cs = 0.0;
            int ne = 0;
            const int32_t* dp = D + c * (L + 1);
            for (int j = 0; j < nst; j++) {
                s1 += dp[j];
                m1 = max(m1, s1);
            }
            auto node_cost = [&](int32_t v) -> double {
                if (v >= n && pos[v] == 0) return 0.0;                        // absent optional node
                return ccls ? cval[cidx[v]] : __ldg(cost_g + v);
            };
            if (swp) {
                for (int j = 0; j < nst; j++) {
                    const int32_t v = __ldg(pk + lo + j);
                    ne += (marks[(lo + j) >> 5] >> ((lo + j) & 31)) & 1u;
                    cs += node_cost(v);
                }
            }
            // block scans: (sum, max-prefix), cost, event counts
            long long ss = s1, mm = m1;
            double cc = cs;
            int ee = ne;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const long long ps = __shfl_up_sync(0xffffffffu, ss, o);
                const long long pm = __shfl_up_sync(0xffffffffu, mm, o);
                const double pc = __shfl_up_sync(0xffffffffu, cc, o);
                const int pe = __shfl_up_sync(0xffffffffu, ee, o);
                if (lane >= o) { monoid(ss, mm, ps, pm); cc += pc; ee += pe; }
            }
            if (lane == 31) { ws_s[warp] = ss; ws_m[warp] = mm; ws_c[warp] = cc; ws_e[warp] = ee; }
            __syncthreads();
            if (warp == 0) {
                long long s2 = lane < kWB ? ws_s[lane] : 0, m2 = lane < kWB ? ws_m[lane] : kNegInfB;
                double c2 = lane < kWB ? ws_c[lane] : 0.0;
                int e2 = lane < kWB ? ws_e[lane] : 0;
                const double cw = c2;
                const int ew = e2;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const long long ps = __shfl_up_sync(0xffffffffu, s2, o);
                    const long long pm = __shfl_up_sync(0xffffffffu, m2, o);
                    const double pc = __shfl_up_sync(0xffffffffu, c2, o);
                    const int pe = __shfl_up_sync(0xffffffffu, e2, o);
                    if (lane >= o) { monoid(s2, m2, ps, pm); c2 += pc; e2 += pe; }
                }
                if (lane < kWB) { ws_c[lane] = c2 - cw; ws_e[lane] = e2 - ew; }   // exclusive warp offsets
                if (lane == kWB - 1) { ctl.s = s2; ctl.m = m2; ctl.c = c2; ctl.nev = e2; }
            }
            __syncthreads();
            if (swp && ne > 0) {
                // the events of this chunk in step order, with the compute-cost
                // prefix before the step within this CTA's half
                double pre = ws_c[warp] + (cc - cs);
                int o = ws_e[warp] + (ee - ne);
                const size_t eb = ((size_t)cid * 2 + rank) * (size_t)pl.max_events;
                for (int j = 0; j < nst; j++) {
                    const int32_t v = __ldg(pk + lo + j);
                    if ((marks[(lo + j) >> 5] >> ((lo + j) & 31)) & 1u) {
                        evk_g[eb + o] = ((unsigned long long)(lo + j) << 32) | (uint32_t)v;
                        evc_g[eb + o] = pre;
                        o++;
                    }
                    pre += node_cost(v);
                }
            }
            __threadfence();
        }
        cl.sync();    // aggregates and event lists of both halves visible
        // ---- phase 6: CTA 0 combines the halves and walks the copy queues
        if (rank == 0 && warp == 0) {
            double lat = INFINITY;
            long long peak = -1;
            if (st_all == 0) {
                const CtlB& q = *ctlp;
                const long long mtot = max(ctl.m, ctl.s + q.m);
                peak = mtot * pl.unit;
                const double ctot = ctl.c + q.c;
                if (!swp) {
                    double bl = 0.0;
                    for (int r = lane; r < R; r += 32)
                        if (dec_s[r] == 1) bl += g.tcost[r];
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) bl += __shfl_xor_sync(0xffffffffu, bl, o);
                    lat = g.base_cost + bl;
                } else if (ctl.nev + q.nev <= lay.evcap) {
                    // the event steps of both halves are resolved by the warp in
                    // parallel into records in shared memory (the node's swapped
                    // inputs and produced tensor; Store / Load with their
                    // transfer time), so the serial walk touches no global memory
                    const int ntot = ctl.nev + q.nev;
                    unsigned long long* ra = (unsigned long long*)(smb + lay.rec);
                    double* rx = (double*)(ra + lay.evcap);
                    for (int e = lane; e < ntot; e += 32) {
                        const int h = e < ctl.nev ? 0 : 1;
                        const size_t idx = ((size_t)cid * 2 + h) * (size_t)pl.max_events + (h ? e - ctl.nev : e);
                        const int32_t w = (int32_t)(evk_g[idx] & 0xffffffffu);
                        unsigned long long a = 0;
                        double x;
                        if (w < n) {
                            // kind 0: bits 0-47 up to three swapped inputs (r, 16 bits
                            // each), 48-55 their count (255: more, walk the list),
                            // 56-61 unused; the produced swapped tensor r+1 in rp
                            const uint2 ni = ninfo[w];
                            const uint32_t rt = ni.x & 0xffffu, cnt = ni.x >> 16;
                            uint32_t ns = 0;
                            for (uint32_t i = 0; i < cnt; i++) {
                                const uint32_t r = lul[ni.y + i];
                                if (dec_s[r] != 2) continue;
                                if (ns < 3) a |= (unsigned long long)r << (16 * ns);
                                ns++;
                            }
                            if (ns > 3) a = ((unsigned long long)ni.y << 16) | cnt;   // long list: walk lul
                            a |= (unsigned long long)min(ns, 255u) << 48;
                            const uint32_t rp = (rt && dec_s[rt - 1] == 2) ? rt : 0u;
                            x = evc_g[idx] + (h ? ctl.c : 0.0);
                            ra[e] = a;
                            rx[e] = x;
                            // producer id kept apart (bits would collide with a long list)
                            ((uint32_t*)(rx + lay.evcap))[e] = rp;
                        } else {
                            const uint32_t qq = (uint32_t)(w - n), r = qq / 3, kd = qq - 3 * r;
                            ra[e] = ((unsigned long long)(kd ? kd : 3u) << 62) | r;   // 3: clone, no queue
                            rx[e] = g.xfer[r];
                            ((uint32_t*)(rx + lay.evcap))[e] = 0u;
                        }
                    }
                    __syncwarp();
                    if (lane == 0) {
                        const uint32_t* rpv = (const uint32_t*)(rx + lay.evcap);
                        double Dl = 0.0, Td = 0.0, Th = 0.0;
                        for (int e = 0; e < ntot; e++) {
                            const unsigned long long a = ra[e];
                            const double x = rx[e];
                            const uint32_t kd = (uint32_t)(a >> 62);
                            if (kd == 0) {
                                const uint32_t ns = (uint32_t)(a >> 48) & 0xffu;
                                if (ns <= 3) {
                                    for (uint32_t i = 0; i < ns; i++)
                                        Dl = fmax(Dl, endb[3 * ((a >> (16 * i)) & 0xffffu) + 2] - x);
                                } else {
                                    const uint32_t off = (uint32_t)(a >> 16) & 0xffffffffu, cnt = (uint32_t)a & 0xffffu;
                                    for (uint32_t i = 0; i < cnt; i++) {
                                        const uint32_t r = lul[off + i];
                                        if (dec_s[r] == 2) Dl = fmax(Dl, endb[3 * r + 2] - x);
                                    }
                                }
                                const uint32_t rp = rpv[e];
                                if (rp) endb[3 * (rp - 1)] = x + Dl + g.tcost[rp - 1];
                            } else if (kd == 1) {
                                const uint32_t r = (uint32_t)a & 0xffffffu;
                                Td = fmax(Td, endb[3 * r]) + x;
                                endb[3 * r + 1] = Td;
                            } else if (kd == 2) {
                                const uint32_t r = (uint32_t)a & 0xffffffu;
                                Th = fmax(Th, endb[3 * r + 1]) + x;
                                endb[3 * r + 2] = Th;
                            }
                        }
                        lat = fmax(fmax(ctot + Dl, Td), Th);
                    }
                } else if (lane == 0) {
                    // three in-order queues over the event steps (reading P7):
                    // endb[3r] producer end, [3r+1] Store end, [3r+2] Load end
                    double Dl = 0.0, Td = 0.0, Th = 0.0;
                    const int ntot = ctl.nev + q.nev;
                    for (int e = 0; e < ntot; e++) {
                        const int h = e < ctl.nev ? 0 : 1;
                        const size_t idx = ((size_t)cid * 2 + h) * (size_t)pl.max_events + (h ? e - ctl.nev : e);
                        const unsigned long long kk = evk_g[idx];
                        const double x = evc_g[idx] + (h ? ctl.c : 0.0);
                        const int32_t w = (int32_t)(kk & 0xffffffffu);
                        if (w < n) {
                            const uint2 ni = ninfo[w];
                            const uint32_t rt = ni.x & 0xffffu, cnt = ni.x >> 16;
                            for (uint32_t i = 0; i < cnt; i++) {              // stalls on swapped inputs
                                const uint32_t r = lul[ni.y + i];
                                if (dec_s[r] == 2) Dl = fmax(Dl, endb[3 * r + 2] - x);
                            }
                            if (rt && dec_s[rt - 1] == 2) endb[3 * (rt - 1)] = x + Dl + g.tcost[rt - 1];
                        } else {
                            const uint32_t qq = (uint32_t)(w - n), r = qq / 3, kd = qq - 3 * r;
                            if (kd == 1) { Td = fmax(Td, endb[3 * r]) + g.xfer[r]; endb[3 * r + 1] = Td; }
                            else if (kd == 2) { Th = fmax(Th, endb[3 * r + 1]) + g.xfer[r]; endb[3 * r + 2] = Th; }
                        }
                    }
                    lat = fmax(fmax(ctot + Dl, Td), Th);
                }
            }
            if (lane == 0) {
                out_status[k] = (uint8_t)st_all;
                out_peak[k] = st_all ? -1 : peak;
                out_lat[k] = st_all ? INFINITY : lat;
            }
        }
        cl.sync();    // the peer is done reading this CTA's deltas and control words
        // ---- phase 7: clear for the next candidate
        for (int i = tid; i <= NTX; i += kB) pos[i] = 0;
        for (int i = tid; i < lay.Sl; i += kB) D[i] = 0;
        for (int i = tid; i < lay.nwm; i += kB) marks[i] = 0;
        if (tid == 0) { ctl.flags = 0; ctl.viol = 0; ctl.swaps = 0; }
        __syncthreads();
    }
    cl.sync();
}

}  // namespace

bool evalb_layout(const Plan2& pl, size_t smem_cap, BLayout* lay) {
    BLayout b{};
    const int32_t NT = pl.NT;
    b.L = std::max(4, ((NT + 2 * kB - 1) / (2 * kB) + 3) & ~3);       // chunk: the two halves cover all steps
    b.S = (NT + b.L - 1) / b.L;
    b.S0 = (b.S + 1) / 2;
    if (b.S0 > kB) return false;
    b.Lm = (uint32_t)((((uint64_t)1 << 32) + (uint64_t)b.L - 1) / (uint64_t)b.L);
    b.Sl = (b.L + 1) * b.S;
    auto a16 = [](size_t x) { return (x + 15) / 16 * 16; };
    size_t o = 0;
    b.stage = pl.cost_cls ? (uint32_t)a16(pl.ccls_idx_off + (size_t)pl.NTX) : 0u;
    o = b.stage;
    b.pos = (uint32_t)o;   o = a16(o + (size_t)(pl.NTX + 1) * 2);
    b.D = (uint32_t)o;     o = a16(o + (size_t)b.Sl * 4);
    b.nwm = (NT + 31) / 32 + 2;
    b.marks = (uint32_t)o; o = a16(o + (size_t)b.nwm * 4);
    b.dec = (uint32_t)o;   o = a16(o + (size_t)std::max(pl.R, 1));
    b.end = (uint32_t)o;   o = a16(o + (size_t)3 * std::max(pl.R, 1) * 8);
    if (o > smem_cap) return false;
    // resolved event records (u64 key, f64 time, u32 producer) for the walk,
    // as many as fit (a candidate with more walks them from global memory)
    b.evcap = (int32_t)std::min<size_t>((size_t)std::max(pl.max_events, 1), (smem_cap - o) / 20);
    b.evcap &= ~7;
    b.rec = (uint32_t)o;   o = a16(o + (size_t)b.evcap * 20);
    b.total = (uint32_t)o;
    *lay = b;
    return true;
}

cudaError_t evalb_launch(const DevGraph& g, const Plan2& pl, const BLayout& lay, const void* blob, int clusters,
                         int64_t K, const int32_t* perm, const uint8_t* dec, uint8_t* status, int64_t* peak,
                         double* lat, void* evscratch, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    cudaError_t e = cudaFuncSetAttribute(evalb_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)lay.total);
    if (e != cudaSuccess) return e;
    const int ncl = (int)std::min<int64_t>(clusters, K);
    unsigned long long* evk = (unsigned long long*)evscratch;
    double* evc = (double*)((char*)evscratch + (size_t)clusters * 2 * pl.max_events * 8);
    evalb_kernel<<<2 * ncl, kB, lay.total, stream>>>(g, pl, (const char*)blob, lay, K, perm, dec, status, peak, lat,
                                                     evk, evc);
    return cudaGetLastError();
}

size_t evalb_scratch_bytes(const Plan2& pl, int clusters) {
    return (size_t)clusters * 2 * std::max(pl.max_events, 1) * 16 + 256;
}

}  // namespace magis
