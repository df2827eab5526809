// magis_eval2.cu -- the shared-memory-resident evaluation kernel (variant 2).
//
// Same per-candidate chain as magis_eval.cu (SURVEY §8(a) a2-a8, P:402-424,
// P:1780-1789), re-laid out for sm_100a:
//  * the graph lives in shared memory as per-thread "streams" (one u32 entry
//    per node header and per edge, interleaved across the 32 lanes of a warp
//    so every stream read is a conflict-free LDS), staged once per CTA with
//    the bulk-copy engine (cp.async.bulk + mbarrier);
//  * P candidates (1, 2 or 4) are scored at once: positions and last-use
//    steps are u16 lanes packed into one 32/64-bit word per node, so each
//    random gather, max and min over the consumer lists serves P candidates
//    (VIMNMX.U16x2 / VIADD.16x2);
//  * activation gates (Fig. 8 rules, reading P6) are folded into data: the
//    positions of inactive optional nodes are zeroed and a late-user edge
//    t_r -> b reads a per-candidate virtual slot holding pos(b) or 0, so the
//    inner loops carry no decision tests;
//  * positions are stored +1 (0 = absent / inactive), so validity is one
//    running min of (q - 1) per node: a violation iff min < pos (unsigned);
//  * alloc/free amounts land in per-step slots (u32 size units) in a
//    transposed layout, so the scan's per-thread contiguous chunks read
//    conflict-free;
//  * the swap-latency sweep (the three in-order queues of reading P7) runs in
//    a dedicated warp, one lane per candidate, fed through a double-buffered
//    shared-memory hand-off guarded by named barriers, so the main warps go on
//    to the next group while it runs.
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "magis_internal.h"

namespace magis {

constexpr uint32_t kKindShift = 29;
constexpr uint32_t kIdMask = (1u << kKindShift) - 1;
constexpr uint32_t kHdrOut = 2, kHdrClone = 3, kNop = 7;   // kHdr = 1, kHdrCopy = 4
constexpr int kBarMain = 1, kBarFull = 2, kBarEmpty = 4;
constexpr int TM = kMainThreads2;
constexpr int WM = TM / 32;

// -------------------------------------------------------------- packed u16 --
template <int P> struct Pk;
template <> struct Pk<1> {
    using V = uint32_t;
    static __device__ __forceinline__ V load(const uint16_t* a, uint32_t i) { return a[i]; }
    static __device__ __forceinline__ void store(uint16_t* a, uint32_t i, V v) { a[i] = (uint16_t)v; }
    static __device__ __forceinline__ uint32_t get(V v, int) { return v & 0xffffu; }
    static __device__ __forceinline__ V vmax(V a, V b) { return max(a, b); }
    static __device__ __forceinline__ V vmin(V a, V b) { return min(a, b); }
    static __device__ __forceinline__ V dec1(V a) { return (a - 1u) & 0xffffu; }
    static __device__ __forceinline__ V ones() { return 0xffffu; }
    static __device__ __forceinline__ V splat(uint32_t x) { return x; }
    static __device__ __forceinline__ V nzmask(V a) { return a ? 0xffffu : 0u; }
    static __device__ __forceinline__ V vand(V a, V b) { return a & b; }
    static __device__ __forceinline__ bool maybe_eq(V a, V b) { return a == b; }
};
template <> struct Pk<2> {
    using V = uint32_t;
    static __device__ __forceinline__ V load(const uint16_t* a, uint32_t i) {
        return reinterpret_cast<const uint32_t*>(a)[i];
    }
    static __device__ __forceinline__ void store(uint16_t* a, uint32_t i, V v) {
        reinterpret_cast<uint32_t*>(a)[i] = v;
    }
    static __device__ __forceinline__ uint32_t get(V v, int c) { return (v >> (16 * c)) & 0xffffu; }
    static __device__ __forceinline__ V vmax(V a, V b) { return __vmaxu2(a, b); }
    static __device__ __forceinline__ V vmin(V a, V b) { return __vminu2(a, b); }
    static __device__ __forceinline__ V dec1(V a) { return __vsub2(a, 0x00010001u); }
    static __device__ __forceinline__ V ones() { return 0xffffffffu; }
    static __device__ __forceinline__ V splat(uint32_t x) { return x | (x << 16); }
    static __device__ __forceinline__ V nzmask(V a) { return __vcmpne2(a, 0u); }
    static __device__ __forceinline__ V vand(V a, V b) { return a & b; }
    static __device__ __forceinline__ bool maybe_eq(V a, V b) {
        const uint32_t x = a ^ b;
        return ((x - 0x00010001u) & ~x & 0x80008000u) != 0;
    }
};
template <> struct Pk<4> {
    using V = uint2;
    static __device__ __forceinline__ V load(const uint16_t* a, uint32_t i) {
        return reinterpret_cast<const uint2*>(a)[i];
    }
    static __device__ __forceinline__ void store(uint16_t* a, uint32_t i, V v) {
        reinterpret_cast<uint2*>(a)[i] = v;
    }
    static __device__ __forceinline__ uint32_t get(V v, int c) {
        return ((c < 2 ? v.x : v.y) >> (16 * (c & 1))) & 0xffffu;
    }
    static __device__ __forceinline__ V vmax(V a, V b) { return make_uint2(__vmaxu2(a.x, b.x), __vmaxu2(a.y, b.y)); }
    static __device__ __forceinline__ V vmin(V a, V b) { return make_uint2(__vminu2(a.x, b.x), __vminu2(a.y, b.y)); }
    static __device__ __forceinline__ V dec1(V a) {
        return make_uint2(__vsub2(a.x, 0x00010001u), __vsub2(a.y, 0x00010001u));
    }
    static __device__ __forceinline__ V ones() { return make_uint2(0xffffffffu, 0xffffffffu); }
    static __device__ __forceinline__ V splat(uint32_t x) { return make_uint2(x | (x << 16), x | (x << 16)); }
    static __device__ __forceinline__ V nzmask(V a) { return make_uint2(__vcmpne2(a.x, 0u), __vcmpne2(a.y, 0u)); }
    static __device__ __forceinline__ V vand(V a, V b) { return make_uint2(a.x & b.x, a.y & b.y); }
    static __device__ __forceinline__ bool maybe_eq(V a, V b) {
        const uint32_t x = a.x ^ b.x, y = a.y ^ b.y;
        return ((((x - 0x00010001u) & ~x) | ((y - 0x00010001u) & ~y)) & 0x80008000u) != 0;
    }
};

// ------------------------------------------------------------- barriers --
// immediate barrier ids so ptxas reserves only the 6 barriers used
__device__ __forceinline__ void bar_sync(int id, int n) {
    switch (id) {
        case 1: asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory"); break;
        case 2: asm volatile("bar.sync 2, %0;" ::"r"(n) : "memory"); break;
        case 3: asm volatile("bar.sync 3, %0;" ::"r"(n) : "memory"); break;
        case 4: asm volatile("bar.sync 4, %0;" ::"r"(n) : "memory"); break;
        default: asm volatile("bar.sync 5, %0;" ::"r"(n) : "memory"); break;
    }
}
__device__ __forceinline__ void bar_arrive(int id, int n) {
    switch (id) {
        case 2: asm volatile("bar.arrive 2, %0;" ::"r"(n) : "memory"); break;
        case 3: asm volatile("bar.arrive 3, %0;" ::"r"(n) : "memory"); break;
        case 4: asm volatile("bar.arrive 4, %0;" ::"r"(n) : "memory"); break;
        default: asm volatile("bar.arrive 5, %0;" ::"r"(n) : "memory"); break;
    }
}

// ------------------------------------------------- bulk copy (TMA engine) --
__device__ __forceinline__ void bulk_stage(void* smem_dst, const void* gsrc, uint32_t bytes,
                                           uint64_t* mbar) {
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(mbar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
        const uint32_t chunk = 1u << 15;
        for (uint32_t o = 0; o < bytes; o += chunk) {
            const uint32_t nb = min(chunk, bytes - o);
            const uint32_t dst = (uint32_t)__cvta_generic_to_shared((char*)smem_dst + o);
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                "l"((const char*)gsrc + o), "r"(nb), "r"(bar)
                : "memory");
        }
    }
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(bar)
            : "memory");
    }
    __syncthreads();
}

// ------------------------------------------------------------ hand-off --
struct SlotHdr {
    long long k[4];
    long long peak[4];      // in size units
    double ctot[4];         // sum of compute costs (from the per-step scan)
    double basel[4];        // base + clone costs (swap-free latency)
    unsigned long long* key[4];   // [2 * cap]: unsorted keys, then sorted keys
    double* cb[4];                // compute-cost prefix before each sorted event
    int status[4];
    int nev[4];
    int cnt[4];             // gather counters
};

struct Ctl {
    int flags[4];           // per-candidate status bits (atomicOr)
    int viol[4];
    int anysw;
};

// per-group results of the cross-warp fold (written by warp 0)
struct Fold {
    long long peak[4];
    double ctot[4];
    double basel[4];
    int nev[4];
    double woff[WM];        // exclusive compute-cost prefix of each warp within its team
};

constexpr long long kNegInf = -(1ll << 62);

// MODE 0: graph tables and step slots in shared memory; 1: tables read from
// the global image; 2: tables and step slots in global memory (large graphs)
template <int P, int LMAX, int MODE>
__global__ void __launch_bounds__(TM + 32, 1)
eval2_kernel(DevGraph g, Plan2 pl, const char* __restrict__ blob, int64_t K,
             const int32_t* __restrict__ perm, const uint8_t* __restrict__ dec,
             uint8_t* __restrict__ out_status, int64_t* __restrict__ out_peak,
             double* __restrict__ out_lat, char* __restrict__ ovf, char* __restrict__ afg) {
    using PK = Pk<P>;
    using V = typename PK::V;
    extern __shared__ __align__(128) char sm[];
    __shared__ uint64_t mbar;
    __shared__ SlotHdr hdr[2];
    __shared__ Ctl ctl;
    __shared__ Fold fold;
    __shared__ long long agg_s[WM];
    __shared__ long long agg_m[WM];
    __shared__ double agg_c[WM];
    __shared__ double agg_b[WM][P];
    __shared__ int agg_n[WM][P];

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int32_t NT = pl.NT, R = pl.R, n = pl.n;
    // optional phase profile (MAGIS_PROFILE=1): cycles between marks, thread 0
    // of the main warps and lane 0 of the latency warp, summed over CTAs
    const bool prof = pl.prof && (tid == 0 || tid == TM);
    unsigned long long pt[16];
#pragma unroll
    for (int i = 0; i < 16; i++) pt[i] = 0;
    long long plast = clock64();
#define PROF_MARK(k) do { if (prof) { const long long _t = clock64(); pt[k] += _t - plast; plast = _t; } } while (0)
    const int32_t L = pl.L, S = pl.S, Sl = pl.L * pl.S, lgL = pl.lgL;

    // graph tables: staged into shared memory once per CTA (bulk copy), or
    // read in place from the global image when they do not fit
    const char* sb = MODE ? blob : sm;
    if (MODE == 0) bulk_stage(sm, blob, pl.static_bytes, &mbar);
    const uint32_t* wtab = (const uint32_t*)(sb + pl.off_wtab);   // [WM][4]: consumer rows, input rows
    const uint2* crow = (const uint2*)(sb + pl.off_crow);
    const uint32_t* chdr = (const uint32_t*)(sb + pl.off_chdr);
    const uint16_t* cent = (const uint16_t*)(sb + pl.off_cent);
    const uint2* frow = (const uint2*)(sb + pl.off_frow);
    const uint32_t* fhdr = (const uint32_t*)(sb + pl.off_fhdr);
    const uint16_t* fent = (const uint16_t*)(sb + pl.off_fent);
    const uint32_t* size_s = (const uint32_t*)(sb + pl.off_size);
    const double2* rtab = (const double2*)(sb + pl.off_rtab);       // [R] (cost(t_r), swap transfer time)
    const double* cost_s = (const double*)(sb + pl.off_cost);
    uint16_t* pos = (uint16_t*)(sm + pl.off_pos);
    uint16_t* last = (uint16_t*)(sm + pl.off_last);
    uint2* AF = MODE == 2 ? (uint2*)(afg + (size_t)blockIdx.x * pl.af_bytes)   // [P][Sl] (alloc, free)
                          : (uint2*)(sm + pl.off_af);                           // size units per step
    uint8_t* dec_s = (uint8_t*)(sm + pl.off_dec);
    double* cofs = (double*)(sm + pl.off_cofs);           // [TM] cost prefix within the warp
    double* endb_all = (double*)(sm + pl.off_end);
    unsigned long long* evk_s = (unsigned long long*)(sm + pl.off_ev);               // [2][P][2*cap]
    double* evcb_s = (double*)(sm + pl.off_ev + (size_t)2 * P * 2 * pl.evcap * 8);  // [2][P][cap]

    // pos / last of the virtual and dummy slots start (and the dummy stays) 0
    for (int i = tid; i < pl.NTX * P; i += blockDim.x) { pos[i] = 0; last[i] = 0; }
    if (tid == 0) {
        for (int c = 0; c < 4; c++) { ctl.flags[c] = 0; ctl.viol[c] = 0; }
        ctl.anysw = 0;
    }
    __syncthreads();

    const int64_t ngroups = (K + P - 1) / P;
    const int ncta = (blockIdx.x < ngroups) ? (int)((ngroups - 1 - blockIdx.x) / gridDim.x + 1) : 0;

    if (warp == WM) {
        // ================= latency sweep warp (reading P7) ==================
        for (int gi = 0; gi < ncta; gi++) {
            const int slot = gi & 1;
            PROF_MARK(13);
            bar_sync(kBarFull + slot, TM + 32);
            PROF_MARK(14);
            const SlotHdr& h = hdr[slot];
            if (lane < P) {
                const long long k = h.k[lane];
                if (k < K) {
                    const int st = h.status[lane];
                    double lat;
                    if (st) {
                        lat = __longlong_as_double(0x7ff0000000000000ll);
                    } else if (h.nev[lane] == 0) {
                        lat = h.basel[lane];
                    } else {
                        const int ne = h.nev[lane];
                        const unsigned long long* key = h.key[lane] + ne;
                        const double* cb = h.cb[lane];
                        double* endb = endb_all + (size_t)lane * 3 * R;
                        double D = 0.0, Td = 0.0, Th = 0.0;
                        // end of producer / Store / Load of r at endb[3r + 0 / 1 / 2]
                        for (int e = 0; e < ne; e++) {
                            const unsigned long long kk = key[e];
                            const uint32_t type = (uint32_t)(kk >> 24) & 0xff;
                            const int32_t r = (int32_t)(kk & 0xffffff);
                            const double c = cb[e];
                            const double2 tx = rtab[r];                 // (cost(t_r), transfer time)
                            if (type == kEvStall) {
                                D = fmax(D, endb[3 * r + 2] - c);
                            } else if (type == kEvProduce) {
                                endb[3 * r + 0] = c + D + tx.x;
                            } else if (type == kEvStore) {
                                Td = fmax(Td, endb[3 * r + 0]) + tx.y;
                                endb[3 * r + 1] = Td;
                            } else {
                                Th = fmax(Th, endb[3 * r + 1]) + tx.y;
                                endb[3 * r + 2] = Th;
                            }
                        }
                        lat = fmax(fmax(h.ctot[lane] + D, Td), Th);
                    }
                    out_status[k] = (uint8_t)st;
                    out_peak[k] = st ? -1 : h.peak[lane] * pl.unit;
                    out_lat[k] = lat;
                }
            }
            __syncwarp();
            PROF_MARK(15);
            if (gi + 2 < ncta) {
                __threadfence_block();
                bar_arrive(kBarEmpty + slot, TM + 32);
            }
        }
        if (prof)
#pragma unroll
            for (int i = 13; i < 16; i++) atomicAdd((unsigned long long*)(ovf + pl.prof_off) + i, pt[i]);
        return;
    }

    // ========================= main warps =====================================
    // phases 1 and 5: candidate cm of the group is handled by team cm (TPC
    // threads, WT warps); thread tt of the team owns steps [lo, lo + L)
    constexpr int TPC = TM / P, WT = WM / P;
    const int cm = tid / TPC, tt = tid - cm * TPC;
    const int32_t lo = tt * L;
    const bool vec4 = (NT & 3) == 0;
    for (int gi = 0; gi < ncta; gi++) {
        const int64_t grp = blockIdx.x + (int64_t)gi * gridDim.x;
        const int slot = gi & 1;
        // candidate c of this group exists iff bit c of vmask is set
        const int64_t kleft = K - grp * P;
        const uint32_t vmask = kleft >= P ? ((1u << P) - 1u) : ((1u << (uint32_t)kleft) - 1u);
        // ---- phase 0: decisions ---------------------------------------------
        {
            int sw = 0;
            uint32_t badm = 0;
            for (int i = tid; i < P * R; i += TM) {
                const int c = i / R, r = i - c * R;
                const uint8_t d = ((vmask >> c) & 1u) ? dec[(grp * P + c) * (int64_t)R + r] : 0;
                dec_s[i] = d;
                sw |= (d == 2);
                if ((d > 2) | ((d == 1) & !(__ldg(g.rflag + r) & kRHasInput))) badm |= 1u << c;
            }
            if (sw) atomicOr(&ctl.anysw, 1);
#pragma unroll
            for (int c = 0; c < P; c++)
                if ((badm >> c) & 1u) atomicOr(&ctl.flags[c], MAGIS_ST_BAD_DEC);
        }
        // ---- phase 1: inverse permutation (pos stored +1); this thread's
        //      chunk of its team's candidate stays in registers for the scan
        constexpr int LR = LMAX <= 16 ? LMAX : 1;      // perm chunk kept in registers when short
        int32_t pr[LR];
        {
            const int32_t* Pp = perm + (grp * P + cm) * (int64_t)NT + lo;
            int bad = 0;
            const bool vc = (vmask >> cm) & 1u;
#pragma unroll
            for (int j = 0; j < LMAX; j += 4) {
                int4 v = make_int4(-1, -1, -1, -1);
                if (vc && j < L && lo + j < NT) {
                    if (vec4) {
                        v = __ldcs(reinterpret_cast<const int4*>(Pp + j));
                    } else {
                        v.x = __ldcs(Pp + j);
                        if (lo + j + 1 < NT) v.y = __ldcs(Pp + j + 1);
                        if (lo + j + 2 < NT) v.z = __ldcs(Pp + j + 2);
                        if (lo + j + 3 < NT) v.w = __ldcs(Pp + j + 3);
                    }
                    const uint32_t i0 = (uint32_t)(lo + j);
                    if ((uint32_t)v.x < (uint32_t)NT) pos[v.x * P + cm] = (uint16_t)(i0 + 1); else bad = 1;
                    if (i0 + 1 < (uint32_t)NT) {
                        if ((uint32_t)v.y < (uint32_t)NT) pos[v.y * P + cm] = (uint16_t)(i0 + 2); else bad = 1;
                    }
                    if (i0 + 2 < (uint32_t)NT) {
                        if ((uint32_t)v.z < (uint32_t)NT) pos[v.z * P + cm] = (uint16_t)(i0 + 3); else bad = 1;
                    }
                    if (i0 + 3 < (uint32_t)NT) {
                        if ((uint32_t)v.w < (uint32_t)NT) pos[v.w * P + cm] = (uint16_t)(i0 + 4); else bad = 1;
                    }
                }
                if (LMAX <= 16) {
                    pr[j % LR] = v.x;
                    if (j + 1 < LR) pr[(j + 1) % LR] = v.y;
                    if (j + 2 < LR) pr[(j + 2) % LR] = v.z;
                    if (j + 3 < LR) pr[(j + 3) % LR] = v.w;
                }
            }
            if (bad) atomicOr(&ctl.flags[cm], MAGIS_ST_NOT_PERM);
        }
        bar_sync(kBarMain, TM);
        PROF_MARK(1);
        const bool anysw = ctl.anysw != 0;
        // ---- phase 2: optional nodes, virtual late-user slots ------------------
        double bl[P];
        int nev[P];
#pragma unroll
        for (int c = 0; c < P; c++) { bl[c] = 0.0; nev[c] = 0; }
        for (int q = tid; q < P * R; q += TM) {
            const int c = q / R, r = q - c * R;
            const int32_t u0 = __ldg(g.U_ptr + r), u1 = __ldg(g.U_ptr + r + 1);
#pragma unroll
            for (int cc = 0; cc < P; cc++) {
                if (cc != c || !((vmask >> cc) & 1u)) continue;
                const uint8_t d = dec_s[cc * R + r];
#pragma unroll
                for (int o = 0; o < 3; o++) {
                    const int32_t id = n + 3 * r + o;
                    const uint32_t p = pos[id * P + cc];
                    if (p == 0) {
                        atomicOr(&ctl.flags[cc], MAGIS_ST_NOT_PERM);
                        continue;
                    }
                    const bool act = (o == 0) ? (d == 1) : (d == 2);
                    if (!act) {
                        const uint32_t st = p - 1;
                        AF[cc * Sl + (st & (L - 1)) * S + (st >> lgL)] = make_uint2(0u, 0u);
                        pos[id * P + cc] = 0;
                    }
                }
                if (d == 1) bl[cc] += __ldg(g.tcost + r);
                if (d == 2) nev[cc] += 3 + (u1 - u0);
                for (int32_t j = u0; j < u1; j++) {
                    const int32_t b = __ldg(g.U_idx + j);
                    pos[(NT + j) * P + cc] = (d == 0) ? pos[b * P + cc] : (uint16_t)0;
                }
            }
        }
        bar_sync(kBarMain, TM);
        PROF_MARK(2);
        // ---- phase 3: validity + last use over the consumer rows -----------------
        {
            int nperm = 0, viol = 0;
            const uint32_t r0 = wtab[warp * 4 + 0], r1 = wtab[warp * 4 + 1];
            for (uint32_t r = r0; r < r1; r++) {
                const uint2 rw = crow[r];                     // (edge offset, degree): warp-uniform
                const uint32_t h = chdr[r * 32 + lane];
                const uint32_t kind = h >> kKindShift, id = h & kIdMask;
                const V p = PK::load(pos, id);
                V lst = p, mn = PK::ones();
                const uint16_t* ent = cent + rw.x + lane;
#pragma unroll 4
                for (uint32_t j = 0; j < rw.y; j++) {
                    const V q = PK::load(pos, ent[j * 32]);
                    mn = PK::vmin(mn, PK::dec1(q));
                    lst = PK::vmax(lst, q);
                }
                if (kind != kNop) {
#pragma unroll
                    for (int c = 0; c < P; c++) {
                        const uint32_t pc = PK::get(p, c);
                        if (kind < kHdrClone && pc == 0) nperm |= 1 << c;
                        if (PK::get(mn, c) < pc) viol |= 1 << c;
                    }
                    V outv;
                    if (kind == kHdrOut) outv = PK::splat((uint32_t)NT);
                    else if (kind >= kHdrClone) outv = PK::vand(lst, PK::nzmask(p));   // inactive halves -> 0
                    else outv = lst;
                    PK::store(last, id, outv);
                }
            }
#pragma unroll
            for (int c = 0; c < P; c++) {
                if (nperm & (1 << c)) atomicOr(&ctl.flags[c], MAGIS_ST_NOT_PERM);
                if (viol & (1 << c)) atomicOr(&ctl.viol[c], MAGIS_ST_EDGE);
            }
        }
        bar_sync(kBarMain, TM);
        PROF_MARK(3);
        // per-candidate status, 4 bits each; okm: valid candidates with status 0
        uint32_t stm = 0, okm = 0;
#pragma unroll
        for (int c = 0; c < P; c++) {
            const int f = ctl.flags[c];
            const uint32_t st = ((vmask >> c) & 1u) ? (uint32_t)(f ? f : ctl.viol[c]) : 0u;
            stm |= st << (4 * c);
            if (((vmask >> c) & 1u) && st == 0) okm |= 1u << c;
        }
        const bool anyok = okm != 0;
        if (anyok) {
            // ---- phase 4: frees over the input rows -> per-step slots ------------
            {
                const uint32_t r0 = wtab[warp * 4 + 2], r1 = wtab[warp * 4 + 3];
                for (uint32_t r = r0; r < r1; r++) {
                    const uint2 rw = frow[r];
                    const uint32_t h = fhdr[r * 32 + lane];
                    const uint32_t kind = h >> kKindShift, id = h & kIdMask;
                    const V p = PK::load(pos, id);
                    const V lv = PK::load(last, id);
                    const uint32_t A = size_s[id];
                    uint32_t fr[P];
#pragma unroll
                    for (int c = 0; c < P; c++) {
                        const uint32_t pc = PK::get(p, c);
                        fr[c] = (pc != 0 && PK::get(lv, c) == pc) ? A : 0u;   // no reader: freed after own step
                    }
                    const uint16_t* ent = fent + rw.x + lane;
#pragma unroll 4
                    for (uint32_t j = 0; j < rw.y; j++) {
                        const uint32_t u = ent[j * 32];
                        const V l = PK::load(last, u);
                        if (PK::maybe_eq(l, p)) {
                            const uint32_t su = size_s[u];
#pragma unroll
                            for (int c = 0; c < P; c++) {
                                const uint32_t pc = PK::get(p, c);
                                if (pc != 0 && PK::get(l, c) == pc) fr[c] += su;
                            }
                        }
                    }
                    if (kind != kNop) {
#pragma unroll
                        for (int c = 0; c < P; c++) {
                            const uint32_t pc = PK::get(p, c);
                            if (pc == 0 || !((okm >> c) & 1u)) continue;
                            const uint32_t st = pc - 1;
                            AF[c * Sl + (st & (L - 1)) * S + (st >> lgL)] = make_uint2(A, fr[c]);
                        }
                    }
                }
            }
            bar_sync(kBarMain, TM);
            PROF_MARK(4);
            // ---- phase 5: scan of the (sum, max-prefix) monoid ------------------
            //      team cm scans candidate cm: alloc = size of the op at each step
            //      (perm chunk in registers), free = Fs slot, compute cost per step
            long long s1 = 0, m1 = kNegInf;
            double cs1 = 0.0;
            const int32_t nst = ((okm >> cm) & 1u) ? min(L, NT - lo) : 0;   // steps of this chunk
#pragma unroll
            for (int j = 0; j < LMAX; j++) {
                if (j < nst) {
                    const uint2 af = AF[cm * Sl + j * S + tt];     // alloc / free of the step (units)
                    s1 += af.x;
                    m1 = max(m1, s1);
                    s1 -= af.y;
                    if (anysw) {
                        const int32_t v = LMAX <= 16 ? pr[j % LR]
                                                     : __ldg(perm + (grp * P + cm) * (int64_t)NT + lo + j);
                        if (v < n || pos[v * P + cm] != 0) cs1 += cost_s[v];
                    }
                }
            }
            {
                // warp-level monoid scan: (s1, m1) then (s2, m2) = (s1 + s2, max(m1, s1 + m2))
                long long ss = s1, mm = m1;
                double cc = cs1;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const long long ps = __shfl_up_sync(0xffffffffu, ss, o);
                    const long long pm = __shfl_up_sync(0xffffffffu, mm, o);
                    const double pc = __shfl_up_sync(0xffffffffu, cc, o);
                    if (lane >= o) { mm = max(pm, ps + mm); ss = ps + ss; cc = pc + cc; }
                }
                if (anysw) cofs[tid] = cc - cs1;
                if (lane == 31) { agg_s[warp] = ss; agg_m[warp] = mm; agg_c[warp] = cc; }
#pragma unroll
                for (int c = 0; c < P; c++) {
                    double b = bl[c];
                    int nn = nev[c];
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) {
                        b += __shfl_xor_sync(0xffffffffu, b, o);
                        nn += __shfl_xor_sync(0xffffffffu, nn, o);
                    }
                    if (lane == 0) { agg_b[warp][c] = b; agg_n[warp][c] = nn; }
                }
            }
            bar_sync(kBarMain, TM);
            PROF_MARK(5);
            if (warp == 0) {
                // fold the WT warp aggregates of each team (segments of WT lanes)
                long long ss = lane < WM ? agg_s[lane] : 0;
                long long mm = lane < WM ? agg_m[lane] : kNegInf;
                double cc = lane < WM ? agg_c[lane] : 0.0;
                const double c0 = cc;
#pragma unroll
                for (int o = 1; o < WT; o <<= 1) {
                    const long long ps = __shfl_up_sync(0xffffffffu, ss, o, WT);
                    const long long pm = __shfl_up_sync(0xffffffffu, mm, o, WT);
                    const double pc = __shfl_up_sync(0xffffffffu, cc, o, WT);
                    if ((lane % WT) >= o) { mm = max(pm, ps + mm); ss = ps + ss; cc = pc + cc; }
                }
                if (lane < WM) fold.woff[lane] = cc - c0;
                if (lane < WM && (lane % WT) == WT - 1) {
                    const int c = lane / WT;
                    fold.peak[c] = mm;
                    fold.ctot[c] = cc;
                }
#pragma unroll
                for (int c = 0; c < P; c++) {
                    double b = lane < WM ? agg_b[lane][c] : 0.0;
                    int nn = lane < WM ? agg_n[lane][c] : 0;
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) {
                        b += __shfl_xor_sync(0xffffffffu, b, o);
                        nn += __shfl_xor_sync(0xffffffffu, nn, o);
                    }
                    if (lane == 0) {
                        fold.basel[c] = g.base_cost + b;
                        fold.nev[c] = ((okm >> c) & 1u) ? nn : 0;
                    }
                }
            }
            bar_sync(kBarMain, TM);
            PROF_MARK(6);
        } else if (tid == 0) {
#pragma unroll
            for (int c = 0; c < P; c++) { fold.peak[c] = 0; fold.ctot[c] = 0.0; fold.basel[c] = 0.0; fold.nev[c] = 0; }
        }
        int nevt[P];
        bool anyev = false;
#pragma unroll
        for (int c = 0; c < P; c++) {
            nevt[c] = anyok ? fold.nev[c] : 0;
            anyev |= nevt[c] > 0;
        }
        // ---- phase 6: swap events -> hand-off slot --------------------------------
        if (gi >= 2) bar_sync(kBarEmpty + slot, TM + 32);
        PROF_MARK(7);
        SlotHdr& h = hdr[slot];
        if (tid == 0) {
#pragma unroll
            for (int c = 0; c < P; c++) {
                h.k[c] = ((vmask >> c) & 1u) ? grp * P + c : LLONG_MAX;
                h.status[c] = (int)((stm >> (4 * c)) & 15u);
                h.peak[c] = fold.peak[c];
                h.ctot[c] = fold.ctot[c];
                h.basel[c] = fold.basel[c];
                h.nev[c] = nevt[c];
                h.cnt[c] = 0;
                if (nevt[c] <= pl.evcap) {
                    h.key[c] = evk_s + (size_t)(slot * P + c) * 2 * pl.evcap;
                    h.cb[c] = evcb_s + (size_t)(slot * P + c) * pl.evcap;
                } else {
                    char* ob = ovf + ((size_t)blockIdx.x * 8 + slot * 4 + c) * pl.ovf_stride;
                    h.key[c] = (unsigned long long*)ob;
                    h.cb[c] = (double*)(ob + (size_t)2 * pl.max_events * 8);
                }
            }
        }
        if (anyev) {
            bar_sync(kBarMain, TM);
            PROF_MARK(8);
            for (int q = tid; q < P * R; q += TM) {
                const int c0 = q / R, r = q - c0 * R;
                const int32_t u0 = __ldg(g.U_ptr + r), u1 = __ldg(g.U_ptr + r + 1);
                const unsigned long long rr = (unsigned long long)r;
#pragma unroll
                for (int c = 0; c < P; c++) {
                    if (c != c0 || nevt[c] == 0 || dec_s[c * R + r] != 2) continue;
                    const int b0 = atomicAdd(&h.cnt[c], 3 + (u1 - u0));
                    unsigned long long* kin = h.key[c];
                    const unsigned long long pt = (unsigned long long)pos[__ldg(g.elig + r) * P + c] - 1;
                    const unsigned long long ps = (unsigned long long)pos[(n + 3 * r + 1) * P + c] - 1;
                    const unsigned long long pq = (unsigned long long)pos[(n + 3 * r + 2) * P + c] - 1;
                    kin[b0 + 0] = (pt << 32) | ((unsigned long long)kEvProduce << 24) | rr;
                    kin[b0 + 1] = (ps << 32) | ((unsigned long long)kEvStore << 24) | rr;
                    kin[b0 + 2] = (pq << 32) | ((unsigned long long)kEvLoad << 24) | rr;
                    for (int32_t j = u0; j < u1; j++) {
                        const unsigned long long pb = (unsigned long long)pos[__ldg(g.U_idx + j) * P + c] - 1;
                        kin[b0 + 3 + (j - u0)] = (pb << 32) | ((unsigned long long)kEvStall << 24) | rr;
                    }
                }
            }
            bar_sync(kBarMain, TM);
            PROF_MARK(9);
            // rank sort (unique keys) + compute-cost prefix before each event:
            // cost of the steps of earlier warps' chunks, earlier lanes of the
            // same warp, then the steps of the owning chunk before the event
            int tot = 0;
#pragma unroll
            for (int c = 0; c < P; c++) tot += nevt[c];
            for (int q = tid; q < tot; q += TM) {
                int c = 0, e = q;
                while (e >= nevt[c]) { e -= nevt[c]; c++; }
                const unsigned long long* kin = h.key[c];
                const int ne = nevt[c];
                const unsigned long long key = kin[e];
                int rank = 0;
                for (int j = 0; j < ne; j++) rank += (kin[j] < key);
                const int32_t stp = (int32_t)(key >> 32);
                const int32_t th = stp >> lgL;
                double cb = fold.woff[c * WT + (th >> 5)] + cofs[c * TPC + th];
                const int32_t* Pp = perm + (grp * P + c) * (int64_t)NT + th * L;
                const int32_t nb = stp - th * L;
#pragma unroll 4
                for (int32_t i = 0; i < nb; i++) {
                    const int32_t v = __ldg(Pp + i);
                    if (v < n || pos[v * P + c] != 0) cb += cost_s[v];
                }
                h.key[c][ne + rank] = key;
                h.cb[c][rank] = cb;
            }
        }
        __threadfence_block();
        bar_arrive(kBarFull + slot, TM + 32);
        PROF_MARK(10);
        // reset the per-group control words for the next group, then make sure
        // every main thread is done with pos / Fs / ctl before they are reused
        if (tid == 0) {
            for (int c = 0; c < 4; c++) { ctl.flags[c] = 0; ctl.viol[c] = 0; }
            ctl.anysw = 0;
        }
        // every main thread must be done reading pos (event keys, cost prefix)
        if (anyev) bar_sync(kBarMain, TM);
        PROF_MARK(11);
        // clear pos so a missing node (duplicate in perm) reads as 0 next group
        {
            const int nb = NT * P * 2;
            uint4* p4 = reinterpret_cast<uint4*>(pos);
            for (int i = tid; i < (nb >> 4); i += TM) p4[i] = make_uint4(0u, 0u, 0u, 0u);
            for (int i = ((nb >> 4) << 3) + tid; i < NT * P; i += TM) pos[i] = 0;
        }
        bar_sync(kBarMain, TM);
        PROF_MARK(12);
    }
    if (prof)
#pragma unroll
        for (int i = 1; i < 13; i++) atomicAdd((unsigned long long*)(ovf + pl.prof_off) + i, pt[i]);
}

template <int P, int MODE>
static const void* kernel_ptr(int lmax) {
    if constexpr (MODE == 0) {
        if (lmax <= 4) return (const void*)eval2_kernel<P, 4, 0>;
        if (lmax <= 8) return (const void*)eval2_kernel<P, 8, 0>;
        if (lmax <= 16) return (const void*)eval2_kernel<P, 16, 0>;
        return (const void*)eval2_kernel<P, 32, 0>;
    } else {
        if (lmax <= 16) return (const void*)eval2_kernel<P, 16, MODE>;
        if (lmax <= 32) return (const void*)eval2_kernel<P, 32, MODE>;
        return (const void*)eval2_kernel<P, 64, MODE>;
    }
}

template <int MODE>
static const void* kernel_mode(const Plan2& pl) {
    return pl.P == 4 ? kernel_ptr<4, MODE>(pl.L) : pl.P == 2 ? kernel_ptr<2, MODE>(pl.L) : kernel_ptr<1, MODE>(pl.L);
}

static const void* kernel_for(const Plan2& pl) {
    const int mode = pl.gmem_af ? 2 : (pl.gmem_static ? 1 : 0);
    return mode == 0 ? kernel_mode<0>(pl) : mode == 1 ? kernel_mode<1>(pl) : kernel_mode<2>(pl);
}

cudaError_t eval2_occupancy(const Plan2& pl, int* blocks) {
    if (pl.L > 64 || (!pl.gmem_static && pl.L > 32)) { *blocks = 0; return cudaSuccess; }
    const void* fn = kernel_for(pl);
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem_total);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
    if (e != cudaSuccess) return e;
    if (std::getenv("MAGIS_DEBUG")) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, fn);
        std::fprintf(stderr, "[magis] eval2 P=%d regs=%d static_smem=%zu local=%zu\n", pl.P, fa.numRegs,
                     fa.sharedSizeBytes, fa.localSizeBytes);
    }
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, TM + 32, pl.smem_total);
}

cudaError_t eval2_launch(const DevGraph& g, const Plan2& pl, const void* blob, void* ovf, void* afg, int grid,
                         int64_t K, const int32_t* perm, const uint8_t* dec, uint8_t* status,
                         int64_t* peak, double* lat, cudaStream_t stream) {
    if (K <= 0) return cudaSuccess;
    const int64_t ngroups = (K + pl.P - 1) / pl.P;
    const int gr = (int)std::min<int64_t>(grid, ngroups);
    void* args[] = {(void*)&g, (void*)&pl, (void*)&blob, (void*)&K, (void*)&perm, (void*)&dec,
                    (void*)&status, (void*)&peak, (void*)&lat, (void*)&ovf, (void*)&afg};
    return cudaLaunchKernel(kernel_for(pl), dim3(gr), dim3(TM + 32), args, pl.smem_total, stream);
}

}  // namespace magis
