// magis_eval2_kernel.cuh -- the shared-memory-resident evaluation kernel (variant 2).
// Included by the per-mode translation units magis_eval2_m*.cu (compiled in
// parallel); the host side (dispatch, occupancy, launch) is magis_eval2.cu.
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
//  * alloc/free amounts land in per-step slots (u32 size units; tier 2: one
//    signed delta) laid out st + st / L, one pad word per scan chunk, so the
//    scan's per-thread contiguous chunks read conflict-free (odd stride);
//  * swap latency (the three in-order queues of reading P7): the steps that
//    raise swap events are marked in a per-candidate bitmap while the gates
//    are resolved (phase 2); the scan threads emit their marked steps with the
//    compute-cost prefix in step order (a warp scan of mark counts gives each
//    thread its slot, so no sort is needed), and one latency warp per
//    candidate walks them.  The hand-off is double-buffered in shared memory
//    and guarded by named barriers, so the main warps go on to the next group
//    while the latency warps run.
#pragma once
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "magis_internal.h"

namespace magis {

constexpr uint32_t kKindShift = 29;
constexpr uint32_t kIdMask = (1u << kKindShift) - 1;
constexpr uint32_t kHdrOut = 2, kHdrClone = 3, kNop = 7;   // kHdr = 1, kHdrCopy = 4, kHdrGated = 5
// named barriers of team t: main 1 + 5t, FULL 2 + 5t + slot, EMPTY 4 + 5t + slot
constexpr int kBarMain = 1, kBarFull = 2, kBarEmpty = 4, kBarTeam = 5;

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
// immediate barrier ids so ptxas reserves only the barriers used (5 per team)
__device__ __forceinline__ void bar_sync(int id, int n) {
    switch (id) {
        case 1: asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory"); break;
        case 2: asm volatile("bar.sync 2, %0;" ::"r"(n) : "memory"); break;
        case 3: asm volatile("bar.sync 3, %0;" ::"r"(n) : "memory"); break;
        case 4: asm volatile("bar.sync 4, %0;" ::"r"(n) : "memory"); break;
        case 5: asm volatile("bar.sync 5, %0;" ::"r"(n) : "memory"); break;
        case 6: asm volatile("bar.sync 6, %0;" ::"r"(n) : "memory"); break;
        case 7: asm volatile("bar.sync 7, %0;" ::"r"(n) : "memory"); break;
        case 8: asm volatile("bar.sync 8, %0;" ::"r"(n) : "memory"); break;
        case 9: asm volatile("bar.sync 9, %0;" ::"r"(n) : "memory"); break;
        default: asm volatile("bar.sync 10, %0;" ::"r"(n) : "memory"); break;
    }
}
__device__ __forceinline__ void bar_arrive(int id, int n) {
    switch (id) {
        case 2: asm volatile("bar.arrive 2, %0;" ::"r"(n) : "memory"); break;
        case 3: asm volatile("bar.arrive 3, %0;" ::"r"(n) : "memory"); break;
        case 4: asm volatile("bar.arrive 4, %0;" ::"r"(n) : "memory"); break;
        case 5: asm volatile("bar.arrive 5, %0;" ::"r"(n) : "memory"); break;
        case 7: asm volatile("bar.arrive 7, %0;" ::"r"(n) : "memory"); break;
        case 8: asm volatile("bar.arrive 8, %0;" ::"r"(n) : "memory"); break;
        case 9: asm volatile("bar.arrive 9, %0;" ::"r"(n) : "memory"); break;
        default: asm volatile("bar.arrive 10, %0;" ::"r"(n) : "memory"); break;
    }
}

// ------------------------------------------------- bulk copy (TMA engine) --
// one or two global ranges -> shared memory (sizes and addresses 16-byte aligned)
__device__ __forceinline__ void bulk_stage(void* smem_dst, const void* gsrc, uint32_t bytes,
                                           uint64_t* mbar, void* smem_dst2 = nullptr,
                                           const void* gsrc2 = nullptr, uint32_t bytes2 = 0) {
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(mbar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes + bytes2) : "memory");
        const uint32_t chunk = 1u << 15;
        for (int part = 0; part < 2; part++) {
            char* d = (char*)(part ? smem_dst2 : smem_dst);
            const char* src = (const char*)(part ? gsrc2 : gsrc);
            const uint32_t nbytes = part ? bytes2 : bytes;
            for (uint32_t o = 0; o < nbytes; o += chunk) {
                const uint32_t nb = min(chunk, nbytes - o);
                const uint32_t dst = (uint32_t)__cvta_generic_to_shared(d + o);
                asm volatile(
                    "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                    "l"(src + o), "r"(nb), "r"(bar)
                    : "memory");
            }
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
// Main warps -> latency warp, one slot per group parity.  Per candidate: the
// steps that raise swap events, in step order, as (step << 32 | node) keys
// with the compute-cost prefix before the step minus the exclusive prefix of
// the owning warp (woff, added by the latency warp), plus the decisions.
struct SlotHdr {
    long long k[4];
    int status[4];
    int nev[4];
    int swp[4];             // candidate swaps some tensor
};

struct Ctl {
    int flags[4];           // per-candidate status bits (atomicOr)
    int viol[4];
    int swm;                // bit c: candidate c swaps some tensor
};

constexpr long long kNegInf = -(1ll << 62);

// mark bits of steps [lo, lo + 64) (the caller masks to its chunk length)
__device__ __forceinline__ unsigned long long mark_bits(const uint32_t* m, int32_t lo) {
    const int32_t w = lo >> 5, sh = lo & 31;
    const unsigned long long a = (unsigned long long)m[w] | ((unsigned long long)m[w + 1] << 32);
    return sh ? (a >> sh) | ((unsigned long long)m[w + 2] << (64 - sh)) : a;
}

struct WalkTabs {
    const uint2* ninfo;
    const uint16_t* lul;
    const double2* rtab;
    int32_t n;
    uint32_t Lm;          // ceil(2^32 / L): step / L = umulhi(step, Lm) (exact for steps < 2^16)
};

// The event steps of a swapping candidate are resolved by the whole latency
// warp (one lane per event) into compact records, so the serial walk (lane 0)
// only chases the queue recurrences:
//   ia (u64): bits 62-63 kind (0 compute, 1 Store, 2 Load); compute: bits
//             48-52 number of swapped tensors the op reads (late-user
//             stalls), bits 0-47 the first three of them (16 bits each)
//   ib (u64): Store / Load: r; compute: bits 0-15 r + 1 of the swapped tensor
//             it produces (0 none), bits 16-46 the swapped mask over the node's
//             late-user list, bits 47-62 the list's offset in lul (used only
//             with more than three stalls)
//   x (f64):  compute: compute-cost prefix before the step; Store / Load:
//             the transfer time lambda + |t_r| / B
__device__ __forceinline__ void resolve_event(unsigned long long& kslot, double& cslot, unsigned long long& islot,
                                              const double* woff, const uint8_t* dd, const WalkTabs& t) {
    const unsigned long long kk = kslot;
    const int32_t stp = (int32_t)(kk >> 32), w = (int32_t)(kk & 0xffffffffu);
    if (w < t.n) {
        const uint2 x = t.ninfo[w];
        const uint32_t rt = x.x & 0xffffu, cnt = x.x >> 16;
        uint32_t m = 0, nw = 0;
        unsigned long long pk = 0;
        for (uint32_t i = 0; i < cnt; i++) {
            const uint32_t r = t.lul[x.y + i];
            if (dd[r] == 2) {
                m |= 1u << i;
                if (nw < 3) pk |= (unsigned long long)r << (16 * nw);
                nw++;
            }
        }
        const bool prod = rt && dd[rt - 1] == 2;
        islot = pk | ((unsigned long long)nw << 48);
        kslot = (unsigned long long)(prod ? rt : 0u) | ((unsigned long long)m << 16) |
                ((unsigned long long)x.y << 47);
        cslot += woff[__umulhi((uint32_t)stp, t.Lm) >> 5];
    } else {
        const uint32_t q = (uint32_t)(w - t.n), r = q / 3, o = q - 3 * r;   // o: 1 Store, 2 Load
        islot = (unsigned long long)o << 62;
        kslot = r;
        cslot = t.rtab[r].y;
    }
}

// The three in-order queues of reading P7 over the resolved records (step
// order): a compute op first stalls on the Loads of the swapped tensors it
// reads, then ends (if it produces a swapped tensor); Store / Load ops run on
// the D2H / H2D queues.  endb[3r + 0 / 1 / 2] = end of producer / Store /
// Load of tensor r.
__device__ __forceinline__ void walk_events(const unsigned long long* ia, const unsigned long long* ib,
                                            const double* xs, int ne, double* endb, const WalkTabs& t,
                                            double& D, double& Td, double& Th) {
    unsigned long long an = ne > 0 ? ia[0] : 0ull, bn = ne > 0 ? ib[0] : 0ull;
    double xn = ne > 0 ? xs[0] : 0.0;
    for (int e = 0; e < ne; e++) {
        const unsigned long long a = an, b = bn;
        const double x = xn;
        if (e + 1 < ne) { an = ia[e + 1]; bn = ib[e + 1]; xn = xs[e + 1]; }   // next record in flight
        const uint32_t kind = (uint32_t)(a >> 62);
        const uint32_t r = (uint32_t)b & 0xffffu;
        if (kind == 0) {
            const uint32_t nw = (uint32_t)(a >> 48) & 31u;
            if (nw <= 3) {
                if (nw > 0) D = fmax(D, endb[3 * ((uint32_t)a & 0xffffu) + 2] - x);
                if (nw > 1) D = fmax(D, endb[3 * ((uint32_t)(a >> 16) & 0xffffu) + 2] - x);
                if (nw > 2) D = fmax(D, endb[3 * ((uint32_t)(a >> 32) & 0xffffu) + 2] - x);
            } else {
                uint32_t m = (uint32_t)(b >> 16) & 0x7fffffffu;
                const uint32_t off = (uint32_t)(b >> 47) & 0xffffu;
                while (m) {
                    const uint32_t i = __ffs(m) - 1;
                    m &= m - 1;
                    D = fmax(D, endb[3 * (uint32_t)t.lul[off + i] + 2] - x);
                }
            }
            if (r) endb[3 * (r - 1)] = x + D + t.rtab[r - 1].x;             // producer of a swapped tensor ends
        } else if (kind == 1) {
            Td = fmax(Td, endb[3 * r]) + x;                                  // Store
            endb[3 * r + 1] = Td;
        } else {
            Th = fmax(Th, endb[3 * r + 1]) + x;                              // Load
            endb[3 * r + 2] = Th;
        }
    }
}

// Latency of one swapping candidate from its event steps (key, cb in step
// order): the warp resolves every step in parallel, then lane 0 walks them.
__device__ __forceinline__ double candidate_latency(unsigned long long* key, double* cbp, unsigned long long* inf,
                                                    int ne, const double* woff, const uint8_t* dd, double* endb,
                                                    const WalkTabs& t, double ctot, int lane) {
    for (int e = lane; e < ne; e += 32) resolve_event(key[e], cbp[e], inf[e], woff, dd, t);
    __syncwarp();
    double lat = 0.0;
    if (lane == 0) {
        double D = 0.0, Td = 0.0, Th = 0.0;
        walk_events(inf, key, cbp, ne, endb, t, D, Td, Th);
        lat = fmax(fmax(ctot + D, Td), Th);
    }
    return lat;
}

// MODE 0: graph tables and step slots in shared memory; 1: tables read from
// the global image; 2: tables and step slots in global memory (large graphs);
// 3: tables read from the global image, one signed delta per step in shared
// memory (large graphs whose (alloc, free) slots do not fit).
// TEAMS: independent teams per CTA (each TM main threads + its latency warps,
// its own per-group state, slots and named barriers; the tables are shared),
// so one team's barrier waits overlap the other's work.
// AM: also emit the first argmax step of the memory curve (SURVEY §8(a) a7's
// optional output: the step whose allocation first reaches M_peak),
// carried as a third monoid field; a separate instantiation, so the default
// kernels are unchanged.
template <int P, int LMAX, int MODE, int TEAMS, bool AM>
__global__ void __launch_bounds__(TEAMS * (kMainThreads2 / TEAMS + 32 * P) < 1024 ? TEAMS * (kMainThreads2 / TEAMS + 32 * P) : 1024, 1)
eval2_kernel(DevGraph g, Plan2 pl, const char* __restrict__ blob, int64_t K,
             const int32_t* __restrict__ perm, const uint8_t* __restrict__ dec,
             uint8_t* __restrict__ out_status, int64_t* __restrict__ out_peak,
             double* __restrict__ out_lat, char* __restrict__ ovf, char* __restrict__ afg,
             int32_t* __restrict__ out_arg) {
    using PK = Pk<P>;
    using V = typename PK::V;
    constexpr int TM = kMainThreads2 / TEAMS;  // main threads of a team
    constexpr int WM = TM / 32;
    constexpr int TL = 32 * P;                 // latency warps: one per candidate of a group
    // per-step slots in shared memory: phase 3 scatters alloc / free into them
    // (smem atomics); in global memory (MODE 2) phase 4 gathers the frees instead
    constexpr bool kScatter = MODE != 2;
    constexpr bool kFO = MODE == 3;            // (tier 2) int32 delta slots: D[i] = alloc(i) - free(i - 1)
    extern __shared__ __align__(128) char sm_all[];
    __shared__ uint64_t mbar;
    __shared__ SlotHdr hdr_t[TEAMS][2];
    __shared__ Ctl ctl_t[TEAMS][2];            // per group parity (reset one group ahead)
    __shared__ long long agg_s_t[TEAMS][2][WM];   // per slot: warp aggregates of the scan,
    __shared__ long long agg_m_t[TEAMS][2][WM];   //   folded by the latency warps
    __shared__ int agg_a_t[TEAMS][2][AM ? WM : 1];   // AM: first argmax step of each warp's max-prefix
    __shared__ double agg_c_t[TEAMS][2][WM];
    __shared__ double lwoff_t[TEAMS][4][WM];   // per latency warp: cost prefix of each team warp
    __shared__ int wcnt_t[TEAMS][WM];          // event steps per warp chunk

    const int team = TEAMS == 1 ? 0 : (int)(threadIdx.x / (TM + TL));
    const int tid = (int)threadIdx.x - team * (TM + TL), lane = tid & 31, warp = tid >> 5;
    const int bb = kBarTeam * team;            // this team's barrier ids: kBar* + bb
    const int64_t cta = (int64_t)blockIdx.x * TEAMS + team, ncta_all = (int64_t)gridDim.x * TEAMS;
    SlotHdr* hdr = hdr_t[team];
    Ctl* ctl = ctl_t[team];
    long long (*agg_s)[WM] = agg_s_t[team];
    long long (*agg_m)[WM] = agg_m_t[team];
    int (*agg_a)[AM ? WM : 1] = agg_a_t[team];
    double (*agg_c)[WM] = agg_c_t[team];
    double (*lwoff)[WM] = lwoff_t[team];
    int* wcnt = wcnt_t[team];
    // this team's state: the static tables (MODE 0) are shared, the state follows at + team * stride
    char* sm = sm_all + (size_t)team * pl.state_stride;
    const int32_t NT = pl.NT, R = pl.R, n = pl.n;
    const int32_t gate_lo = pl.gate_lo;      // ids >= gate_lo may be absent in a candidate
    // optional phase profile (MAGIS_PROFILE=1): cycles between marks, thread 0
    // of the main warps and lane 0 of the latency warp, summed over CTAs
    const bool prof = pl.prof && (tid == 0 || tid == TM);
    unsigned long long pt[16];
#pragma unroll
    for (int i = 0; i < 16; i++) pt[i] = 0;
    long long plast = clock64();
#define PROF_MARK(k) do { if (prof) { const long long _t = clock64(); pt[k] += _t - plast; plast = _t; } } while (0)
    // per-step slots of a candidate: step st at st + st / L (one pad word per scan
    // chunk of L steps, L a multiple of 4), so thread tt's chunk [tt L, tt L + L)
    // is contiguous at tt (L + 1) and the lanes of a warp read it conflict-free
    // (odd stride); st / L = umulhi(st, Lm)
    const int32_t L = pl.L, S = pl.S, Sl = ((pl.L + 1) * pl.S + 3) & ~3;
    const uint32_t Lm = pl.Lm;

    // graph tables: staged into shared memory once per CTA (bulk copy), or
    // read in place from the global image when they do not fit
    const char* sb = MODE ? blob : sm_all;
    if (MODE == 0) bulk_stage(sm_all, blob, pl.static_bytes, &mbar);
    else if (pl.cost_sm)
        bulk_stage(sm_all, blob + (pl.cost_cls ? pl.off_ccls : pl.off_cost), pl.stage_bytes, &mbar,
                   sm_all + pl.rows_off, blob + pl.off_wtab, pl.rows_bytes);
    // tier 1 with rows_sm: the consumer-row tables [wtab, crow, chdr, cent] were staged too
    const char* sr = (MODE == 1 && pl.rows_sm) ? (const char*)sm_all + pl.rows_off - pl.off_wtab : sb;
    const uint32_t* wtab = (const uint32_t*)(sr + pl.off_wtab);   // [WM][4]: consumer rows, input rows
    const uint2* crow = (const uint2*)(sr + pl.off_crow);
    const uint32_t* chdr = (const uint32_t*)(sr + pl.off_chdr);
    const uint32_t* csize = (const uint32_t*)(sb + pl.off_csize);   // size units of each header, row order
    const uint16_t* cent = (const uint16_t*)(sr + pl.off_cent);
    const uint2* frow = (const uint2*)(sb + pl.off_frow);
    const uint32_t* fhdr = (const uint32_t*)(sb + pl.off_fhdr);
    const uint16_t* fent = (const uint16_t*)(sb + pl.off_fent);
    const uint32_t* size_s = (const uint32_t*)(sb + pl.off_size);
    const double2* rtab = (const double2*)(sb + pl.off_rtab);       // [R] (cost(t_r), swap transfer time)
    const double* cost_s = (MODE != 0 && pl.cost_sm) ? (const double*)sm_all : (const double*)(sb + pl.off_cost);
    // tier 2 with cost classes: cost(v) = class value [class index of v], both staged
    const bool ccls = (MODE == 1 || MODE == 3) && pl.cost_sm && pl.cost_cls;
    const uint8_t* ccls_idx = (const uint8_t*)(sm_all + pl.ccls_idx_off);
    const uint2* ninfo = (const uint2*)(sb + pl.off_ninfo);
    const uint16_t* lul = (const uint16_t*)(sb + pl.off_lul);
    const uint32_t* urow = (const uint32_t*)(sb + pl.off_urow);     // [R] U_r offset | |U_r| << 16
    const uint16_t* ubs = (const uint16_t*)(sb + pl.off_ubs);       // [nU] late users, by r
    const uint16_t* utr = (const uint16_t*)(sb + pl.off_utr);       // [R] t_r
    uint16_t* pos = (uint16_t*)(sm + pl.off_pos);
    uint16_t* last = (uint16_t*)(sm + pl.off_last);
    uint2* AF = MODE == 2 ? (uint2*)(afg + (size_t)cta * pl.af_bytes)         // [P][Sl] (alloc, free)
                          : (uint2*)(sm + pl.off_af);                           // size units per step
    uint8_t* dec_s = (uint8_t*)(sm + pl.off_dec);
    uint32_t* evm = (uint32_t*)(sm + pl.off_evm);          // [P][nwm] event-step marks
    uint8_t* sdec = (uint8_t*)(sm + pl.off_sdec);          // [2][P][Rw] decisions for the latency warp
    // decision row: R eligible tensors, then F F-Trans regions (NEXT-4)
    const int32_t F = pl.F, Rd = pl.Rd;
    const int32_t Rw = (Rd + 15) & ~15;                    // padded row of sdec
    const uint32_t* rnl = (const uint32_t*)(sb + pl.off_rn);        // [nRN] region nodes
    const uint8_t* nvarr = (const uint8_t*)(sb + pl.off_nvar);      // [F]
    const double* vcost = (const double*)(sb + pl.off_vcost);        // [4F]
    const int32_t nwm = pl.nwm, cap = pl.evcap;
    unsigned long long* evk_s = (unsigned long long*)(sm + pl.off_ev);             // [2][P][cap]
    double* evc_s = (double*)(sm + pl.off_ev + (size_t)2 * P * cap * 8);          // [2][P][cap]
    unsigned long long* evi_s = (unsigned long long*)(sm + pl.off_ev + (size_t)2 * P * cap * 16);   // [2][P][cap]

    // pos / last of the virtual and dummy slots start (and the dummy stays) 0
    for (int i = tid; i < pl.NTX * P; i += TM + TL) {
        pos[i] = 0;
        if constexpr (!kScatter) last[i] = 0;
    }
    for (int i = tid; i < P * nwm; i += TM + TL) evm[i] = 0;
    if constexpr (kScatter) {
        uint4* af4 = reinterpret_cast<uint4*>(AF);
        for (int i = tid; i < P * Sl / (kFO ? 4 : 2); i += TM + TL) af4[i] = make_uint4(0u, 0u, 0u, 0u);
    }
    // MODE 3: [P][Sl] one signed delta per step in size units, D[i] = alloc(i)
    // - free(i - 1), so M_i = sum_{j <= i} D[j] and the peak is the max-prefix of D
    int32_t* Ds = reinterpret_cast<int32_t*>(AF);
    if (tid == 0) {
        for (int b = 0; b < 2; b++) {
            for (int c = 0; c < 4; c++) ctl[b].flags[c] = ctl[b].viol[c] = 0;
            ctl[b].swm = 0;
        }
    }
    __syncthreads();

    const int64_t ngroups = (K + P - 1) / P;
    const int ncta = (cta < ngroups) ? (int)((ngroups - 1 - cta) / ncta_all + 1) : 0;
    constexpr int TPC = TM / P, WT = WM / P;

    if (warp >= WM) {
        // ================= latency warps (reading P7) ======================
        //      warp WM + c walks the event steps of candidate c of each group
        const int c = warp - WM;
        double* endb = (double*)(sm + pl.off_end) + (size_t)c * 3 * R;
        const WalkTabs wt{ninfo, lul, rtab, n, Lm};
        for (int gi = 0; gi < ncta; gi++) {
            const int slot = gi & 1;
            PROF_MARK(13);
            bar_sync(kBarFull + slot + bb, TM + TL);
            PROF_MARK(14);
            const SlotHdr& h = hdr[slot];
            const long long k = h.k[c];
            if (k < K) {
                const int st = h.status[c];
                const uint8_t* dd = sdec + (size_t)(slot * P + c) * Rw;
                double lat = __longlong_as_double(0x7ff0000000000000ll);
                long long pk = 0;
                int am_step = -1;
                double ctot = 0.0;
                if (!st) {
                    // fold the team's WT warp aggregates: (sum, max-prefix) -> peak,
                    // cost sums -> per-warp exclusive prefix and the total
                    const int a = c * WT + (lane < WT ? lane : 0);
                    long long ss = lane < WT ? agg_s[slot][a] : 0;
                    long long mm = lane < WT ? agg_m[slot][a] : kNegInf;
                    double cc = lane < WT ? agg_c[slot][a] : 0.0;
                    int aa = 0;
                    if constexpr (AM) aa = lane < WT ? agg_a[slot][a] : -1;
                    const double c0 = cc;
#pragma unroll
                    for (int o = 1; o < WT; o <<= 1) {
                        const long long ps = __shfl_up_sync(0xffffffffu, ss, o);
                        const long long pm = __shfl_up_sync(0xffffffffu, mm, o);
                        const double pc = __shfl_up_sync(0xffffffffu, cc, o);
                        if constexpr (AM) {
                            // the earlier part keeps the argmax on ties (first argmax)
                            const int pa = __shfl_up_sync(0xffffffffu, aa, o);
                            if (lane >= o && pm >= ps + mm) aa = pa;
                        }
                        if (lane >= o) { mm = max(pm, ps + mm); ss = ps + ss; cc = pc + cc; }
                    }
                    if (lane < WT) lwoff[c][lane] = cc - c0;
                    if constexpr (AM) am_step = __shfl_sync(0xffffffffu, aa, WT - 1);
                    pk = __shfl_sync(0xffffffffu, mm, WT - 1);
                    ctot = __shfl_sync(0xffffffffu, cc, WT - 1);
                    __syncwarp();
                }
                PROF_MARK(10);
                if (st) {
                } else if (!h.swp[c]) {
                    double bl = 0.0;                 // no swap: base cost + re-computations
                    for (int r = lane; r < R; r += 32)
                        if (dd[r] == 1) bl += rtab[r].x;
                    for (int i = lane; i < F; i += 32) bl += vcost[4 * i + dd[R + i]];   // chosen variants
#pragma unroll
                    for (int o = 16; o > 0; o >>= 1) bl += __shfl_xor_sync(0xffffffffu, bl, o);
                    lat = g.base_cost + bl;
                } else {
                    const double* woff = lwoff[c];
                    const int ne = h.nev[c];
#ifdef MAGIS_ABL_WALK
                    if (true) { lat = ctot; } else   // ablation (timing only): no latency walk
#endif
                    if (ne <= cap) {
                        const size_t b0 = (size_t)(slot * P + c) * cap;
                        unsigned long long* key = evk_s + b0;
                        unsigned long long* inf = evi_s + b0;
                        double* cbp = evc_s + b0;
                        for (int e = lane; e < ne; e += 32) resolve_event(key[e], cbp[e], inf[e], woff, dd, wt);
                        __syncwarp();
                        PROF_MARK(11);
                        if (lane == 0) {
                            double D = 0.0, Td = 0.0, Th = 0.0;
                            walk_events(inf, key, cbp, ne, endb, wt, D, Td, Th);
                            lat = fmax(fmax(ctot + D, Td), Th);
                        }
                        PROF_MARK(12);
                    } else {
                        char* ob = ovf + ((size_t)cta * 8 + slot * 4 + c) * pl.ovf_stride;
                        const size_t me = (size_t)pl.max_events;
                        lat = candidate_latency((unsigned long long*)ob, (double*)(ob + me * 8),
                                                (unsigned long long*)(ob + me * 16), ne, woff, dd, endb, wt, ctot,
                                                lane);
                    }
                }
                if (lane == 0) {
                    out_status[k] = (uint8_t)st;
                    out_peak[k] = st ? -1 : pk * pl.unit;
                    if constexpr (AM) out_arg[k] = st ? -1 : am_step;
                    out_lat[k] = lat;
                }
            }
            __syncwarp();
            PROF_MARK(15);
            if (gi + 2 < ncta) bar_arrive(kBarEmpty + slot + bb, TM + TL);
        }
        if (prof)
#pragma unroll
            for (int i = 10; i < 16; i++) atomicAdd((unsigned long long*)(ovf + pl.prof_off) + i, pt[i]);
        return;
    }

    // ========================= main warps =====================================
    // phases 1 and 5: candidate cm of the group is handled by team cm (TPC
    // threads, WT warps); thread tt of the team owns steps [lo, lo + L)
    const int cm = tid / TPC, tt = tid - cm * TPC;
    // (candidate, tensor) of this thread's first item in the P x R loops and the
    // per-iteration step (TM / R, TM % R): no division inside the group loop
    const int c_0 = R > 0 ? tid / R : 0, r_0 = tid - c_0 * R, dc_ = R > 0 ? TM / R : 0, dr_ = TM - dc_ * R;
    // the same over the whole decision row (R + F)
    const int c_0d = Rd > 0 ? tid / Rd : 0, r_0d = tid - c_0d * Rd, dc_d = Rd > 0 ? TM / Rd : 0, dr_d = TM - dc_d * Rd;
    const int32_t lo = tt * L;
    const bool vec4 = (NT & 3) == 0;
    // perm chunk kept in registers when short (32 steps only where the
    // tables sit in shared memory and the register budget allows it)
    constexpr int kRegL = MODE <= 1 ? 32 : 16;
    constexpr int LR = LMAX <= kRegL ? LMAX : 1;
    int32_t pr[LR];
    // this thread's chunk of candidate cm of group grp_ (-1 past the end)
    // the chunk's alignment in its row (warp-uniform: a warp serves one
    // candidate): 16-byte vectors when the row offset allows, else 8-byte
    // pairs (n_total even), else scalars; a vector never reads past the row
    auto load_chunk = [&](int64_t grp_) {
        const bool vc = grp_ * P + cm < K;
        const int64_t eo = (grp_ * P + cm) * (int64_t)NT + lo;
        const int32_t* Pp = perm + eo;
        const bool a16 = vec4 || (eo & 3) == 0, a8 = (eo & 1) == 0;
#pragma unroll
        for (int j = 0; j < LR; j += 4) {
            int4 v = make_int4(-1, -1, -1, -1);
            if (vc && j < L && lo + j < NT) {
                if (vec4 || (a16 && lo + j + 3 < NT)) {
                    v = __ldcs(reinterpret_cast<const int4*>(Pp + j));
                } else if (a8 && lo + j + 3 < NT) {
                    const int2 x = __ldcs(reinterpret_cast<const int2*>(Pp + j));
                    const int2 y = __ldcs(reinterpret_cast<const int2*>(Pp + j + 2));
                    v = make_int4(x.x, x.y, y.x, y.y);
                } else {
                    v.x = __ldcs(Pp + j);
                    if (lo + j + 1 < NT) v.y = __ldcs(Pp + j + 1);
                    if (lo + j + 2 < NT) v.z = __ldcs(Pp + j + 2);
                    if (lo + j + 3 < NT) v.w = __ldcs(Pp + j + 3);
                }
            }
            pr[j] = v.x;
            if (j + 1 < LR) pr[j + 1] = v.y;
            if (j + 2 < LR) pr[j + 2] = v.z;
            if (j + 3 < LR) pr[j + 3] = v.w;
        }
    };
    if constexpr (LMAX <= kRegL) {
        if (ncta > 0) load_chunk(cta);
    }
    // the group's decisions (<= 2 bytes per thread) are prefetched into
    // registers one group ahead, like the perm chunk
    const bool dreg = P * Rd <= 2 * TM;
    uint32_t dq0 = 0, dq1 = 0;
    auto load_dec = [&](int64_t grp_) {
        const int64_t b = grp_ * P * (int64_t)Rd, lim = K * (int64_t)Rd;
        dq0 = (tid < P * Rd && b + tid < lim) ? (uint32_t)__ldcs(dec + b + tid) : 0u;
        dq1 = (tid + TM < P * Rd && b + tid + TM < lim) ? (uint32_t)__ldcs(dec + b + tid + TM) : 0u;
    };
    if (dreg && Rd > 0 && ncta > 0) load_dec(cta);
    // streamed perm (tier 2, chunks longer than the register budget): the perm
    // rows of the group two ahead are pulled into L2 by the bulk-copy engine
    // (no registers, no shared memory), so phase 1 reads them from L2 (A/B: C4
    // -1.9%; with the chunk prefetched into registers it is neutral to +1.2%)
    constexpr bool kL2Pf = LMAX > kRegL;
    auto l2_prefetch = [&](int64_t grp_) {
        const int64_t k0 = grp_ * P, k1 = min(K, k0 + P);
        if (k0 >= K) return;
        uint64_t a = (uint64_t)(perm + k0 * (int64_t)NT), e = (uint64_t)(perm + k1 * (int64_t)NT);
        a = (a + 15) & ~15ull;                       // whole 16-byte units inside the rows
        e &= ~15ull;
        for (; a + 16 <= e; a += 32768) {
            const uint32_t nb = (uint32_t)min((uint64_t)32768, e - a);
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"(nb) : "memory");
        }
    };
    if (kL2Pf && tid == 0 && ncta > 1) l2_prefetch(cta + ncta_all);
    for (int gi = 0; gi < ncta; gi++) {
        const int64_t grp = cta + (int64_t)gi * ncta_all;
        const int slot = gi & 1;
        Ctl& cl = ctl[slot];
        if (kL2Pf && tid == 0 && gi + 2 < ncta) l2_prefetch(grp + 2 * ncta_all);
        // candidate c of this group exists iff bit c of vmask is set
        const int64_t kleft = K - grp * P;
        const uint32_t vmask = kleft >= P ? ((1u << P) - 1u) : ((1u << (uint32_t)kleft) - 1u);
        // ---- phase 0: decisions ---------------------------------------------
        {
            uint32_t badm = 0, swm = 0;
            int it = 0;
            for (int i = tid, c = c_0d, r = r_0d; i < P * Rd; i += TM, c += dc_d, r += dr_d, it++) {
                if (r >= Rd) { r -= Rd; c++; }
                // the group's decision rows are contiguous: dec[grp * P * Rd + i]
                uint8_t d;
                if (dreg) d = (uint8_t)(it == 0 ? dq0 : dq1);
                else d = ((vmask >> c) & 1u) ? dec[grp * P * (int64_t)Rd + i] : 0;
                dec_s[i] = d;
                if (r < R) {
                    if (d == 2) swm |= 1u << c;
                    if ((d > 2) | ((d == 1) & !(__ldg(g.rflag + r) & kRHasInput))) badm |= 1u << c;
                } else if (d >= nvarr[r - R]) {
                    badm |= 1u << c;                       // reading F1: not a variant of region r - R
                }
            }
            // one shared atomic per warp
            swm = __reduce_or_sync(0xffffffffu, swm);
            badm = __reduce_or_sync(0xffffffffu, badm);
            if (lane == 0) {
                if (swm) atomicOr(&cl.swm, (int)swm);
#pragma unroll
                for (int c = 0; c < P; c++)
                    if ((badm >> c) & 1u) atomicOr(&cl.flags[c], MAGIS_ST_BAD_DEC);
            }
        }
        // ---- phase 1: inverse permutation (pos stored +1); this thread's
        //      chunk of its team's candidate is in registers (loaded during the
        //      previous group) when short, else streamed here
        {
            int bad = 0;
            const bool vc = (vmask >> cm) & 1u;
            if constexpr (LMAX <= kRegL) {
                if (vc && L == LMAX && lo + LMAX <= NT) {
                    // full chunk: no per-step tests; an out-of-range id goes to
                    // the trash slot NTX (never read) and flags the candidate
                    const uint32_t trash = (uint32_t)pl.NTX;
                    uint16_t* pc_ = pos + cm;
#pragma unroll
                    for (int j = 0; j < LMAX; j++) {
                        const uint32_t v = (uint32_t)pr[j];
                        // every id >= NT (not only >= NTX) goes to the trash slot:
                        // the virtual slots and the dummy NTX - 1 read by row padding
                        // must stay untouched by a bad permutation
                        const bool oob = v >= (uint32_t)NT;
                        bad |= oob;
                        pc_[(oob ? trash : v) * P] = (uint16_t)(lo + j + 1);
                    }
                } else {
#pragma unroll
                    for (int j = 0; j < LMAX; j++) {
                        if (vc && j < L && lo + j < NT) {
                            const int32_t v = pr[j];
                            if ((uint32_t)v < (uint32_t)NT) pos[v * P + cm] = (uint16_t)(lo + j + 1); else bad = 1;
                        }
                    }
                }
            } else {
                // (default caching: the swap cost loop of phase 5 reads the chunk again)
                const int64_t eo = (grp * P + cm) * (int64_t)NT + lo;
                const int32_t* Pp = perm + eo;
                const bool a16 = vec4 || (eo & 3) == 0, a8 = (eo & 1) == 0;
                // batches of 16 steps: the 4 vector loads of a batch are issued
                // before its scatters (the compiler does not move loads across
                // the shared stores), so a chunk costs LMAX / 16 round trips
                // (tier 1; on tier 2 the L2 prefetch covers it and batching
                // measured +1.4%)
                constexpr int kB = MODE == 1 ? 16 : 4;
#pragma unroll
                for (int jb = 0; jb < LMAX; jb += kB) {
                    int4 vb[kB / 4];
#pragma unroll
                    for (int u = 0; u < kB / 4; u++) {
                        const int j = jb + 4 * u;
                        int4 v = make_int4(-1, -1, -1, -1);
                        if (j < LMAX && vc && j < L && lo + j < NT) {
                            if (vec4 || (a16 && lo + j + 3 < NT)) {
                                v = __ldg(reinterpret_cast<const int4*>(Pp + j));
                            } else if (a8 && lo + j + 3 < NT) {
                                const int2 x = __ldg(reinterpret_cast<const int2*>(Pp + j));
                                const int2 y = __ldg(reinterpret_cast<const int2*>(Pp + j + 2));
                                v = make_int4(x.x, x.y, y.x, y.y);
                            } else {
                                v.x = __ldg(Pp + j);
                                if (lo + j + 1 < NT) v.y = __ldg(Pp + j + 1);
                                if (lo + j + 2 < NT) v.z = __ldg(Pp + j + 2);
                                if (lo + j + 3 < NT) v.w = __ldg(Pp + j + 3);
                            }
                        }
                        vb[u] = v;
                    }
#pragma unroll
                    for (int u = 0; u < kB / 4; u++) {
                        const int j = jb + 4 * u;
                        if (j < LMAX && vc && j < L && lo + j < NT) {
                            const int4 v = vb[u];
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
                    }
                }
            }
            if (bad) atomicOr(&cl.flags[cm], MAGIS_ST_NOT_PERM);
        }
        // the control words of the next group (last read one group ago)
        if (tid == 0) {
            Ctl& cn = ctl[slot ^ 1];
            for (int c = 0; c < 4; c++) { cn.flags[c] = 0; cn.viol[c] = 0; }
            cn.swm = 0;
        }
        bar_sync(kBarMain + bb, TM);
        PROF_MARK(1);
        // ---- phase 2: optional nodes, virtual late-user slots, swap-event
        //      steps (producer, Store, Load and late users of swapped tensors)
        for (int q = tid, c = c_0, r = r_0; q < P * R; q += TM, c += dc_, r += dr_) {
            if (r >= R) { r -= R; c++; }
            if (!((vmask >> c) & 1u)) continue;
            const uint32_t ur = urow[r];                       // (U offset, |U_r|) packed
            const uint32_t u0 = ur & 0xffffu, u1 = u0 + (ur >> 16);
            const uint8_t d = dec_s[c * Rd + r];
            uint32_t* em = evm + c * nwm;
            uint16_t* pc_ = pos + c;
#pragma unroll
            for (int o = 0; o < 3; o++) {
                const int32_t id = n + 3 * r + o;
                const uint32_t p = pc_[id * P];
                if (p == 0) {
                    atomicOr(&cl.flags[c], MAGIS_ST_NOT_PERM);
                    continue;
                }
                const bool act = (o == 0) ? (d == 1) : (d == 2);
                const uint32_t st = p - 1;
                if (!act) {
                    // slots in shared memory start the group at 0 and phase 3 adds
                    // nothing at an absent node's step (no alloc, and no tensor has
                    // its last reader there); the global slots (MODE 2) are not cleared
                    if constexpr (!kScatter) AF[c * Sl + st + __umulhi(st, Lm)] = make_uint2(0u, 0u);
                    pc_[id * P] = 0;
                } else if (o > 0) {
                    atomicOr(em + (st >> 5), 1u << (st & 31));
                }
            }
            if (d == 2) {
                const uint32_t pt_ = pc_[(uint32_t)utr[r] * P];
                if (pt_) atomicOr(em + ((pt_ - 1) >> 5), 1u << ((pt_ - 1) & 31));
            }
            for (uint32_t j = u0; j < u1; j++) {
                const uint32_t pb = pc_[(uint32_t)ubs[j] * P];
                pc_[(NT + j) * P] = (d == 0) ? (uint16_t)pb : (uint16_t)0;
                if (d == 2 && pb) atomicOr(em + ((pb - 1) >> 5), 1u << ((pb - 1) & 31));
            }
        }
        // F-Trans regions (NEXT-4, reading F1): a node of an unchosen variant is
        // absent (position 0); every region node must still be in the
        // permutation
        if (F > 0) {
            // a thread takes region nodes k = tid + i TM and serves every
            // candidate of the group with one table read; the reads of 4 nodes
            // are issued together (the table is in global memory on tiers 1-3)
            const int32_t nRN = pl.nRN;
            for (int k0 = tid; k0 < nRN; k0 += 4 * TM) {
                uint32_t ev[4];
#pragma unroll
                for (int u = 0; u < 4; u++) ev[u] = k0 + u * TM < nRN ? rnl[k0 + u * TM] : 0u;
#pragma unroll
                for (int u = 0; u < 4; u++) {
                    if (k0 + u * TM >= nRN) break;
                    const uint32_t e = ev[u];
                    const uint32_t id = e & 0xffffu, reg = (e >> 16) & 0x3fffu, var = e >> 30;
#pragma unroll
                    for (int c = 0; c < P; c++) {
                        if (!((vmask >> c) & 1u)) continue;
                        uint16_t* pp = pos + id * P + c;
                        if (*pp == 0) atomicOr(&cl.flags[c], MAGIS_ST_NOT_PERM);
                        else if (dec_s[c * Rd + R + reg] != var) *pp = 0;
                    }
                }
            }
        }
        bar_sync(kBarMain + bb, TM);
        PROF_MARK(2);
        // ---- phase 3: validity + last use over the consumer rows -----------------
        {
            int nperm = 0, viol = 0;
            const uint32_t r0 = wtab[warp * 4 + 0], r1 = wtab[warp * 4 + 1];
            // tables in global memory: the next row's (offset, degree), header and
            // size are loaded one row ahead, hiding an L2 round trip (measured: C3
            // -13%, C4 -13% time; with the tables in shared memory it costs 0.3-1%)
            constexpr bool kRowPf = MODE != 0;
            // tier 2 (C4, one candidate per group): the first kEP edge entries of
            // the next row are also loaded with its header (one row ahead) and
            // its (offset, degree) two rows ahead, so the pos gathers of a row do
            // not wait on L2 (measured: C4 37.47 -> 36.15 ms; on tier 1 / C3 it
            // costs 6%: more registers and instructions than latency saved at P = 2)
            constexpr bool kEntPf = MODE == 3;
            constexpr int kEP = 4;
            uint2 rw_n = make_uint2(0u, 0u), rw_nn = make_uint2(0u, 0u);
            uint32_t h_n = 0u, a_n = 0u;
            uint32_t e_n[kEP], e_c[kEP];
#pragma unroll
            for (int k = 0; k < kEP; k++) e_n[k] = e_c[k] = 0u;
            if (kRowPf && r0 < r1) {
                rw_n = crow[r0];
                h_n = chdr[r0 * 32 + lane];
                a_n = csize[r0 * 32 + lane];
                if constexpr (kEntPf) {
#pragma unroll
                    for (int k = 0; k < kEP; k++)
                        if ((uint32_t)k < rw_n.y) e_n[k] = cent[rw_n.x + lane + k * 32];
                    if (r0 + 1 < r1) rw_nn = crow[r0 + 1];
                }
            }
            for (uint32_t r = r0; r < r1; r++) {
                uint2 rw;                                     // (edge offset, degree): warp-uniform
                uint32_t h, a_r;
                if constexpr (kRowPf) {
                    rw = rw_n; h = h_n; a_r = a_n;
                    if constexpr (kEntPf) {
#pragma unroll
                        for (int k = 0; k < kEP; k++) e_c[k] = e_n[k];
                        if (r + 1 < r1) {
                            rw_n = rw_nn;
                            h_n = chdr[(r + 1) * 32 + lane];
                            a_n = csize[(r + 1) * 32 + lane];
#pragma unroll
                            for (int k = 0; k < kEP; k++)
                                if ((uint32_t)k < rw_n.y) e_n[k] = cent[rw_n.x + lane + k * 32];
                        }
                        if (r + 2 < r1) rw_nn = crow[r + 2];
                    } else if (r + 1 < r1) {
                        rw_n = crow[r + 1];
                        h_n = chdr[(r + 1) * 32 + lane];
                        a_n = csize[(r + 1) * 32 + lane];
                    }
                } else {
                    rw = crow[r];
                    h = chdr[r * 32 + lane];
                    a_r = csize[r * 32 + lane];
                }
                const uint32_t kind = h >> kKindShift, id = h & kIdMask;
                const V p = PK::load(pos, id);
                V lst = p, mn = PK::ones();
                const uint16_t* ent = cent + rw.x + lane;
                uint32_t j0 = 0;
                if constexpr (kEntPf) {
#pragma unroll
                    for (int k = 0; k < kEP; k++) {
                        if ((uint32_t)k < rw.y) {
                            const V q = PK::load(pos, e_c[k]);
                            mn = PK::vmin(mn, PK::dec1(q));
                            lst = PK::vmax(lst, q);
                        }
                    }
                    j0 = kEP;
                }
#pragma unroll 4
                for (uint32_t j = j0; j < rw.y; j++) {
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
                    if constexpr (kScatter) {
                        // alloc at the own step, free after the last reader's step
                        // (a tensor without readers after its own step; graph
                        // outputs live to the end): scattered straight into the
                        // per-step slots, no second pass over the input rows
                        const uint32_t A = a_r;                    // row order (conflict-free)
#pragma unroll
                        for (int c = 0; c < P; c++) {
                            const uint32_t pc = PK::get(p, c);
                            if (pc == 0) continue;                  // absent (inactive) in candidate c
                            const uint32_t st = pc - 1;
                            if constexpr (kFO) {
                                if (A == 0) continue;
                                atomicAdd(&Ds[c * Sl + st + __umulhi(st, Lm)], (int32_t)A);
                                // freed after its last reader's step: the delta of the next step
                                const uint32_t f1 = PK::get(lst, c);
                                if (kind != kHdrOut && f1 < (uint32_t)NT)
                                    atomicAdd(&Ds[c * Sl + f1 + __umulhi(f1, Lm)], -(int32_t)A);
                                continue;
                            }
                            AF[c * Sl + st + __umulhi(st, Lm)].x = A;
                            if (kind != kHdrOut && A != 0) {
                                const uint32_t fs = PK::get(lst, c) - 1;
                                atomicAdd(&AF[c * Sl + fs + __umulhi(fs, Lm)].y, A);
                            }
                        }
                    } else {
                        V outv;
                        if (kind == kHdrOut) outv = PK::splat((uint32_t)NT);
                        else if (kind >= kHdrClone) outv = PK::vand(lst, PK::nzmask(p));   // inactive halves -> 0
                        else outv = lst;
                        PK::store(last, id, outv);
                    }
                }
            }
#pragma unroll
            for (int c = 0; c < P; c++) {
                if (nperm & (1 << c)) atomicOr(&cl.flags[c], MAGIS_ST_NOT_PERM);
                if (viol & (1 << c)) atomicOr(&cl.viol[c], MAGIS_ST_EDGE);
            }
        }
        bar_sync(kBarMain + bb, TM);
        PROF_MARK(3);
        // per-candidate status, 4 bits each; okm: valid candidates with status 0
        uint32_t stm = 0, okm = 0;
#pragma unroll
        for (int c = 0; c < P; c++) {
            const int f = cl.flags[c];
            const uint32_t st = ((vmask >> c) & 1u) ? (uint32_t)(f ? f : cl.viol[c]) : 0u;
            stm |= st << (4 * c);
            if (((vmask >> c) & 1u) && st == 0) okm |= 1u << c;
        }
        const uint32_t swm = (uint32_t)cl.swm & okm;       // valid candidates with swaps
        const bool mysw = (swm >> cm) & 1u;
        // event steps of this thread's chunk and their order within the warp
        const int32_t nst = ((okm >> cm) & 1u) ? max(0, min(L, NT - lo)) : 0;   // steps of this chunk
        const unsigned long long mbits =
            (mysw && nst > 0) ? mark_bits(evm + cm * nwm, lo) & (~0ull >> (64 - nst)) : 0ull;
        int evx = __popcll(mbits);
        {
            int inc = evx;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int x = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += x;
            }
            if (lane == 31) wcnt[warp] = inc;
            evx = inc - evx;
        }
        if (!kScatter && okm != 0) {
            // ---- phase 4 (slots in global memory): frees over the input rows ------
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
                        AF[c * Sl + st + __umulhi(st, Lm)] = make_uint2(A, fr[c]);
                    }
                }
            }
        }
        // the slot of this group parity is free once the latency warp is done
        // with group gi - 2
        PROF_MARK(9);
        if (gi >= 2) bar_sync(kBarEmpty + slot + bb, TM + TL);
        else bar_sync(kBarMain + bb, TM);
        PROF_MARK(4);
        SlotHdr& h = hdr[slot];
        // event list of candidate cm: shared-memory slot, or global overflow
        int ntot = 0, wpre = 0;
#pragma unroll
        for (int w = 0; w < WT; w++) {
            const int x = wcnt[cm * WT + w];
            ntot += x;
            if (w < warp - cm * WT) wpre += x;
        }
        unsigned long long* kout;
        double* cout_;
        if (ntot <= cap) {
            kout = evk_s + (size_t)(slot * P + cm) * cap;
            cout_ = evc_s + (size_t)(slot * P + cm) * cap;
        } else {
            char* ob = ovf + ((size_t)cta * 8 + slot * 4 + cm) * pl.ovf_stride;
            kout = (unsigned long long*)ob;
            cout_ = (double*)(ob + (size_t)pl.max_events * 8);
        }
        if (okm != 0) {
            // ---- phase 5: scan of the (sum, max-prefix) monoid ------------------
            //      team cm scans candidate cm: alloc = size of the op at each step,
            //      free = slot; with swaps also the compute-cost prefix, and the
            //      event steps of the chunk are emitted in order
            long long s1 = 0, m1 = kNegInf;
            int a1 = -1;                                     // AM: first step reaching m1
            double cs1 = 0.0;
            int o = wpre + evx;
            const int o0 = o;
            constexpr int kUnroll5 = LR > 1 ? LMAX : 8;     // full unroll only with the chunk in registers
            const uint2* afp = AF + cm * Sl + tt * (L + 1);  // step lo + j of candidate cm at afp[j]
            if constexpr (kFO) {
                // memory: max-prefix of the per-step deltas
                const int32_t* dp = Ds + cm * Sl + tt * (L + 1);   // step lo + j of candidate cm at dp[j]
#pragma unroll kUnroll5
                for (int j = 0; j < LMAX; j++) {
                    if (j < nst) {
                        s1 += dp[j];
                        if constexpr (AM) { if (s1 > m1) { m1 = s1; a1 = lo + j; } } else m1 = max(m1, s1);
                    }
                }
            } else
            // memory: alloc = size of the op at each step, free = slot
            if (L == LMAX && nst == LMAX) {
#pragma unroll
                for (int j = 0; j < LMAX; j++) {
                    const uint2 af = afp[j];
                    s1 += af.x;
                    if constexpr (AM) { if (s1 > m1) { m1 = s1; a1 = lo + j; } } else m1 = max(m1, s1);
                    s1 -= af.y;
                }
            } else {
#pragma unroll kUnroll5
                for (int j = 0; j < LMAX; j++) {
                    if (j < nst) {
                        const uint2 af = afp[j];
                        s1 += af.x;
                        if constexpr (AM) { if (s1 > m1) { m1 = s1; a1 = lo + j; } } else m1 = max(m1, s1);
                        s1 -= af.y;
                    }
                }
            }
#ifdef MAGIS_ABL_COST
            if (false) {                     // ablation (timing only): no swap cost loop / events
#else
            if (mysw) {
#endif
                // swapping candidate: compute-cost prefix (two partial sums
                // halve the dependent fp64 chain) and the chunk's event steps in
                // step order; an inactive clone (pos 0) costs nothing
                double ca = 0.0, cb = 0.0;
                if constexpr (LMAX <= kRegL) {
#pragma unroll kUnroll5
                    for (int j = 0; j < LMAX; j++) {
                        if (j < nst) {
                            const int32_t v = pr[j % LR];
                            if ((mbits >> j) & 1ull) {
                                kout[o] = ((unsigned long long)(lo + j) << 32) | (uint32_t)v;
                                cout_[o] = ca + cb;
                                o++;
                            }
                            double c = ccls ? cost_s[ccls_idx[v]] : cost_s[v];
                            if (v >= gate_lo && pos[v * P + cm] == 0) c = 0.0;
                            if (j & 1) cb += c; else ca += c;
                        }
                    }
                } else {
                    // perm chunk re-read from global: batches of 8 steps with the perm
                    // and cost loads issued ahead of the event stores (which the
                    // compiler cannot move loads across)
                    const int64_t eo = (grp * P + cm) * (int64_t)NT + lo;
                    const int32_t* pp = perm + eo;
                    const bool a16 = vec4 || (eo & 3) == 0, a8 = (eo & 1) == 0;
                    for (int jb = 0; jb < LMAX; jb += 8) {
                        if (jb >= nst) break;
                        int32_t vv[8];
                        double cv[8];
                        if (jb + 8 <= nst && (a16 || a8)) {              // last read, as vectors
                            if (a16) {
                                const int4 x = __ldcs(reinterpret_cast<const int4*>(pp + jb));
                                const int4 y = __ldcs(reinterpret_cast<const int4*>(pp + jb + 4));
                                vv[0] = x.x; vv[1] = x.y; vv[2] = x.z; vv[3] = x.w;
                                vv[4] = y.x; vv[5] = y.y; vv[6] = y.z; vv[7] = y.w;
                            } else {
#pragma unroll
                                for (int u = 0; u < 8; u += 2) {
                                    const int2 x = __ldcs(reinterpret_cast<const int2*>(pp + jb + u));
                                    vv[u] = x.x; vv[u + 1] = x.y;
                                }
                            }
                        } else {
#pragma unroll
                            for (int u = 0; u < 8; u++) vv[u] = jb + u < nst ? __ldcs(pp + jb + u) : 0;   // last read
                        }
#pragma unroll
                        for (int u = 0; u < 8; u++)
                            cv[u] = jb + u < nst ? (ccls ? cost_s[ccls_idx[vv[u]]] : cost_s[vv[u]]) : 0.0;
#pragma unroll
                        for (int u = 0; u < 8; u++) {
                            const int j = jb + u;
                            if (j < nst) {
                                const int32_t v = vv[u];
                                if ((mbits >> j) & 1ull) {
                                    kout[o] = ((unsigned long long)(lo + j) << 32) | (uint32_t)v;
                                    cout_[o] = ca + cb;
                                    o++;
                                }
                                double c = cv[u];
                                if (v >= gate_lo && pos[v * P + cm] == 0) c = 0.0;
                                if (u & 1) cb += c; else ca += c;
                            }
                        }
                    }
                }
                cs1 = ca + cb;
            }
            {
                // warp-level monoid scan: (s1, m1) then (s2, m2) = (s1 + s2, max(m1, s1 + m2))
                long long ss = s1, mm = m1;
                double cc = cs1;
                int aa = a1;
#pragma unroll
                for (int o2 = 1; o2 < 32; o2 <<= 1) {
                    const long long ps = __shfl_up_sync(0xffffffffu, ss, o2);
                    const long long pm = __shfl_up_sync(0xffffffffu, mm, o2);
                    const double pc = __shfl_up_sync(0xffffffffu, cc, o2);
                    if constexpr (AM) {
                        const int pa = __shfl_up_sync(0xffffffffu, aa, o2);
                        if (lane >= o2 && pm >= ps + mm) aa = pa;      // earlier steps win ties
                    }
                    if (lane >= o2) { mm = max(pm, ps + mm); ss = ps + ss; cc = pc + cc; }
                }
                if (lane == 31) {
                    agg_s[slot][warp] = ss; agg_m[slot][warp] = mm; agg_c[slot][warp] = cc;
                    if constexpr (AM) agg_a[slot][warp] = aa;
                }
                // add the lane's exclusive cost prefix within the warp to its events
                const double pre = cc - cs1;
                for (int e = o0; e < o; e++) cout_[e] += pre;
            }
        }
        // the next group's chunk and decisions are loaded while this group finishes
        if constexpr (LMAX <= kRegL) {
            if (gi + 1 < ncta) load_chunk(grp + ncta_all);
        }
        if (dreg && Rd > 0 && gi + 1 < ncta) load_dec(grp + ncta_all);
        bar_sync(kBarMain + bb, TM);
        PROF_MARK(5);
        // ---- phase 6: hand-off to the latency warps (they fold the aggregates) ----
        if (tid < P) {
            const int c = tid;
            int ne = 0;
#pragma unroll
            for (int w = 0; w < WT; w++) ne += wcnt[c * WT + w];
            h.k[c] = ((vmask >> c) & 1u) ? grp * P + c : LLONG_MAX;
            h.status[c] = (int)((stm >> (4 * c)) & 15u);
            h.swp[c] = (int)((swm >> c) & 1u);
            h.nev[c] = ne;
        }
        if (Rd > 0) {
            // decisions of the group -> the slot (rows padded to 16 bytes)
            const int nw = Rw >> 2;
            uint32_t* dst = reinterpret_cast<uint32_t*>(sdec + (size_t)slot * P * Rw);
            for (int i = tid; i < P * nw; i += TM) {
                const int c = i / nw, w = i - c * nw;
                uint32_t x = 0;
#pragma unroll
                for (int b = 0; b < 4; b++) {
                    const int r = 4 * w + b;
                    if (r < Rd) x |= (uint32_t)dec_s[c * Rd + r] << (8 * b);
                }
                dst[i] = x;
            }
        }
        // bar.arrive orders this thread's prior shared / global writes for the
        // threads that sync on the barrier (no membar: it would also wait for
        // the next group's perm loads already in flight)
        bar_arrive(kBarFull + slot + bb, TM + TL);
        PROF_MARK(6);
        // clear pos and the event marks for the next group
        {
            const int nb = NT * P * 2;
            uint4* p4 = reinterpret_cast<uint4*>(pos);
            for (int i = tid; i < (nb >> 4); i += TM) p4[i] = make_uint4(0u, 0u, 0u, 0u);
            for (int i = ((nb >> 4) << 3) + tid; i < NT * P; i += TM) pos[i] = 0;
            for (int i = tid; i < P * nwm; i += TM) evm[i] = 0;
            if constexpr (kScatter) {           // the per-step slots start from 0 for the scatter
                uint4* af4 = reinterpret_cast<uint4*>(AF);
                for (int i = tid; i < P * Sl / (kFO ? 4 : 2); i += TM) af4[i] = make_uint4(0u, 0u, 0u, 0u);
            }
        }
        bar_sync(kBarMain + bb, TM);
        PROF_MARK(7);
    }
    if (prof)
#pragma unroll
        for (int i = 1; i < 13; i++) atomicAdd((unsigned long long*)(ovf + pl.prof_off) + i, pt[i]);
}


template <int P, int MODE, int TEAMS, bool AM>
static const void* kernel_ptr(int lmax) {
    if constexpr (MODE == 0) {
        if (lmax <= 4) return (const void*)eval2_kernel<P, 4, 0, TEAMS, AM>;
        if (lmax <= 8) return (const void*)eval2_kernel<P, 8, 0, TEAMS, AM>;
        if (lmax <= 12) return (const void*)eval2_kernel<P, 12, 0, TEAMS, AM>;
        if (lmax <= 16) return (const void*)eval2_kernel<P, 16, 0, TEAMS, AM>;
        if (lmax <= 20) return (const void*)eval2_kernel<P, 20, 0, TEAMS, AM>;
        if (lmax <= 24) return (const void*)eval2_kernel<P, 24, 0, TEAMS, AM>;
        if (lmax <= 28) return (const void*)eval2_kernel<P, 28, 0, TEAMS, AM>;
        return (const void*)eval2_kernel<P, 32, 0, TEAMS, AM>;
    } else {
        if (lmax <= 16) return (const void*)eval2_kernel<P, 16, MODE, 1, AM>;
        if (lmax <= 24) return (const void*)eval2_kernel<P, 24, MODE, 1, AM>;
        if (lmax <= 28) return (const void*)eval2_kernel<P, 28, MODE, 1, AM>;
        if (lmax <= 32) return (const void*)eval2_kernel<P, 32, MODE, 1, AM>;
        if (lmax <= 48) return (const void*)eval2_kernel<P, 48, MODE, 1, AM>;
        return (const void*)eval2_kernel<P, 64, MODE, 1, AM>;
    }
}

template <int MODE, int TEAMS, bool AM = false>
static const void* kernel_mode(const Plan2& pl) {
    return pl.P == 4 ? kernel_ptr<4, MODE, TEAMS, AM>(pl.L)
                     : pl.P == 2 ? kernel_ptr<2, MODE, TEAMS, AM>(pl.L) : kernel_ptr<1, MODE, TEAMS, AM>(pl.L);
}

}  // namespace magis
