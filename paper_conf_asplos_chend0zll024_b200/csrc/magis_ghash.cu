// magis_ghash.cu -- batched GraphHash (Alg. 3 lines 3-6,
// P:1693-1700; the Weisfeiler-Lehman idea).  Readings G1-G4 are
// in DESIGN.md §3.  The duplicate filter (lines 10-12) is magis_hashset.cu.
//
// The graph of candidate k is its transformed graph (Fig. 8 rules applied to
// the decisions dec[k]; the schedule does not enter, reading G4).  Per node,
// in one fixed topological order of the super-graph:
//     x_v = hash( hash(label_v) (+) x_{u_1} (+) ... (+) x_{u_d} )   (line 5)
// with u_1..u_d = pre(v) in ascending order of x (reading G2), and
//     GraphHash = hash( sum_v x_v mod 2^64 )                         (line 6)
// hash() over 64-bit words: h = GAMMA (m + 1), h = mix64(h ^ w_i) (reading G1).
//
// B200 layout.
//  * Lane = candidate; a warp carries C = 1 or 2 candidates per lane (two
//    independent mix64 chains per node for ILP) and walks the node table
//    with warp-uniform, L1-broadcast loads.  Decisions only switch which
//    value a late-user edge reads (t_r, the clone or the Load) and whether an
//    optional node is active, so control flow stays uniform.
//  * Work that does not depend on the decisions is done once at create
//    time: the first absorbed word of every node (h1 = mix64(GAMMA (d+2) ^
//    hash(label))), and the complete x of every node no decision can reach
//    (sources, weights, and everything upstream of the first late user):
//    those nodes leave the loop, their values are read from a constant table
//    and their sum is a constant.
//  * x values of the remaining nodes live in "slots" assigned by a linear
//    scan over the order (reused once the last potential reader has run):
//    short-lived values in shared memory ([slot][c][lane], conflict-free),
//    long-lived ones in a per-warp global region with the same layout
//    (256-byte coalesced rows, L2-resident).
//  * Predecessor values are sorted in registers: exact networks for in-degree
//    1-4 (the bulk of a DNN graph), bitonic networks up to 32, a rank sort in
//    global scratch beyond.
#include <algorithm>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <new>
#include <string>
#include <vector>

#include "magis_internal.h"

namespace magis {

constexpr uint64_t kGamma = 0x9E3779B97F4A7C15ull;
constexpr uint64_t kTagStore = 0x45524F5453ull;   // "STORE" (reading G3)
constexpr uint64_t kTagLoad = 0x44414F4Cull;      // "LOAD"
// value references (pent entries, slots): LU = late-user edge of r (the
// decision picks t_r / clone_r / load_r); Const = x0 table index;
// Glob = per-warp global slot; otherwise a shared-memory slot
constexpr uint32_t kLU = 0x80000000u, kConst = 0x40000000u, kGlob = 0x20000000u, kIdx = 0x1FFFFFFFu;
constexpr uint32_t kNoSlot = 0xFFFFFFFFu;
constexpr int kGhWarps = 4;                        // warps per CTA
constexpr int kGhCtasPerSm = 4;
constexpr uint32_t kLabStore = 0xFFFFFFFEu, kLabLoad = 0xFFFFFFFDu;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

struct GhDev {
    int32_t nloop;            // nodes walked per candidate
    int32_t R, NS;            // eligible tensors, shared slots per warp (per candidate column)
    int32_t gslots;           // global slots per warp (per candidate column)
    int32_t maxdeg;           // in-degree of the rank-sort path (0 if none > 32)
    int32_t Rw;               // u32 words of packed decisions per candidate (16 per word)
    const uint4* nrec;        // [nloop] (h1 lo, h1 hi, own slot, gate); gate ~0 = always active
    const uint2* nadj;        // [nloop] (pent offset or x0 index, deg | kind << 24); kind 1 = constant node
    const uint32_t* pent;     // value references of the predecessors
    const uint4* rslot;       // [R] value references of (t_r, clone_r, load_r, t_r)
    const uint8_t* rflag;     // [R] kRHasInput
    const unsigned long long* x0;   // [NT] x of the decision-independent nodes
    const unsigned long long* c0;   // [1] sum of x0 over decision-independent original nodes
    unsigned long long* gbuf; // [warps][gslots + 2 maxdeg][C][32]
};

}  // namespace magis

struct magis_ghash {
    const magis_graph* g = nullptr;
    int device = 0;
    magis::GhDev dev{};
    void* tables = nullptr;
    void* scratch = nullptr;
    size_t scratch_bytes = 0;
    int grid = 0;
    size_t smem = 0;
    int64_t n_global_nodes = 0;   // walked nodes whose x lives in global slots
    int64_t n_const_nodes = 0;    // nodes no decision can reach
    int64_t n_grouped = 0;        // walked nodes hashed in same-level groups
};

namespace magis {
namespace {

// ------------------------------------------------------------ setup kernels --
// h1[v] = hash state after the first word of line 5: mix64(GAMMA (d + 2) ^ hash([label_v]))
__global__ void ghash_h1_kernel(int32_t NT, const uint32_t* lsrc, const int32_t* deg, const uint64_t* label,
                                unsigned long long* h1) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= NT) return;
    const uint32_t s = lsrc[i];
    const uint64_t lab = s == kLabStore ? kTagStore : s == kLabLoad ? kTagLoad : label[s];
    const uint64_t hl = mix64((kGamma * 2ull) ^ lab);                   // hash([label])
    h1[i] = mix64((kGamma * (uint64_t)(deg[i] + 2)) ^ hl);
}

// x of the decision-independent nodes, in order (one thread; runs once)
__global__ void ghash_const_kernel(int32_t nc, const int32_t* cnode, const int32_t* cptr, const int32_t* cpred,
                                   const uint8_t* corig, const unsigned long long* h1, unsigned long long* x0,
                                   unsigned long long* tmp, unsigned long long* c0) {
    if (blockIdx.x || threadIdx.x) return;
    unsigned long long sum = 0;
    for (int32_t i = 0; i < nc; i++) {
        const int32_t v = cnode[i], b = cptr[i], e = cptr[i + 1];
        int32_t m = 0;
        for (int32_t j = b; j < e; j++) {                // insertion sort, ascending
            const unsigned long long x = x0[cpred[j]];
            int32_t q = m++;
            while (q > 0 && tmp[q - 1] > x) { tmp[q] = tmp[q - 1]; q--; }
            tmp[q] = x;
        }
        unsigned long long h = h1[v];
        for (int32_t j = 0; j < m; j++) h = mix64(h ^ tmp[j]);
        x0[v] = h;
        if (corig[i]) sum += h;
    }
    *c0 = sum;
}

__global__ void ghash_fill_kernel(int32_t nloop, const int32_t* lnode, const unsigned long long* h1, uint4* nrec) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nloop) return;
    const unsigned long long h = h1[lnode[i]];
    nrec[i].x = (uint32_t)h;
    nrec[i].y = (uint32_t)(h >> 32);
}

// ------------------------------------------------------------- main kernel --
template <int D>
__device__ __forceinline__ void bitonic(uint64_t (&a)[D]) {
#pragma unroll
    for (int k = 2; k <= D; k <<= 1)
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1)
#pragma unroll
            for (int i = 0; i < D; i++) {
                const int l = i ^ j;
                if (l > i) {
                    const bool up = (i & k) == 0;
                    const uint64_t lo = min(a[i], a[l]), hi = max(a[i], a[l]);
                    a[i] = up ? lo : hi;
                    a[l] = up ? hi : lo;
                }
            }
}

__device__ __forceinline__ void cex(uint64_t& a, uint64_t& b) {
    const uint64_t lo = min(a, b), hi = max(a, b);
    a = lo;
    b = hi;
}

struct Lanes {
    const GhDev& d;
    unsigned long long* xs;            // shared slots of this warp: [NS][32]
    unsigned long long* gb;            // global slots of this warp: [gslots][32]
    const uint32_t* decp;              // packed decisions of this warp: [Rw][32]
    int lane;
    __device__ __forceinline__ uint32_t dec(uint32_t r) const {
        return (decp[(r >> 4) * 32 + lane] >> (2 * (r & 15))) & 3u;
    }
    __device__ __forceinline__ uint64_t get(uint32_t e) const {
        if (!(e & (kLU | kConst | kGlob))) return xs[e * 32 + lane];     // the common case first
        uint32_t s = e;
        if (e & kLU) {
            const uint4 rs = __ldg(d.rslot + (e & kIdx));
            const uint32_t dd = dec(e & kIdx);
            s = dd == 1 ? rs.y : dd == 2 ? rs.z : rs.x;
        }
        if (s & kConst) return __ldg(d.x0 + (s & kIdx));
        if (s & kGlob) return gb[(size_t)(s & kIdx) * 32 + lane];
        return xs[s * 32 + lane];
    }
    __device__ __forceinline__ void put(uint32_t s, uint64_t h) const {
        if (!(s & kGlob)) xs[s * 32 + lane] = h;                        // kNoSlot has every bit set
        else if (s != kNoSlot) gb[(size_t)(s & kIdx) * 32 + lane] = h;
    }
};

// exact sorting networks for D <= 4 values
template <int D>
__device__ __forceinline__ void sortn(uint64_t (&a)[D]) {
    if constexpr (D == 2) {
        cex(a[0], a[1]);
    } else if constexpr (D == 3) {
        cex(a[0], a[1]); cex(a[1], a[2]); cex(a[0], a[1]);
    } else if constexpr (D == 4) {
        cex(a[0], a[1]); cex(a[2], a[3]); cex(a[0], a[2]); cex(a[1], a[3]); cex(a[1], a[2]);
    }
}

// G independent nodes of one topological level with in-degree D each (always
// active): G interleaved mix64 chains.  Node records i .. i+G-1, their
// predecessor references are contiguous at ent (G x D).
template <int G, int D>
__device__ __forceinline__ void group_nodes(const Lanes& L, const uint4* rec, const uint32_t* ent, uint64_t& sum) {
    uint64_t a[G][D], h[G];
    uint32_t e[G * D];
#pragma unroll
    for (int j = 0; j < G * D; j++) e[j] = __ldg(ent + j);
#pragma unroll
    for (int g = 0; g < G; g++) {
#pragma unroll
        for (int j = 0; j < D; j++) a[g][j] = L.get(e[g * D + j]);
        sortn<D>(a[g]);
        h[g] = ((uint64_t)rec[g].y << 32) | rec[g].x;
    }
#pragma unroll
    for (int j = 0; j < D; j++)
#pragma unroll
        for (int g = 0; g < G; g++) h[g] = mix64(h[g] ^ a[g][j]);
#pragma unroll
    for (int g = 0; g < G; g++) {
        sum += h[g];
        L.put(rec[g].z, h[g]);
    }
}

template <int G>
__device__ __forceinline__ void group_dispatch(const Lanes& L, int D, const uint4* rec, const uint32_t* ent,
                                               uint64_t& sum) {
    switch (D) {
        case 1: group_nodes<G, 1>(L, rec, ent, sum); break;
        case 2: group_nodes<G, 2>(L, rec, ent, sum); break;
        case 3: group_nodes<G, 3>(L, rec, ent, sum); break;
        default: group_nodes<G, 4>(L, rec, ent, sum); break;
    }
}

__global__ void __launch_bounds__(32 * kGhWarps, kGhCtasPerSm)
ghash_kernel(GhDev d, int64_t K, const uint8_t* __restrict__ dec, int vec, uint8_t* __restrict__ out_status,
             uint64_t* __restrict__ out_hash) {
    extern __shared__ __align__(16) unsigned long long ghsm[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int64_t wg = (int64_t)blockIdx.x * kGhWarps + wib, nw = (int64_t)gridDim.x * kGhWarps;
    const size_t per_warp = (size_t)d.NS * 32 + (size_t)d.Rw * 16;     // u64 units
    unsigned long long* xs = ghsm + per_warp * wib;
    uint32_t* decp = reinterpret_cast<uint32_t*>(xs + (size_t)d.NS * 32);
    unsigned long long* gb = d.gbuf + (size_t)wg * (size_t)(d.gslots + 2 * d.maxdeg) * 32;
    const Lanes L{d, xs, gb, decp, lane};
    const unsigned long long c0 = *d.c0;

    for (int64_t grp = wg; grp * 32 < K; grp += nw) {
        const int64_t k = grp * 32 + lane;
        const bool valid = k < K;
        // decisions -> 2-bit lanes; bad decision status (reading P12, R-noinput)
        uint32_t bad = 0;
        const uint8_t* dk = dec + (valid ? k : 0) * (int64_t)d.R;
        for (int w = 0; w < d.Rw; w++) {
            uint32_t word = 0;
            if (valid) {
                if (vec) {
                    const uint4 q = __ldcs(reinterpret_cast<const uint4*>(dk + 16 * w));
                    const uint32_t qq[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                    for (int b = 0; b < 16; b++) {
                        const uint32_t dv = (qq[b >> 2] >> (8 * (b & 3))) & 0xffu;
                        bad |= (dv > 2u) | ((dv == 1u) & !(__ldg(d.rflag + 16 * w + b) & kRHasInput));
                        word |= (dv & 3u) << (2 * b);
                    }
                } else {
                    for (int b = 0; b < 16 && 16 * w + b < d.R; b++) {
                        const uint32_t dv = dk[16 * w + b];
                        bad |= (dv > 2u) | ((dv == 1u) & !(__ldg(d.rflag + 16 * w + b) & kRHasInput));
                        word |= (dv & 3u) << (2 * b);
                    }
                }
            }
            decp[w * 32 + lane] = word;
        }
        __syncwarp();
        uint64_t sum = c0;
        for (int32_t i = 0; i < d.nloop;) {
            const uint2 adj = __ldg(d.nadj + i);
            const int deg = (int)(adj.y & 0xFFFFFFu);
            const uint32_t kind = (adj.y >> 24) & 3u;
            if (kind == 2) {                                  // a group of G same-level nodes
                const int G = (int)(adj.y >> 26);
                uint4 rec[4];
#pragma unroll
                for (int g = 0; g < 4; g++)
                    if (g < G) rec[g] = __ldg(d.nrec + i + g);
                const uint32_t* ent = d.pent + adj.x;
                switch (G) {
                    case 2: group_dispatch<2>(L, deg, rec, ent, sum); break;
                    case 3: group_dispatch<3>(L, deg, rec, ent, sum); break;
                    default: group_dispatch<4>(L, deg, rec, ent, sum); break;
                }
                i += G;
                continue;
            }
            const uint4 rec = __ldg(d.nrec + i);
            i++;
            bool act = true;
            if (rec.w != 0xFFFFFFFFu) {                       // optional node: active iff dec[r] == gate
                act = L.dec(rec.w >> 2) == (rec.w & 3u);
                if (!__any_sync(0xffffffffu, act)) continue;
            }
            if (kind == 1) {                                  // decision-independent optional node
                if (act) sum += __ldg(d.x0 + adj.x);
                continue;
            }
            const uint32_t* ent = d.pent + adj.x;
            uint64_t h = ((uint64_t)rec.y << 32) | rec.x;
            if (deg == 1) {
                h = mix64(h ^ L.get(__ldg(ent)));
            } else if (deg == 2) {
                uint64_t a[2] = {L.get(__ldg(ent)), L.get(__ldg(ent + 1))};
                sortn<2>(a);
                h = mix64(mix64(h ^ a[0]) ^ a[1]);
            } else if (deg == 3) {
                uint64_t a[3] = {L.get(__ldg(ent)), L.get(__ldg(ent + 1)), L.get(__ldg(ent + 2))};
                sortn<3>(a);
                h = mix64(mix64(mix64(h ^ a[0]) ^ a[1]) ^ a[2]);
            } else if (deg == 4) {
                uint64_t a[4] = {L.get(__ldg(ent)), L.get(__ldg(ent + 1)), L.get(__ldg(ent + 2)),
                                 L.get(__ldg(ent + 3))};
                sortn<4>(a);
                h = mix64(mix64(mix64(mix64(h ^ a[0]) ^ a[1]) ^ a[2]) ^ a[3]);
            } else if (deg == 0) {
            } else if (deg <= 8) {
                uint64_t a[8];
#pragma unroll
                for (int j = 0; j < 8; j++) a[j] = j < deg ? L.get(__ldg(ent + j)) : ~0ull;
                bitonic<8>(a);
#pragma unroll
                for (int j = 0; j < 8; j++)
                    if (j < deg) h = mix64(h ^ a[j]);
            } else if (deg <= 32) {
                uint64_t a[32];
#pragma unroll
                for (int j = 0; j < 32; j++) a[j] = j < deg ? L.get(__ldg(ent + j)) : ~0ull;
                bitonic<32>(a);
#pragma unroll
                for (int j = 0; j < 32; j++)
                    if (j < deg) h = mix64(h ^ a[j]);
            } else {
                // rank sort in this lane's global scratch column (merges of > 32 parts)
                unsigned long long* t0 = gb + (size_t)d.gslots * 32;
                unsigned long long* t1 = t0 + (size_t)d.maxdeg * 32;
                for (int j = 0; j < deg; j++) t0[j * 32 + lane] = L.get(__ldg(ent + j));
                for (int j = 0; j < deg; j++) {
                    const uint64_t v = t0[j * 32 + lane];
                    int rk = 0;
                    for (int q = 0; q < deg; q++) {
                        const uint64_t u = t0[q * 32 + lane];
                        rk += (u < v) | ((u == v) & (q < j));
                    }
                    t1[rk * 32 + lane] = v;
                }
                for (int j = 0; j < deg; j++) h = mix64(h ^ t1[j * 32 + lane]);
            }
            if (act) {
                sum += h;
                L.put(rec.z, h);
            }
            // no __syncwarp: every lane reads and writes only its own column
        }
        if (valid) {
            out_status[k] = bad ? (uint8_t)MAGIS_ST_BAD_DEC : (uint8_t)0;
            out_hash[k] = bad ? 0ull : mix64((kGamma * 2ull) ^ sum);       // line 6: hash([sum])
        }
        __syncwarp();
    }
}

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) { cudaGetDevice(&prev); cudaSetDevice(d); }
    ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

#define GCK(call)                                                                             \
    do {                                                                                      \
        cudaError_t _e = (call);                                                              \
        if (_e != cudaSuccess) {                                                              \
            cudaGetLastError();                                                               \
            return set_error(MAGIS_E_CUDA, std::string(#call ": ") + cudaGetErrorString(_e)); \
        }                                                                                     \
    } while (0)

}  // namespace
}  // namespace magis

using namespace magis;

// ------------------------------------------------------------------- host --
extern "C" int magis_ghash_create(const magis_graph* g, const uint64_t* h_label, magis_ghash** out) {
    clear_error();
    if (!out) return set_error(MAGIS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (!g || !h_label) return set_error(MAGIS_E_INVAL, "null argument");
    if (g->dev.F > 0) return set_error(MAGIS_E_UNSUPPORTED, "magis_ghash_create: not available on graphs with F-Trans regions");
    const int32_t n = g->dev.n, R = g->dev.R, NT = g->dev.NT;
    const auto& pp = g->h_pred_ptr;
    const auto& pr = g->h_pred;
    // r_of and late-user membership (reading P6)
    std::vector<int32_t> r_of(n, -1);
    for (int32_t r = 0; r < R; r++) r_of[g->h_elig[r]] = r;
    std::vector<std::vector<int32_t>> Umem(n);   // Umem[b] = r's with b in U_r
    for (int32_t r = 0; r < R; r++)
        for (int32_t j = g->h_Uptr[r]; j < g->h_Uptr[r + 1]; j++) Umem[g->h_Uidx[j]].push_back(r);
    // fixed topological order of the super-graph: originals in load-time
    // topological order, clone / Store / Load right after their t_r
    std::vector<int32_t> order;
    order.reserve(NT);
    for (int32_t v : g->h_topo) {
        order.push_back(v);
        if (r_of[v] >= 0) for (int o = 0; o < 3; o++) order.push_back(n + 3 * r_of[v] + o);
    }
    // predecessor entries: node id, or kLU | r for a late-user edge
    std::vector<std::vector<uint32_t>> ent(NT);
    for (int32_t v = 0; v < n; v++)
        for (int32_t e = pp[v]; e < pp[v + 1]; e++) {
            const int32_t u = pr[e], r = r_of[u];
            bool lu = false;
            if (r >= 0) for (int32_t rr : Umem[v]) if (rr == r) { lu = true; break; }
            ent[v].push_back(lu ? (kLU | (uint32_t)r) : (uint32_t)u);
        }
    for (int32_t r = 0; r < R; r++) {
        const int32_t t = g->h_elig[r], c = n + 3 * r;
        for (int32_t e = pp[t]; e < pp[t + 1]; e++) ent[c].push_back((uint32_t)pr[e]);
        ent[c + 1].push_back((uint32_t)t);
        ent[c + 2].push_back((uint32_t)(c + 1));
    }
    // decision-dependent nodes: a late-user edge, or a predecessor that is
    std::vector<uint8_t> aff(NT, 0);
    for (int32_t x : order)
        for (uint32_t e : ent[x])
            if ((e & kLU) || aff[e]) { aff[x] = 1; break; }
    // launch shape and the shared slot budget
    int sms = 0;
    {
        DeviceGuard guard(g->device);
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device) != cudaSuccess) {
            cudaGetLastError();
            return set_error(MAGIS_E_CUDA, "cudaDeviceGetAttribute failed");
        }
    }
    const int32_t Rw = (R + 15) / 16;
    const size_t smem_cap = 227 * 1024 / kGhCtasPerSm;
    const size_t dec_bytes = (size_t)Rw * 32 * 4;
    int32_t NS = (int32_t)std::max<int64_t>(0, ((int64_t)smem_cap / kGhWarps - (int64_t)dec_bytes) / 256);
    if (const char* e = std::getenv("MAGIS_GH_NS")) NS = std::min(NS, std::atoi(e));
    int32_t maxdeg = 0;
    for (int32_t x = 0; x < NT; x++)
        if (aff[x]) maxdeg = std::max<int32_t>(maxdeg, (int32_t)ent[x].size());
    // Two walking orders are planned and the one that keeps fewer values in
    // global slots wins (ties: levels):
    //  * levels: topological levels of the super-graph (every gated edge
    //    included, so they hold for every candidate), by in-degree inside a
    //    level, so that runs of same-level, same-degree nodes form groups whose
    //    hash chains interleave (ILP within one candidate);
    //  * topo: the load-time topological order (shorter value lifetimes on
    //    graphs whose levels are wide, e.g. many fissioned parts side by side).
    // Slots by linear scan over the walked values; a value that dies within
    // TS positions prefers shared memory; TS minimises the values sent to global.
    const std::vector<int32_t> order_topo = order;
    std::vector<int32_t> lvl(NT, 0), pos0(NT);
    for (int32_t i = 0; i < NT; i++) pos0[order_topo[i]] = i;
    for (int32_t x : order_topo)
        for (uint32_t e : ent[x]) {
            if (e & kLU) {
                const int32_t r = (int32_t)(e & kIdx);
                for (int32_t y : {g->h_elig[r], n + 3 * r, n + 3 * r + 2}) lvl[x] = std::max(lvl[x], lvl[y] + 1);
            } else {
                lvl[x] = std::max(lvl[x], lvl[e] + 1);
            }
        }
    const char* ordenv = std::getenv("MAGIS_GH_ORDER");
    std::vector<uint32_t> best_slot;
    int32_t best_gs = 0;
    int64_t best_glob = -1;
    for (int mode = 0; mode < 2; mode++) {                 // 0 levels, 1 topo
        if (ordenv && std::string(ordenv) == (mode ? "level" : "topo")) continue;
        std::vector<int32_t> ord = order_topo;
        if (mode == 0) {
            auto dclass = [&](int32_t x) { return x >= n ? 8 : std::min<int32_t>((int32_t)ent[x].size(), 5); };
            std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) {
                if (lvl[a] != lvl[b]) return lvl[a] < lvl[b];
                if (dclass(a) != dclass(b)) return dclass(a) < dclass(b);
                return pos0[a] < pos0[b];
            });
        }
        std::vector<int32_t> hp(NT);
        for (int32_t i = 0; i < NT; i++) hp[ord[i]] = i;
        // potential readers of the walked values -> last position
        std::vector<int32_t> lastp(NT);
        for (int32_t i = 0; i < NT; i++) lastp[ord[i]] = i;
        for (int32_t x = 0; x < NT; x++) {
            if (!aff[x]) continue;
            for (uint32_t e : ent[x]) {
                if (e & kLU) {
                    const int32_t r = (int32_t)(e & kIdx);
                    for (int32_t y : {g->h_elig[r], n + 3 * r, n + 3 * r + 2}) lastp[y] = std::max(lastp[y], hp[x]);
                } else {
                    lastp[e] = std::max(lastp[e], hp[x]);
                }
            }
        }
        for (int32_t TS : {1, 2, 4, 8, 16, 32, 64, 128, 256, 1 << 30}) {
            std::vector<uint32_t> slot(NT, kNoSlot);
            std::vector<std::vector<int32_t>> dies(NT + 1);
            std::vector<uint32_t> sfree, gfree;
            for (int32_t s2 = NS - 1; s2 >= 0; s2--) sfree.push_back((uint32_t)s2);
            int32_t gused = 0;
            int64_t nglob = 0;
            for (int32_t i = 0; i < NT; i++) {
                const int32_t x = ord[i];
                if (i > 0)
                    for (int32_t y : dies[i - 1]) {
                        if (slot[y] & kGlob) gfree.push_back(slot[y]);
                        else sfree.push_back(slot[y]);
                    }
                if (!aff[x] || lastp[x] == i) continue;   // constant, or no reader after it
                const bool shortl = lastp[x] - i <= TS;
                if (shortl && !sfree.empty()) { slot[x] = sfree.back(); sfree.pop_back(); }
                else if (!gfree.empty()) { slot[x] = gfree.back(); gfree.pop_back(); nglob++; }
                else { slot[x] = kGlob | (uint32_t)gused++; nglob++; }
                dies[lastp[x]].push_back(x);
            }
            if (best_glob < 0 || nglob < best_glob) {
                best_glob = nglob;
                best_slot = slot;
                best_gs = gused;
                order = ord;
            }
        }
    }
    auto ref = [&](int32_t y) -> uint32_t { return aff[y] ? best_slot[y] : (kConst | (uint32_t)y); };
    // walked nodes: decision-dependent nodes, and constant optional nodes
    // (their activity still depends on the decisions)
    std::vector<uint4> nrec;
    std::vector<uint2> nadj;
    std::vector<int32_t> lnode;
    std::vector<uint32_t> pent;
    int64_t ngrouped = 0;
    for (int32_t i = 0; i < NT; i++) {
        const int32_t x = order[i];
        if (!aff[x] && x < n) continue;
        // a group: up to 4 consecutive always-active walked nodes of one level
        // with the same in-degree D in 1..4 (no edges among them)
        if (x < n) {
            const int32_t D = (int32_t)ent[x].size();
            int32_t G = 1;
            while (D >= 1 && D <= 4 && G < 4 && i + G < NT) {
                const int32_t y = order[i + G];
                if (y >= n || !aff[y] || (int32_t)ent[y].size() != D) break;
                bool same = true;       // same level: y reads none of the group
                for (int32_t q = 0; q < G && same; q++)
                    for (uint32_t e : ent[y]) {
                        const int32_t z = order[i + q];
                        if (e == (uint32_t)z) same = false;
                        if ((e & kLU) && (g->h_elig[e & kIdx] == z)) same = false;
                    }
                if (!same) break;
                G++;
            }
            if (G > 1) {
                const uint32_t off = (uint32_t)pent.size();
                for (int32_t q = 0; q < G; q++) {
                    const int32_t y = order[i + q];
                    lnode.push_back(y);
                    nrec.push_back(make_uint4(0u, 0u, best_slot[y], 0xFFFFFFFFu));
                    nadj.push_back(make_uint2(q == 0 ? off : (uint32_t)pent.size(),
                                              q == 0 ? ((uint32_t)D | (2u << 24) | ((uint32_t)G << 26)) : (uint32_t)D));
                    for (uint32_t e : ent[y]) {
                        const uint32_t v = (e & kLU) ? e : ref((int32_t)e);
                        if (v == kNoSlot) return set_error(MAGIS_E_INVAL, "internal: reader of an unslotted value");
                        pent.push_back(v);
                    }
                }
                ngrouped += G;
                i += G - 1;
                continue;
            }
        }
        uint32_t gate = 0xFFFFFFFFu;
        if (x >= n) {
            const int32_t r = (x - n) / 3, o = (x - n) % 3;
            gate = ((uint32_t)r << 2) | (o == 0 ? 1u : 2u);
        }
        lnode.push_back(x);
        nrec.push_back(make_uint4(0u, 0u, aff[x] ? best_slot[x] : kNoSlot, gate));
        if (!aff[x]) {
            nadj.push_back(make_uint2((uint32_t)x, (uint32_t)ent[x].size() | (1u << 24)));
            continue;
        }
        nadj.push_back(make_uint2((uint32_t)pent.size(), (uint32_t)ent[x].size()));
        for (uint32_t e : ent[x]) {
            const uint32_t v = (e & kLU) ? e : ref((int32_t)e);
            if (v == kNoSlot) return set_error(MAGIS_E_INVAL, "internal: reader of an unslotted value");
            pent.push_back(v);
        }
    }
    std::vector<uint4> rslot(std::max(R, 1));
    for (int32_t r = 0; r < R; r++) {
        const int32_t t = g->h_elig[r];
        rslot[r] = make_uint4(ref(t), ref(n + 3 * r), ref(n + 3 * r + 2), ref(t));
    }
    // constant nodes in order, with their predecessors (all constant)
    std::vector<int32_t> cnode, cptr(1, 0), cpred;
    std::vector<uint8_t> corig;
    for (int32_t x : order) {
        if (aff[x]) continue;
        cnode.push_back(x);
        corig.push_back(x < n ? 1 : 0);
        for (uint32_t e : ent[x]) cpred.push_back((int32_t)e);
        cptr.push_back((int32_t)cpred.size());
    }
    // per node: label source and in-degree (for h1)
    std::vector<uint32_t> lsrc(NT);
    std::vector<int32_t> degv(NT);
    int32_t cmaxdeg = 1;
    for (int32_t x = 0; x < NT; x++) {
        if (x < n) lsrc[x] = (uint32_t)x;
        else {
            const int32_t r = (x - n) / 3, o = (x - n) % 3;
            lsrc[x] = o == 0 ? (uint32_t)g->h_elig[r] : o == 1 ? kLabStore : kLabLoad;
        }
        degv[x] = (int32_t)ent[x].size();
        cmaxdeg = std::max(cmaxdeg, degv[x]);
    }
    const int32_t nloop = (int32_t)lnode.size(), nc = (int32_t)cnode.size();

    magis_ghash* h = new (std::nothrow) magis_ghash();
    if (!h) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    h->g = g;
    h->device = g->device;
    DeviceGuard guard(g->device);
    size_t off = 0;
    auto al = [&](size_t bytes) { const size_t o = off; off = (off + std::max<size_t>(bytes, 1) + 255) / 256 * 256; return o; };
    const size_t o_nrec = al(16 * (size_t)nloop), o_nadj = al(8 * (size_t)nloop), o_pent = al(4 * pent.size()),
                 o_rslot = al(16 * rslot.size()), o_x0 = al(8 * (size_t)NT), o_c0 = al(8), o_h1 = al(8 * (size_t)NT),
                 o_lab = al(8 * (size_t)n), o_lsrc = al(4 * (size_t)NT), o_deg = al(4 * (size_t)NT),
                 o_cnode = al(4 * (size_t)nc), o_cptr = al(4 * cptr.size()), o_cpred = al(4 * cpred.size()),
                 o_corig = al(corig.size()), o_tmp = al(8 * (size_t)cmaxdeg), o_lnode = al(4 * (size_t)nloop);
    if (cudaMalloc(&h->tables, off) != cudaSuccess) {
        cudaGetLastError();
        delete h;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc GraphHash tables failed");
    }
    char* b = (char*)h->tables;
    cudaError_t e = cudaSuccess;
    auto up = [&](size_t o, const void* src, size_t bytes) {
        if (e == cudaSuccess && bytes) e = cudaMemcpy(b + o, src, bytes, cudaMemcpyHostToDevice);
    };
    up(o_nrec, nrec.data(), 16 * (size_t)nloop);
    up(o_nadj, nadj.data(), 8 * (size_t)nloop);
    up(o_pent, pent.data(), 4 * pent.size());
    up(o_rslot, rslot.data(), 16 * rslot.size());
    up(o_lab, h_label, 8 * (size_t)n);
    up(o_lsrc, lsrc.data(), 4 * (size_t)NT);
    up(o_deg, degv.data(), 4 * (size_t)NT);
    up(o_cnode, cnode.data(), 4 * (size_t)nc);
    up(o_cptr, cptr.data(), 4 * cptr.size());
    up(o_cpred, cpred.data(), 4 * cpred.size());
    up(o_corig, corig.data(), corig.size());
    up(o_lnode, lnode.data(), 4 * (size_t)nloop);
    auto* h1 = (unsigned long long*)(b + o_h1);
    auto* x0 = (unsigned long long*)(b + o_x0);
    auto* c0 = (unsigned long long*)(b + o_c0);
    if (e == cudaSuccess) {
        ghash_h1_kernel<<<(NT + 255) / 256, 256>>>(NT, (const uint32_t*)(b + o_lsrc), (const int32_t*)(b + o_deg),
                                                   (const uint64_t*)(b + o_lab), h1);
        ghash_const_kernel<<<1, 1>>>(nc, (const int32_t*)(b + o_cnode), (const int32_t*)(b + o_cptr),
                                     (const int32_t*)(b + o_cpred), (const uint8_t*)(b + o_corig), h1, x0,
                                     (unsigned long long*)(b + o_tmp), c0);
        if (nloop)
            ghash_fill_kernel<<<(nloop + 255) / 256, 256>>>(nloop, (const int32_t*)(b + o_lnode), h1,
                                                             (uint4*)(b + o_nrec));
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    GhDev& d = h->dev;
    d.nloop = nloop; d.R = R; d.NS = NS; d.gslots = best_gs; d.maxdeg = maxdeg > 32 ? maxdeg : 0; d.Rw = Rw;
    d.nrec = (const uint4*)(b + o_nrec);
    d.nadj = (const uint2*)(b + o_nadj);
    d.pent = (const uint32_t*)(b + o_pent);
    d.rslot = (const uint4*)(b + o_rslot);
    d.rflag = g->dev.rflag;
    d.x0 = x0;
    d.c0 = c0;
    h->n_global_nodes = best_glob;
    h->n_const_nodes = nc;
    h->n_grouped = ngrouped;
    h->smem = (size_t)kGhWarps * ((size_t)NS * 256 + (size_t)Rw * 128);
    const void* fn = (const void*)ghash_kernel;
    if (e == cudaSuccess) e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)h->smem);
    int occ = 0;
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, 32 * kGhWarps, h->smem);
    if (e == cudaSuccess && occ < 1) e = cudaErrorInvalidConfiguration;
    if (e == cudaSuccess) {
        h->grid = sms * occ;
        const size_t per_warp = (size_t)(d.gslots + 2 * d.maxdeg) * 32 * 8;
        h->scratch_bytes = std::max<size_t>(per_warp * (size_t)h->grid * kGhWarps, 256);
        if (cudaMalloc(&h->scratch, h->scratch_bytes) != cudaSuccess) e = cudaErrorMemoryAllocation;
        d.gbuf = (unsigned long long*)h->scratch;
    }
    if (e != cudaSuccess) {
        cudaGetLastError();
        if (h->tables) cudaFree(h->tables);
        if (h->scratch) cudaFree(h->scratch);
        delete h;
        return set_error(e == cudaErrorMemoryAllocation ? MAGIS_E_NOMEM : MAGIS_E_CUDA,
                         std::string("GraphHash setup: ") + cudaGetErrorString(e));
    }
    if (std::getenv("MAGIS_DEBUG"))
        std::fprintf(stderr,
                     "[magis] ghash NT=%d walked=%d const=%d grouped=%lld NS=%d gslots=%d global-nodes=%lld maxdeg=%d "
                     "grid=%d occ=%d smem=%zu scratch=%zu\n",
                     NT, nloop, nc, (long long)ngrouped, NS, d.gslots, (long long)best_glob, maxdeg, h->grid, occ, h->smem,
                     h->scratch_bytes);
    *out = h;
    return MAGIS_SUCCESS;
}

extern "C" int magis_ghash_free(magis_ghash* h) {
    clear_error();
    if (!h) return MAGIS_SUCCESS;
    DeviceGuard guard(h->device);
    cudaDeviceSynchronize();
    if (h->tables) cudaFree(h->tables);
    if (h->scratch) cudaFree(h->scratch);
    cudaGetLastError();
    delete h;
    return MAGIS_SUCCESS;
}

extern "C" int magis_graph_hash(magis_ghash* h, int64_t K, const uint8_t* d_dec, uint8_t* d_status,
                                uint64_t* d_hash, void* cuda_stream) {
    clear_error();
    if (!h) return set_error(MAGIS_E_INVAL, "ghash is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_status || !d_hash) return set_error(MAGIS_E_INVAL, "null device pointer");
    if (h->dev.R > 0 && !d_dec) return set_error(MAGIS_E_INVAL, "d_dec is NULL but R > 0");
    DeviceGuard guard(h->device);
    const int64_t groups = (K + 31) / 32;
    const int grid = (int)std::min<int64_t>(h->grid, (groups + kGhWarps - 1) / kGhWarps);
    // 16-byte decision loads when every row starts 16-byte aligned
    const int vec = (h->dev.R % 16 == 0) && ((uintptr_t)d_dec % 16 == 0);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    ghash_kernel<<<grid, 32 * kGhWarps, h->smem, st>>>(h->dev, K, d_dec, vec, d_status, d_hash);
    GCK(cudaGetLastError());
    return MAGIS_SUCCESS;
}

extern "C" int magis_ghash_info(const magis_ghash* h, int32_t* shared_slots, int32_t* global_slots,
                                int64_t* global_nodes, int32_t* grid) {
    clear_error();
    if (!h) return set_error(MAGIS_E_INVAL, "ghash is NULL");
    if (shared_slots) *shared_slots = h->dev.NS;
    if (global_slots) *global_slots = h->dev.gslots;
    if (global_nodes) *global_nodes = h->n_global_nodes;
    if (grid) *grid = h->grid;
    return MAGIS_SUCCESS;
}
