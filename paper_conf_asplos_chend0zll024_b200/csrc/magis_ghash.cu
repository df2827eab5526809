// magis_ghash.cu -- batched GraphHash and the duplicate filter (SURVEY §8(f)
// NEXT-2; Alg. 3 lines 3-6 and 10-12; the Weisfeiler-Lehman
// idea).  Readings G1-G4 are in DESIGN.md §3.
//
// The graph of candidate k is its transformed graph (Fig. 8 rules applied to
// the decisions dec[k]; the schedule does not enter, reading G4).  Per node,
// in one fixed topological order of the super-graph:
//     x_v = hash( hash(label_v) (+) x_{u_1} (+) ... (+) x_{u_d} )   (line 5)
// with u_1..u_d = pre(v) in ascending order of x (reading G2), and
//     GraphHash = hash( sum_v x_v mod 2^64 )                         (line 6)
// hash() over 64-bit words: h = GAMMA (m + 1), h = mix64(h ^ w_i) (reading G1).
//
// B200 layout: lane = candidate.  A warp walks the node table (warp-uniform,
// L1-broadcast loads) for 32 candidates at once; the decisions only switch
// which slot a late-user edge reads (t_r, the clone or the Load) and whether
// an optional node is active, so control flow stays uniform.  x values live
// in "slots" assigned at create time by a linear scan over the order (a slot
// is reused once its last potential reader has run): short-lived values in
// shared memory ([slot][lane], conflict-free), long-lived ones (forward
// activations read by the backward pass) in a per-warp global region with
// the same lane-interleaved layout (256-byte coalesced rows, L2-resident).
// Predecessor values are sorted in registers by a bitonic network sized to
// the warp-uniform in-degree.
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
constexpr uint32_t kNoSlot = 0xFFFFFFFFu;
constexpr uint32_t kLU = 0x80000000u;             // late-user entry: low bits = r
constexpr int kGhWarps = 4;                        // warps per CTA
constexpr int kGhCtasPerSm = 4;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

struct GhDev {
    int32_t NT, R, NS;        // nodes in the order, eligible tensors, shared slots per warp
    int32_t gslots;           // global slots per warp
    int32_t maxdeg;           // largest in-degree (> 32 uses the rank sort in global scratch)
    int32_t Rw;               // u32 words of packed decisions per candidate (16 per word)
    const uint4* nrec;        // [NT] (hash(label) lo, hi, slot, gate); gate ~0 = always active
    const uint2* nadj;        // [NT] (offset into pent, in-degree)
    const uint32_t* pent;     // slot, or kLU | r
    const uint4* rslot;       // [R] (slot of t_r, clone_r, load_r, slot of t_r)
    const uint8_t* rflag;     // [R] kRHasInput
    unsigned long long* gbuf; // [warps][gslots + 2 maxdeg][32]
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
    int64_t n_global_nodes = 0;   // nodes whose x lives in the global slots
};

struct magis_hashset {
    int device = 0;
    uint64_t cap = 0;                  // power of two
    unsigned long long* keys = nullptr;     // [cap] 0 = empty
    unsigned long long* owner = nullptr;    // [cap + 1] (epoch << 40 | first id); [cap] = key 0
    unsigned long long* stats = nullptr;    // [2] occupied slots, overflowed inserts
    uint32_t epoch = 0;
};

namespace magis {
namespace {

// ------------------------------------------------------------------ device --
__global__ void ghash_label_kernel(uint4* nrec, int32_t NT, const uint64_t* label) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= NT) return;
    uint4 r = nrec[i];
    // label source: r.x = original id (or t_r), r.y = kind (0 op / clone, 1 Store, 2 Load)
    const uint64_t lab = r.y == 0 ? label[r.x] : (r.y == 1 ? kTagStore : kTagLoad);
    const uint64_t h = mix64((kGamma * 2ull) ^ lab);             // hash([label]), m = 1
    r.x = (uint32_t)h;
    r.y = (uint32_t)(h >> 32);
    nrec[i] = r;
}

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

struct Lane {
    const GhDev& d;
    const unsigned long long* xs;      // shared slots of this warp
    unsigned long long* gb;            // global slots of this warp
    const uint32_t* decp;              // packed decisions of this warp
    int lane;
    __device__ __forceinline__ uint32_t dec(uint32_t r) const {
        return (decp[(r >> 4) * 32 + lane] >> (2 * (r & 15))) & 3u;
    }
    __device__ __forceinline__ uint32_t slot_of(uint32_t e) const {
        if (!(e & kLU)) return e;
        const uint4 rs = __ldg(d.rslot + (e & ~kLU));
        const uint32_t dd = dec(e & ~kLU);
        return dd == 1 ? rs.y : dd == 2 ? rs.z : rs.x;
    }
    __device__ __forceinline__ uint64_t get(uint32_t e) const {
        const uint32_t s = slot_of(e);
        return s < (uint32_t)d.NS ? xs[s * 32 + lane] : gb[(size_t)(s - d.NS) * 32 + lane];
    }
};

template <int D>
__device__ __forceinline__ uint64_t hash_preds(const Lane& L, const uint32_t* ent, int deg, uint64_t h) {
    uint64_t a[D];
#pragma unroll
    for (int j = 0; j < D; j++) a[j] = j < deg ? L.get(__ldg(ent + j)) : ~0ull;
    bitonic<D>(a);
#pragma unroll
    for (int j = 0; j < D; j++)
        if (j < deg) h = mix64(h ^ a[j]);
    return h;
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
    const Lane L{d, xs, gb, decp, lane};

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
        uint64_t sum = 0;
        for (int32_t i = 0; i < d.NT; i++) {
            const uint4 rec = __ldg(d.nrec + i);
            bool act = true;
            if (rec.w != 0xFFFFFFFFu) act = L.dec(rec.w >> 2) == (rec.w & 3u);
            if (!__any_sync(0xffffffffu, act)) continue;
            const uint2 adj = __ldg(d.nadj + i);
            const uint32_t* ent = d.pent + adj.x;
            const int deg = (int)adj.y;
            uint64_t h = mix64((kGamma * (uint64_t)(deg + 2)) ^ (((uint64_t)rec.y << 32) | rec.x));
            if (deg <= 4) {
                h = hash_preds<4>(L, ent, deg, h);
            } else if (deg <= 8) {
                h = hash_preds<8>(L, ent, deg, h);
            } else if (deg <= 32) {
                h = hash_preds<32>(L, ent, deg, h);
            } else {
                // rank sort in this lane's global scratch column (rare: merges of > 32 parts)
                unsigned long long* t0 = gb + (size_t)d.gslots * 32;
                unsigned long long* t1 = t0 + (size_t)d.maxdeg * 32;
                for (int j = 0; j < deg; j++) t0[(size_t)j * 32 + lane] = L.get(__ldg(ent + j));
                for (int j = 0; j < deg; j++) {
                    const uint64_t v = t0[(size_t)j * 32 + lane];
                    int rk = 0;
                    for (int q = 0; q < deg; q++) {
                        const uint64_t u = t0[(size_t)q * 32 + lane];
                        rk += (u < v) | ((u == v) & (q < j));
                    }
                    t1[(size_t)rk * 32 + lane] = v;
                }
                for (int j = 0; j < deg; j++) h = mix64(h ^ t1[(size_t)j * 32 + lane]);
            }
            if (act) {
                sum += h;
                const uint32_t s = rec.z;
                if (s < (uint32_t)d.NS) xs[s * 32 + lane] = h;
                else if (s != kNoSlot) gb[(size_t)(s - d.NS) * 32 + lane] = h;
            }
            __syncwarp();
        }
        if (valid) {
            out_status[k] = bad ? (uint8_t)MAGIS_ST_BAD_DEC : (uint8_t)0;
            out_hash[k] = bad ? 0ull : mix64((kGamma * 2ull) ^ sum);       // line 6: hash([sum])
        }
        __syncwarp();
    }
}

// hash set: open addressing, linear probing, 64-bit keys (0 = empty; the
// key 0 has its own owner word at [cap])
__device__ __forceinline__ uint64_t probe_start(uint64_t h, uint64_t mask) { return mix64(h) & mask; }

__global__ void hs_insert_kernel(magis_hashset s, int64_t K, const uint64_t* __restrict__ hash,
                                 const uint8_t* __restrict__ status) {
    const uint64_t mask = s.cap - 1;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        if (status && status[k]) continue;
        const unsigned long long h = hash[k];
        const unsigned long long me = ((unsigned long long)s.epoch << 40) | (unsigned long long)k;
        if (h == 0) { atomicMin(s.owner + s.cap, me); continue; }
        uint64_t i = probe_start(h, mask);
        bool done = false;
        for (uint64_t p = 0; p < s.cap; p++) {
            const unsigned long long prev = atomicCAS(s.keys + i, 0ull, h);
            if (prev == 0ull || prev == h) {
                if (prev == 0ull) atomicAdd(s.stats, 1ull);
                atomicMin(s.owner + i, me);
                done = true;
                break;
            }
            i = (i + 1) & mask;
        }
        if (!done) atomicAdd(s.stats + 1, 1ull);
    }
}

__global__ void hs_mark_kernel(magis_hashset s, int64_t K, const uint64_t* __restrict__ hash,
                               const uint8_t* __restrict__ status, uint8_t* __restrict__ is_new) {
    const uint64_t mask = s.cap - 1;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        if (status && status[k]) { is_new[k] = 0; continue; }
        const unsigned long long h = hash[k];
        const unsigned long long me = ((unsigned long long)s.epoch << 40) | (unsigned long long)k;
        uint8_t r = 1;                           // not found (table full): kept as new
        if (h == 0) {
            r = s.owner[s.cap] == me;
        } else {
            uint64_t i = probe_start(h, mask);
            for (uint64_t p = 0; p < s.cap; p++) {
                const unsigned long long key = s.keys[i];
                if (key == h) { r = s.owner[i] == me; break; }
                if (key == 0ull) break;
                i = (i + 1) & mask;
            }
        }
        is_new[k] = r;
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
    std::vector<int32_t> hp(NT);
    for (int32_t i = 0; i < NT; i++) hp[order[i]] = i;
    // potential readers -> last position; predecessor entries
    std::vector<int32_t> lastp(NT);
    for (int32_t i = 0; i < NT; i++) lastp[order[i]] = i;
    auto rd = [&](int32_t u, int32_t at) { lastp[u] = std::max(lastp[u], at); };
    std::vector<std::vector<uint32_t>> ent(NT);   // node -> entries (node ids / kLU|r), slots filled later
    int32_t maxdeg = 0;
    for (int32_t v = 0; v < n; v++) {
        for (int32_t e = pp[v]; e < pp[v + 1]; e++) {
            const int32_t u = pr[e];
            const int32_t r = r_of[u];
            bool lu = false;
            if (r >= 0) for (int32_t rr : Umem[v]) if (rr == r) { lu = true; break; }
            if (lu) {
                ent[v].push_back(kLU | (uint32_t)r);
                rd(u, hp[v]); rd(n + 3 * r, hp[v]); rd(n + 3 * r + 2, hp[v]);
            } else {
                ent[v].push_back((uint32_t)u);
                rd(u, hp[v]);
            }
        }
        maxdeg = std::max<int32_t>(maxdeg, (int32_t)ent[v].size());
    }
    for (int32_t r = 0; r < R; r++) {
        const int32_t t = g->h_elig[r], c = n + 3 * r, st = c + 1, ld = c + 2;
        for (int32_t e = pp[t]; e < pp[t + 1]; e++) { ent[c].push_back((uint32_t)pr[e]); rd(pr[e], hp[c]); }
        ent[st].push_back((uint32_t)t); rd(t, hp[st]);
        ent[ld].push_back((uint32_t)st); rd(st, hp[ld]);
        maxdeg = std::max<int32_t>(maxdeg, (int32_t)ent[c].size());
    }
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
    // slots by linear scan; a value that dies within TS positions prefers shared
    // memory.  TS is picked to minimise the number of values sent to global.
    std::vector<uint32_t> best_slot;
    int32_t best_gs = 0;
    int64_t best_glob = -1;
    for (int32_t TS : {1, 2, 4, 8, 16, 32, 64, 128, 256, 1 << 30}) {
        std::vector<uint32_t> slot(NT, kNoSlot);
        std::vector<std::vector<int32_t>> dies(NT + 1);
        std::vector<uint32_t> sfree, gfree;
        for (int32_t s = NS - 1; s >= 0; s--) sfree.push_back((uint32_t)s);
        int32_t gused = 0;
        int64_t nglob = 0;
        for (int32_t i = 0; i < NT; i++) {
            const int32_t x = order[i];
            if (i > 0)
                for (int32_t y : dies[i - 1]) {
                    if (slot[y] < (uint32_t)NS) sfree.push_back(slot[y]);
                    else gfree.push_back(slot[y]);
                }
            if (lastp[x] == i) continue;             // no reader after it: x is only summed
            const bool shortl = lastp[x] - i <= TS;
            if (shortl && !sfree.empty()) { slot[x] = sfree.back(); sfree.pop_back(); }
            else if (!gfree.empty()) { slot[x] = gfree.back(); gfree.pop_back(); nglob++; }
            else { slot[x] = (uint32_t)(NS + gused++); nglob++; }
            dies[lastp[x]].push_back(x);
        }
        if (best_glob < 0 || nglob < best_glob) { best_glob = nglob; best_slot = slot; best_gs = gused; }
    }
    // tables: nrec, nadj, pent, rslot
    std::vector<uint4> nrec(NT);
    std::vector<uint2> nadj(NT);
    std::vector<uint32_t> pent;
    for (int32_t i = 0; i < NT; i++) {
        const int32_t x = order[i];
        uint32_t src = 0, kind = 0, gate = 0xFFFFFFFFu;
        if (x < n) src = (uint32_t)x;
        else {
            const int32_t r = (x - n) / 3, o = (x - n) % 3;
            src = (uint32_t)g->h_elig[r];
            kind = (uint32_t)o;                      // 0 clone (label of t_r), 1 Store, 2 Load
            gate = ((uint32_t)r << 2) | (o == 0 ? 1u : 2u);
        }
        nrec[i] = make_uint4(src, kind, best_slot[x], gate);
        nadj[i] = make_uint2((uint32_t)pent.size(), (uint32_t)ent[x].size());
        for (uint32_t e : ent[x]) pent.push_back((e & kLU) ? e : best_slot[e]);
    }
    std::vector<uint4> rslot(std::max(R, 1));
    for (int32_t r = 0; r < R; r++) {
        const int32_t t = g->h_elig[r];
        rslot[r] = make_uint4(best_slot[t], best_slot[n + 3 * r], best_slot[n + 3 * r + 2], best_slot[t]);
    }
    for (uint32_t e : pent)
        if (!(e & kLU) && e == kNoSlot) return set_error(MAGIS_E_INVAL, "internal: reader of an unslotted value");

    magis_ghash* h = new (std::nothrow) magis_ghash();
    if (!h) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    h->g = g;
    h->device = g->device;
    DeviceGuard guard(g->device);
    auto al = [](size_t x) { return (x + 255) / 256 * 256; };
    const size_t o_nrec = 0, o_nadj = al(o_nrec + 16 * (size_t)NT), o_pent = al(o_nadj + 8 * (size_t)NT),
                 o_rslot = al(o_pent + 4 * std::max<size_t>(pent.size(), 1)),
                 o_lab = al(o_rslot + 16 * rslot.size()), total = al(o_lab + 8 * (size_t)n);
    if (cudaMalloc(&h->tables, total) != cudaSuccess) {
        cudaGetLastError();
        delete h;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc GraphHash tables failed");
    }
    char* b = (char*)h->tables;
    cudaError_t e = cudaMemcpy(b + o_nrec, nrec.data(), 16 * (size_t)NT, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(b + o_nadj, nadj.data(), 8 * (size_t)NT, cudaMemcpyHostToDevice);
    if (e == cudaSuccess && !pent.empty()) e = cudaMemcpy(b + o_pent, pent.data(), 4 * pent.size(), cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(b + o_rslot, rslot.data(), 16 * rslot.size(), cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemcpy(b + o_lab, h_label, 8 * (size_t)n, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) {
        ghash_label_kernel<<<(NT + 255) / 256, 256>>>((uint4*)(b + o_nrec), NT, (const uint64_t*)(b + o_lab));
        e = cudaGetLastError();
    }
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    GhDev& d = h->dev;
    d.NT = NT; d.R = R; d.NS = NS; d.gslots = best_gs; d.maxdeg = maxdeg > 32 ? maxdeg : 0; d.Rw = Rw;
    d.nrec = (const uint4*)(b + o_nrec);
    d.nadj = (const uint2*)(b + o_nadj);
    d.pent = (const uint32_t*)(b + o_pent);
    d.rslot = (const uint4*)(b + o_rslot);
    d.rflag = g->dev.rflag;
    h->n_global_nodes = best_glob;
    h->smem = (size_t)kGhWarps * ((size_t)NS * 256 + dec_bytes);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(ghash_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)h->smem);
    int occ = 0;
    if (e == cudaSuccess)
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ghash_kernel, 32 * kGhWarps, h->smem);
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
        std::fprintf(stderr, "[magis] ghash NT=%d NS=%d gslots=%d global-nodes=%lld maxdeg=%d grid=%d occ=%d smem=%zu\n",
                     NT, NS, d.gslots, (long long)best_glob, maxdeg, h->grid, occ, h->smem);
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
    ghash_kernel<<<grid, 32 * kGhWarps, h->smem, (cudaStream_t)cuda_stream>>>(h->dev, K, d_dec, vec, d_status,
                                                                              d_hash);
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

extern "C" int magis_hashset_create(int device, int64_t capacity, magis_hashset** out) {
    clear_error();
    if (!out) return set_error(MAGIS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (capacity < 1 || capacity > (1ll << 40)) return set_error(MAGIS_E_INVAL, "capacity out of range");
    if (!magis_device_supported(device))
        return set_error(MAGIS_E_UNSUPPORTED, "device " + std::to_string(device) +
                         " is not an sm_100 (B200) GPU; there is no CPU fallback");
    DeviceGuard guard(device);
    magis_hashset* s = new (std::nothrow) magis_hashset();
    if (!s) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    uint64_t cap = 1;
    while (cap < (uint64_t)capacity) cap <<= 1;
    s->device = device;
    s->cap = cap;
    if (cudaMalloc(&s->keys, cap * 8) != cudaSuccess || cudaMalloc(&s->owner, (cap + 1) * 8) != cudaSuccess ||
        cudaMalloc(&s->stats, 16) != cudaSuccess) {
        cudaGetLastError();
        if (s->keys) cudaFree(s->keys);
        if (s->owner) cudaFree(s->owner);
        delete s;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc hash set failed");
    }
    const int rc = magis_hashset_clear(s, nullptr);
    if (rc != MAGIS_SUCCESS || cudaDeviceSynchronize() != cudaSuccess) {
        cudaGetLastError();
        cudaFree(s->keys);
        cudaFree(s->owner);
        cudaFree(s->stats);
        delete s;
        return set_error(MAGIS_E_CUDA, "hash set initialisation failed");
    }
    *out = s;
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_clear(magis_hashset* s, void* cuda_stream) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    DeviceGuard guard(s->device);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    GCK(cudaMemsetAsync(s->keys, 0, s->cap * 8, st));
    GCK(cudaMemsetAsync(s->owner, 0xFF, (s->cap + 1) * 8, st));
    GCK(cudaMemsetAsync(s->stats, 0, 16, st));
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_free(magis_hashset* s) {
    clear_error();
    if (!s) return MAGIS_SUCCESS;
    DeviceGuard guard(s->device);
    cudaDeviceSynchronize();
    cudaFree(s->keys);
    cudaFree(s->owner);
    cudaFree(s->stats);
    cudaGetLastError();
    delete s;
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_filter(magis_hashset* s, int64_t K, const uint64_t* d_hash, const uint8_t* d_status,
                                    uint8_t* d_new, void* cuda_stream) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    if (K < 0 || K >= (1ll << 40)) return set_error(MAGIS_E_INVAL, "K out of range");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_hash || !d_new) return set_error(MAGIS_E_INVAL, "null device pointer");
    if (s->epoch + 1 >= (1u << 24)) return set_error(MAGIS_E_CAPACITY, "hash set epoch exhausted: clear it");
    DeviceGuard guard(s->device);
    s->epoch++;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    const int grid = (int)std::min<int64_t>((K + 255) / 256, 148 * 16);
    hs_insert_kernel<<<grid, 256, 0, st>>>(*s, K, d_hash, d_status);
    GCK(cudaGetLastError());
    hs_mark_kernel<<<grid, 256, 0, st>>>(*s, K, d_hash, d_status, d_new);
    GCK(cudaGetLastError());
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_stats(const magis_hashset* s, int64_t* n_keys, int64_t* n_overflow) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    DeviceGuard guard(s->device);
    unsigned long long h[2] = {0, 0};
    GCK(cudaMemcpy(h, s->stats, 16, cudaMemcpyDeviceToHost));
    unsigned long long z = 0;
    GCK(cudaMemcpy(&z, s->owner + s->cap, 8, cudaMemcpyDeviceToHost));
    if (n_keys) *n_keys = (int64_t)h[0] + (z != ~0ull ? 1 : 0);
    if (n_overflow) *n_overflow = (int64_t)h[1];
    return MAGIS_SUCCESS;
}
