// magis_internal.h -- shared declarations of the B200 evaluation library.
// Not part of the ABI (see include/magis.h).
#pragma once

#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "magis.h"

namespace magis {

// Activation gate of a super-graph node or edge (reading P6, Fig. 8):
// -1 = always active, otherwise (r << 2) | d = active iff dec[r] == d.
constexpr int32_t kAlways = -1;

// Per-node flags.
constexpr uint8_t kFlagOutput = 1;    // outs(G): live to the end (reading P2)
constexpr uint8_t kFlagCompute = 2;   // runs on the compute queue (original op or clone)

// Per-eligible flags.
constexpr uint8_t kRHasInput = 1;     // t_r has inputs: re-mat allowed

// Swap-latency event types, in the order events at one step are applied.
constexpr uint32_t kEvStall = 0;      // compute op waits for a Load it reads
constexpr uint32_t kEvProduce = 1;    // producer t_r of a swapped tensor finishes
constexpr uint32_t kEvStore = 2;      // Store on the D2H queue
constexpr uint32_t kEvLoad = 3;       // Load on the H2D queue

// Device view of one loaded graph (all pointers are device memory).
struct DevGraph {
    int32_t n;           // original nodes
    int32_t R;           // eligible tensors
    int32_t NT;          // n + 3R
    int32_t max_events;  // 3R + |U| (swap events of one candidate, upper bound)
    const int32_t* cons_ptr;   // [NT+1]
    const int2* cons_ent;      // (consumer id, gate)
    const int32_t* in_ptr;     // [NT+1]
    const int2* in_ent;        // (input id, gate)
    const int64_t* size;       // [NT] device bytes of the node's output when active (P5, P9)
    const double* cost;        // [NT] compute cost (0 for Store / Load)
    const int32_t* ngate;      // [NT]
    const uint8_t* nflag;      // [NT]
    const int32_t* elig;       // [R] t_r
    const int32_t* U_ptr;      // [R+1]
    const int32_t* U_idx;      // U_r
    const double* xfer;        // [R] swap_latency + |t_r| / bytes_per_s
    const double* tcost;       // [R] cost(t_r)
    const uint8_t* rflag;      // [R]
    double base_cost;          // sum of cost over original nodes
    const int32_t* dtin;       // [n] dominator-tree preorder index (NEXT-3)
    const int32_t* dtout;      // [n] end of the node's preorder range
    const int32_t* pred_ptr;   // [n+1] predecessors in G (deduplicated)
    const int32_t* pred;
    // F-Trans variant regions (NEXT-4, reading F1): a candidate's decision
    // row is [R eligible decisions | F region variants]; gates of region
    // nodes index dec[R + i]
    int32_t F;                 // regions (0: none)
    int32_t Rd;                // decision row length R + F
    const int32_t* nvar;       // [F] variants per region (<= 4)
    const double* vcost;       // [4F] sum of cost over the nodes of (region, variant)
};

// Variant-2 plan (magis_eval2.cu): graph as per-thread streams in shared
// memory, P candidates packed per u16 lane group.  Built on the host by
// plan2_build; all offsets are bytes into the dynamic shared memory.
#ifndef MAGIS_MAIN_THREADS
#define MAGIS_MAIN_THREADS 512
#endif
constexpr int kMainThreads2 = MAGIS_MAIN_THREADS;   // main (non-latency) threads of a variant-2 CTA

struct Plan2 {
    int32_t P;            // candidates per group (1, 2, 4); 0 = not applicable
    int32_t NT, NTX, n, R, nU;
    int32_t L, S;         // scan chunk length / slot stride (L * S >= NT, S <= kMainThreads2)
    int64_t unit;         // bytes per size unit (gcd of sizes)
    int32_t max_events;   // 3R + |U|
    uint32_t Lm;          // ceil(2^32 / L) (L a multiple of 4): st / L = umulhi(st, Lm)
    uint32_t static_bytes;   // bulk-staged prefix (graph rows + size units)
    uint32_t off_wtab;       // [WM][4]: consumer rows [b, e), input rows [b, e)
    uint32_t off_crow, off_chdr, off_cent;                  // consumer rows: (offset, degree), headers, edges
    uint32_t off_csize;                                     // consumer rows: size units per header (row order)
    uint32_t off_frow, off_fhdr, off_fent;                  // input rows
    uint32_t off_size;       // [NTX] size units
    uint32_t off_rtab;       // [R] double2 (cost(t_r), swap transfer time)
    uint32_t off_cost;       // [NTX] compute cost (f64; clone = cost(t_r), Store / Load 0)
    uint32_t off_ninfo;      // [n] uint2: x = (r + 1 if node is t_r, else 0) | |{r : node in U_r}| << 16,
                             //            y = offset of that r list in lul
    uint32_t off_lul;        // u16 r lists (late-user -> tensors), see off_ninfo
    uint32_t off_urow;       // [R] u32: offset of U_r in ubs | |U_r| << 16
    uint32_t off_ubs;        // [nU] u16 late users, grouped by r
    uint32_t off_utr;        // [R] u16 t_r
    int32_t F, Rd;           // F-Trans regions (NEXT-4) and the decision row length R + F
    int32_t nRN;             // nodes inside regions (every variant)
    uint32_t off_rn;         // [nRN] u32: node id | region << 16 | variant << 30
    uint32_t off_nvar;       // [F] u8 variants per region
    uint32_t off_vcost;      // [4F] f64 cost sum of (region, variant)
    int32_t gate_lo;         // smallest id of a node that may be absent (region nodes, then n)
    uint64_t l2win_bytes;    // tiers 1-3: bytes of the graph image under an L2 persisting window (0: none)
    int32_t cost_cls;        // tier 2: the cost table staged as u8 class indices + <= 256 class values
    uint32_t off_ccls;       // image offset of [class values f64 (a16) | class index u8 [NTX]]
    uint32_t ccls_idx_off;   // offset of the class index inside that region
    uint32_t stage_bytes;    // bytes staged into shared memory on tiers 1 / 2 (cost table or classes)
    int32_t rows_sm;         // tier 1: [wtab, crow, chdr, cent] also staged, at shared offset rows_off
    uint32_t rows_off, rows_bytes;
    uint32_t image_bytes;    // whole device image (static_bytes staged on tier 0, then the class tables)
    uint32_t off_pos, off_last, off_af, off_dec, off_end;
    uint32_t off_evm;        // [P][NW] swap-event step marks (bit per step)
    uint32_t off_sdec;       // [2][P][Rw] decisions handed to the latency warp
    uint32_t off_ev;         // [2][P][evcap] event keys (u64) then [2][P][evcap] cost prefixes (f64)
    int32_t evcap;           // event steps per candidate held in shared memory
    int32_t nwm;             // NW: u32 words of marks per candidate
    uint64_t ovf_stride;     // bytes per overflow event region (global)
    uint32_t smem_total;
    int32_t gmem_static;  // graph tables read from the global image instead of shared memory
    int32_t gmem_af;      // per-step slots in a per-CTA global slice (af_bytes each)
    int32_t cost_sm;      // tables in global, but the cost table staged at shared offset 0
    int32_t delta_slots;  // tier 2: one signed int32 per step in shared memory, alloc(i) - free(i - 1)
    uint32_t state_base;  // offset of the per-candidate state in shared memory
    uint64_t af_bytes;
    int32_t prof;         // MAGIS_PROFILE: accumulate per-phase cycles
    uint64_t prof_off;    // byte offset of the 16 u64 phase counters in the scratch buffer
    int32_t teams;        // independent teams per CTA (1 or 2), each with its own per-group state and barriers
    uint32_t state_stride;   // bytes of shared memory per team's state (team t at + t * state_stride)
};

// Base-graph adjacency for the device candidate generator (magis_gen.cu).
struct GenTables {
    const int32_t* succ_ptr;   // [n+1]
    const int32_t* succ;
    const int32_t* pred_ptr;   // [n+1]
    const int32_t* pred;
    // fast path (magis_gen.cu gen2_kernel): sources of G in id order, and the
    // nodes whose base position the optional-node placement reads (t_r, its
    // inputs, U_r) as a compact slot map
    const int32_t* src;        // [S]
    const uint16_t* qmap;      // [n] slot or 0xffff
    const int32_t* qnode;      // [nq] node of each slot
    const uint2* sinfo;        // [n] (successor offset, count | slot << 16)
    const uint2* rec;          // [E] successor records in succ order: s | o0 << 16, o1 | o2 << 16
                               //     (the other inputs of s, 0xffff none; o0 = 0xfffe: more than 3
                               //     other inputs, then o1 = the node's wide slot, o2 = its in-degree)
    int32_t W;                 // wide nodes (in-degree > 4): per-candidate emitted-input counters
    int32_t S, nq;
    int32_t fast;              // n, nq < 65535 and R < 32768: the fast kernel applies
};

struct GenSpec {
    uint64_t seed;
    int32_t pct_random, pct_local, p_remat, p_swap, wmax, slack;
};

// One launch plan of the generator for a call of K candidates: grid threads of
// the fast kernel (0: the fast kernel does not apply) and of the sequential
// kernel (the whole call, or the re-run of the candidates whose ready set
// outgrew the fast kernel's on-chip heap), and the scratch they need.
struct GenPlan {
    int64_t T2 = 0, T1 = 0;
    int hc = 0, bsm = 0;       // fast kernel: on-chip heap entries, bitset on chip
    size_t w2 = 0;             // fast kernel scratch bytes per thread
    size_t bytes = 0;          // total scratch
};
GenPlan gen_plan(int device, const DevGraph& g, const GenTables& gt, int64_t K);
cudaError_t gen_launch(const DevGraph& g, const GenTables& gt, const GenSpec& sp, uint64_t id0, int64_t K,
                       int32_t* perm, uint8_t* dec, void* scratch, const GenPlan& gp, cudaStream_t stream);

// Base schedule for windowed delta evaluation (magis_window.cu).
struct BaseHdr {
    int status;
    int nev;
    long long peak;
    double latency;
    double ctot;
};
struct BaseDev {
    BaseHdr* hdr;
    int32_t* perm;      // [NT] step -> node
    int32_t* pos;       // [NT] node -> step
    int32_t* last;      // [NT] last reader step (NT for outputs, own step if none, -1 inactive)
    uint8_t* active;    // [NT]
    long long* carry;   // [NT+1] bytes live entering step i (before its allocation)
    long long* pm;      // [NT+1] max_{j<i} M_j (-1 if none)
    long long* sm;      // [NT+1] max_{j>=i} M_j (-1 if none)
    double* cb;         // [NT+1] compute cost before step i
    long long* mstep;   // [NT] M_i
    uint8_t* dec;       // [R]
    double* endb;       // [3R] scratch of the base sweep
    unsigned long long* evk;   // swap events of the base, step order
    double* snap;       // [(max_events + 1) * 3] (D, Td, Th) of the base sweep before each event
    int32_t* evix;      // [3R] index of the base event that writes endb[x] (INT_MAX: none)
};
size_t base_bytes(const DevGraph& g);
BaseDev base_layout(const DevGraph& g, void* mem);
cudaError_t base_launch(const DevGraph& g, const BaseDev& b, const int32_t* perm, const uint8_t* dec,
                        cudaStream_t s);
int window_grid(int device);
int window_wmax_supported();
cudaError_t window_launch(const DevGraph& g, const BaseDev& b, int grid, double* endb_ws, int64_t K,
                          const int32_t* wstart, const int32_t* wlen, const int32_t* wperm, int32_t wmax,
                          uint8_t* st, int64_t* pk, double* lt, cudaStream_t s);

struct EvalConfig {
    int variant;          // 0: per-candidate state in shared memory, 1: in global workspace,
                          // 2: packed streams (magis_eval2.cu)
    int grid;
    int block;
    size_t smem;          // dynamic shared memory per CTA
    size_t state_bytes;   // per-CTA candidate state
};

// Per-CTA candidate state layout (same in shared or global memory).
struct StateLayout {
    size_t pos, last, A, Fr, C, evkey_in, evkey_out, evcb, endT, endS, endL, dec, total;
};
StateLayout state_layout(int32_t NT, int32_t R, int32_t max_events, int32_t Rd);

// Host-side inputs of the variant-2 planner (super-graph in CSR form).
struct SuperGraphHost {
    int32_t n, R, NT;
    const int32_t* cons_ptr;   // [NT+1]
    const int2* cons_ent;      // (consumer, gate)
    const int32_t* in_ptr;     // [NT+1]
    const int2* in_ent;        // (input, gate)
    const int64_t* size;       // [NT]
    const double* cost;        // [NT]
    const uint8_t* nflag;      // [NT]
    const int32_t* U_ptr;      // [R+1]
    const int32_t* U_idx;
    const double* rtab;        // [R][2] (cost(t_r), swap transfer time)
    const int32_t* elig;       // [R] t_r
    // F-Trans variant regions (NEXT-4, reading F1); F = 0: none
    int32_t F;
    const int32_t* ngate;      // [n] gate of an original node: -1 or (R + region) << 2 | variant
    const int32_t* nvar;       // [F] variants per region
    const double* vcost;       // [4F] cost sum of (region, variant)
};

// Build the variant-2 plan and its static shared-memory image for a given P.
// Returns false if the graph does not fit (ids >= 65535, sizes beyond u32
// units, or shared memory).
bool plan2_build(const SuperGraphHost& sg, int P, int teams, bool gmem_static, bool gmem_af, bool delta_slots,
                 size_t smem_cap, Plan2* plan,
                 std::vector<char>* image, int row_groups = 1);
cudaError_t eval2_launch(const DevGraph& g, const Plan2& pl, const void* blob, void* ovf, void* afg, int grid,
                         int64_t K, const int32_t* perm, const uint8_t* dec, uint8_t* status,
                         int64_t* peak, double* lat, cudaStream_t stream, int32_t* argmax = nullptr);
cudaError_t eval2_occupancy(const Plan2& pl, int* blocks_per_sm);

// Kernel B (magis_evalb.cu): one candidate per two-CTA cluster, tier-2
// semantics; a plan built with row_groups = 2.  Shared-memory layout per CTA:
struct BLayout {
    int32_t L, S, S0;     // steps per scan chunk, chunks, chunks of CTA 0
    uint32_t Lm;          // ceil(2^32 / L)
    int32_t Sl;           // padded per-step delta slots (step st at st + st / L)
    int32_t nwm;          // u32 words of event-step marks
    uint32_t stage;       // staged cost-class bytes at offset 0 (0: none)
    uint32_t pos, D, marks, dec, end, total;
    uint32_t rec;         // resolved event records [evcap]: u64 key, f64 time, u32 producer
    int32_t evcap;
};
bool evalb_layout(const Plan2& pl, size_t smem_cap, BLayout* lay);
cudaError_t evalb_launch(const DevGraph& g, const Plan2& pl, const BLayout& lay, const void* blob, int clusters,
                         int64_t K, const int32_t* perm, const uint8_t* dec, uint8_t* status, int64_t* peak,
                         double* lat, void* evscratch, cudaStream_t stream);
size_t evalb_scratch_bytes(const Plan2& pl, int clusters);
int eval2_block(const Plan2& pl);      // threads per CTA

size_t hotspot_ws_per_cta(const DevGraph& g);
cudaError_t hotspot_launch(const DevGraph& g, int grid, void* ws, int64_t K, const int32_t* perm, const uint8_t* dec,
                           int32_t nsplit, uint8_t* status, int64_t* peak, uint8_t* hot, int64_t* heat,
                           double* score, cudaStream_t stream);

cudaError_t eval_configure(const DevGraph& g, int device, EvalConfig* cfg);
cudaError_t eval_launch(const DevGraph& g, const EvalConfig& cfg, void* gws, int64_t K,
                        const int32_t* perm, const uint8_t* dec, uint8_t* status,
                        int64_t* peak, double* lat, cudaStream_t stream);

int64_t pareto_workspace_size(int64_t n);
cudaError_t pareto_launch(int64_t n, const int64_t* peak, const double* lat,
                          const uint8_t* status, const int64_t* id, int64_t id_base,
                          int64_t cap, int64_t* front_id, int64_t* front_peak,
                          double* front_lat, int64_t* front_n, int64_t mem_limit,
                          double lat_limit, int64_t* best, void* ws, cudaStream_t stream);

// thread-local error reporting
int set_error(int code, const std::string& msg);
void clear_error();

}  // namespace magis

// The opaque graph handle.
struct magis_graph {
    int device = 0;
    magis::DevGraph dev{};
    magis::EvalConfig cfg{};
    void* blob = nullptr;          // device tables
    size_t blob_bytes = 0;
    void* gws = nullptr;           // global per-CTA workspace (variant 1)
    magis::Plan2 plan2{};          // variant 2 plan (also kernel B's tables, variant 3)
    magis::BLayout layb{};         // variant 3 (kernel B) shared-memory layout
    int clustersb = 0;             // variant 3: two-CTA clusters in the grid
    void* evb = nullptr;           // variant 3: event scratch
    void* blob2 = nullptr;         // variant 2 static shared-memory image
    size_t blob2_bytes = 0;
    void* ovf2 = nullptr;          // variant 2 event overflow scratch
    void* afg2 = nullptr;          // variant 2 per-CTA global step slots (gmem_af)
    magis::GenTables gen{};        // base-graph adjacency (device)
    void* gen_scratch = nullptr;   // candidate generator scratch (lazily allocated)
    size_t gen_bytes = 0;
    size_t gws_bytes = 0;
    int64_t n_edges = 0;
    int64_t n_super_edges = 0;
    std::vector<int32_t> idom;     // dominator tree of G (host copy)
    // host copies of the load-time tables (plans built later: GraphHash)
    std::vector<int32_t> h_pred_ptr, h_pred, h_topo, h_elig, h_Uptr, h_Uidx;
    std::vector<uint8_t> h_rflag;
    void* hs_ws = nullptr;         // hot-spot query workspace (lazily allocated)
    size_t hs_ws_bytes = 0;
    // host-buffer (end-to-end) path: lazily allocated staging
    cudaStream_t aux = nullptr;
    int64_t stage_K = 0;
    void* stage[2] = {nullptr, nullptr};
    cudaEvent_t ev_h2d[2] = {nullptr, nullptr};
    cudaEvent_t ev_done[2] = {nullptr, nullptr};
};

struct magis_base {
    const magis_graph* g = nullptr;
    void* mem = nullptr;
    magis::BaseDev dev{};
    double* endb_ws = nullptr;
    int grid = 0;
};
