/*
 * magis.h -- C ABI of the B200-native batched schedule evaluator for MAGIS
 * (Chen et al., "MAGIS: Memory Optimization via Coordinated Graph
 * Transformation and Scheduling for DNN", ASPLOS '24).
 *
 * Citations "P:a-b" are line ranges of the paper text; readings
 * "Pn" are listed in DESIGN.md §Readings.
 *
 * The library scores K candidate schedules of one computation graph at once.
 * A candidate is a topological order of the super-graph (original ops plus,
 * per eligible tensor, an optional re-materialised clone, Store and Load,
 * §5.2) and one decision per eligible tensor (0 keep,
 * 1 re-materialise, 2 swap).  Its score is the exact peak memory M_peak
 * and the modelled latency.
 *
 * All calls are thread-safe with respect to distinct graphs; a graph is
 * immutable after load and may be used from several streams (each call uses
 * graph-owned workspace, so concurrent calls on ONE graph must be serialised
 * by the caller on one stream).  Every entry point returns MAGIS_SUCCESS or a
 * negative error code; magis_last_error() gives a thread-local message.
 * There is no CPU fallback: without an sm_100 device every call that needs
 * one returns MAGIS_E_UNSUPPORTED.
 */
#ifndef MAGIS_H
#define MAGIS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#pragma GCC visibility push(default)   /* the library builds with -fvisibility=hidden */
#endif

#define MAGIS_ABI_VERSION 2

enum {
    MAGIS_SUCCESS = 0,
    MAGIS_E_INVAL = -1,        /* bad argument or malformed graph            */
    MAGIS_E_CYCLE = -2,        /* the graph is not a DAG          */
    MAGIS_E_NOMEM = -3,        /* host or device allocation failed            */
    MAGIS_E_CUDA = -4,         /* a CUDA runtime call failed                  */
    MAGIS_E_UNSUPPORTED = -5,  /* no sm_100 device / graph too large          */
    MAGIS_E_CAPACITY = -6      /* output capacity too small (see pareto)      */
};

/* Candidate status bits (per-candidate problems are data, not errors;
 * reading P12).  Any nonzero status => peak = -1, latency = +inf. */
enum {
    MAGIS_ST_NOT_PERM = 1,     /* perm is not a permutation of [0, n_total)  */
    MAGIS_ST_EDGE = 2,         /* a dependency of the transformed graph is violated
                                  (only reported when bits 0 and 2 are clear) */
    MAGIS_ST_BAD_DEC = 4       /* a decision is not 0/1/2, or 1 on a tensor
                                  without inputs (re-mat needs A's inputs) */
};

/*
 * Graph description (host memory; copied by magis_graph_load, the caller
 * keeps ownership).  Table 1 / §2.1:
 *   n_nodes       |V|; node ids 0..n_nodes-1.  Every op has one output tensor
 *                 (reading P4); inputs/labels/weights are ordinary zero-cost
 *                 nodes (reading P3).
 *   out_bytes     [n_nodes] size(v) = |v| in bytes, >= 0 (int64: sums exceed 2^31).
 *   cost          [n_nodes] cost(v) in seconds, finite, >= 0 (the operator
 *                 performance cache of P:1780-1783).
 *   is_output     [n_nodes] nonzero for outs(G) (live to the end, reading P2).
 *   n_edges, edge_src, edge_dst
 *                 E subset of V x V; (u, v) means v reads u's output.  E is a
 *                 set: duplicates are merged (reading P17); self-loops rejected.
 *   n_eligible    R, tensors the re-mat / swap rules may touch (the hot-spot
 *                 filter of P:1619-1625).
 *   eligible_tensor [R] t_r: not a graph output, no duplicates.
 *   late_user_ptr [R+1], late_user_idx: U_r, non-empty, U_r subset of
 *                 cons(t_r), no duplicates: the users served by the clone /
 *                 the Load (reading P6; Fig. 8 "one user B" generalised).
 *   swap_bytes_per_s > 0, swap_latency_s >= 0: a Store / Load of t takes
 *                 swap_latency_s + |t| / swap_bytes_per_s on its copy queue
 *                 (reading P7).  Ignored when R == 0.
 *
 * Super-graph ids: original v -> v; for eligible r: clone_r = n+3r,
 * store_r = n+3r+1, load_r = n+3r+2; n_total = n + 3R.
 */
typedef struct magis_graph_desc {
    int32_t n_nodes;
    const int64_t* out_bytes;
    const double* cost;
    const uint8_t* is_output;
    int64_t n_edges;
    const int32_t* edge_src;
    const int32_t* edge_dst;
    int32_t n_eligible;
    const int32_t* eligible_tensor;
    const int64_t* late_user_ptr;
    const int32_t* late_user_idx;
    double swap_bytes_per_s;
    double swap_latency_s;
} magis_graph_desc;

typedef struct magis_graph magis_graph;   /* opaque, library-owned */

typedef struct magis_graph_info {
    int32_t n_nodes;           /* n */
    int32_t n_eligible;        /* R */
    int32_t n_total;           /* n + 3R: length of one candidate perm */
    int64_t n_edges;           /* deduplicated |E| */
    int64_t n_super_edges;     /* edges of the super-graph (all gates) */
    int32_t device;            /* CUDA device ordinal */
    int32_t variant;           /* eval kernel: 0/1 = per-candidate state in smem/global, 2 = packed streams */
    int32_t grid;              /* persistent CTAs per eval launch */
    int32_t block;             /* threads per CTA */
    int64_t smem_bytes;        /* dynamic shared memory per CTA */
    int64_t table_bytes;       /* device bytes of the graph tables */
    double base_cost;          /* sum of cost(v) over original nodes */
    int32_t pack;              /* candidates scored together per CTA step (variant 2), else 1 */
    int32_t n_regions;         /* F-Trans variant regions F (decision row = R + F bytes) */
} magis_graph_info;

/*
 * Validate and upload a graph.  Builds, on `device`, the consumer and input
 * CSRs of the super-graph with per-edge activation gates, the node tables and
 * the swap-event tables, plus the eval workspace (Table 1
 * P:356-369).  When the evaluation plan reads its graph image from global
 * memory (large graphs), the call raises the device's persisting-L2 limit
 * (cudaLimitPersistingL2CacheSize) to cover the image, and every evaluation
 * launch carries an L2 access-policy window over it; no stream attribute is
 * changed.
 * Errors: MAGIS_E_INVAL (null pointer, n_nodes < 1, id out of range, self
 * loop, negative size or cost, non-finite cost, output marked eligible,
 * duplicate eligible tensor, empty U_r, U_r not a subset of cons(t_r),
 * duplicate in U_r, swap_bytes_per_s <= 0 with R > 0), MAGIS_E_CYCLE,
 * MAGIS_E_NOMEM, MAGIS_E_CUDA, MAGIS_E_UNSUPPORTED (device is not sm_100,
 * or n_total > 2^30).  On error *out is set to NULL.
 */
int magis_graph_load(const magis_graph_desc* desc, int device, magis_graph** out);

/*
 * F-Trans variant regions (§4.2-4.3, §5.1
 * P:1295-1326; reading F1 in DESIGN.md).  An F-Trans f = (S, D, n) replaces
 * the sub-graph S by n parts plus slices and merges (Fig. 5).  A region holds
 * several such versions of one S side by side in the graph (variant 0 = S
 * unsplit, variant j = one factor n_j): the caller materialises them as
 * ordinary nodes and labels each with (region, variant).  A candidate picks
 * one variant per region; a node of region i exists iff the candidate's
 * choice for i equals its variant, an edge exists iff both ends exist, and
 * nodes that do not exist are no-ops wherever the schedule puts them (they
 * hold no memory and cost no time).  The decision row of a candidate becomes
 * [R eligible decisions | F region variants] (uint8, R + F bytes).
 *   n_regions     F >= 0.
 *   n_variants    [F] 1..4.
 *   node_region   [n_nodes] region of the node, or -1 (present in every variant).
 *   node_variant  [n_nodes] variant of that region (< n_variants[region]).
 * Constraints (MAGIS_E_INVAL otherwise): an edge joins nodes of at most one
 * (region, variant) (regions do not touch; a consumer outside a region reads
 * every variant's version of a region output); eligible tensors, their
 * inputs and their late users are outside regions (the Fig. 8 rules act on
 * the ops present in every variant).  A variant index >= n_variants in a
 * candidate is MAGIS_ST_BAD_DEC.  Graphs with regions are scored by the
 * general gated kernel (variant 0/1); magis_generate_candidates,
 * magis_base_create, magis_hotspots and magis_ghash_create return
 * MAGIS_E_UNSUPPORTED on them.  magis_graph_load(d, dev, out) is
 * magis_graph_load_regions(d, NULL, dev, out).
 */
typedef struct magis_region_desc {
    int32_t n_regions;
    const int32_t* n_variants;
    const int32_t* node_region;
    const uint8_t* node_variant;
} magis_region_desc;

int magis_graph_load_regions(const magis_graph_desc* desc, const magis_region_desc* regions, int device,
                             magis_graph** out);

/* Release a graph (NULL is a no-op).  Synchronises the graph's device. */
int magis_graph_free(magis_graph* g);

int magis_graph_info_get(const magis_graph* g, magis_graph_info* info);

/*
 * Score K candidates (the hot path):
 *   perm -> inverse permutation -> validity of every active super-graph edge
 *   -> last-use step per tensor -> alloc/free events -> prefix scan -> max,
 *   plus the latency model (sum of compute costs; with swaps, the three
 *   in-order queues compute / D2H / H2D of reading P7).
 * d_perm     [K x n_total] int32, row-major, device memory: step -> super id.
 * d_dec      [K x (R + F)] uint8 device memory (F = n_regions, usually 0), or
 *            NULL when R + F == 0.
 * d_status   [K] uint8  out: MAGIS_ST_* bits.
 * d_peak     [K] int64  out: M_peak in bytes (-1 if status != 0).
 * d_latency  [K] double out: seconds (+inf if status != 0).
 * cuda_stream: cudaStream_t (NULL = legacy default stream).
 * Asynchronous on the stream, no allocation, no host synchronisation.
 * Errors: MAGIS_E_INVAL (K < 0, null pointer, dec NULL with R > 0),
 * MAGIS_E_CUDA (launch failure).
 */
int magis_eval_schedules(const magis_graph* g, int64_t K, const int32_t* d_perm,
                         const uint8_t* d_dec, uint8_t* d_status, int64_t* d_peak,
                         double* d_latency, void* cuda_stream);

/*
 * magis_eval_schedules plus the optional output of step a7:
 * d_argmax [K] int32 out: the first step of the candidate's permutation
 * (0-based index into d_perm's row, inactive optional nodes included) whose
 * allocation brings the memory M_i to M_peak -- the first step of the
 * memory hot-spot; -1 if status != 0.  It is always the step of
 * an active node.  Same execution as magis_eval_schedules (one launch, the
 * argmax is a third field of the scan's (sum, max-prefix) monoid).
 * Errors: as magis_eval_schedules, plus MAGIS_E_UNSUPPORTED when the graph
 * is evaluated by the simple kernel (n_total + |U| >= 65,535).
 */
int magis_eval_schedules_argmax(const magis_graph* g, int64_t K, const int32_t* d_perm, const uint8_t* d_dec,
                                uint8_t* d_status, int64_t* d_peak, double* d_latency, int32_t* d_argmax,
                                void* cuda_stream);

/*
 * The same evaluation with HOST buffers (end-to-end path): the candidates are
 * copied host->device in chunks on `cuda_stream` and a second graph-owned
 * stream, overlapped with evaluation, and the results copied back.  Pinned
 * host memory gives overlap; pageable memory works but serialises.  Blocks
 * until the results are in h_status / h_peak / h_latency.
 * Errors as magis_eval_schedules.
 */
int magis_eval_schedules_host(magis_graph* g, int64_t K, const int32_t* h_perm,
                              const uint8_t* h_dec, uint8_t* h_status, int64_t* h_peak,
                              double* h_latency, void* cuda_stream);

/*
 * As magis_eval_schedules_host with the schedules in the compact wire format:
 * h_perm [K x n_total] uint16 host memory (n_total <= 65535).  Half the
 * host->device bytes; the library widens each chunk on the device before
 * evaluating it.  Errors as magis_eval_schedules_host, plus
 * MAGIS_E_UNSUPPORTED if n_total > 65535.
 */
int magis_eval_schedules_host_u16(magis_graph* g, int64_t K, const uint16_t* h_perm,
                                  const uint8_t* h_dec, uint8_t* h_status, int64_t* h_peak,
                                  double* h_latency, void* cuda_stream);

/*
 * As magis_eval_schedules_host with the schedules in the delta8 wire format
 * (n_total <= 65535): per step one signed byte, the difference between this
 * step's node id and the previous step's (a row starts from 0); the byte -128
 * means "the next value of this row's exception list", an absolute uint16
 * id.  h_delta [K x n_total] int8; h_exc_ptr [K + 1] int32 (row k's
 * exceptions are h_exc[h_exc_ptr[k] .. h_exc_ptr[k+1]), nondecreasing);
 * h_exc uint16 (may be NULL if there are none).  Random topological orders
 * of DNN graphs move by small id steps, so this is ~1.1 bytes per step
 * instead of 2 (u16) or 4 (int32) across PCIe; the device decodes each
 * chunk (a segmented warp scan) before evaluating it.  Ids >= n_total (e.g. a
 * clamped out-of-range id) give MAGIS_ST_NOT_PERM as usual.
 * Errors as magis_eval_schedules_host_u16, plus MAGIS_E_INVAL for
 * decreasing offsets.
 */
int magis_eval_schedules_host_delta8(magis_graph* g, int64_t K, const int8_t* h_delta, const int32_t* h_exc_ptr,
                                     const uint16_t* h_exc, const uint8_t* h_dec, uint8_t* h_status,
                                     int64_t* h_peak, double* h_latency, void* cuda_stream);

/*
 * As magis_eval_schedules_host_delta8 with one nibble per step (the delta4
 * wire format, n_total <= 65535): row k is h_code[k * ceil(n_total / 2) ..],
 * step j in byte j / 2, the low nibble first; nibble c = 0 means "the next
 * value of this row's exception list" (an absolute uint16 id), any other c a
 * difference of c - 8 (-7 .. +7) to the previous step's id (the row starts
 * from 0); the pad nibble of an odd-length row is ignored.  ~0.5 byte per step
 * plus 2 bytes per escaped step across PCIe (C2: 87% of steps move by at most
 * 7 ids).  Errors as magis_eval_schedules_host_delta8.
 */
int magis_eval_schedules_host_delta4(magis_graph* g, int64_t K, const uint8_t* h_code, const int32_t* h_exc_ptr,
                                     const uint16_t* h_exc, const uint8_t* h_dec, uint8_t* h_status,
                                     int64_t* h_peak, double* h_latency, void* cuda_stream);

/*
 * Seeded candidate generation on the device.  Candidate k
 * (global id id0 + i) depends only on (spec->seed, k), so ranks generate
 * their shards independently.  The recipe stands in for MAGIS's rule
 * application + re-ordering (§5.2, Alg. 2; DESIGN.md
 * §5): per eligible tensor a decision (re-mat with probability
 * p_remat/10000 if the tensor has inputs, else swap with p_swap/10000);
 * pct_random % random-priority Kahn orders (the ready node of smallest
 * (16-bit priority, id) first), pct_local % local moves (a window of <= wmax
 * natural-order steps re-ordered by the same keyed Kahn), the rest a random
 * order with one random transposition (may be invalid); Stores right after
 * their producer, Loads / clones 0..slack steps before the first
 * late user, inactive optional nodes last.  Byte-identical to the C generator
 * magis_inputs/csrc/candgen.c (the test side).
 * d_perm [K x n_total] int32, d_dec [K x max(R,1)] uint8 (R = 0: one zero pad
 * byte per row): device memory, caller-owned.
 * Asynchronous on the stream.  The first call allocates graph-owned scratch
 * (grown when a later call needs more), so calls on one graph must not overlap
 * in time on different streams.
 * Errors: MAGIS_E_INVAL (K < 0, null pointer, bad spec), MAGIS_E_NOMEM / MAGIS_E_CUDA.
 */
typedef struct magis_gen_spec {
    uint64_t seed;
    int32_t pct_random;   /* % random topological orders                       */
    int32_t pct_local;    /* % local moves; the rest: one random transposition */
    int32_t p_remat;      /* per 10000 eligible tensors                         */
    int32_t p_swap;       /* per 10000 eligible tensors                         */
    int32_t wmax;         /* max local-move window (>= 2)                       */
    int32_t slack;        /* Load / clone placement slack in steps (>= 0)       */
} magis_gen_spec;

int magis_generate_candidates(magis_graph* g, const magis_gen_spec* spec, uint64_t id0, int64_t K,
                              int32_t* d_perm, uint8_t* d_dec, void* cuda_stream);

/*
 * Windowed delta evaluation of local moves (the
 * incremental-scheduling idea of Alg. 2, applied to scoring).
 * A base schedule (perm + decisions) is evaluated once into a device-resident
 * profile; a local-move candidate k re-orders the base steps
 * [wstart[k], wstart[k] + wlen[k]) and keeps the base decisions.  Outside the
 * window the memory curve cannot change, so each candidate costs
 * O(window + incident edges + swap events) and the result equals the full
 * evaluation of the expanded schedule (tested bit-exactly on peak/status,
 * 1e-9 on latency).
 *
 * magis_base_create: d_perm [n_total] / d_dec [R] device memory (may be
 *   reused by the caller after the call's stream work completes); the base is
 *   evaluated asynchronously on the stream.  *out is library-owned.
 * magis_base_info: synchronises and returns the base's status / peak / latency.
 * magis_eval_windows: d_wstart [K], d_wlen [K] (1..wmax), d_wperm [K x wmax]
 *   int32 (the window's super-graph node ids in their new order; entry j of
 *   row k for j < wlen[k]), device memory; wmax <= 64.  Outputs as
 *   magis_eval_schedules.  A window that is not a permutation of the base
 *   window's nodes gets MAGIS_ST_NOT_PERM; a violated dependency inside the
 *   window MAGIS_ST_EDGE; an invalid base passes its status on.
 *   Asynchronous on the stream.  Errors: MAGIS_E_INVAL, MAGIS_E_UNSUPPORTED
 *   (wmax > 64), MAGIS_E_NOMEM, MAGIS_E_CUDA.
 */
typedef struct magis_base magis_base;   /* opaque, library-owned */

int magis_base_create(magis_graph* g, const int32_t* d_perm, const uint8_t* d_dec, magis_base** out,
                      void* cuda_stream);
int magis_base_info(const magis_base* b, int* status, int64_t* peak, double* latency);
int magis_base_free(magis_base* b);
int magis_eval_windows(const magis_base* b, int64_t K, const int32_t* d_wstart, const int32_t* d_wlen,
                       const int32_t* d_wperm, int32_t wmax, uint8_t* d_status, int64_t* d_peak,
                       double* d_latency, void* cuda_stream);

/*
 * Memory hot-spots and F-Trans heat / score of K candidate schedules
 * (Eq. 3-4), for the schedules
 * the search selects (one CTA per candidate; not the batch hot loop).
 * H = the tensors live at some step where M_i = M_peak; over the original
 * graph a live clone or Load of t_r stands for t_r and a Store does not count
 * (reading H1).  T = the dominator tree of G, sources under a
 * virtual root (built by magis_graph_load; see magis_graph_idom).
 *   heat(v)  = sum of |w| over w in H and T.des(v)                      (Eq. 3)
 *   score(v) = (1 - 1/nsplit) heat(v) - sum of |u| over the inputs of
 *              T.des(v) not in H                                         (Eq. 4)
 * d_perm [K x n_total] int32, d_dec [K x R] u8 (may be NULL if R == 0):
 *             device memory, as magis_eval_schedules.
 * nsplit      n of Eq. 4 (>= 1; the paper uses 2).
 * d_status [K] u8, d_peak [K] int64 out: as magis_eval_schedules.
 * d_hot [K x n_nodes] u8 out: 1 iff original tensor v is a hot-spot.
 * d_heat [K x n_nodes] int64 out (bytes) or NULL; d_score [K x n_nodes] f64
 *             out or NULL.  Invalid candidates: status != 0, peak -1, rows 0.
 * Asynchronous on the stream; the workspace is library-owned (allocated on
 * first use, freed with the graph).
 * Errors: MAGIS_E_INVAL, MAGIS_E_NOMEM, MAGIS_E_CUDA.
 */
int magis_hotspots(magis_graph* g, int64_t K, const int32_t* d_perm, const uint8_t* d_dec, int32_t nsplit,
                   uint8_t* d_status, int64_t* d_peak, uint8_t* d_hot, int64_t* d_heat, double* d_score,
                   void* cuda_stream);

/*
 * Immediate dominators of the original graph: idom[v] = the
 * nearest strict dominator of v, or -1 if only the sources' virtual root
 * dominates it.  idom: host array [n_nodes], caller-owned.
 * Errors: MAGIS_E_INVAL.
 */
int magis_graph_idom(const magis_graph* g, int32_t* idom);

/*
 * Pareto front of (peak, latency) over valid points,
 * plus the BetterThan-best point of Alg. 3 in both optimisation
 * modes.  a dominates b iff a.peak <= b.peak, a.lat <= b.lat and
 * one is strict; among exact duplicates the smallest id survives (reading P10).
 * Used for the per-rank front and again on the all-gathered fronts; it is
 * collective-agnostic (the caller all-gathers, e.g. via NCCL).
 * n           number of input points (>= 0).
 * d_peak, d_lat [n] device memory.
 * d_status    [n] device memory (status != 0 => ignored), or NULL (all valid).
 * d_id        [n] int64 candidate ids, or NULL => id = id_base + index.
 *             Points with a negative id are ignored (padding of gathered fronts).
 * cap         capacity of the front outputs (>= 0).
 * d_front_id, d_front_peak, d_front_lat [cap] out, ascending peak
 *             (strictly decreasing latency); the first min(front, cap)
 *             entries are the front, entries [front, cap) are padding
 *             (id -1, peak -1, latency +inf), so a padded front can be
 *             all-gathered and fed back into this call as is.
 * d_front_n   [1] out: the true front size (may exceed cap: the caller
 *             checks; the call itself stays asynchronous).
 * mem_limit   >= 0: d_best[0] = argmin over valid points of
 *             (max(peak, M), lat, peak, id) (Alg. 3 mode 1, reading P10b); -1 if
 *             mem_limit < 0 or no valid point.
 * lat_limit   >= 0: d_best[1] = argmin of (max(lat, L), peak, lat, id) (mode 2);
 *             -1 if lat_limit < 0 or no valid point.  d_best may be NULL.
 * d_workspace / workspace_bytes: caller-owned device scratch of at least
 *             magis_pareto_workspace_size(n) bytes.
 * Asynchronous on the stream; no allocation; no host synchronisation.
 * Errors: MAGIS_E_INVAL, MAGIS_E_CAPACITY (workspace too small), MAGIS_E_CUDA.
 */
int64_t magis_pareto_workspace_size(int64_t n);

int magis_pareto_merge(int64_t n, const int64_t* d_peak, const double* d_lat,
                       const uint8_t* d_status, const int64_t* d_id, int64_t id_base,
                       int64_t cap, int64_t* d_front_id, int64_t* d_front_peak,
                       double* d_front_lat, int64_t* d_front_n, int64_t mem_limit,
                       double lat_limit, int64_t* d_best, void* d_workspace,
                       int64_t workspace_bytes, void* cuda_stream);

/*
 * Batched GraphHash (Alg. 3 lines 3-6, and
 * the Weisfeiler-Lehman test of P:1776-1778; readings G1-G4 in DESIGN.md).
 * The graph of candidate k is its transformed graph (the Fig. 8 rules of
 * dec[k] applied to G; the schedule does not enter, G4).  For
 * every active node v, in topological order,
 *     x_v = hash( hash(label_v) (+) x_{u_1} (+) ... (+) x_{u_d} )      (line 5)
 * where u_1..u_d = pre(v) sorted by ascending x (G2) and (+) concatenates
 * 64-bit words; GraphHash = hash( sum_v x_v mod 2^64 ) (line 6).
 * hash(w_0..w_{m-1}) = fold h = mix64(h ^ w_i) from h = 0x9E3779B97F4A7C15 *
 * (m + 1), mix64 = the SplitMix64 output function (G1).  A clone carries
 * label(t_r); Store / Load carry 0x45524F5453 / 0x44414F4C (G3).
 *
 * magis_ghash_create: h_label [n_nodes] uint64 host memory (copied; the
 *   caller's op signature, e.g. type + attributes + shape), builds the node
 *   order, value slots and tables on the graph's device (synchronous).
 *   *out is library-owned and tied to g (free it before g).
 *   Errors: MAGIS_E_INVAL, MAGIS_E_NOMEM, MAGIS_E_CUDA.
 * magis_graph_hash: d_dec [K x R] uint8 device memory (NULL if R == 0);
 *   d_status [K] uint8 out (MAGIS_ST_BAD_DEC or 0); d_hash [K] uint64 out
 *   (0 if status != 0).  Asynchronous on the stream, no allocation; the
 *   scratch belongs to *h, so calls on one h are serialised by the caller.
 *   Errors: MAGIS_E_INVAL (K < 0, null pointer), MAGIS_E_CUDA.
 * magis_ghash_info: shared / global value slots per warp, the number of
 *   values kept in global slots, persistent grid (any pointer may be NULL).
 */
typedef struct magis_ghash magis_ghash;   /* opaque, library-owned */

int magis_ghash_create(const magis_graph* g, const uint64_t* h_label, magis_ghash** out);
int magis_ghash_free(magis_ghash* h);
int magis_graph_hash(magis_ghash* h, int64_t K, const uint8_t* d_dec, uint8_t* d_status, uint64_t* d_hash,
                     void* cuda_stream);
int magis_ghash_info(const magis_ghash* h, int32_t* shared_slots, int32_t* global_slots, int64_t* global_nodes,
                     int32_t* grid);

/*
 * The duplicate filter of Alg. 3 lines 10-12 over a batch: a
 * device hash set X of graph hashes.  magis_hashset_filter processes the
 * batch as if in candidate-id order: d_new[k] = 1 iff d_status[k] == 0 (or
 * d_status is NULL), d_hash[k] is not in X and no smaller k' of the batch
 * with status 0 has the same hash; then every valid hash joins X.  All hash
 * values (0 included) are ordinary keys.
 * capacity: keys the set can hold (rounded up to a power of two, <= 2^40).
 *   Open addressing: keep the load below ~0.7.  If the set is full an insert
 *   is dropped, counted in n_overflow, and that candidate is reported new
 *   (never a false duplicate).
 * d_hash [K] uint64, d_status [K] uint8 or NULL, d_new [K] uint8 out: device
 *   memory.  Asynchronous on the stream; calls on one set are serialised by
 *   the caller (one stream).  K < 2^40; at most 2^24 - 2 filter calls between
 *   clears (MAGIS_E_CAPACITY after that).
 * magis_hashset_stats synchronises and returns |X| and dropped inserts.
 * Errors: MAGIS_E_INVAL, MAGIS_E_NOMEM, MAGIS_E_CUDA, MAGIS_E_UNSUPPORTED
 *   (no sm_100 device), MAGIS_E_CAPACITY.
 */
typedef struct magis_hashset magis_hashset;   /* opaque, library-owned */

int magis_hashset_create(int device, int64_t capacity, magis_hashset** out);
int magis_hashset_free(magis_hashset* s);
int magis_hashset_clear(magis_hashset* s, void* cuda_stream);
int magis_hashset_filter(magis_hashset* s, int64_t K, const uint64_t* d_hash, const uint8_t* d_status,
                         uint8_t* d_new, void* cuda_stream);
int magis_hashset_stats(const magis_hashset* s, int64_t* n_keys, int64_t* n_overflow);

/* Thread-local message for the last nonzero return on this thread. */
const char* magis_last_error(void);

/* ABI version (MAGIS_ABI_VERSION) and whether an sm_100 device is visible. */
int magis_abi_version(void);
int magis_device_supported(int device);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif

#ifdef __cplusplus
}
#endif

#endif /* MAGIS_H */
