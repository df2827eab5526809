// magis_graph.cu -- graph loader and ABI glue.
//
// Validates the graph of Table 1 / §2.1, deduplicates E (a set,
// reading P17), checks acyclicity (a schedule must satisfy every dependency,
// P:402-405), and builds the super-graph the re-materialisation and swapping
// rules can produce (§5.2, Fig. 8): per eligible tensor t_r an
// optional clone (reads pre(t_r), serves U_r), Store (reads t_r) and Load
// (reads the Store, serves U_r).  Every super-graph edge carries an
// activation gate so that one static CSR serves every decision vector.
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <vector>

#include "magis_internal.h"

namespace magis {

static thread_local std::string g_err;

int set_error(int code, const std::string& msg) {
    g_err = msg;
    return code;
}
void clear_error() { g_err.clear(); }

}  // namespace magis

using namespace magis;

extern "C" const char* magis_last_error(void) { return g_err.c_str(); }
extern "C" int magis_abi_version(void) { return MAGIS_ABI_VERSION; }

extern "C" int magis_device_supported(int device) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    if (device < 0 || device >= n) return 0;
    cudaDeviceProp p;
    if (cudaGetDeviceProperties(&p, device) != cudaSuccess) return 0;
    return p.major == 10 ? 1 : 0;
}

namespace {

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) {
        cudaGetDevice(&prev);
        cudaSetDevice(d);
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

#define CK(call)                                                                   \
    do {                                                                           \
        cudaError_t _e = (call);                                                   \
        if (_e != cudaSuccess) {                                                   \
            cudaGetLastError();                                                    \
            return set_error(MAGIS_E_CUDA, std::string(#call ": ") + cudaGetErrorString(_e)); \
        }                                                                          \
    } while (0)

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

cudaError_t dispatch_eval(const magis_graph* g, int64_t K, const int32_t* perm, const uint8_t* dec,
                          uint8_t* st, int64_t* pk, double* lt, cudaStream_t s) {
    if (g->cfg.variant == 2) {
        cudaError_t e = eval2_launch(g->dev, g->plan2, g->blob2, g->ovf2, g->afg2, g->cfg.grid, K, perm, dec, st, pk,
                                     lt, s);
        if (e == cudaSuccess && g->plan2.prof) {
            // diagnostics only: per-phase cycles summed over CTAs (thread 0 / latency lane 0)
            unsigned long long h[16];
            cudaStreamSynchronize(s);
            cudaMemcpy(h, (char*)g->ovf2 + g->plan2.prof_off, 128, cudaMemcpyDeviceToHost);
            cudaMemset((char*)g->ovf2 + g->plan2.prof_off, 0, 128);
            unsigned long long tot = 0;
            for (int i = 1; i < 10; i++) tot += h[i];
            std::fprintf(stderr, "[magis-prof] main:");
            for (int i = 1; i < 10; i++) std::fprintf(stderr, " p%d=%.1f%%", i, tot ? 100.0 * h[i] / tot : 0.0);
            std::fprintf(stderr,
                         " | latency warp: wait=%llu fold=%llu resolve=%llu walk=%llu rest=%llu arrive=%llu"
                         " (main total %llu)\n",
                         h[14], h[10], h[11], h[12], h[15], h[13], tot);
        }
        return e;
    }
    if (g->cfg.variant == 3)
        return evalb_launch(g->dev, g->plan2, g->layb, g->blob2, g->clustersb, K, perm, dec, st, pk, lt, g->evb, s);
    return eval_launch(g->dev, g->cfg, g->gws, K, perm, dec, st, pk, lt, s);
}

}  // namespace

extern "C" int magis_graph_load(const magis_graph_desc* d, int device, magis_graph** out) {
    return magis_graph_load_regions(d, nullptr, device, out);
}

extern "C" int magis_graph_load_regions(const magis_graph_desc* d, const magis_region_desc* rd, int device,
                                        magis_graph** out) {
    clear_error();
    if (!out) return set_error(MAGIS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (!d) return set_error(MAGIS_E_INVAL, "desc is NULL");
    const int32_t n = d->n_nodes;
    const int32_t R = d->n_eligible;
    if (n < 1) return set_error(MAGIS_E_INVAL, "n_nodes < 1");
    if (R < 0) return set_error(MAGIS_E_INVAL, "n_eligible < 0");
    if (d->n_edges < 0) return set_error(MAGIS_E_INVAL, "n_edges < 0");
    if (!d->out_bytes || !d->cost || !d->is_output)
        return set_error(MAGIS_E_INVAL, "null node array");
    // --- F-Trans variant regions (NEXT-4, reading F1) -------------------------
    const int32_t F = rd ? rd->n_regions : 0;
    if (F < 0) return set_error(MAGIS_E_INVAL, "n_regions < 0");
    if (F > 0 && (!rd->n_variants || !rd->node_region || !rd->node_variant))
        return set_error(MAGIS_E_INVAL, "null region array");
    if ((int64_t)R + F > (1 << 23)) return set_error(MAGIS_E_UNSUPPORTED, "n_eligible + n_regions > 2^23");
    std::vector<int32_t> nreg(n, -1);         // gate of an original node: -1 or (R + region) << 2 | variant
    for (int32_t i = 0; i < F; i++)
        if (rd->n_variants[i] < 1 || rd->n_variants[i] > 4)
            return set_error(MAGIS_E_INVAL, "n_variants must be in 1..4 (region " + std::to_string(i) + ")");
    if (F > 0)
        for (int32_t v = 0; v < n; v++) {
            const int32_t ri = rd->node_region[v];
            if (ri < -1 || ri >= F) return set_error(MAGIS_E_INVAL, "node_region out of range at node " + std::to_string(v));
            if (ri >= 0) {
                if (rd->node_variant[v] >= rd->n_variants[ri])
                    return set_error(MAGIS_E_INVAL, "node_variant out of range at node " + std::to_string(v));
                nreg[v] = ((R + ri) << 2) | rd->node_variant[v];
            }
        }
    if (d->n_edges > 0 && (!d->edge_src || !d->edge_dst))
        return set_error(MAGIS_E_INVAL, "null edge array");
    if (R > 0 && (!d->eligible_tensor || !d->late_user_ptr || !d->late_user_idx))
        return set_error(MAGIS_E_INVAL, "null eligible array");
    if ((int64_t)n + 3 * (int64_t)R > (1 << 30))
        return set_error(MAGIS_E_UNSUPPORTED, "n_total > 2^30");
    if (R > (1 << 23)) return set_error(MAGIS_E_UNSUPPORTED, "n_eligible > 2^23");
    for (int32_t v = 0; v < n; v++) {
        if (d->out_bytes[v] < 0) return set_error(MAGIS_E_INVAL, "negative out_bytes at node " + std::to_string(v));
        if (!(d->cost[v] >= 0.0) || !std::isfinite(d->cost[v]))
            return set_error(MAGIS_E_INVAL, "negative or non-finite cost at node " + std::to_string(v));
    }
    if (R > 0 && !(d->swap_bytes_per_s > 0.0 && std::isfinite(d->swap_bytes_per_s)))
        return set_error(MAGIS_E_INVAL, "swap_bytes_per_s must be > 0");
    if (R > 0 && !(d->swap_latency_s >= 0.0 && std::isfinite(d->swap_latency_s)))
        return set_error(MAGIS_E_INVAL, "swap_latency_s must be >= 0");

    // --- E as a set (reading P17) ------------------------------------------
    std::vector<uint64_t> keys;
    keys.reserve((size_t)d->n_edges);
    for (int64_t e = 0; e < d->n_edges; e++) {
        int32_t u = d->edge_src[e], v = d->edge_dst[e];
        if (u < 0 || u >= n || v < 0 || v >= n)
            return set_error(MAGIS_E_INVAL, "edge id out of range at edge " + std::to_string(e));
        if (u == v) return set_error(MAGIS_E_INVAL, "self-loop at node " + std::to_string(u));
        if (nreg[u] >= 0 && nreg[v] >= 0 && nreg[u] != nreg[v])
            return set_error(MAGIS_E_INVAL, "edge between different F-Trans variants at edge " + std::to_string(e));
        keys.push_back(((uint64_t)(uint32_t)u << 32) | (uint32_t)v);
    }
    std::sort(keys.begin(), keys.end());
    keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
    const int64_t E = (int64_t)keys.size();
    std::vector<int32_t> succ_ptr(n + 1, 0), succ(E), pred_ptr(n + 1, 0), pred(E);
    for (auto k : keys) { succ_ptr[(k >> 32) + 1]++; pred_ptr[(uint32_t)k + 1]++; }
    for (int32_t v = 0; v < n; v++) { succ_ptr[v + 1] += succ_ptr[v]; pred_ptr[v + 1] += pred_ptr[v]; }
    {
        std::vector<int32_t> fs(succ_ptr.begin(), succ_ptr.end() - 1), fp(pred_ptr.begin(), pred_ptr.end() - 1);
        for (auto k : keys) {
            int32_t u = (int32_t)(k >> 32), v = (int32_t)(uint32_t)k;
            succ[fs[u]++] = v;
            pred[fp[v]++] = u;
        }
    }
    // --- acyclicity --------------------------------------------
    std::vector<int32_t> topo;
    topo.reserve(n);
    {
        std::vector<int32_t> indeg(n), stack;
        for (int32_t v = 0; v < n; v++) {
            indeg[v] = pred_ptr[v + 1] - pred_ptr[v];
            if (!indeg[v]) stack.push_back(v);
        }
        while (!stack.empty()) {
            int32_t u = stack.back();
            stack.pop_back();
            topo.push_back(u);
            for (int32_t e = succ_ptr[u]; e < succ_ptr[u + 1]; e++)
                if (--indeg[succ[e]] == 0) stack.push_back(succ[e]);
        }
        if ((int32_t)topo.size() != n) return set_error(MAGIS_E_CYCLE, "the graph has a cycle");
    }
    // --- dominator tree T(G) (for NEXT-3 heat / score) ----------
    // Sources hang off a virtual root (-1).  On a DAG in topological order the
    // immediate dominator of v is the nearest common dominator-tree ancestor
    // of its predecessors; tin / tout number the tree in preorder, so the
    // descendants of v are the preorder range [tin(v), tout(v)).
    std::vector<int32_t> idom(n, -1), dtin(n), dtout(n);
    {
        std::vector<int32_t> ti(n);
        for (int32_t i = 0; i < n; i++) ti[topo[i]] = i;
        for (int32_t v : topo) {
            int32_t cur = -2;                       // -2: no predecessor seen yet
            for (int32_t e = pred_ptr[v]; e < pred_ptr[v + 1]; e++) {
                int32_t a = pred[e];
                if (cur == -2) { cur = a; continue; }
                int32_t b = cur;
                while (a != b && a >= 0 && b >= 0) {
                    if (ti[a] > ti[b]) a = idom[a]; else b = idom[b];
                }
                cur = (a == b) ? a : -1;
            }
            idom[v] = cur == -2 ? -1 : cur;
        }
        std::vector<int32_t> cptr(n + 2, 0), cidx(n);
        for (int32_t v = 0; v < n; v++) cptr[idom[v] + 2]++;
        for (int32_t i = 0; i <= n; i++) cptr[i + 1] += cptr[i];
        {
            std::vector<int32_t> fill(cptr.begin(), cptr.end() - 1);
            for (int32_t v = 0; v < n; v++) cidx[fill[idom[v] + 1]++] = v;
        }
        // iterative preorder from the virtual root (children slot 0)
        int32_t t = 0;
        std::vector<std::pair<int32_t, int32_t>> st;   // (node, next child index)
        st.push_back({-1, cptr[0]});
        while (!st.empty()) {
            auto& top = st.back();
            const int32_t u = top.first;
            if (top.second < cptr[u + 2]) {
                const int32_t c = cidx[top.second++];
                dtin[c] = t++;
                st.push_back({c, cptr[c + 1]});
            } else {
                if (u >= 0) dtout[u] = t;
                st.pop_back();
            }
        }
    }
    // --- eligible tensors (reading P6) -------------------------------------
    std::vector<int32_t> r_of(n, -1);
    int64_t nU = R > 0 ? d->late_user_ptr[R] : 0;
    if (R > 0 && d->late_user_ptr[0] != 0) return set_error(MAGIS_E_INVAL, "late_user_ptr[0] != 0");
    for (int32_t r = 0; r < R; r++) {
        int32_t t = d->eligible_tensor[r];
        if (t < 0 || t >= n) return set_error(MAGIS_E_INVAL, "eligible id out of range");
        if (d->is_output[t]) return set_error(MAGIS_E_INVAL, "graph output marked eligible: " + std::to_string(t));
        if (nreg[t] >= 0) return set_error(MAGIS_E_INVAL, "eligible tensor inside an F-Trans region: " + std::to_string(t));
        for (int32_t e = pred_ptr[t]; e < pred_ptr[t + 1]; e++)
            if (nreg[pred[e]] >= 0)
                return set_error(MAGIS_E_INVAL, "eligible tensor reads an F-Trans region: " + std::to_string(t));
        if (r_of[t] >= 0) return set_error(MAGIS_E_INVAL, "duplicate eligible tensor " + std::to_string(t));
        r_of[t] = r;
        int64_t a = d->late_user_ptr[r], b = d->late_user_ptr[r + 1];
        if (b <= a) return set_error(MAGIS_E_INVAL, "empty U_r for r=" + std::to_string(r));
        std::vector<int32_t> us(d->late_user_idx + a, d->late_user_idx + b);
        std::sort(us.begin(), us.end());
        if (std::unique(us.begin(), us.end()) != us.end())
            return set_error(MAGIS_E_INVAL, "duplicate late user for r=" + std::to_string(r));
        for (int32_t bb : us) {
            if (bb < 0 || bb >= n || !std::binary_search(succ.begin() + succ_ptr[t], succ.begin() + succ_ptr[t + 1], bb))
                return set_error(MAGIS_E_INVAL, "U_r not a subset of cons(t_r) for r=" + std::to_string(r));
            if (nreg[bb] >= 0) return set_error(MAGIS_E_INVAL, "late user inside an F-Trans region for r=" + std::to_string(r));
        }
    }
    const int32_t NT = n + 3 * R;

    // --- super-graph edges with gates (Fig. 8) ------------------------------
    struct SE { int32_t u, v, gate; };
    std::vector<SE> se;
    se.reserve((size_t)E + 2 * (size_t)nU + 2 * (size_t)R + 16);
    std::vector<std::vector<int32_t>> Uset(R);
    for (int32_t r = 0; r < R; r++) {
        Uset[r].assign(d->late_user_idx + d->late_user_ptr[r], d->late_user_idx + d->late_user_ptr[r + 1]);
        std::sort(Uset[r].begin(), Uset[r].end());
    }
    for (auto k : keys) {
        int32_t u = (int32_t)(k >> 32), v = (int32_t)(uint32_t)k;
        int32_t r = r_of[u];
        if (r >= 0 && std::binary_search(Uset[r].begin(), Uset[r].end(), v)) {
            se.push_back({u, v, (r << 2) | 0});              // t_r -> b kept (dec 0)
            se.push_back({n + 3 * r, v, (r << 2) | 1});      // clone_r -> b (dec 1)
            se.push_back({n + 3 * r + 2, v, (r << 2) | 2});  // load_r -> b (dec 2)
        } else {
            se.push_back({u, v, nreg[u] >= 0 ? nreg[u] : nreg[v]});   // kAlways (-1) outside regions
        }
    }
    for (int32_t r = 0; r < R; r++) {
        int32_t t = d->eligible_tensor[r];
        for (int32_t e = pred_ptr[t]; e < pred_ptr[t + 1]; e++)
            se.push_back({pred[e], n + 3 * r, (r << 2) | 1});   // A' reads A's inputs
        se.push_back({t, n + 3 * r + 1, (r << 2) | 2});          // A -> Store
        se.push_back({n + 3 * r + 1, n + 3 * r + 2, (r << 2) | 2});  // Store -> Load
    }
    const int64_t SEn = (int64_t)se.size();
    if (SEn > INT32_MAX) return set_error(MAGIS_E_UNSUPPORTED, "too many super-graph edges");

    std::vector<int32_t> cons_ptr(NT + 1, 0), in_ptr(NT + 1, 0);
    for (auto& x : se) { cons_ptr[x.u + 1]++; in_ptr[x.v + 1]++; }
    for (int32_t v = 0; v < NT; v++) { cons_ptr[v + 1] += cons_ptr[v]; in_ptr[v + 1] += in_ptr[v]; }
    std::vector<int2> cons_ent(SEn), in_ent(SEn);
    {
        std::sort(se.begin(), se.end(), [](const SE& a, const SE& b) { return a.u != b.u ? a.u < b.u : a.v < b.v; });
        for (int64_t i = 0; i < SEn; i++) cons_ent[i] = make_int2(se[i].v, se[i].gate);
        std::sort(se.begin(), se.end(), [](const SE& a, const SE& b) { return a.v != b.v ? a.v < b.v : a.u < b.u; });
        for (int64_t i = 0; i < SEn; i++) in_ent[i] = make_int2(se[i].u, se[i].gate);
    }
    // --- node tables (reading P5, P9) ----------------------------------------
    std::vector<int64_t> size(NT);
    std::vector<double> cost(NT, 0.0);
    std::vector<int32_t> ngate(NT, kAlways);
    std::vector<uint8_t> nflag(NT, 0);
    double base_cost = 0.0;
    std::vector<int32_t> nvar(std::max(F, 1), 1);
    std::vector<double> vcost((size_t)4 * std::max(F, 1), 0.0);
    for (int32_t i = 0; i < F; i++) nvar[i] = rd->n_variants[i];
    for (int32_t v = 0; v < n; v++) {
        size[v] = d->out_bytes[v];
        cost[v] = d->cost[v];
        nflag[v] = (uint8_t)((d->is_output[v] ? kFlagOutput : 0) | kFlagCompute);
        ngate[v] = nreg[v];
        if (nreg[v] >= 0) vcost[(size_t)4 * ((nreg[v] >> 2) - R) + (nreg[v] & 3)] += d->cost[v];
        else base_cost += d->cost[v];
    }
    std::vector<int32_t> elig(R), U_ptr(R + 1, 0), U_idx((size_t)nU);
    std::vector<double> xfer(R), tcost(R);
    std::vector<uint8_t> rflag(R);
    for (int32_t r = 0; r < R; r++) {
        int32_t t = d->eligible_tensor[r];
        elig[r] = t;
        size[n + 3 * r] = d->out_bytes[t];        // clone A' = |A|
        size[n + 3 * r + 1] = 0;                   // Store: data in external storage
        size[n + 3 * r + 2] = d->out_bytes[t];    // Load = |A|
        cost[n + 3 * r] = d->cost[t];              // cost(A') = cost(A)
        ngate[n + 3 * r] = (r << 2) | 1;
        ngate[n + 3 * r + 1] = (r << 2) | 2;
        ngate[n + 3 * r + 2] = (r << 2) | 2;
        nflag[n + 3 * r] = kFlagCompute;
        xfer[r] = d->swap_latency_s + (double)d->out_bytes[t] / d->swap_bytes_per_s;
        tcost[r] = d->cost[t];
        rflag[r] = (uint8_t)(pred_ptr[t + 1] > pred_ptr[t] ? kRHasInput : 0);
        U_ptr[r + 1] = U_ptr[r] + (int32_t)Uset[r].size();
        std::copy(Uset[r].begin(), Uset[r].end(), U_idx.begin() + U_ptr[r]);
    }

    // --- upload ----------------------------------------------------------------
    if (!magis_device_supported(device))
        return set_error(MAGIS_E_UNSUPPORTED, "device " + std::to_string(device) +
                         " is not an sm_100 (B200) GPU; there is no CPU fallback");
    DeviceGuard guard(device);
    magis_graph* g = new (std::nothrow) magis_graph();
    if (!g) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    g->device = device;
    g->n_edges = E;
    g->n_super_edges = SEn;
    struct Part { const void* src; size_t bytes; size_t off; };
    std::vector<Part> parts;
    size_t off = 0;
    auto add = [&](const void* p, size_t b) { parts.push_back({p, b, off}); size_t o = off; off = align_up(off + std::max<size_t>(b, 1), 256); return o; };
    size_t o_cons_ptr = add(cons_ptr.data(), cons_ptr.size() * 4);
    size_t o_cons_ent = add(cons_ent.data(), cons_ent.size() * 8);
    size_t o_in_ptr = add(in_ptr.data(), in_ptr.size() * 4);
    size_t o_in_ent = add(in_ent.data(), in_ent.size() * 8);
    size_t o_size = add(size.data(), size.size() * 8);
    size_t o_cost = add(cost.data(), cost.size() * 8);
    size_t o_ngate = add(ngate.data(), ngate.size() * 4);
    size_t o_nflag = add(nflag.data(), nflag.size());
    size_t o_elig = add(elig.data(), elig.size() * 4);
    size_t o_Uptr = add(U_ptr.data(), U_ptr.size() * 4);
    size_t o_Uidx = add(U_idx.data(), U_idx.size() * 4);
    size_t o_xfer = add(xfer.data(), xfer.size() * 8);
    size_t o_tcost = add(tcost.data(), tcost.size() * 8);
    size_t o_rflag = add(rflag.data(), rflag.size());
    // generator fast path: sources, and the slot map of the nodes whose base
    // position places the optional nodes (t_r, pre(t_r), U_r)
    std::vector<int32_t> gsrc, gqnode;
    std::vector<uint16_t> gqmap(n, 0xffffu);
    for (int32_t v = 0; v < n; v++)
        if (pred_ptr[v + 1] == pred_ptr[v]) gsrc.push_back(v);
    auto addq = [&](int32_t v) {
        if (gqmap[v] == 0xffffu && gqnode.size() < 0xffffu) {
            gqmap[v] = (uint16_t)gqnode.size();
            gqnode.push_back(v);
        }
    };
    for (int32_t r = 0; r < R; r++) {
        addq(elig[r]);
        for (int32_t e = pred_ptr[elig[r]]; e < pred_ptr[elig[r] + 1]; e++) addq(pred[e]);
        for (int32_t j = U_ptr[r]; j < U_ptr[r + 1]; j++) addq(U_idx[j]);
    }
    std::vector<uint32_t> gsinfo((size_t)2 * n), grec((size_t)2 * std::max<int64_t>(E, 1), 0);
    std::vector<int32_t> gwide(n, -1);            // wide slot of a node with more than 4 inputs
    int32_t gW = 0;
    for (int32_t v = 0; v < n; v++)
        if (pred_ptr[v + 1] - pred_ptr[v] > 4 && gW < 0xfffe) gwide[v] = gW++;
    for (int32_t u = 0; u < n; u++) {
        gsinfo[2 * u] = (uint32_t)succ_ptr[u];
        gsinfo[2 * u + 1] = (uint32_t)(succ_ptr[u + 1] - succ_ptr[u]) | ((uint32_t)gqmap[u] << 16);
        for (int32_t e = succ_ptr[u]; e < succ_ptr[u + 1]; e++) {
            const int32_t s2 = succ[e];
            uint32_t o[3] = {0xffffu, 0xffffu, 0xffffu};
            int no = 0;
            for (int32_t f = pred_ptr[s2]; f < pred_ptr[s2 + 1]; f++) {
                if (pred[f] == u) continue;
                if (no < 3) o[no] = (uint32_t)pred[f];
                no++;
            }
            if (no > 3) {
                o[0] = 0xfffeu;
                const int32_t deg = pred_ptr[s2 + 1] - pred_ptr[s2];
                if (gwide[s2] >= 0 && deg < 0xffff) {
                    o[1] = (uint32_t)gwide[s2];
                    o[2] = (uint32_t)deg;
                } else {
                    o[1] = o[2] = 0xffffu;                // no counter: the kernel scans the inputs
                }
            }
            grec[2 * e] = (uint32_t)s2 | (o[0] << 16);
            grec[2 * e + 1] = o[1] | (o[2] << 16);
        }
    }
    size_t o_gsinfo = add(gsinfo.data(), gsinfo.size() * 4);
    size_t o_grec = add(grec.data(), grec.size() * 4);
    size_t o_gsrc = add(gsrc.data(), gsrc.size() * 4);
    size_t o_gqmap = add(gqmap.data(), gqmap.size() * 2);
    size_t o_gqnode = add(gqnode.data(), gqnode.size() * 4);
    size_t o_sp = add(succ_ptr.data(), succ_ptr.size() * 4);
    size_t o_s = add(succ.data(), succ.size() * 4);
    size_t o_pp = add(pred_ptr.data(), pred_ptr.size() * 4);
    size_t o_p = add(pred.data(), pred.size() * 4);
    size_t o_dtin = add(dtin.data(), dtin.size() * 4);
    size_t o_dtout = add(dtout.data(), dtout.size() * 4);
    size_t o_nvar = add(nvar.data(), nvar.size() * 4);
    size_t o_vcost = add(vcost.data(), vcost.size() * 8);
    g->blob_bytes = off;
    cudaError_t e = cudaMalloc(&g->blob, off);
    if (e != cudaSuccess) {
        cudaGetLastError();
        delete g;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc graph tables failed");
    }
    std::vector<char> host(off, 0);
    for (auto& p : parts)
        if (p.bytes) std::memcpy(host.data() + p.off, p.src, p.bytes);
    e = cudaMemcpy(g->blob, host.data(), off, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        cudaGetLastError();
        cudaFree(g->blob);
        delete g;
        return set_error(MAGIS_E_CUDA, "upload of graph tables failed");
    }
    char* b = (char*)g->blob;
    DevGraph& dg = g->dev;
    dg.n = n;
    dg.R = R;
    dg.NT = NT;
    dg.max_events = 3 * R + (int32_t)nU;
    dg.cons_ptr = (const int32_t*)(b + o_cons_ptr);
    dg.cons_ent = (const int2*)(b + o_cons_ent);
    dg.in_ptr = (const int32_t*)(b + o_in_ptr);
    dg.in_ent = (const int2*)(b + o_in_ent);
    dg.size = (const int64_t*)(b + o_size);
    dg.cost = (const double*)(b + o_cost);
    dg.ngate = (const int32_t*)(b + o_ngate);
    dg.nflag = (const uint8_t*)(b + o_nflag);
    dg.elig = (const int32_t*)(b + o_elig);
    dg.U_ptr = (const int32_t*)(b + o_Uptr);
    dg.U_idx = (const int32_t*)(b + o_Uidx);
    dg.xfer = (const double*)(b + o_xfer);
    dg.tcost = (const double*)(b + o_tcost);
    dg.rflag = (const uint8_t*)(b + o_rflag);
    dg.base_cost = base_cost;
    dg.dtin = (const int32_t*)(b + o_dtin);
    dg.dtout = (const int32_t*)(b + o_dtout);
    dg.pred_ptr = (const int32_t*)(b + o_pp);
    dg.pred = (const int32_t*)(b + o_p);
    dg.F = F;
    dg.Rd = R + F;
    dg.nvar = (const int32_t*)(b + o_nvar);
    dg.vcost = (const double*)(b + o_vcost);
    g->idom = idom;
    // host copies for plans built after load (GraphHash, NEXT-2)
    g->h_pred_ptr = pred_ptr;
    g->h_pred = pred;
    g->h_topo = topo;
    g->h_elig = elig;
    g->h_Uptr = U_ptr;
    g->h_Uidx = U_idx;
    g->h_rflag = rflag;
    g->gen.succ_ptr = (const int32_t*)(b + o_sp);
    g->gen.succ = (const int32_t*)(b + o_s);
    g->gen.pred_ptr = (const int32_t*)(b + o_pp);
    g->gen.pred = (const int32_t*)(b + o_p);
    g->gen.src = (const int32_t*)(b + o_gsrc);
    g->gen.qmap = (const uint16_t*)(b + o_gqmap);
    g->gen.qnode = (const int32_t*)(b + o_gqnode);
    g->gen.sinfo = (const uint2*)(b + o_gsinfo);
    g->gen.rec = (const uint2*)(b + o_grec);
    g->gen.S = (int32_t)gsrc.size();
    g->gen.W = gW;
    g->gen.nq = (int32_t)gqnode.size();
    g->gen.fast = (n < 0xffff && gqnode.size() < 0xffffu && R < 32768) ? 1 : 0;

    e = eval_configure(dg, device, &g->cfg);
    if (e != cudaSuccess) {
        cudaGetLastError();
        cudaFree(g->blob);
        delete g;
        return set_error(MAGIS_E_CUDA, std::string("eval_configure: ") + cudaGetErrorString(e));
    }
    // --- variant 2: packed streams in shared memory (magis_eval2.cu) -----------
    {
        const char* force = std::getenv("MAGIS_VARIANT");
        const char* pforce = std::getenv("MAGIS_P");
        const bool allow2 = !(force && std::atoi(force) != 2);
        cudaDeviceProp prop;
        if (allow2 && cudaGetDeviceProperties(&prop, device) == cudaSuccess) {
            std::vector<double> rtab((size_t)2 * R);
            for (int32_t r = 0; r < R; r++) { rtab[2 * r] = tcost[r]; rtab[2 * r + 1] = xfer[r]; }
            SuperGraphHost sg{n, R, NT, cons_ptr.data(), cons_ent.data(), in_ptr.data(), in_ent.data(),
                              size.data(), cost.data(), nflag.data(), U_ptr.data(), U_idx.data(), rtab.data(),
                              elig.data(), F, ngate.data(), nvar.data(), vcost.data()};
            const size_t cap = (size_t)prop.sharedMemPerBlockOptin - 4096;
            // pick the packing with the most candidates in flight per SM
            // (P x resident CTAs; ties go to more CTAs, which hide barriers).
            // Tiers, in order: graph tables and step slots in shared memory;
            // tables read from global (L2); tables and slots in global.
            // Teams (two independent warp groups per CTA sharing the tables)
            // count as extra resident groups: candidates in flight = P x teams
            // x CTAs; ties prefer one team with the wider packing (measured on
            // C2 / C5: 1 team x P=4 beats 2 teams x P=2 by 16-19%, the packed
            // u16x4 work outweighs the overlapped barrier waits).
            const int cands[3] = {4, 2, 1};
            const char* tforce = std::getenv("MAGIS_TEAMS");
            int bestP = 0, bestOcc = 0, bestT = 1;
            Plan2 bestPl{};
            std::vector<char> bestImg;
            // tier 2 = tables in global, one signed delta per step in shared
            // memory (alloc - free of the previous step); tier 3 = tables and
            // slots in global
            const char* tierf = std::getenv("MAGIS_TIER");
            for (int tier = 0; tier < 4 && bestP == 0; tier++) {
                if (tierf && std::atoi(tierf) != tier) continue;
                const bool gs = tier >= 1, fo = tier == 2, ga = tier == 3;
                for (int T = 2; T >= 1; T--) {
                    if (tforce && std::atoi(tforce) != T) continue;
                    if (T == 2 && gs) continue;                     // teams only with the tables in smem
                    for (int ci = 0; ci < 3; ci++) {
                        const int P = cands[ci];
                        if (pforce && std::atoi(pforce) != P) continue;
                        Plan2 pl;
                        std::vector<char> img;
                        if (!plan2_build(sg, P, T, gs, ga, fo, cap, &pl, &img)) continue;
                        int occ = 0;
                        cudaError_t oe = eval2_occupancy(pl, &occ);
                        if (std::getenv("MAGIS_DEBUG"))
                            std::fprintf(stderr,
                                         "[magis] plan tier=%d teams=%d P=%d L=%d S=%d smem=%u static=%u occ=%d err=%d\n",
                                         tier, T, P, pl.L, pl.S, pl.smem_total, pl.static_bytes, occ, (int)oe);
                        if (std::getenv("MAGIS_DEBUG") && std::atoi(std::getenv("MAGIS_DEBUG")) > 1)
                            std::fprintf(stderr,
                                         "[magis]   tables: wtab %u crow %u chdr %u csize %u cent %u (rows_sm %d) frow %u fhdr %u fent %u "
                                         "size %u cost %u rtab %u ninfo %u lul %u urow %u ubs %u utr %u rn %u | state: pos %u "
                                         "last %u af %u dec %u end %u evm %u sdec %u ev %u (cap %d) stage %u\n",
                                         pl.off_crow - pl.off_wtab, pl.off_chdr - pl.off_crow, pl.off_cent - pl.off_chdr,
                                         pl.off_frow - pl.off_csize, pl.off_csize - pl.off_cent, pl.rows_sm, pl.off_fhdr - pl.off_frow,
                                         pl.off_fent - pl.off_fhdr, pl.off_size - pl.off_fent, pl.off_cost - pl.off_size,
                                         pl.off_rtab - pl.off_cost, pl.off_ninfo - pl.off_rtab, pl.off_lul - pl.off_ninfo,
                                         pl.off_urow - pl.off_lul, pl.off_ubs - pl.off_urow, pl.off_utr - pl.off_ubs,
                                         pl.off_rn - pl.off_utr, pl.off_nvar - pl.off_rn, pl.off_last - pl.off_pos,
                                         pl.off_af - pl.off_last, pl.off_dec - pl.off_af, pl.off_end - pl.off_dec,
                                         pl.off_evm - pl.off_end, pl.off_sdec - pl.off_evm, pl.off_ev - pl.off_sdec,
                                         pl.smem_total - pl.off_ev, pl.evcap, pl.stage_bytes);
                        if (oe != cudaSuccess || occ < 1) { cudaGetLastError(); continue; }
                        const int a = P * T * occ, b = bestP * bestT * bestOcc;
                        if (a > b || (a == b && (T < bestT || (T == bestT && occ > bestOcc)))) {
                            bestP = P;
                            bestT = T;
                            bestOcc = occ;
                            bestPl = pl;
                            bestImg.swap(img);
                        }
                    }
                }
            }
            if (bestP > 0) {
                void* b2 = nullptr;
                void* ov = nullptr;
                const int grid = prop.multiProcessorCount * bestOcc;
                bool ok = cudaMalloc(&b2, bestImg.size()) == cudaSuccess;
                ok = ok && cudaMemcpy(b2, bestImg.data(), bestImg.size(), cudaMemcpyHostToDevice) == cudaSuccess;
                bestPl.prof = std::getenv("MAGIS_PROFILE") ? 1 : 0;
                // graph image read from global memory: reserve persisting L2 for it
                // (SURVEY §8(a) a0 "L2 window"); the launch sets the window
                bestPl.l2win_bytes = 0;
                if (bestPl.gmem_static && !std::getenv("MAGIS_NO_L2WIN") && prop.persistingL2CacheMaxSize > 0) {
                    const size_t want = std::min<size_t>(bestImg.size(), (size_t)prop.accessPolicyMaxWindowSize);
                    size_t cur = 0;
                    cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
                    const size_t lim = std::min<size_t>((size_t)prop.persistingL2CacheMaxSize, std::max(cur, want));
                    if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, lim) == cudaSuccess)
                        bestPl.l2win_bytes = std::min(want, lim);
                    else
                        cudaGetLastError();
                }
                bestPl.prof_off = (uint64_t)grid * bestT * 8 * bestPl.ovf_stride;   // 8 regions per team
                ok = ok && cudaMalloc(&ov, bestPl.prof_off + 256) == cudaSuccess;
                ok = ok && cudaMemset(ov, 0, bestPl.prof_off + 256) == cudaSuccess;
                void* ag = nullptr;
                if (ok && bestPl.gmem_af) ok = cudaMalloc(&ag, (size_t)grid * bestT * bestPl.af_bytes) == cudaSuccess;
                g->afg2 = ag;
                if (ok) {
                    g->plan2 = bestPl;
                    g->blob2 = b2;
                    g->blob2_bytes = bestImg.size();
                    g->ovf2 = ov;
                    g->cfg.variant = 2;
                    g->cfg.grid = grid;
                    g->cfg.block = eval2_block(bestPl);
                    g->cfg.smem = bestPl.smem_total;
                } else {
                    cudaGetLastError();
                    if (b2) cudaFree(b2);
                    if (ov) cudaFree(ov);
                }
            }
        }
    }
    // --- kernel B (magis_evalb.cu): one candidate per two-CTA cluster, opt-in
    //     (MAGIS_KERNELB=1; measured against the single-CTA plans)
    const char* kbenv = std::getenv("MAGIS_KERNELB");
    if (kbenv && kbenv[0] == '1' && F == 0) {
        cudaDeviceProp prop;
        if (cudaGetDeviceProperties(&prop, device) == cudaSuccess) {
            std::vector<double> rtab((size_t)2 * R);
            for (int32_t r = 0; r < R; r++) { rtab[2 * r] = tcost[r]; rtab[2 * r + 1] = xfer[r]; }
            SuperGraphHost sg{n, R, NT, cons_ptr.data(), cons_ent.data(), in_ptr.data(), in_ent.data(),
                              size.data(), cost.data(), nflag.data(), U_ptr.data(), U_idx.data(), rtab.data(),
                              elig.data(), F, ngate.data(), nvar.data(), vcost.data()};
            const size_t cap = (size_t)prop.sharedMemPerBlockOptin - 4096;
            Plan2 pl;
            std::vector<char> img;
            BLayout lay;
            if (plan2_build(sg, 1, 1, true, false, true, cap, &pl, &img, 2) && evalb_layout(pl, cap, &lay)) {
                const int clusters = prop.multiProcessorCount / 2;
                void* b2 = nullptr;
                void* ev = nullptr;
                bool ok = cudaMalloc(&b2, img.size()) == cudaSuccess;
                ok = ok && cudaMemcpy(b2, img.data(), img.size(), cudaMemcpyHostToDevice) == cudaSuccess;
                ok = ok && cudaMalloc(&ev, evalb_scratch_bytes(pl, clusters)) == cudaSuccess;
                if (ok) {
                    if (g->blob2) cudaFree(g->blob2);
    if (g->evb) cudaFree(g->evb);
                    if (g->ovf2) { cudaFree(g->ovf2); g->ovf2 = nullptr; }
                    if (g->afg2) { cudaFree(g->afg2); g->afg2 = nullptr; }
                    g->plan2 = pl;
                    g->blob2 = b2;
                    g->blob2_bytes = img.size();
                    g->layb = lay;
                    g->clustersb = clusters;
                    g->evb = ev;
                    g->cfg.variant = 3;
                    g->cfg.grid = 2 * clusters;
                    g->cfg.block = 512;
                    g->cfg.smem = lay.total;
                } else {
                    cudaGetLastError();
                    if (b2) cudaFree(b2);
                    if (ev) cudaFree(ev);
                }
            }
        }
    }
    if (g->cfg.variant == 1) {
        g->gws_bytes = g->cfg.state_bytes * (size_t)g->cfg.grid;
        e = cudaMalloc(&g->gws, g->gws_bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            cudaFree(g->blob);
            delete g;
            return set_error(MAGIS_E_NOMEM, "cudaMalloc eval workspace failed");
        }
    }
    *out = g;
    return MAGIS_SUCCESS;
}

extern "C" int magis_graph_free(magis_graph* g) {
    clear_error();
    if (!g) return MAGIS_SUCCESS;
    DeviceGuard guard(g->device);
    cudaDeviceSynchronize();
    if (g->blob) cudaFree(g->blob);
    if (g->gws) cudaFree(g->gws);
    if (g->blob2) cudaFree(g->blob2);
    if (g->evb) cudaFree(g->evb);
    if (g->ovf2) cudaFree(g->ovf2);
    if (g->hs_ws) cudaFree(g->hs_ws);
    if (g->afg2) cudaFree(g->afg2);
    if (g->gen_scratch) cudaFree(g->gen_scratch);
    for (int i = 0; i < 2; i++) {
        if (g->stage[i]) cudaFree(g->stage[i]);
        if (g->ev_h2d[i]) cudaEventDestroy(g->ev_h2d[i]);
        if (g->ev_done[i]) cudaEventDestroy(g->ev_done[i]);
    }
    if (g->aux) cudaStreamDestroy(g->aux);
    cudaGetLastError();
    delete g;
    return MAGIS_SUCCESS;
}

extern "C" int magis_graph_info_get(const magis_graph* g, magis_graph_info* info) {
    clear_error();
    if (!g || !info) return set_error(MAGIS_E_INVAL, "null argument");
    info->n_nodes = g->dev.n;
    info->n_eligible = g->dev.R;
    info->n_total = g->dev.NT;
    info->n_edges = g->n_edges;
    info->n_super_edges = g->n_super_edges;
    info->device = g->device;
    info->variant = g->cfg.variant;
    info->grid = g->cfg.grid;
    info->block = g->cfg.block;
    info->smem_bytes = (int64_t)g->cfg.smem;
    info->table_bytes = (int64_t)g->blob_bytes;
    info->base_cost = g->dev.base_cost;
    info->pack = g->cfg.variant == 2 ? g->plan2.P : 1;
    info->n_regions = g->dev.F;
    return MAGIS_SUCCESS;
}

extern "C" int magis_eval_schedules(const magis_graph* g, int64_t K, const int32_t* d_perm,
                                    const uint8_t* d_dec, uint8_t* d_status, int64_t* d_peak,
                                    double* d_latency, void* cuda_stream) {
    clear_error();
    if (!g) return set_error(MAGIS_E_INVAL, "graph is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_perm || !d_status || !d_peak || !d_latency)
        return set_error(MAGIS_E_INVAL, "null device pointer");
    if (g->dev.Rd > 0 && !d_dec) return set_error(MAGIS_E_INVAL, "d_dec is NULL but R + n_regions > 0");
    DeviceGuard guard(g->device);
    cudaError_t e = dispatch_eval(g, K, d_perm, d_dec, d_status, d_peak, d_latency,
                                  (cudaStream_t)cuda_stream);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("eval launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}

// a7's optional output: the step that first reaches the peak, in the batch call
extern "C" int magis_eval_schedules_argmax(const magis_graph* g, int64_t K, const int32_t* d_perm,
                                           const uint8_t* d_dec, uint8_t* d_status, int64_t* d_peak,
                                           double* d_latency, int32_t* d_argmax, void* cuda_stream) {
    clear_error();
    if (!g) return set_error(MAGIS_E_INVAL, "graph is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_perm || !d_status || !d_peak || !d_latency || !d_argmax)
        return set_error(MAGIS_E_INVAL, "null device pointer");
    if (g->dev.Rd > 0 && !d_dec) return set_error(MAGIS_E_INVAL, "d_dec is NULL but R + n_regions > 0");
    if (g->cfg.variant != 2)
        return set_error(MAGIS_E_UNSUPPORTED, "argmax output needs the packed kernel (the graph is too large for it)");
    DeviceGuard guard(g->device);
    cudaError_t e = eval2_launch(g->dev, g->plan2, g->blob2, g->ovf2, g->afg2, g->cfg.grid, K, d_perm, d_dec,
                                 d_status, d_peak, d_latency, (cudaStream_t)cuda_stream, d_argmax);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("eval launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}

// NEXT-3: hot-spots and heat / score of selected candidates.
extern "C" int magis_hotspots(magis_graph* g, int64_t K, const int32_t* d_perm, const uint8_t* d_dec,
                              int32_t nsplit, uint8_t* d_status, int64_t* d_peak, uint8_t* d_hot,
                              int64_t* d_heat, double* d_score, void* cuda_stream) {
    clear_error();
    if (g && g->dev.F > 0) return set_error(MAGIS_E_UNSUPPORTED, "magis_hotspots: not available on graphs with F-Trans regions");
    if (!g) return set_error(MAGIS_E_INVAL, "graph is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (nsplit < 1) return set_error(MAGIS_E_INVAL, "nsplit < 1");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_perm || !d_status || !d_peak || !d_hot) return set_error(MAGIS_E_INVAL, "null device pointer");
    if (g->dev.Rd > 0 && !d_dec) return set_error(MAGIS_E_INVAL, "d_dec is NULL but R + n_regions > 0");
    DeviceGuard guard(g->device);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, g->device);
    const int grid = std::max(1, sms) * 2;
    const size_t need = hotspot_ws_per_cta(g->dev) * (size_t)grid;
    if (g->hs_ws_bytes < need) {
        if (g->hs_ws) { cudaDeviceSynchronize(); cudaFree(g->hs_ws); g->hs_ws = nullptr; g->hs_ws_bytes = 0; }
        if (cudaMalloc(&g->hs_ws, need) != cudaSuccess) {
            cudaGetLastError();
            return set_error(MAGIS_E_NOMEM, "cudaMalloc hot-spot workspace failed");
        }
        g->hs_ws_bytes = need;
    }
    cudaError_t e = hotspot_launch(g->dev, grid, g->hs_ws, K, d_perm, d_dec, nsplit, d_status, d_peak, d_hot, d_heat,
                                   d_score, (cudaStream_t)cuda_stream);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("hotspot launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}

extern "C" int magis_graph_idom(const magis_graph* g, int32_t* idom) {
    clear_error();
    if (!g || !idom) return set_error(MAGIS_E_INVAL, "null argument");
    for (size_t v = 0; v < g->idom.size(); v++) idom[v] = g->idom[v];
    return MAGIS_SUCCESS;
}

// End-to-end host path: chunked, double-buffered H2D -> eval -> D2H.
namespace {

__global__ void widen_u16(const uint16_t* __restrict__ src, int32_t* __restrict__ dst, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = (int32_t)src[i];
}

// Delta wire formats: per step the difference to the previous step's id (the
// row starts from 0), or an escape = "take the next value of the row's
// exception list" (an absolute uint16 id).  delta8: one int8 per step, escape
// -128.  delta4: one nibble per step (step j in byte j / 2, low nibble first),
// code c: 0 = escape, else delta c - 8 (-7 .. +7).  One warp per row: the
// exception ranks come from a ballot, and a segmented scan over (reset, value)
// pairs rebuilds the ids 32 steps at a time.
template <int BITS>
__global__ void decode_delta(const uint8_t* __restrict__ code, int64_t row_b, const int32_t* __restrict__ exc_ptr,
                             const uint16_t* __restrict__ exc, int64_t kc, int32_t NT, int32_t* __restrict__ out) {
    const int lane = threadIdx.x & 31;
    const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int32_t e0 = exc_ptr[0];
    for (int64_t k = w0; k < kc; k += nw) {
        const uint8_t* dr = code + k * row_b;
        int32_t* orow = out + k * (int64_t)NT;
        int32_t carry = 0, ec = exc_ptr[k] - e0;
        for (int32_t t = 0; t < NT; t += 32) {
            const int32_t j = t + lane;
            int32_t b = 0;
            bool isx = false;
            if (j < NT) {
                if (BITS == 8) {
                    b = (int32_t)(int8_t)dr[j];
                    isx = b == -128;
                } else {
                    const int32_t c = (dr[j >> 1] >> ((j & 1) * 4)) & 15;
                    isx = c == 0;
                    b = c - 8;
                }
            }
            const unsigned m = __ballot_sync(0xffffffffu, isx);
            int32_t v = isx ? (int32_t)exc[ec + __popc(m & ((1u << lane) - 1u))] : b;
            bool rs = isx;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int32_t pv = __shfl_up_sync(0xffffffffu, v, o);
                const bool pr = __shfl_up_sync(0xffffffffu, (int)rs, o);
                if (lane >= o && !rs) { v += pv; rs = pr; }
            }
            if (!rs) v += carry;
            if (j < NT) orow[j] = v;
            carry = __shfl_sync(0xffffffffu, v, 31);
            ec += __popc(m);
        }
    }
}

// pb = the host wire format (4: int32, 2: uint16 widened on the device,
// 1: delta8, 0: delta4 -- both decoded on the device, h_exc_ptr / h_exc then
// hold the exception lists)
int host_path(magis_graph* g, int64_t K, const void* h_perm, int pb, const uint8_t* h_dec, uint8_t* h_status,
              int64_t* h_peak, double* h_latency, void* cuda_stream, const int32_t* h_exc_ptr = nullptr,
              const uint16_t* h_exc = nullptr) {
    clear_error();
    if (!g) return set_error(MAGIS_E_INVAL, "graph is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!h_perm || !h_status || !h_peak || !h_latency)
        return set_error(MAGIS_E_INVAL, "null host pointer");
    const int32_t R = g->dev.Rd, NT = g->dev.NT;          // decision row: R eligible + F regions
    if (R > 0 && !h_dec) return set_error(MAGIS_E_INVAL, "h_dec is NULL but R + n_regions > 0");
    if (pb <= 2 && NT > 65535) return set_error(MAGIS_E_UNSUPPORTED, "compact schedules need n_total <= 65535");
    const size_t row_b = pb == 0 ? (size_t)(NT + 1) / 2 : (size_t)NT * pb;   // host bytes per schedule
    if (pb <= 1) {
        if (!h_exc_ptr) return set_error(MAGIS_E_INVAL, "null exception pointer array");
        for (int64_t k = 0; k < K; k++) {
            if (h_exc_ptr[k + 1] < h_exc_ptr[k]) return set_error(MAGIS_E_INVAL, "exception offsets decrease");
            // no row has more escapes than steps (bounds the staging copy)
            if (h_exc_ptr[k + 1] - h_exc_ptr[k] > NT)
                return set_error(MAGIS_E_INVAL, "more exceptions than steps in schedule " + std::to_string(k));
        }
        if (h_exc_ptr[K] > h_exc_ptr[0] && !h_exc) return set_error(MAGIS_E_INVAL, "null exception array");
    }
    DeviceGuard guard(g->device);
    cudaStream_t s0 = (cudaStream_t)cuda_stream;
    // chunk of ~64 MiB of int32 perms
    int64_t chunk = std::max<int64_t>(1, (64ll << 20) / ((int64_t)NT * 4));
    chunk = std::min<int64_t>(chunk, K);
    const size_t perm_b = align_up((size_t)chunk * NT * 4, 256);
    const size_t narrow_b = align_up((size_t)chunk * NT * 2, 256);
    const size_t dec_b = align_up((size_t)chunk * std::max(R, 1), 256);
    const size_t out_b = align_up((size_t)chunk * 17, 256);
    const size_t excp_b = align_up((size_t)(chunk + 1) * 4, 256);   // delta8: exception offsets, then values
    if (g->stage_K < chunk) {
        for (int i = 0; i < 2; i++) {
            if (g->stage[i]) cudaFree(g->stage[i]);
            g->stage[i] = nullptr;
            CK(cudaMalloc(&g->stage[i], perm_b + narrow_b + dec_b + out_b + 256 + excp_b + narrow_b + 256));
            if (!g->ev_h2d[i]) CK(cudaEventCreateWithFlags(&g->ev_h2d[i], cudaEventDisableTiming));
            if (!g->ev_done[i]) CK(cudaEventCreateWithFlags(&g->ev_done[i], cudaEventDisableTiming));
        }
        if (!g->aux) CK(cudaStreamCreateWithFlags(&g->aux, cudaStreamNonBlocking));
        g->stage_K = chunk;
    }
    // copies on aux, compute on s0; two buffers alternate.
    int64_t nchunks = (K + chunk - 1) / chunk;
    for (int64_t c = 0; c < nchunks; c++) {
        int b = (int)(c & 1);
        int64_t k0 = c * chunk, kc = std::min(chunk, K - k0);
        char* base = (char*)g->stage[b];
        int32_t* dp = (int32_t*)base;
        uint16_t* dn = (uint16_t*)(base + perm_b);
        uint8_t* dd = (uint8_t*)(base + perm_b + narrow_b);
        char* ob = base + perm_b + narrow_b + dec_b;
        int64_t* dpk = (int64_t*)ob;
        double* dlt = (double*)(ob + align_up((size_t)chunk * 8, 64));
        uint8_t* dst = (uint8_t*)(ob + 2 * align_up((size_t)chunk * 8, 64));
        // buffer b is free once the D2H of chunk c-2 finished
        if (c >= 2) CK(cudaStreamWaitEvent(g->aux, g->ev_done[b], 0));
        const char* hp = (const char*)h_perm + (size_t)k0 * row_b;
        int32_t* dxp = (int32_t*)(ob + out_b + 256);    // past the outputs (which may spill 128 B over out_b)
        uint16_t* dxv = (uint16_t*)((char*)dxp + excp_b);
        CK(cudaMemcpyAsync(pb == 4 ? (void*)dp : (void*)dn, hp, (size_t)kc * row_b, cudaMemcpyHostToDevice, g->aux));
        if (pb <= 1) {
            const int64_t x0 = h_exc_ptr[k0], x1 = h_exc_ptr[k0 + kc];
            CK(cudaMemcpyAsync(dxp, h_exc_ptr + k0, (size_t)(kc + 1) * 4, cudaMemcpyHostToDevice, g->aux));
            if (x1 > x0) CK(cudaMemcpyAsync(dxv, h_exc + x0, (size_t)(x1 - x0) * 2, cudaMemcpyHostToDevice, g->aux));
        }
        if (R > 0) CK(cudaMemcpyAsync(dd, h_dec + k0 * R, (size_t)kc * R, cudaMemcpyHostToDevice, g->aux));
        CK(cudaEventRecord(g->ev_h2d[b], g->aux));
        CK(cudaStreamWaitEvent(s0, g->ev_h2d[b], 0));
        if (pb <= 1) {
            const int blocks = (int)std::min<int64_t>((kc + 7) / 8, 4096);
            if (pb == 1) decode_delta<8><<<blocks, 256, 0, s0>>>((const uint8_t*)dn, (int64_t)row_b, dxp, dxv, kc, NT, dp);
            else decode_delta<4><<<blocks, 256, 0, s0>>>((const uint8_t*)dn, (int64_t)row_b, dxp, dxv, kc, NT, dp);
        }
        if (pb == 2) {
            const int64_t ne = kc * (int64_t)NT;
            const int blocks = (int)std::min<int64_t>((ne + 255) / 256, 4096);
            widen_u16<<<blocks, 256, 0, s0>>>(dn, dp, ne);
        }
        cudaError_t e = dispatch_eval(g, kc, dp, R > 0 ? dd : nullptr, dst, dpk, dlt, s0);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return set_error(MAGIS_E_CUDA, std::string("eval launch: ") + cudaGetErrorString(e));
        }
        CK(cudaMemcpyAsync(h_status + k0, dst, (size_t)kc, cudaMemcpyDeviceToHost, s0));
        CK(cudaMemcpyAsync(h_peak + k0, dpk, (size_t)kc * 8, cudaMemcpyDeviceToHost, s0));
        CK(cudaMemcpyAsync(h_latency + k0, dlt, (size_t)kc * 8, cudaMemcpyDeviceToHost, s0));
        CK(cudaEventRecord(g->ev_done[b], s0));
    }
    CK(cudaStreamSynchronize(s0));
    return MAGIS_SUCCESS;
}

}  // namespace

extern "C" int magis_eval_schedules_host(magis_graph* g, int64_t K, const int32_t* h_perm,
                                         const uint8_t* h_dec, uint8_t* h_status,
                                         int64_t* h_peak, double* h_latency,
                                         void* cuda_stream) {
    return host_path(g, K, h_perm, 4, h_dec, h_status, h_peak, h_latency, cuda_stream);
}

extern "C" int magis_eval_schedules_host_u16(magis_graph* g, int64_t K, const uint16_t* h_perm,
                                             const uint8_t* h_dec, uint8_t* h_status,
                                             int64_t* h_peak, double* h_latency,
                                             void* cuda_stream) {
    return host_path(g, K, h_perm, 2, h_dec, h_status, h_peak, h_latency, cuda_stream);
}

extern "C" int magis_eval_schedules_host_delta8(magis_graph* g, int64_t K, const int8_t* h_delta,
                                                const int32_t* h_exc_ptr, const uint16_t* h_exc,
                                                const uint8_t* h_dec, uint8_t* h_status, int64_t* h_peak,
                                                double* h_latency, void* cuda_stream) {
    return host_path(g, K, h_delta, 1, h_dec, h_status, h_peak, h_latency, cuda_stream, h_exc_ptr, h_exc);
}

extern "C" int magis_eval_schedules_host_delta4(magis_graph* g, int64_t K, const uint8_t* h_code,
                                                const int32_t* h_exc_ptr, const uint16_t* h_exc,
                                                const uint8_t* h_dec, uint8_t* h_status, int64_t* h_peak,
                                                double* h_latency, void* cuda_stream) {
    return host_path(g, K, h_code, 0, h_dec, h_status, h_peak, h_latency, cuda_stream, h_exc_ptr, h_exc);
}

extern "C" int magis_generate_candidates(magis_graph* g, const magis_gen_spec* spec, uint64_t id0, int64_t K,
                                         int32_t* d_perm, uint8_t* d_dec, void* cuda_stream) {
    clear_error();
    if (g && g->dev.F > 0) return set_error(MAGIS_E_UNSUPPORTED, "magis_generate_candidates: not available on graphs with F-Trans regions");
    if (!g || !spec) return set_error(MAGIS_E_INVAL, "null argument");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_perm || !d_dec) return set_error(MAGIS_E_INVAL, "null device pointer");
    if (spec->pct_random < 0 || spec->pct_local < 0 || spec->pct_random + spec->pct_local > 100 ||
        spec->p_remat < 0 || spec->p_swap < 0 || spec->p_remat + spec->p_swap > 10000 || spec->wmax < 2 ||
        spec->slack < 0)
        return set_error(MAGIS_E_INVAL, "bad generator spec");
    DeviceGuard guard(g->device);
    // scratch of the launch plan (grown on demand)
    const GenPlan gp = gen_plan(g->device, g->dev, g->gen, K);
    if (!g->gen_scratch || g->gen_bytes < gp.bytes) {
        if (g->gen_scratch) cudaFree(g->gen_scratch);
        g->gen_scratch = nullptr;
        g->gen_bytes = 0;
        CK(cudaMalloc(&g->gen_scratch, gp.bytes));
        g->gen_bytes = gp.bytes;
    }
    GenSpec sp{spec->seed, spec->pct_random, spec->pct_local, spec->p_remat, spec->p_swap, spec->wmax, spec->slack};
    cudaError_t e = gen_launch(g->dev, g->gen, sp, id0, K, d_perm, d_dec, g->gen_scratch, gp,
                               (cudaStream_t)cuda_stream);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("generator launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}

// ------------------------------------------------ windowed delta evaluation --
extern "C" int magis_base_create(magis_graph* g, const int32_t* d_perm, const uint8_t* d_dec, magis_base** out,
                                 void* cuda_stream) {
    clear_error();
    if (g && g->dev.F > 0) return set_error(MAGIS_E_UNSUPPORTED, "magis_base_create: not available on graphs with F-Trans regions");
    if (!out) return set_error(MAGIS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (!g || !d_perm) return set_error(MAGIS_E_INVAL, "null argument");
    if (g->dev.Rd > 0 && !d_dec) return set_error(MAGIS_E_INVAL, "d_dec is NULL but R + n_regions > 0");
    DeviceGuard guard(g->device);
    magis_base* b = new (std::nothrow) magis_base();
    if (!b) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    b->g = g;
    b->grid = window_grid(g->device);
    const size_t wsb = (size_t)b->grid * 8 * 3 * std::max(g->dev.R, 1) * sizeof(double);
    if (cudaMalloc(&b->mem, base_bytes(g->dev)) != cudaSuccess ||
        cudaMalloc((void**)&b->endb_ws, wsb) != cudaSuccess) {
        cudaGetLastError();
        if (b->mem) cudaFree(b->mem);
        delete b;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc base failed");
    }
    b->dev = base_layout(g->dev, b->mem);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    cudaMemsetAsync(b->dev.endb, 0, (size_t)std::max(g->dev.R, 1) * 24, s);
    cudaError_t e = base_launch(g->dev, b->dev, d_perm, d_dec ? d_dec : (const uint8_t*)b->dev.dec, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        cudaFree(b->mem);
        cudaFree(b->endb_ws);
        delete b;
        return set_error(MAGIS_E_CUDA, std::string("base launch: ") + cudaGetErrorString(e));
    }
    *out = b;
    return MAGIS_SUCCESS;
}

extern "C" int magis_base_info(const magis_base* b, int* status, int64_t* peak, double* latency) {
    clear_error();
    if (!b) return set_error(MAGIS_E_INVAL, "base is NULL");
    DeviceGuard guard(b->g->device);
    BaseHdr h;
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(&h, b->dev.hdr, sizeof(h), cudaMemcpyDeviceToHost));
    if (status) *status = h.status;
    if (peak) *peak = h.status ? -1 : h.peak;
    if (latency) *latency = h.status ? INFINITY : h.latency;
    return MAGIS_SUCCESS;
}

extern "C" int magis_base_free(magis_base* b) {
    clear_error();
    if (!b) return MAGIS_SUCCESS;
    DeviceGuard guard(b->g->device);
    cudaDeviceSynchronize();
    cudaFree(b->mem);
    cudaFree(b->endb_ws);
    cudaGetLastError();
    delete b;
    return MAGIS_SUCCESS;
}

extern "C" int magis_eval_windows(const magis_base* b, int64_t K, const int32_t* d_wstart, const int32_t* d_wlen,
                                  const int32_t* d_wperm, int32_t wmax, uint8_t* d_status, int64_t* d_peak,
                                  double* d_latency, void* cuda_stream) {
    clear_error();
    if (!b) return set_error(MAGIS_E_INVAL, "base is NULL");
    if (K < 0) return set_error(MAGIS_E_INVAL, "K < 0");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_wstart || !d_wlen || !d_wperm || !d_status || !d_peak || !d_latency)
        return set_error(MAGIS_E_INVAL, "null device pointer");
    if (wmax < 1) return set_error(MAGIS_E_INVAL, "wmax < 1");
    if (wmax > window_wmax_supported()) return set_error(MAGIS_E_UNSUPPORTED, "wmax > 64");
    DeviceGuard guard(b->g->device);
    cudaError_t e = window_launch(b->g->dev, b->dev, b->grid, b->endb_ws, K, d_wstart, d_wlen, d_wperm, wmax,
                                  d_status, d_peak, d_latency, (cudaStream_t)cuda_stream);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("window launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}

extern "C" int64_t magis_pareto_workspace_size(int64_t n) {
    return n < 0 ? 0 : pareto_workspace_size(n);
}

extern "C" int magis_pareto_merge(int64_t n, const int64_t* d_peak, const double* d_lat,
                                  const uint8_t* d_status, const int64_t* d_id, int64_t id_base,
                                  int64_t cap, int64_t* d_front_id, int64_t* d_front_peak,
                                  double* d_front_lat, int64_t* d_front_n, int64_t mem_limit,
                                  double lat_limit, int64_t* d_best, void* d_workspace,
                                  int64_t workspace_bytes, void* cuda_stream) {
    clear_error();
    if (n < 0 || cap < 0) return set_error(MAGIS_E_INVAL, "n < 0 or cap < 0");
    if (!d_front_n) return set_error(MAGIS_E_INVAL, "d_front_n is NULL");
    if (n > 0 && (!d_peak || !d_lat))
        return set_error(MAGIS_E_INVAL, "null input pointer");
    if (cap > 0 && (!d_front_id || !d_front_peak || !d_front_lat))
        return set_error(MAGIS_E_INVAL, "null front pointer");
    if (workspace_bytes < pareto_workspace_size(n) || (n > 0 && !d_workspace))
        return set_error(MAGIS_E_CAPACITY, "workspace smaller than magis_pareto_workspace_size(n)");
    cudaError_t e = pareto_launch(n, d_peak, d_lat, d_status, d_id, id_base, cap, d_front_id,
                                  d_front_peak, d_front_lat, d_front_n, mem_limit, lat_limit,
                                  d_best, d_workspace, (cudaStream_t)cuda_stream);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return set_error(MAGIS_E_CUDA, std::string("pareto launch: ") + cudaGetErrorString(e));
    }
    return MAGIS_SUCCESS;
}
