// magis_plan.cu -- host-side planner of the variant-2 kernel (magis_eval2.cu).
//
// Turns the gated super-graph into warp-aligned "rows" held in shared memory:
//  * a consumer row = 32 nodes (one per lane) of similar out-degree: a header
//    (node id + kind) and deg edge entries stored lane-major, so every read is
//    a conflict-free LDS and all lanes of a warp step through headers and
//    edges in lock-step (no divergence); a late-user edge t_r -> b (active iff
//    dec[r] == 0, reading P6) is redirected to the virtual slot NT + j
//    (j = position of b in U) that the kernel fills per candidate;
//  * an input row = 32 nodes of similar in-degree with their inputs (every
//    gate: inactive ones never match, see magis_eval2.cu) plus the node's size
//    units and compute cost;
//  * rows are dealt longest-first onto the least loaded warp;
//  * tensor sizes are stored in units of their gcd (u32), which keeps the
//    scan exact (reading P14: sizes are multiples of the allocation grain).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <queue>

#include "magis_internal.h"

namespace magis {

namespace {
constexpr uint32_t kKindShift = 29;
// kHdrGated: an original node inside an F-Trans region (present iff its variant is chosen)
constexpr uint32_t kEdge = 0, kHdr = 1, kHdrOut = 2, kHdrClone = 3, kHdrCopy = 4, kHdrGated = 5, kNop = 7;

uint64_t gcd64(uint64_t a, uint64_t b) {
    while (b) { uint64_t t = a % b; a = b; b = t; }
    return a;
}
size_t a16(size_t x) { return (x + 15) / 16 * 16; }

struct Rows {
    std::vector<uint32_t> row;   // (offset, degree) pairs
    std::vector<uint32_t> hdr;   // [nrows * 32]
    std::vector<uint16_t> ent;   // edge entries (node ids), lane-major per row
    std::vector<int32_t> node;   // [nrows * 32] node id or -1
    std::vector<uint32_t> wtab;  // per warp [begin, end) rows
};

// Group nodes into rows of 32 by descending degree, deal rows onto warps.
Rows make_rows(const std::vector<std::vector<uint32_t>>& lists, const std::vector<uint32_t>& hdrs,
               uint16_t nop_entry, uint32_t nop_hdr, int WM) {
    const int32_t N = (int32_t)lists.size();
    std::vector<int32_t> order(N);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(),
                     [&](int32_t a, int32_t b) { return lists[a].size() > lists[b].size(); });
    const int32_t nrows = (N + 31) / 32;
    std::vector<uint32_t> deg(nrows, 0);
    for (int32_t r = 0; r < nrows; r++)
        for (int l = 0; l < 32 && r * 32 + l < N; l++)
            deg[r] = std::max<uint32_t>(deg[r], (uint32_t)lists[order[r * 32 + l]].size());
    // deal rows onto warps (longest first, least loaded)
    std::vector<std::vector<int32_t>> wr(WM);
    {
        using It = std::pair<uint64_t, int>;
        std::priority_queue<It, std::vector<It>, std::greater<It>> q;
        for (int w = 0; w < WM; w++) q.push({0, w});
        for (int32_t r = 0; r < nrows; r++) {   // rows already in descending degree
            It it = q.top();
            q.pop();
            wr[it.second].push_back(r);
            it.first += 1 + deg[r];
            q.push(it);
        }
    }
    Rows out;
    out.wtab.resize(WM * 2);
    for (int w = 0; w < WM; w++) {
        out.wtab[2 * w] = (uint32_t)(out.row.size() / 2);
        for (int32_t r : wr[w]) {
            const uint32_t off = (uint32_t)out.ent.size();
            out.row.push_back(off);
            out.row.push_back(deg[r]);
            out.ent.resize(off + (size_t)deg[r] * 32, nop_entry);
            for (int l = 0; l < 32; l++) {
                const int32_t i = r * 32 + l;
                if (i < N) {
                    const int32_t v = order[i];
                    out.hdr.push_back(hdrs[v]);
                    out.node.push_back(v);
                    for (size_t j = 0; j < lists[v].size(); j++)
                        out.ent[off + j * 32 + l] = (uint16_t)(lists[v][j] & 0xffffu);
                } else {
                    out.hdr.push_back(nop_hdr);
                    out.node.push_back(-1);
                }
            }
        }
        out.wtab[2 * w + 1] = (uint32_t)(out.row.size() / 2);
    }
    return out;
}
}  // namespace

bool plan2_build(const SuperGraphHost& sg, int P, int teams, bool gmem_static, bool gmem_af, bool delta_slots,
                 size_t smem_cap,
                 Plan2* pl, std::vector<char>* img, int row_groups) {
    const int32_t NT = sg.NT, n = sg.n, R = sg.R;
    const int32_t nU = R > 0 ? sg.U_ptr[R] : 0;
    const int64_t NTX = (int64_t)NT + nU + 1;
    if (NTX >= 65535 || NT < 1 || R >= 65535) return false;   // u16 positions (stored +1), u16 tensor ids
    // size units
    uint64_t gg = 0;
    for (int32_t v = 0; v < NT; v++) if (sg.size[v] > 0) gg = gcd64(gg, (uint64_t)sg.size[v]);
    if (gg == 0) gg = 1;
    for (int32_t v = 0; v < NT; v++) {
        uint64_t s = (uint64_t)sg.size[v] / gg;
        for (int32_t e = sg.in_ptr[v]; e < sg.in_ptr[v + 1]; e++) s += (uint64_t)sg.size[sg.in_ent[e].x] / gg;
        if (s > 0xffffffffull) return false;
        if (delta_slots && s > 0x7fffffffull) return false;  // tier 2: signed per-step deltas (int32)
    }
    auto virt = [&](int32_t r, int32_t b) -> int32_t {
        for (int32_t j = sg.U_ptr[r]; j < sg.U_ptr[r + 1]; j++)
            if (sg.U_idx[j] == b) return NT + j;
        return -1;
    };
    std::vector<std::vector<uint32_t>> cons(NT), ins(NT);
    std::vector<uint32_t> hdrs(NT);
    // F-Trans regions (reading F1): every node of every variant is listed; the
    // kernel zeroes the positions of the nodes of unchosen variants per
    // candidate, so edges need no gates (an edge exists iff both ends do)
    const int32_t F = sg.F;
    std::vector<uint32_t> rn;
    int32_t gate_lo = n;
    for (int32_t v = 0; v < n && F > 0; v++) {
        const int32_t gt = sg.ngate[v];
        if (gt < 0) continue;
        const int32_t reg = (gt >> 2) - R, var = gt & 3;
        if (reg < 0 || reg >= F || reg >= (1 << 14) || (sg.nflag[v] & kFlagOutput)) return false;
        rn.push_back((uint32_t)v | ((uint32_t)reg << 16) | ((uint32_t)var << 30));
        gate_lo = std::min(gate_lo, v);
    }
    for (int32_t u = 0; u < NT; u++) {
        uint32_t kind;
        if (u < n) kind = (sg.nflag[u] & kFlagOutput) ? kHdrOut : (F > 0 && sg.ngate[u] >= 0) ? kHdrGated : kHdr;
        else kind = ((u - n) % 3 == 0) ? kHdrClone : kHdrCopy;
        hdrs[u] = (kind << kKindShift) | (uint32_t)u;
        for (int32_t e = sg.cons_ptr[u]; e < sg.cons_ptr[u + 1]; e++) {
            const int2 ce = sg.cons_ent[e];
            int32_t c = ce.x;
            if (ce.y >= 0 && (ce.y >> 2) < R && (ce.y & 3) == 0) {   // t_r -> b, b in U_r (region gates have r >= R)
                c = virt(ce.y >> 2, ce.x);
                if (c < 0) return false;
            }
            cons[u].push_back((kEdge << kKindShift) | (uint32_t)c);
        }
        for (int32_t e = sg.in_ptr[u]; e < sg.in_ptr[u + 1]; e++)
            ins[u].push_back((kEdge << kKindShift) | (uint32_t)sg.in_ent[e].x);
    }
    // teams: independent groups of warps in one CTA, each scoring its own
    // candidates with its own per-group state and barriers (the graph tables
    // are shared); main threads per team = kMainThreads2 / teams
    if (teams != 1 && teams != 2) return false;
    const int TMt = kMainThreads2 / teams;
    const int WM = TMt / 32;
    if (WM % P != 0 || kMainThreads2 + teams * 32 * P > 1024) return false;   // whole warps per candidate
    const uint32_t dummy = (uint32_t)(NTX - 1);
    const uint16_t nop = (uint16_t)dummy;
    const uint32_t nophdr = (kNop << kKindShift) | dummy;
    // row_groups > 1 (kernel B): rows dealt onto row_groups x WM warps, the
    // warps of CTA r of a cluster take [r WM, (r + 1) WM)
    const int WMr = WM * row_groups;
    Rows cr = make_rows(cons, hdrs, nop, nophdr, WMr);
    // input rows only where the frees are gathered (slots in global memory);
    // with the slots in shared memory phase 3 scatters the frees instead
    Rows fr;
    if (gmem_af) fr = make_rows(ins, hdrs, nop, nophdr, WMr);
    std::vector<uint32_t> wtab(WMr * 4, 0);
    for (int w = 0; w < WMr; w++) {
        wtab[4 * w + 0] = cr.wtab[2 * w];
        wtab[4 * w + 1] = cr.wtab[2 * w + 1];
        if (gmem_af) {
            wtab[4 * w + 2] = fr.wtab[2 * w];
            wtab[4 * w + 3] = fr.wtab[2 * w + 1];
        }
    }
    std::vector<uint32_t> size_u(NTX, 0);
    std::vector<double> cost_u(NTX, 0.0);
    for (int32_t v = 0; v < NT; v++) {
        size_u[v] = (uint32_t)((uint64_t)sg.size[v] / gg);
        cost_u[v] = (sg.nflag[v] & kFlagCompute) ? sg.cost[v] : 0.0;
    }

    Plan2 p{};
    p.P = P;
    p.NT = NT;
    p.NTX = (int32_t)NTX;
    p.n = n;
    p.R = R;
    p.nU = nU;
    {
        // scan chunk: the fewest steps per thread, a multiple of 4 (int4 perm
        // loads, odd padded slot stride); the kernel divides by L with a magic
        const int32_t tpc = TMt / P;                    // threads per candidate in the scan
        const int32_t Lmin = std::max(4, (NT + tpc - 1) / tpc);
        p.L = (Lmin + 3) & ~3;
        if (p.L > 64) return false;                     // LMAX <= 64 steps per thread
        p.Lm = (uint32_t)((((uint64_t)1 << 32) + (uint64_t)p.L - 1) / (uint64_t)p.L);
        p.S = (NT + p.L - 1) / p.L;
    }
    p.unit = (int64_t)gg;
    p.max_events = 3 * R + nU;
    size_t o = 0;
    p.off_wtab = (uint32_t)o;  o = a16(o + wtab.size() * 4);
    p.off_crow = (uint32_t)o;  o = a16(o + cr.row.size() * 4);
    p.off_chdr = (uint32_t)o;  o = a16(o + cr.hdr.size() * 4);
    p.off_cent = (uint32_t)o;  o = a16(o + cr.ent.size() * 2);
    // [wtab, crow, chdr, cent] contiguous: the row tables tier 1 may stage
    p.off_csize = (uint32_t)o; o = a16(o + cr.hdr.size() * 4);   // size units of each header, row order
    p.off_frow = (uint32_t)o;  o = a16(o + fr.row.size() * 4);
    p.off_fhdr = (uint32_t)o;  o = a16(o + fr.hdr.size() * 4);
    p.off_fent = (uint32_t)o;  o = a16(o + fr.ent.size() * 2);
    p.off_size = (uint32_t)o;  o = a16(o + size_u.size() * 4);
    p.off_cost = (uint32_t)o;  o = a16(o + cost_u.size() * 8);
    p.off_rtab = (uint32_t)o;  o = a16(o + (size_t)std::max(R, 1) * 16);
    p.off_ninfo = (uint32_t)o; o = a16(o + (size_t)n * 8);
    p.off_lul = (uint32_t)o;   o = a16(o + (size_t)std::max(nU, 1) * 2);
    p.off_urow = (uint32_t)o;  o = a16(o + (size_t)std::max(R, 1) * 4);
    p.off_ubs = (uint32_t)o;   o = a16(o + (size_t)std::max(nU, 1) * 2);
    p.off_utr = (uint32_t)o;   o = a16(o + (size_t)std::max(R, 1) * 2);
    p.F = F;
    p.Rd = R + F;
    p.nRN = (int32_t)rn.size();
    p.gate_lo = gate_lo;
    p.off_rn = (uint32_t)o;    o = a16(o + std::max<size_t>(rn.size(), 1) * 4);
    p.off_nvar = (uint32_t)o;  o = a16(o + (size_t)std::max(F, 1));
    p.off_vcost = (uint32_t)o; o = a16(o + (size_t)4 * std::max(F, 1) * 8);
    p.static_bytes = (uint32_t)o;
    // tier 2: the cost table as class indices (the graphs' costs take few
    // distinct values: C4 200 of 23,562) so the swap scan's cost gather is a
    // shared-memory lookup instead of an L2 round trip
    std::vector<double> cvals(cost_u.begin(), cost_u.end());
    std::sort(cvals.begin(), cvals.end());
    cvals.erase(std::unique(cvals.begin(), cvals.end()), cvals.end());
    const bool have_cls = cvals.size() <= 256;
    p.off_ccls = (uint32_t)o;
    p.ccls_idx_off = (uint32_t)a16(cvals.size() * 8);
    if (have_cls) o = a16(o + p.ccls_idx_off + (size_t)NTX);
    p.image_bytes = (uint32_t)o;
    // graph tables in shared memory (staged) or read from the global image
    // (L1/L2; the row reads stay coalesced); per-step slots in shared memory or
    // in a per-CTA global slice
    p.gmem_static = gmem_static ? 1 : 0;
    p.gmem_af = gmem_af ? 1 : 0;
    p.delta_slots = (delta_slots && !gmem_af) ? 1 : 0;
    if (p.delta_slots && !gmem_static) return false;      // MODE 3 reads the tables from the global image
    const size_t Sl = ((size_t)(p.L + 1) * p.S + 3) & ~(size_t)3;   // padded per-candidate slots (magis_eval2.cu)
    p.af_bytes = (uint64_t)((P * Sl * 8 + 255) / 256 * 256);
    const size_t static_end = o;
    // tables read from the global image: the cost table (the swap scan's
    // random gather) is still staged into shared memory when it fits with
    // at least 32 event slots per candidate.  Tier 1 first tries to stage the
    // consumer-row tables too ([wtab, crow, chdr, cent]; the row sizes stay in
    // global memory, loaded a row ahead), with the cost table as u8 classes to
    // make room: the row pass then gathers from shared memory only (rows_sm).
    struct Att { int rs, csm; };
    Att atts[3];
    int na = 0;
    const char* nors = std::getenv("MAGIS_NO_ROWSM");
    if (gmem_static) {
        if (!delta_slots && !gmem_af && have_cls && !(nors && std::atoi(nors) != 0)) atts[na++] = {1, 1};
        atts[na++] = {0, 1};
        atts[na++] = {0, 0};
    } else {
        atts[na++] = {0, 0};
    }
    bool planned = false;
    for (int ai = 0; ai < na; ai++) {
    const int csm = atts[ai].csm;
    p.rows_sm = atts[ai].rs;
    p.cost_cls = (have_cls && (delta_slots || p.rows_sm)) ? 1 : 0;   // tier 1 without rows_sm: f64 (classes +2.6%, A/B)
    p.stage_bytes = (uint32_t)(p.cost_cls ? a16(p.ccls_idx_off + (size_t)NTX) : a16((size_t)NTX * 8));
    p.rows_off = p.stage_bytes;
    p.rows_bytes = p.rows_sm ? (uint32_t)(p.off_csize - p.off_wtab) : 0u;
    o = gmem_static ? (csm ? (size_t)p.stage_bytes + p.rows_bytes : 0) : static_end;
    p.cost_sm = csm;
    p.state_base = (uint32_t)o;
    // pos: NTX slots + one trash slot (out-of-range ids of a bad permutation
    // are written there); last: only where phase 4 gathers the frees
    p.off_pos = (uint32_t)o;  o = a16(o + (size_t)(NTX + 1) * P * 2);
    p.off_last = (uint32_t)o; o = a16(o + (gmem_af ? (size_t)NTX * P * 2 : 0));
    p.off_af = (uint32_t)o;   o = a16(o + (gmem_af ? 0 : (size_t)P * Sl * (p.delta_slots ? 4 : 8)));   // tier 2: int32 delta
    p.off_dec = (uint32_t)o;  o = a16(o + (size_t)P * std::max(R + F, 1));
    p.off_end = (uint32_t)o;  o = a16(o + (size_t)P * 3 * std::max(R, 1) * 8);
    p.nwm = (NT + 31) / 32 + 3;                         // mark_bits reads up to 2 words past a chunk start
    p.off_evm = (uint32_t)o;  o = a16(o + (size_t)P * p.nwm * 4);
    p.off_sdec = (uint32_t)o; o = a16(o + (size_t)2 * P * ((std::max(R + F, 1) + 15) & ~15));
    p.off_ev = (uint32_t)o;
    // event steps of a candidate: at most the marked steps (<= 3R + |U|)
    int cap = std::min(std::max(p.max_events, 1), 128);
    p.teams = teams;
    bool fit = false;
    while (true) {
        const size_t st = a16(o + (size_t)2 * P * cap * 24) - p.state_base;     // one team's state
        const size_t need = p.state_base + (size_t)teams * st;
        if (need <= smem_cap) {
            p.smem_total = (uint32_t)a16(need);
            p.state_stride = (uint32_t)st;
            fit = true;
            break;
        }
        if (cap <= (csm ? 32 : 8)) break;
        cap /= 2;
    }
    if (!fit) continue;
    p.evcap = cap;
    planned = true;
    break;
    }
    if (!planned) return false;
    p.ovf_stride = (uint64_t)((std::max(p.max_events, 1) * 24 + 255) / 256 * 256);
    *pl = p;
    img->assign(p.image_bytes, 0);
    auto put = [&](uint32_t off, const void* src, size_t bytes) {
        if (bytes) std::memcpy(img->data() + off, src, bytes);
    };
    put(p.off_wtab, wtab.data(), wtab.size() * 4);
    put(p.off_crow, cr.row.data(), cr.row.size() * 4);
    put(p.off_chdr, cr.hdr.data(), cr.hdr.size() * 4);
    {
        std::vector<uint32_t> cs(cr.hdr.size(), 0);
        for (size_t i = 0; i < cr.node.size(); i++)
            if (cr.node[i] >= 0) cs[i] = size_u[cr.node[i]];
        put(p.off_csize, cs.data(), cs.size() * 4);
    }
    put(p.off_cent, cr.ent.data(), cr.ent.size() * 2);
    put(p.off_frow, fr.row.data(), fr.row.size() * 4);
    put(p.off_fhdr, fr.hdr.data(), fr.hdr.size() * 4);
    put(p.off_fent, fr.ent.data(), fr.ent.size() * 2);
    put(p.off_size, size_u.data(), size_u.size() * 4);
    put(p.off_cost, cost_u.data(), cost_u.size() * 8);
    if (have_cls) {
        put(p.off_ccls, cvals.data(), cvals.size() * 8);
        std::vector<uint8_t> ci(NTX);
        for (int64_t v = 0; v < NTX; v++)
            ci[v] = (uint8_t)(std::lower_bound(cvals.begin(), cvals.end(), cost_u[v]) - cvals.begin());
        put(p.off_ccls + p.ccls_idx_off, ci.data(), (size_t)NTX);
    }
    put(p.off_rtab, sg.rtab, (size_t)R * 16);
    // per original node: the tensor it produces (if eligible) and the eligible
    // tensors it is a late user of -- the swap events it can raise (reading P7)
    {
        std::vector<std::vector<uint16_t>> lu(n);
        for (int32_t r = 0; r < R; r++)
            for (int32_t j = sg.U_ptr[r]; j < sg.U_ptr[r + 1]; j++) lu[sg.U_idx[j]].push_back((uint16_t)r);
        std::vector<uint32_t> ninfo((size_t)2 * n, 0);
        std::vector<uint16_t> lul;
        for (int32_t v = 0; v < n; v++) {
            if (lu[v].size() > 31) return false;       // swapped-late-user mask of the event steps
            ninfo[2 * v] = (uint32_t)lu[v].size() << 16;
            ninfo[2 * v + 1] = (uint32_t)lul.size();
            lul.insert(lul.end(), lu[v].begin(), lu[v].end());
        }
        for (int32_t r = 0; r < R; r++) ninfo[2 * sg.elig[r]] |= (uint32_t)(r + 1);
        put(p.off_ninfo, ninfo.data(), ninfo.size() * 4);
        put(p.off_lul, lul.data(), lul.size() * 2);
        std::vector<uint32_t> urow(std::max(R, 1), 0);
        std::vector<uint16_t> ubs(std::max(nU, 1), 0), utr(std::max(R, 1), 0);
        for (int32_t r = 0; r < R; r++) {
            const int32_t u0 = sg.U_ptr[r], cnt = sg.U_ptr[r + 1] - u0;
            if (cnt > 0xffff) return false;
            urow[r] = (uint32_t)u0 | ((uint32_t)cnt << 16);
            utr[r] = (uint16_t)sg.elig[r];
            for (int32_t j = u0; j < u0 + cnt; j++) ubs[j] = (uint16_t)sg.U_idx[j];
        }
        put(p.off_rn, rn.data(), rn.size() * 4);
    if (F > 0) {
        std::vector<uint8_t> nv(F);
        for (int32_t i = 0; i < F; i++) nv[i] = (uint8_t)sg.nvar[i];
        put(p.off_nvar, nv.data(), (size_t)F);
        put(p.off_vcost, sg.vcost, (size_t)4 * F * 8);
    }
    put(p.off_urow, urow.data(), (size_t)R * 4);
        put(p.off_ubs, ubs.data(), (size_t)nU * 2);
        put(p.off_utr, utr.data(), (size_t)R * 2);
    }
    return true;
}

}  // namespace magis
