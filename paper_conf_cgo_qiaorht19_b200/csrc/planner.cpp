// planner.cpp -- the fusion planner of Qiao et al. (CGO'19), host side.
//
//   edge weights   Eqs. 3-12, scenario per edge
//   IsLegal        dependence (Fig. 2), resources (Eq. 2,
//                  PAPER.md:296-321), header, profitability
//
//   MinCut         Stoer-Wagner [14] on the undirected view
//   Alg. 1         GetLegalPartitions
//
// Readings of the garbled/silent passages are listed in DESIGN.md §3 (R-1..R-9).
// Weights are lexicographic pairs (q, eps): q = floor(w * 2^20 + 0.5) in
// fixed point so that sums and ties are exact (R-9), eps counts the
// "arbitrarily small positive" weights of illegal edges.
#include <algorithm>
#include <cmath>
#include <deque>
#include <functional>

#include "kf_internal.h"

namespace kf {

namespace {

struct W2 {
    int64_t q = 0, e = 0;
    W2 operator+(const W2 &o) const { return {q + o.q, e + o.e}; }
    bool operator<(const W2 &o) const { return q != o.q ? q < o.q : e < o.e; }
};

int64_t quantize(double w) { return (int64_t)std::floor(w * 1048576.0 + 0.5); }

double f_mshared(const kf_pipeline *p, int k, const kf_model_params &m)
{
    const Op &o = p->ops[k];
    if (o.kind != LOCAL) return 0.0;
    return (double)((int64_t)(m.tile_w + 2 * o.rx()) * (m.tile_h + 2 * o.ry()) * 4);
}

}  // namespace

// Fig. 2 reading (R-1): exactly one sink kd; every other kernel has
// all its consumers inside and is not a pipeline output (2c); every image a
// non-source kernel reads from outside is also read by a source kernel (2b vs 2d).
bool dependence_legal(const kf_pipeline *p, const std::set<int> &P)
{
    auto co = consumers(p);
    auto pr = producers(p);
    int sink = -1, nsink = 0;
    for (int k : P) {
        bool inner = false;
        for (int c : co[k]) inner |= P.count(c) > 0;
        if (!inner) { sink = k; nsink++; }
    }
    if (nsink != 1) return false;
    std::set<int> outs(p->outputs.begin(), p->outputs.end());
    for (int k : P) {
        if (k == sink) continue;
        if (outs.count(p->n_inputs + k)) return false;
        for (int c : co[k])
            if (!P.count(c)) return false;
    }
    std::set<int> src_reads;
    std::set<int> sources;
    for (int k : P) {
        bool has_prod = false;
        for (int s : pr[k]) has_prod |= P.count(s) > 0;
        if (!has_prod) {
            sources.insert(k);
            for (int img : p->ops[k].inputs) src_reads.insert(img);
        }
    }
    for (int k : P) {
        if (sources.count(k)) continue;
        for (int img : p->ops[k].inputs) {
            bool inside = img >= p->n_inputs && P.count(img - p->n_inputs);
            if (!inside && !src_reads.count(img)) return false;
        }
    }
    return true;
}

// Eq. 2 with fMshared(vP) = sum of the block's local kernels' staged tiles (R-2).
static bool resource_legal(const kf_pipeline *p, const std::set<int> &P, const kf_model_params &m)
{
    double s = 0.0, mx = 0.0;
    bool any = false;
    for (int k : P) {               // std::set iterates ascending, as the reference does
        if (p->ops[k].kind != LOCAL) continue;
        any = true;
        s += f_mshared(p, k, m);
        mx = std::max(mx, f_mshared(p, k, m));
    }
    if (!any) return true;
    return s / mx <= m.c_mshared;
}

// Header compatibility: one iteration space per pipeline is
// enforced at creation; access-granularity reading R-8: the local kernels of a
// fused block all use REPEAT or none does.
bool header_legal(const kf_pipeline *p, const std::set<int> &P)
{
    int rep = 0, loc = 0;
    for (int k : P)
        if (p->ops[k].kind == LOCAL) {
            loc++;
            rep += p->ops[k].mode == KF_REPEAT;
        }
    return rep == 0 || rep == loc;
}

static bool context_legal(const kf_pipeline *p, const std::set<int> &P, const kf_model_params &m)
{
    return dependence_legal(p, P) && resource_legal(p, P, m) && header_legal(p, P);
}

// ROOFLINE reading (phi_mode 2, R-20): SM-cycles per pixel of the
// kernel set {ks} or {ks, kd} run as one kernel -- the larger of its DRAM
// time (bpp bytes per distinct external image and per output) and its issue
// time (Eq. 6 costs as issue slots, the producer recomputed on the staged halo).
static double roof_time(const kf_pipeline *p, int ks, int kd, const kf_model_params &m)
{
    const double ch = p->dtype == KF_U8X4 ? 2.0 : 1.0;
    auto issue = [&](int k) {
        const Op &o = p->ops[k];
        double n = 0.0;
        for (const Instr &in : o.prog) n += op_issue_slots(in.op);
        if (o.kind == LOCAL)
            for (double v : o.mask) n += v != 0.0;
        return n * ch;
    };
    std::set<int> ext(p->ops[ks].inputs.begin(), p->ops[ks].inputs.end());
    double slots = issue(ks);
    if (kd >= 0) {
        const Op &d = p->ops[kd];
        for (int i : d.inputs)
            if (i != p->n_inputs + ks) ext.insert(i);
        const double r = d.kind == LOCAL ? ((double)(m.tile_w + 2 * d.rx()) * (double)(m.tile_h + 2 * d.ry())) /
                                                   ((double)m.tile_w * (double)m.tile_h)
                                         : 1.0;
        slots = issue(ks) * r + issue(kd);
    }
    const double mem = 4.0 * (double)(ext.size() + 1) / m.bw_bytes_clk;
    const double iss = slots / m.issue_lanes_clk;
    return std::max(mem, iss) + m.overlap * std::min(mem, iss);
}

// Benefit of one edge, Eqs. 3-11 plus gamma (Eq. 12 before clamping).
static EdgeInfo benefit(const kf_pipeline *p, int ks, int kd, const kf_model_params &m)
{
    const Op &s = p->ops[ks], &d = p->ops[kd];
    const double IS = 1.0;                                    // R-5
    const double costop = m.c_alu * s.n_alu + m.c_sfu * s.n_sfu;   // Eq. 6
    const double is_ks = (double)s.inputs.size();
    EdgeInfo e{};
    e.ks = ks;
    e.kd = kd;
    if (m.phi_mode == 2) {                                    // ROOFLINE (R-20)
        e.scenario = d.kind == POINT ? 0 : s.kind == POINT ? 1 : 2;
        e.w = roof_time(p, ks, -1, m) + roof_time(p, kd, -1, m) - roof_time(p, ks, kd, m) + m.gamma;
        return e;
    }
    if (d.kind == POINT) {                                    // point-based, Eqs. 4-5
        e.scenario = 0;
        e.w = IS * m.tg + m.gamma;
        return e;
    }
    double fac;
    if (m.phi_mode == 1)                                      // STAGED (R-4)
        fac = ((double)(m.tile_w + 2 * d.rx()) * (double)(m.tile_h + 2 * d.ry())) /
              ((double)m.tile_w * (double)m.tile_h);   // in double: large tiles must not overflow int
    else if (s.kind == POINT)
        fac = (double)((2 * d.rx() + 1) * (2 * d.ry() + 1)); // sz(kd), Eq. 7
    else
        fac = (double)((2 * d.rx() + 1 + 2 * s.rx()) * (2 * d.ry() + 1 + 2 * s.ry()));  // Eq. 9 (R-6)
    const double phi = costop * is_ks * fac;                  // Eqs. 7 / 10
    if (s.kind == POINT) {
        e.scenario = 1;
        e.w = IS * m.tg - phi + m.gamma;                      // Eq. 8
    } else {
        e.scenario = 2;
        double dsh = m.eq3_mode == 0 ? IS * m.tg / m.ts : IS * (m.tg - m.ts);   // Eq. 3 (R-7)
        e.w = dsh - phi + m.gamma;                            // Eq. 11
    }
    return e;
}

static std::vector<EdgeInfo> edge_weights(const kf_pipeline *p, const kf_model_params &m)
{
    std::vector<EdgeInfo> out;
    auto pr = producers(p);
    for (int kd = 0; kd < (int)p->ops.size(); kd++)
        for (int ks : pr[kd]) {
            EdgeInfo e = benefit(p, ks, kd, m);
            e.profitable = e.w > 0.0;
            e.ctx_legal = context_legal(p, {ks, kd}, m);
            if (e.profitable && e.ctx_legal) { e.q = quantize(e.w); e.eps = 0; }
            else { e.q = 0; e.eps = 1; }                      // w_e = eps (Eq. 12)
            out.push_back(e);
        }
    return out;
}

static bool is_legal(const kf_pipeline *p, const std::set<int> &P, const kf_model_params &m,
                     const std::vector<EdgeInfo> &E)
{
    if (P.size() == 1) return true;
    for (const EdgeInfo &e : E)
        if (P.count(e.ks) && P.count(e.kd) && !e.profitable) return false;   // R-3
    return context_legal(p, P, m);
}

// Stoer-Wagner global minimum cut with the deterministic tie-breaks of R-9:
// start vertex = first active vertex in declaration order, most tightly
// connected next (ties: lowest declaration index), merged vertex keeps s's
// slot, keep the first minimum encountered (strict <).
static CutInfo stoer_wagner(const std::vector<int> &verts, const std::vector<EdgeInfo> &E)
{
    const int n = (int)verts.size();
    std::map<int, int> idx;
    for (int i = 0; i < n; i++) idx[verts[i]] = i;
    std::vector<std::vector<W2>> Wm(n, std::vector<W2>(n));
    for (const EdgeInfo &e : E) {
        auto a = idx.find(e.ks), b = idx.find(e.kd);
        if (a == idx.end() || b == idx.end()) continue;
        W2 w{e.q, e.eps};
        Wm[a->second][b->second] = Wm[a->second][b->second] + w;
        Wm[b->second][a->second] = Wm[b->second][a->second] + w;
    }
    std::vector<std::vector<int>> groups(n);
    for (int i = 0; i < n; i++) groups[i] = {verts[i]};
    std::vector<int> active(n);
    for (int i = 0; i < n; i++) active[i] = i;
    bool have = false;
    W2 best;
    std::vector<int> best_group;
    int phases = 0;
    while (active.size() > 1) {
        phases++;
        std::vector<int> A{active[0]};
        std::vector<int> rest(active.begin() + 1, active.end());   // ascending positions
        std::vector<W2> conn(n);
        for (int v : rest) conn[v] = Wm[active[0]][v];
        W2 last;
        while (!rest.empty()) {
            size_t bi = 0;
            for (size_t i = 1; i < rest.size(); i++)
                if (conn[rest[bi]] < conn[rest[i]]) bi = i;      // strictly larger wins; ties keep lowest
            int v = rest[bi];
            last = conn[v];
            rest.erase(rest.begin() + bi);
            A.push_back(v);
            for (int u : rest) conn[u] = conn[u] + Wm[v][u];
        }
        int s = A[A.size() - 2], t = A.back();
        if (!have || last < best) {
            have = true;
            best = last;
            best_group = groups[t];
        }
        groups[s].insert(groups[s].end(), groups[t].begin(), groups[t].end());
        for (int u = 0; u < n; u++) {
            Wm[s][u] = Wm[s][u] + Wm[t][u];
            Wm[u][s] = Wm[u][s] + Wm[u][t];
        }
        Wm[s][s] = W2{};
        active.erase(std::find(active.begin(), active.end(), t));
    }
    std::sort(best_group.begin(), best_group.end());
    return CutInfo{best_group, best.q, best.e, phases};
}

static void finish_plan(kf_pipeline *p, kf_plan *plan)
{
    for (auto &b : plan->blocks) std::sort(b.begin(), b.end());
    std::sort(plan->blocks.begin(), plan->blocks.end(),
              [](const std::vector<int> &a, const std::vector<int> &b) { return a.back() < b.back(); });
    plan->beta_q = plan->beta_eps = 0;
    for (auto &b : plan->blocks) {
        std::set<int> S(b.begin(), b.end());
        for (const EdgeInfo &e : plan->edges)
            if (S.count(e.ks) && S.count(e.kd)) { plan->beta_q += e.q; plan->beta_eps += e.eps; }
    }
    for (auto &b : plan->blocks) plan->info.push_back(analyse_block(p, b));
    // band halo: max accumulated vertical radius from an input to an output
    std::vector<int> dist(p->n_images(), -1);
    for (int o : p->outputs) dist[o] = 0;
    for (int k = (int)p->ops.size() - 1; k >= 0; k--) {
        int d = dist[p->n_inputs + k];
        if (d < 0) d = 0;                // dead kernels still run
        for (int img : p->ops[k].inputs) dist[img] = std::max(dist[img], d + p->ops[k].ry());
    }
    plan->halo_rows = 0;
    for (int i = 0; i < p->n_inputs; i++) plan->halo_rows = std::max(plan->halo_rows, dist[i]);
    plan->pipe = p;
    p->frozen = true;
}

kf_plan *plan_fusion(kf_pipeline *p, const kf_model_params &m)
{
    if (p->ops.empty()) fail(KF_ERR_ARG, "pipeline has no kernels");
    if (!(m.ts > 0) || m.tile_w <= 0 || m.tile_h <= 0 || !(m.c_mshared > 0))
        fail(KF_ERR_ARG, "invalid model parameters");
    auto plan = std::make_unique<kf_plan>();
    plan->edges = edge_weights(p, m);                         // Alg. 1 lines 2-4
    std::deque<std::vector<int>> Sp;                          // line 6
    std::vector<int> all(p->ops.size());
    for (size_t i = 0; i < all.size(); i++) all[i] = (int)i;
    Sp.push_back(all);
    while (!Sp.empty()) {                                     // lines 7-17
        std::vector<int> blk = Sp.front();
        Sp.pop_front();
        std::set<int> S(blk.begin(), blk.end());
        if (blk.size() == 1 || is_legal(p, S, m, plan->edges)) {
            plan->blocks.push_back(blk);                      // line 10
        } else {
            CutInfo c = stoer_wagner(blk, plan->edges);       // line 13
            std::vector<int> other;
            std::set<int> side(c.side.begin(), c.side.end());
            for (int k : blk)
                if (!side.count(k)) other.push_back(k);
            plan->cuts.push_back(c);
            Sp.push_back(c.side);
            Sp.push_back(other);
        }
    }
    finish_plan(p, plan.get());
    return plan.release();
}

// ---------------------------------------------------------------------------
// §8(f)3 -- the "basic" fusion of the authors' previous work [12], the paper's
// comparison column: only point-to-point,
// local-to-point and point-to-local fusion; a shared input (Fig. 2b) is
// treated as an external dependence and rejected.  Reading R-18:
// a block is basic-legal iff it is legal for Alg. 1 (dependence, resources,
// header, profitability) AND it has exactly one source kernel, no kernel but
// that source reads an image from outside the block, and no local kernel has
// a local kernel upstream inside the block (that would be local-to-local).
// [12] fuses pair-wise: edges are visited by decreasing benefit (ties: lower
// producer, then lower consumer) and the two blocks an edge joins are merged
// when the union is basic-legal, until a full pass merges nothing.
static bool basic_legal(const kf_pipeline *p, const std::set<int> &P, const kf_model_params &m,
                        const std::vector<EdgeInfo> &E)
{
    if (P.size() == 1) return true;
    if (!is_legal(p, P, m, E)) return false;
    auto pr = producers(p);
    int nsrc = 0;
    for (int k : P) {
        bool has_prod = false;
        for (int s : pr[k]) has_prod |= P.count(s) > 0;
        if (has_prod) {
            for (int img : p->ops[k].inputs)
                if (!(img >= p->n_inputs && P.count(img - p->n_inputs))) return false;   // shared/external input
        } else {
            nsrc++;
        }
    }
    if (nsrc != 1) return false;
    for (int k : P) {
        if (p->ops[k].kind != LOCAL) continue;
        std::vector<int> st(pr[k].begin(), pr[k].end());   // walk the producers inside P
        std::set<int> seen;
        while (!st.empty()) {
            int u = st.back();
            st.pop_back();
            if (!P.count(u) || !seen.insert(u).second) continue;
            if (p->ops[u].kind == LOCAL) return false;   // local-to-local
            for (int v : pr[u]) st.push_back(v);
        }
    }
    return true;
}

kf_plan *plan_basic(kf_pipeline *p, const kf_model_params &m)
{
    if (p->ops.empty()) fail(KF_ERR_ARG, "pipeline has no kernels");
    auto plan = std::make_unique<kf_plan>();
    plan->edges = edge_weights(p, m);
    const int n = (int)p->ops.size();
    std::vector<int> lab(n);
    for (int k = 0; k < n; k++) lab[k] = k;
    std::vector<const EdgeInfo *> order;
    for (const EdgeInfo &e : plan->edges)
        if (e.profitable) order.push_back(&e);
    std::stable_sort(order.begin(), order.end(), [](const EdgeInfo *a, const EdgeInfo *b) {
        if (a->w != b->w) return a->w > b->w;
        return a->ks != b->ks ? a->ks < b->ks : a->kd < b->kd;
    });
    for (bool changed = true; changed;) {
        changed = false;
        for (const EdgeInfo *e : order) {
            const int a = lab[e->ks], b = lab[e->kd];
            if (a == b) continue;
            std::set<int> U;
            for (int k = 0; k < n; k++)
                if (lab[k] == a || lab[k] == b) U.insert(k);
            if (!basic_legal(p, U, m, plan->edges)) continue;
            for (int k = 0; k < n; k++)
                if (lab[k] == b) lab[k] = a;
            changed = true;
        }
    }
    std::map<int, std::vector<int>> byl;
    for (int k = 0; k < n; k++) byl[lab[k]].push_back(k);
    for (auto &kv : byl) plan->blocks.push_back(kv.second);
    finish_plan(p, plan.get());
    return plan.release();
}

// ---------------------------------------------------------------------------
// §8(f)4 -- exact planner: the maximum of Eq. 1 (sum of the weights of the
// edges inside blocks, lexicographic (q, eps) as in Alg. 1) over ALL
// partitions into legal blocks -- the exhaustive alternative the paper rules
// out for large graphs (minimum-weight k-cut, NP-complete).
// Subset DP, O(3^n): best(S) = max over legal B, min(S) in B, B subset of S,
// of w(B) + best(S \ B).  Limited to n <= 16 kernels.  Ties keep the first
// candidate in increasing sub-mask order (deterministic).
kf_plan *plan_exact(kf_pipeline *p, const kf_model_params &m)
{
    const int n = (int)p->ops.size();
    if (n == 0) fail(KF_ERR_ARG, "pipeline has no kernels");
    if (n > 16) fail(KF_ERR_ARG, "exact planner is limited to 16 kernels (O(3^n))");
    auto plan = std::make_unique<kf_plan>();
    plan->edges = edge_weights(p, m);
    const uint32_t full = (1u << n) - 1;
    std::vector<char> legal(full + 1, 0);
    std::vector<W2> w(full + 1);
    for (uint32_t s = 1; s <= full; s++) {
        std::set<int> S;
        for (int k = 0; k < n; k++)
            if (s >> k & 1) S.insert(k);
        legal[s] = S.size() == 1 || is_legal(p, S, m, plan->edges);
        if (!legal[s]) continue;
        for (const EdgeInfo &e : plan->edges)
            if ((s >> e.ks & 1) && (s >> e.kd & 1)) w[s] = w[s] + W2{e.q, e.eps};
    }
    std::vector<W2> best(full + 1);
    std::vector<uint32_t> pick(full + 1, 0);
    for (uint32_t s = 1; s <= full; s++) {
        const uint32_t low = s & (~s + 1u), rest = s ^ low;
        bool have = false;
        // sub-masks B = low | r, r a sub-mask of rest, in increasing order
        for (uint32_t r = 0;; r = (r - rest) & rest) {
            const uint32_t B = low | r;
            if (legal[B]) {
                W2 c = w[B] + best[s ^ B];
                if (!have || best[s] < c) { best[s] = c; pick[s] = B; have = true; }
            }
            if (r == rest) break;
        }
    }
    for (uint32_t s = full; s; s ^= pick[s]) {
        std::vector<int> b;
        for (int k = 0; k < n; k++)
            if (pick[s] >> k & 1) b.push_back(k);
        plan->blocks.push_back(b);
    }
    finish_plan(p, plan.get());
    return plan.release();
}

kf_plan *plan_from_blocks(kf_pipeline *p, std::vector<std::vector<int>> blocks, bool check)
{
    auto plan = std::make_unique<kf_plan>();
    kf_model_params m;
    kf_model_params_paper(&m);
    plan->edges = edge_weights(p, m);
    for (auto &b : blocks) {
        if (check && b.size() > 1) {
            std::set<int> S(b.begin(), b.end());
            if (!dependence_legal(p, S) || !header_legal(p, S)) {
                std::string s;
                for (int k : b) s += " " + std::to_string(k);
                fail(KF_ERR_ILLEGAL_BLOCK, "block {" + s + " } is not legal (dependence/header)");
            }
        }
    }
    plan->blocks = std::move(blocks);
    finish_plan(p, plan.get());
    return plan.release();
}

// Block analysis: sink, external images, halos, staged kernels.
BlockInfo analyse_block(const kf_pipeline *p, const std::vector<int> &kernels)
{
    BlockInfo b;
    b.kernels = kernels;
    std::sort(b.kernels.begin(), b.kernels.end());
    std::set<int> S(b.kernels.begin(), b.kernels.end());
    auto co = consumers(p);
    for (int k : b.kernels) {
        bool inner = false;
        for (int c : co[k]) inner |= S.count(c) > 0;
        if (!inner) b.sink = k;                 // legal blocks have exactly one
    }
    for (auto it = b.kernels.rbegin(); it != b.kernels.rend(); ++it) {
        int k = *it;
        int hx = 0, hy = 0;
        for (int c : co[k])
            if (S.count(c)) {
                hx = std::max(hx, b.hx[c] + p->ops[c].rx());
                hy = std::max(hy, b.hy[c] + p->ops[c].ry());
                if (p->ops[c].kind == LOCAL) b.staged.insert(k);
            }
        b.hx[k] = hx;
        b.hy[k] = hy;
    }
    std::set<int> ext;
    for (int k : b.kernels)
        for (int img : p->ops[k].inputs) {
            bool inside = img >= p->n_inputs && S.count(img - p->n_inputs);
            if (inside) continue;
            ext.insert(img);
            b.ext_hx[img] = std::max(b.ext_hx.count(img) ? b.ext_hx[img] : 0, b.hx[k] + p->ops[k].rx());
            b.ext_hy[img] = std::max(b.ext_hy.count(img) ? b.ext_hy[img] : 0, b.hy[k] + p->ops[k].ry());
        }
    b.ext.assign(ext.begin(), ext.end());
    for (int img : b.ext) {
        b.Rx = std::max(b.Rx, b.ext_hx[img]);
        b.Ry = std::max(b.Ry, b.ext_hy[img]);
    }
    int loc = 0, rep = 0;
    for (int k : b.kernels)
        if (p->ops[k].kind == LOCAL) { loc++; rep += p->ops[k].mode == KF_REPEAT; }
    b.torus = loc > 0 && rep == loc;
    return b;
}

}  // namespace kf
