// Host-side preprocessing rows of DiGraph (sec. 3.2.1 / 3.2.3):
//   (1) Algorithm 1 path decomposition per subgraph (OpenMP), short-path
//       merging, hot/cold classification;
//   (2) path dependency graph, Tarjan SCC condensation (DAG sketch),
//       layering, priority Pri(p), partitions and vertex->partition maps;
//   (5) multi-rank path partitioning and the boundary (replica) vertex set.
// Deterministic for a given dg_path_params (independent of the number of
// OpenMP threads): subgraph outputs are concatenated in subgraph order.
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <parallel/algorithm>
#include <stdexcept>

#include "dg_internal.h"

namespace dg {
namespace {

struct SubOut {
    std::vector<int32_t> pv;     // path vertices, concatenated
    std::vector<int32_t> pw;     // weight of the edge into each path vertex (0 at heads)
    std::vector<int64_t> start;  // path starts into pv (+ final size)
};

// ---------------------------------------------------------------------------
// Algorithm 1 on one subgraph [lo, hi).
// An expansion of v visits *all* of v's local edges (the for loop of lines
// 6-17 runs to completion and only expansions of v visit v's edges), so
// "v has unvisited local edges" == "v is local, has out-edges and was never
// expanded"; no per-edge visited flags are needed.
// ---------------------------------------------------------------------------
struct Decomposer {
    const HostCSR& g;
    const std::vector<int32_t>& scol;   // successors of each row, sorted (line 5)
    const std::vector<int32_t>& sw;     // their weights
    const std::vector<int64_t>& deg;
    std::vector<uint8_t>& expanded;     // global, disjoint per subgraph
    std::vector<uint8_t>& inner;        // global (line 13), benign byte races
    std::vector<uint32_t>& visited;     // per thread, stamp = subgraph id + 1
    uint32_t stamp;
    int64_t lo, hi;
    int d_max;
    SubOut& out;
    bool open = false;

    void new_path() {  // lines 14 / 19: close the current path
        if (open) { out.start.push_back((int64_t)out.pv.size()); open = false; }
    }
    void insert(int32_t u, int32_t v, int32_t w) {  // line 9
        if (!open) { out.pv.push_back(u); out.pw.push_back(0); open = true; }
        out.pv.push_back(v); out.pw.push_back(w);
    }
    bool has_unvisited(int64_t v) const {
        return v >= lo && v < hi && !expanded[v] && g.row_ptr[v + 1] > g.row_ptr[v];
    }
    void graphp(int32_t v_root, int d) {
        visited[v_root] = stamp;                                    // line 2
        if (has_unvisited(v_root) && d < d_max) {                   // line 3
            expanded[v_root] = 1;
            for (int64_t e = g.row_ptr[v_root]; e < g.row_ptr[v_root + 1]; e++) {  // lines 4-6
                int32_t v = scol[e];
                insert(v_root, v, sw[e]);                           // lines 7-9
                if (visited[v] != stamp) {                          // line 10
                    graphp(v, d + 1);                               // line 11
                } else {
                    __atomic_store_n(&inner[v], (uint8_t)1, __ATOMIC_RELAXED);  // line 13
                    new_path();                                     // line 14
                }
            }
        } else {
            new_path();                                             // line 19
        }
    }
};

// Iterative Tarjan over a CSR graph (node ids < 2^31); comp[v] = SCC id in
// completion order (reverse topological order of the condensation).
int32_t tarjan(int32_t N, const std::vector<int64_t>& ptr, const std::vector<int32_t>& adj,
               std::vector<int32_t>& comp) {
    std::vector<int32_t> index(N, -1), low(N, 0);
    std::vector<int64_t> it(N, 0);
    std::vector<uint8_t> onst(N, 0);
    std::vector<int32_t> st, work;
    st.reserve(1024); work.reserve(1024);
    comp.assign(N, -1);
    int32_t counter = 0, ncomp = 0;
    for (int32_t r = 0; r < N; r++) {
        if (index[r] != -1) continue;
        index[r] = low[r] = counter++;
        st.push_back(r); onst[r] = 1; it[r] = ptr[r];
        work.push_back(r);
        while (!work.empty()) {
            int32_t v = work.back();
            if (it[v] < ptr[v + 1]) {
                int32_t u = adj[it[v]++];
                if (index[u] == -1) {
                    index[u] = low[u] = counter++;
                    st.push_back(u); onst[u] = 1; it[u] = ptr[u];
                    work.push_back(u);
                } else if (onst[u]) {
                    low[v] = std::min(low[v], index[u]);
                }
            } else {
                work.pop_back();
                if (!work.empty()) { int32_t q = work.back(); low[q] = std::min(low[q], low[v]); }
                if (low[v] == index[v]) {
                    while (true) {
                        int32_t x = st.back(); st.pop_back(); onst[x] = 0;
                        comp[x] = ncomp;
                        if (x == v) break;
                    }
                    ncomp++;
                }
            }
        }
    }
    return ncomp;
}

}  // namespace

void build_layout(const HostCSR& g, const dg_path_params& p, HostLayout& L) {
    auto t0 = std::chrono::steady_clock::now();
    auto tp = t0;
    const bool verbose = std::getenv("DG_VERBOSE") != nullptr;
    auto phase = [&](const char* name) {
        auto now = std::chrono::steady_clock::now();
        if (verbose)
            std::fprintf(stderr, "[dg_build_paths] %-22s %9.1f ms\n", name,
                         std::chrono::duration<double, std::milli>(now - tp).count());
        tp = now;
    };
    const int64_t n = g.n, m = g.m;
    L = HostLayout();
    L.params = p;
    std::vector<int64_t> deg(n);
    for (int64_t v = 0; v < n; v++) deg[v] = (int64_t)g.indeg[v] + g.outdeg[v];

    // ---- line 5: successors sorted by (degree desc, id asc), stable in CSR order
    std::vector<int32_t> scol(g.col), sw(m);
    if (g.has_w) sw = g.w; else std::fill(sw.begin(), sw.end(), 1);
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; v++) {
        int64_t b = g.row_ptr[v], e = g.row_ptr[v + 1];
        if (e - b < 2) continue;
        std::vector<std::pair<int32_t, int32_t>> tmp(e - b);
        for (int64_t i = b; i < e; i++) tmp[i - b] = {scol[i], sw[i]};
        if (p.order == 0)
            std::stable_sort(tmp.begin(), tmp.end(), [&](const auto& x, const auto& y) {
                if (deg[x.first] != deg[y.first]) return deg[x.first] > deg[y.first];
                return x.first < y.first;
            });
        else
            std::stable_sort(tmp.begin(), tmp.end(),
                             [](const auto& x, const auto& y) { return x.first < y.first; });
        for (int64_t i = b; i < e; i++) { scol[i] = tmp[i - b].first; sw[i] = tmp[i - b].second; }
    }

    phase("sort successors");
    // ---- subgraphs: contiguous vertex ranges of ~m/T out-edges (reading R-SUB)
    const int T = std::max(1, p.n_sub);
    std::vector<int64_t> bounds(T + 1, 0);
    for (int k = 1; k < T; k++) {
        int64_t target = (int64_t)(((__int128)k * m) / T);
        int64_t v = std::lower_bound(g.row_ptr.begin(), g.row_ptr.begin() + n + 1, target) - g.row_ptr.begin();
        bounds[k] = std::max(bounds[k - 1], std::min(v, n));
    }
    bounds[T] = n;

    // ---- Algorithm 1 on every subgraph (parallel over subgraphs)
    std::vector<SubOut> subs(T);
    std::vector<uint8_t> expanded(n, 0), inner(n, 0);
    const int nthr = omp_get_max_threads();
    std::vector<std::vector<uint32_t>> vis(nthr);
    #pragma omp parallel for schedule(dynamic, 1)
    for (int k = 0; k < T; k++) {
        auto& visited = vis[omp_get_thread_num()];
        if (visited.empty()) visited.assign(n, 0);
        int64_t lo = bounds[k], hi = bounds[k + 1];
        SubOut& out = subs[k];
        out.start.push_back(0);
        Decomposer D{g, scol, sw, deg, expanded, inner, visited, (uint32_t)(k + 1), lo, hi, p.d_max, out};
        std::vector<int32_t> roots(hi - lo);
        std::iota(roots.begin(), roots.end(), (int32_t)lo);
        if (p.order == 0)
            std::stable_sort(roots.begin(), roots.end(),
                             [&](int32_t a, int32_t b) { return deg[a] > deg[b]; });
        for (int32_t r : roots)
            if (D.has_unvisited(r)) D.graphp(r, 0);
        D.new_path();
    }

    phase("algorithm 1");
    // ---- concatenate (subgraph order)
    std::vector<int64_t> poff{0};
    std::vector<int32_t> pv, pw;
    {
        int64_t tot = 0;
        for (auto& s : subs) tot += (int64_t)s.pv.size();
        pv.reserve(tot); pw.reserve(tot);
        for (auto& s : subs) {
            int64_t base = (int64_t)pv.size();
            pv.insert(pv.end(), s.pv.begin(), s.pv.end());
            pw.insert(pw.end(), s.pw.begin(), s.pw.end());
            for (size_t i = 1; i < s.start.size(); i++) poff.push_back(base + s.start[i]);
            std::vector<int32_t>().swap(s.pv);
            std::vector<int32_t>().swap(s.pw);
            std::vector<int64_t>().swap(s.start);
        }
    }
    const int64_t P0 = (int64_t)poff.size() - 1;
    L.paths_before_merge = P0;
    if (P0 >= INT32_MAX || P0 + n >= INT32_MAX) throw std::runtime_error("too many paths for 32-bit path ids");
    { std::vector<SubOut>().swap(subs); std::vector<std::vector<uint32_t>>().swap(vis); }

    phase("concatenate");
    // ---- short-path merging (reading R-MERGE):
    // pair the k-th path ending at x with the k-th path starting at x, cut
    // cycles before their lowest index, cut chains into <= l_merge edges,
    // order merged paths by their first piece.
    std::vector<int32_t> nxt(P0, -1), prv(P0, -1);
    if (p.l_merge > 0 && P0 > 1) {
        std::vector<int64_t> eptr(n + 1, 0), sptr(n + 1, 0);
        std::vector<int32_t> elist(P0), slist(P0);
        for (int64_t i = 0; i < P0; i++) { eptr[pv[poff[i + 1] - 1] + 1]++; sptr[pv[poff[i]] + 1]++; }
        for (int64_t v = 0; v < n; v++) { eptr[v + 1] += eptr[v]; sptr[v + 1] += sptr[v]; }
        {
            std::vector<int64_t> fe(eptr.begin(), eptr.end() - 1), fs(sptr.begin(), sptr.end() - 1);
            for (int64_t i = 0; i < P0; i++) {
                elist[fe[pv[poff[i + 1] - 1]]++] = (int32_t)i;
                slist[fs[pv[poff[i]]]++] = (int32_t)i;
            }
        }
        #pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t x = 0; x < n; x++) {
            const int64_t na = eptr[x + 1] - eptr[x], nb = sptr[x + 1] - sptr[x];
            if (!na || !nb) continue;
            if (p.merge_rule == 0 && g.indeg[x] > 1 && g.outdeg[x] > 1 && inner[x]) continue;
            int32_t* A = &elist[eptr[x]];
            int32_t* B = &slist[sptr[x]];
            for (int64_t k = 0; k < std::min(na, nb); k++) {
                if (A[k] == B[k]) {
                    if (k + 1 < nb) std::swap(B[k], B[k + 1]);
                    else continue;
                }
                nxt[A[k]] = B[k];
                prv[B[k]] = A[k];
            }
        }
    }
    // chains (start where nothing links in), then cycles cut before their lowest index
    std::vector<uint8_t> seen(P0, 0);
    std::vector<int32_t> seg_first, seg_len;   // segments: first piece, #pieces
    std::vector<int32_t> seg_pieces;           // pieces in chain order, segments contiguous per chain
    auto walk_chain = [&](int32_t s0, std::vector<int32_t>& pieces, std::vector<int32_t>& sf, std::vector<int32_t>& sl) {
        int64_t cur_len = 0;
        int32_t cur_n = 0;
        for (int32_t j = s0; j != -1 && !seen[j]; j = nxt[j]) {
            seen[j] = 1;
            const int64_t e = poff[j + 1] - poff[j] - 1;
            if (cur_n && cur_len + e > p.l_merge) { sl.push_back(cur_n); cur_n = 0; cur_len = 0; }
            if (!cur_n) sf.push_back(j);
            pieces.push_back(j);
            cur_n++; cur_len += e;
        }
        if (cur_n) sl.push_back(cur_n);
    };
    {
        const int nth = omp_get_max_threads();
        std::vector<std::vector<int32_t>> tp(nth), tf(nth), tl(nth);
        #pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t i = 0; i < P0; i++)
            if (prv[i] == -1) { int t = omp_get_thread_num(); walk_chain((int32_t)i, tp[t], tf[t], tl[t]); }
        for (int t = 0; t < nth; t++) {
            seg_pieces.insert(seg_pieces.end(), tp[t].begin(), tp[t].end());
            seg_first.insert(seg_first.end(), tf[t].begin(), tf[t].end());
            seg_len.insert(seg_len.end(), tl[t].begin(), tl[t].end());
        }
        for (int64_t i = 0; i < P0; i++)
            if (!seen[i]) walk_chain((int32_t)i, seg_pieces, seg_first, seg_len);
    }
    { std::vector<int32_t>().swap(nxt); std::vector<int32_t>().swap(prv); std::vector<uint8_t>().swap(seen); }
    const int64_t P = (int64_t)seg_first.size();
    std::vector<int64_t> seg_start(P + 1, 0);   // into seg_pieces
    for (int64_t s2 = 0; s2 < P; s2++) seg_start[s2 + 1] = seg_start[s2] + seg_len[s2];
    std::vector<int32_t> sorder(P);
    std::iota(sorder.begin(), sorder.end(), 0);
    std::sort(sorder.begin(), sorder.end(), [&](int32_t a, int32_t b) { return seg_first[a] < seg_first[b]; });
    // materialise merged paths (merge order) in parallel
    std::vector<int64_t> moff(P + 1, 0);
    for (int64_t r = 0; r < P; r++) {
        int64_t sgi = sorder[r], len = 1;
        for (int64_t q = seg_start[sgi]; q < seg_start[sgi + 1]; q++) len += poff[seg_pieces[q] + 1] - poff[seg_pieces[q]] - 1;
        moff[r + 1] = moff[r] + len;
    }
    std::vector<int32_t> mv(moff[P]), mw(moff[P]);
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t r = 0; r < P; r++) {
        int64_t sgi = sorder[r], o = moff[r];
        bool first = true;
        for (int64_t q = seg_start[sgi]; q < seg_start[sgi + 1]; q++) {
            int64_t c = seg_pieces[q];
            for (int64_t k = poff[c] + (first ? 0 : 1); k < poff[c + 1]; k++) { mv[o] = pv[k]; mw[o] = pw[k]; o++; }
            first = false;
        }
    }
    { std::vector<int32_t>().swap(pv); std::vector<int32_t>().swap(pw); }

    phase("merge");
    // ---- path statistics (reading R-HOT)
    std::vector<double> dbar(P);
    std::vector<int64_t> nvert(P);
    std::vector<uint8_t> hot(P);
    const double mean_deg = n ? 2.0 * (double)m / (double)n : 0.0;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < P; i++) {
        double s = 0;
        for (int64_t k = moff[i]; k < moff[i + 1]; k++) s += (double)deg[mv[k]];
        nvert[i] = moff[i + 1] - moff[i];
        dbar[i] = s / (double)nvert[i];
        hot[i] = dbar[i] >= (double)p.hot_factor * mean_deg;
    }

    phase("path stats");
    // ---- dependency graph G' as a bipartite path/vertex graph (reading R-DEP):
    // path node i -> vertex node P+x for every x entered by an edge of i;
    // vertex node P+x -> path node j for every x left by an edge of j.
    // Reachability between path nodes equals reachability in G'.
    const int64_t N = P + n;
    std::vector<int64_t> aptr(N + 1, 0);
    std::vector<int32_t> adj;
    std::vector<int64_t> layer_of_path(P, 0), scc_label(P, 0);
    int64_t n_layers = 0, n_dep_sccs = 0, giant = 0;
    {
        for (int64_t i = 0; i < P; i++) {
            int64_t len = moff[i + 1] - moff[i];
            aptr[i + 1] += len - 1;                                   // entered vertices
            for (int64_t k = moff[i]; k < moff[i + 1] - 1; k++) aptr[P + mv[k] + 1]++;  // left vertices
        }
        for (int64_t x = 0; x < N; x++) aptr[x + 1] += aptr[x];
        adj.resize(aptr[N]);
        std::vector<int64_t> fill(aptr.begin(), aptr.end() - 1);
        for (int64_t i = 0; i < P; i++) {
            for (int64_t k = moff[i] + 1; k < moff[i + 1]; k++) adj[fill[i]++] = (int32_t)(P + mv[k]);
            for (int64_t k = moff[i]; k < moff[i + 1] - 1; k++) adj[fill[P + mv[k]]++] = (int32_t)i;
        }
        std::vector<int32_t> comp;
        int64_t nc = tarjan((int32_t)N, aptr, adj, comp);
        // group nodes by comp; comps are numbered in reverse topological order
        std::vector<int64_t> cptr(nc + 1, 0), cnodes(N);
        for (int64_t x = 0; x < N; x++) cptr[comp[x] + 1]++;
        for (int64_t c = 0; c < nc; c++) cptr[c + 1] += cptr[c];
        {
            std::vector<int64_t> fill2(cptr.begin(), cptr.end() - 1);
            for (int64_t x = 0; x < N; x++) cnodes[fill2[comp[x]]++] = x;
        }
        std::vector<int64_t> f(nc, 0), minpath(nc, INT64_MAX), npaths(nc, 0);
        for (int64_t i = 0; i < P; i++) {
            minpath[comp[i]] = std::min(minpath[comp[i]], i);
            npaths[comp[i]]++;
        }
        // topological order = decreasing comp id (sources first)
        for (int64_t c = nc - 1; c >= 0; c--) {
            int64_t add = npaths[c] > 0 ? 1 : 0;
            for (int64_t q = cptr[c]; q < cptr[c + 1]; q++) {
                int64_t x = cnodes[q];
                for (int64_t e = aptr[x]; e < aptr[x + 1]; e++) {
                    int64_t d = comp[adj[e]];
                    if (d != c) f[d] = std::max(f[d], f[c] + add);
                }
            }
        }
        for (int64_t i = 0; i < P; i++) {
            layer_of_path[i] = f[comp[i]];
            scc_label[i] = minpath[comp[i]];
            n_layers = std::max(n_layers, f[comp[i]] + 1);
        }
        for (int64_t c = 0; c < nc; c++)
            if (npaths[c] > 0) { n_dep_sccs++; giant = std::max(giant, npaths[c]); }
    }
    { std::vector<int32_t>().swap(adj); std::vector<int64_t>().swap(aptr); }

    phase("dependency DAG");
    // ---- priority Pri(p) = alpha*D(p)*N(p) - L(p)
    double dmax = 0; int64_t nmax = 0;
    for (int64_t i = 0; i < P; i++) { dmax = std::max(dmax, dbar[i]); nmax = std::max(nmax, nvert[i]); }
    const double alpha = (dmax > 0 && nmax > 0) ? 1.0 / (dmax * (double)nmax) : 0.0;
    std::vector<double> pri(P);
    for (int64_t i = 0; i < P; i++) pri[i] = alpha * dbar[i] * (double)nvert[i] - (double)layer_of_path[i];
    std::vector<int64_t> order(P);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](int64_t a, int64_t b) { return pri[a] > pri[b]; });

    // ---- partitions over the priority order (greedy, whole paths)
    // part_entries == 0: auto -- about 16K partitions (several per resident
    // warp of a 148-SM grid), between 128 and 2048 entries each
    int64_t target = p.part_entries;
    if (target <= 0) {
        int64_t tot = 0;
        for (int64_t i = 0; i < P; i++) tot += nvert[i];
        target = std::min<int64_t>(2048, std::max<int64_t>(128, tot / 16384));
    }
    std::vector<int64_t> gpart_first{0};  // global partition -> first index in `order`
    {
        int64_t acc = 0;
        for (int64_t r = 0; r < P; r++) {
            if (acc >= target) { gpart_first.push_back(r); acc = 0; }
            acc += nvert[order[r]];
        }
        gpart_first.push_back(P);
        if (P == 0) gpart_first.assign(1, 0);
    }
    const int64_t G = (int64_t)gpart_first.size() - 1;
    const int world = std::max(1, p.world), rank = p.rank;

    // ---- internal numbering: vertices in degree-descending order (ties by id).
    // The H highest-degree vertices get ids [0, H) so the path kernel keeps them
    // as shared-memory proxies; the rest are packed by degree so the vertex
    // states that most path entries touch share cache sectors and stay in L2.
    const int64_t H = std::min<int64_t>(std::max<int32_t>(0, p.n_proxy), n);
    L.n_proxy = H;
    L.new_id.resize(n);
    L.orig.resize(n);
    {
        std::vector<int32_t> byd(n);
        std::iota(byd.begin(), byd.end(), 0);
        __gnu_parallel::sort(byd.begin(), byd.end(), [&](int32_t a, int32_t b) {
            return deg[a] != deg[b] ? deg[a] > deg[b] : a < b;
        });
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < n; i++) {
            L.new_id[byd[i]] = (int32_t)i;
            L.orig[i] = byd[i];
        }
    }
    // CSR in internal ids
    L.prow_ptr.assign(n + 1, 0);
    L.poutdeg.resize(n);
    for (int64_t u = 0; u < n; u++) {
        L.poutdeg[u] = g.outdeg[L.orig[u]];
        L.prow_ptr[u + 1] = L.prow_ptr[u] + L.poutdeg[u];
    }
    L.pcol.resize(m);
    if (g.has_w) L.pw.resize(m);
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < n; u++) {
        const int64_t src0 = g.row_ptr[L.orig[u]], len = L.poutdeg[u], dst0 = L.prow_ptr[u];
        for (int64_t k = 0; k < len; k++) {
            L.pcol[dst0 + k] = L.new_id[g.col[src0 + k]];
            if (g.has_w) L.pw[dst0 + k] = g.w[src0 + k];
        }
    }

    // ---- boundary vertices: present in partitions of >1 rank (round-robin owner q % world)
    if (world > 1) {
        std::vector<uint64_t> present(n, 0);  // ranks whose partitions hold v
        for (int64_t q = 0; q < G; q++) {
            uint64_t bit = 1ull << ((q % world) & 63);
            for (int64_t r = gpart_first[q]; r < gpart_first[q + 1]; r++) {
                int64_t i = order[r];
                for (int64_t k = moff[i]; k < moff[i + 1]; k++) present[mv[k]] |= bit;
            }
        }
        for (int64_t v = 0; v < n; v++)
            if (__builtin_popcountll(present[v]) > 1) L.boundary.push_back(L.new_id[v]);
        std::sort(L.boundary.begin(), L.boundary.end());
    }

    phase("priority+partitions");
    // ---- this rank's layout
    L.part_off.push_back(0);
    L.path_off.push_back(0);
    for (int64_t q = rank; q < G; q += world) {
        for (int64_t r = gpart_first[q]; r < gpart_first[q + 1]; r++) {
            int64_t i = order[r];
            for (int64_t k = moff[i]; k < moff[i + 1]; k++) {
                uint32_t code = (uint32_t)L.new_id[mv[k]];
                if (k == moff[i]) code |= kHead;
                if (k == moff[i + 1] - 1) code |= kTail;
                L.e_idx.push_back(code);
                L.e_w.push_back(mw[k]);
            }
            L.path_off.push_back((int64_t)L.e_idx.size());
            L.layer.push_back((int32_t)layer_of_path[i]);
            L.scc.push_back(scc_label[i]);
            L.merged_index.push_back(i);
            L.hot.push_back(hot[i]);
            L.n_hot += hot[i];
        }
        L.part_off.push_back((int64_t)L.e_idx.size());
    }

    phase("layout");
    L.n_layers = n_layers;
    L.n_dep_sccs = n_dep_sccs;
    L.giant = giant;
    L.built = true;
    L.preprocess_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

}  // namespace dg
