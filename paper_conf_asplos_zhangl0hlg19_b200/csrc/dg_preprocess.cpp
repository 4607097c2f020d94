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
#include <functional>
#include <numeric>
#include <parallel/algorithm>
#include <stdexcept>

#include "dg_internal.h"

namespace dg {
namespace {

// Vector whose resize() leaves PODs uninitialised (the big temporaries are
// overwritten in parallel right after; value-initialising them is a
// single-threaded memset of tens of GB at Twitter scale).
template <class T>
struct NoInit : std::allocator<T> {
    template <class U> struct rebind { using other = NoInit<U>; };
    NoInit() = default;
    template <class U> NoInit(const NoInit<U>&) noexcept {}
    template <class U> void construct(U* p) noexcept { ::new ((void*)p) U; }
    template <class U, class... A> void construct(U* p, A&&... a) { ::new ((void*)p) U(std::forward<A>(a)...); }
};
template <class T> using rvec = std::vector<T, NoInit<T>>;

// Parallel stable group-by (radix partition + per-bucket counting sort):
// items [0, n_items) each emit (key, value) pairs through
// emit(item, sink); the result is a CSR over keys [0, n_keys) whose lists
// hold the values in item order (then emission order) -- deterministic and
// independent of the thread count.  Cache-friendly: pass 1 counts pairs per
// (thread, bucket of 2^16 keys), pass 2 scatters them into bucket-major
// runs, pass 3 sorts each bucket by key with a bucket-local cursor array.
template <class Emit>
void group_by(int64_t n_items, int64_t n_keys, Emit&& emit, std::vector<int64_t>& ptr, rvec<int32_t>& vals) {
    constexpr int kShift = 16;
    const int64_t B = std::max<int64_t>(1, (n_keys + (1 << kShift) - 1) >> kShift);
    const int T = omp_get_max_threads();
    std::vector<int64_t> cnt((size_t)T * B, 0);
    auto chunk = [&](int t, int64_t& lo, int64_t& hi) {
        lo = n_items * t / T;
        hi = n_items * (t + 1) / T;
    };
    #pragma omp parallel num_threads(T)
    {
        const int t = omp_get_thread_num();
        int64_t lo, hi;
        chunk(t, lo, hi);
        int64_t* c = &cnt[(size_t)t * B];
        for (int64_t i = lo; i < hi; i++) emit(i, [&](int32_t key, int32_t) { c[key >> kShift]++; });
    }
    std::vector<int64_t> off((size_t)T * B), bstart(B + 1, 0);
    {
        int64_t acc = 0;
        for (int64_t b = 0; b < B; b++) {
            bstart[b] = acc;
            for (int t = 0; t < T; t++) { off[(size_t)t * B + b] = acc; acc += cnt[(size_t)t * B + b]; }
        }
        bstart[B] = acc;
    }
    const int64_t total = bstart[B];
    rvec<int32_t> tk(total), tv(total);
    #pragma omp parallel num_threads(T)
    {
        const int t = omp_get_thread_num();
        int64_t lo, hi;
        chunk(t, lo, hi);
        int64_t* o = &off[(size_t)t * B];
        for (int64_t i = lo; i < hi; i++)
            emit(i, [&](int32_t key, int32_t v) { const int64_t q = o[key >> kShift]++; tk[q] = key; tv[q] = v; });
    }
    ptr.assign(n_keys + 1, 0);
    vals.resize(total);
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t b = 0; b < B; b++) {
        const int64_t k0 = b << kShift, k1 = std::min<int64_t>(n_keys, (b + 1) << kShift);
        std::vector<int64_t> cur(k1 - k0 + 1, 0);
        for (int64_t q = bstart[b]; q < bstart[b + 1]; q++) cur[tk[q] - k0 + 1]++;
        for (int64_t k = 0; k < k1 - k0; k++) cur[k + 1] += cur[k];
        for (int64_t k = k0; k < k1; k++) ptr[k] = bstart[b] + cur[k - k0];
        for (int64_t q = bstart[b]; q < bstart[b + 1]; q++) vals[bstart[b] + cur[tk[q] - k0]++] = tv[q];
    }
    ptr[n_keys] = total;
}


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

// ---------------------------------------------------------------------------
// Dependency graph G' and its DAG sketch (readings
// R-DEP, R-LAYER), as a bipartite path/vertex graph with implicit adjacency:
//   path node i    -> vertex node P+x  for every x entered by an edge of i
//   vertex node P+x -> path node j     for every x left by an edge of j
// Reachability between path nodes equals reachability in G'.  SCCs are found
// by the parallel trim / forward-backward / Tarjan scheme: (1) nodes with no
// remaining predecessor or successor are peeled off in rounds (singleton SCCs;
// the peel rounds are a topological order of them); (2) the SCC of a pivot is
// the intersection of its forward and backward reachable sets (the giant SCC
// of power-law graphs); (3) the rest is split into the pivot's upstream,
// unrelated and downstream classes, each closed under SCCs, and condensed by
// sequential Tarjan.  Components are numbered in a topological order and the
// layers are longest-path depths over it.  SCC sets and layers are unique, so
// the result equals a plain Tarjan + topological DP (tests/test_host_preprocess.py).
// ---------------------------------------------------------------------------
struct DepGraph {
    int64_t P, n, N;
    const std::vector<int64_t>& moff;
    const rvec<int32_t>& mv;
    std::vector<int64_t> lptr, eptr;   // vertex x: paths leaving x / entering x
    rvec<int32_t> ladj, eadj;

    DepGraph(int64_t P_, int64_t n_, const std::vector<int64_t>& moff_, const rvec<int32_t>& mv_)
        : P(P_), n(n_), N(P_ + n_), moff(moff_), mv(mv_) {
        group_by(P, n, [&](int64_t i, auto&& sink) {
            for (int64_t k = moff[i]; k < moff[i + 1] - 1; k++) sink(mv[k], (int32_t)i);
        }, lptr, ladj);
        group_by(P, n, [&](int64_t i, auto&& sink) {
            for (int64_t k = moff[i] + 1; k < moff[i + 1]; k++) sink(mv[k], (int32_t)i);
        }, eptr, eadj);
    }
    template <class F> void for_out(int64_t u, F&& f) const {
        if (u < P) { for (int64_t k = moff[u] + 1; k < moff[u + 1]; k++) f(P + mv[k]); }
        else { const int64_t x = u - P; for (int64_t e = lptr[x]; e < lptr[x + 1]; e++) f((int64_t)ladj[e]); }
    }
    template <class F> void for_in(int64_t u, F&& f) const {
        if (u < P) { for (int64_t k = moff[u]; k < moff[u + 1] - 1; k++) f(P + mv[k]); }
        else { const int64_t x = u - P; for (int64_t e = eptr[x]; e < eptr[x + 1]; e++) f((int64_t)eadj[e]); }
    }
    int64_t outdeg(int64_t u) const { return u < P ? moff[u + 1] - moff[u] - 1 : lptr[u - P + 1] - lptr[u - P]; }
    int64_t indeg(int64_t u) const { return u < P ? moff[u + 1] - moff[u] - 1 : eptr[u - P + 1] - eptr[u - P]; }
};

// append per-thread vectors in thread order
template <class T>
void gather_threads(std::vector<std::vector<T>>& parts, std::vector<T>& out) {
    out.clear();
    size_t tot = 0;
    for (auto& p : parts) tot += p.size();
    out.reserve(tot);
    for (auto& p : parts) { out.insert(out.end(), p.begin(), p.end()); p.clear(); }
}

// Iterative Tarjan restricted to the nodes with cls[u] == c; components are
// appended to `comps` (members) in completion order = reverse topological order.
void tarjan_class(const DepGraph& G, const std::vector<int32_t>& nodes, const std::vector<uint8_t>& cls, uint8_t c,
                  std::vector<int32_t>& local, std::vector<std::vector<int32_t>>& comps) {
    if (nodes.empty()) return;
    const int32_t K = (int32_t)nodes.size();
    for (int32_t q = 0; q < K; q++) local[nodes[q]] = q;  // classes are disjoint: no race
    // local CSR of the class-internal out-edges
    std::vector<int64_t> ptr(K + 1, 0);
    std::vector<int32_t> adj;
    for (int32_t q = 0; q < K; q++) {
        G.for_out(nodes[q], [&](int64_t v) { if (cls[v] == c) adj.push_back(local[v]); });
        ptr[q + 1] = (int64_t)adj.size();
    }
    std::vector<int32_t> index(K, -1), low(K, 0), st, work;
    std::vector<int64_t> it(K, 0);
    std::vector<uint8_t> onst(K, 0);
    int32_t counter = 0;
    for (int32_t r = 0; r < K; r++) {
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
                    comps.emplace_back();
                    while (true) {
                        int32_t x = st.back(); st.pop_back(); onst[x] = 0;
                        comps.back().push_back(nodes[x]);
                        if (x == v) break;
                    }
                }
            }
        }
    }
}

struct DagResult {
    std::vector<int64_t> layer, scc;  // per path
    int64_t n_layers = 0, n_dep_sccs = 0, giant = 0;
};

void dependency_dag(const DepGraph& G, DagResult& R, const std::function<void(const char*)>& phase) {
    const int64_t P = G.P, N = G.N;
    const int nth = omp_get_max_threads();
    // ---- (1) trim
    std::vector<int32_t> indeg(N), outdeg(N), rnd(N, -1);
    std::vector<uint8_t> side(N, 0);  // 1 peeled as source, 2 peeled as sink
    std::vector<std::atomic<uint8_t>> claimed(N);
    std::vector<std::vector<int32_t>> parts(nth);
    #pragma omp parallel for schedule(static)
    for (int64_t u = 0; u < N; u++) {
        indeg[u] = (int32_t)G.indeg(u);
        outdeg[u] = (int32_t)G.outdeg(u);
        const bool s = indeg[u] == 0, t = outdeg[u] == 0;
        claimed[u].store(s || t, std::memory_order_relaxed);
        if (s || t) { side[u] = s ? 1 : 2; rnd[u] = 0; parts[omp_get_thread_num()].push_back((int32_t)u); }
    }
    std::vector<int32_t> frontier, peeled_src, peeled_snk;
    std::vector<int32_t> src_round_off{0}, snk_round_off{0};
    gather_threads(parts, frontier);
    for (int32_t r = 0; !frontier.empty(); r++) {
        std::sort(frontier.begin(), frontier.end());
        for (int32_t u : frontier) (side[u] == 1 ? peeled_src : peeled_snk).push_back(u);
        src_round_off.push_back((int32_t)peeled_src.size());
        snk_round_off.push_back((int32_t)peeled_snk.size());
        #pragma omp parallel for schedule(dynamic, 256)
        for (size_t q = 0; q < frontier.size(); q++) {
            const int32_t u = frontier[q];
            auto& out = parts[omp_get_thread_num()];
            auto claim = [&](int64_t v, uint8_t sd) {
                uint8_t z = 0;
                if (claimed[v].compare_exchange_strong(z, 1)) { side[v] = sd; rnd[v] = r + 1; out.push_back((int32_t)v); }
            };
            if (side[u] == 1) {
                G.for_out(u, [&](int64_t v) {
                    if (__atomic_sub_fetch(&indeg[v], 1, __ATOMIC_RELAXED) == 0) claim(v, 1);
                });
            } else {
                G.for_in(u, [&](int64_t w) {
                    if (__atomic_sub_fetch(&outdeg[w], 1, __ATOMIC_RELAXED) == 0) claim(w, 2);
                });
            }
        }
        gather_threads(parts, frontier);
    }
    phase("dag: trim");
    // ---- (2) forward / backward reachability of a pivot among the remaining nodes
    std::vector<uint8_t> cls(N, 0);  // 0 peeled, 1 upstream (B\F), 2 pivot SCC, 3 unrelated, 4 downstream (F\B)
    int64_t pivot = -1, best = -1;
    for (int64_t u = 0; u < P; u++)
        if (!claimed[u].load(std::memory_order_relaxed)) {
            const int64_t sc = (G.indeg(u) + 1) * (G.outdeg(u) + 1);
            if (sc > best) { best = sc; pivot = u; }
        }
    std::vector<uint8_t> F(N, 0), B(N, 0);
    auto bfs = [&](std::vector<uint8_t>& mark, bool fwd) {
        std::vector<int32_t> fr{(int32_t)pivot};
        mark[pivot] = 1;
        while (!fr.empty()) {
            #pragma omp parallel for schedule(dynamic, 256)
            for (size_t q = 0; q < fr.size(); q++) {
                auto& out = parts[omp_get_thread_num()];
                auto visit = [&](int64_t v) {
                    if (claimed[v].load(std::memory_order_relaxed) || __atomic_load_n(&mark[v], __ATOMIC_RELAXED)) return;
                    if (!__atomic_exchange_n(&mark[v], (uint8_t)1, __ATOMIC_RELAXED)) out.push_back((int32_t)v);
                };
                if (fwd) G.for_out(fr[q], visit); else G.for_in(fr[q], visit);
            }
            gather_threads(parts, fr);
        }
    };
    if (pivot >= 0) { bfs(F, true); bfs(B, false); }
    phase("dag: fw-bw");
    std::vector<std::vector<int32_t>> cls_nodes(5);
    {
        std::vector<std::vector<std::vector<int32_t>>> tp(nth, std::vector<std::vector<int32_t>>(5));
        #pragma omp parallel for schedule(static)
        for (int64_t u = 0; u < N; u++) {
            if (claimed[u].load(std::memory_order_relaxed)) continue;
            const uint8_t c = (F[u] && B[u]) ? 2 : B[u] ? 1 : F[u] ? 4 : 3;
            cls[u] = c;
            tp[omp_get_thread_num()][c].push_back((int32_t)u);
        }
        for (int c = 1; c <= 4; c++) {
            std::vector<std::vector<int32_t>> pc(nth);
            for (int t = 0; t < nth; t++) pc[t].swap(tp[t][c]);
            gather_threads(pc, cls_nodes[c]);
        }
    }
    { std::vector<uint8_t>().swap(F); std::vector<uint8_t>().swap(B); }
    phase("dag: classes");
    // ---- (3) Tarjan on the three remaining classes (in parallel)
    std::vector<std::vector<std::vector<int32_t>>> ccomps(5);
    {
        std::vector<int32_t> local(N, -1);
        #pragma omp parallel for schedule(dynamic, 1)
        for (int c = 1; c <= 4; c++)
            if (c != 2) tarjan_class(G, cls_nodes[c], cls, (uint8_t)c, local, ccomps[c]);
    }
    phase("dag: tarjan");
    // ---- component ids in a topological order:
    // source peel rounds, upstream comps, pivot SCC, unrelated comps,
    // downstream comps, sink peel rounds in reverse
    std::vector<int32_t> comp(N, -1);
    std::vector<int64_t> cstart{0};  // members of comp c (for the non-singleton blocks)
    int64_t nc = 0;
    for (int32_t u : peeled_src) comp[u] = (int32_t)nc++;
    const int64_t c_src_end = nc;
    std::vector<std::pair<int64_t, const std::vector<int32_t>*>> seq_comps;  // (id, members) of Tarjan comps
    auto add_tarjan = [&](int c) {
        auto& cc = ccomps[c];
        for (size_t q = cc.size(); q-- > 0;) {  // completion order reversed = topological
            for (int32_t u : cc[q]) comp[u] = (int32_t)nc;
            seq_comps.push_back({nc, &cc[q]});
            nc++;
        }
    };
    add_tarjan(1);
    const int64_t c_giant = cls_nodes[2].empty() ? -1 : nc;
    if (c_giant >= 0) { for (int32_t u : cls_nodes[2]) comp[u] = (int32_t)c_giant; nc++; }
    const size_t seq_mid = seq_comps.size();
    add_tarjan(3);
    add_tarjan(4);
    std::vector<int64_t> snk_comp_base(snk_round_off.size(), 0);
    for (int64_t r = (int64_t)snk_round_off.size() - 2; r >= 0; r--)
        for (int32_t q = snk_round_off[r]; q < snk_round_off[r + 1]; q++) comp[peeled_snk[q]] = (int32_t)nc++;
    // ---- per-comp path counts and smallest path index
    std::vector<int64_t> npaths(nc, 0), minpath(nc, INT64_MAX);
    for (int64_t i = 0; i < P; i++) {
        npaths[comp[i]]++;
        minpath[comp[i]] = std::min(minpath[comp[i]], i);
    }
    phase("dag: comp ids");
    // ---- layers: f[d] = max over condensation edges c->d of f[c] + (c holds a path)
    std::vector<int64_t> f(nc, 0);
    auto push = [&](int64_t u) {
        const int64_t cu = comp[u], val = f[cu] + (npaths[cu] > 0 ? 1 : 0);
        G.for_out(u, [&](int64_t v) {
            const int64_t cv = comp[v];
            if (cv == cu) return;
            int64_t cur = __atomic_load_n(&f[cv], __ATOMIC_RELAXED);
            while (val > cur && !__atomic_compare_exchange_n(&f[cv], &cur, val, true, __ATOMIC_RELAXED, __ATOMIC_RELAXED)) {}
        });
    };
    for (size_t r = 0; r + 1 < src_round_off.size(); r++) {
        #pragma omp parallel for schedule(dynamic, 256)
        for (int32_t q = src_round_off[r]; q < src_round_off[r + 1]; q++) push(peeled_src[q]);
    }
    for (size_t q = 0; q < seq_mid; q++) for (int32_t u : *seq_comps[q].second) push(u);
    if (c_giant >= 0) {
        #pragma omp parallel for schedule(dynamic, 256)
        for (size_t q = 0; q < cls_nodes[2].size(); q++) push(cls_nodes[2][q]);
    }
    for (size_t q = seq_mid; q < seq_comps.size(); q++) for (int32_t u : *seq_comps[q].second) push(u);
    for (int64_t r = (int64_t)snk_round_off.size() - 2; r >= 0; r--) {
        #pragma omp parallel for schedule(dynamic, 256)
        for (int32_t q = snk_round_off[r]; q < snk_round_off[r + 1]; q++) push(peeled_snk[q]);
    }
    (void)c_src_end;
    (void)snk_comp_base;
    phase("dag: layers");
    R.layer.assign(P, 0);
    R.scc.assign(P, 0);
    for (int64_t i = 0; i < P; i++) {
        R.layer[i] = f[comp[i]];
        R.scc[i] = minpath[comp[i]];
        R.n_layers = std::max(R.n_layers, f[comp[i]] + 1);
    }
    for (int64_t c = 0; c < nc; c++)
        if (npaths[c] > 0) { R.n_dep_sccs++; R.giant = std::max(R.giant, npaths[c]); }
}

}  // namespace

void build_layouts(const HostCSR& g, const dg_path_params& p, const std::vector<int>& ranks,
                   const std::function<void(int, HostLayout&)>& emit) {
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
    HostLayout L;
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
        static thread_local std::vector<std::pair<int32_t, int32_t>> tmp;
        tmp.resize(e - b);
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
    // ---- concatenate (subgraph order), in parallel over subgraphs
    rvec<int64_t> poff;
    rvec<int32_t> pv, pw;
    {
        std::vector<int64_t> voff(T + 1, 0), qoff(T + 1, 0);
        for (int k = 0; k < T; k++) {
            voff[k + 1] = voff[k] + (int64_t)subs[k].pv.size();
            qoff[k + 1] = qoff[k] + (int64_t)subs[k].start.size() - 1;
        }
        pv.resize(voff[T]); pw.resize(voff[T]);
        poff.resize(qoff[T] + 1);
        poff[0] = 0;
        #pragma omp parallel for schedule(dynamic, 1)
        for (int k = 0; k < T; k++) {
            SubOut& s2 = subs[k];
            std::copy(s2.pv.begin(), s2.pv.end(), pv.begin() + voff[k]);
            std::copy(s2.pw.begin(), s2.pw.end(), pw.begin() + voff[k]);
            for (size_t i = 1; i < s2.start.size(); i++) poff[qoff[k] + i] = voff[k] + s2.start[i];
            std::vector<int32_t>().swap(s2.pv);
            std::vector<int32_t>().swap(s2.pw);
            std::vector<int64_t>().swap(s2.start);
        }
    }
    phase("concatenate: copy");
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
        // paths by end vertex / by start vertex, each bucket in path order
        std::vector<int64_t> eptr, sptr;
        rvec<int32_t> elist, slist;
        group_by(P0, n, [&](int64_t i, auto&& sink) { sink(pv[poff[i + 1] - 1], (int32_t)i); }, eptr, elist);
        group_by(P0, n, [&](int64_t i, auto&& sink) { sink(pv[poff[i]], (int32_t)i); }, sptr, slist);
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
    phase("merge: pairing");
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
        // chains from their heads are disjoint; each thread walks 16 of them
        // round-robin so 16 independent pointer-chasing misses are in flight
        // (segment order is irrelevant: segments are sorted by first piece below)
        #pragma omp parallel
        {
            const int t = omp_get_thread_num(), T = omp_get_num_threads();
            constexpr int K = 16;
            struct Cur { int32_t j = -1; int64_t len = 0; int32_t cnt = 0; std::vector<int32_t> pieces, sf, sl; };
            std::vector<Cur> cs(K);
            int64_t i = P0 * t / T;
            const int64_t iend = P0 * (t + 1) / T;
            int active = 0;
            auto start = [&](Cur& c) {
                while (i < iend && prv[i] != -1) i++;
                if (i >= iend) return false;
                c.j = (int32_t)i++; c.len = 0; c.cnt = 0;
                return true;
            };
            for (auto& c : cs) if (start(c)) active++;
            while (active) {
                for (auto& c : cs) {
                    if (c.j < 0) continue;
                    const int32_t j = c.j;
                    seen[j] = 1;
                    const int64_t e = poff[j + 1] - poff[j] - 1;
                    if (c.cnt && c.len + e > p.l_merge) { c.sl.push_back(c.cnt); c.cnt = 0; c.len = 0; }
                    if (!c.cnt) c.sf.push_back(j);
                    c.pieces.push_back(j);
                    c.cnt++; c.len += e;
                    const int32_t nj = nxt[j];
                    if (nj != -1) {
                        __builtin_prefetch(&nxt[nj]);
                        __builtin_prefetch(&poff[nj]);
                        c.j = nj;
                    } else {
                        c.sl.push_back(c.cnt);
                        tp[t].insert(tp[t].end(), c.pieces.begin(), c.pieces.end());
                        tf[t].insert(tf[t].end(), c.sf.begin(), c.sf.end());
                        tl[t].insert(tl[t].end(), c.sl.begin(), c.sl.end());
                        c.pieces.clear(); c.sf.clear(); c.sl.clear();
                        c.j = -1;
                        if (!start(c)) active--;
                    }
                }
            }
        }
        for (int t = 0; t < nth; t++) {
            seg_pieces.insert(seg_pieces.end(), tp[t].begin(), tp[t].end());
            seg_first.insert(seg_first.end(), tf[t].begin(), tf[t].end());
            seg_len.insert(seg_len.end(), tl[t].begin(), tl[t].end());
        }
        for (int64_t i = 0; i < P0; i++)
            if (!seen[i]) walk_chain((int32_t)i, seg_pieces, seg_first, seg_len);
    }
    { std::vector<int32_t>().swap(nxt); std::vector<int32_t>().swap(prv); std::vector<uint8_t>().swap(seen); }
    phase("merge: chains");
    const int64_t P = (int64_t)seg_first.size();
    std::vector<int64_t> seg_start(P + 1, 0);   // into seg_pieces
    for (int64_t s2 = 0; s2 < P; s2++) seg_start[s2 + 1] = seg_start[s2] + seg_len[s2];
    std::vector<int32_t> sorder(P);
    std::iota(sorder.begin(), sorder.end(), 0);
    __gnu_parallel::sort(sorder.begin(), sorder.end(), [&](int32_t a, int32_t b) { return seg_first[a] < seg_first[b]; });
    phase("merge: order");
    // materialise merged paths (merge order) in parallel
    std::vector<int64_t> moff(P + 1, 0);
    #pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < P; r++) {
        int64_t sgi = sorder[r], len = 1;
        for (int64_t q = seg_start[sgi]; q < seg_start[sgi + 1]; q++) len += poff[seg_pieces[q] + 1] - poff[seg_pieces[q]] - 1;
        moff[r + 1] = len;
    }
    for (int64_t r = 0; r < P; r++) moff[r + 1] += moff[r];
    rvec<int32_t> mv(moff[P]), mw(moff[P]);
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
    { rvec<int32_t>().swap(pv); rvec<int32_t>().swap(pw); }

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
    // ---- dependency graph G' and DAG sketch (reading R-DEP, R-LAYER)
    DagResult dag;
    {
        DepGraph DG(P, n, moff, mv);
        phase("dag: bipartite CSR");
        dependency_dag(DG, dag, phase);
    }
    const std::vector<int64_t>& layer_of_path = dag.layer;
    const std::vector<int64_t>& scc_label = dag.scc;
    const int64_t n_layers = dag.n_layers, n_dep_sccs = dag.n_dep_sccs, giant = dag.giant;

    phase("dependency DAG");
    // ---- priority Pri(p) = alpha*D(p)*N(p) - L(p)
    double dmax = 0; int64_t nmax = 0;
    for (int64_t i = 0; i < P; i++) { dmax = std::max(dmax, dbar[i]); nmax = std::max(nmax, nvert[i]); }
    const double alpha = (dmax > 0 && nmax > 0) ? 1.0 / (dmax * (double)nmax) : 0.0;
    std::vector<double> pri(P);
    for (int64_t i = 0; i < P; i++) pri[i] = alpha * dbar[i] * (double)nvert[i] - (double)layer_of_path[i];
    std::vector<int64_t> order(P);
    std::iota(order.begin(), order.end(), 0);
    __gnu_parallel::stable_sort(order.begin(), order.end(), [&](int64_t a, int64_t b) { return pri[a] > pri[b]; });

    // ---- partitions over the priority order (greedy, whole paths)
    // part_entries == 0: auto -- about 16K partitions (several per resident
    // warp of a 148-SM grid), between 512 and 2048 entries each (smaller
    // partitions only add dispatch round trips: R-MAT-16 SSSP 0.35 -> 0.30 ms
    // kernel time from 137- to 512-entry partitions)
    int64_t target = p.part_entries;
    if (target <= 0) {
        int64_t tot = 0;
        for (int64_t i = 0; i < P; i++) tot += nvert[i];
        target = std::min<int64_t>(2048, std::max<int64_t>(512, tot / 16384));
    }
    const int world = std::max(1, p.world), rank = p.rank;
    // ---- path -> rank placement (world > 1, placement 1; reading R-PLACE,
    // a dispatch unit goes to "the GPU with the most number
    // of its direct precursors"): paths in priority order, each to the rank
    // already holding most of its vertices among the ranks whose entry load
    // stays within 2 % of an even share (ties: the least loaded) -- a greedy
    // vertex-cut that keeps replicas (the boundary) few.  The order is then
    // regrouped rank by rank (priority order inside a rank) so a partition
    // never spans two ranks.  placement 0: partitions round-robin (below).
    std::vector<int32_t> grp_owner;  // owner rank of each group of `order` (placement 1)
    std::vector<int64_t> grp_first{0, P};
    if (world > 1 && p.placement == 1) {
        int64_t tot = 0;
        for (int64_t i = 0; i < P; i++) tot += nvert[i];
        const double cap = 1.02 * (double)tot / world;
        std::vector<uint64_t> pres(n, 0);
        std::vector<int64_t> load(world, 0), cnt(world);
        std::vector<int32_t> path_owner(P);
        for (int64_t r = 0; r < P; r++) {
            const int64_t i = order[r];
            std::fill(cnt.begin(), cnt.end(), 0);
            for (int64_t k = moff[i]; k < moff[i + 1]; k++)
                for (uint64_t b = pres[mv[k]]; b; b &= b - 1) cnt[__builtin_ctzll(b)]++;
            int best = -1;
            for (int w = 0; w < world; w++) {
                if ((double)(load[w] + nvert[i]) > cap) continue;
                if (best < 0 || cnt[w] > cnt[best] || (cnt[w] == cnt[best] && load[w] < load[best])) best = w;
            }
            if (best < 0) best = (int)(std::min_element(load.begin(), load.end()) - load.begin());
            path_owner[i] = best;
            load[best] += nvert[i];
            const uint64_t bit = 1ull << best;
            for (int64_t k = moff[i]; k < moff[i + 1]; k++) pres[mv[k]] |= bit;
        }
        std::vector<int64_t> grouped;
        grouped.reserve(P);
        grp_first.assign(1, 0);
        for (int w = 0; w < world; w++) {
            for (int64_t r = 0; r < P; r++)
                if (path_owner[order[r]] == w) grouped.push_back(order[r]);
            grp_first.push_back((int64_t)grouped.size());
            grp_owner.push_back(w);
        }
        order.swap(grouped);
    }
    // ---- partitions over the (grouped) priority order (greedy, whole paths)
    std::vector<int64_t> gpart_first{0};  // global partition -> first index in `order`
    std::vector<int32_t> owner;           // global partition -> rank
    for (size_t grp = 0; grp + 1 < grp_first.size(); grp++) {
        int64_t acc = 0;
        for (int64_t r = grp_first[grp]; r < grp_first[grp + 1]; r++) {
            if (acc >= target && r > gpart_first.back()) {
                gpart_first.push_back(r);
                owner.push_back(grp_owner.empty() ? 0 : grp_owner[grp]);
                acc = 0;
            }
            acc += nvert[order[r]];
        }
        if (grp_first[grp + 1] > gpart_first.back()) {
            gpart_first.push_back(grp_first[grp + 1]);
            owner.push_back(grp_owner.empty() ? 0 : grp_owner[grp]);
        }
    }
    if (P == 0) { gpart_first.assign(1, 0); owner.clear(); }
    const int64_t G = (int64_t)gpart_first.size() - 1;
    if (grp_owner.empty())  // placement 0 (or one rank): round-robin over the priority order
        for (int64_t q = 0; q < G; q++) owner[q] = (int32_t)(q % world);

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

    // ---- the boundary: vertices present in partitions of more than one rank
    if (world > 1) {
        std::vector<uint64_t> present(n, 0);  // ranks whose partitions hold v
        for (int64_t q = 0; q < G; q++) {
            const uint64_t bit = 1ull << owner[q];
            for (int64_t r = gpart_first[q]; r < gpart_first[q + 1]; r++) {
                const int64_t i = order[r];
                for (int64_t k = moff[i]; k < moff[i + 1]; k++) present[mv[k]] |= bit;
            }
        }
        // boundary vertices (internal ids, ascending) and their holder ranks
        std::vector<std::pair<int32_t, uint64_t>> bh;
        for (int64_t v = 0; v < n; v++)
            if (__builtin_popcountll(present[v]) > 1) bh.emplace_back(L.new_id[v], present[v]);
        std::sort(bh.begin(), bh.end());
        for (const auto& x : bh) {
            L.boundary.push_back(x.first);
            L.bnd_hold.push_back(x.second);
        }
    }

    // per-vertex sum of out-edge weights (Adsorption's W(u), reading R-ADS), so
    // a layout needs no CSR on the device for it
    L.wsum.assign(n, 0.f);
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < n; u++) {
        double ws = 0;
        for (int64_t e = L.prow_ptr[u]; e < L.prow_ptr[u + 1]; e++) ws += g.has_w ? (double)L.pw[e] : 1.0;
        L.wsum[u] = (float)ws;
    }
    L.n_layers = n_layers;
    L.n_dep_sccs = n_dep_sccs;
    L.giant = giant;

    phase("priority+partitions");
    // ---- each requested rank's layout (the steps above ran once for all)
    for (const int rank : ranks) {
        L.params.rank = rank;
        L.path_off.clear(); L.part_off.clear();
        // this rank's paths (priority order within its partitions) and offsets
        std::vector<int64_t> sel;
        L.part_off.push_back(0);
        std::vector<int64_t> part_paths{0};
        for (int64_t q = 0; q < G; q++) {
            if (owner[q] != rank) continue;
            for (int64_t r = gpart_first[q]; r < gpart_first[q + 1]; r++) sel.push_back(order[r]);
            part_paths.push_back((int64_t)sel.size());
        }
        const int64_t Q = (int64_t)sel.size();
        L.path_off.assign(Q + 1, 0);
        for (int64_t r = 0; r < Q; r++) L.path_off[r + 1] = L.path_off[r] + (moff[sel[r] + 1] - moff[sel[r]]);
        for (size_t q = 1; q < part_paths.size(); q++) L.part_off.push_back(L.path_off[part_paths[q]]);
        L.e_idx.resize(L.path_off[Q]);
        L.e_w.resize(L.path_off[Q]);
        L.layer.resize(Q); L.scc.resize(Q); L.merged_index.resize(Q); L.hot.resize(Q);
        int64_t nh = 0;
        #pragma omp parallel for schedule(dynamic, 1024) reduction(+ : nh)
        for (int64_t r = 0; r < Q; r++) {
            const int64_t i = sel[r];
            int64_t o = L.path_off[r];
            for (int64_t k = moff[i]; k < moff[i + 1]; k++, o++) {
                uint32_t code = (uint32_t)L.new_id[mv[k]];
                if (k == moff[i]) code |= kHead;
                if (k == moff[i + 1] - 1) code |= kTail;
                L.e_idx[o] = code;
                L.e_w[o] = mw[k];
            }
            L.layer[r] = (int32_t)layer_of_path[i];
            L.scc[r] = scc_label[i];
            L.merged_index[r] = i;
            L.hot[r] = hot[i];
            nh += hot[i];
        }
        L.n_hot = nh;
        L.built = true;
        L.preprocess_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        phase("layout");
        emit(rank, L);
    }
}

void build_layout(const HostCSR& g, const dg_path_params& p, HostLayout& out) {
    build_layouts(g, p, {p.rank}, [&](int, HostLayout& L) { out = std::move(L); });
}

}  // namespace dg
