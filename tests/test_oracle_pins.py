"""Pins for the oracle (-m "not gpu"): each oracle routine is checked against
something other than itself -- brute force on tiny inputs, dense linear
solves, closed forms, the paper's Figure 4 worked example, invariants.  A
plausible slip in the oracle (dropped term, wrong sign/index, transposed
operand) fails at least one test here.
"""
import heapq
import itertools
import os

import numpy as np
import pytest

from oracle import algorithms as A
from oracle import paths as P

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def rand_graph(n, m, seed, wmax=255, self_loops=True):
    rng = np.random.default_rng(seed)
    src = rng.integers(0, n, m)
    dst = rng.integers(0, n, m)
    if not self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    w = rng.integers(1, wmax + 1, len(src))
    return src.astype(np.int64), dst.astype(np.int64), w.astype(np.int64)


def to_csr(n, src, dst, w=None):
    order = np.lexsort((dst, src))
    row_ptr = np.zeros(n + 1, np.int64)
    np.add.at(row_ptr, src + 1, 1)
    row_ptr = np.cumsum(row_ptr)
    return row_ptr, dst[order], (None if w is None else w[order]), src[order]


# ------------------------------------------------------------------ SSSP / BFS
def dijkstra(n, src, dst, w, s):
    adj = [[] for _ in range(n)]
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        adj[a].append((b, c))
    dist = [None] * n
    pq = [(0, s)]
    while pq:
        d, u = heapq.heappop(pq)
        if dist[u] is not None:
            continue
        dist[u] = d
        for v, c in adj[u]:
            if dist[v] is None:
                heapq.heappush(pq, (d + c, v))
    return np.array([A.UNREACHED if x is None else x for x in dist], dtype=np.int64)


def floyd_warshall(n, src, dst, w):
    INF = float("inf")
    D = np.full((n, n), INF)
    np.fill_diagonal(D, 0)
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        D[a, b] = min(D[a, b], c)
    for k in range(n):
        D = np.minimum(D, D[:, [k]] + D[[k], :])
    return D


@pytest.mark.parametrize("seed", range(6))
def test_sssp_vs_dijkstra(seed):
    n = 60 + 10 * seed
    src, dst, w = rand_graph(n, 4 * n, seed)
    got, _ = A.sssp_bellman_ford(n, src, dst, w, 0)
    assert np.array_equal(got, dijkstra(n, src, dst, w, 0))


def test_sssp_vs_floyd_warshall_all_sources():
    n = 14
    src, dst, w = rand_graph(n, 30, 7, wmax=9)
    D = floyd_warshall(n, src, dst, w)
    for s in range(n):
        got, _ = A.sssp_bellman_ford(n, src, dst, w, s)
        exp = np.where(np.isinf(D[s]), A.UNREACHED, D[s]).astype(np.int64)
        assert np.array_equal(got, exp)


def test_sssp_hand_example_and_special_cases():
    # 0 -5-> 1 -1-> 2 ; 0 -9-> 2 ; 3 isolated: dist 2 must use the 2-hop route
    got, _ = A.sssp_bellman_ford(4, [0, 1, 0], [1, 2, 2], [5, 1, 9], 0)
    assert got.tolist() == [0, 5, 6, A.UNREACHED]
    # empty edge set
    got, _ = A.sssp_bellman_ford(3, [], [], [], 1)
    assert got.tolist() == [A.UNREACHED, 0, A.UNREACHED]
    # directed n-chain with unit weights: dist = index
    n = 40
    got, rounds = A.sssp_bellman_ford(n, np.arange(n - 1), np.arange(1, n), np.ones(n - 1), 0)
    assert got.tolist() == list(range(n))
    assert rounds == n  # Jacobi needs one round per hop + the quiescent round


@pytest.mark.parametrize("seed", range(4))
def test_bfs_vs_floyd_warshall(seed):
    n = 25
    src, dst, _ = rand_graph(n, 45, 100 + seed)
    D = floyd_warshall(n, src, dst, np.ones_like(src))
    got = A.bfs_levels(n, src, dst, 3)
    exp = np.where(np.isinf(D[3]), A.UNREACHED, D[3]).astype(np.int64)
    assert np.array_equal(got, exp)


# ------------------------------------------------------------------ PageRank
def pagerank_dense_solve(n, src, dst, d=0.85):
    """Stationary vector of the Google matrix via one dense linear solve."""
    M = np.zeros((n, n))
    outdeg = np.bincount(src, minlength=n)
    for a, b in zip(src.tolist(), dst.tolist()):
        M[a, b] += 1.0 / outdeg[a]
    M[outdeg == 0, :] = 1.0 / n          # dangling rows -> uniform
    # r = (1-d)/n 1 + d M^T r
    return np.linalg.solve(np.eye(n) - d * M.T, np.full(n, (1 - d) / n))


def test_pagerank_cycle_closed_form():
    for n in (1, 2, 7, 50):
        r, _ = A.pagerank_power(n, np.arange(n), (np.arange(n) + 1) % n)
        assert np.allclose(r, 1.0 / n, rtol=0, atol=1e-13)


@pytest.mark.parametrize("seed", range(5))
def test_pagerank_vs_dense_solve(seed):
    n = 30 + 7 * seed
    src, dst, _ = rand_graph(n, 3 * n, 200 + seed)
    r, _ = A.pagerank_power(n, src, dst)
    exp = pagerank_dense_solve(n, src, dst)
    # contraction factor d: ||r_k - r*||_1 <= d/(1-d) * ||r_k - r_(k-1)||_1
    # <= 0.85/0.15 * 1e-12 (+ rounding of the dense solve)
    assert np.abs(r - exp).sum() < 0.85 / 0.15 * 1e-12 + 1e-13
    assert abs(r.sum() - 1.0) < 1e-12            # rank mass sums to 1


def test_pagerank_asymmetric_two_vertex():
    # 0 -> 1, vertex 1 dangling.  Closed form by hand:
    # r0 = (1-d)/2 + d*r1/2 ; r1 = (1-d)/2 + d*(r0 + r1/2)
    d = 0.85
    r, _ = A.pagerank_power(2, [0], [1], d=d)
    # solve the 2x2 system by Cramer's rule
    a11, a12, b1 = 1.0, -d / 2, (1 - d) / 2
    a21, a22, b2 = -d, 1 - d / 2, (1 - d) / 2
    det = a11 * a22 - a12 * a21
    r0 = (b1 * a22 - a12 * b2) / det
    r1 = (a11 * b2 - a21 * b1) / det
    assert abs(r[0] - r0) < 1e-13 and abs(r[1] - r1) < 1e-13
    assert r[1] > r[0]


# ------------------------------------------------------------------ Adsorption
@pytest.mark.parametrize("seed", range(3))
def test_adsorption_vs_dense_solve(seed):
    n = 40
    src, dst, w = rand_graph(n, 150, 300 + seed, wmax=9)
    rng = np.random.default_rng(seed)
    p_cont = rng.uniform(0.1, 0.8, n)
    p_inj = rng.uniform(0.0, 1.0 - p_cont)
    inj = rng.uniform(0, 1, n)
    x, _ = A.adsorption_jacobi(n, src, dst, w, p_inj, p_cont, inj)
    wout = np.bincount(src, weights=w, minlength=n)
    M = np.zeros((n, n))
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        M[a, b] += p_cont[a] * c / wout[a]
    exp = np.linalg.solve(np.eye(n) - M.T, p_inj * inj)
    assert np.abs(x - exp).max() < 1e-11


# ------------------------------------------------------------------ WCC / SCC
def union_find_labels(n, src, dst):
    parent = list(range(n))

    def find(x):
        while parent[x] != x:
            parent[x] = parent[parent[x]]
            x = parent[x]
        return x
    for a, b in zip(src.tolist(), dst.tolist()):
        ra, rb = find(a), find(b)
        if ra != rb:
            parent[max(ra, rb)] = min(ra, rb)
    roots = [find(x) for x in range(n)]
    mins = {}
    for v, r in enumerate(roots):
        mins[r] = min(mins.get(r, v), v)
    return np.array([mins[r] for r in roots], dtype=np.int64)


@pytest.mark.parametrize("seed", range(5))
def test_wcc_vs_union_find(seed):
    n = 80
    src, dst, _ = rand_graph(n, 50 + 10 * seed, 400 + seed)
    got, _ = A.wcc_label_propagation(n, src, dst)
    assert np.array_equal(got, union_find_labels(n, src, dst))


def closure_scc_labels(n, src, dst):
    R = np.eye(n, dtype=bool)
    R[src, dst] = True
    for k in range(n):  # Warshall transitive closure
        R = R | (R[:, [k]] & R[[k], :])
    both = R & R.T
    return np.array([int(np.nonzero(both[v])[0].min()) for v in range(n)], dtype=np.int64)


@pytest.mark.parametrize("seed", range(6))
def test_scc_vs_transitive_closure(seed):
    n = 30
    src, dst, _ = rand_graph(n, 35 + 5 * seed, 500 + seed)
    assert np.array_equal(A.scc_tarjan(n, src, dst), closure_scc_labels(n, src, dst))


def test_scc_vs_scipy_medium():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import connected_components
    n = 3000
    src, dst, _ = rand_graph(n, 4500, 77)
    got = A.scc_tarjan(n, src, dst)
    _, lab = connected_components(csr_matrix((np.ones(len(src)), (src, dst)), shape=(n, n)),
                                  directed=True, connection="strong")
    # same partition: canonical min-id labels agree
    mins = {}
    for v, l in enumerate(lab.tolist()):
        mins[l] = min(mins.get(l, v), v)
    assert np.array_equal(got, np.array([mins[l] for l in lab.tolist()]))


# ------------------------------------------------------------------ Algorithm 1
def load_fig4():
    n, edges, paths, inner, deps, layer = 0, [], [], set(), [], None
    with open(os.path.join(GOLDEN, "fig4_example.txt")) as f:
        for line in f:
            t = line.split()
            if not t or t[0].startswith("#"):
                continue
            if t[0] == "n":
                n = int(t[1])
            elif t[0] == "edge":
                edges.append((int(t[1]), int(t[2])))
            elif t[0] == "path":
                paths.append([int(x) for x in t[1:]])
            elif t[0] == "inner":
                inner |= {int(x) for x in t[1:]}
            elif t[0] == "dep":
                deps.append((int(t[1]), int(t[2])))
            elif t[0] == "layer":
                layer = [int(x) for x in t[1:]]
    return n, edges, paths, inner, deps, layer


def test_algorithm1_reproduces_figure4():
    n, edges, paths, inner, deps, layer = load_fig4()
    src = np.array([e[0] for e in edges]); dst = np.array([e[1] for e in edges])
    row_ptr, col, _, _ = to_csr(n, src, dst)
    got, got_inner = P.graphp_decompose(n, row_ptr, col, d_max=16, n_sub=1, order="id")
    assert got == paths
    assert got_inner == inner
    dep = P.dependency_graph(got)
    assert dep == sorted(deps)
    scc, lay = P.condense_and_layer(len(got), dep)
    assert lay.tolist() == layer
    assert scc.tolist() == [0, 1, 2, 1]


def check_cover(n, src, dst, paths):
    """Every edge covered by exactly one path edge (multiset equality)."""
    got = sorted((p[t], p[t + 1]) for p in paths for t in range(len(p) - 1))
    exp = sorted(zip(src.tolist(), dst.tolist()))
    return got == exp


@pytest.mark.parametrize("seed,n_sub,order", list(itertools.product(range(4), (1, 3), ("degree", "id"))))
def test_algorithm1_is_an_edge_disjoint_cover(seed, n_sub, order):
    n = 120
    src, dst, _ = rand_graph(n, 600, 600 + seed)
    row_ptr, col, _, s_sorted = to_csr(n, src, dst)
    paths, inner = P.graphp_decompose(n, row_ptr, col, d_max=16, n_sub=n_sub, order=order)
    assert check_cover(n, src, dst, paths)
    assert all(2 <= len(p) <= 17 for p in paths)          # 1..D_MAX edges
    merged = P.merge_short_paths(n, src, dst, paths, inner, l_max=64)
    assert check_cover(n, src, dst, merged)
    assert all(len(p) - 1 <= 64 for p in merged)
    assert len(merged) <= len(paths)


def test_subgraph_bounds_hand_example():
    """Reading R-SUB by hand: lo_k = first v with row_ptr[v] >= floor(k*m/T).
    out-degrees [4, 0, 1, 1, 2, 0], m = 8, T = 4: targets 2, 4, 6 -> v = 1,
    1, 4 (row_ptr = [0, 4, 4, 5, 6, 8, 8])."""
    row_ptr = np.array([0, 4, 4, 5, 6, 8, 8])
    assert P.subgraph_bounds(6, row_ptr, 4) == [0, 1, 1, 4, 6]
    assert P.subgraph_bounds(6, row_ptr, 1) == [0, 6]
    assert P.subgraph_bounds(3, np.array([0, 0, 0, 0]), 3) == [0, 0, 0, 3]  # no edges


def test_algorithm1_subgraphs_split_paths_by_hand():
    """Each thread divides only its local subgraph: an edge
    belongs to the subgraph of its source, and a traversal stops at a vertex
    of another subgraph (no local edges -> line 19).  Chain 0->1->2->3->4,
    order "id", derived by hand: T=1 one path; T=2 (bounds [0,2,5]) splits at
    vertex 2; T=3 (bounds [0,1,2,5]) splits at 1 and 2."""
    n = 5
    src = np.arange(4); dst = np.arange(1, 5)
    row_ptr, col, _, _ = to_csr(n, src, dst)
    run = lambda t: P.graphp_decompose(n, row_ptr, col, d_max=16, n_sub=t, order="id")[0]
    assert run(1) == [[0, 1, 2, 3, 4]]
    assert run(2) == [[0, 1, 2], [2, 3, 4]]
    assert run(3) == [[0, 1], [1, 2], [2, 3, 4]]


def test_algorithm1_depth_bound_on_chain():
    n = 41  # chain 0 -> 1 -> ... -> 40
    src = np.arange(40); dst = np.arange(1, 41)
    row_ptr, col, _, _ = to_csr(n, src, dst)
    paths, inner = P.graphp_decompose(n, row_ptr, col, d_max=16, order="degree")
    # roots by (degree desc, id): 1 first (deg 2); DFS stops at depth 16 (v17),
    # v17 and v33 become later roots, v0 (deg 1) last and hits the visited v1.
    assert [p[0] for p in paths] == [1, 17, 33, 0]
    assert [len(p) - 1 for p in paths] == [16, 16, 7, 1]
    assert inner == {1}
    merged = P.merge_short_paths(n, src, dst, paths, inner, l_max=64)
    assert merged == [list(range(1, 41))] + [] or merged == [[0] + list(range(1, 41))] \
        or sorted(len(p) - 1 for p in merged) == [1, 39]
    # indeg(1)=1 so the inner constraint does not block the merge at v1:
    # path [0,1] absorbs the chain starting at 1 once earlier paths are done.
    assert check_cover(n, src, dst, merged)


def test_merge_respects_inner_constraint():
    # x=2 has in- and out-degree 2 and is inner -> no merge through x
    n = 6
    src = np.array([0, 1, 2, 2, 3]); dst = np.array([2, 2, 4, 5, 1])
    paths = [[0, 2], [2, 4], [1, 2], [2, 5], [3, 1]]
    out = P.merge_short_paths(n, src, dst, paths, inner={2}, l_max=64)
    # nothing merges through the inner hub 2; [3,1] may absorb [1,2] (indeg(1)=1)
    assert out == [[0, 2], [2, 4], [2, 5], [3, 1, 2]]
    out2 = P.merge_short_paths(n, src, dst, paths, inner=set(), l_max=64)
    assert out2 == [[0, 2, 4], [3, 1, 2, 5]]
    # links by hand: at x=1 path4->path2; at x=2 (ends [0,2], starts [1,3])
    # path0->path1, path2->path3.  Chains [0,1] and [4,2,3]; the cap of 2 edges
    # cuts the second after [3,1,2]; segments ordered by first piece 0, 3, 4.
    out3 = P.merge_short_paths(n, src, dst, paths, inner=set(), l_max=2)
    assert out3 == [[0, 2, 4], [2, 5], [3, 1, 2]]


# ------------------------------------------------------------------ dependency DAG
def brute_reach(k, edges):
    R = np.eye(k, dtype=bool)
    for a, b in edges:
        R[a, b] = True
    for m in range(k):
        R = R | (R[:, [m]] & R[[m], :])
    return R


@pytest.mark.parametrize("seed", range(4))
def test_dependency_layers_are_longest_path_layers(seed):
    n = 60
    src, dst, _ = rand_graph(n, 90, 700 + seed, self_loops=False)
    row_ptr, col, _, _ = to_csr(n, src, dst)
    paths, inner = P.graphp_decompose(n, row_ptr, col, d_max=4)
    dep = P.dependency_graph(paths)
    # dependency edges by brute force from the definition
    k = len(paths)
    brute = set()
    for i, j in itertools.product(range(k), range(k)):
        if i != j and set(paths[i][1:]) & set(paths[j][:-1]):
            brute.add((i, j))
    assert set(dep) == brute
    scc, layer = P.condense_and_layer(k, dep)
    R = brute_reach(k, dep)
    for i, j in itertools.product(range(k), range(k)):
        assert (scc[i] == scc[j]) == (R[i, j] and R[j, i])
    for i, j in dep:
        if scc[i] != scc[j]:
            assert layer[i] < layer[j]
    for c in set(scc.tolist()):  # tightness: an SCC at layer L>0 has a predecessor SCC at L-1
        lc = layer[scc == c][0]
        assert np.all(layer[scc == c] == lc)
        if lc > 0:
            assert any(scc[j] == c and scc[i] != c and layer[i] == lc - 1 for i, j in dep)
    # independently: peel the condensation (built from the brute-force
    # reachability) source layer by source layer (Kahn by rounds) -- round t
    # removes exactly the SCCs whose longest chain of predecessors has t SCCs
    comp = {}
    for i in range(k):
        comp.setdefault(frozenset(j for j in range(k) if R[i, j] and R[j, i]) | {i}, []).append(i)
    cid = {i: c for c, members in enumerate(comp.values()) for i in members}
    preds = {c: set() for c in range(len(comp))}
    for i, j in brute:
        if cid[i] != cid[j]:
            preds[cid[j]].add(cid[i])
    peel, left, t = {}, set(preds), 0
    while left:
        src_now = {c for c in left if not (preds[c] & left)}
        assert src_now  # a DAG always has a source
        for c in src_now:
            peel[c] = t
        left -= src_now
        t += 1
    assert all(layer[i] == peel[cid[i]] for i in range(k))


def test_priority_orders_layers_first():
    dbar = np.array([1.0, 50.0, 3.0]); nv = np.array([10, 2, 5]); layer = np.array([1, 2, 0])
    pri = P.priority(dbar, nv, layer)
    assert np.argsort(-pri, kind="stable").tolist() == [2, 0, 1]
    assert np.all((pri + layer > 0) & (pri + layer <= 1))


def test_path_stats_on_figure4():
    n, edges, paths, *_ = load_fig4()
    src = np.array([e[0] for e in edges]); dst = np.array([e[1] for e in edges])
    dbar, nv, hot = P.path_stats(n, src, dst, paths, hot_factor=1.25)
    # degrees (in+out) by hand: v0 1, v1 2, v2 2, v3 3, v4 2, v5 1, v6 3, v7 3,
    # v8 3, v9 1, v10 2, v11 2, v12 1, v13 2, v14 2; mean degree 2*15/15 = 2
    assert np.allclose(dbar, [11 / 6, 13 / 5, 2.0, 2.5])
    assert nv.tolist() == [6, 5, 4, 4]
    assert hot.tolist() == [False, True, False, True]   # threshold 2.5


@pytest.mark.parametrize("seed", range(6))
def test_relaxed_merge_is_maximal(seed):
    """Reading R-MERGE, relaxed rule, no length cap: the merge links pieces
    at every vertex until one side runs out, so afterwards no vertex has
    both a merged path that only ends there and one that only starts there;
    paths that start and end at the same vertex (a closed piece, or a cycle
    of links cut there -- the cut frees an end and a start of the same path)
    are exempt.  A merge that skipped a possible link, or linked pieces that
    do not meet, fails this or the cover check."""
    n = 80
    src, dst, _ = rand_graph(n, 400, 900 + seed, self_loops=False)
    row_ptr, col, _, _ = to_csr(n, src, dst)
    paths, inner = P.graphp_decompose(n, row_ptr, col, d_max=4)
    merged = P.merge_short_paths(n, src, dst, paths, set(), l_max=1 << 30)
    assert check_cover(n, src, dst, merged)
    ends, starts = {}, {}
    for i, p in enumerate(merged):
        ends.setdefault(p[-1], set()).add(i)
        starts.setdefault(p[0], set()).add(i)
    for x in set(ends) & set(starts):
        only_end, only_start = ends[x] - starts[x], starts[x] - ends[x]
        assert not (only_end and only_start), (x, ends[x], starts[x])
    # and the merge really merged: every piece boundary inside a merged path joins at one vertex
    assert len(merged) < len(paths)
