"""Oracle vertex programs (test infrastructure only -- see oracle/__init__.py).

Every routine is the plain synchronous (Jacobi) definition of the iterative
algorithm the paper benchmarks (sec. 4, "four iterative directed graph
algorithms ... (1) pagerank [29]; (2) adsorption [3]; (3) SSSP [28]") plus the
label-propagation WCC / SCC rows of BASELINE.json's north_star.  All
algorithms "execute until convergence" (sec. 4).

Graph convention: ``n`` vertices 0..n-1 and a directed edge list
``src[k] -> dst[k]`` (numpy int64), optional integer weights ``w[k]``.
Duplicate edges are kept (they count in out-degrees); self loops are allowed.

No code here is shared with, or imported from, the CUDA path.
"""
from __future__ import annotations

import numpy as np

# DESIGN.md reading R-INF: an unreachable vertex reports 2**31 - 1.
UNREACHED = 2**31 - 1


def _edges(src, dst, w=None):
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    if w is not None:
        w = np.asarray(w, dtype=np.int64)
    return src, dst, w


# ---------------------------------------------------------------------------
# SSSP -- synchronous Bellman-Ford (min-plus relaxation), sec. 2
# ("executing SSSP ... the shortest distance from v1 to v2") and sec. 4 (3).
# ---------------------------------------------------------------------------
def sssp_bellman_ford(n, src, dst, w, source, max_rounds=None):
    """dist[v] = min over paths source~>v of the summed integer weights.

    Jacobi rounds: every round relaxes every edge from the previous round's
    distances, dist'[v] = min(dist[v], min_{u->v} dist[u] + w(u,v)), until no
    distance changes.  Returns (dist int64 with UNREACHED, rounds).
    """
    src, dst, w = _edges(src, dst, w)
    if w is None:
        w = np.ones_like(src)
    if np.any(w < 0):
        raise ValueError("Bellman-Ford oracle: negative weights are out of scope")
    dist = np.full(n, UNREACHED, dtype=np.int64)
    if n == 0:
        return dist, 0
    dist[source] = 0
    rounds = 0
    limit = n if max_rounds is None else max_rounds
    while rounds < limit + 1:
        rounds += 1
        reached = dist[src] < UNREACHED
        cand = dist[src[reached]] + w[reached]
        new = dist.copy()
        np.minimum.at(new, dst[reached], cand)
        if np.array_equal(new, dist):
            return dist, rounds
        dist = new
    raise RuntimeError("Bellman-Ford did not converge")


def bfs_levels(n, src, dst, source):
    """Hop distance from ``source`` (level-synchronous frontier BFS).

    BFS is SSSP with unit weights (north_star "SSSP/BFS min-plus relaxation");
    written here as the textbook frontier expansion so it does not reuse the
    Bellman-Ford routine.  Unreached vertices report UNREACHED.
    """
    src, dst, _ = _edges(src, dst)
    level = np.full(n, UNREACHED, dtype=np.int64)
    if n == 0:
        return level
    # adjacency lists in plain Python for obviousness
    adj = [[] for _ in range(n)]
    for a, b in zip(src.tolist(), dst.tolist()):
        adj[a].append(b)
    level[source] = 0
    frontier = [source]
    depth = 0
    while frontier:
        depth += 1
        nxt = []
        for u in frontier:
            for v in adj[u]:
                if level[v] == UNREACHED:
                    level[v] = depth
                    nxt.append(v)
        frontier = nxt
    return level


# ---------------------------------------------------------------------------
# PageRank -- PAPER.md sec. 4 benchmark (1) pagerank [29]; d = 0.85
# (BASELINE.json north_star).  DESIGN.md reading R-PR: the textbook
# stochastic PageRank, teleport (1-d)/n, dangling mass spread uniformly,
# so the rank vector sums to 1.
# ---------------------------------------------------------------------------
def pagerank_power(n, src, dst, d=0.85, tol=1e-12, max_iter=100000):
    """fp64 power iteration  r' = (1-d)/n + d*(sum_{u->v} r_u/outdeg(u) + D/n)
    where D = sum of r over dangling (outdeg 0) vertices.  Iterates until the
    L1 change between iterates is <= tol.  Returns (r, iterations)."""
    src, dst, _ = _edges(src, dst)
    if n == 0:
        return np.zeros(0), 0
    outdeg = np.bincount(src, minlength=n).astype(np.float64)
    dangling = outdeg == 0
    r = np.full(n, 1.0 / n)
    for it in range(1, max_iter + 1):
        share = np.zeros(n)
        np.add.at(share, dst, r[src] / outdeg[src])
        dmass = r[dangling].sum()
        new = (1.0 - d) / n + d * (share + dmass / n)
        diff = np.abs(new - r).sum()
        r = new
        if diff <= tol:
            return r, it
    raise RuntimeError("PageRank power iteration did not converge")


# ---------------------------------------------------------------------------
# Adsorption -- PAPER.md sec. 4 benchmark (2) adsorption [3] (Baluja et al.).
# DESIGN.md reading R-ADS: the scalar accumulative form used by graph
# systems:  x_v = p_inj(v) * I(v) + sum_{u->v} p_cont(u) * w(u,v)/W(u) * x_u,
# W(u) = sum of u's out-edge weights.  Converges because p_cont < 1.
# ---------------------------------------------------------------------------
def adsorption_jacobi(n, src, dst, w, p_inj, p_cont, inj, tol=1e-12, max_iter=100000):
    src, dst, w = _edges(src, dst, w)
    if w is None:
        w = np.ones_like(src)
    p_inj = np.asarray(p_inj, dtype=np.float64)
    p_cont = np.asarray(p_cont, dtype=np.float64)
    inj = np.asarray(inj, dtype=np.float64)
    wout = np.zeros(n)
    np.add.at(wout, src, w.astype(np.float64))
    coef = p_cont[src] * w / wout[src]
    base = p_inj * inj
    x = base.copy()
    for it in range(1, max_iter + 1):
        acc = np.zeros(n)
        np.add.at(acc, dst, coef * x[src])
        new = base + acc
        diff = np.abs(new - x).sum()
        x = new
        if diff <= tol:
            return x, it
    raise RuntimeError("Adsorption Jacobi iteration did not converge")


# ---------------------------------------------------------------------------
# WCC -- north_star "WCC/SCC label propagation".  DESIGN.md reading R-CC:
# a vertex's label is the smallest vertex id in its component.
# ---------------------------------------------------------------------------
def wcc_label_propagation(n, src, dst):
    """Jacobi min-label propagation over both directions of every edge."""
    src, dst, _ = _edges(src, dst)
    label = np.arange(n, dtype=np.int64)
    rounds = 0
    while True:
        rounds += 1
        new = label.copy()
        np.minimum.at(new, dst, label[src])
        np.minimum.at(new, src, label[dst])
        if np.array_equal(new, label):
            return label, rounds
        label = new


def scc_tarjan(n, src, dst):
    """Tarjan's algorithm [40] (sec. 3.2.1 uses it for the DAG
    sketch), written iteratively.  Returns label[v] = smallest vertex id of
    v's strongly connected component."""
    src, dst, _ = _edges(src, dst)
    adj = [[] for _ in range(n)]
    for a, b in zip(src.tolist(), dst.tolist()):
        adj[a].append(b)
    index = [-1] * n
    low = [0] * n
    on_stack = [False] * n
    stack = []
    comp = [-1] * n
    counter = 0
    for root in range(n):
        if index[root] != -1:
            continue
        work = [(root, 0)]
        index[root] = low[root] = counter
        counter += 1
        stack.append(root)
        on_stack[root] = True
        while work:
            v, i = work[-1]
            if i < len(adj[v]):
                work[-1] = (v, i + 1)
                u = adj[v][i]
                if index[u] == -1:
                    index[u] = low[u] = counter
                    counter += 1
                    stack.append(u)
                    on_stack[u] = True
                    work.append((u, 0))
                elif on_stack[u]:
                    low[v] = min(low[v], index[u])
            else:
                work.pop()
                if work:
                    p = work[-1][0]
                    low[p] = min(low[p], low[v])
                if low[v] == index[v]:
                    members = []
                    while True:
                        x = stack.pop()
                        on_stack[x] = False
                        members.append(x)
                        if x == v:
                            break
                    m = min(members)
                    for x in members:
                        comp[x] = m
    return np.asarray(comp, dtype=np.int64)
