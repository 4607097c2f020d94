"""Oracle for DiGraph's preprocessing rows (test infrastructure only).

Follows PAPER.md sec. 3.1 / 3.2.1 / 3.2.3 step by step, in the paper's order
and notation, for small graphs:

  graphp_decompose   -- Algorithm 1 "Path-based Graph Partitioning on CPU"
                        (PAPER.md lines 118-145), one DFS forest per subgraph.
  merge_short_paths  -- head-to-tail merging of short paths with the
                        inner-vertex constraint.
  path_stats         -- average vertex degree D(p), hot/cold class, N(p)
                        (PAPER.md lines 112, 192).
  dependency_graph   -- G' = (V', E'), <p_i, p_j> when some v is entered by an
                        edge of p_i and left by an edge of p_j.
  condense_and_layer -- DAG sketch G'' by contracting SCCs of G' (Tarjan [40],
                        PAPER.md line 159) and layer numbers.
  priority           -- Pri(p) = alpha * D(p) * N(p) - L(p),
                        alpha = 1/(Dmax * Nmax).

Where the paper is silent the DESIGN.md reading is named in the docstring.
Nothing here is shared with the CUDA/C++ product path.
"""
from __future__ import annotations

from collections import defaultdict

import numpy as np

D_MAX_DEFAULT = 16  # "its maximum value is D_MAX=16 by default"


def _degrees(n, src, dst):
    outdeg = np.bincount(src, minlength=n).astype(np.int64)
    indeg = np.bincount(dst, minlength=n).astype(np.int64)
    return indeg, outdeg


def subgraph_bounds(n, row_ptr, n_sub):
    """DESIGN.md reading R-SUB: "divides the graph into several subgraphs and
    evenly assigns them to CPU threads" -> contiguous
    vertex ranges holding ~E/T out-edges each: lo_k = first v with
    row_ptr[v] >= floor(k*E/T)."""
    m = int(row_ptr[n])
    bounds = [0]
    for k in range(1, n_sub):
        target = (k * m) // n_sub
        v = int(np.searchsorted(row_ptr[: n + 1], target, side="left"))
        bounds.append(max(bounds[-1], min(v, n)))
    bounds.append(n)
    return bounds


def graphp_decompose(n, row_ptr, col, d_max=D_MAX_DEFAULT, n_sub=1, order="degree"):
    """Algorithm 1 over every subgraph; returns (paths, inner) where each path
    is the list of its vertices x0..xk (edges <x_t, x_t+1>), in the order the
    edge queues create them, and ``inner`` is the set marked at line 13.

    ``order`` (reading R-ORD): "degree" sorts successors -- and
    picks roots -- by total degree (in+out) descending, ties by vertex id
    (line 5 "Sort them based on degrees"; line 112 "the one with the highest
    degree is first chosen"); "id" sorts by vertex id, which reproduces the
    paper's Figure 4 layout.
    Roots (line 114 "repeatedly takes the vertex with unvisited local edges as
    the root"): every vertex of the subgraph in root order, whenever it still
    has unvisited local edges.  Visited flags are private to a subgraph
    ("each thread only divides its local subgraph", line 145).
    """
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(row_ptr))
    indeg, outdeg = _degrees(n, src, col)
    deg = indeg + outdeg

    def key(v):
        return (-int(deg[v]), int(v)) if order == "degree" else (int(v),)

    all_paths = []
    inner = set()
    bounds = subgraph_bounds(n, row_ptr, n_sub)
    for lo, hi in zip(bounds[:-1], bounds[1:]):
        visited_v = set()
        visited_e = set()           # CSR positions of visited local edges
        queue = []                  # the edge queue pointed to by p
        starts = [0]                # offsets of path starts in the queue

        def local_edges(v):
            if lo <= v < hi:
                return list(range(int(row_ptr[v]), int(row_ptr[v + 1])))
            return []

        def has_unvisited(v):
            return any(e not in visited_e for e in local_edges(v))

        def new_path():
            if starts[-1] != len(queue):
                starts.append(len(queue))

        def graphp(v_root, d):
            visited_v.add(v_root)                                  # line 2
            if has_unvisited(v_root) and d < d_max:                # line 3
                s_suc = local_edges(v_root)                        # line 4
                s_suc.sort(key=lambda e: key(int(col[e])) + (e,))  # line 5
                for e in s_suc:                                    # line 6
                    v = int(col[e])
                    if e not in visited_e:                         # line 7
                        visited_e.add(e)                           # line 8
                        queue.append((v_root, v))                  # line 9
                        if v not in visited_v:                     # line 10
                            graphp(v, d + 1)                       # line 11
                        else:
                            inner.add(v)                           # line 13
                            new_path()                             # line 14
            else:
                new_path()                                         # line 19

        for v_root in sorted(range(lo, hi), key=key):
            if has_unvisited(v_root):
                graphp(v_root, 0)
        new_path()
        for a, b in zip(starts[:-1], starts[1:]):
            edges = queue[a:b]
            if not edges:
                continue
            path = [edges[0][0]]
            for (x, y) in edges:
                assert x == path[-1], "Algorithm 1 produced a disconnected path"
                path.append(y)
            all_paths.append(path)
    return all_paths, inner


def merge_short_paths(n, src, dst, paths, inner, l_max):
    """"the paths are rechecked to merge the short ones in
    a head-to-tail way ... if both in-degree and out-degree of their
    intersected vertex are more than one, they are merged only when their
    intersected vertex is not an inner vertex".  DESIGN.md reading R-MERGE:

      1. at every vertex x where merging is allowed, the k-th path (by index)
         ending at x is linked to the k-th path starting at x; a path is never
         linked to itself (a closed path swaps with the next starter);
      2. links form chains and cycles; each cycle is cut before its
         lowest-indexed path;
      3. every chain is walked from its start and cut into merged paths of at
         most l_max edges (a piece that does not fit starts a new path);
      4. merged paths are ordered by the index of their first piece.

    ``inner`` holds the line-13 vertices for the paper-literal rule, or is
    empty for the relaxed rule."""
    indeg, outdeg = _degrees(n, np.asarray(src), np.asarray(dst))
    P = len(paths)
    ends, starts = defaultdict(list), defaultdict(list)
    for i, p in enumerate(paths):
        ends[p[-1]].append(i)
        starts[p[0]].append(i)
    nxt, prv = [-1] * P, [-1] * P
    for x in sorted(set(ends) & set(starts)):
        if indeg[x] > 1 and outdeg[x] > 1 and x in inner:
            continue
        A, B = ends[x], list(starts[x])
        for k in range(min(len(A), len(B))):
            if A[k] == B[k]:
                if k + 1 < len(B):
                    B[k], B[k + 1] = B[k + 1], B[k]
                else:
                    continue
            nxt[A[k]], prv[B[k]] = B[k], A[k]
    seen = [False] * P
    chains = []
    for i in range(P):                      # chains: start where nothing links in
        if prv[i] == -1:
            c, j = [], i
            while j != -1:
                seen[j] = True
                c.append(j)
                j = nxt[j]
            chains.append(c)
    for i in range(P):                      # cycles: cut before the lowest index
        if not seen[i]:
            c, j = [], i
            while not seen[j]:
                seen[j] = True
                c.append(j)
                j = nxt[j]
            chains.append(c)
    segs = []
    for c in chains:
        cur, cur_len = [], 0
        for j in c:
            e = len(paths[j]) - 1
            if cur and cur_len + e > l_max:
                segs.append(cur)
                cur, cur_len = [], 0
            cur.append(j)
            cur_len += e
        if cur:
            segs.append(cur)
    segs.sort(key=lambda sg: sg[0])
    out = []
    for sg in segs:
        p = list(paths[sg[0]])
        for j in sg[1:]:
            p += paths[j][1:]
        out.append(p)
    return out


def path_stats(n, src, dst, paths, hot_factor=2.0):
    """D(p) = average (in+out) degree of the path's vertex entries; N(p) = its
    vertex count (all initially active); hot iff
    D(p) >= hot_factor * mean degree (reading R-HOT)."""
    indeg, outdeg = _degrees(n, np.asarray(src), np.asarray(dst))
    deg = indeg + outdeg
    mean_deg = (2.0 * len(src) / n) if n else 0.0
    dbar = np.array([deg[np.asarray(p)].mean() for p in paths], dtype=np.float64)
    nvert = np.array([len(p) for p in paths], dtype=np.int64)
    hot = dbar >= hot_factor * mean_deg
    return dbar, nvert, hot


def dependency_graph(paths):
    """E' of PAPER.md line 98: <p_i, p_j> iff some vertex v is the head of an
    edge of p_i (v = p_i[t], t >= 1) and the tail of an edge of p_j
    (v = p_j[t], t < len-1).  Self loops are dropped.  Returns a sorted list
    of (i, j)."""
    into = defaultdict(set)
    out_of = defaultdict(set)
    for i, p in enumerate(paths):
        for t, v in enumerate(p):
            if t >= 1:
                into[v].add(i)
            if t < len(p) - 1:
                out_of[v].add(i)
    edges = set()
    for v, ins in into.items():
        for i in ins:
            for j in out_of.get(v, ()):
                if i != j:
                    edges.add((i, j))
    return sorted(edges)


def condense_and_layer(n_paths, dep_edges):
    """Tarjan SCCs of G', DAG sketch G'' and layer numbers
    ("SCC-vertices at each layer only depend on the
    SCC-vertices at the lower layer"; reading R-LAYER: longest-path
    layering, sources at layer 0).  Returns (scc_label, layer) per path where
    scc_label = smallest path index in the path's SCC."""
    from .algorithms import scc_tarjan
    if n_paths == 0:
        return np.zeros(0, np.int64), np.zeros(0, np.int64)
    e = np.asarray(dep_edges, dtype=np.int64).reshape(-1, 2)
    label = scc_tarjan(n_paths, e[:, 0], e[:, 1])
    comps = sorted(set(label.tolist()))
    preds = defaultdict(set)
    for a, b in e.tolist():
        if label[a] != label[b]:
            preds[int(label[b])].add(int(label[a]))
    layer_of = {}

    def layer(c):
        # iterative longest-path-from-source evaluation (memoised DFS)
        stack = [c]
        while stack:
            x = stack[-1]
            if x in layer_of:
                stack.pop()
                continue
            pending = [p for p in preds[x] if p not in layer_of]
            if pending:
                stack.extend(pending)
                continue
            layer_of[x] = 0 if not preds[x] else 1 + max(layer_of[p] for p in preds[x])
            stack.pop()
        return layer_of[c]

    for c in comps:
        layer(c)
    return label, np.array([layer_of[int(label[i])] for i in range(n_paths)], dtype=np.int64)


def priority(dbar, nvert, layer):
    """Pri(p) = alpha * D(p) * N(p) - L(p), alpha = 1/(Dmax * Nmax)
    (PAPER.md line 192)."""
    if len(dbar) == 0:
        return np.zeros(0)
    alpha = 1.0 / (dbar.max() * nvert.max()) if dbar.max() > 0 else 0.0
    return alpha * dbar * nvert - layer
