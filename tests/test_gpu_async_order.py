"""-m gpu: the asynchronous path walk must not depend on WHEN a partition is
walked (sec. 3.1: paths are handled concurrently and asynchronously;
any interleaving of the pushes reaches the same fixed point).  The dispatch
order of the partitions is permuted through the kernel's developer knob
(DG_PART_ORDER: 1 = reversed, k > 1 = t -> t*k mod #partitions) and the
results are compared with the oracle: bit-exact for the min-plus algorithms,
within the PageRank tolerance for the accumulative one.

Also checks the bytes the public API moves: dg_upload copies only what every
run needs, SSSP adds the path-edge weights and the vertex-centric ablation
the CSR, each once.
"""
import os

import numpy as np
import pytest

import inputs
from oracle import algorithms as OA
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _cuda(cuda_required):
    pass


@pytest.fixture(scope="module")
def graph():
    return inputs.rmat(13, 8192, 90000, seed=21)


@pytest.fixture(params=["1", "7919", "65537"])
def order(request):
    old = os.environ.get("DG_PART_ORDER")
    os.environ["DG_PART_ORDER"] = request.param
    yield request.param
    if old is None:
        os.environ.pop("DG_PART_ORDER", None)
    else:
        os.environ["DG_PART_ORDER"] = old


def test_sssp_bfs_wcc_exact_under_any_dispatch_order(graph, order):
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths(part_entries=128)
    src, dst, w = g.edges()
    dg.run("sssp", source=0)
    assert np.array_equal(dg.get_states().astype(np.int64), OA.sssp_bellman_ford(g.n, src, dst, w, 0)[0])
    dg.run("bfs", source=0)
    assert np.array_equal(dg.get_states().astype(np.int64), OA.bfs_levels(g.n, src, dst, 0))
    dg.run("wcc")
    assert np.array_equal(dg.get_states().astype(np.int64), OA.wcc_label_propagation(g.n, src, dst)[0])
    dg.run("scc")
    assert np.array_equal(dg.get_states().astype(np.int64), OA.scc_tarjan(g.n, src, dst))


def test_pagerank_within_tolerance_under_any_dispatch_order(graph, order):
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths(part_entries=128)
    dg.run("pagerank", epsilon=1e-7)
    got = dg.get_states().astype(np.float64)
    src, dst, _ = g.edges()
    exp, _ = OA.pagerank_power(g.n, src, dst, d=0.85, tol=1e-12)
    assert np.abs(got - exp).sum() <= 1e-4
    assert (np.abs(got - exp) / exp).max() <= 1e-3


def test_upload_moves_only_what_the_algorithm_reads(graph):
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    dg.upload()
    info = dg.layout_info()
    base = info["h2d_bytes"]
    M, n = info["n_entries"], g.n
    # e_idx + part_off + per-vertex maps (out-degree, both id maps); no weights, no CSR
    assert base == 4 * M + 8 * (info["n_partitions"] + 1) + 12 * n
    dg.run("pagerank")
    assert dg.layout_info()["h2d_bytes"] == base
    dg.run("sssp", source=0)
    assert dg.layout_info()["h2d_bytes"] == base + 4 * M           # path-edge weights, once
    dg.run("sssp", source=0)
    assert dg.layout_info()["h2d_bytes"] == base + 4 * M
    dg.run("sssp", source=0, mode="vertex")                        # the ablation reads the CSR
    assert dg.layout_info()["h2d_bytes"] == base + 4 * M + 8 * (n + 1) + 8 * g.m
    dg.upload()                                                    # a new upload starts over
    assert dg.layout_info()["h2d_bytes"] == base


@pytest.mark.parametrize("delta", [None, 0, 1, 37, 255, 100000])
def test_sssp_exact_for_every_bucket_width(graph, delta):
    # reading R-DELTA: the bucket width trades redundant updates for rounds;
    # the distances are exact for every width (None = library default 2*w_max,
    # 0 = unbounded)
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    src, dst, w = g.edges()
    exp = OA.sssp_bellman_ford(g.n, src, dst, w, 5)[0]
    st = dg.run("sssp", source=5, delta=delta)
    assert np.array_equal(dg.get_states().astype(np.int64), exp)
    assert st["converged"]


def test_bfs_unit_buckets_are_level_synchronous(graph):
    # with Delta = 1 a BFS round commits exactly one level: every reachable
    # vertex but the source is updated once, like the level-synchronous ablation
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    src, dst, _ = g.edges()
    exp = OA.bfs_levels(g.n, src, dst, 0)
    st = dg.run("bfs", source=0, delta=1)
    assert np.array_equal(dg.get_states().astype(np.int64), exp)
    reached = int((exp < OA.UNREACHED).sum())
    assert st["vertex_updates"] == reached - 1
    sv = dg.run("bfs", source=0, mode="vertex")
    assert sv["vertex_updates"] == st["vertex_updates"]


def test_default_bucket_width_cuts_sssp_updates(graph):
    g = graph
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    st_def = dg.run("sssp", source=0)
    st_unb = dg.run("sssp", source=0, delta=0)
    assert st_def["vertex_updates"] <= st_unb["vertex_updates"]


@pytest.fixture(params=["0", "1", "16"])
def sparse_div(request):
    # DG_SPARSE_DIV: 0 = dense rounds only; k > 0 = a round with at most n/4
    # signalled vertices whose out-edges are at most M/k walks from them (1:
    # every such round, 16: the library default)
    # (DG_SPARSE_MIN_M = 0: also on these small graphs)
    old = {k: os.environ.get(k) for k in ("DG_SPARSE_DIV", "DG_SPARSE_MIN_M")}
    os.environ["DG_SPARSE_DIV"] = request.param
    os.environ["DG_SPARSE_MIN_M"] = "0"
    yield request.param
    for k, v in old.items():
        if v is None:
            del os.environ[k]
        else:
            os.environ[k] = v


@pytest.mark.parametrize("gname", ["rmat", "chains", "uniform_dup"])
@pytest.mark.parametrize("delta", [None, 1, 0])
def test_min_plus_exact_in_sparse_and_dense_rounds(graph, sparse_div, gname, delta):
    # walking from the signalled vertices through the
    # occurrence index relaxes the same edges as the window walk, so SSSP and
    # BFS stay bit-exact whichever kind of round runs, for every bucket width
    g = {"rmat": graph,
         "chains": inputs.chains(20000, 26000, chain_len=700, seed=13),
         "uniform_dup": inputs.uniform(3000, 9000, seed=12, dedupe=False, drop_self=False)}[gname]
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    src, dst, w = g.edges()
    st = dg.run("sssp", source=0, delta=delta)
    assert np.array_equal(dg.get_states().astype(np.int64), OA.sssp_bellman_ford(g.n, src, dst, w, 0)[0])
    assert st["converged"]
    st = dg.run("bfs", source=0, delta=delta)
    exp = OA.bfs_levels(g.n, src, dst, 0)
    assert np.array_equal(dg.get_states().astype(np.int64), exp)
    if delta == 1:  # level-synchronous in either kind of round
        assert st["vertex_updates"] == int((exp < OA.UNREACHED).sum()) - 1
    if delta is None:  # SCC colouring and WCC labels walk sparse too
        dg.run("scc")
        assert np.array_equal(dg.get_states().astype(np.int64), OA.scc_tarjan(g.n, src, dst))
        dg.run("wcc")
        assert np.array_equal(dg.get_states().astype(np.int64), OA.wcc_label_propagation(g.n, src, dst)[0])


@pytest.mark.parametrize("gname", ["rmat", "chains", "uniform_dup"])
def test_accumulative_in_sparse_and_dense_rounds(graph, sparse_div, gname):
    # DESIGN.md "Sparse rounds" (accumulative): walks from the signalled
    # vertices forward pending totals with the same per-entry rule; PageRank and
    # Adsorption stay within the north_star tolerance (L1 <= 1e-4, per-vertex
    # relative error <= 1e-3 against the oracle converged to 1e-12)
    g = {"rmat": graph,
         "chains": inputs.chains(20000, 26000, chain_len=700, seed=13),
         "uniform_dup": inputs.uniform(3000, 9000, seed=12, dedupe=False, drop_self=False)}[gname]
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    src, dst, w = g.edges()
    st = dg.run("pagerank", epsilon=1e-7, damping=0.85)
    got = dg.get_states().astype(np.float64)
    exp, _ = OA.pagerank_power(g.n, src, dst, d=0.85, tol=1e-12)
    assert np.abs(got - exp).sum() <= 1e-4
    assert (np.abs(got - exp) / exp).max() <= 1e-3
    assert st["converged"]
    p_inj, p_cont, inj = inputs.adsorption_params(g.n, seed=3)
    dg.set_vertex_params(p_inj, p_cont, inj)
    dg.run("adsorption", epsilon=1e-7)
    got = dg.get_states().astype(np.float64)
    exp, _ = OA.adsorption_jacobi(g.n, src, dst, w, p_inj, p_cont, inj, tol=1e-12)
    assert np.abs(got - exp).sum() / np.abs(exp).sum() <= 1e-4
    # every vertex: relative 1e-3 plus an absolute floor of 100 * eps (a
    # vertex stops at a pending delta < eps; states near 0 -- p_inj ~ 0 --
    # have no meaningful relative error)
    assert np.all(np.abs(got - exp) <= 1e-3 * exp + 100 * 1e-7), (np.abs(got - exp) - 1e-3 * exp).max()


def test_edge_cases_in_sparse_rounds(sparse_div):
    # empty edge set, single vertex, self loop only, source without out-edges,
    # a two-vertex cycle: every algorithm with sparse rounds forced on / off
    for n, e in [(1, []), (5, []), (3, [(1, 1)]), (4, [(1, 2), (2, 3)]), (3, [(0, 1), (1, 0), (1, 2)])]:
        src = np.array([a for a, _ in e], np.int64)
        dst = np.array([b for _, b in e], np.int64)
        w = [3] * len(e)
        g = inputs.from_edges(n, list(src), list(dst), w)
        dg = DiGraph()
        dg.load_graph(g)
        dg.build_paths()
        dg.run("sssp", source=0)
        assert np.array_equal(dg.get_states().astype(np.int64), OA.sssp_bellman_ford(n, src, dst, w, 0)[0])
        dg.run("bfs", source=0)
        assert np.array_equal(dg.get_states().astype(np.int64), OA.bfs_levels(n, src, dst, 0))
        dg.run("scc")
        assert np.array_equal(dg.get_states().astype(np.int64), OA.scc_tarjan(n, src, dst))
        dg.run("wcc")
        assert np.array_equal(dg.get_states().astype(np.int64), OA.wcc_label_propagation(n, src, dst)[0])
        dg.run("pagerank")
        assert np.abs(dg.get_states() - OA.pagerank_power(n, src, dst)[0]).sum() <= 1e-4


@pytest.fixture(params=["0", "1"])
def probe_free(request):
    """DG_PROBE_FREE=0 probes the signal bitmap in every dense min-plus round;
    1 (the default) walks every window without probing when most vertices are
    signalled (DESIGN.md sec. 4 "Probe-free dense min-plus rounds")."""
    old = os.environ.get("DG_PROBE_FREE")
    os.environ["DG_PROBE_FREE"] = request.param
    yield request.param
    if old is None:
        os.environ.pop("DG_PROBE_FREE", None)
    else:
        os.environ["DG_PROBE_FREE"] = old


def test_min_plus_exact_with_and_without_probing(probe_free):
    # large enough (> 2^23 path entries) that sparse rounds, probing dense
    # rounds and probe-free dense rounds all occur in one SSSP run
    g = inputs.rmat(19, 1 << 19, 9_000_000, seed=5, oversample=1.15)
    src, dst, w = g.edges()
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths()
    st = dg.run("sssp", source=0)
    assert st["dense_rounds"] >= 1 and st["rounds"] > st["dense_rounds"]
    assert np.array_equal(dg.get_states().astype(np.int64), OA.sssp_bellman_ford(g.n, src, dst, w, 0)[0])
    dg.run("bfs", source=0)
    assert np.array_equal(dg.get_states().astype(np.int64), OA.bfs_levels(g.n, src, dst, 0))
    dg.run("wcc")
    assert np.array_equal(dg.get_states().astype(np.int64), OA.wcc_label_propagation(g.n, src, dst)[0])
