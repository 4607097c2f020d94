"""-m "not gpu": the C-ABI library loads and exports every symbol of
include/digraph.h, and its host preprocessing rows (Algorithm 1, merging,
dependency DAG, layers, priority order, partitions) agree exactly with the
oracle -- the product and the oracle share no code."""
import itertools
import os
import re

import numpy as np
import pytest

import inputs
from oracle import paths as OP
from paper_conf_asplos_zhangl0hlg19_b200 import _abi, DiGraph, DGError

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_header_symbol():
    hdr = open(os.path.join(ROOT, "include", "digraph.h")).read()
    declared = sorted(set(re.findall(r"^\s*(?:int|void|const char \*)\s*\*?\s*(dg_\w+)\s*\(", hdr, re.M)))
    assert declared, "no declarations parsed"
    L = _abi.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert sorted(_abi.EXPORTS) == declared


def oracle_layout(g, d_max, n_sub, order, l_merge, rule="relaxed"):
    src, dst, _ = g.edges()
    paths, inner = OP.graphp_decompose(g.n, g.row_ptr, g.col, d_max=d_max, n_sub=n_sub, order=order)
    # reading R-MERGE: "relaxed" ignores the inner-vertex constraint (oracle: inner = {})
    inner_used = inner if rule == "paper" else set()
    merged = OP.merge_short_paths(g.n, src, dst, paths, inner_used, l_max=l_merge) if l_merge else paths
    dep = OP.dependency_graph(merged)
    scc, layer = OP.condense_and_layer(len(merged), dep)
    dbar, nv, hot = OP.path_stats(g.n, src, dst, merged, hot_factor=2.0)
    pri = OP.priority(dbar, nv, layer)
    return paths, merged, scc, layer, hot, pri


def product_layout(g, d_max, n_sub, order, l_merge, part_entries=64, rule="relaxed"):
    dg = DiGraph()
    dg.load_graph(g)
    dg.build_paths(d_max=d_max, l_merge=l_merge, n_sub=n_sub, order=order, part_entries=part_entries,
                   merge_rule=rule)
    return dg, dg.export_paths(), dg.layout_info()


def split(ex):
    off, v = ex["path_off"], ex["vertices"]
    return [v[off[i]:off[i + 1]].tolist() for i in range(len(off) - 1)]


def fig4_graph():
    edges = [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5), (3, 6), (6, 7), (7, 8), (8, 9), (8, 10),
             (10, 11), (11, 12), (7, 13), (13, 14), (14, 6)]
    return inputs.from_edges(15, [e[0] for e in edges], [e[1] for e in edges], [1] * len(edges))


def test_product_reproduces_figure4_layout():
    g = fig4_graph()
    dg, ex, info = product_layout(g, 16, 1, "id", 0)
    paths = split(ex)
    by_merge = [p for _, p in sorted(zip(ex["merged_index"].tolist(), paths))]
    assert by_merge == [[0, 1, 2, 3, 4, 5], [3, 6, 7, 8, 9], [8, 10, 11, 12], [7, 13, 14, 6]]
    lay = dict(zip(ex["merged_index"].tolist(), ex["layer"].tolist()))
    assert [lay[i] for i in range(4)] == [0, 1, 2, 1]
    scc = dict(zip(ex["merged_index"].tolist(), ex["scc"].tolist()))
    assert [scc[i] for i in range(4)] == [0, 1, 2, 1]
    # priority order: layer 0 first, layer 2 last
    assert ex["layer"].tolist() == sorted(ex["layer"].tolist())
    assert info["n_layers"] == 3 and info["n_dep_sccs"] == 3 and info["giant_scc_paths"] == 2


CASES = list(itertools.product([0, 1, 2], [1, 3], ["degree", "id"], [0, 64], [16, 3], ["paper", "relaxed"]))


@pytest.mark.parametrize("seed,n_sub,order,l_merge,d_max,rule", CASES)
def test_product_preprocessing_matches_oracle(seed, n_sub, order, l_merge, d_max, rule):
    g = inputs.rmat(9, 400, 2500, seed=seed, weights=(1, 9)) if seed != 2 else \
        inputs.uniform(300, 1200, seed=seed, weights=(1, 9))
    o_paths, o_merged, o_scc, o_layer, o_hot, o_pri = oracle_layout(g, d_max, n_sub, order, l_merge, rule)
    dg, ex, info = product_layout(g, d_max, n_sub, order, l_merge, rule=rule)
    assert info["paths_before_merge"] == len(o_paths)
    paths = split(ex)
    midx = ex["merged_index"]
    assert sorted(midx.tolist()) == list(range(len(o_merged)))
    for p, i in zip(paths, midx.tolist()):
        assert p == o_merged[i]
    # dependency SCC labels and layers
    assert np.array_equal(ex["scc"], o_scc[midx])
    assert np.array_equal(ex["layer"], o_layer[midx])
    assert np.array_equal(ex["hot"], o_hot[midx])
    # priority order = stable sort by Pri desc
    assert midx.tolist() == np.argsort(-o_pri, kind="stable").tolist()
    # partitions cover whole paths in order
    po = ex["part_off"]
    assert po[0] == 0 and po[-1] == ex["path_off"][-1]
    assert set(po.tolist()) <= set(ex["path_off"].tolist())


def test_edge_weights_follow_paths():
    g = inputs.rmat(8, 256, 1500, seed=5, weights=(1, 255))
    dg, ex, info = product_layout(g, 16, 2, "degree", 64)
    # every path edge is a graph edge; weights are the graph's
    wmap = {}
    src, dst, w = g.edges()
    for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
        wmap[(a, b)] = c
    cover = []
    for p in split(ex):
        cover += list(zip(p[:-1], p[1:]))
    assert sorted(cover) == sorted(zip(src.tolist(), dst.tolist()))


@pytest.mark.parametrize("placement", ["locality", "round_robin"])
def test_multirank_partitioning_is_a_disjoint_cover(placement):
    g = inputs.rmat(10, 1000, 8000, seed=3)
    world = 3
    covers, bnd_sets, presence, entries = [], [], [], []
    for r in range(world):
        dg = DiGraph()
        dg.load_graph(g)
        dg.build_paths(part_entries=128, rank=r, world=world, placement=placement)
        entries.append(dg.layout_info()["n_entries"])
        ex = dg.export_paths()
        cov = []
        for p in split(ex):
            cov += list(zip(p[:-1], p[1:]))
        covers.append(cov)
        bnd_sets.append(dg.boundary_vertices().tolist())
        presence.append(set(ex["vertices"].tolist()))
    src, dst, _ = g.edges()
    assert sorted(sum(covers, [])) == sorted(zip(src.tolist(), dst.tolist()))
    assert bnd_sets[0] == bnd_sets[1] == bnd_sets[2]
    # boundary = vertices replicated on more than one rank's paths
    multi = sorted(v for v in range(g.n) if sum(v in s_ for s_ in presence) > 1)
    assert bnd_sets[0] == multi
    # balanced in path entries (what a rank's kernel walks): within 2 % of an
    # even share plus one partition for the locality placement
    assert max(entries) - min(entries) <= 0.1 * max(entries), entries


def test_locality_placement_shrinks_the_boundary():
    """Reading R-PLACE: paths go to the rank already holding most of their
    vertices, so fewer vertices are replicated than with round-robin
    partitions (same graph, same world)."""
    for g, gain in ((inputs.chains(40000, 60000, chain_len=512, seed=5), 0.6),
                    (inputs.rmat(13, 8192, 80000, seed=31), 1.0)):
        nb = {}
        for pl in ("round_robin", "locality"):
            dg = DiGraph().load_graph(g).build_paths(part_entries=256, rank=0, world=2, placement=pl)
            nb[pl] = dg.layout_info()["n_boundary"]
        assert nb["locality"] < gain * nb["round_robin"], nb


def test_run_without_cuda_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("CUDA present")
    dg = DiGraph()
    dg.load_graph(fig4_graph())
    dg.build_paths()
    with pytest.raises(DGError, match="DG_ENOCUDA"):
        dg.run("sssp", source=0)


def test_bad_arguments_are_rejected():
    dg = DiGraph()
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.build_paths()
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.load_csr(3, np.array([0, 1, 2, 9]), np.array([1, 2, 0]))
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.load_csr(3, np.array([0, 1, 2, 3]), np.array([1, 2, 7]))


def test_failed_load_keeps_the_previous_graph():
    """A dg_load_csr that fails validation leaves the handle as it was
    (include/digraph.h): the previous graph and its layout stay usable, so a
    later upload cannot read host arrays sized for the rejected graph."""
    dg = DiGraph()
    g = fig4_graph()
    dg.load_graph(g).build_paths()
    before = dg.layout_info()
    big = 100
    for rp, col, w in [
        (np.r_[0, np.full(big, 1)], np.array([big + 5]), None),        # column out of range
        (np.r_[0, np.full(big, 1)], np.array([3]), np.array([-1])),     # negative weight
        (np.r_[0, 2, 1, np.full(big - 2, 2)], np.array([1, 2]), None),  # decreasing row_ptr
    ]:
        with pytest.raises(DGError, match="DG_EINVAL"):
            dg.load_csr(big, rp, col, w)
        assert dg.n == g.n and dg.m == g.m
        assert dg.layout_info() == before
    ex = dg.export_paths()
    assert len(ex["vertices"]) == before["n_entries"]


def test_p2p_exchange_lifecycle_is_checked():
    """dg_p2p_alloc needs an uploaded layout, dg_p2p_open an allocated region,
    dg_boundary_exchange a run in progress (include/digraph.h)."""
    dg = DiGraph()
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.p2p_alloc(2, 0)
    dg.load_graph(fig4_graph())
    dg.build_paths(rank=0, world=2)
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.p2p_alloc(2, 0)  # not uploaded
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.p2p_open([b"\0" * 64, b"\0" * 64])
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.boundary_exchange()


def test_layout_file_round_trip(tmp_path):
    """dg_save_layout / dg_load_layout: the loaded handle exports exactly the
    saved layout (paths, layers, SCC labels, partitions, boundary)."""
    g = inputs.rmat(11, 2048, 20000, seed=13)
    a = DiGraph().load_graph(g).build_paths(part_entries=256)
    path = str(tmp_path / "lay.0")
    a.save_layout(path)
    b = DiGraph().load_layout(path)
    ea, eb = a.export_paths(), b.export_paths()
    for k in ea:
        assert np.array_equal(ea[k], eb[k]), k
    ia, ib = a.layout_info(), b.layout_info()
    for k in ("n", "m", "n_paths", "n_entries", "n_partitions", "n_hot_paths", "n_layers", "n_dep_sccs",
              "giant_scc_paths", "n_boundary", "paths_before_merge"):
        assert ia[k] == ib[k], k
    assert b.n == g.n and b.m == g.m
    # a layout file carries no CSR: re-preprocessing it is refused
    with pytest.raises(DGError, match="DG_EINVAL"):
        b.build_paths()


def test_shared_build_equals_per_rank_builds(tmp_path):
    """dg_build_paths_shared (one preprocessing pass) writes, for every rank,
    the layout a per-rank dg_build_paths(rank, world) builds."""
    g = inputs.rmat(11, 2048, 20000, seed=17)
    world = 3
    prefix = str(tmp_path / "shared")
    own = DiGraph().load_graph(g).build_paths_shared(prefix, world=world, rank=1, part_entries=128)
    for r in range(world):
        ref = DiGraph().load_graph(g).build_paths(part_entries=128, rank=r, world=world)
        got = DiGraph().load_layout(f"{prefix}.{r}")
        er, eg = ref.export_paths(), got.export_paths()
        for k in er:
            assert np.array_equal(er[k], eg[k]), (r, k)
        assert np.array_equal(ref.boundary_vertices(), got.boundary_vertices())
    eo, e1 = own.export_paths(), DiGraph().load_layout(f"{prefix}.1").export_paths()
    for k in eo:
        assert np.array_equal(eo[k], e1[k]), k


def test_bad_layout_file_keeps_the_handle(tmp_path):
    g = fig4_graph()
    dg = DiGraph().load_graph(g).build_paths()
    before = dg.layout_info()
    p = tmp_path / "bad"
    p.write_bytes(b"DGLAYOUT" + b"\0" * 16)
    for path in (str(p), str(tmp_path / "missing")):
        with pytest.raises(DGError, match="DG_EINVAL"):
            dg.load_layout(path)
        assert dg.layout_info() == before
    good = str(tmp_path / "good")
    dg.save_layout(good)
    data = open(good, "rb").read()
    open(str(p), "wb").write(data[: len(data) // 2])  # truncated
    with pytest.raises(DGError, match="DG_EINVAL"):
        dg.load_layout(str(p))
    assert dg.layout_info() == before


def test_auto_partitions_hold_at_least_512_entries():
    # part_entries = 0 (auto): about 16 K partitions of 512..2048 whole-path
    # entries (DESIGN.md sec. 4 "Small graphs"); a partition may exceed the
    # target only by the path that crosses it
    for scale, m in ((12, 40_000), (16, 1 << 20)):
        g = inputs.rmat(scale, 1 << scale, m, seed=4)
        dg = DiGraph().load_graph(g).build_paths()
        info = dg.layout_info()
        part_off = dg.export_paths()["part_off"]
        sizes = np.diff(part_off)
        assert info["n_partitions"] == len(sizes)
        # every partition but the last reaches the 512-entry target
        assert sizes[:-1].min() >= 512
        assert info["n_partitions"] <= info["n_entries"] // 512 + 1
