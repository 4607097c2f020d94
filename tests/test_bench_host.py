"""CPU: the bench line's host-side accounting -- the
compulsory-byte model, the roofline fields and the hub share the L2
operation count excludes -- on a layout built on the CPU box (no GPU run:
the launch statistics are supplied)."""
import importlib.util
import os

import numpy as np
import pytest

import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_compulsory_bytes_by_hand(bench):
    st = {"entries_processed": 1000, "vertex_updates": 700, "rounds": 3, "dense_rounds": 2}
    n, M = 50, 400
    # PageRank: 24 B per walked entry + 40 B per vertex and round
    assert bench.algorithmic_bytes("pagerank", st, n, M) == 24 * 1000 + 40 * 50 * 3
    # SSSP: index stream of the dense rounds + 8 B per walked entry + 8 B per update + two bitmaps
    assert bench.algorithmic_bytes("sssp", st, n, M) == 4 * 400 * 2 + 8 * 1000 + 8 * 700 + 50 * 3 // 4
    # BFS / WCC / SCC read 4-byte masters only
    assert bench.algorithmic_bytes("bfs", st, n, M) == 4 * 400 * 2 + 4 * 1000 + 8 * 700 + 50 * 3 // 4


def test_roofline_fields_and_hub_share(bench):
    st = {"entries_processed": 10_000, "vertex_updates": 6_000, "rounds": 5, "dense_rounds": 5, "kernel_ms": 2.0}
    r = bench.roofline("pagerank", "nonexistent", st, 100, 1000, "path", hub_frac=0.25)
    for k in ("bound", "achieved", "peak", "unit", "frac", "traffic"):
        assert k in r
    assert r["bound"] == "hbm" and r["unit"] == "GB/s"
    assert r["achieved"] == pytest.approx(bench.algorithmic_bytes("pagerank", st, 100, 1000) / 2e-3 / 1e9)
    assert r["frac"] == pytest.approx(r["achieved"] / r["peak"])
    # hub entries are shared-memory operations: only 75 % of the gathers/REDs reach L2
    assert r["l2_random"]["ops_per_launch"] == pytest.approx(0.75 * 16_000)
    assert r["l2_random"]["frac"] == pytest.approx(0.75 * 16_000 / 2e-3 / bench.L2_MIX_CEILING)
    # min-plus walks have no proxies: every gather/atomicMin counts
    r2 = bench.roofline("sssp", "nonexistent", st, 100, 1000, "path", hub_frac=0.25)
    assert r2["l2_random"]["ops_per_launch"] == 16_000
    assert r2["l2_random"]["peak"] == bench.L2_GATHER_CEILING


def test_hub_entries_counts_the_proxied_vertices():
    g = inputs.rmat(12, 4096, 40_000, seed=3)
    dg = DiGraph().load_graph(g)
    dg.build_paths(n_proxy=64)
    info = dg.layout_info()
    ex = dg.export_paths()
    # internal ids are degree-descending: the 64 proxies are the 64 highest-degree vertices
    src, dst, _ = g.edges()
    deg = np.bincount(src, minlength=g.n) + np.bincount(dst, minlength=g.n)
    order = sorted(range(g.n), key=lambda v: (-deg[v], v))
    hubs = set(order[:64])
    verts = ex["vertices"]
    assert info["hub_entries"] == sum(1 for v in verts if v in hubs)
    assert 0 < info["hub_entries"] < info["n_entries"]
