#!/usr/bin/env python
"""Boundary size and peer-exchange volume of multi-rank layouts (CPU only):
for world 2/4/8 and both placements (round-robin partitions, locality paths;
DESIGN.md reading R-PLACE), the boundary vertices n_bnd (replicated on > 1
rank) and the bytes one rank reads per exchange in the peer-memory exchange:
holder-aware, 8 B x boundary_reads (the peer slots of the boundary vertices
its own paths hold; dg_layout_info), next to the all-peers volume
8 B x n_bnd x (world - 1) the exchange read before it became holder-aware.  Prints one JSON line per case.

  python scripts/boundary_table.py <config> [worlds]
"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "lj"
worlds = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [2, 4, 8]
g = inputs.make(cfg)
n, m = g.n, g.m
dg = DiGraph().load_graph(g)
del g
for w in worlds:
    for pl in ("round_robin", "locality"):
        t = time.time()
        dg.build_paths(rank=0, world=w, placement=pl)
        i = dg.layout_info()
        nb = i["n_boundary"]
        print(json.dumps({"config": cfg, "n": n, "m": m, "world": w, "placement": pl, "n_boundary": nb,
                          "boundary_frac": nb / n, "rank0_entries": i["n_entries"],
                          "boundary_reads_rank0": i["boundary_reads"],
                          "exchange_bytes_rank0": 8 * i["boundary_reads"],
                          "all_peers_bytes_per_rank": 8 * nb * (w - 1), "build_s": time.time() - t}), flush=True)
