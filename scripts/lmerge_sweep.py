#!/usr/bin/env python
"""Path-length sweep (readings R-MERGE and Algorithm 1's depth
bound D_MAX; verdict r01 item 7): for each (d_max, l_merge) rebuild the
layout and time PageRank, SSSP and BFS to convergence (3 timed runs after 2
warm-ups, L2 flushed).  Prints one JSON line per (d_max, l_merge, algo).

  python scripts/lmerge_sweep.py <config> [l1,l2,...] [d1,d2,...] [algo,...]
"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "lj"
lms = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [64, 256, 1024, 0]
dms = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [16]
algos = sys.argv[4].split(",") if len(sys.argv) > 4 else ["pagerank", "sssp", "bfs"]
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
del g
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for dm, lm in [(d, l) for d in dms for l in lms]:
    # l_merge 0 = no cap: merged chains are cut only by the 2^20 sanity bound
    t = time.time()
    dg.build_paths(d_max=dm, l_merge=lm if lm > 0 else 1 << 20)
    tp = time.time() - t
    dg.upload()
    info = dg.layout_info()
    for algo in algos:
        for _ in range(2):
            dg.run(algo, source=0)
        ts, st = [], None
        for _ in range(3):
            flush.zero_(); torch.cuda.synchronize()
            a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
            a.record(); st = dg.run(algo, source=0); b.record(); torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        print(json.dumps({"config": cfg, "d_max": dm, "l_merge": lm or "unbounded", "algo": algo, "ms": sorted(ts),
                          "rounds": st["rounds"], "updates": st["vertex_updates"],
                          "entries": st["entries_processed"], "n_paths": info["n_paths"],
                          "mean_path_edges": (info["n_entries"] - info["n_paths"]) / max(1, info["n_paths"]),
                          "preprocess_s": tp}), flush=True)
