#!/usr/bin/env python
"""A/B of a developer knob (environment variable read at each launch):
generate + preprocess once, then for every value time each algorithm to
convergence (3 timed runs after 2 warm-ups, L2 flushed, kernel CUDA-event
time) and check that the states equal those of the first value (exact for
SSSP/BFS/WCC/SCC, L1 for PageRank).  One JSON line per (value, algo).

  python scripts/knob_ab.py <config> <algo,...> <ENV_NAME> <v1,v2,...>   ('-' = unset)
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg, algos, name, vals = sys.argv[1], sys.argv[2].split(","), sys.argv[3], sys.argv[4].split(",")
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
del g
# DG_BUILD_NPROXY: the layout's proxy count (default: the library's 8192)
npx = os.environ.get("DG_BUILD_NPROXY")
dg.build_paths(**({"n_proxy": int(npx)} if npx else {}))
dg.upload()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
first = {}
for v in vals:
    if v == "-":
        os.environ.pop(name, None)
    else:
        os.environ[name] = v
    for algo in algos:
        for _ in range(2):
            dg.run(algo, source=0)
        ts = []
        for _ in range(3):
            flush.zero_()
            torch.cuda.synchronize()
            st = dg.run(algo, source=0)
            ts.append(st["kernel_ms"])
        x = dg.get_states()
        if algo not in first:
            first[algo] = x.copy()
            same = None
        elif algo == "pagerank":
            same = float(np.abs(x.astype(np.float64) - first[algo]).sum())
        else:
            same = bool(np.array_equal(x, first[algo]))
        print(json.dumps({"config": cfg, name: v, "algo": algo, "kernel_ms": sorted(ts), "rounds": st["rounds"],
                          "dense_rounds": st["dense_rounds"], "updates": st["vertex_updates"],
                          "entries": st["entries_processed"], "same_as_first": same}), flush=True)
