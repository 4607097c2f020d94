#!/usr/bin/env python
"""PageRank to convergence under DG_EXP settings (developer experiment; the
DG_EXP build, scripts/build_exp.sh, via DG_LIB_PATH): rounds, entries, time
and the result's L1 distance to the DG_EXP=0 run.  32: gathers read a
snapshot of the masters taken at the start of the round; 64: one taken at
the start of the previous round (the staleness of a scheme that learns a
vertex's pending amount from its own atomic one round late).

  DG_LIB_PATH=... python scripts/pr_exp_runs.py <config> 0,32,64
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "lj"
exps = sys.argv[2].split(",") if len(sys.argv) > 2 else ["0", "32", "64"]
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
del g
dg.build_paths()
dg.upload()
ref = None
for ex in exps:
    os.environ["DG_EXP"] = ex
    dg.run("pagerank")
    st = dg.run("pagerank")
    x = dg.get_states().astype(np.float64)
    if ref is None:
        ref = x
    print(json.dumps({"config": cfg, "DG_EXP": ex, "rounds": st["rounds"], "kernel_ms": st["kernel_ms"],
                      "entries": st["entries_processed"], "updates": st["vertex_updates"],
                      "l1_vs_first": float(np.abs(x - ref).sum())}), flush=True)
os.environ.pop("DG_EXP", None)
