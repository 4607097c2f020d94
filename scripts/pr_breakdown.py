#!/usr/bin/env python
"""PageRank cost breakdown of the accumulative walk (developer experiment; the
DG_EXP build of scripts/build_exp.sh, loaded through DG_LIB_PATH): the first
R rounds of PageRank (all windows active on the large graphs) timed with parts
of the per-entry work switched off -- 1: master REDs, 2: master gathers,
4: S_val stores, 16: S_val + coefficient loads -- and with the shared-memory
proxies off (DG_N_PROXY=0).  Results with switches on are wrong by design;
only the time per round matters.  One JSON line per case.

  DG_LIB_PATH=.../libdigraph_exp.so python scripts/pr_breakdown.py <config> [rounds]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "lj"
R = int(sys.argv[2]) if len(sys.argv) > 2 else 10
cases = [("base", "0", None), ("no_red", "1", None), ("no_gather", "2", None), ("no_sval_store", "4", None),
         ("no_stream_sval_coef", "16", None), ("no_red_no_gather", "3", None), ("stream_only", "7", None),
         ("no_proxy", "0", "0"), ("proxy_2k", "0", "2048"), ("base_again", "0", None)]
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
m = g.m
del g
dg.build_paths()
dg.upload()
info = dg.layout_info()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for name, ex, npx in cases:
    os.environ["DG_EXP"] = ex
    if npx is None:
        os.environ.pop("DG_N_PROXY", None)
    else:
        os.environ["DG_N_PROXY"] = npx
    ts = []
    for k in range(4):
        flush.zero_()
        torch.cuda.synchronize()
        st = dg.run("pagerank", max_rounds=R, allow_noconv=True)
        if k:
            ts.append(st["kernel_ms"])
    print(json.dumps({"config": cfg, "case": name, "DG_EXP": ex, "n_proxy": npx, "rounds": st["rounds"],
                      "kernel_ms": sorted(ts), "ms_per_round": min(ts) / st["rounds"],
                      "entries": st["entries_processed"], "updates": st["vertex_updates"],
                      "M": info["n_entries"], "m": m}), flush=True)
os.environ.pop("DG_EXP", None)
