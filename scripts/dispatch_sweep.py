#!/usr/bin/env python
"""Dispatch and proxy-refresh sweep (readings R-DISPATCH, R-PX):
PageRank and SSSP to convergence with the global ticket (DG_DISPATCH=0, the
default) and per-CTA hot-first queues with work stealing (DG_DISPATCH=1),
and PageRank under several DG_PROXY_REFRESH intervals.  3 timed runs after
2 warm-ups, L2 flushed.  One JSON line per case.

  python scripts/dispatch_sweep.py <config> [refresh,refresh,...]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "lj"
refresh = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [8, 32, 128]
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
del g
dg.build_paths()
dg.upload()
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def timed(algo):
    for _ in range(2):
        dg.run(algo, source=0)
    ts, st = [], None
    for _ in range(3):
        flush.zero_()
        torch.cuda.synchronize()
        st = dg.run(algo, source=0)
        ts.append(st["kernel_ms"])
    return sorted(ts), st


cases = [("dispatch", d, None) for d in ("0", "1")] + [("refresh", "0", r) for r in refresh]
for kind, d, r in cases:
    os.environ["DG_DISPATCH"] = d
    if r is None:
        os.environ.pop("DG_PROXY_REFRESH", None)
    else:
        os.environ["DG_PROXY_REFRESH"] = str(r)
    for algo in (("pagerank", "sssp") if kind == "dispatch" else ("pagerank",)):
        ts, st = timed(algo)
        print(json.dumps({"config": cfg, "kind": kind, "DG_DISPATCH": d, "DG_PROXY_REFRESH": r or "auto",
                          "algo": algo, "kernel_ms": ts, "rounds": st["rounds"],
                          "updates": st["vertex_updates"]}), flush=True)
