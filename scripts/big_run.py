#!/usr/bin/env python
"""Large-config run (configs[2..4] at N=1): generate once, preprocess once,
time each algorithm to convergence (3 timed runs after 2 warm-ups), and one
vertex-centric ablation run for SSSP / BFS / PageRank / WCC (vertex updates next to
the path kernel's).  Prints one JSON object.

  python scripts/big_run.py <config> <algo,algo,...> [--no-ablation | --ablation=algo,algo]
"""
import json, os, resource, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "twitter"
algos = sys.argv[2].split(",") if len(sys.argv) > 2 else ["pagerank", "sssp", "wcc"]
ablation = "--no-ablation" not in sys.argv
abl_only = next((a.split("=", 1)[1].split(",") for a in sys.argv if a.startswith("--ablation=")), None)
res = {"config": cfg}
t = time.time(); g = inputs.make(cfg); res["gen_s"] = time.time() - t; res["n"] = g.n; res["m"] = g.m
print(f"[big] generated {g.name} in {res['gen_s']:.1f}s", file=sys.stderr, flush=True)
dg = DiGraph(); dg.load_graph(g)
n = g.n
del g  # the library holds its own copy of the CSR
t = time.time(); dg.build_paths(); res["preprocess_s"] = time.time() - t
t = time.time(); dg.upload(); res["upload_s"] = time.time() - t
res["layout"] = dg.layout_info()
res["host_peak_rss_gb"] = resource.getrusage(resource.RUSAGE_SELF).ru_maxrss / 1e6
print(f"[big] preprocess {res['preprocess_s']:.1f}s layout {res['layout']}", file=sys.stderr, flush=True)
for algo in algos:
    if algo == "adsorption":
        dg.set_vertex_params(*inputs.adsorption_params(n))
    for _ in range(2):
        dg.run(algo, source=0)
    times, st = [], None
    for _ in range(3):
        torch.cuda.synchronize(); a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); st = dg.run(algo, source=0); b.record(); torch.cuda.synchronize(); times.append(a.elapsed_time(b))
    ms = sum(times) / len(times)
    res[algo] = {"ms": ms, "edges_per_s": res["m"] / (ms / 1e3), "rounds": st["rounds"],
                 "vertex_updates": st["vertex_updates"], "entries_processed": st["entries_processed"],
                 "kernel_ms": st["kernel_ms"]}
    print(f"[big] {algo}: {res[algo]}", file=sys.stderr, flush=True)
    if ablation and algo in ("pagerank", "sssp", "bfs", "wcc") and (abl_only is None or algo in abl_only):
        st = dg.run(algo, source=0, mode="vertex")
        res[algo]["ablation_vertex_centric"] = {"ms": st["time_ms"], "rounds": st["rounds"],
                                                "vertex_updates": st["vertex_updates"],
                                                "edges_processed": st["edges_processed"]}
        print(f"[big] {algo} ablation: {res[algo]['ablation_vertex_centric']}", file=sys.stderr, flush=True)
res["device_peak_gb"] = torch.cuda.max_memory_allocated() / 1e9
print(json.dumps(res), flush=True)
