#!/usr/bin/env python
"""Small-graph sweep (configs[0]-sized graphs are bound by per-round latency):
partition size x resident min-plus CTAs per SM (DG_MP_CTAS), SSSP and BFS
timed as bench.py does (CUDA events around dg_run, L2 flushed, 5 runs after
3 warm-ups) with the kernel time next to it.  One JSON line per case.

  python scripts/small_sweep.py <config> [part_entries,...] [ctas,...]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import inputs
from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph

cfg = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
pes = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [0, 256, 512, 1024]
ctas = sys.argv[3].split(",") if len(sys.argv) > 3 else ["3", "2", "1"]
g = inputs.make(cfg)
dg = DiGraph().load_graph(g)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
ref = {}
for pe in pes:
    dg.build_paths(part_entries=pe)
    dg.upload()
    info = dg.layout_info()
    for c in ctas:
        os.environ["DG_MP_CTAS"] = c
        for algo in ("sssp", "bfs"):
            for _ in range(3):
                dg.run(algo, source=0)
            ms, kms = [], []
            for _ in range(5):
                flush.zero_()
                torch.cuda.synchronize()
                a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
                a.record(); st = dg.run(algo, source=0); b.record(); torch.cuda.synchronize()
                ms.append(a.elapsed_time(b)); kms.append(st["kernel_ms"])
            x = dg.get_states()
            same = bool(np.array_equal(x, ref[algo])) if algo in ref else None
            ref.setdefault(algo, x.copy())
            print(json.dumps({"config": cfg, "part_entries": pe, "n_partitions": info["n_partitions"], "ctas_per_sm": c,
                              "algo": algo, "ms_per_run": float(np.median(ms)), "kernel_ms": float(np.median(kms)),
                              "rounds": st["rounds"], "updates": st["vertex_updates"], "same": same}), flush=True)
os.environ.pop("DG_MP_CTAS", None)
