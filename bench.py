#!/usr/bin/env python
"""DiGraph benchmark (driver contract).

A step = one dg_run to convergence (every hot-path row: the persistent
path-propagation kernel with its device-side work lists and active counter)
on a graph already resident in HBM.  Default workload = BASELINE.json
configs[1]: PageRank d=0.85 (eps 1e-7, fp32 states) on a LiveJournal-shaped
R-MAT digraph (4,847,571 vertices, 68,993,773 edges).

  python bench.py [--gpus N --steps K --warmup W --algo pagerank|sssp --config lj|rmat16|...]
  python bench.py --impl reference ...   # the CPU oracle (a deliberately slow baseline)

One JSON line is printed by rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    ("pagerank", "lj"): "PageRank d=0.85, eps=1e-7, fp32 states, on LiveJournal-shaped R-MAT digraph "
                        "(4.8M vertices, 69M edges), 1 GPU (BASELINE configs[1])",
    ("sssp", "rmat16"): "SSSP on R-MAT scale-16 digraph (65K vertices, 1M edges, int weights 1..255), "
                        "source 0 (BASELINE configs[0])",
    ("sssp", "lj"): "SSSP (int weights 1..255) from source 0 on LiveJournal-shaped R-MAT digraph (4.8M V, 69M E)",
    ("pagerank", "twitter"): "PageRank d=0.85 on Twitter-shaped power-law digraph (41.6M V, 1.47B E) (configs[2])",
    ("sssp", "twitter"): "SSSP on Twitter-shaped power-law digraph (41.6M V, 1.47B E) (configs[2])",
    ("wcc", "lj"): "WCC label propagation on LiveJournal-shaped R-MAT digraph",
    ("scc", "lj"): "SCC colouring on LiveJournal-shaped R-MAT digraph",
}
METRIC = "time-to-convergence & edges/s"
DTYPE = {"pagerank": "f32", "adsorption": "f32", "sssp": "u32", "bfs": "u32", "wcc": "i32", "scc": "i32"}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ----------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi samples during the timed region (B200_PROFILING.md clocks line)."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        how = "sampled every 100 ms during the timed region"
        if not any(len(ln.split(",")) >= 7 for ln in self.lines):
            # the timed region was shorter than one sampling period: one query
            # right after it (clocks and throttle reasons of the same warm state)
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=10)
                self.lines = out.stdout.strip().splitlines()
                how = "timed region < 100 ms: one query right after it"
            except Exception:
                pass
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "how": how}


# ----------------------------------------------------------------- roofline
def algorithmic_bytes(algo, st):
    """Useful bytes one launch of the propagation kernel moves (DESIGN.md
    sec. 0(d)), from the launch's device counters: E = path entries walked,
    U = master updates.
      PageRank/Adsorption: per walked entry 4 B e_idx + 4 B path-edge
        coefficient + 8 B mirror S_val read + 8 B master total T read (24 B);
        per update 8 B RED on T + 8 B mirror write (16 B).
      SSSP/BFS: per walked entry 4 B e_idx + 4 B weight + 4 B distance read;
        per improvement 8 B atomicMin read-modify-write.
      WCC/SCC: per walked entry 4 B e_idx + 4 B label; 8 B per improvement."""
    E, U = st["entries_processed"], st["vertex_updates"]
    if algo in ("pagerank", "adsorption"):
        return E * 24 + U * 16
    if algo in ("sssp", "bfs"):
        return E * (12 if algo == "sssp" else 8) + U * 8
    return E * 8 + U * 8


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_random_ceiling():
    """Measured random-access ceilings (G ops/s) over an L2-resident array:
    8-byte gathers alone and an even gather/RED mix (scripts/ubench_l2_random.cu,
    profiles/r01_l2_random_ubench.txt)."""
    p = os.path.join(ROOT, "profiles", "r01_l2_random_ubench.txt")
    best = {}
    try:
        with open(p) as f:
            for ln in f:
                parts = ln.split()
                if len(parts) > 3 and parts[0] in ("gather", "g+red") and "G" in parts:
                    mb = float(ln.split("S=")[1].split("MB")[0])
                    if mb < 100:
                        v = float(ln.split(":")[1].split("G")[0])
                        best[parts[0]] = max(best.get(parts[0], 0.0), v)
    except Exception:
        pass
    return best


def load_traffic(algo, config):
    """ncu DRAM bytes per launch of the dominant kernel, from the committed
    profile summary (profiles/ncu_traffic.json), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{algo}/{config}", {}).get("dram_bytes_per_launch")
    except Exception:
        return None


# ----------------------------------------------------------------- reference arm (CPU oracle)
def oracle_sample(algo, seed):
    """A bounded sample of the workload (the oracle needs a few seconds per run
    of it): the same generator at a smaller scale with the same edge factor
    (PageRank), or the whole configs[0] graph (SSSP)."""
    import inputs
    if algo == "pagerank":
        g = inputs.rmat(20, 1 << 20, int((1 << 20) * 68993773 / 4847571), seed=seed, oversample=1.15)
        desc = "R-MAT scale 20 (1.05M vertices), LiveJournal edge factor 14.2, oracle PageRank to residual 1e-12"
    else:
        g = inputs.make("rmat16", seed=seed)
        desc = "configs[0] graph (R-MAT scale 16, 1M edges), oracle Bellman-Ford from source 0"
    return g, desc


def run_oracle_once(algo, g):
    from oracle import algorithms as OA
    src, dst, w = g.edges()
    t = time.perf_counter()
    if algo == "pagerank":
        OA.pagerank_power(g.n, src, dst, d=0.85, tol=1e-12)
    else:
        OA.sssp_bellman_ford(g.n, src, dst, w, 0)
    return time.perf_counter() - t


def cpu_baseline(algo, seed=1, min_s=10.0):
    """The oracle as it stands, run back to back on the sample until >= min_s
    seconds of CPU work; value = edges of the sample per second of one run."""
    g, desc = oracle_sample(algo, seed)
    runs, tot = 0, 0.0
    while runs == 0 or tot < min_s:
        tot += run_oracle_once(algo, g)
        runs += 1
    return {"value": g.m * runs / tot, "unit": "edges/s", "cores": 1, "kind": "oracle",
            "sample": f"{desc}: m={g.m}, {runs} run(s) in {tot:.2f} s (numpy, single-threaded)"}


def reference_arm(args, rank, world):
    if rank != 0:
        return
    algo = args.algo
    g, desc = oracle_sample(algo, args.seed)
    for _ in range(args.warmup):
        run_oracle_once(algo, g)
    times = [run_oracle_once(algo, g) for _ in range(args.steps)]
    ms = 1e3 * sum(times) / len(times)
    v = g.m / (ms / 1e3)
    line = {"metric": METRIC, "value": v, "unit": "edges/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": WORKLOADS.get((algo, args.config), f"{algo} on {args.config}"),
                       "sample": desc},
            "cpu_baseline": {"kind": "oracle", "cores": 1, "sample": desc, "value": v, "unit": "edges/s"},
            "e2e": {"value": v, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="digraph", choices=["digraph", "reference"])
    ap.add_argument("--algo", default="pagerank", choices=["pagerank", "sssp", "bfs", "wcc", "scc"])
    ap.add_argument("--config", default=None)
    ap.add_argument("--mode", default="path", choices=["path", "vertex"])
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--eps", type=float, default=1e-7)
    ap.add_argument("--part-entries", type=int, default=0)
    ap.add_argument("--merge-rule", default="relaxed")
    ap.add_argument("--n-proxy", type=int, default=4096)
    ap.add_argument("--l2-flush-mb", type=int, default=512)
    ap.add_argument("--no-extras", action="store_true", help="skip ablation/e2e/cpu baseline (profiling runs)")
    args = ap.parse_args()
    if args.config is None:
        args.config = "lj" if args.algo in ("pagerank", "wcc", "scc") else "rmat16"
    args.warmup = max(args.warmup, 3) if args.impl == "digraph" else args.warmup

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        reference_arm(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    import inputs
    from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph, parallel

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    t0 = time.time()
    g = inputs.make(args.config, seed=args.seed)
    t_gen = time.time() - t0
    dg = DiGraph(device=local)
    dg.load_graph(g)
    t0 = time.time()
    dg.build_paths(part_entries=args.part_entries, rank=rank, world=world, merge_rule=args.merge_rule,
                   n_proxy=args.n_proxy)
    t_pre = time.time() - t0
    dg.upload()
    info = dg.layout_info()
    log(f"[bench] rank {rank}: graph {g.name} gen {t_gen:.1f}s preprocess {t_pre:.1f}s layout {info}")

    run_kw = dict(source=0, epsilon=args.eps, damping=0.85)

    def step():
        if world == 1:
            return dg.run(args.algo, mode=args.mode, **run_kw), None
        return parallel.run_distributed(dg, args.algo, device=torch.device("cuda", local), **run_kw)

    for _ in range(args.warmup):
        step()
    flush = torch.empty(args.l2_flush_mb << 20, dtype=torch.uint8, device="cuda")
    clocks = ClockSampler(local)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    stats, syncs = [], []
    for k in range(args.steps):
        flush.zero_()                      # L2 flush (> 126 MB) outside the step's events
        ev[k][0].record()
        st, sy = step()
        ev[k][1].record()
        stats.append(st)
        syncs.append(sy)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    times = [a.elapsed_time(b) for a, b in ev]
    ms_local = sum(times) / len(times)
    ms_t = torch.tensor([ms_local], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    kernel_ms = sum(s["kernel_ms"] for s in stats) / len(stats)
    st0 = stats[-1]

    # roofline of the dominant kernel (the persistent propagation kernel)
    peak, peak_src = load_peaks()
    ab = algorithmic_bytes(args.algo, st0)
    achieved = ab / (st0["kernel_ms"] / 1e3) / 1e9 if st0["kernel_ms"] > 0 else 0.0
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": load_traffic(args.algo, args.config), "peak_source": peak_src,
            "kernel": f"path_kernel<{args.algo}>" if args.mode == "path" else f"vertex_kernel<{args.algo}>",
            "algorithmic_bytes_per_launch": ab, "kernel_ms": st0["kernel_ms"],
            "kernel_share_of_step": kernel_ms / ms if ms else None}

    # the resource that actually binds the path walk: random 8-byte L2 accesses
    # (one master gather per walked entry + one RED / atomicMin per update)
    ceil = load_random_ceiling()
    ops = st0["entries_processed"] + st0["vertex_updates"]
    kind = "g+red" if args.algo in ("pagerank", "adsorption") else "gather"
    ach_ops = ops / (st0["kernel_ms"] / 1e3) / 1e9 if st0["kernel_ms"] > 0 else 0.0
    rand = {"bound": "l2_random_access", "achieved": ach_ops, "unit": "G ops/s", "ops_per_launch": ops,
            "ceiling": ceil.get(kind), "ceiling_kind": f"measured {kind} over a 34-67 MB array "
                                                      "(profiles/r01_l2_random_ubench.txt)",
            "frac": (ach_ops / ceil[kind]) if ceil.get(kind) else None}

    extras = {}
    if not args.no_extras:
        # end-to-end through the public API with host buffers, every step: H2D
        # upload of the graph layout, the run (multi-rank protocol for N > 1),
        # D2H of the states (gathered over ranks for N > 1)
        e2e_t = []
        for _ in range(max(2, min(args.steps, 3))):
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t = time.perf_counter()
            dg.upload()
            t_up = time.perf_counter()
            if world == 1:
                dg.run(args.algo, mode=args.mode, **run_kw)
                t_run = time.perf_counter()
                out = dg.get_states()
                d2h = int(out.nbytes)
                log(f"[bench] e2e step: upload {1e3 * (t_up - t):.1f} ms, run {1e3 * (t_run - t_up):.1f} ms, "
                    f"get_states {1e3 * (time.perf_counter() - t_run):.1f} ms")
            else:
                parallel.run_distributed(dg, args.algo, device=torch.device("cuda", local), **run_kw)
                out = parallel.gather_states(dg, args.algo, g.n, device=torch.device("cuda", local)).cpu()
                d2h = out.numel() * out.element_size()
            torch.cuda.synchronize()
            dt = torch.tensor([time.perf_counter() - t], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(dt, op=dist.ReduceOp.MAX)
            e2e_t.append(float(dt.item()))
        info2 = dg.layout_info()
        e2e_s = statistics.median(e2e_t)
        extras["e2e"] = {"value": g.m / e2e_s, "unit": "edges/s", "h2d_bytes_per_step": info2["h2d_bytes"],
                         "d2h_bytes_per_step": d2h, "ms_per_step": e2e_s * 1e3}
    if not args.no_extras and rank == 0 and world == 1:
        # vertex-centric ablation (north_star: total vertex updates next to it)
        if args.algo in ("pagerank", "sssp", "bfs", "wcc"):
            other = "vertex" if args.mode == "path" else "path"
            ab_st = dg.run(args.algo, mode=other, **run_kw)
            extras["ablation"] = {"mode": other, "ms": ab_st["time_ms"], "rounds": ab_st["rounds"],
                                  "vertex_updates": ab_st["vertex_updates"],
                                  "edges_processed": ab_st["edges_processed"]}
        extras["cpu_baseline"] = cpu_baseline(args.algo, args.seed)

    value = g.m / (ms / 1e3)
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": DTYPE[args.algo], "data": "synthetic",
            "config": {"workload": WORKLOADS.get((args.algo, args.config), f"{args.algo} on {args.config}"),
                       "graph": g.name, "n": g.n, "m": g.m, "algo": args.algo, "mode": args.mode,
                       "epsilon": args.eps if args.algo == "pagerank" else None,
                       "delta": ("library default (SSSP 2*max weight, BFS 1; DESIGN.md R-DELTA)"
                                 if args.algo in ("sssp", "bfs") else None),
                       "l2": f"flushed between steps ({args.l2_flush_mb} MB write outside the step events)",
                       "parallelism": f"paths partitioned over {world} GPU(s)",
                       "preprocess_s": t_pre, "n_paths": info["n_paths"], "n_entries": info["n_entries"],
                       "n_partitions": info["n_partitions"], "n_layers": info["n_layers"],
                       "n_boundary": info["n_boundary"]},
            "time_to_convergence_ms": ms,
            "rounds": st0["rounds"], "vertex_updates": st0["vertex_updates"],
            "edges_processed": st0["edges_processed"], "kernel_ms": kernel_ms,
            "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
            "roofline": roof, "random_access_roofline": rand, "clocks": clk,
        }
        if syncs[-1]:
            line["sync"] = syncs[-1]
        line.update(extras)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
