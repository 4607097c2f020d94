#!/usr/bin/env python
"""DiGraph benchmark (driver contract; DESIGN.md sec. 0(d) "Measurement").

A step = one dg_run to convergence (every hot-path row: the persistent
path-propagation kernel with its device-side work lists and active counter)
on a graph already resident in HBM.  Default workload = BASELINE.json
configs[2], the metric's own config: PageRank d=0.85 (eps 1e-7, fp32 states)
on a Twitter-shaped power-law R-MAT digraph (41,652,230 vertices,
1,468,365,182 edges); the same graph and preprocessing then also time SSSP
(the metric's second algorithm) as the line's `sssp` record.

  python bench.py [--gpus N --steps K --warmup W --algo pagerank|sssp|... --config twitter|lj|rmat16|...]
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
    ("pagerank", "twitter"): "PageRank d=0.85, eps=1e-7, fp32 states, on Twitter-shaped power-law R-MAT digraph "
                             "(41.6M vertices, 1.47B edges) (BASELINE configs[2])",
    ("sssp", "twitter"): "SSSP (int weights 1..255) from source 0 on Twitter-shaped power-law R-MAT digraph "
                         "(41.6M vertices, 1.47B edges) (BASELINE configs[2])",
    ("pagerank", "lj"): "PageRank d=0.85, eps=1e-7, fp32 states, on LiveJournal-shaped R-MAT digraph "
                        "(4.8M vertices, 69M edges), 1 GPU (BASELINE configs[1])",
    ("sssp", "rmat16"): "SSSP on R-MAT scale-16 digraph (65K vertices, 1M edges, int weights 1..255), "
                        "source 0 (BASELINE configs[0])",
    ("sssp", "lj"): "SSSP (int weights 1..255) from source 0 on LiveJournal-shaped R-MAT digraph (4.8M V, 69M E)",
    ("wcc", "lj"): "WCC label propagation on LiveJournal-shaped R-MAT digraph",
    ("scc", "lj"): "SCC colouring on LiveJournal-shaped R-MAT digraph",
}
DEFAULT_CONFIG = {"pagerank": "twitter", "sssp": "twitter", "bfs": "twitter", "wcc": "lj", "scc": "lj"}
# The paper's own numbers (context only, other hardware): DiGraph on four
# Tesla K80 (26 SMX, 24 GB each) against Gunrock and Groute on the same GPUs,
# PAPER.md:37 (abstract), 196 (sec. 4 setup), 249 (sec. 4.2).
PAPER_CONTEXT = {"hardware": "4 x NVIDIA Tesla K80 (PAPER.md:196)",
                 "speedup_vs_gunrock": "2.25-7.39x (PAPER.md:37, 249)",
                 "speedup_vs_groute": "1.59-3.54x (PAPER.md:37, 249)",
                 "note": "context only: another machine and other graphs; not a target for this line"}
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
def algorithmic_bytes(algo, st, n, M):
    """Compulsory HBM bytes of one launch of the propagation kernel (DESIGN.md
    sec. 0(d)): what the walk must stream from / to HBM whatever the cache
    does, from the launch's device counters -- E = path entries walked, U =
    master updates, R = rounds, Rd = rounds that streamed every window (dense),
    n vertices, M path entries.  Random master gathers / REDs are counted once
    per vertex and round (the masters are re-read every round); every further
    access to a master is an L2 operation, not compulsory HBM traffic (ncu's
    `traffic` shows what the cache really let through).
      PageRank/Adsorption: 24 E (4 B e_idx + 4 B coefficient + 8 B S_val read
        + 8 B S_val write per walked entry) + 40 n R (per round and vertex: the
        master read + write, 16 B; the end-of-round sweep's T read and sigma
        read + write, 24 B).
      SSSP / BFS / WCC / SCC: 4 M Rd (the index stream of a dense round) +
        8 E (SSSP: 4 B weight + 4 B master per walked entry; 4 B master for
        the others) + 8 U (master read-modify-write) + n R / 4 (two bitmaps)."""
    E, U, R = st["entries_processed"], st["vertex_updates"], st["rounds"]
    Rd = st.get("dense_rounds", R)
    if algo in ("pagerank", "adsorption"):
        return 24 * E + 40 * n * R
    per = 8 if algo == "sssp" else 4
    return 4 * M * Rd + per * E + 8 * U + n * R // 4


L2_MIX_CEILING = 145e9  # random 8-byte gather/RED mix over an L2-resident array (r02d ubench: 142-149 G ops/s)
L2_GATHER_CEILING = 280e9  # random gathers alone (r02d ubench: 278-287 G/s)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_ncu(algo, config):
    """The committed ncu capture of the dominant kernel for this workload
    (profiles/ncu_traffic.json, written by scripts/summarize_ncu.py): DRAM
    bytes (read + write) per launch and the launch's duration under ncu."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            return json.load(f).get(f"{algo}/{config}")
    except Exception:
        return None


def roofline(algo, config, st, n, M, mode, hub_frac=None):
    """`roofline` of the dominant kernel: compulsory bytes / CUDA-event time of
    this run's launch (`achieved`), against the measured HBM copy bandwidth;
    `traffic` and `hbm_measured` from the committed ncu capture (what the
    kernel really moved: DRAM bytes / its ncu duration)."""
    peak, peak_src = load_peaks()
    ab = algorithmic_bytes(algo, st, n, M)
    kms = st["kernel_ms"]
    achieved = ab / (kms / 1e3) / 1e9 if kms > 0 else 0.0
    nc = load_ncu(algo, config) if mode == "path" else None
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": nc["dram_bytes_per_launch"] if nc else None, "peak_source": peak_src,
            "kernel": f"path_kernel<{algo}>" if mode == "path" else f"vertex_kernel<{algo}>",
            "algorithmic_bytes_per_launch": ab, "kernel_ms": kms,
            "model": "compulsory HBM bytes (bench.py algorithmic_bytes, DESIGN.md sec. 0(d))"}
    if nc and nc.get("kernel_ms"):
        gbs = nc["dram_bytes_per_launch"] / (nc["kernel_ms"] / 1e3) / 1e9
        roof["hbm_measured"] = {"dram_bytes": nc["dram_bytes_per_launch"], "ncu_kernel_ms": nc["kernel_ms"],
                                "gbs": gbs, "frac": gbs / peak, "report": nc.get("summary")}
    # the L2 side: random master operations per second -- one gather per
    # walked entry, one RED / atomicMin per update; for PageRank/Adsorption
    # the hub entries (shared-memory proxies) are not L2 operations: both
    # counts are scaled by the non-hub share of the layout's entries
    ops = st["entries_processed"] + st["vertex_updates"]
    if algo in ("pagerank", "adsorption") and hub_frac is not None:
        ops *= 1.0 - hub_frac
        roof["hub_entry_share"] = hub_frac
    rate = ops / (kms / 1e3) if kms > 0 else 0.0
    roof["l2_random_ops_per_s"] = rate
    # the resource that binds the walks (DESIGN.md sec. 4 "Bound"): random
    # master operations against the measured L2 gather/RED-mix ceiling
    accum = algo in ("pagerank", "adsorption")
    ceil = L2_MIX_CEILING if accum else L2_GATHER_CEILING
    roof["l2_random"] = {"achieved": rate, "peak": ceil, "unit": "ops/s", "frac": rate / ceil, "ops_per_launch": ops,
                         "peak_source": "measured: scripts/ubench_l2_random.cu, profiles/r02d_l2_random_ubench.txt " +
                                        ("(8-byte gathers and 64-bit REDs, even mix, L2-resident array)" if accum else
                                         "(random gathers over an L2-resident array; the min-plus walk's atomicMins "
                                         "are a few percent of its operations)")}
    return roof


# ----------------------------------------------------------------- reference arm (CPU oracle)
def oracle_sample(algo, config, seed):
    """A bounded sample of the workload (the oracle needs seconds per run of
    it): the same generator at a smaller scale with the same edge factor."""
    import inputs
    if config == "rmat16":
        g = inputs.make("rmat16", seed=seed)
        return g, "configs[0] graph (R-MAT scale 16, 1M edges)"
    ef = {"twitter": 1468365182 / 41652230, "lj": 68993773 / 4847571,
          "friendster": 1806067135 / 65608366}.get(config, 1468365182 / 41652230)
    scale = 19 if algo == "pagerank" else 20
    g = inputs.rmat(scale, 1 << scale, int((1 << scale) * ef), seed=seed, oversample=1.15)
    return g, f"R-MAT scale {scale} ({1 << scale} vertices), {config} edge factor {ef:.1f}"


def run_oracle_once(algo, g):
    from oracle import algorithms as OA
    src, dst, w = g.edges()
    t = time.perf_counter()
    if algo == "pagerank":
        OA.pagerank_power(g.n, src, dst, d=0.85, tol=1e-12)
    elif algo == "sssp":
        OA.sssp_bellman_ford(g.n, src, dst, w, 0)
    elif algo == "bfs":
        OA.bfs_levels(g.n, src, dst, 0)
    elif algo == "wcc":
        OA.wcc_label_propagation(g.n, src, dst)
    else:
        OA.scc_tarjan(g.n, src, dst)
    return time.perf_counter() - t


ORACLE_DESC = {"pagerank": "oracle fp64 power iteration to residual 1e-12", "sssp": "oracle Bellman-Ford from source 0",
               "bfs": "oracle level BFS from 0", "wcc": "oracle label propagation", "scc": "oracle Tarjan"}


def cpu_baseline(algo, config, seed=1, min_s=10.0):
    """The oracle as it stands, run back to back on the sample until >= min_s
    seconds of CPU work; value = edges of the sample per second of one run."""
    g, desc = oracle_sample(algo, config, seed)
    runs, tot = 0, 0.0
    while runs == 0 or tot < min_s:
        tot += run_oracle_once(algo, g)
        runs += 1
    return {"value": g.m * runs / tot, "unit": "edges/s", "cores": 1, "kind": "oracle",
            "sample": f"{desc}, {ORACLE_DESC[algo]}: m={g.m}, {runs} run(s) in {tot:.2f} s (numpy, single-threaded)"}


def reference_arm(args, rank, world):
    if rank != 0:
        return
    algo = args.algo
    g, desc = oracle_sample(algo, args.config, args.seed)
    desc = f"{desc}, {ORACLE_DESC[algo]}"
    for _ in range(args.warmup):
        run_oracle_once(algo, g)
    times = [run_oracle_once(algo, g) for _ in range(args.steps)]
    ms = 1e3 * sum(times) / len(times)
    v = g.m / (ms / 1e3)
    line = {"metric": METRIC, "value": v, "unit": "edges/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64" if algo == "pagerank" else "i64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": WORKLOADS.get((algo, args.config), f"{algo} on {args.config}"),
                       "sample": desc, "m_sample": g.m},
            "cpu_baseline": {"kind": "oracle", "cores": 1, "sample": desc, "value": v, "unit": "edges/s"},
            "e2e": {"value": v, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------- our arm
def timed_runs(step, steps, warmup, flush, world, clocks=None):
    """W untimed runs, then K runs bracketed by CUDA events (L2 flushed before
    each, outside the events); `clocks` samples nvidia-smi during the K runs.
    Returns (per-run ms list, stats list, sync list)."""
    import torch
    import torch.distributed as dist
    for _ in range(warmup):
        step()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    if clocks:
        clocks.start()
    stats, syncs = [], []
    for k in range(steps):
        flush.zero_()                      # L2 flush (> 126 MB) outside the step's events
        ev[k][0].record()
        st, sy = step()
        ev[k][1].record()
        stats.append(st)
        syncs.append(sy)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    return [a.elapsed_time(b) for a, b in ev], stats, syncs


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
    ap.add_argument("--l-merge", type=int, default=64)
    ap.add_argument("--n-proxy", type=int, default=8192)
    ap.add_argument("--l2-flush-mb", type=int, default=512)
    ap.add_argument("--no-extras", action="store_true", help="skip ablation/e2e/cpu baseline/sssp (profiling runs)")
    ap.add_argument("--no-sssp", action="store_true", help="skip the SSSP record of the default PageRank line")
    ap.add_argument("--layout-cache", default=None,
                    help="N=1 profiling runs only: load the layout from this file if it exists, else build it and "
                         "save it there (a loaded layout has no CSR, so use with --no-extras)")
    args = ap.parse_args()
    if args.config is None:
        args.config = DEFAULT_CONFIG[args.algo]
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

    bp = dict(part_entries=args.part_entries, merge_rule=args.merge_rule, n_proxy=args.n_proxy,
              l_merge=args.l_merge)
    dg = DiGraph(device=local)
    t_gen = t_load = t_pre = 0.0
    gname = f"{args.config}-seed{args.seed}"
    if world == 1 and args.layout_cache and os.path.exists(args.layout_cache):
        t0 = time.time()
        dg.load_layout(args.layout_cache)
        t_load = time.time() - t0
        gname = f"{args.config}-seed{args.seed} (layout file)"
    elif world == 1:
        t0 = time.time()
        g = inputs.make(args.config, seed=args.seed)
        t_gen = time.time() - t0
        gname = g.name
        t0 = time.time()
        dg.load_graph(g)
        t_load = time.time() - t0
        del g  # the library holds its own copy of the CSR
        t0 = time.time()
        dg.build_paths(**bp)
        t_pre = time.time() - t0
        if args.layout_cache:
            try:
                dg.save_layout(args.layout_cache)
            except Exception as e:  # a profiling convenience only
                log(f"[bench] layout cache not written: {e}")
    else:
        # preprocess ONCE (rank 0) and hand every rank its share through layout
        # files (dg_build_paths_shared / dg_load_layout):
        # the other ranks neither generate the graph nor run Algorithm 1
        shm = "/dev/shm" if os.path.isdir("/dev/shm") else "/tmp"
        prefix = os.path.join(shm, f"dg_layout_{os.environ.get('MASTER_PORT', '0')}_{args.config}_{args.seed}")
        if rank == 0:
            t0 = time.time()
            g = inputs.make(args.config, seed=args.seed)
            t_gen = time.time() - t0
            gname = g.name
            dg.load_graph(g)
            del g
            t0 = time.time()
            dg.build_paths_shared(prefix, world=world, rank=0, **bp)
            t_pre = time.time() - t0
        dist.barrier()
        if rank != 0:
            t0 = time.time()
            dg.load_layout(f"{prefix}.{rank}")
            t_load = time.time() - t0
        dist.barrier()
        if rank == 0:
            for r in range(world):
                try:
                    os.remove(f"{prefix}.{r}")
                except OSError:
                    pass
    info0 = dg.layout_info()
    n, m = info0["n"], info0["m"]
    dg.upload()
    info = dg.layout_info()
    M = info["n_entries"]
    log(f"[bench] rank {rank}: graph {gname} gen {t_gen:.1f}s load {t_load:.1f}s preprocess {t_pre:.1f}s "
        f"layout {info}")

    def make_step(algo, mode):
        kw = dict(source=0, epsilon=args.eps, damping=0.85)
        if world == 1:
            return lambda: (dg.run(algo, mode=mode, **kw), None)
        return lambda: parallel.run_distributed(dg, algo, device=torch.device("cuda", local), **kw)

    flush = torch.empty(args.l2_flush_mb << 20, dtype=torch.uint8, device="cuda")
    clocks = ClockSampler(local)
    times, stats, syncs = timed_runs(make_step(args.algo, args.mode), args.steps, args.warmup, flush, world, clocks)
    clk = clocks.stop()
    ms_t = torch.tensor([sum(times) / len(times)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    kernel_ms = sum(s["kernel_ms"] for s in stats) / len(stats)
    st0 = stats[-1]
    hub_frac = info["hub_entries"] / M if M else None
    roof = roofline(args.algo, args.config, st0, n, M, args.mode, hub_frac)
    roof["kernel_share_of_step"] = kernel_ms / ms if ms else None

    extras = {}
    if not args.no_extras:
        # end-to-end through the public API with host buffers, every step: H2D
        # upload of the graph layout from pinned host memory, the run
        # (multi-rank protocol for N > 1), D2H of the states (gathered over
        # ranks for N > 1).  Host preprocessing (dg_build_paths, once per
        # graph) is reported next to it, not inside it.
        e2e_t = []
        for _ in range(max(2, min(args.steps, 3))):
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t = time.perf_counter()
            dg.upload()
            t_up = time.perf_counter()
            if world == 1:
                dg.run(args.algo, mode=args.mode, source=0, epsilon=args.eps, damping=0.85)
                t_run = time.perf_counter()
                out = dg.get_states()
                d2h = int(out.nbytes)
                log(f"[bench] e2e step: upload {1e3 * (t_up - t):.1f} ms, run {1e3 * (t_run - t_up):.1f} ms, "
                    f"get_states {1e3 * (time.perf_counter() - t_run):.1f} ms")
            else:
                parallel.run_distributed(dg, args.algo, device=torch.device("cuda", local), source=0,
                                         epsilon=args.eps, damping=0.85)
                out = parallel.gather_states(dg, args.algo, n, device=torch.device("cuda", local)).cpu()
                d2h = out.numel() * out.element_size()
            torch.cuda.synchronize()
            dt = torch.tensor([time.perf_counter() - t], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(dt, op=dist.ReduceOp.MAX)
            e2e_t.append(float(dt.item()))
        info2 = dg.layout_info()
        e2e_s = statistics.median(e2e_t)
        extras["e2e"] = {"value": m / e2e_s, "unit": "edges/s", "h2d_bytes_per_step": info2["h2d_bytes"],
                         "d2h_bytes_per_step": d2h, "ms_per_step": e2e_s * 1e3,
                         "excludes": "host preprocessing (dg_build_paths, once per graph): see preprocess_s",
                         "preprocess_s": t_pre, "graph_gen_s": t_gen, "load_csr_s": t_load}
        # the metric's second algorithm on the same graph and preprocessing
        if args.algo == "pagerank" and not args.no_sssp and args.mode == "path":
            st_times, st_stats, st_syncs = timed_runs(make_step("sssp", "path"), max(args.steps, 5), 3, flush, world)
            sms = torch.tensor([sum(st_times) / len(st_times)], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(sms, op=dist.ReduceOp.MAX)
            sms = float(sms.item())
            s0 = st_stats[-1]
            rec = {"workload": WORKLOADS.get(("sssp", args.config), f"sssp on {args.config}"),
                   "time_to_convergence_ms": sms, "value": m / (sms / 1e3), "unit": "edges/s",
                   "steps": len(st_times), "rounds": s0["rounds"], "dense_rounds": s0["dense_rounds"],
                   "vertex_updates": s0["vertex_updates"], "entries_processed": s0["entries_processed"],
                   "kernel_ms": sum(x["kernel_ms"] for x in st_stats) / len(st_stats),
                   "roofline": roofline("sssp", args.config, s0, n, M, "path"), "dtype": "u32",
                   "delta": "library default (2*max weight; DESIGN.md R-DELTA)"}
            if st_syncs[-1]:
                rec["sync"] = st_syncs[-1]
            if rank == 0 and world == 1:
                ab_st = dg.run("sssp", mode="vertex", source=0)
                rec["ablation"] = {"mode": "vertex", "ms": ab_st["time_ms"], "rounds": ab_st["rounds"],
                                   "vertex_updates": ab_st["vertex_updates"],
                                   "edges_processed": ab_st["edges_processed"]}
            extras["sssp"] = rec
    if not args.no_extras and rank == 0 and world == 1:
        # vertex-centric ablation (north_star: total vertex updates next to it)
        if args.algo in ("pagerank", "sssp", "bfs", "wcc"):
            other = "vertex" if args.mode == "path" else "path"
            ab_st = dg.run(args.algo, mode=other, source=0, epsilon=args.eps, damping=0.85)
            extras["ablation"] = {"mode": other, "ms": ab_st["time_ms"], "rounds": ab_st["rounds"],
                                  "vertex_updates": ab_st["vertex_updates"],
                                  "edges_processed": ab_st["edges_processed"]}
        extras["cpu_baseline"] = cpu_baseline(args.algo, args.config, args.seed)

    value = m / (ms / 1e3)
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": DTYPE[args.algo], "data": "synthetic (seeded R-MAT, inputs/gen.c)",
            "config": {"workload": WORKLOADS.get((args.algo, args.config), f"{args.algo} on {args.config}"),
                       "graph": gname, "n": n, "m": m, "algo": args.algo, "mode": args.mode,
                       "epsilon": args.eps if args.algo == "pagerank" else None,
                       "delta": ("library default (SSSP 2*max weight, BFS 1; DESIGN.md R-DELTA)"
                                 if args.algo in ("sssp", "bfs") else None),
                       "l2": f"flushed between steps ({args.l2_flush_mb} MB write outside the step events)",
                       "parallelism": f"paths partitioned over {world} GPU(s)",
                       "preprocess_s": t_pre, "preprocess": ("once on rank 0, shares handed out as layout files"
                                                             if world > 1 else "dg_build_paths"),
                       "n_paths": info["n_paths"], "n_entries": M,
                       "n_partitions": info["n_partitions"], "n_layers": info["n_layers"],
                       "n_boundary": info["n_boundary"], "l_merge": args.l_merge},
            "time_to_convergence_ms": ms,
            "rounds": st0["rounds"], "dense_rounds": st0["dense_rounds"], "vertex_updates": st0["vertex_updates"],
            "edges_processed": st0["edges_processed"], "entries_processed": st0["entries_processed"],
            "kernel_ms": kernel_ms,
            "gpu_launches": int(sum(s["kernel_launches"] for s in stats)),
            "roofline": roof, "clocks": clk, "paper_context": PAPER_CONTEXT,
        }
        if syncs[-1]:
            sy = syncs[-1]
            line["sync"] = sy
            # NVLink traffic of the replica synchronisation (north_star reporting)
            line["exchanges"] = sy.get("syncs")
            line["nvlink_bytes_per_exchange"] = sy.get("nvlink_bytes_per_sync")
            line["nvlink_bytes_per_round"] = (sy.get("nvlink_bytes_per_sync", 0) * sy.get("syncs", 0) /
                                              max(1, st0["rounds"]))
        line.update(extras)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
