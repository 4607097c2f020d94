"""Multi-GPU driver (north_star (5)): one process per GPU, paths partitioned
across ranks (dg_build_paths(rank, world): round-robin over the priority-
ordered partitions), only replica/boundary vertex states cross NVLink.

Protocol per outer iteration ("state propagation between
paths is done through state synchronization of vertex replicas ... in
batches"):
  1. every rank runs ``local_rounds`` local rounds (default 4: the sync cost --
     one NCCL all-reduce of the boundary over NVLink -- is amortised over a
     few rounds while replicas stay at most a few rounds apart), or fewer if
     its local active counter reaches zero;
  2. boundary states are packed (device kernel) and all-reduced with NCCL:
     MIN for SSSP/BFS/WCC, SUM of pending deltas for PageRank/Adsorption;
  3. unpack (device kernel) re-activates partitions of changed vertices;
  4. the activated-partition counts are all-reduced; zero everywhere = done.

The engine argument only needs the ``DiGraph`` protocol methods (run_begin,
rounds, boundary_pack, boundary_unpack, run_end, get_states), so the host
logic is testable with a CPU engine under the gloo backend.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

SUM_ALGOS = ("pagerank", "adsorption")
MIN_ALGOS = ("sssp", "bfs", "wcc")


def boundary_buffer(n_boundary, algo, device):
    # SUM algorithms exchange exact 64-bit fixed-point growth of the totals
    dtype = torch.int64 if algo in SUM_ALGOS else torch.int32
    return torch.zeros(max(int(n_boundary), 1), dtype=dtype, device=device)


def run_distributed(engine, algo, source=0, epsilon=1e-7, damping=0.85, local_rounds=4,
                    max_outer=1_000_000, device=None, group=None):
    """Run ``algo`` to global convergence.  Returns (stats, sync_info)."""
    if algo not in SUM_ALGOS + MIN_ALGOS:
        raise ValueError(f"{algo}: no multi-rank protocol (SCC is single-rank)")
    device = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                                if torch.cuda.is_available() else torch.device("cpu"))
    nb = len(engine.boundary_vertices())
    buf = boundary_buffer(nb, algo, device)
    op = dist.ReduceOp.SUM if algo in SUM_ALGOS else dist.ReduceOp.MIN
    active = torch.zeros(1, dtype=torch.int64, device=device)
    engine.run_begin(algo, source=source, epsilon=epsilon, damping=damping)
    syncs, bytes_per_sync = 0, buf.numel() * buf.element_size()
    for _ in range(max_outer):
        engine.rounds(local_rounds)
        if nb:
            engine.boundary_pack(buf)
        dist.all_reduce(buf, op=op, group=group)
        act = engine.boundary_unpack(buf)
        syncs += 1
        active.fill_(int(act))
        dist.all_reduce(active, op=dist.ReduceOp.SUM, group=group)
        if int(active.item()) == 0:
            break
    else:
        raise RuntimeError("multi-rank run did not converge")
    stats = engine.run_end()
    return stats, {"syncs": syncs, "boundary": nb, "nvlink_bytes_per_sync": bytes_per_sync}


def gather_states(engine, algo, n, device=None, group=None):
    """Global final states on every rank (device tensor): MIN over ranks for
    SSSP/BFS/WCC (a rank not holding a vertex keeps its initial value), MAX
    for PageRank/Adsorption totals (monotone from the same initial value on
    every rank), then PageRank is normalised."""
    device = device if device is not None else torch.device("cuda", torch.cuda.current_device())
    dtype = torch.float32 if algo in SUM_ALGOS else torch.int32
    out = torch.empty(n, dtype=dtype, device=device)
    engine.get_states(out)
    op = dist.ReduceOp.MAX if algo in SUM_ALGOS else dist.ReduceOp.MIN
    dist.all_reduce(out, op=op, group=group)
    if algo == "pagerank":
        engine.normalize_states(out)
    return out
