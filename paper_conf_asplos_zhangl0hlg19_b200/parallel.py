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
  2. boundary states are exchanged: MIN for SSSP/BFS/WCC, SUM of pending
     deltas for PageRank/Adsorption.  ``exchange="fused"`` (default on
     GPUs): the whole run is ONE dg_run_fused launch per rank -- the
     persistent kernel does the peer-memory exchange below between its
     rounds and tests global convergence on the devices (steps 1-4 without
     any host involvement).  ``exchange="p2p"``: one
     dg_boundary_exchange -- pack, device-side epoch flags and an elementwise
     reduction read straight from every peer's HBM (CUDA IPC over
     NVLink/NVSwitch), unpack; no host collective moves boundary states.
     ``exchange="collective"``: pack kernel, ``dist.all_reduce`` of the
     buffer (NCCL on GPUs, gloo in the CPU tests), unpack kernel;
  3. unpack re-activates the changed vertices;
  4. the activated counts are all-reduced (8 bytes); zero everywhere = done.

The engine argument only needs the ``DiGraph`` protocol methods (run_begin,
rounds, boundary_pack, boundary_unpack, run_end, get_states), so the host
logic is testable with a CPU engine under the gloo backend.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

SUM_ALGOS = ("pagerank", "adsorption")
MIN_ALGOS = ("sssp", "bfs", "wcc", "scc")  # SCC phases exchange colours / marks with MIN


def boundary_buffer(n_boundary, algo, device):
    # SUM algorithms exchange exact 64-bit fixed-point growth of the totals
    dtype = torch.int64 if algo in SUM_ALGOS else torch.int32
    return torch.zeros(max(int(n_boundary), 1), dtype=dtype, device=device)


def p2p_setup(engine, group=None, device=None):
    """Allocate this rank's exchange region and map every peer's (once per
    layout): the 64-byte IPC handles travel through ``dist.all_gather_object``.
    Returns None when every rank mapped every peer, else the first error (all
    ranks agree, so they all fall back to the collective exchange together --
    e.g. when each process sees only its own GPU and CUDA IPC cannot map a
    peer's memory)."""
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    key = (world, rank, len(engine.boundary_vertices()))
    if getattr(engine, "p2p_key", None) == key:
        return None
    err = None
    try:
        h = engine.p2p_alloc(world, rank)
    except Exception as e:  # noqa: BLE001 -- reported to every rank below
        h, err = b"", f"dg_p2p_alloc: {e}"
    hs = [None] * world
    dist.all_gather_object(hs, h, group=group)
    if err is None and all(len(x) == len(h) for x in hs):
        try:
            engine.p2p_open(hs)
        except Exception as e:  # noqa: BLE001
            err = f"dg_p2p_open: {e}"
    elif err is None:
        err = "a peer failed dg_p2p_alloc"
    errs = [None] * world
    dist.all_gather_object(errs, err, group=group)
    first = next((e for e in errs if e), None)
    if first is None:
        engine.p2p_key = key
    return first


def _converge(engine, exchange, nb, buf, op, local_rounds, max_outer, group, device):
    """One multi-rank run (or SCC phase) to global convergence; returns the
    number of boundary exchanges."""
    if exchange == "fused":
        syncs, converged = engine.run_fused(local_rounds)
        if not converged:
            raise RuntimeError("multi-rank run did not converge")
        return syncs
    active = torch.zeros(1, dtype=torch.int64, device=device)
    for syncs in range(1, max_outer + 1):
        engine.rounds(local_rounds)
        if exchange == "p2p":
            act = engine.boundary_exchange()
        else:
            if nb:
                engine.boundary_pack(buf)
            dist.all_reduce(buf, op=op, group=group)
            act = engine.boundary_unpack(buf)
        active.fill_(int(act))
        dist.all_reduce(active, op=dist.ReduceOp.SUM, group=group)
        if int(active.item()) == 0:
            return syncs
    raise RuntimeError("multi-rank run did not converge")


def run_distributed(engine, algo, source=0, epsilon=1e-7, damping=0.85, local_rounds=4,
                    max_outer=1_000_000, device=None, group=None, exchange=None):
    """Run ``algo`` to global convergence.  Returns (stats, sync_info).
    ``exchange``: "fused" (default on CUDA devices), "p2p" or "collective".
    SCC runs its colouring iterations (include/digraph.h dg_scc_phase): per
    iteration a forward-colouring phase and a backward-marking phase, each a
    multi-rank run with MIN exchanges, then dg_scc_assign; the iterations stop
    when no rank has an unassigned vertex."""
    if algo not in SUM_ALGOS + MIN_ALGOS:
        raise ValueError(f"{algo}: no multi-rank protocol")
    device = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                                if torch.cuda.is_available() else torch.device("cpu"))
    if exchange is None:
        exchange = "fused" if device.type == "cuda" else "collective"
    if exchange not in ("fused", "p2p", "collective"):
        raise ValueError(f"exchange={exchange!r}: 'fused', 'p2p' or 'collective'")
    nb = len(engine.boundary_vertices())
    buf = boundary_buffer(nb, algo, device)
    op = dist.ReduceOp.SUM if algo in SUM_ALGOS else dist.ReduceOp.MIN
    engine.run_begin(algo, source=source, epsilon=epsilon, damping=damping)
    p2p_error = None
    if exchange in ("fused", "p2p"):
        p2p_error = p2p_setup(engine, group)
        if p2p_error:
            import sys
            print(f"[parallel] peer-memory exchange unavailable ({p2p_error}); using the collective",
                  file=sys.stderr, flush=True)
            exchange = "collective"
    args = (exchange, nb, buf, op, local_rounds, max_outer, group, device)
    syncs, iterations = 0, 0
    if algo == "scc":
        rem = torch.zeros(1, dtype=torch.int64, device=device)
        while True:
            for phase in (0, 1):
                engine.scc_phase(phase)
                syncs += _converge(engine, *args)
            rem.fill_(int(engine.scc_assign()))
            dist.all_reduce(rem, op=dist.ReduceOp.SUM, group=group)
            iterations += 1
            if int(rem.item()) == 0:
                break
    else:
        syncs = _converge(engine, *args)
    stats = engine.run_end()
    bytes_per_sync = buf.numel() * buf.element_size()
    if exchange in ("fused", "p2p"):
        # a rank reads, for each boundary vertex its paths hold, the 8-byte slot
        # of every other rank holding it (dg_layout_info.boundary_reads)
        reads = engine.layout_info().get("boundary_reads") if hasattr(engine, "layout_info") else None
        bytes_per_sync = 8 * (reads if reads is not None else nb * (dist.get_world_size(group) - 1))
    info = {"syncs": syncs, "boundary": nb, "nvlink_bytes_per_sync": bytes_per_sync, "exchange": exchange}
    if algo == "scc":
        info["scc_iterations"] = iterations
    if p2p_error:
        info["p2p_error"] = p2p_error
    return stats, info


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
