"""-m gpu: the real multi-rank device path (dg_run_begin / dg_rounds and
either the peer-memory exchange dg_boundary_exchange -- CUDA IPC between the
two processes, device-side epoch flags -- or dg_boundary_pack / all-reduce /
dg_boundary_unpack) with two ranks time-sharing cuda:0.  NCCL refuses two
ranks on one GPU, so the host collective here is gloo on CUDA tensors."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import inputs
from oracle import algorithms as OA

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _graph():
    return inputs.rmat(13, 8192, 80000, seed=31)


def _worker(rank, world, port, algo, q, sparse=False, exchange="fused"):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if sparse:  # every round with <= n/4 signalled vertices walks sparse
        os.environ.update(DG_SPARSE_DIV="1", DG_SPARSE_MIN_M="0")
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph, parallel
    g = _graph()
    dg = DiGraph(device=0)
    dg.load_graph(g).build_paths(part_entries=256, rank=rank, world=world)
    if algo == "adsorption":
        dg.set_vertex_params(*inputs.adsorption_params(g.n, seed=3))
    dev = torch.device("cuda", 0)
    stats, info = parallel.run_distributed(dg, algo, source=0, epsilon=1e-7, device=dev, exchange=exchange)
    out = parallel.gather_states(dg, algo, g.n, device=dev)
    if rank == 0:
        q.put((out.cpu().numpy().copy(), info, stats))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("exchange", ["fused", "p2p", "collective"])
@pytest.mark.parametrize("sparse", [False, True])
@pytest.mark.parametrize("algo", ["sssp", "wcc", "pagerank", "adsorption", "scc"])
def test_two_ranks_on_one_gpu_match_oracle(algo, sparse, exchange, cuda_required):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, algo, q, sparse, exchange)) for r in range(2)]
    for p in procs:
        p.start()
    got, info, stats = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    g = _graph()
    src, dst, w = g.edges()
    assert info["boundary"] > 0 and info["exchange"] == exchange
    if algo == "sssp":
        exp, _ = OA.sssp_bellman_ford(g.n, src, dst, w, 0)
        assert np.array_equal(got.view(np.uint32).astype(np.int64), exp)
    elif algo == "wcc":
        exp, _ = OA.wcc_label_propagation(g.n, src, dst)
        assert np.array_equal(got.astype(np.int64), exp)
    elif algo == "scc":
        exp = OA.scc_tarjan(g.n, src, dst)
        assert np.array_equal(got.astype(np.int64), exp)
        assert info["scc_iterations"] >= 1
    elif algo == "adsorption":
        p_inj, p_cont, inj = inputs.adsorption_params(g.n, seed=3)
        exp, _ = OA.adsorption_jacobi(g.n, src, dst, w, p_inj, p_cont, inj, tol=1e-12)
        got = got.astype(np.float64)
        assert np.abs(got - exp).sum() / np.abs(exp).sum() <= 1e-4
        assert np.all(np.abs(got - exp) <= 1e-3 * exp + 100 * 1e-7)
    else:
        exp, _ = OA.pagerank_power(g.n, src, dst)
        assert np.abs(got.astype(np.float64) - exp).sum() <= 1e-4
        assert (np.abs(got.astype(np.float64) - exp) / exp).max() <= 1e-3
