"""Multi-GPU host logic on CPU (-m "not gpu"): world-size-2 gloo runs of the
real multi-rank preprocessing (dg_build_paths with rank/world: path
partitioning and boundary set) and of the real driver protocol
(`parallel.run_distributed` / `gather_states`), with a test-only CPU engine
that walks the rank's exported paths with the kernel's semantics.  The
product itself has no CPU path; this engine exists only in the tests.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import inputs
from oracle import algorithms as OA

FX = 1 << 32


class CpuPathEngine:
    """Mimics libdigraph's per-rank semantics on the rank's own paths."""

    def __init__(self, g, rank, world):
        from paper_conf_asplos_zhangl0hlg19_b200 import DiGraph
        dg = DiGraph()
        dg.load_graph(g)
        dg.build_paths(part_entries=64, rank=rank, world=world)
        ex = dg.export_paths()
        self.bnd = dg.boundary_vertices().astype(np.int64)
        off, v = ex["path_off"], ex["vertices"].astype(np.int64)
        self.paths = [v[off[i]:off[i + 1]] for i in range(len(off) - 1)]
        src, dst, w = g.edges()
        self.wmap = {}
        for a, b, c in zip(src.tolist(), dst.tolist(), w.tolist()):
            self.wmap.setdefault((a, b), []).append(c)
        self.n = g.n
        self.outdeg = np.diff(g.row_ptr)
        # per-path weights / mirrors
        self.pw = []
        used = {}
        for p in self.paths:
            ws = []
            for a, b in zip(p[:-1].tolist(), p[1:].tolist()):
                k = used.get((a, b), 0)
                ws.append(self.wmap[(a, b)][k])
                used[(a, b)] = k + 1
            self.pw.append(ws)

    def boundary_vertices(self):
        return self.bnd

    def set_vertex_params(self, p_inj, p_cont, inj):
        """Adsorption inputs (DESIGN.md R-ADS), as dg_set_vertex_params."""
        self.ads = (np.asarray(p_inj, np.float64), np.asarray(p_cont, np.float64), np.asarray(inj, np.float64))

    def run_begin(self, algo, source=0, epsilon=1e-7, damping=0.85):
        self.algo = algo
        if algo == "scc":
            # vertices on none of this rank's paths carry their own id (MIN-gathered)
            present = np.zeros(self.n, bool)
            for p in self.paths:
                present[p] = True
            self.label = np.where(present, -1, np.arange(self.n)).astype(np.int64)
            self.x = np.full(self.n, OA.UNREACHED, np.int64)
            self.mark = np.zeros(self.n, bool)
            self.phase = -1
            return
        if algo in ("sssp", "wcc"):
            self.x = np.full(self.n, OA.UNREACHED, np.int64)
            if algo == "sssp":
                self.x[source] = 0
            else:
                self.x = np.arange(self.n, dtype=np.int64)
        else:
            self.eps = int(epsilon * FX)
            if algo == "adsorption":
                # x_v = p_inj I + sum_u p_cont(u) w(u,v)/W(u) x_u: path edge t of a
                # path carries p_cont(p[t]) * w / W(p[t])
                p_inj, p_cont, inj = self.ads
                self.T = np.array([int(x * FX) for x in (p_inj * inj)], np.int64)
                W = np.zeros(self.n)
                for (a, _), ws in self.wmap.items():
                    W[a] += sum(ws)
                self.ecoef = [[p_cont[u] * wt / W[u] for u, wt in zip(p[:-1].tolist(), ws)]
                              for p, ws in zip(self.paths, self.pw)]
            else:
                self.T = np.full(self.n, int((1 - damping) * FX), np.int64)
                coef = np.where(self.outdeg > 0, damping / np.maximum(self.outdeg, 1), 0.0)
                self.ecoef = [[coef[u] for u in p[:-1].tolist()] for p in self.paths]
            self.S = [np.zeros(len(p), np.int64) for p in self.paths]
            self.base = self.T[self.bnd].copy()

    def _walk_min(self):
        changed = 0
        for p, ws in zip(self.paths, self.pw):
            cur = None
            for t, v in enumerate(p.tolist()):
                a = self.x[v]
                if cur is not None:
                    cand = cur + (ws[t - 1] if self.algo == "sssp" else 0)
                    if cand < a:
                        self.x[v] = cand
                        changed += 1
                        a = cand
                cur = a
            if self.algo == "wcc":  # backward along the path
                cur = None
                for v in p[::-1].tolist():
                    a = self.x[v]
                    if cur is not None and cur < a:
                        self.x[v] = cur
                        changed += 1
                        a = cur
                    cur = a
        return changed

    def _walk_accum(self):
        pushed = 0
        for p, S, ec in zip(self.paths, self.S, self.ecoef):
            carry = 0.0
            for t, v in enumerate(p.tolist()):
                pin = carry if t > 0 else 0.0
                pfx = int(pin * FX)
                if pfx:
                    self.T[v] += pfx
                    pushed += 1
                if t < len(p) - 1:
                    pend = (self.T[v] - pfx) - S[t]      # the total before this walk's push
                    pend = pend if pend >= self.eps else 0
                    carry = ec[t] * ((pend / FX) + pin)
                    S[t] += pend + pfx
                else:
                    carry = 0.0
        return pushed

    # ---- SCC colouring phases (include/digraph.h dg_scc_phase / dg_scc_assign)
    def scc_phase(self, phase):
        self.phase = phase
        un = self.label < 0
        if phase == 0:
            self.x = np.where(un, np.arange(self.n), OA.UNREACHED).astype(np.int64)
            self.mark[:] = False
            return int(un.sum())
        self.mark = un & (self.x == np.arange(self.n))
        return int(self.mark.sum())

    def scc_assign(self):
        sel = self.mark & (self.label < 0)
        self.label[sel] = self.x[sel]
        self.phase = -1
        return int((self.label < 0).sum())

    def _walk_scc(self):
        changed = 0
        for p in self.paths:
            vs = p.tolist()
            if self.phase == 0:  # forward min colour; assigned vertices break the path
                cur = None
                for v in vs:
                    if self.label[v] >= 0:
                        cur = None
                        continue
                    if cur is not None and cur < self.x[v]:
                        self.x[v] = cur
                        changed += 1
                    cur = self.x[v]
            else:  # backward marks inside a colour
                for a, b in zip(vs[-2::-1], vs[:0:-1]):
                    if (self.mark[b] and not self.mark[a] and self.label[a] < 0 and self.label[b] < 0
                            and self.x[a] == self.x[b]):
                        self.mark[a] = True
                        changed += 1
        return changed

    def rounds(self, k):
        walk = (self._walk_scc if self.algo == "scc" else
                self._walk_min if self.algo in ("sssp", "wcc") else self._walk_accum)
        for _ in range(100000):
            if walk() == 0:
                return 0
        raise RuntimeError("local rounds did not converge")

    def boundary_pack(self, buf):
        if self.algo == "scc" and self.phase == 1:  # marks: 0 = marked, MIN = OR
            buf.copy_(torch.from_numpy(np.where(self.mark[self.bnd], 0, 1).astype(np.int32)))
        elif self.algo in ("sssp", "wcc", "scc"):
            buf.copy_(torch.from_numpy(self.x[self.bnd].astype(np.int32)))
        else:
            buf.copy_(torch.from_numpy(self.T[self.bnd] - self.base))

    def boundary_unpack(self, buf):
        if len(self.bnd) == 0:
            return 0
        b = buf.numpy().astype(np.int64)
        if self.algo == "scc" and self.phase == 1:
            new = (b == 0) & ~self.mark[self.bnd] & (self.label[self.bnd] < 0)
            self.mark[self.bnd[new]] = True
            return int(new.sum())
        if self.algo in ("sssp", "wcc", "scc"):
            new = np.minimum(self.x[self.bnd], b)
            act = int((new < self.x[self.bnd]).sum())
            self.x[self.bnd] = new
            return act
        t = self.base + b
        act = int(((t - self.T[self.bnd]) > 0).sum())
        self.T[self.bnd] = t
        self.base = t.copy()
        return act

    def run_end(self):
        return {}

    def get_states(self, out):
        if self.algo == "scc":
            out.copy_(torch.from_numpy(self.label.astype(np.int32)))
        elif self.algo in ("sssp", "wcc"):
            out.copy_(torch.from_numpy(self.x.astype(np.int32)))
        else:
            out.copy_(torch.from_numpy((self.T / FX).astype(np.float32)))
        return out

    def normalize_states(self, buf):
        buf /= buf.sum()
        return buf


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


class NoPeerEngine(CpuPathEngine):
    """Peer mapping fails on rank 1 only (as when a process cannot see its
    peers' GPUs): every rank must fall back to the collective together."""

    def p2p_alloc(self, world, rank):
        if rank == 1:
            raise RuntimeError("no peer access")
        return b"h" * 64

    def p2p_open(self, handles):
        raise AssertionError("must not be reached: rank 1 failed dg_p2p_alloc")


class FusedModelEngine(CpuPathEngine):
    """Host model of dg_run_fused's protocol (path_kernel + mr_exchange):
    between local round batches every rank publishes its activity =
    signalled work + boundary values that differ from the previous
    exchange's result (MIN) or non-zero growth (SUM); the boundary is
    reduced; the run stops when the summed activity of an exchange is 0.
    Here a rendezvous is a gloo collective, in the kernel an epoch flag."""

    def p2p_alloc(self, world, rank):
        return b"m" * 64

    def p2p_open(self, handles):
        pass

    def run_fused(self, local_rounds=4, max_rounds=0):
        nb = len(self.bnd)
        minalgo = self.algo in ("sssp", "wcc", "scc")
        last = None
        for ex in range(1, 100000):
            act = self.rounds(local_rounds)
            buf = torch.zeros(max(nb, 1), dtype=torch.int32 if minalgo else torch.int64)
            if nb:
                self.boundary_pack(buf)
            vals = buf.numpy()[:nb].astype(np.int64)
            dirty = int((vals != last).sum()) if (minalgo and last is not None) else (
                nb if minalgo else int((vals != 0).sum()))
            total = torch.tensor([act + dirty], dtype=torch.int64)
            dist.all_reduce(total)
            dist.all_reduce(buf, op=dist.ReduceOp.MIN if minalgo else dist.ReduceOp.SUM)
            self.boundary_unpack(buf)
            if minalgo:
                last = buf.numpy()[:nb].astype(np.int64)
            if int(total.item()) == 0:
                return ex, True
        return ex, False


def _worker(rank, world, port, algo, q, exchange=None):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_asplos_zhangl0hlg19_b200 import parallel
    g = inputs.rmat(10, 1024, 6000, seed=21, weights=(1, 20))
    eng = {"p2p": NoPeerEngine, "fused": FusedModelEngine}.get(exchange, CpuPathEngine)(g, rank, world)
    if algo == "adsorption":
        eng.set_vertex_params(*inputs.adsorption_params(g.n, seed=3))
    stats, info = parallel.run_distributed(eng, algo, source=0, epsilon=1e-7, device=torch.device("cpu"),
                                           exchange=exchange)
    out = parallel.gather_states(eng, algo, g.n, device=torch.device("cpu"))
    if rank == 0:
        q.put((out.numpy().copy(), info))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("algo,exchange", [("sssp", None), ("wcc", None), ("pagerank", None), ("adsorption", None),
                                           ("sssp", "p2p"), ("sssp", "fused"), ("wcc", "fused"),
                                           ("pagerank", "fused"), ("adsorption", "fused"), ("scc", None),
                                           ("scc", "fused")])
def test_two_rank_protocol_matches_oracle(algo, exchange):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, algo, q, exchange)) for r in range(2)]
    for p in procs:
        p.start()
    got, info = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = inputs.rmat(10, 1024, 6000, seed=21, weights=(1, 20))
    src, dst, w = g.edges()
    assert info["boundary"] > 0 and info["syncs"] >= 1
    assert info["exchange"] == ("fused" if exchange == "fused" else "collective")
    assert ("p2p_error" in info) == (exchange == "p2p")
    if algo == "sssp":
        exp, _ = OA.sssp_bellman_ford(g.n, src, dst, w, 0)
        assert np.array_equal(got.astype(np.int64), exp)
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
        assert np.abs(got - exp).sum() / np.abs(exp).sum() <= 1e-4
        assert np.all(np.abs(got - exp) <= 1e-3 * exp + 100 * 1e-7)
    else:
        exp, _ = OA.pagerank_power(g.n, src, dst)
        assert np.abs(got - exp).sum() <= 1e-4
        assert (np.abs(got - exp) / exp).max() <= 1e-3
