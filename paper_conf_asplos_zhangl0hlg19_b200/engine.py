"""Python face of the C ABI (same operations as include/digraph.h, marshalled
with ctypes).  Host arrays are numpy; device buffers are anything exposing a
CUDA ``data_ptr()`` (torch tensors)."""
from __future__ import annotations

import ctypes

import numpy as np

from . import _abi
from ._abi import check

ALGOS = {"sssp": _abi.DG_SSSP, "bfs": _abi.DG_BFS, "pagerank": _abi.DG_PAGERANK,
         "wcc": _abi.DG_WCC, "scc": _abi.DG_SCC, "adsorption": _abi.DG_ADSORPTION}
MODES = {"path": _abi.DG_MODE_PATH, "vertex": _abi.DG_MODE_VERTEX}
STATE_DTYPE = {"sssp": np.uint32, "bfs": np.uint32, "pagerank": np.float32,
               "adsorption": np.float32, "wcc": np.int32, "scc": np.int32}
INF = _abi.DG_INF


def _p(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


def default_params():
    p = _abi.dg_path_params()
    _abi.lib().dg_default_params(ctypes.byref(p))
    return p


class DiGraph:
    """One graph on one CUDA device (dg_create ... dg_destroy)."""

    def __init__(self, device=0):
        self._L = _abi.lib()
        self._h = ctypes.c_void_p()
        check(self._L.dg_create(ctypes.byref(self._h), int(device)), "dg_create")
        self.n = 0
        self.m = 0
        self.algo = None

    # -- lifecycle -----------------------------------------------------------
    def close(self):
        if self._h:
            self._L.dg_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- dg_load_csr / dg_build_paths / dg_upload ----------------------------
    def load_csr(self, n, row_ptr, col, weight=None):
        self._row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        self._col = np.ascontiguousarray(col, dtype=np.int32)
        self._w = None if weight is None else np.ascontiguousarray(weight, dtype=np.int32)
        n_new, m_new = int(n), int(self._row_ptr[-1])
        rc = self._L.dg_load_csr(self._h, n_new, m_new, _p(self._row_ptr), _p(self._col), _p(self._w))
        self._row_ptr = self._col = self._w = None  # dg_load_csr copied them
        check(rc, "dg_load_csr")  # on failure the handle keeps the previous graph
        self.n, self.m = n_new, m_new
        self.p2p_key = None  # the library freed any exchange region
        return self

    def load_graph(self, g):
        """Load an ``inputs.Graph``."""
        return self.load_csr(g.n, g.row_ptr, g.col, g.w)

    @staticmethod
    def _path_params(d_max=16, l_merge=64, n_sub=64, order="degree", hot_factor=2.0,
                     part_entries=0, rank=0, world=1, merge_rule="relaxed", n_proxy=8192, placement="locality"):
        p = default_params()
        p.d_max, p.l_merge, p.n_sub = d_max, l_merge, n_sub
        p.order = 0 if order == "degree" else 1
        p.hot_factor, p.part_entries, p.rank, p.world = hot_factor, part_entries, rank, world
        p.merge_rule = {"paper": 0, "relaxed": 1}[merge_rule]
        p.n_proxy = n_proxy
        p.placement = {"round_robin": 0, "locality": 1}[placement]
        return p

    def build_paths(self, d_max=16, l_merge=64, n_sub=64, order="degree", hot_factor=2.0,
                    part_entries=0, rank=0, world=1, merge_rule="relaxed", n_proxy=8192, placement="locality"):
        p = self._path_params(d_max, l_merge, n_sub, order, hot_factor, part_entries, rank, world, merge_rule,
                              n_proxy, placement)
        check(self._L.dg_build_paths(self._h, ctypes.byref(p)), "dg_build_paths")
        self.p2p_key = None  # the library freed any exchange region
        return self

    def build_paths_shared(self, prefix, world, rank=0, **kw):
        """dg_build_paths_shared: one preprocessing pass for `world` ranks, rank
        r's layout written to "<prefix>.<r>"; this handle keeps `rank`'s."""
        p = self._path_params(rank=rank, world=world, **kw)
        check(self._L.dg_build_paths_shared(self._h, ctypes.byref(p), prefix.encode()), "dg_build_paths_shared")
        self.p2p_key = None
        return self

    def save_layout(self, path):
        check(self._L.dg_save_layout(self._h, path.encode()), "dg_save_layout")
        return self

    def load_layout(self, path):
        """dg_load_layout: this handle's graph and layout from a layout file."""
        check(self._L.dg_load_layout(self._h, path.encode()), "dg_load_layout")
        info = self.layout_info()
        self.n, self.m = info["n"], info["m"]
        self.p2p_key = None
        return self

    def upload(self):
        check(self._L.dg_upload(self._h), "dg_upload")
        return self

    def set_vertex_params(self, p_inj, p_cont, inj):
        a = [np.ascontiguousarray(x, dtype=np.float64) for x in (p_inj, p_cont, inj)]
        check(self._L.dg_set_vertex_params(self._h, *[_p(x) for x in a]), "dg_set_vertex_params")

    # -- dg_run / dg_get_states ----------------------------------------------
    @staticmethod
    def _param(algo, damping, delta):
        """dg_run's `param`: PageRank damping; SSSP/BFS bucket width (None: library
        default, 0: unbounded, k > 0: k; include/digraph.h, DESIGN.md R-DELTA)."""
        if algo in ("sssp", "bfs"):
            return 0.0 if delta is None else (-1.0 if delta == 0 else float(delta))
        return float(damping)

    def run(self, algo, source=0, epsilon=1e-7, damping=0.85, mode="path", max_rounds=0,
            allow_noconv=False, delta=None):
        st = _abi.dg_run_stats()
        rc = self._L.dg_run(self._h, ALGOS[algo], int(source), float(epsilon), self._param(algo, damping, delta),
                            MODES[mode], int(max_rounds), ctypes.byref(st))
        if rc != 0 and not (allow_noconv and rc == -4):
            check(rc, "dg_run")
        self.algo = algo
        d = st.as_dict()
        d["converged"] = rc == 0
        return d

    def get_states(self, out=None):
        """Final states: numpy array (host) or, if ``out`` is a CUDA tensor, filled in place."""
        if out is not None and hasattr(out, "data_ptr") and getattr(out, "is_cuda", False):
            check(self._L.dg_get_states(self._h, ctypes.c_void_p(out.data_ptr()), self.n, 1), "dg_get_states")
            return out
        res = out if out is not None else np.empty(self.n, dtype=STATE_DTYPE[self.algo])
        check(self._L.dg_get_states(self._h, _p(res), self.n, 0), "dg_get_states")
        return res

    # -- inspection ------------------------------------------------------------
    def layout_info(self):
        info = _abi.dg_layout_info()
        check(self._L.dg_get_layout_info(self._h, ctypes.byref(info)), "dg_get_layout_info")
        return info.as_dict()

    def export_paths(self):
        info = self.layout_info()
        P, M, Q = info["n_paths"], info["n_entries"], info["n_partitions"]
        path_off = np.empty(P + 1, np.int64)
        verts = np.empty(max(M, 1), np.int32)
        layer = np.empty(max(P, 1), np.int32)
        scc = np.empty(max(P, 1), np.int64)
        midx = np.empty(max(P, 1), np.int64)
        hot = np.empty(max(P, 1), np.uint8)
        part_off = np.empty(Q + 1, np.int64)
        check(self._L.dg_export_paths(self._h, _p(path_off), _p(verts), _p(layer), _p(scc), _p(midx),
                                      _p(hot), _p(part_off)), "dg_export_paths")
        return dict(path_off=path_off, vertices=verts[:M], layer=layer[:P], scc=scc[:P],
                    merged_index=midx[:P], hot=hot[:P].astype(bool), part_off=part_off)

    # -- multi-GPU protocol ----------------------------------------------------
    def boundary_vertices(self):
        nb = ctypes.c_int64()
        check(self._L.dg_boundary_size(self._h, ctypes.byref(nb)), "dg_boundary_size")
        out = np.empty(max(nb.value, 1), np.int32)
        check(self._L.dg_boundary_vertices(self._h, _p(out)), "dg_boundary_vertices")
        return out[: nb.value]

    def run_begin(self, algo, source=0, epsilon=1e-7, damping=0.85, delta=None):
        check(self._L.dg_run_begin(self._h, ALGOS[algo], int(source), float(epsilon),
                                   self._param(algo, damping, delta)), "dg_run_begin")
        self.algo = algo

    def rounds(self, max_rounds):
        a = ctypes.c_int64()
        check(self._L.dg_rounds(self._h, int(max_rounds), ctypes.byref(a)), "dg_rounds")
        return a.value

    def boundary_pack(self, buf):
        check(self._L.dg_boundary_pack(self._h, ctypes.c_void_p(buf.data_ptr())), "dg_boundary_pack")

    def boundary_unpack(self, buf):
        a = ctypes.c_int64()
        check(self._L.dg_boundary_unpack(self._h, ctypes.c_void_p(buf.data_ptr()), ctypes.byref(a)),
              "dg_boundary_unpack")
        return a.value

    # ---- peer-memory boundary exchange (include/digraph.h dg_p2p_*) ----
    P2P_HANDLE_BYTES = 64

    def p2p_alloc(self, world, rank):
        """Allocate this rank's exchange region; returns its IPC handle (bytes)."""
        h = ctypes.create_string_buffer(self.P2P_HANDLE_BYTES)
        check(self._L.dg_p2p_alloc(self._h, int(world), int(rank), h), "dg_p2p_alloc")
        return h.raw

    def p2p_open(self, handles):
        """Map every peer's region; ``handles`` = list of IPC handles in rank order."""
        blob = b"".join(handles)
        assert len(blob) == self.P2P_HANDLE_BYTES * len(handles)
        check(self._L.dg_p2p_open(self._h, ctypes.create_string_buffer(blob, len(blob))), "dg_p2p_open")

    def boundary_exchange(self):
        a = ctypes.c_int64()
        check(self._L.dg_boundary_exchange(self._h, ctypes.byref(a)), "dg_boundary_exchange")
        return a.value

    def scc_phase(self, phase):
        """dg_scc_phase: 0 forward colouring, 1 backward marks; returns the
        vertices this rank signalled."""
        a = ctypes.c_int64()
        check(self._L.dg_scc_phase(self._h, int(phase), ctypes.byref(a)), "dg_scc_phase")
        return a.value

    def scc_assign(self):
        """dg_scc_assign: returns this rank's unassigned vertices."""
        a = ctypes.c_int64()
        check(self._L.dg_scc_assign(self._h, ctypes.byref(a)), "dg_scc_assign")
        return a.value

    def run_fused(self, local_rounds=4, max_rounds=0):
        """The whole multi-rank run in one launch (dg_run_fused); returns
        (exchanges, converged)."""
        ex, conv = ctypes.c_int64(), ctypes.c_int64()
        check(self._L.dg_run_fused(self._h, int(local_rounds), int(max_rounds), ctypes.byref(ex), ctypes.byref(conv)),
              "dg_run_fused")
        return ex.value, bool(conv.value)

    def normalize_states(self, buf):
        check(self._L.dg_normalize_states(self._h, ctypes.c_void_p(buf.data_ptr()), buf.numel()),
              "dg_normalize_states")
        return buf

    def run_end(self):
        st = _abi.dg_run_stats()
        check(self._L.dg_run_end(self._h, ctypes.byref(st)), "dg_run_end")
        return st.as_dict()
