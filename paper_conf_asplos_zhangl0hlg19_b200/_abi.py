"""Thin ctypes binding of libdigraph.so (include/digraph.h).

Argument marshalling only: every computation step runs in the native
library (host preprocessing in C++, the hot path in CUDA kernels).  The
function names are the C names.  Loading fails loudly if the library is
missing; there is no Python or CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DG_LIB_PATH") or os.path.join(_HERE, "libdigraph.so")  # env: developer builds only

DG_SSSP, DG_BFS, DG_PAGERANK, DG_WCC, DG_SCC, DG_ADSORPTION = range(6)
DG_MODE_PATH, DG_MODE_VERTEX = 0, 1
DG_INF = 0x7FFFFFFF
ERRORS = {-1: "DG_EINVAL", -2: "DG_ENOMEM", -3: "DG_ENOCUDA", -4: "DG_ENOCONV"}

# every symbol include/digraph.h declares
EXPORTS = [
    "dg_default_params", "dg_create", "dg_destroy", "dg_last_error", "dg_load_csr",
    "dg_build_paths", "dg_upload", "dg_set_vertex_params", "dg_run", "dg_get_states",
    "dg_get_layout_info", "dg_export_paths", "dg_boundary_size", "dg_boundary_vertices",
    "dg_run_begin", "dg_rounds", "dg_boundary_pack", "dg_boundary_unpack", "dg_run_end",
    "dg_normalize_states", "dg_p2p_alloc", "dg_p2p_open", "dg_boundary_exchange", "dg_run_fused",
    "dg_build_paths_shared", "dg_save_layout", "dg_load_layout", "dg_scc_phase", "dg_scc_assign",
]


class dg_path_params(ctypes.Structure):
    _fields_ = [("d_max", ctypes.c_int32), ("l_merge", ctypes.c_int32), ("n_sub", ctypes.c_int32),
                ("order", ctypes.c_int32), ("hot_factor", ctypes.c_float),
                ("part_entries", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("merge_rule", ctypes.c_int32), ("n_proxy", ctypes.c_int32), ("placement", ctypes.c_int32)]


class dg_run_stats(ctypes.Structure):
    _fields_ = [("time_ms", ctypes.c_double), ("rounds", ctypes.c_int64),
                ("vertex_updates", ctypes.c_int64), ("edges_processed", ctypes.c_int64),
                ("units_processed", ctypes.c_int64), ("kernel_launches", ctypes.c_int64),
                ("outer_iterations", ctypes.c_int64), ("entries_processed", ctypes.c_int64),
                ("csr_edges", ctypes.c_int64), ("kernel_ms", ctypes.c_double),
                ("dense_rounds", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class dg_layout_info(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("m", ctypes.c_int64), ("n_paths", ctypes.c_int64),
                ("n_entries", ctypes.c_int64), ("n_partitions", ctypes.c_int64),
                ("n_hot_paths", ctypes.c_int64), ("n_layers", ctypes.c_int64),
                ("n_dep_sccs", ctypes.c_int64), ("giant_scc_paths", ctypes.c_int64),
                ("n_boundary", ctypes.c_int64), ("paths_before_merge", ctypes.c_int64),
                ("preprocess_ms", ctypes.c_double), ("device_bytes", ctypes.c_int64),
                ("h2d_bytes", ctypes.c_int64), ("boundary_reads", ctypes.c_int64),
                ("hub_entries", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


_lib = None


def lib():
    """Load libdigraph.so (building it first if the sources are newer)."""
    global _lib
    if _lib is not None:
        return _lib
    from . import build as _build
    if _build.needs_build():
        _build.build()
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libdigraph.so missing at {LIB_PATH}; run __graft_entry__.build()")
    L = ctypes.CDLL(LIB_PATH)
    P, i64, i32, f64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
    pp = ctypes.POINTER
    sig = {
        "dg_default_params": (None, [pp(dg_path_params)]),
        "dg_create": (i32, [pp(P), i32]),
        "dg_destroy": (None, [P]),
        "dg_last_error": (ctypes.c_char_p, []),
        "dg_load_csr": (i32, [P, i64, i64, P, P, P]),
        "dg_build_paths": (i32, [P, pp(dg_path_params)]),
        "dg_upload": (i32, [P]),
        "dg_set_vertex_params": (i32, [P, P, P, P]),
        "dg_run": (i32, [P, i32, i64, f64, f64, i32, i64, pp(dg_run_stats)]),
        "dg_get_states": (i32, [P, P, i64, i32]),
        "dg_get_layout_info": (i32, [P, pp(dg_layout_info)]),
        "dg_export_paths": (i32, [P, P, P, P, P, P, P, P]),
        "dg_boundary_size": (i32, [P, pp(i64)]),
        "dg_boundary_vertices": (i32, [P, P]),
        "dg_run_begin": (i32, [P, i32, i64, f64, f64]),
        "dg_rounds": (i32, [P, i64, pp(i64)]),
        "dg_boundary_pack": (i32, [P, P]),
        "dg_boundary_unpack": (i32, [P, P, pp(i64)]),
        "dg_run_end": (i32, [P, pp(dg_run_stats)]),
        "dg_normalize_states": (i32, [P, P, i64]),
        "dg_p2p_alloc": (i32, [P, i32, i32, P]),
        "dg_p2p_open": (i32, [P, P]),
        "dg_boundary_exchange": (i32, [P, pp(i64)]),
        "dg_run_fused": (i32, [P, i64, i64, pp(i64), pp(i64)]),
        "dg_build_paths_shared": (i32, [P, pp(dg_path_params), ctypes.c_char_p]),
        "dg_save_layout": (i32, [P, ctypes.c_char_p]),
        "dg_load_layout": (i32, [P, ctypes.c_char_p]),
        "dg_scc_phase": (i32, [P, i32, pp(i64)]),
        "dg_scc_assign": (i32, [P, pp(i64)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


class DGError(RuntimeError):
    def __init__(self, code, where):
        msg = lib().dg_last_error().decode()
        super().__init__(f"{where}: {ERRORS.get(code, code)}: {msg}")
        self.code = code


def check(code, where):
    if code != 0:
        raise DGError(code, where)
    return code
