"""Seeded synthetic input generators shared by the oracle tests and the
product benchmarks.

This module draws graphs and random per-vertex parameters only; it holds none
of DiGraph's arithmetic and imports neither ``oracle`` nor the product
package.  The heavy lifting is C (``gen.c``, OpenMP, counter-based splitmix64
streams, so results do not depend on the thread count).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libdginputs.so")
_lib = None

# Workload shapes of BASELINE.json "configs".
RMAT_ABC = (0.57, 0.19, 0.19)          # Graph500 R-MAT quadrant probabilities
CONFIGS = {
    # configs[0]: SSSP on R-MAT scale-16 (65K vertices, 1M edges, w 1..255)
    "rmat16": dict(kind="rmat", scale=16, n=1 << 16, m=1 << 20),
    # configs[1]: LiveJournal-shaped R-MAT (4.8M vertices, 69M edges)
    "lj": dict(kind="rmat", scale=23, n=4_847_571, m=68_993_773),
    # configs[2]: Twitter-shaped power-law (41.6M vertices, 1.47B edges)
    "twitter": dict(kind="rmat", scale=26, n=41_652_230, m=1_468_365_182),
    # configs[2] at half scale (same edge factor; 167 MB of PageRank masters,
    # still beyond the 126 MB L2): the tuning proxy of the headline workload
    "twitter_h": dict(kind="rmat", scale=25, n=20_826_115, m=734_182_591),
    # configs[3]: Friendster-shaped (65.6M vertices, 1.8B edges)
    "friendster": dict(kind="rmat", scale=26, n=65_608_366, m=1_806_067_135),
    # configs[4]: long-chain-heavy digraph (100M vertices, 2B edges)
    "chains": dict(kind="chains", n=100_000_000, m=2_000_000_000, chain_len=4096),
    # configs[4] at 1/4 scale for one host (same chain length and cross-edge mix)
    "chains_q": dict(kind="chains", n=25_000_000, m=500_000_000, chain_len=4096),
    # configs[4] at 1/40 scale (CPU-side checks)
    "chains_s": dict(kind="chains", n=2_500_000, m=50_000_000, chain_len=4096),
}


def build(force=False):
    """Compile libdginputs.so (gcc -O3 -fopenmp)."""
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-shared", "-fPIC",
                               src, "-o", _SO, "-lm"])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        i64, u64, i32, f64 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32, ctypes.c_double
        lib.dgi_rmat.argtypes = [ctypes.c_int, i64, i64, f64, f64, f64, u64, ctypes.c_int, P, P]
        lib.dgi_chains.argtypes = [i64, i64, i64, f64, u64, P, P]
        lib.dgi_chains.restype = i64
        lib.dgi_uniform.argtypes = [i64, i64, u64, P, P]
        lib.dgi_build_csr.argtypes = [i64, i64, P, P, ctypes.c_int, ctypes.c_int, i64, u64, P, P]
        lib.dgi_build_csr.restype = i64
        lib.dgi_weights.argtypes = [i64, P, P, i32, i32, u64, P]
        lib.dgi_uniform_f64.argtypes = [i64, u64, u64, f64, f64, P]
        lib.dgi_perm.argtypes = [u64, u64, u64]
        lib.dgi_perm.restype = u64
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


class Graph:
    """CSR digraph: row_ptr int64[n+1], col int32[m], w int32[m] (or None)."""

    def __init__(self, n, row_ptr, col, w=None, name=""):
        self.n = int(n)
        self.row_ptr = row_ptr
        self.col = col
        self.w = w
        self.name = name

    @property
    def m(self):
        return int(self.row_ptr[-1])

    def edges(self):
        """(src, dst, w) as int64 arrays (CSR order)."""
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.row_ptr))
        return src, self.col.astype(np.int64), (None if self.w is None else self.w.astype(np.int64))


def _csr_from_edges(n, src, dst, seed, dedupe=True, drop_self=True, keep_m=0,
                    weights=(1, 255)):
    lib = _load()
    m = len(src)
    row_ptr = np.empty(n + 1, np.int64)
    col = np.empty(max(m, 1), np.int32)
    mm = lib.dgi_build_csr(n, m, _ptr(src), _ptr(dst), int(dedupe), int(drop_self),
                           int(keep_m), seed, _ptr(row_ptr), _ptr(col))
    col = col[:mm].copy() if mm < len(col) else col
    w = None
    if weights is not None:
        w = np.empty(max(mm, 1), np.int32)
        lib.dgi_weights(n, _ptr(row_ptr), _ptr(col), int(weights[0]), int(weights[1]), seed, _ptr(w))
        w = w[:mm]
    return Graph(n, row_ptr, col[:mm], w)


def rmat(scale, n, m, seed=1, abc=RMAT_ABC, permute=True, oversample=1.0,
         weights=(1, 255), dedupe=True):
    """R-MAT digraph on [0, n) with ~m distinct edges (self loops dropped,
    duplicates merged; ``oversample`` > 1 draws extra raw edges and thins
    back to exactly m).  Vertex ids are scrambled except 0, the R-MAT hub."""
    lib = _load()
    raw = int(m * oversample)
    src = np.empty(raw, np.int32)
    dst = np.empty(raw, np.int32)
    lib.dgi_rmat(int(scale), raw, int(n), abc[0], abc[1], abc[2], seed, int(permute), _ptr(src), _ptr(dst))
    g = _csr_from_edges(n, src, dst, seed, dedupe=dedupe, keep_m=m if oversample > 1 else 0,
                        weights=weights)
    g.name = f"rmat-s{scale}-n{n}-m{g.m}-seed{seed}"
    return g


def chains(n, m, chain_len=4096, back_frac=0.01, seed=1, weights=(1, 255)):
    """Long-chain-heavy digraph (deep path dependencies)."""
    lib = _load()
    n_chains = (n + chain_len - 1) // chain_len
    m_extra = max(0, m - (n - n_chains))
    src = np.empty(n - n_chains + m_extra, np.int32)
    dst = np.empty_like(src)
    lib.dgi_chains(n, chain_len, m_extra, back_frac, seed, _ptr(src), _ptr(dst))
    g = _csr_from_edges(n, src, dst, seed, weights=weights)
    g.name = f"chains-n{n}-L{chain_len}-m{g.m}-seed{seed}"
    return g


def uniform(n, m, seed=1, weights=(1, 255), dedupe=False, drop_self=False):
    """G(n, m) with replacement (duplicates/self loops kept unless asked)."""
    lib = _load()
    src = np.empty(m, np.int32)
    dst = np.empty(m, np.int32)
    lib.dgi_uniform(n, m, seed, _ptr(src), _ptr(dst))
    g = _csr_from_edges(n, src, dst, seed, dedupe=dedupe, drop_self=drop_self, weights=weights)
    g.name = f"uniform-n{n}-m{g.m}-seed{seed}"
    return g


def from_edges(n, src, dst, w=None):
    """Small hand-made graphs (tests): CSR in the given per-row edge order."""
    src = np.asarray(src, np.int64)
    dst = np.asarray(dst, np.int64)
    order = np.argsort(src, kind="stable")
    row_ptr = np.zeros(n + 1, np.int64)
    np.add.at(row_ptr, src + 1, 1)
    row_ptr = np.cumsum(row_ptr)
    wv = None if w is None else np.asarray(w, np.int32)[order]
    return Graph(n, row_ptr, dst[order].astype(np.int32), wv, name="custom")


def vertex_uniform(n, seed, stream, lo=0.0, hi=1.0):
    lib = _load()
    out = np.empty(n, np.float64)
    lib.dgi_uniform_f64(n, seed, stream, lo, hi, _ptr(out))
    return out


def adsorption_params(n, seed=1):
    """Per-vertex Adsorption inputs (reading R-ADS): p_cont in
    [0.3, 0.7), p_inj in [0, 1 - p_cont), injected value I in [0, 1)."""
    p_cont = vertex_uniform(n, seed, 101, 0.3, 0.7)
    p_inj = vertex_uniform(n, seed, 102, 0.0, 1.0) * (1.0 - p_cont)
    inj = vertex_uniform(n, seed, 103, 0.0, 1.0)
    return p_inj, p_cont, inj


def make(config, seed=1):
    """Graph for a named BASELINE config (see CONFIGS)."""
    c = CONFIGS[config]
    if c["kind"] == "rmat":
        return rmat(c["scale"], c["n"], c["m"], seed=seed, oversample=1.15)
    return chains(c["n"], c["m"], chain_len=c["chain_len"], seed=seed)
