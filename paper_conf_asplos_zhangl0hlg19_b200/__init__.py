"""B200-native DiGraph: path-based asynchronous iterative directed-graph
processing (Zhang et al., ASPLOS'19) on sm_100a.

The product is ``libdigraph.so`` (C ABI in include/digraph.h): host C++
preprocessing (Algorithm 1 paths, dependency DAG, partitions) plus CUDA
kernels for the propagation hot path.  This package is the thin Python
binding (``DiGraph``) and the multi-GPU driver (``parallel``).
"""
from ._abi import (DG_ADSORPTION, DG_BFS, DG_INF, DG_MODE_PATH, DG_MODE_VERTEX, DG_PAGERANK,  # noqa: F401
                   DG_SCC, DG_SSSP, DG_WCC, DGError, EXPORTS, LIB_PATH)
from .engine import ALGOS, INF, MODES, STATE_DTYPE, DiGraph, default_params  # noqa: F401
