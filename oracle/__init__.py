"""DiGraph ORACLE -- test infrastructure only.

This package is a plain, slow, obviously-correct CPU implementation of what
the DiGraph hot path computes (Zhang et al., "DiGraph: An Efficient
Path-based Iterative Directed Graph Processing System on Multiple GPUs",
ASPLOS'19; /root/reference/PAPER.md).  It exists so the CUDA path in
``paper_conf_asplos_zhangl0hlg19_b200`` can be checked element by element.

Rules:
  * only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
    ``cpu_baseline`` / ``--impl reference`` legs may import anything here;
  * it shares no code, header, constant or table with the CUDA path, and
    imports nothing from the product package;
  * floating point is fp64 unless the paper fixes the precision.

Modules
  algorithms -- synchronous (Jacobi) vertex programs: Bellman-Ford SSSP,
                BFS, PageRank power iteration, Adsorption, label-propagation
                WCC, Tarjan SCC.  Every function cites the PAPER.md passage
                (or DESIGN.md reading) it follows.
  paths      -- Algorithm 1 path decomposition, short-path merging, hot/cold
                classification, path dependency graph, SCC condensation,
                layering and the soft priority Pri(p) (sec. 3.1-3.2.3).

Pinning (tests/test_oracle_pins.py): every function here is checked against
something other than itself -- Dijkstra / Floyd-Warshall brute force, dense
linear solves, closed forms, the paper's Figure 4 worked example, transitive
closure, invariants.  No function is "parity unpinned".
"""
