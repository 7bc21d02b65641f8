"""Seeded synthetic workloads shared by the oracle tests, the GPU parity tests and bench.py.

This package holds NO arithmetic of the method (no BFS, no path counting, no
dependency accumulation).  It only builds graphs in CSR form, samples roots and
produces edge-insertion streams, following the paper's experimental protocol
(Sec. IV: "100 edges are chosen at random to be removed from the
graph ... then reinserted into the graph one at a time"; k source nodes "also at
random").  Both `oracle/` and the CUDA path consume these inputs; neither imports
the other.

CSR convention: `row_ptr` int64[n+1], `col` int32[2m],
undirected (every edge stored in both rows), no self loops, no duplicates, each
row sorted ascending by neighbour id.  That row order is the *canonical
adjacency order*; inserted edges are appended after the row in insertion order.
"""

from .graphs import (
    CSR,
    csr_from_edges,
    karate,
    rmat,
    delaunay,
    watts_strogatz,
    path_graph,
    star_graph,
    cycle_graph,
    complete_graph,
    grid_graph,
    random_gnm,
    edges_of,
)
from .streams import (
    sample_roots,
    remove_then_reinsert,
    uniform_non_edges,
    Workload,
    make_workload,
    CONFIGS,
)

__all__ = [
    "CSR", "csr_from_edges", "karate", "rmat", "delaunay", "watts_strogatz",
    "path_graph", "star_graph", "cycle_graph", "complete_graph", "grid_graph",
    "random_gnm", "edges_of", "sample_roots", "remove_then_reinsert",
    "uniform_non_edges", "Workload", "make_workload", "CONFIGS",
]
