"""Graph generators (CSR, canonical order = ascending neighbour id per row).

Shapes follow SURVEY.md Sec. 8(d) "Configs as concrete synthetic inputs", which
stand in for the paper's DIMACS-10 graphs (Table I: a
Kronecker graph, a Delaunay triangulation, a small-world graph, ...).
"""

from __future__ import annotations

from dataclasses import dataclass

import numpy as np

# Zachary karate club, 34 vertices, 78 edges (embedded so
# nothing depends on a networkx version).
KARATE_EDGES = [
    (0, 1), (0, 2), (0, 3), (0, 4), (0, 5), (0, 6), (0, 7), (0, 8), (0, 10), (0, 11),
    (0, 12), (0, 13), (0, 17), (0, 19), (0, 21), (0, 31), (1, 2), (1, 3), (1, 7),
    (1, 13), (1, 17), (1, 19), (1, 21), (1, 30), (2, 3), (2, 7), (2, 8), (2, 9),
    (2, 13), (2, 27), (2, 28), (2, 32), (3, 7), (3, 12), (3, 13), (4, 6), (4, 10),
    (5, 6), (5, 10), (5, 16), (6, 16), (8, 30), (8, 32), (8, 33), (9, 33), (13, 33),
    (14, 32), (14, 33), (15, 32), (15, 33), (18, 32), (18, 33), (19, 33), (20, 32),
    (20, 33), (22, 32), (22, 33), (23, 25), (23, 27), (23, 29), (23, 32), (23, 33),
    (24, 25), (24, 27), (24, 31), (25, 31), (26, 29), (26, 33), (27, 33), (28, 31),
    (28, 33), (29, 32), (29, 33), (30, 32), (30, 33), (31, 32), (31, 33), (32, 33),
]


@dataclass
class CSR:
    """Undirected graph in CSR form (both directions stored)."""

    n: int
    row_ptr: np.ndarray  # int64 [n+1]
    col: np.ndarray  # int32 [row_ptr[n]]

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def m(self) -> int:
        return self.nnz // 2

    def degree(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def neighbors(self, v: int) -> np.ndarray:
        return self.col[self.row_ptr[v]:self.row_ptr[v + 1]]


def csr_from_edges(n: int, u, v) -> CSR:
    """Symmetrise, drop self loops and duplicate edges, sort each row ascending."""
    u = np.asarray(u, dtype=np.int64).ravel()
    v = np.asarray(v, dtype=np.int64).ravel()
    keep = u != v
    u, v = u[keep], v[keep]
    a = np.concatenate([u, v])
    b = np.concatenate([v, u])
    key = _sorted_unique(a * n + b)  # sorted by (row, col) and deduplicated
    rows = key // n
    cols = key % n
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    row_ptr[1:] = np.cumsum(np.bincount(rows, minlength=n))
    return CSR(n, row_ptr, cols.astype(np.int32))


def _sorted_unique(key):
    """np.unique(key) for int64 keys (sort + adjacent dedup: np.unique takes
    ~50x longer on the 10^8-key Kronecker inputs)."""
    key = np.sort(key, kind="stable")
    if key.size == 0:
        return key
    keep = np.empty(key.size, dtype=bool)
    keep[0] = True
    np.not_equal(key[1:], key[:-1], out=keep[1:])
    return key[keep]


def edges_of(g: CSR):
    """Undirected edge list (u < v), sorted."""
    rows = np.repeat(np.arange(g.n, dtype=np.int64), g.degree())
    cols = g.col.astype(np.int64)
    m = rows < cols
    return rows[m].astype(np.int32), cols[m].astype(np.int32)


def karate() -> CSR:
    e = np.array(KARATE_EDGES, dtype=np.int64)
    return csr_from_edges(34, e[:, 0], e[:, 1])


def path_graph(n: int) -> CSR:
    i = np.arange(n - 1)
    return csr_from_edges(n, i, i + 1)


def cycle_graph(n: int) -> CSR:
    i = np.arange(n)
    return csr_from_edges(n, i, (i + 1) % n)


def star_graph(n: int) -> CSR:
    """Centre 0 joined to leaves 1..n-1 (n vertices)."""
    i = np.arange(1, n)
    return csr_from_edges(n, np.zeros_like(i), i)


def complete_graph(n: int) -> CSR:
    u, v = np.triu_indices(n, 1)
    return csr_from_edges(n, u, v)


def grid_graph(a: int, b: int) -> CSR:
    """a x b grid, vertex (i, j) -> i*b + j."""
    idx = np.arange(a * b).reshape(a, b)
    u = np.concatenate([idx[:, :-1].ravel(), idx[:-1, :].ravel()])
    v = np.concatenate([idx[:, 1:].ravel(), idx[1:, :].ravel()])
    return csr_from_edges(a * b, u, v)


def random_gnm(n: int, m: int, seed: int) -> CSR:
    """Uniform random simple graph with (up to) m edges; may be disconnected."""
    rng = np.random.default_rng(seed)
    u = rng.integers(0, n, size=m)
    v = rng.integers(0, n, size=m)
    return csr_from_edges(n, u, v)


def rmat(scale: int, edgefactor: int, seed: int, a=0.57, b=0.19, c=0.19) -> CSR:
    """Graph500 Kronecker/R-MAT generator (A,B,C = .57/.19/.19, D = .05).

    2^scale vertices, edgefactor * 2^scale tuples, random vertex permutation,
    symmetrised, self loops and duplicates dropped (SURVEY.md Sec. 8(d) cfg 2, 4, 5).
    """
    rng = np.random.default_rng(seed)
    n = 1 << scale
    m = edgefactor * n
    ab = a + b
    c_norm = c / (1.0 - ab)
    a_norm = a / ab
    ii = np.zeros(m, dtype=np.int64)
    jj = np.zeros(m, dtype=np.int64)
    for ib in range(scale):
        ii_bit = rng.random(m) > ab
        thr = np.where(ii_bit, c_norm, a_norm)
        jj_bit = rng.random(m) > thr
        ii |= ii_bit.astype(np.int64) << ib
        jj |= jj_bit.astype(np.int64) << ib
        del ii_bit, jj_bit, thr
    perm = rng.permutation(n)
    return csr_from_edges(n, perm[ii], perm[jj])


def delaunay(n_points: int, seed: int) -> CSR:
    """Delaunay triangulation of uniform points in [0,1)^2 (cfg 3, cf. delaunay_n20)."""
    from scipy.spatial import Delaunay

    rng = np.random.default_rng(seed)
    pts = rng.random((n_points, 2))
    tri = Delaunay(pts).simplices.astype(np.int64)
    u = np.concatenate([tri[:, 0], tri[:, 1], tri[:, 2]])
    v = np.concatenate([tri[:, 1], tri[:, 2], tri[:, 0]])
    return csr_from_edges(n_points, u, v)


def watts_strogatz(n: int, k: int, p: float, seed: int) -> CSR:
    """Watts-Strogatz small world (ring lattice, each vertex to k/2 right neighbours,
    each such edge's far endpoint rewired with probability p); cf. smallworld."""
    rng = np.random.default_rng(seed)
    src = np.repeat(np.arange(n), k // 2)
    off = np.tile(np.arange(1, k // 2 + 1), n)
    dst = (src + off) % n
    rew = rng.random(src.size) < p
    dst = dst.copy()
    dst[rew] = rng.integers(0, n, size=int(rew.sum()))
    return csr_from_edges(n, src, dst)
