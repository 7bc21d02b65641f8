"""Generators produce valid undirected CSR in canonical order (no method arithmetic here)."""
import numpy as np
import pytest

import workloads as W


def check_csr(g):
    rp, col = g.row_ptr, g.col
    assert rp.dtype == np.int64 and col.dtype == np.int32
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0) and rp[-1] == col.size
    rows = np.repeat(np.arange(g.n), np.diff(rp))
    assert np.all(col >= 0) and np.all(col < g.n)
    assert np.all(rows != col)  # no self loops
    key = rows.astype(np.int64) * g.n + col
    assert np.all(np.diff(key) > 0)  # rows sorted ascending, no duplicates
    rkey = np.sort(col.astype(np.int64) * g.n + rows)
    assert np.array_equal(rkey, key)  # symmetric


@pytest.mark.parametrize("g", [W.karate(), W.path_graph(7), W.star_graph(6), W.cycle_graph(9),
                               W.complete_graph(5), W.grid_graph(4, 6), W.random_gnm(50, 120, 3),
                               W.rmat(10, 8, 1), W.delaunay(500, 2), W.watts_strogatz(300, 6, 0.2, 4)])
def test_generators_valid(g):
    check_csr(g)


def test_karate_shape():
    g = W.karate()
    assert g.n == 34 and g.m == 78


def test_rmat16_shape():
    g = W.rmat(16, 8, 1)
    check_csr(g)
    assert 440_000 < g.m < 500_000  # ~477k undirected edges
    assert 0.3 < (g.degree() == 0).mean() < 0.45


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12", "delaunay12u"])
def test_workload_streams(name):
    wl = W.make_workload(name)
    check_csr(wl.graph)
    eu, ev = W.edges_of(wl.graph)
    present = set(zip(eu.tolist(), ev.tolist()))
    seen = set()
    for u, v in zip(wl.ins_u.tolist(), wl.ins_v.tolist()):
        a, b = min(u, v), max(u, v)
        assert a != b and (a, b) not in present and (a, b) not in seen
        seen.add((a, b))
    assert len(set(wl.roots.tolist())) == wl.roots.size
    assert np.all(wl.graph.degree()[wl.roots] > 0)


def test_seeded_reproducible():
    a = W.make_workload("rmat10", seed=5)
    b = W.make_workload("rmat10", seed=5)
    assert np.array_equal(a.graph.col, b.graph.col) and np.array_equal(a.roots, b.roots)
    assert np.array_equal(a.ins_u, b.ins_u)
