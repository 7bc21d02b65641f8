"""Pins for the CPU oracle (oracle/), independent of the CUDA path.

Each pin fixes the oracle against something other than itself (SURVEY.md
Sec. 8(c) "Pins"): brute-force path enumeration, closed forms, networkx, and
invariants the mathematics fixes.
"""

from __future__ import annotations

import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import workloads as W
from tests.bruteforce import brute_force

INF = oracle.INF
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def run(g, roots=None):
    roots = np.arange(g.n, dtype=np.int32) if roots is None else np.asarray(roots, np.int32)
    return oracle.brandes_csr(g, roots)


# --------------------------------------------------------------------------
# brute force on tiny graphs: d and sigma exact, delta and BC to 1e-12
# --------------------------------------------------------------------------
@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_random_tiny(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(4, 9))
    m = int(rng.integers(n - 1, min(n * (n - 1) // 2, 2 * n) + 1))
    g = W.random_gnm(n, m, seed)  # may be disconnected: exercises INF
    eu, ev = W.edges_of(g)
    roots = rng.choice(n, size=int(rng.integers(1, n + 1)), replace=False).astype(np.int32)
    bc, d, sig, dl = run(g, roots)
    bd, bs, bdl, bbc = brute_force(n, list(zip(eu.tolist(), ev.tolist())), roots.tolist())
    for i in range(roots.size):
        assert d[i].tolist() == bd[i]
        assert sig[i].tolist() == [float(x) for x in bs[i]]
        for v in range(n):
            assert dl[i, v] == pytest.approx(float(bdl[i][v]), rel=1e-12, abs=1e-12)
    for v in range(n):
        assert bc[v] == pytest.approx(float(bbc[v]), rel=1e-12, abs=1e-12)


def test_bruteforce_catches_unreachable_root_conventions():
    # two components: {0,1,2} path and {3,4} edge, vertex 5 isolated
    g = W.csr_from_edges(6, [0, 1, 3], [1, 2, 4])
    bc, d, sig, dl = run(g, [0, 5])
    assert d[0].tolist() == [0, 1, 2, INF, INF, INF]
    assert sig[0].tolist() == [1, 1, 1, 0, 0, 0]
    assert dl[0].tolist() == [0, 1, 0, 0, 0, 0]
    assert d[1].tolist() == [INF] * 5 + [0]
    assert sig[1].tolist() == [0] * 5 + [1]
    assert bc.tolist() == [0, 1, 0, 0, 0, 0]


# --------------------------------------------------------------------------
# closed forms (ordered pairs, R = V)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("n", [2, 3, 5, 8, 13])
def test_path_closed_form(n):
    bc, *_ = run(W.path_graph(n))
    assert bc.tolist() == [2.0 * i * (n - 1 - i) for i in range(n)]


@pytest.mark.parametrize("n", [3, 4, 7, 12])
def test_star_closed_form(n):
    bc, *_ = run(W.star_graph(n))
    assert bc[0] == (n - 1) * (n - 2)
    assert np.all(bc[1:] == 0)


@pytest.mark.parametrize("n", [3, 4, 5, 6, 7, 10, 11])
def test_cycle_closed_form(n):
    bc, *_ = run(W.cycle_graph(n))
    want = (n - 1) * (n - 3) / 4 if n % 2 else (n - 2) ** 2 / 4
    np.testing.assert_allclose(bc, want, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("n", [2, 3, 6, 9])
def test_complete_closed_form(n):
    bc, d, sig, _ = run(W.complete_graph(n))
    assert np.all(bc == 0)
    assert np.all(sig == 1)


@pytest.mark.parametrize("a,b", [(3, 4), (6, 6), (20, 25)])
def test_grid_sigma_binomial(a, b):
    g = W.grid_graph(a, b)
    _, d, sig, _ = run(g, [0])
    for i in range(a):
        for j in range(b):
            assert d[0, i * b + j] == i + j
            assert sig[0, i * b + j] == math.comb(i + j, i)


# --------------------------------------------------------------------------
# library pin: networkx (unnormalised undirected BC x 2 == ordered pairs)
# --------------------------------------------------------------------------
def _nx_bc(g):
    nx = pytest.importorskip("networkx")
    G = nx.Graph()
    G.add_nodes_from(range(g.n))
    eu, ev = W.edges_of(g)
    G.add_edges_from(zip(eu.tolist(), ev.tolist()))
    r = nx.betweenness_centrality(G, normalized=False)
    return np.array([2.0 * r[v] for v in range(g.n)])


def test_karate_networkx_and_survey_values():
    g = W.karate()
    bc, d, sig, _ = run(g)
    np.testing.assert_allclose(bc, _nx_bc(g), rtol=1e-12, atol=1e-12)
    with open(os.path.join(GOLDEN, "karate_bc.json")) as f:
        gold = json.load(f)
    for v, val in gold["bc"].items():
        assert bc[int(v)] == pytest.approx(val, rel=1e-12)
    for v in gold["zero"]:
        assert bc[v] == 0.0
    assert bc.sum() == pytest.approx(gold["sum"], rel=1e-12)
    assert int(d[d != INF].max()) == gold["diameter"]
    assert sig.max() == gold["max_sigma"]


@pytest.mark.parametrize("seed", range(4))
def test_random_graphs_networkx(seed):
    g = W.random_gnm(60, 150, seed)
    bc, *_ = run(g)
    np.testing.assert_allclose(bc, _nx_bc(g), rtol=1e-11, atol=1e-11)


# --------------------------------------------------------------------------
# invariants
# --------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12"])
def test_sum_bc_equals_sum_pair_distances(name):
    """sum_v BC(v) = sum_{s in R} sum_{t reachable, t != s} (d_s(t) - 1): every
    shortest s-t path has d_s(t)-1 interior vertices (Eq. (1) summed over v)."""
    wl = W.make_workload(name)
    bc, d, sig, dl = oracle.brandes_csr(wl.graph, wl.roots)
    fin = d[(d != INF) & (d > 0)]
    assert bc.sum() == pytest.approx(float((fin - 1).sum()), rel=1e-11)
    # structural invariants on every root's state
    g = wl.graph
    rows = np.repeat(np.arange(g.n), g.degree())
    for i in range(min(8, wl.roots.size)):
        dd = d[i].astype(np.int64)
        reach = dd != INF
        e_ok = reach[rows] == reach[g.col]
        assert e_ok.all()  # components are closed
        both = reach[rows] & reach[g.col]
        assert np.all(np.abs(dd[rows][both] - dd[g.col][both]) <= 1)
        assert np.all((sig[i] >= 1) == reach)
        assert np.all(dl[i] >= 0)
        leaf = (g.degree() == 1) & (np.arange(g.n) != wl.roots[i])
        assert np.all(dl[i][leaf] == 0)


# --------------------------------------------------------------------------
# naive dynamic rule
# --------------------------------------------------------------------------
@pytest.mark.parametrize("n", [5, 6, 9, 10])
def test_dynamic_path_to_cycle(n):
    """P_n + (0, n-1) = C_n: exercises Cases 1/2/3 over the roots."""
    dyn = oracle.NaiveDynamicBC(W.path_graph(n), np.arange(n, dtype=np.int32))
    dyn.insert(0, n - 1)
    bc, *_ = dyn.compute()
    want = (n - 1) * (n - 3) / 4 if n % 2 else (n - 2) ** 2 / 4
    np.testing.assert_allclose(bc, want, rtol=1e-13, atol=1e-13)


def test_dynamic_star_to_complete():
    n = 7
    dyn = oracle.NaiveDynamicBC(W.star_graph(n), np.arange(n, dtype=np.int32))
    for a in range(1, n):
        for b in range(a + 1, n):
            dyn.insert(a, b)
    bc, d, sig, _ = dyn.compute()
    np.testing.assert_allclose(bc, 0.0, atol=1e-15)
    assert np.all(sig == 1)


def test_dynamic_canonical_order_appends_in_insertion_order():
    g = W.path_graph(4)  # rows: 0:[1] 1:[0,2] 2:[1,3] 3:[2]
    dyn = oracle.NaiveDynamicBC(g, [0])
    dyn.insert(3, 0)
    dyn.insert(1, 3)
    rp, col = dyn.csr()
    rows = [col[rp[v]:rp[v + 1]].tolist() for v in range(4)]
    assert rows == [[1, 3], [0, 2, 3], [1, 3], [2, 0, 1]]


def test_dynamic_matches_networkx_after_insertions():
    wl = W.make_workload("karate")
    dyn = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        dyn.insert(u, v)
    bc, *_ = dyn.compute()
    eu, ev = W.edges_of(wl.graph)
    final = W.csr_from_edges(34, np.concatenate([eu, wl.ins_u]), np.concatenate([ev, wl.ins_v]))
    np.testing.assert_allclose(bc, _nx_bc(final), rtol=1e-12, atol=1e-12)


def test_case1_insertion_leaves_state_bitwise_unchanged():
    """Case 1: |d_s(u) - d_s(v)| = 0 for every root => no change."""
    g = W.grid_graph(5, 5)
    roots = np.array([0, 24, 12], dtype=np.int32)
    bc0, d0, s0, dl0 = oracle.brandes_csr(g, roots)
    eu, ev = W.edges_of(g)
    adj = set(zip(eu.tolist(), ev.tolist()))
    found = None
    for a in range(25):
        for b in range(a + 1, 25):
            if (a, b) in adj:
                continue
            if all(d0[i, a] == d0[i, b] for i in range(roots.size)):
                found = (a, b)
                break
        if found:
            break
    assert found is not None
    dyn = oracle.NaiveDynamicBC(g, roots)
    dyn.insert(*found)
    bc1, d1, s1, dl1 = dyn.compute()
    assert np.array_equal(d0, d1) and np.array_equal(s0, s1)
    assert np.array_equal(dl0, dl1) and np.array_equal(bc0, bc1)


def test_dynamic_bruteforce_tiny_streams():
    """Naive rule vs brute force after each insertion of a tiny random stream."""
    rng = np.random.default_rng(7)
    for trial in range(6):
        n = 7
        g = W.random_gnm(n, 6, 100 + trial)
        roots = np.arange(n, dtype=np.int32)
        eu, ev = W.edges_of(g)
        edges = list(zip(eu.tolist(), ev.tolist()))
        dyn = oracle.NaiveDynamicBC(g, roots)
        non = [(a, b) for a in range(n) for b in range(a + 1, n) if (a, b) not in set(edges)]
        rng.shuffle(non)
        for a, b in non[:3]:
            dyn.insert(a, b)
            edges.append((a, b))
            bc, d, sig, _ = dyn.compute()
            bd, bs, _, bbc = brute_force(n, edges, roots.tolist())
            assert d.tolist() == bd
            assert sig.tolist() == [[float(x) for x in r] for r in bs]
            np.testing.assert_allclose(bc, [float(x) for x in bbc], rtol=1e-12, atol=1e-12)


def test_paper_table_arithmetic():
    """Consistency of the paper's own numbers (Tables II/III): node totals over
    100 insertions / 100 = Table III averages; mean of recompute/avg ~ 45x."""
    with open(os.path.join(GOLDEN, "paper_tables.json")) as f:
        t = json.load(f)
    ratios = []
    for gname, row in t["table3"].items():
        assert row["average"] * 100 == pytest.approx(t["table2_node_total"][gname], rel=2e-3)
        ratios.append(row["recompute"] / row["average"])
        assert row["recompute"] / row["average"] == pytest.approx(row["avg_speedup"], rel=1e-2)  # times printed to 2-3 digits
    assert np.mean(ratios) == pytest.approx(45.0, abs=0.5)


# --------------------------------------------------------------------------
# scenario classification and touched sets (Fig. 2 / Fig. 4 diagnostics)
# --------------------------------------------------------------------------
def _with_edge(g, u, v):
    dyn = oracle.NaiveDynamicBC(g, np.zeros(1, np.int32))
    dyn.insert(u, v)
    return dyn.csr()


@pytest.mark.parametrize("seed", range(10))
def test_scenarios_match_all_pairs_characterisation(seed):
    """Case from brute-force distances; Case-2 touched set = every v != s on a
    shortest s-t path (new graph) to some t whose path count changed
    (sigma changes exactly below u_low)."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(5, 9))
    m = int(rng.integers(n - 1, min(n * (n - 1) // 2 - 1, 2 * n) + 1))
    g = W.random_gnm(n, m, 100 + seed)
    eu, ev = W.edges_of(g)
    old = list(zip(eu.tolist(), ev.tolist()))
    present = set(old)
    cand = [(a, b) for a in range(n) for b in range(a + 1, n) if (a, b) not in present]
    roots = np.arange(n, dtype=np.int32)
    bd0, bs0, _, _ = brute_force(n, old, list(range(n)))
    seen2 = 0
    for ci in rng.permutation(len(cand))[:8]:
        u, v = cand[int(ci)]
        rp1, col1 = _with_edge(g, u, v)
        case, touched, down = oracle.scenarios(g.row_ptr, g.col, rp1, col1, roots, u, v)
        bd1, bs1, _, _ = brute_force(n, old + [(u, v)], list(range(n)))
        for s in range(n):
            du, dv = bd0[s][u], bd0[s][v]
            want = 1 if du == dv else (2 if abs(du - dv) == 1 else 3)
            assert case[s] == want
            if want != 2:
                continue
            seen2 += 1
            changed = [t for t in range(n) if bs1[s][t] != bs0[s][t]]
            assert down[s] == len(changed)
            on_path = {x for x in range(n) if x != s and any(
                bd1[s][x] + bd1[x][t] == bd1[s][t] for t in changed)}
            assert touched[s] == len(on_path)
    assert seen2 > 0  # the Case-2 branch is exercised


def test_scenarios_path_graph_closed_form():
    """P_n plus (0, n-1): root r sees d(0) = r, d(n-1) = n-1-r, so Case 1 iff
    2r = n-1, Case 2 iff |n-1-2r| = 1, else Case 3."""
    n = 7
    g = W.path_graph(n)
    rp1, col1 = _with_edge(g, 0, n - 1)
    roots = np.arange(n, dtype=np.int32)
    case, touched, _ = oracle.scenarios(g.row_ptr, g.col, rp1, col1, roots, 0, n - 1)
    for r in range(n):
        diff = abs((n - 1 - r) - r)
        assert case[r] == (1 if diff == 0 else 2 if diff == 1 else 3)
    # n = 7: r = 3 is Case 1; no r has |6 - 2r| = 1 (even) -> no Case 2
    assert case.tolist() == [3, 3, 3, 1, 3, 3, 3]
    n = 6  # C_6 after the insertion; r = 2: d(0) = 2, d(5) = 3 -> Case 2, u_low = 5
    g = W.path_graph(n)
    rp1, col1 = _with_edge(g, 0, n - 1)
    case, touched, down = oracle.scenarios(g.row_ptr, g.col, rp1, col1, np.arange(n, dtype=np.int32), 0, n - 1)
    assert case.tolist() == [3, 3, 2, 2, 3, 3]
    # root 2 on C_6: sigma changes only at 5 (paths 2-1-0-5 and 2-3-4-5);
    # on shortest paths to 5: 1, 0, 3, 4, 5 -> touched 5
    assert touched[2] == 5 and touched[3] == 5
    assert down[2] == 1 and down[3] == 1


# --------------------------------------------------------------------------
# the CPU dynamic baseline (Alg. 2 + Case 3, oracle/cpu_dynamic.c) vs the
# naive rule: d / sigma bit-exact, delta and BC within the GPU's tolerance
# --------------------------------------------------------------------------
def _check_cpu_dynamic(g, roots, us, vs, every=1):
    cd = oracle.CpuDynamicBC(g, roots)
    ref = oracle.NaiveDynamicBC(g, roots)
    for i, (u, v) in enumerate(zip(us, vs)):
        cd.insert(u, v)
        ref.insert(u, v)
        if (i + 1) % every and i + 1 != len(us):
            continue
        bc, d, s, dl = cd.state()
        rbc, rd, rs, rdl = ref.compute()
        assert np.array_equal(d, rd)
        assert np.array_equal(s, rs)
        assert np.all(np.abs(dl - rdl) <= 1e-10 * np.maximum(np.abs(rdl), 1.0))
        assert np.all(np.abs(bc - rbc) <= 1e-9 * np.maximum(np.abs(rbc), 1.0))
    return cd.scenarios()


@pytest.mark.parametrize("seed", range(6))
def test_cpu_dynamic_random_multicomponent(seed):
    rng = np.random.default_rng(300 + seed)
    n = int(rng.integers(20, 60))
    g = W.random_gnm(n, int(n * 0.9), 300 + seed)  # several components: Case 3 from INF
    eu, ev = W.edges_of(g)
    present = set(zip(eu.tolist(), ev.tolist()))
    us, vs = [], []
    while len(us) < 25:
        a, b = sorted(int(x) for x in rng.choice(n, 2, replace=False))
        if (a, b) not in present:
            present.add((a, b))
            us.append(a)
            vs.append(b)
    sc = _check_cpu_dynamic(g, np.arange(n, dtype=np.int32), us, vs)
    assert sc[1] > 0 and sc[2] > 0  # Case 2 and Case 3 both exercised


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u"])
def test_cpu_dynamic_configs(name):
    wl = W.make_workload(name)
    B = min(30, wl.ins_u.size)
    _check_cpu_dynamic(wl.graph, wl.roots, wl.ins_u[:B], wl.ins_v[:B], every=5)


def test_cpu_dynamic_path_to_cycle():
    n = 9
    g = W.path_graph(n)
    cd = oracle.CpuDynamicBC(g, np.arange(n, dtype=np.int32))
    cd.insert(0, n - 1)
    bc, *_ = cd.state()
    ref, *_ = oracle.brandes_csr(W.cycle_graph(n), np.arange(n, dtype=np.int32))
    assert np.all(np.abs(bc - ref) <= 1e-12 * np.maximum(ref, 1))


def test_cpu_dynamic_grid_sigma_above_2_53():
    """sigma up to 2^84 on a 45x45 grid: the pull form stays bit-exact."""
    g = W.grid_graph(45, 45)
    rng = np.random.default_rng(7)
    eu, ev = W.edges_of(g)
    present = set(zip(eu.tolist(), ev.tolist()))
    us, vs = [], []
    while len(us) < 6:
        a, b = sorted(int(x) for x in rng.choice(g.n, 2, replace=False))
        if (a, b) not in present:
            present.add((a, b))
            us.append(a)
            vs.append(b)
    _check_cpu_dynamic(g, np.array([0, 44, 1012, 2024], np.int32), us, vs)


# --------------------------------------------------------------------------
# the naive rule for edge deletion
# --------------------------------------------------------------------------
@pytest.mark.parametrize("n", [5, 8, 11])
def test_delete_cycle_edge_gives_path(n):
    """C_n minus (0, n-1) = P_n: BC(i) = 2 i (n-1-i)."""
    g = W.cycle_graph(n)
    dyn = oracle.NaiveDynamicBC(g, np.arange(n, dtype=np.int32))
    dyn.delete(0, n - 1)
    bc, *_ = dyn.compute()
    assert bc.tolist() == [2.0 * i * (n - 1 - i) for i in range(n)]


def test_delete_complete_to_star():
    """K_7 minus every edge between leaves = S_7: BC(0) = 6*5, leaves 0."""
    n = 7
    g = W.complete_graph(n)
    dyn = oracle.NaiveDynamicBC(g, np.arange(n, dtype=np.int32))
    for a in range(1, n):
        for b in range(a + 1, n):
            dyn.delete(a, b)
    bc, *_ = dyn.compute()
    assert bc[0] == (n - 1) * (n - 2) and np.all(bc[1:] == 0)


@pytest.mark.parametrize("seed", range(8))
def test_delete_bruteforce_tiny(seed):
    """Random deletions (and re-insertions) on tiny graphs vs path enumeration."""
    rng = np.random.default_rng(500 + seed)
    n = int(rng.integers(5, 9))
    m = int(rng.integers(n, min(n * (n - 1) // 2, 2 * n) + 1))
    g = W.random_gnm(n, m, 500 + seed)
    eu, ev = W.edges_of(g)
    edges = list(zip(eu.tolist(), ev.tolist()))
    roots = np.arange(n, dtype=np.int32)
    dyn = oracle.NaiveDynamicBC(g, roots)
    for step in range(4):
        a, b = edges.pop(int(rng.integers(len(edges))))
        dyn.delete(a, b)
        if step == 2:  # re-insert one: appended at the row ends
            dyn.insert(a, b)
            edges.append((a, b))
        bc, d, sig, dl = dyn.compute()
        bd, bs, bdl, bbc = brute_force(n, edges, roots.tolist())
        for i in range(n):
            assert d[i].tolist() == bd[i]
            assert sig[i].tolist() == [float(x) for x in bs[i]]
        for v in range(n):
            assert bc[v] == pytest.approx(float(bbc[v]), rel=1e-12, abs=1e-12)


def test_delete_keeps_row_order():
    g = W.csr_from_edges(4, [0, 0, 0], [1, 2, 3])
    dyn = oracle.NaiveDynamicBC(g, np.array([0], np.int32))
    dyn.insert(1, 2)
    dyn.delete(0, 2)
    rp, col = dyn.csr()
    assert col[rp[0]:rp[1]].tolist() == [1, 3]
    assert col[rp[1]:rp[2]].tolist() == [0, 2]
    assert col[rp[2]:rp[3]].tolist() == [1]


# --------------------------------------------------------------------------
# root-parallel leg (SURVEY.md Sec. 8(d) oracle timing (ii)): the same per-root
# computation spread over host threads, Eq. (3) summed in slot order -- must be
# bit-identical to the single-thread path (and so inherits all its pins)
# --------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u", "grid", "multi"])
@pytest.mark.parametrize("threads", [1, 3, 8])
def test_brandes_parallel_bitwise_equals_single_thread(name, threads):
    if name == "grid":
        g = W.grid_graph(30, 30)
        roots = np.array([0, 31, 450, 899, 17], np.int32)
    elif name == "multi":
        g = W.random_gnm(300, 280, 5)  # several components: INF rows
        roots = np.arange(0, 300, 7, dtype=np.int32)
    else:
        wl = W.make_workload(name)
        g, roots = wl.graph, wl.roots
    bc, d, sig, dl = oracle.brandes(g.n, g.row_ptr, g.col, roots)
    slots = np.array(sorted({0, roots.size - 1, roots.size // 2}), np.int64)
    pbc, pd, psig, pdl = oracle.brandes_parallel(g.n, g.row_ptr, g.col, roots, threads=threads,
                                                 state_slots=slots)
    assert np.array_equal(pbc.view(np.int64), bc.view(np.int64))  # bitwise, incl. signed zeros
    assert np.array_equal(pd, d[slots])
    assert np.array_equal(psig.view(np.int64), sig[slots].view(np.int64))
    assert np.array_equal(pdl.view(np.int64), dl[slots].view(np.int64))
    pbc2, pd2, _, _ = oracle.brandes_parallel(g.n, g.row_ptr, g.col, roots, threads=threads)
    assert pd2 is None and np.array_equal(pbc2.view(np.int64), bc.view(np.int64))
