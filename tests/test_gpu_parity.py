"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle.

Bar (BASELINE.json north_star): d and sigma bit-exact,
BC within |bc - ref| <= 1e-9 * max(|ref|, 1), delta within 1e-12 * max(|ref|, 1)
(delta is a diagnostic; derivation in DESIGN.md).
"""

from __future__ import annotations

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

BC_TOL = 1e-9
DELTA_TOL = 1e-12  # SURVEY.md Sec. 8(c) item 14 (hybrid delta, relative, floor 1)


_TUNE: dict = {}


@pytest.fixture
def tune():
    """dbc_tuning fields (launch configuration) for the contexts _dbc creates in a test."""
    _TUNE.clear()
    yield _TUNE
    _TUNE.clear()


def _dbc(g, roots, **kw):
    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC

    if _TUNE:
        kw.setdefault("tuning", dict(_TUNE))
    return DynamicBC(g.n, g.row_ptr, g.col, roots, **kw)


def assert_bc(bc, ref, tol=BC_TOL):
    err = np.abs(bc - ref) / np.maximum(np.abs(ref), 1.0)
    assert err.max(initial=0.0) <= tol, f"BC rel err {err.max()} at {int(err.argmax())}"


def assert_state(dbc, d_ref, s_ref, dl_ref, slots):
    for slot in slots:
        d, s, dl = dbc.get_root_state(slot)
        assert np.array_equal(d, d_ref[slot]), f"d mismatch at slot {slot}"
        bad = np.nonzero(s != s_ref[slot])[0]
        assert bad.size == 0, f"sigma mismatch slot {slot} at {bad[:5]}: {s[bad[:5]]} vs {s_ref[slot][bad[:5]]}"
        err = np.abs(dl - dl_ref[slot]) / np.maximum(np.abs(dl_ref[slot]), 1.0)
        assert err.max(initial=0.0) <= DELTA_TOL, f"delta rel err {err.max()} slot {slot}"


def check_all(dbc, ref_out, k):
    bc_ref, d_ref, s_ref, dl_ref = ref_out
    assert_bc(dbc.get_bc(), bc_ref)
    assert_state(dbc, d_ref, s_ref, dl_ref, range(k))


# ---------------------------------------------------------------- static ----
def _big_sigma_hub(fan=5000):
    """A hub whose row (> 4,096 entries: a single-row chunk, row sums by shared
    atomics) sums predecessors with sigma ~ 2^56 of two different values, so the
    result above 2^53 depends on the order: it must be the canonical one."""
    eu, ev = [], []
    nxt = [1]

    def new():
        nxt[0] += 1
        return nxt[0] - 1

    def diamonds(src, k):  # k diamonds: sigma doubles per diamond
        cur = src
        for _ in range(k):
            a, b, z = new(), new(), new()
            eu.extend([cur, cur, a, b])
            ev.extend([a, b, z, z])
            cur = z
        return cur

    def path(src, k):
        cur = src
        for _ in range(k):
            x = new()
            eu.append(cur)
            ev.append(x)
            cur = x
        return cur

    s = 0
    t = diamonds(s, 56)                 # level 112, sigma 2^56
    t2 = path(diamonds(s, 5), 102)      # level 112, sigma 2^5
    hub = new()
    for i in range(fan):
        a = new()
        eu.extend([t, a])
        ev.extend([a, hub])
        if i % 2 == 0:
            eu.append(t2)
            ev.append(a)
    g = W.csr_from_edges(nxt[0], eu, ev)
    return g, np.array([0, 1, hub], np.int32)


STATIC_CASES = {
    "big_sigma_hub": _big_sigma_hub,
    "star6k": lambda: (W.star_graph(6000), np.array([0, 1, 5999])),
    "karate": lambda: (W.karate(), np.arange(34)),
    "path9": lambda: (W.path_graph(9), np.arange(9)),
    "star12": lambda: (W.star_graph(12), np.arange(12)),
    "complete8": lambda: (W.complete_graph(8), np.arange(8)),
    "grid_big_sigma": lambda: (W.grid_graph(45, 45), np.array([0, 44, 1012, 2024])),
    "disconnected": lambda: (W.random_gnm(300, 280, 5), np.arange(0, 300, 7)),
    "isolated_root": lambda: (W.csr_from_edges(6, [0, 1], [1, 2]), np.array([5, 0, 3])),
    "rmat10": lambda: (W.make_workload("rmat10").graph, W.make_workload("rmat10").roots),
    "delaunay12": lambda: (W.make_workload("delaunay12").graph, W.make_workload("delaunay12").roots),
    "hub": lambda: (W.star_graph(3000), np.array([0, 1, 2, 2999])),
}


@pytest.mark.parametrize("name", sorted(STATIC_CASES))
def test_static_matches_oracle(name):
    g, roots = STATIC_CASES[name]()
    roots = np.asarray(roots, np.int32)
    ref = oracle.brandes_csr(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        check_all(dbc, ref, roots.size)


@pytest.mark.parametrize("sblock", ["128", "256", "512"])
@pytest.mark.parametrize("name", ["grid_big_sigma", "disconnected", "rmat10", "delaunay12", "hub", "big_sigma_hub"])
def test_static_other_widths_match_oracle(name, sblock, tune):
    """The static kernel at the non-default CTA widths (tuning.static_block; default 1024)."""
    tune["static_block"] = int(sblock)
    g, roots = STATIC_CASES[name]()
    roots = np.asarray(roots, np.int32)
    ref = oracle.brandes_csr(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        check_all(dbc, ref, roots.size)


MS_CASES = dict(STATIC_CASES)
MS_CASES.update({
    "smallworld_small": lambda: (W.make_workload("smallworld_small").graph,
                                 W.make_workload("smallworld_small").roots),
    "rmat10_all": lambda: (W.make_workload("rmat10").graph,
                           np.arange(0, W.make_workload("rmat10").graph.n, 9, dtype=np.int32)),
    "grid60_sigma": lambda: (W.grid_graph(60, 60), np.array([0, 61, 1830, 3599, 29], np.int32)),
})


@pytest.mark.parametrize("width", ["32", "64"])
@pytest.mark.parametrize("chunk", [None, "4"])
@pytest.mark.parametrize("name", sorted(MS_CASES))
def test_static_multisource_matches_oracle(name, chunk, width, tune):
    """The multi-source static kernel (msbrandes.cu, 32 roots per warp) forced on
    every graph: d and sigma bit-exact, delta 1e-12 (Eq. (2) regrouped as
    sigma(w) * sum q(y)), BC 1e-9.  chunk 4 splits every row longer than 4
    entries over several warp tasks (sigma partials added atomically, re-summed
    in canonical order at or above 2^53: grid60 and big_sigma_hub reach 2^56
    and more); one 32-root group per wave, so the roots of karate / rmat10_all
    / disconnected run in several waves.  width 64: two roots per lane (64-bit
    masks)."""
    tune["static_ms"] = 1
    tune["static_groups"] = 1
    tune["static_width"] = int(width)
    if chunk:
        tune["static_chunk"] = int(chunk)
    g, roots = MS_CASES[name]()
    roots = np.asarray(roots, np.int32)
    ref = oracle.brandes_csr(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        check_all(dbc, ref, roots.size)


@pytest.mark.parametrize("chunk", [None, "4"])
@pytest.mark.parametrize("name", ["rmat10_all", "grid60_sigma", "big_sigma_hub", "disconnected"])
def test_static_multisource_pull_delta_is_bitwise(name, chunk, tune):
    """DBC_FLAG_PULL_DELTA with the multi-source kernel requested: it regroups
    Eq. (2), so the static pass falls back to the per-root kernel, whose delta
    is bit-identical to the oracle."""
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_PULL_DELTA

    tune["static_ms"] = 1
    if chunk:
        tune["static_chunk"] = int(chunk)
    g, roots = MS_CASES[name]()
    roots = np.asarray(roots, np.int32)
    bc_ref, d_ref, s_ref, dl_ref = oracle.brandes_csr(g, roots)
    with _dbc(g, roots, flags=FLAG_PULL_DELTA) as dbc:
        dbc.static_compute()
        assert_bc(dbc.get_bc(), bc_ref)
        for slot in range(roots.size):
            d, s, dl = dbc.get_root_state(slot)
            assert np.array_equal(d, d_ref[slot]) and np.array_equal(s, s_ref[slot])
            assert np.array_equal(dl.view(np.int64), dl_ref[slot].view(np.int64)), f"delta slot {slot}"


def test_static_multisource_deep_graph_falls_back(tune):
    """A BFS deeper than 254 levels (byte levels) makes the multi-source kernel
    give up; the per-root kernel recomputes and the result is still exact."""
    tune["static_ms"] = 1
    g = W.path_graph(600)
    roots = np.array([0, 299, 599], np.int32)
    ref = oracle.brandes_csr(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        check_all(dbc, ref, roots.size)


@pytest.mark.parametrize("name", ["rmat10", "smallworld_small"])
def test_static_multisource_then_dynamic(name, tune):
    """The multi-source state (and its level-2 masks) feeds the update kernels:
    a stream of insertions after it matches the naive dynamic oracle."""
    tune["static_ms"] = 1
    wl = W.make_workload(name)
    g, roots = wl.graph, wl.roots
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        us, vs = wl.ins_u[:40], wl.ins_v[:40]
        for b in range(0, 40, 10):
            dbc.insert_edges(us[b:b + 10], vs[b:b + 10])
            for u, v in zip(us[b:b + 10], vs[b:b + 10]):
                ref.insert(int(u), int(v))
        check_all(dbc, ref.compute(), roots.size)


def test_static_no_edges_and_zero_roots():
    g = W.csr_from_edges(5, [], [])
    with _dbc(g, np.array([0, 3], np.int32)) as dbc:
        dbc.static_compute()
        assert np.all(dbc.get_bc() == 0)
        d, s, dl = dbc.get_root_state(1)
        assert d[3] == 0 and s[3] == 1 and np.all(d[[0, 1, 2, 4]] == oracle.INF)
    with _dbc(W.path_graph(4), np.array([], np.int32)) as dbc:
        dbc.static_compute()
        assert np.all(dbc.get_bc() == 0)


# --------------------------------------------------------------- dynamic ----
def run_stream_single(g, roots, us, vs, check_every=1, flags=0, workers=0):
    """Insert one edge per call; compare with the naive dynamic oracle."""
    roots = np.asarray(roots, np.int32)
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots, flags=flags, workers=workers) as dbc:
        dbc.static_compute()
        for i, (u, v) in enumerate(zip(us, vs)):
            dbc.insert_edges([u], [v])
            ref.insert(u, v)
            if (i + 1) % check_every == 0 or i + 1 == len(us):
                check_all(dbc, ref.compute(), roots.size)


@pytest.mark.parametrize("n", [5, 6, 9, 10])
def test_path_to_cycle(n):
    run_stream_single(W.path_graph(n), np.arange(n), [0], [n - 1])


def test_star_to_complete():
    n = 7
    pairs = [(a, b) for a in range(1, n) for b in range(a + 1, n)]
    run_stream_single(W.star_graph(n), np.arange(n), [p[0] for p in pairs], [p[1] for p in pairs])


def test_karate_config1_every_insertion():
    wl = W.make_workload("karate")
    run_stream_single(wl.graph, wl.roots, wl.ins_u, wl.ins_v)


@pytest.mark.parametrize("seed", range(6))
def test_random_multicomponent(seed):
    """Components merge: Case 3 with an unreachable endpoint pulls whole components up."""
    rng = np.random.default_rng(seed)
    n = 80
    g = W.random_gnm(n, 70, 40 + seed)
    u, v = W.uniform_non_edges(g, 30, seed)
    roots = rng.choice(n, size=20, replace=False)
    run_stream_single(g, roots, u, v)


@pytest.mark.parametrize("name", ["rmat10", "delaunay12", "delaunay12u"])
def test_config_shapes_single(name):
    wl = W.make_workload(name)
    run_stream_single(wl.graph, wl.roots, wl.ins_u, wl.ins_v, check_every=5)


def test_grid_sigma_above_2p53_dynamic():
    """sigma > 2^53 (Delaunay-like meshes reach 2^100): pull sums in canonical order stay bit-exact."""
    g = W.grid_graph(60, 60)
    roots = np.array([0, 59, 3599, 1830], np.int32)
    rng = np.random.default_rng(3)
    eu, ev = W.edges_of(g)
    # diagonal shortcuts inside the mesh (Case 2/3 mixes)
    cand = [(i * 60 + j, (i + 1) * 60 + j + 1) for i in range(0, 59, 7) for j in range(0, 59, 11)]
    pick = [cand[i] for i in rng.permutation(len(cand))[:12]]
    run_stream_single(g, roots, [p[0] for p in pick], [p[1] for p in pick], check_every=3)


@pytest.mark.parametrize("lean", [True, False])  # per-insertion jobs on update_lean.cu / update.cu
@pytest.mark.parametrize("flags", [0, 1, 0x10])  # Mode A merged, Mode S, Mode A one job per insertion
@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u"])
def test_batch_modes_match_oracle(name, flags, lean, tune):
    if flags == 0 and not lean:
        pytest.skip("merged batches do not use the per-insertion kernel")
    if not lean:
        tune["disable"] = 0x4  # DBC_TUNE_NO_LEAN
    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
        dbc.static_compute()
        half = wl.ins_u.size // 2
        for sl in (slice(0, half), slice(half, None)):
            st = dbc.insert_edges(wl.ins_u[sl], wl.ins_v[sl], stats=True)
            for u, v in zip(wl.ins_u[sl], wl.ins_v[sl]):
                ref.insert(u, v)
            assert st["case1"] + st["case2"] + st["case3"] == wl.roots.size * wl.ins_u[sl].size
            check_all(dbc, ref.compute(), wl.roots.size)


def test_mode_a_equals_mode_s_and_static_bitwise():
    wl = W.make_workload("delaunay12")
    outs = []
    for flags in (0, 1):
        with _dbc(wl.graph, wl.roots, flags=flags, workers=7) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            outs.append([dbc.get_root_state(s)[:2] for s in range(wl.roots.size)])
            dbc.static_compute()  # GPU recompute on the final graph
            outs.append([dbc.get_root_state(s)[:2] for s in range(wl.roots.size)])
    for o in outs[1:]:
        for (d0, s0), (d1, s1) in zip(outs[0], o):
            assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


def test_exact_bc_flag():
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_EXACT_BC

    wl = W.make_workload("rmat10")
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots, flags=FLAG_EXACT_BC) as dbc:
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u, wl.ins_v)
        for u, v in zip(wl.ins_u, wl.ins_v):
            ref.insert(u, v)
        bc_ref = ref.compute()[0]
        assert_bc(dbc.get_bc(), bc_ref, tol=1e-12)


def test_device_batch_api():
    import torch

    wl = W.make_workload("rmat10")
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        u = torch.from_numpy(wl.ins_u).cuda()
        v = torch.from_numpy(wl.ins_v).cuda()
        dbc.insert_edges(u, v)
        for a, b in zip(wl.ins_u, wl.ins_v):
            ref.insert(a, b)
        check_all(dbc, ref.compute(), wl.roots.size)


def test_fake_multi_gpu_shards_sum_to_single():
    """Two rank contexts (world=2) on one device: partials sum to the 1-rank BC."""
    wl = W.make_workload("rmat10")
    outs = []
    for world in (1, 2):
        parts = []
        for rank in range(world):
            with _dbc(wl.graph, wl.roots, rank=rank, world=world) as dbc:
                dbc.static_compute()
                dbc.insert_edges(wl.ins_u, wl.ins_v)
                parts.append(dbc.get_bc() if world == 1 else dbc.get_bc_partial())
                assert dbc.num_local_roots() == len(range(rank, wl.roots.size, world))
        outs.append(np.sum(parts, axis=0))
    assert_bc(outs[1], outs[0], tol=1e-12)


# ----------------------------------------------------------- error paths ----
def test_error_paths_leave_state_unchanged():
    from paper_conf_ipps_mclaughlinb14_b200 import DBCError

    g = W.karate()
    roots = np.arange(34, dtype=np.int32)
    with _dbc(g, roots, edge_capacity=4) as dbc:
        with pytest.raises(DBCError) as e:
            dbc.insert_edges([0], [9])
        assert e.value.name == "DBC_ESTATE"
        dbc.static_compute()
        bc0 = dbc.get_bc().copy()
        st0 = dbc.get_root_state(5)
        bad = {
            "self loop": ([3], [3]),
            "range": ([0], [34]),
            "negative": ([-1], [2]),
            "present": ([0], [1]),
            "present reversed": ([1], [0]),
            "dup in batch": ([0, 9], [9, 0]),
            "bad later in batch": ([0, 4], [9, 4]),
        }
        for name, (u, v) in bad.items():
            with pytest.raises(DBCError) as e:
                dbc.insert_edges(u, v)
            assert e.value.name == "DBC_EEDGE", name
        with pytest.raises(DBCError) as e:
            dbc.insert_edges([0, 0, 0, 0, 0], [9, 14, 15, 16, 18])
        assert e.value.name == "DBC_ECAPACITY"
        assert np.array_equal(dbc.get_bc(), bc0)
        for a, b in zip(dbc.get_root_state(5), st0):
            assert np.array_equal(a, b)
        with pytest.raises(DBCError) as e:
            dbc.get_root_state(34)
        assert e.value.name == "DBC_EINVAL"
        dbc.insert_edges([], [])  # empty batch is fine
        dbc.insert_edges([0, 9], [9, 14])
        dbc.insert_edges([0, 9], [15, 16])
        with pytest.raises(DBCError) as e:
            dbc.insert_edges([0], [18])
        assert e.value.name == "DBC_ECAPACITY"


def test_host_and_device_validation_agree():
    """Host-array batches are validated on the host against the context's host
    copy of the adjacency (no device round trip), device-array batches on the
    device: the same batches get the same verdicts, and the host copy follows
    insertions through either path and deletions (an inserted edge deleted and
    re-inserted, an original edge deleted and re-inserted); the final state
    matches the oracle after the same operations."""
    import torch

    from paper_conf_ipps_mclaughlinb14_b200 import DBCError

    g = W.karate()
    roots = np.arange(34, dtype=np.int32)
    ref = oracle.NaiveDynamicBC(g, roots)

    def dev(a):
        return torch.tensor(a, dtype=torch.int32, device="cuda")

    with _dbc(g, roots, edge_capacity=16) as dbc:
        dbc.static_compute()

        def verdict(u, v, device):
            try:
                if device:
                    dbc.insert_edges(dev(u), dev(v))
                else:
                    dbc.insert_edges(np.array(u, np.int32), np.array(v, np.int32))
                return "ok"
            except DBCError as e:
                return e.name

        bad = [([3], [3]), ([0], [34]), ([-1], [2]), ([0], [1]), ([1], [0]), ([0, 9], [9, 0]),
               ([0, 4], [9, 4]), ([0, 2], [9, 40])]
        for u, v in bad:
            assert verdict(u, v, False) == verdict(u, v, True) == "DBC_EEDGE", (u, v)
        assert verdict([0], [9], True) == "ok"  # through the device path ...
        ref.insert(0, 9)
        assert verdict([9], [0], False) == "DBC_EEDGE"  # ... is present for the host path
        assert verdict([14], [0], False) == "ok"
        ref.insert(14, 0)
        assert verdict([0], [14], True) == "DBC_EEDGE"
        dbc.delete_edges([0], [1])  # an original edge
        ref.delete(0, 1)
        assert verdict([1], [0], False) == "ok"
        ref.insert(1, 0)
        dbc.delete_edges([9], [0])  # an inserted edge
        ref.delete(9, 0)
        assert verdict([0], [9], False) == "ok"
        ref.insert(0, 9)
        assert verdict([9], [0], False) == "DBC_EEDGE"
        check_all(dbc, ref.compute(), roots.size)


def test_async_host_inserts_with_timing():
    """Host-array insertions do not synchronise: back-to-back calls right after
    dbc_static_compute with DBC_FLAG_TIMING (whose events the next call folds)
    must work and give the oracle's state; the timings are filled in."""
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING

    wl = W.make_workload("karate")
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots, flags=FLAG_TIMING) as dbc:
        dbc.static_compute()  # no synchronize: the next call folds the static events
        for u, v in zip(wl.ins_u.tolist(), wl.ins_v.tolist()):
            dbc.insert_edges([u], [v])
            ref.insert(u, v)
        t = dbc.timings()
        assert t["static_ms"] > 0 and t["update_ms"] > 0 and t["insertions_total"] == wl.ins_u.size
        check_all(dbc, ref.compute(), wl.roots.size)


def test_scenario_log_oversized_batch_leaves_state_unchanged():
    """A batch larger than the scenario log is rejected before anything changes
    (the live graph, d/sigma/delta, BC): a later insertion of the same edges
    succeeds and matches the oracle."""
    from paper_conf_ipps_mclaughlinb14_b200 import DBCError

    wl = W.make_workload("karate")
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        bc0 = dbc.get_bc().copy()
        st0 = [dbc.get_root_state(s) for s in (0, 5, 33)]
        dbc.scenario_log(3)
        with pytest.raises(DBCError) as e:
            dbc.insert_edges(wl.ins_u[:5], wl.ins_v[:5])
        assert e.value.name == "DBC_EINVAL"
        assert np.array_equal(dbc.get_bc(), bc0)
        for s, want in zip((0, 5, 33), st0):
            for a, b in zip(dbc.get_root_state(s), want):
                assert np.array_equal(a, b)
        dbc.scenario_log(0)
        dbc.insert_edges(wl.ins_u[:5], wl.ins_v[:5])  # not "already present": nothing was applied
        ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
        for u, v in zip(wl.ins_u[:5], wl.ins_v[:5]):
            ref.insert(u, v)
        check_all(dbc, ref.compute(), wl.roots.size)


def test_device_deletions_ordered_on_the_context_stream():
    """dbc_delete_edges_device reads a batch the caller wrote on the context
    stream after work already queued there (the batch is read on that stream)."""
    import torch

    wl = W.make_workload("rmat10")
    g = wl.graph
    eu, ev = W.edges_of(g)
    pick = np.random.default_rng(4).choice(eu.size, 6, replace=False)
    du, dv = eu[pick].astype(np.int32), ev[pick].astype(np.int32)
    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        with _dbc(g, wl.roots, stream=stream.cuda_stream) as dbc:
            dbc.static_compute()
            tu = torch.full((6,), -1, dtype=torch.int32, device="cuda")
            tv = torch.full((6,), -1, dtype=torch.int32, device="cuda")
            torch.cuda._sleep(50_000_000)  # keep the stream busy: the copies below land late
            tu.copy_(torch.from_numpy(du).cuda(non_blocking=True))
            tv.copy_(torch.from_numpy(dv).cuda(non_blocking=True))
            dbc.delete_edges(tu, tv)
            ref = oracle.NaiveDynamicBC(g, wl.roots)
            for a, b in zip(du, dv):
                ref.delete(int(a), int(b))
            check_all(dbc, ref.compute(), wl.roots.size)


# ------------------------------------------------- full size (configs[1]) ----
def test_rmat16_full_size_batch_parity():
    """BASELINE configs[1] at full size, in the launch configuration bench.py times
    (Mode A, one batch): BC over all 256 roots vs the oracle recompute, d/sigma/delta
    on sampled roots, and GPU dynamic == GPU static (bitwise d/sigma) on the final graph."""
    wl = W.make_workload("rmat16")
    g = wl.graph
    with _dbc(g, wl.roots) as dbc:
        dbc.static_compute()
        c0 = dbc.debug_counters()
        st = dbc.insert_edges(wl.ins_u, wl.ins_v, stats=True)
        assert st["case1"] + st["case2"] + st["case3"] == 256 * 1000
        c1 = dbc.debug_counters()
        # the cooperative help path (idle CTAs take blocks of a heavy C2 push) ran
        assert c1["help_blocks_by_helpers"] > c0["help_blocks_by_helpers"]
        bc = dbc.get_bc()
        ref = oracle.NaiveDynamicBC(g, wl.roots)
        for u, v in zip(wl.ins_u, wl.ins_v):
            ref.insert(u, v)
        rp, col = ref.csr()
        sample = np.array([0, 17, 101, 255], np.int32)
        bc_ref, d_ref, s_ref, dl_ref = oracle.brandes(g.n, rp, col, wl.roots[sample])
        for i, slot in enumerate(sample):
            d, s, dl = dbc.get_root_state(int(slot))
            assert np.array_equal(d, d_ref[i]) and np.array_equal(s, s_ref[i])
            err = np.abs(dl - dl_ref[i]) / np.maximum(np.abs(dl_ref[i]), 1.0)
            assert err.max() <= DELTA_TOL
        full_bc_ref = oracle.brandes(g.n, rp, col, wl.roots, want_state=False)[0]
        assert_bc(bc, full_bc_ref)
        dyn = [dbc.get_root_state(s)[:2] for s in range(0, 256, 15)]
        dbc.static_compute()
        for (d0, s0), s in zip(dyn, range(0, 256, 15)):
            d1, s1, _ = dbc.get_root_state(s)
            assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u"])
def test_no_reorder_flag_matches_oracle(name):
    """Internal BFS relabelling (default) and the caller's numbering give the same results."""
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_NO_REORDER

    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    want = ref.compute()
    outs = []
    for flags in (FLAG_NO_REORDER, 0):
        with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            check_all(dbc, want, wl.roots.size)
            outs.append([dbc.get_root_state(s) for s in range(wl.roots.size)])
    for (d0, s0, _), (d1, s1, _) in zip(*outs):
        assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u"])
def test_block128_kernels_match_oracle(name, tune):
    """The 128-thread kernel build (chosen when there are more roots than 2 x SMs)."""
    tune["update_block"] = 128
    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        check_all(dbc, ref.compute(), wl.roots.size)
        dbc.insert_edges(wl.ins_u, wl.ins_v)
        for u, v in zip(wl.ins_u, wl.ins_v):
            ref.insert(u, v)
        check_all(dbc, ref.compute(), wl.roots.size)


@pytest.mark.parametrize("block", ["256", "512"])
def test_heavy_lane_batches_match_oracle(tune, block):
    """Several Mode-A batches so the adaptive heavy lane (2x-wide CTAs for the
    slowest roots of the previous batch: 512 threads beside the 256-thread
    build, 1024 beside the 512-thread one) is exercised; d/sigma bit-exact."""
    tune["update_block"] = int(block)
    tune["heavy_factor"] = 1.0  # any root slower than the median
    tune["window"] = 8  # several jobs per root and batch
    wl = W.make_workload("rmat10", insertions=120)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        heavy = 0
        for b in range(4):
            sl = slice(30 * b, 30 * (b + 1))
            dbc.insert_edges(wl.ins_u[sl], wl.ins_v[sl])
            for u, v in zip(wl.ins_u[sl], wl.ins_v[sl]):
                ref.insert(u, v)
            heavy = max(heavy, dbc.timings()["heavy_roots"])
        check_all(dbc, ref.compute(), wl.roots.size)
        assert heavy > 0  # the heavy lane was used


def _sampled_full_size(name, insertions, sample):
    """Full-size config in the bench launch configuration (Mode A, one batch):
    sampled roots' d/sigma bit-exact and delta within tolerance vs the oracle on
    the final graph; incremental BC vs the GPU's own column sum of delta
    (Eq. (3), DBC_FLAG_EXACT_BC rebase) within 1e-9; GPU dynamic == GPU static."""
    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, FLAG_EXACT_BC

    wl = W.make_workload(name, insertions=insertions)
    g = wl.graph
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots) as dbc:
        dbc.static_compute()
        half = insertions // 2
        dbc.insert_edges(wl.ins_u[:half], wl.ins_v[:half])  # two batches: heavy lanes engage
        dbc.insert_edges(wl.ins_u[half:], wl.ins_v[half:])
        bc_inc = dbc.get_bc()
        ref = oracle.NaiveDynamicBC(g, wl.roots)
        for u, v in zip(wl.ins_u, wl.ins_v):
            ref.insert(u, v)
        rp, col = ref.csr()
        slots = np.linspace(0, wl.roots.size - 1, sample).astype(np.int32)
        _, d_ref, s_ref, dl_ref = oracle.brandes(g.n, rp, col, wl.roots[slots])
        dyn = {}
        for i, slot in enumerate(slots):
            d, s, dl = dbc.get_root_state(int(slot))
            assert np.array_equal(d, d_ref[i]), f"d slot {slot}"
            assert np.array_equal(s, s_ref[i]), f"sigma slot {slot}"
            err = np.abs(dl - dl_ref[i]) / np.maximum(np.abs(dl_ref[i]), 1.0)
            assert err.max() <= DELTA_TOL
            dyn[int(slot)] = (d, s)
        dbc.static_compute()  # GPU recompute on the final graph
        for slot, (d0, s0) in dyn.items():
            d1, s1, _ = dbc.get_root_state(slot)
            assert np.array_equal(d0, d1) and np.array_equal(s0, s1)
    # Eq. (3) column sum on a fresh context that replays the same batches
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_EXACT_BC) as dbc:
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u[:half], wl.ins_v[:half])
        dbc.insert_edges(wl.ins_u[half:], wl.ins_v[half:])
        bc_exact = dbc.get_bc()
    assert_bc(bc_inc, bc_exact)


def test_delaunay18_full_size_sampled():
    _sampled_full_size("delaunay18", 1000, 4)


def test_kron20_full_size_sampled():
    _sampled_full_size("kron20", 600, 3)


def test_help_off_matches_help_on(tune):
    """DBC_TUNE_NO_HELP (every C2 push done by its owner CTA) and the default
    cooperative path give bitwise-equal d/sigma and BC within tolerance."""
    wl = W.make_workload("rmat16", insertions=400)
    g = wl.graph
    outs = []
    for off in (1, 0):
        tune["disable"] = off  # DBC_TUNE_NO_HELP
        with _dbc(g, wl.roots) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            outs.append((dbc.get_bc(), [dbc.get_root_state(s)[:2] for s in range(0, 256, 9)]))
    assert_bc(outs[1][0], outs[0][0])
    for (d0, s0), (d1, s1) in zip(outs[0][1], outs[1][1]):
        assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u", "smallworld"])
def test_case2_groups_match_oracle_and_no_merge(name):
    """Runs of Case-2 insertions repaired as one multi-seed job (default) give the
    oracle's d/sigma bit-exact and BC within tolerance, and the same d/sigma as
    DBC_FLAG_NO_MERGE (one job per insertion); group jobs actually formed."""
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_NO_MERGE

    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    want = ref.compute()
    outs = []
    for flags in (FLAG_NO_MERGE, 0):
        with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
            dbc.static_compute()
            c0 = dbc.debug_counters()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            c1 = dbc.debug_counters()
            check_all(dbc, want, wl.roots.size)
            outs.append([dbc.get_root_state(s)[:2] for s in range(wl.roots.size)])
            groups = c1["case2_groups"] - c0["case2_groups"]
            assert (groups == 0) if flags else (groups > 0 or name == "karate")
    for (d0, s0), (d1, s1) in zip(*outs):
        assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


@pytest.mark.parametrize("window", ["2", "7", "64"])
@pytest.mark.parametrize("name", ["rmat10", "delaunay12u"])
def test_window_sizes_match_oracle(name, window, tune):
    """Jobs of `window` insertions (seed injection across several windows per
    batch, Case 3 inside windows): oracle d/sigma bit-exact, BC within tolerance."""
    tune["window"] = int(window)
    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u, wl.ins_v)
        check_all(dbc, ref.compute(), wl.roots.size)


# ------------------------------------------------ scenario log (Fig. 2/4) ----
@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12", "delaunay12u"])
def test_scenario_log_matches_oracle(name):
    """dbc_get_scenarios: case of every (root, insertion) bit-exact against the
    oracle's classification of P:148-159; for every Case-2 scenario the down
    set |D| (sigma changed) and the touched count -- Alg. 2's
    {i | t[i] != untouched}: D plus every ancestor, the root excluded
    -- exactly equal to the oracle's (R19)."""
    wl = W.make_workload(name)
    g, roots = wl.graph, wl.roots
    B = min(40, wl.ins_u.size)
    u, v = wl.ins_u[:B], wl.ins_v[:B]
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        dbc.scenario_log(B)
        dbc.insert_edges(u, v)
        case, touched, down = dbc.scenarios()
        assert case.shape == (B, roots.size)
        n2 = 0
        for i in range(B):
            rp0, col0 = ref.csr()
            ref.insert(u[i], v[i])
            rp1, col1 = ref.csr()
            oc, ot, od = oracle.scenarios(rp0, col0, rp1, col1, roots, int(u[i]), int(v[i]))
            assert np.array_equal(case[i], oc), f"case mismatch at insertion {i}"
            c2 = oc == 2
            n2 += int(c2.sum())
            assert np.array_equal(down[i][c2], od[c2]), f"|D| mismatch at insertion {i}"
            assert np.array_equal(touched[i][c2], ot[c2]), f"touched mismatch at insertion {i}"
            assert np.all(touched[i][oc == 1] == 0) and np.all(down[i][oc == 1] == 0)
        assert n2 > 0
        # the batch itself still matches the naive rule
        check_all(dbc, ref.compute(), roots.size)


# ------------------------------------------- edge-parallel variant (Table II) ----
EDGE = 0x20  # DBC_FLAG_EDGE_PARALLEL


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12", "delaunay12u", "smallworld_small"])
def test_edge_parallel_matches_oracle(name):
    """Alg. 4 / Alg. 6 edge-based kernel: same d/sigma (bit-exact) and BC as the
    oracle, batch by batch."""
    if name == "smallworld_small":
        g = W.watts_strogatz(2000, 6, 0.1, seed=4)
        roots = np.arange(0, 2000, 37, dtype=np.int32)
        eu, ev = W.edges_of(g)
        rng = np.random.default_rng(9)
        pick = rng.choice(eu.size, 40, replace=False)
        # reinsert: drop the picked edges from the graph first
        keep = np.ones(eu.size, bool)
        keep[pick] = False
        g = W.csr_from_edges(g.n, eu[keep], ev[keep])
        us, vs = eu[pick], ev[pick]
    else:
        wl = W.make_workload(name)
        g, roots, us, vs = wl.graph, wl.roots, wl.ins_u, wl.ins_v
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots, flags=EDGE) as dbc:
        dbc.static_compute()
        half = us.size // 2
        for sl in (slice(0, half), slice(half, None)):
            st = dbc.insert_edges(us[sl], vs[sl], stats=True)
            for u, v in zip(us[sl], vs[sl]):
                ref.insert(u, v)
            assert st["case1"] + st["case2"] + st["case3"] == roots.size * us[sl].size
            check_all(dbc, ref.compute(), roots.size)


def test_edge_parallel_multicomponent_and_big_sigma():
    """Case 3 from an unreachable endpoint, and sigma > 2^53 (the canonical re-sum)."""
    g = W.random_gnm(300, 280, 5)
    eu, ev = W.edges_of(g)
    present = set(zip(eu.tolist(), ev.tolist()))
    rng = np.random.default_rng(11)
    pairs = []
    while len(pairs) < 12:
        a, b = sorted(int(x) for x in rng.choice(300, 2, replace=False))
        if (a, b) not in present:
            present.add((a, b))
            pairs.append((a, b))
    run_stream_single(g, np.arange(0, 300, 7), [p[0] for p in pairs], [p[1] for p in pairs],
                      check_every=3, flags=EDGE)
    g = W.grid_graph(60, 60)
    cand = [(i * 60 + j, (i + 1) * 60 + j + 1) for i in range(0, 59, 7) for j in range(0, 59, 11)]
    run_stream_single(g, np.array([0, 59, 3599, 1830], np.int32), [p[0] for p in cand[:8]],
                      [p[1] for p in cand[:8]], check_every=4, flags=EDGE)


def test_edge_parallel_equals_node_parallel_bitwise():
    wl = W.make_workload("delaunay12")
    outs = []
    for flags in (0, EDGE):
        with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            outs.append([dbc.get_root_state(s)[:2] for s in range(wl.roots.size)])
    for (d0, s0), (d1, s1) in zip(outs[0], outs[1]):
        assert np.array_equal(d0, d1) and np.array_equal(s0, s1)


# ------------------------------------------------ edge deletion (Sec. 8(f) #4) ----
def _existing_edges(g, count, seed, roots=None, incident_to_roots=0):
    eu, ev = W.edges_of(g)
    rng = np.random.default_rng(seed)
    pick = list(rng.permutation(eu.size)[:count])
    out = [(int(eu[i]), int(ev[i])) for i in pick]
    if incident_to_roots and roots is not None:  # also edges at the roots (level-1 changes)
        rs = set(int(r) for r in roots)
        inc = [(int(a), int(b)) for a, b in zip(eu, ev) if int(a) in rs or int(b) in rs]
        for i in rng.permutation(len(inc))[:incident_to_roots]:
            if inc[i] not in out:
                out.append(inc[i])
    return out


def run_delete_stream(g, roots, pairs, batch=1, check_every=1, flags=0):
    roots = np.asarray(roots, np.int32)
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots, flags=flags) as dbc:
        dbc.static_compute()
        for b0 in range(0, len(pairs), batch):
            chunk = pairs[b0:b0 + batch]
            st = dbc.delete_edges([p[0] for p in chunk], [p[1] for p in chunk], stats=True)
            assert st["case1"] + st["case2"] + st["case3"] == roots.size * len(chunk)
            for a, b in chunk:
                ref.delete(a, b)
            if (b0 // batch + 1) % check_every == 0 or b0 + batch >= len(pairs):
                check_all(dbc, ref.compute(), roots.size)
        return dbc


@pytest.mark.parametrize("n", [5, 8, 9])
def test_delete_cycle_to_path_and_split(n):
    g = W.cycle_graph(n)
    # C_n -> P_n (distances grow), then cut the path in two (unreachable halves)
    run_delete_stream(g, np.arange(n), [(0, n - 1), (2, 3)])


def test_delete_complete_to_star():
    n = 7
    pairs = [(a, b) for a in range(1, n) for b in range(a + 1, n)]
    run_delete_stream(W.complete_graph(n), np.arange(n), pairs)
    run_delete_stream(W.complete_graph(n), np.arange(n), pairs, batch=len(pairs))


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12"])
def test_delete_single_and_batch_match_oracle(name):
    wl = W.make_workload(name)
    pairs = _existing_edges(wl.graph, 30, 1, wl.roots, incident_to_roots=6)
    run_delete_stream(wl.graph, wl.roots, pairs, batch=1, check_every=3)
    run_delete_stream(wl.graph, wl.roots, pairs, batch=12)


def test_delete_multicomponent_and_isolating():
    g = W.random_gnm(200, 230, 8)
    roots = np.arange(0, 200, 9)
    pairs = _existing_edges(g, 60, 2)  # tree-like graph: many deletions disconnect
    run_delete_stream(g, roots, pairs, batch=1, check_every=5)


def test_delete_grid_sigma_above_2_53():
    g = W.grid_graph(45, 45)
    roots = np.array([0, 44, 1012, 2024], np.int32)
    run_delete_stream(g, roots, _existing_edges(g, 10, 3), batch=1, check_every=5)


def test_delete_insert_mixed_stream():
    """Insert a batch, delete some of those and some original edges, re-insert."""
    wl = W.make_workload("rmat10")
    g, roots = wl.graph, wl.roots
    ref = oracle.NaiveDynamicBC(g, roots)
    orig = _existing_edges(g, 10, 5)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        ins = list(zip(wl.ins_u[:20].tolist(), wl.ins_v[:20].tolist()))
        dbc.insert_edges([p[0] for p in ins], [p[1] for p in ins])
        for a, b in ins:
            ref.insert(a, b)
        dele = ins[3:9] + orig
        dbc.delete_edges([p[0] for p in dele], [p[1] for p in dele])
        for a, b in dele:
            ref.delete(a, b)
        check_all(dbc, ref.compute(), roots.size)
        back = dele[:4] + dele[-3:]
        dbc.insert_edges([p[0] for p in back], [p[1] for p in back])
        for a, b in back:
            ref.insert(a, b)
        check_all(dbc, ref.compute(), roots.size)
        dbc.static_compute()  # GPU recompute on the final graph == the oracle too
        check_all(dbc, ref.compute(), roots.size)


def test_delete_rejects_bad_batches_atomically():
    from paper_conf_ipps_mclaughlinb14_b200 import DBCError

    wl = W.make_workload("karate")
    g, roots = wl.graph, wl.roots
    ref = oracle.brandes_csr(g, roots)
    eu, ev = W.edges_of(g)
    with _dbc(g, roots) as dbc:
        dbc.static_compute()
        for bad in ([(int(eu[0]), int(ev[0])), (5, 9)],          # (5, 9) absent in karate
                    [(int(eu[0]), int(ev[0])), (int(ev[0]), int(eu[0]))],  # duplicate pair
                    [(3, 3)], [(0, 34)]):
            with pytest.raises(DBCError):
                dbc.delete_edges([p[0] for p in bad], [p[1] for p in bad])
        check_all(dbc, ref, roots.size)  # nothing changed


@pytest.mark.timeout(240)
@pytest.mark.parametrize("rep", range(3))
def test_heavy_lane_with_help_completes_rmat16(rep):
    """Heavy lane (1024-thread CTAs) beside the normal lane with the help board
    on: a normal grid that fills every SM must not wait on heavy roots (the
    lanes steal each other's roots).  Full-size R-MAT 16, several batches from
    host arrays; d/sigma of sampled roots bit-exact vs the GPU's own recompute."""
    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC

    wl = W.make_workload("rmat16", insertions=4000, seed=1 + rep)
    g = wl.graph
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots) as dbc:
        dbc.static_compute()
        heavy = 0
        for b in range(4):
            dbc.insert_edges(wl.ins_u[1000 * b:1000 * (b + 1)], wl.ins_v[1000 * b:1000 * (b + 1)])
            heavy = max(heavy, dbc.timings()["heavy_roots"])
        dyn = [dbc.get_root_state(s)[:2] for s in range(0, wl.roots.size, 37)]
        dbc.static_compute()
        for i, s in enumerate(range(0, wl.roots.size, 37)):
            d, sg, _ = dbc.get_root_state(s)
            assert np.array_equal(d, dyn[i][0]) and np.array_equal(sg, dyn[i][1])


@pytest.mark.parametrize("block", [None, "512"])
@pytest.mark.parametrize("name", ["rmat10", "delaunay12u", "smallworld"])
def test_forced_help_paths_match_oracle(name, block, tune):
    """Every cooperative path forced on at small sizes: helped down levels
    (kind 1, 32-item blocks), entry-balanced long rows of every down level
    (kind 4), the Case-3 removal pass as help blocks (kind 3), helped delta-pull
    / push passes (kinds 2 / 0, 256-entry blocks), busy workers taking blocks of
    any pass; several batches (heavy lanes).  d/sigma bit-exact vs the oracle,
    BC within tolerance."""
    tune.update(help_down_min=1, help_down_block=32, down_long_min=1, help_min_blocks=1,
                help_entries=256, busy_min=1, busy_help=4, heavy_factor=1.0)
    if block:  # 512-thread CTAs (128 registers) beside the default width
        tune["update_block"] = int(block)
    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        c0 = dbc.debug_counters()
        nb = 3
        step = (wl.ins_u.size + nb - 1) // nb
        for b in range(nb):
            sl = slice(b * step, (b + 1) * step)
            dbc.insert_edges(wl.ins_u[sl], wl.ins_v[sl])
            for u, v in zip(wl.ins_u[sl], wl.ins_v[sl]):
                ref.insert(u, v)
        c1 = dbc.debug_counters()
        check_all(dbc, ref.compute(), wl.roots.size)
        assert c1["help_requests"] > c0["help_requests"]


@pytest.mark.parametrize("block", [None, "512"])
def test_wide_up_levels_deferred_chunks_match_oracle(block, tune):
    """Wide up levels walked with short rows in-lane (published as help blocks,
    kind 5) and long rows in chunks, more than one chunk of them deferred
    (DBC_WIDE_INLANE forces the mode on every level wider than a CTA): R-MAT
    2^14 / edgefactor 16, 64 roots, 400 insertions in two batches; d/sigma
    bit-exact vs the oracle, BC in tolerance."""
    tune["wide_inlane"] = 100000
    tune["busy_min"] = 1  # every pass worth publishing (kind-5 help blocks too)
    if block:
        tune["update_block"] = int(block)
    wl = W.make_workload("rmat14")
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    with _dbc(wl.graph, wl.roots) as dbc:
        dbc.static_compute()
        c0 = dbc.debug_counters()
        for sl in (slice(0, 200), slice(200, 400)):
            dbc.insert_edges(wl.ins_u[sl], wl.ins_v[sl])
            for u, v in zip(wl.ins_u[sl], wl.ins_v[sl]):
                ref.insert(u, v)
        c1 = dbc.debug_counters()
        check_all(dbc, ref.compute(), wl.roots.size)
        assert c1["deferred_rows"] > c0["deferred_rows"]  # more than one chunk of long rows
        assert c1["up_passes_helped"] > c0["up_passes_helped"]  # kind-5 help blocks ran



# ------------------------------------------------ per-insertion kernel (update_lean.cu) ----
@pytest.mark.parametrize("name", ["rmat10", "delaunay12u", "smallworld_small"])
def test_lean_fewer_workers_than_roots(name, tune):
    """Per-insertion jobs with 3 worker CTAs for all roots (dynamic root counter,
    several roots per worker and launch), one-job-per-insertion batch and Mode S."""
    tune["lean_workers"] = 3
    wl = W.make_workload(name)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    want = ref.compute()
    for flags in (0x10, 0x1):
        with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            check_all(dbc, want, wl.roots.size)


def test_lean_two_builds_per_launch_kind():
    """A hub graph with more roots than SMs: single-insertion launches run the
    128-register 512-thread build (one per SM), a launch over many insertions
    the 64-register build (two per SM, every root resident) -- both against the
    oracle, and the two orders of use within one context."""
    wl = W.make_workload("rmat10", k=300)
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    want = ref.compute()
    h = wl.ins_u.size // 2
    with _dbc(wl.graph, wl.roots, flags=0x10) as dbc:  # DBC_FLAG_NO_MERGE
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u[:h], wl.ins_v[:h])  # many insertions: two CTAs per SM
        for u, v in zip(wl.ins_u[h:].tolist(), wl.ins_v[h:].tolist()):
            dbc.insert_edges([u], [v])  # single insertions: one CTA per SM
        check_all(dbc, want, wl.roots.size)


@pytest.mark.parametrize("width", [128, 256, 512, 1024])
def test_lean_every_cta_width(width, tune):
    """The per-insertion kernel at every CTA width (128/256/512/1024 threads:
    meshes' multi-insertion launches, meshes, hub graphs, million-vertex hub
    graphs), one-job-per-insertion batch, Mode S and single-edge calls."""
    tune["lean_block"] = width
    wl = W.make_workload("rmat10")
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    want = ref.compute()
    for flags in (0x10, 0x1, 0):
        with _dbc(wl.graph, wl.roots, flags=flags) as dbc:
            dbc.static_compute()
            if flags:
                dbc.insert_edges(wl.ins_u, wl.ins_v)
            else:
                for u, v in zip(wl.ins_u.tolist(), wl.ins_v.tolist()):
                    dbc.insert_edges([u], [v])
            check_all(dbc, want, wl.roots.size)


@pytest.mark.parametrize("mult", ["0", "1"])
def test_lean_level2_shortcut_forced(mult, tune):
    """Level-2 up vertices resolved against adj(root) (probing the sorted rows)
    whenever the root's row is cached, on hub-heavy and mesh graphs."""
    tune["lean_short"] = int(mult)
    for name in ("rmat10", "rmat14", "delaunay12u"):
        wl = W.make_workload(name, insertions=60)
        ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
        with _dbc(wl.graph, wl.roots, flags=0x10) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            for u, v in zip(wl.ins_u, wl.ins_v):
                ref.insert(u, v)
            check_all(dbc, ref.compute(), wl.roots.size)


def test_lean_push_stash_overflow():
    """A down vertex with more predecessors outside D than the per-chunk push
    stash holds (600 > 512): the pushes run in a second pass over its row."""
    # s = 0; a_i = 1..600 (level 1) all adjacent to x = 601 (level 2); b = 602
    # adjacent to s; tail 603 -- 604 below x.  Inserting (b, x) gives x one
    # more predecessor (Case 2): x in D, the 600 a_i are not.
    fan = 600
    x, b = fan + 1, fan + 2
    eu = [0] * fan + list(range(1, fan + 1)) + [0, x, fan + 3]
    ev = list(range(1, fan + 1)) + [x] * fan + [b, fan + 3, fan + 4]
    g = W.csr_from_edges(fan + 5, eu, ev)
    roots = np.array([0, 1, fan + 4, b], np.int32)
    run_stream_single(g, roots, [b, 5], [x, fan + 4])
    for flags in (0x10, 0x1):
        ref = oracle.NaiveDynamicBC(g, roots)
        with _dbc(g, roots, flags=flags) as dbc:
            dbc.static_compute()
            dbc.insert_edges([b, 5], [x, fan + 4])
            ref.insert(b, x)
            ref.insert(5, fan + 4)
            check_all(dbc, ref.compute(), roots.size)


def test_lean_single_edge_calls_match_batch_kernel():
    """Single-edge calls (the per-insertion kernel) and the same insertions as
    one merged batch (update.cu) give bitwise equal d and sigma."""
    wl = W.make_workload("rmat14", insertions=80)
    outs = []
    for single in (True, False):
        with _dbc(wl.graph, wl.roots) as dbc:
            dbc.static_compute()
            if single:
                for u, v in zip(wl.ins_u, wl.ins_v):
                    dbc.insert_edges([u], [v])
            else:
                dbc.insert_edges(wl.ins_u, wl.ins_v)
            outs.append([dbc.get_root_state(s)[:2] for s in range(0, wl.roots.size, 5)] + [dbc.get_bc()])
    for (d0, s0), (d1, s1) in zip(outs[0][:-1], outs[1][:-1]):
        assert np.array_equal(d0, d1) and np.array_equal(s0, s1)
    assert_bc(outs[0][-1], outs[1][-1])


# ------------------------------------------------ DBC_FLAG_PULL_DELTA (bitwise delta) ----
def _bitwise_state(dbc, ref_out, k, what):
    bc_ref, d_ref, s_ref, dl_ref = ref_out
    for slot in range(k):
        d, s, dl = dbc.get_root_state(slot)
        assert np.array_equal(d, d_ref[slot]), f"{what}: d slot {slot}"
        assert np.array_equal(s.view(np.int64), s_ref[slot].view(np.int64)), f"{what}: sigma slot {slot}"
        bad = np.nonzero(dl.view(np.int64) != dl_ref[slot].view(np.int64))[0]
        assert bad.size == 0, f"{what}: delta slot {slot} at {bad[:4]}: {dl[bad[:4]]} vs {dl_ref[slot][bad[:4]]}"


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u", "grid60", "multi"])
def test_pull_delta_mode_is_bitwise(name):
    """DBC_FLAG_PULL_DELTA + DBC_FLAG_EXACT_BC at world 1 (SURVEY.md Sec. 8(c)
    items 14-15): every touched vertex pulls delta in canonical order, so d,
    sigma, delta AND BC are bit-identical to the oracle -- after the static pass
    and after insertion batches (Case 3 heavy streams, sigma > 2^53, several
    components included)."""
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_EXACT_BC, FLAG_PULL_DELTA

    if name == "grid60":
        g = W.grid_graph(60, 60)
        roots = np.array([0, 61, 1830, 3599, 29], np.int32)
        rng = np.random.default_rng(3)
        pairs = set()
        while len(pairs) < 30:
            a, b = (int(x) for x in rng.integers(0, g.n, 2))
            if a != b and b not in set(g.col[g.row_ptr[a]:g.row_ptr[a + 1]].tolist()):
                pairs.add((min(a, b), max(a, b)))
        us = np.array([p[0] for p in pairs], np.int32)
        vs = np.array([p[1] for p in pairs], np.int32)
    elif name == "multi":
        g = W.random_gnm(400, 380, 11)
        roots = np.arange(0, 400, 9, dtype=np.int32)
        rng = np.random.default_rng(5)
        eu, ev = W.edges_of(g)
        existing = set(zip(eu.tolist(), ev.tolist()))
        pairs = []
        while len(pairs) < 60:
            a, b = sorted(int(x) for x in rng.integers(0, g.n, 2))
            if a != b and (a, b) not in existing and (a, b) not in pairs:
                pairs.append((a, b))
        us = np.array([p[0] for p in pairs], np.int32)
        vs = np.array([p[1] for p in pairs], np.int32)
    else:
        wl = W.make_workload(name)
        g, roots, us, vs = wl.graph, wl.roots, wl.ins_u, wl.ins_v
    ref = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots, flags=FLAG_PULL_DELTA | FLAG_EXACT_BC) as dbc:
        dbc.static_compute()
        out = ref.compute()
        _bitwise_state(dbc, out, roots.size, "static")
        assert np.array_equal(dbc.get_bc().view(np.int64), out[0].view(np.int64))
        half = us.size // 2
        for sl in (slice(0, half), slice(half, None)):
            dbc.insert_edges(us[sl], vs[sl])
            for u, v in zip(us[sl], vs[sl]):
                ref.insert(u, v)
            out = ref.compute()
            _bitwise_state(dbc, out, roots.size, f"after {sl.stop}")
            assert np.array_equal(dbc.get_bc().view(np.int64), out[0].view(np.int64)), "BC not bitwise"
    # without the rebase: BC incremental (within the north star's tolerance), delta still bitwise
    ref2 = oracle.NaiveDynamicBC(g, roots)
    with _dbc(g, roots, flags=FLAG_PULL_DELTA) as dbc:
        dbc.static_compute()
        dbc.insert_edges(us, vs)
        for u, v in zip(us, vs):
            ref2.insert(u, v)
        out = ref2.compute()
        _bitwise_state(dbc, out, roots.size, "incremental BC")
        assert_bc(dbc.get_bc(), out[0])


def test_pull_delta_rejects_deletions():
    from paper_conf_ipps_mclaughlinb14_b200 import FLAG_PULL_DELTA, DBCError

    g = W.cycle_graph(8)
    with _dbc(g, np.array([0, 3], np.int32), flags=FLAG_PULL_DELTA) as dbc:
        dbc.static_compute()
        with pytest.raises(DBCError) as e:
            dbc.delete_edges([0], [1])
        assert e.value.name == "DBC_EINVAL"
