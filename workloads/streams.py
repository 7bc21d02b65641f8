"""Root sampling and edge-insertion streams (Sec. IV).

Readings (restated in DESIGN.md):
* roots: uniform without replacement among vertices of degree >= 1 in the
  initial graph, fixed seed (config 1 uses all 34 karate vertices);
* insertions: the paper's remove-then-reinsert protocol -- sample edges of the
  full graph, build the initial graph without them, reinsert in sampled order --
  or, for config 1 and the stress variant, uniform random non-edges.
"""

from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .graphs import CSR, csr_from_edges, edges_of, karate, rmat, delaunay, watts_strogatz


def sample_roots(g: CSR, k: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    cand = np.nonzero(g.degree() > 0)[0]
    if k >= cand.size:
        return cand.astype(np.int32)
    return rng.choice(cand, size=k, replace=False).astype(np.int32)


def remove_then_reinsert(g: CSR, count: int, seed: int):
    """Returns (initial graph without the sampled edges, u[], v[]) in reinsertion order."""
    rng = np.random.default_rng(seed)
    eu, ev = edges_of(g)
    count = min(count, eu.size)
    pick = rng.choice(eu.size, size=count, replace=False)
    keep = np.ones(eu.size, dtype=bool)
    keep[pick] = False
    g0 = csr_from_edges(g.n, eu[keep], ev[keep])
    # random orientation of each reinserted edge (the ABI is symmetric anyway)
    flip = rng.random(count) < 0.5
    u = np.where(flip, ev[pick], eu[pick]).astype(np.int32)
    v = np.where(flip, eu[pick], ev[pick]).astype(np.int32)
    return g0, u, v


def uniform_non_edges(g: CSR, count: int, seed: int):
    """`count` distinct uniformly random non-edges (u != v) of g, in sampled order."""
    rng = np.random.default_rng(seed)
    n = g.n
    eu, ev = edges_of(g)
    existing = set((eu.astype(np.int64) * n + ev).tolist()) if eu.size < 5_000_000 else None
    max_pairs = n * (n - 1) // 2 - eu.size
    count = min(count, max_pairs)
    chosen: list[int] = []
    seen: set[int] = set()
    if n <= 2048:
        # small graph: sample exactly among all non-edges
        iu, iv = np.triu_indices(n, 1)
        keys = iu.astype(np.int64) * n + iv
        mask = ~np.isin(keys, eu.astype(np.int64) * n + ev)
        cand = keys[mask]
        sel = rng.choice(cand.size, size=count, replace=False)
        chosen = cand[sel].tolist()
    else:
        ekeys = np.sort(eu.astype(np.int64) * n + ev)
        while len(chosen) < count:
            a = rng.integers(0, n, size=2 * count)
            b = rng.integers(0, n, size=2 * count)
            lo, hi = np.minimum(a, b), np.maximum(a, b)
            ok = lo != hi
            keys = lo[ok].astype(np.int64) * n + hi[ok]
            pos = np.searchsorted(ekeys, keys)
            pos = np.minimum(pos, ekeys.size - 1)
            isnew = ekeys[pos] != keys if ekeys.size else np.ones(keys.size, bool)
            for kk in keys[isnew].tolist():
                if kk not in seen:
                    seen.add(kk)
                    chosen.append(kk)
                    if len(chosen) == count:
                        break
    del existing
    keys = np.array(chosen, dtype=np.int64)
    lo, hi = keys // n, keys % n
    flip = rng.random(keys.size) < 0.5
    u = np.where(flip, hi, lo).astype(np.int32)
    v = np.where(flip, lo, hi).astype(np.int32)
    return u, v


@dataclass
class Workload:
    name: str
    graph: CSR  # initial graph (before any insertion)
    roots: np.ndarray  # int32 [k]
    ins_u: np.ndarray  # int32 [B]
    ins_v: np.ndarray  # int32 [B]
    meta: dict = field(default_factory=dict)


# BASELINE.json configs (made concrete in SURVEY.md Sec. 8(d)).
CONFIGS = {
    "karate": dict(graph="karate", k=34, insertions=10, mode="non_edges"),
    "rmat16": dict(graph="rmat", scale=16, ef=8, k=256, insertions=1000, mode="reinsert"),
    "delaunay18": dict(graph="delaunay", npts=1 << 18, k=512, insertions=1000, mode="reinsert"),
    # config 3's stress variant: uniform random
    # non-edges -- long-range Case-3 pull-ups on a high-diameter mesh
    "delaunay18u": dict(graph="delaunay", npts=1 << 18, k=512, insertions=1000, mode="non_edges"),
    "kron20": dict(graph="rmat", scale=20, ef=16, k=1024, insertions=10000, mode="reinsert"),
    "kron22": dict(graph="rmat", scale=22, ef=16, k=4096, insertions=10000, mode="reinsert"),
    "smallworld": dict(graph="ws", n=100_000, kk=10, p=0.1, k=256, insertions=100, mode="reinsert"),
    # small shapes of the same families for oracle-speed parity tests
    "rmat10": dict(graph="rmat", scale=10, ef=8, k=64, insertions=40, mode="reinsert"),
    "rmat14": dict(graph="rmat", scale=14, ef=16, k=64, insertions=400, mode="reinsert"),
    "delaunay12": dict(graph="delaunay", npts=1 << 12, k=48, insertions=40, mode="reinsert"),
    "delaunay12u": dict(graph="delaunay", npts=1 << 12, k=48, insertions=40, mode="non_edges"),
    "smallworld_small": dict(graph="ws", n=2000, kk=6, p=0.1, k=54, insertions=40, mode="reinsert"),
}


def _full_graph(cfg: dict, seed: int) -> CSR:
    kind = cfg["graph"]
    if kind == "karate":
        return karate()
    if kind == "rmat":
        return rmat(cfg["scale"], cfg["ef"], seed)
    if kind == "delaunay":
        return delaunay(cfg["npts"], seed)
    if kind == "ws":
        return watts_strogatz(cfg["n"], cfg["kk"], cfg["p"], seed)
    raise ValueError(kind)


def make_workload(name: str, seed: int = 1, insertions: int | None = None,
                  k: int | None = None, mode: str | None = None) -> Workload:
    cfg = dict(CONFIGS[name])
    if insertions is not None:
        cfg["insertions"] = insertions
    if k is not None:
        cfg["k"] = k
    if mode is not None:
        cfg["mode"] = mode
    full = _full_graph(cfg, seed)
    if cfg["mode"] == "reinsert":
        g0, u, v = remove_then_reinsert(full, cfg["insertions"], seed + 1000)
    else:
        g0 = full
        u, v = uniform_non_edges(full, cfg["insertions"], seed + 1000)
    roots = sample_roots(g0, cfg["k"], seed + 2000)
    meta = dict(cfg, seed=seed, n=g0.n, m=g0.m)
    return Workload(name, g0, roots, u, v, meta)
