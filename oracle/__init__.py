"""CPU oracle for dynamic betweenness centrality -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
`--impl reference`) may import this package.  The product path
(paper_conf_ipps_mclaughlinb14_b200) never imports it, and this package never
imports the product.  Inputs come from `workloads/` (no method arithmetic).

* `brandes(g, roots)` -- static Brandes over a root set (Alg. 1, PAPER.md
  P:69-124, Eqs. (2)-(3) P:52-57), implemented in plain C (oracle/brandes.c,
  fp64, -ffp-contract=off), wrapped with ctypes.
* `CpuDynamicBC` -- NOT part of the oracle: the paper's dynamic sequential
  CPU comparison algorithm (Alg. 2, with Case 3), single thread,
  in oracle/cpu_dynamic.c; pinned against the naive rule, timed by bench.py.
* `NaiveDynamicBC` -- the naive dynamic rule of the north star: after each edge
  insertion (u, v) ("E' = E u {e}") append v to adj(u) and u to
  adj(v) (canonical order: original row, then inserted neighbours in insertion
  order) and recompute everything from scratch; after a deletion (the
  decremental counterpart) remove the two entries, the rows keeping the order
  of their remaining entries, and recompute.

Pins (tests/test_oracle.py): brute-force path enumeration on n <= 9, closed
forms (path, star, cycle, complete graph, grid binomials), networkx on karate
and random graphs, the Sigma-BC = Sigma (d-1) identity, Case-1 invariance.
"""

from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

INF = np.iinfo(np.int32).max


def build(force: bool = False) -> str:
    """Compile oracle/brandes.c (+ the CPU dynamic baseline cpu_dynamic.c) ->
    oracle/liboracle.so (gcc, fp64, no FMA contraction)."""
    srcs = [os.path.join(_HERE, f) for f in ("brandes.c", "cpu_dynamic.c")]
    newest = max(os.path.getmtime(f) for f in srcs)
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < newest:
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c99",
                               "-fPIC", "-shared", "-o", tmp] + srcs)
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB_PATH)
            P = ctypes.c_void_p
            lib.oracle_brandes.argtypes = [ctypes.c_int32, P, P, P, ctypes.c_int32, P, P, P, P]
            lib.oracle_brandes.restype = ctypes.c_int
            lib.cd_create.argtypes = [ctypes.c_int32, P, P, P, ctypes.c_int32]
            lib.cd_create.restype = P
            lib.cd_destroy.argtypes = [P]
            lib.cd_destroy.restype = None
            lib.cd_insert.argtypes = [P, ctypes.c_int32, ctypes.c_int32]
            lib.cd_insert.restype = ctypes.c_int
            lib.cd_insert_roots.argtypes = [P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32]
            lib.cd_insert_roots.restype = ctypes.c_int
            lib.cd_get.argtypes = [P, P, P, P, P]
            lib.cd_get.restype = None
            lib.cd_scenarios.argtypes = [P, P]
            lib.cd_scenarios.restype = None
            _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def brandes(n, row_ptr, col, roots, want_state=True):
    """Static Brandes over `roots` (slot order).  Returns (bc[n], d[k,n], sigma[k,n], delta[k,n])."""
    lib = _load()
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    roots = np.ascontiguousarray(roots, dtype=np.int32)
    k = roots.size
    bc = np.zeros(n, dtype=np.float64)
    d = sig = dl = None
    if want_state:
        d = np.empty((k, n), dtype=np.int32)
        sig = np.empty((k, n), dtype=np.float64)
        dl = np.empty((k, n), dtype=np.float64)
    rc = lib.oracle_brandes(n, _ptr(row_ptr), _ptr(col), _ptr(roots), k,
                            _ptr(d), _ptr(sig), _ptr(dl), _ptr(bc))
    if rc != 0:
        raise RuntimeError(f"oracle_brandes failed: {rc}")
    return bc, d, sig, dl


def brandes_csr(g, roots, want_state=True):
    return brandes(g.n, g.row_ptr, g.col, roots, want_state)


def host_threads() -> int:
    """Host cores this process may use (the root-parallel leg's thread count)."""
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return max(1, os.cpu_count() or 1)


def brandes_parallel(n, row_ptr, col, roots, threads=None, state_slots=None):
    """Root-parallel leg of `brandes` (SURVEY.md Sec. 8(d) oracle timing (ii)).

    The SAME per-root computation (oracle_brandes called with one root, so
    Alg. 1 / Eq. (2) run unchanged, in canonical order) is spread over host
    threads; BC is then Eq. (3) summed in slot order -- bc = ((0 + delta_0) +
    delta_1) + ..., one IEEE add per slot and vertex exactly as brandes.c does
    (delta_s(s) = 0, so adding slot s's whole row equals skipping v = s).  The
    result is therefore bit-identical to `brandes` (pinned in
    tests/test_oracle.py).  Roots run in waves of `threads` so only
    threads x n deltas are held at once.

    state_slots: None -> no per-root state returned; an index array -> (d,
    sigma, delta) of those slots (rows in the order given).
    Returns (bc[n], d, sigma, delta)."""
    from concurrent.futures import ThreadPoolExecutor

    lib = _load()
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    roots = np.ascontiguousarray(roots, dtype=np.int32)
    k = roots.size
    T = max(1, int(threads or host_threads()))
    want = {} if state_slots is None else {int(s): i for i, s in enumerate(state_slots)}
    m = len(want)
    d = np.empty((m, n), np.int32) if m else None
    sig = np.empty((m, n), np.float64) if m else None
    dl = np.empty((m, n), np.float64) if m else None
    bc = np.zeros(n, dtype=np.float64)
    wave = np.empty((min(T, max(k, 1)), n), np.float64)
    rbuf = [np.empty(1, np.int32) for _ in range(wave.shape[0])]

    def one(slot, j):
        rbuf[j][0] = roots[slot]
        i = want.get(slot)
        rc = lib.oracle_brandes(n, _ptr(row_ptr), _ptr(col), _ptr(rbuf[j]), 1,
                                None if i is None else _ptr(d[i]),
                                None if i is None else _ptr(sig[i]),
                                _ptr(wave[j]), None)
        if rc != 0:
            raise RuntimeError(f"oracle_brandes failed: {rc}")
        if i is not None:
            dl[i] = wave[j]

    with ThreadPoolExecutor(max_workers=T) as ex:
        for s0 in range(0, k, T):
            s1 = min(k, s0 + T)
            list(ex.map(lambda a: one(*a), [(s, s - s0) for s in range(s0, s1)]))
            for s in range(s0, s1):  # Eq. (3) in slot order
                bc += wave[s - s0]
    return bc, d, sig, dl


class NaiveDynamicBC:
    """Naive dynamic rule: keep the canonical adjacency, recompute after each insertion."""

    def __init__(self, g, roots):
        self.n = g.n
        self.base_rp = np.asarray(g.row_ptr, dtype=np.int64)
        self.base_col = np.asarray(g.col, dtype=np.int32)
        self.roots = np.asarray(roots, dtype=np.int32)
        self.ins = []  # (u, v) in insertion order

    def insert(self, u: int, v: int):
        if getattr(self, "adj", None) is not None:
            self.adj[int(u)].append(int(v))
            self.adj[int(v)].append(int(u))
            return
        self.ins.append((int(u), int(v)))

    def delete(self, u: int, v: int):
        """Edge deletion (decremental update): E' = E minus
        {(u, v)}; each row keeps the order of its remaining entries."""
        if getattr(self, "adj", None) is None:  # switch to explicit neighbour lists
            rp, col = self.csr()
            self.adj = [col[rp[x]:rp[x + 1]].tolist() for x in range(self.n)]
        self.adj[int(u)].remove(int(v))
        self.adj[int(v)].remove(int(u))

    def csr(self):
        """Canonical adjacency: base row, then inserted neighbours in insertion order
        (after a deletion: explicit per-vertex lists, removal keeps the order)."""
        n = self.n
        if getattr(self, "adj", None) is not None:
            deg = np.array([len(a) for a in self.adj], dtype=np.int64)
            rp = np.zeros(n + 1, dtype=np.int64)
            rp[1:] = np.cumsum(deg)
            col = np.fromiter((y for a in self.adj for y in a), dtype=np.int32, count=int(rp[-1]))
            return rp, col
        if not self.ins:
            return self.base_rp.copy(), self.base_col.copy()
        e = np.array(self.ins, dtype=np.int64)
        # directed extra entries in insertion order: for edge i, (u -> v) and (v -> u)
        src = np.empty(2 * len(e), dtype=np.int64)
        dst = np.empty(2 * len(e), dtype=np.int64)
        src[0::2], dst[0::2] = e[:, 0], e[:, 1]
        src[1::2], dst[1::2] = e[:, 1], e[:, 0]
        order = np.argsort(src, kind="stable")  # stable: keeps insertion order within a row
        src, dst = src[order], dst[order]
        extra_deg = np.bincount(src, minlength=n)
        base_deg = np.diff(self.base_rp)
        rp = np.zeros(n + 1, dtype=np.int64)
        rp[1:] = np.cumsum(base_deg + extra_deg)
        col = np.empty(rp[-1], dtype=np.int32)
        # base entries
        base_rows = np.repeat(np.arange(n), base_deg)
        base_pos = rp[base_rows] + (np.arange(self.base_col.size) - self.base_rp[base_rows])
        col[base_pos] = self.base_col
        # extra entries after the base row, in insertion order
        first = np.zeros(n + 1, dtype=np.int64)
        first[1:] = np.cumsum(extra_deg)
        rank = np.arange(src.size) - first[src]
        col[rp[src] + base_deg[src] + rank] = dst
        return rp, col

    def compute(self, want_state=True):
        rp, col = self.csr()
        return brandes(self.n, rp, col, self.roots, want_state)


def scenarios(rp_old, col_old, rp_new, col_new, roots, u, v):
    """Scenario of each root for the insertion of (u, v) (Fig. 2 / Fig. 4).

    rp_old/col_old: the graph before the insertion; rp_new/col_new: after it.
    Returns (case[k], touched[k], down[k]) int64:
      case: 1 if d_s(u) == d_s(v) (both unreachable included),
        2 if |d_s(u) - d_s(v)| == 1, else 3 (one endpoint unreachable is 3);
      touched ("{i in V | t[i] != untouched}") for Case 2, following
        Alg. 2: the down-touched set D = u_low and every vertex
        reached from it along the NEW shortest-path DAG (t[w] = down, lines
        9-20), plus every vertex reached from D by predecessor steps (t[v] = up,
        lines 21-35), the root itself excluded (its delta is never used,
        P:221-223).  0 for Case 1, -1 for Case 3 (not defined by the paper);
      down = |D| for Case 2 (the vertices whose sigma changes), 0 / -1 likewise.
    Pinned in tests/test_oracle.py against an all-pairs characterisation
    (sigma changed / lies on a shortest path to such a vertex)."""
    n = rp_old.size - 1
    _, d0, _, _ = brandes(n, rp_old, col_old, roots)
    _, d1, _, _ = brandes(n, rp_new, col_new, roots)
    k = len(roots)
    case = np.zeros(k, dtype=np.int64)
    touched = np.zeros(k, dtype=np.int64)
    down = np.zeros(k, dtype=np.int64)
    for j in range(k):
        du, dv = int(d0[j, u]), int(d0[j, v])
        if du == dv:
            case[j] = 1
            continue
        if min(du, dv) + 1 != max(du, dv):
            case[j] = 3
            touched[j] = -1
            down[j] = -1
            continue
        case[j] = 2
        d = d1[j]
        ul = v if du < dv else u
        t = np.zeros(n, dtype=bool)
        t[ul] = True
        queue = [ul]
        qi = 0
        while qi < len(queue):  # down: successors in the new DAG
            w = queue[qi]
            qi += 1
            for y in col_new[rp_new[w]:rp_new[w + 1]]:
                if d[y] == d[w] + 1 and not t[y]:
                    t[y] = True
                    queue.append(int(y))
        down[j] = len(queue)
        qi = 0
        while qi < len(queue):  # up: predecessors of touched vertices
            x = queue[qi]
            qi += 1
            for p in col_new[rp_new[x]:rp_new[x + 1]]:
                if d[p] == d[x] - 1 and not t[p]:
                    t[p] = True
                    queue.append(int(p))
        t[roots[j]] = False
        touched[j] = int(t.sum())
    return case, touched, down


class CpuDynamicBC:
    """The dynamic sequential CPU baseline (oracle/cpu_dynamic.c): Alg. 2 of
    the paper (Green et al.) with Case 3, one thread.  A comparison
    program for bench.py (`cpu_dynamic`), pinned against NaiveDynamicBC."""

    def __init__(self, g, roots):
        lib = _load()
        self.n = g.n
        self.k = len(roots)
        rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(g.col, dtype=np.int32)
        self.roots = np.ascontiguousarray(roots, dtype=np.int32)
        self._h = lib.cd_create(g.n, _ptr(rp), _ptr(col), _ptr(self.roots), self.k)
        if not self._h:
            raise MemoryError("cd_create failed")
        self._lib = lib

    def insert(self, u: int, v: int, roots: tuple | None = None):
        if roots is None:
            rc = self._lib.cd_insert(self._h, int(u), int(v))
        else:
            rc = self._lib.cd_insert_roots(self._h, int(u), int(v), int(roots[0]), int(roots[1]))
        if rc != 0:
            raise MemoryError("cd_insert failed")

    def state(self):
        bc = np.empty(self.n, np.float64)
        d = np.empty((self.k, self.n), np.int32)
        sig = np.empty((self.k, self.n), np.float64)
        dl = np.empty((self.k, self.n), np.float64)
        self._lib.cd_get(self._h, _ptr(bc), _ptr(d), _ptr(sig), _ptr(dl))
        return bc, d, sig, dl

    def scenarios(self):
        out = np.zeros(3, np.int64)
        self._lib.cd_scenarios(self._h, _ptr(out))
        return out

    def close(self):
        if getattr(self, "_h", None):
            self._lib.cd_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()
