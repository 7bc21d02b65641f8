"""CPU oracle for dynamic betweenness centrality -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
`--impl reference`) may import this package.  The product path
(paper_conf_ipps_mclaughlinb14_b200) never imports it, and this package never
imports the product.  Inputs come from `workloads/` (no method arithmetic).

* `brandes(g, roots)` -- static Brandes over a root set (Alg. 1, PAPER.md
  P:69-124, Eqs. (2)-(3) P:52-57), implemented in plain C (oracle/brandes.c,
  fp64, -ffp-contract=off), wrapped with ctypes.
* `NaiveDynamicBC` -- the naive dynamic rule of the north star: after each edge
  insertion (u, v) ("E' = E u {e}") append v to adj(u) and u to
  adj(v) (canonical order: original row, then inserted neighbours in insertion
  order) and recompute everything from scratch.

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
    """Compile oracle/brandes.c -> oracle/liboracle.so (gcc, fp64, no FMA contraction)."""
    src = os.path.join(_HERE, "brandes.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c99",
                               "-fPIC", "-shared", "-o", tmp, src])
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


class NaiveDynamicBC:
    """Naive dynamic rule: keep the canonical adjacency, recompute after each insertion."""

    def __init__(self, g, roots):
        self.n = g.n
        self.base_rp = np.asarray(g.row_ptr, dtype=np.int64)
        self.base_col = np.asarray(g.col, dtype=np.int32)
        self.roots = np.asarray(roots, dtype=np.int32)
        self.ins = []  # (u, v) in insertion order

    def insert(self, u: int, v: int):
        self.ins.append((int(u), int(v)))

    def csr(self):
        """Canonical adjacency: base row, then inserted neighbours in insertion order."""
        n = self.n
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
