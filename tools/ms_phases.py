"""Phase clock of the multi-source static kernel (msbrandes.cu): the time of
every grid-barrier-separated pass (block 0's %globaltimer after each barrier).

    python tools/ms_phases.py config [tuning k=v,...]   -> one JSON line per config
"""
import ctypes
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

K_TRACE_N, K_TRACE0, K_COUNT = 34, 35, 35 + 2048
KIND = {1: "init", 2: "expand", 3: "sigma", 4: "delta", 5: "transpose"}

name = sys.argv[1]
tune = {"static_ms": 1}
for kv in (sys.argv[2].split(",") if len(sys.argv) > 2 else []):
    k, v = kv.split("=")
    tune[k] = int(v)
wl = W.make_workload(name, insertions=10)
g = wl.graph
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning=tune) as d:
    for _ in range(2):
        d.static_compute()
    t = d.timings()
    raw = np.zeros(K_COUNT, np.int64)
    rc = d._lib.dbc_debug_counters(d._ctx, raw.ctypes.data_as(ctypes.c_void_p), K_COUNT)
    assert rc == 0
nev = int(raw[K_TRACE_N])
ev = raw[K_TRACE0:K_TRACE0 + 2 * nev].reshape(-1, 2)
tot = {}
rows = []
for i in range(1, nev):
    kind, lev = int(ev[i, 0]) >> 16, int(ev[i, 0]) & 0xffff
    dt = (int(ev[i, 1]) - int(ev[i - 1, 1])) / 1e3
    tot[KIND[kind]] = tot.get(KIND[kind], 0.0) + dt
    rows.append([KIND[kind], lev, round(dt, 1)])
print(json.dumps({"config": name, "tune": tune, "static_ms": t["static_ms"],
                  "kernel_us": (int(ev[-1, 1]) - int(ev[0, 1])) / 1e3 if nev else None,
                  "totals_us": {k: round(v, 1) for k, v in tot.items()}, "passes": rows}), flush=True)
