"""Static Brandes recompute time per mapping (diagnostic).

    python tools/static_probe.py config [variants...]   variants: dbc_tuning fields, e.g.
        static_ms=0   static_ms=1,static_groups=8,static_chunk=256   -> JSON lines
Every variant's state is compared with the first variant's on 8 sampled root
slots (d and sigma bitwise, delta relative error) and BC (relative error).
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name = sys.argv[1]
wl = W.make_workload(name, insertions=10)
g = wl.graph
k = wl.roots.size
slots = np.unique(np.linspace(0, k - 1, min(8, k)).astype(int))
first = None
for var in sys.argv[2:] or ["default"]:
    tune = {}
    if var != "default":
        for kv in var.split(","):
            key, v = kv.split("=")
            tune[key] = int(v)
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning=tune or None) as d:
        ts = []
        for _ in range(3):
            d.static_compute()
            t = d.timings()
            ts.append((t["static_ms"], t["static_alg_bytes"]))
        ms, nb = min(ts)
        bc = d.get_bc()
        st = {int(s): d.get_root_state(int(s)) for s in slots}
    res = {"config": name, "variant": var, "static_ms": ms, "all_ms": [round(x[0], 3) for x in ts],
           "alg_GBps": nb / (ms / 1e3) / 1e9}
    if first is None:
        first = (bc, st)
    else:
        bc0, st0 = first
        res["bc_rel_err"] = float((np.abs(bc - bc0) / np.maximum(np.abs(bc0), 1)).max())
        res["d_sigma_equal"] = all(np.array_equal(st[s][0], st0[s][0]) and np.array_equal(st[s][1], st0[s][1])
                                   for s in st)
        res["delta_rel_err"] = max(float((np.abs(st[s][2] - st0[s][2]) / np.maximum(np.abs(st0[s][2]), 1)).max())
                                   for s in st)
    print(json.dumps(res), flush=True)
