"""Per-root profile of single-edge calls (diagnostic): for each call, the
slowest root's time, levels, touched vertices and scanned entries.

    python tools/lean_profile.py [config] [calls]   -> JSON lines
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
wl = W.make_workload(name, insertions=N)
g = wl.graph
rows = []
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING) as dbc:
    dbc.static_compute()
    dbc.synchronize()
    dbc.root_profile(enable=True, read=False)
    ph = ["sc_down", "sc_removal", "sc_dpull", "sc_dpush", "sc_up2", "sc_up3"]
    for i in range(N):
        c0 = dbc.debug_counters()
        dbc.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        c1 = dbc.debug_counters()
        t = dbc.timings()
        p = dbc.root_profile(enable=True, read=True)
        dt = (p[:, 1] - p[:, 0]) / 1e3  # us
        w = p[:, 2] > 0
        j = int(np.argmax(dt))
        rows.append({"i": i, "update_us": t["update_ms"] * 1e3, "working": int(w.sum()), "max_slot": j,
                     "max_us": float(dt[j]), "max_levels": int(p[j, 5]), "max_touched": int(p[j, 3]),
                     "max_scanned": int(p[j, 4]),
                     "median_working_us": float(np.median(dt[w])) if w.any() else 0.0,
                     "mean_working_levels": float(p[w, 5].mean()) if w.any() else 0.0,
                     "mean_working_touched": float(p[w, 3].mean()) if w.any() else 0.0,
                     "mean_working_scanned": float(p[w, 4].mean()) if w.any() else 0.0,
                     "us_per_level_median": float(np.median(dt[w] / np.maximum(p[w, 5], 1))) if w.any() else 0.0,
                     "scanned_by_phase": {k: c1[k] - c0[k] for k in ph}})
        print(json.dumps(rows[-1]), flush=True)
