"""Anatomy of single-edge update launches (diagnostic): for N single-edge
dbc_insert_edges calls, the update kernel's device time (dbc_get_timings) beside
the per-root profile of the launch (globaltimer start/end, touched, entries,
level steps): launch span, the slowest root's chain and what it touched, the
median working root, and the cost of a Case-1-only root.

    python tools/lean_anatomy.py config N [tuning k=v,...]   -> JSON lines
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, N = sys.argv[1], int(sys.argv[2])
tune = {}
if len(sys.argv) > 3:
    for kv in sys.argv[3].split(","):
        k, v = kv.split("=")
        tune[k] = int(v)
wl = W.make_workload(name, insertions=N)
g = wl.graph
rows = []
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning=tune or None) as d:
    d.static_compute()
    d.synchronize()
    d.root_profile(True, read=False)
    for i in range(N):
        d.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        t = d.timings()
        p = d.root_profile(True, read=True).astype(np.float64)
        st, en, jobs, touch, ent, lev = p.T
        dur = (en - st) / 1e3  # us
        span = (en.max() - st.min()) / 1e3
        cp = d.cta_profile().astype(np.float64)
        cp = cp[cp[:, 0] > 0]
        w = jobs > 0
        j = int(np.argmax(dur))
        rows.append({
            "i": i, "kernel_us": t["update_ms"] * 1e3, "span_us": span,
            "start_spread_us": (st.max() - st.min()) / 1e3,
            "working": int(w.sum()),
            "max_us": dur[j], "max_touched": int(touch[j]), "max_entries": int(ent[j]), "max_levels": int(lev[j]),
            "med_working_us": float(np.median(dur[w])) if w.any() else 0.0,
            "med_working_levels": float(np.median(lev[w])) if w.any() else 0.0,
            "med_working_touched": float(np.median(touch[w])) if w.any() else 0.0,
            "cta_entry_to_first_root_us": (st.min() - cp[:, 0].min()) / 1e3,
            "cta_entry_spread_us": (cp[:, 0].max() - cp[:, 0].min()) / 1e3,
            "last_root_to_last_loop_end_us": (cp[:, 1].max() - en.max()) / 1e3,
            "last_loop_end_to_last_exit_us": (cp[:, 2].max() - cp[:, 1].max()) / 1e3,
            "cta_first_entry_to_last_exit_us": (cp[:, 2].max() - cp[:, 0].min()) / 1e3,
            "med_idle_us": float(np.median(dur[~w])) if (~w).any() else 0.0,
        })
for r in rows:
    print(json.dumps({k: (round(v, 2) if isinstance(v, float) else v) for k, v in r.items()}))
agg = {k: float(np.mean([r[k] for r in rows])) for k in rows[0] if k != "i"}
agg["config"] = name
agg["calls"] = N
print(json.dumps({"mean": {k: (round(v, 2) if isinstance(v, float) else v) for k, v in agg.items()}}))
