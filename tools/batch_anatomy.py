"""Anatomy of window-merged batch launches (diagnostic): per-root chain times
of the batch kernel (dbc_debug_root_profile) against the launch's device time:
how much of the launch is the slowest root's chain, how the chains are spread,
what the slowest roots touched.

    python tools/batch_anatomy.py config batches [batch] [tuning k=v,...]   -> JSON lines
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, NB = sys.argv[1], int(sys.argv[2])
B = int(sys.argv[3]) if len(sys.argv) > 3 else 1000
tune = {}
if len(sys.argv) > 4:
    for kv in sys.argv[4].split(","):
        k, v = kv.split("=")
        tune[k] = int(v)
wl = W.make_workload(name, insertions=NB * B)
g = wl.graph
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, edge_capacity=NB * B,
               tuning=tune or None) as d:
    d.static_compute()
    d.synchronize()
    d.root_profile(True, read=False)
    for b in range(NB):
        d.insert_edges(wl.ins_u[b * B:(b + 1) * B], wl.ins_v[b * B:(b + 1) * B])
        t = d.timings()
        p = d.root_profile(True, read=True).astype(np.float64)
        st, en, jobs, touch, ent, lev = p.T
        ok = en > 0
        dur = (en - st)[ok] / 1e3
        order = np.argsort(-dur)
        top = [{"us": round(float(dur[j]), 1), "touched": int(touch[ok][j]), "scanned": int(ent[ok][j]),
                "levels": int(lev[ok][j]), "jobs": int(jobs[ok][j])} for j in order[:5]]
        print(json.dumps({
            "batch": b, "kernel_us": round(t["update_ms"] * 1e3, 1),
            "span_us": round(float((en[ok].max() - st[ok].min()) / 1e3), 1),
            "chain_us_quantiles": {q: round(float(np.quantile(dur, q)), 1) for q in (0.1, 0.5, 0.9, 0.99, 1.0)},
            "sum_chain_us": round(float(dur.sum()), 1),
            "start_spread_us": round(float((st[ok].max() - st[ok].min()) / 1e3), 1),
            "heavy_roots": t.get("heavy_roots"),
            "top": top}))
