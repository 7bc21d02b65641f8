"""Fig. 2, Fig. 4 and Table III of the paper, measured on this implementation.

    python tools/paper_figures.py [config] [insertions]  -> one JSON object on stdout

* Fig. 2: distribution of the k x B scenarios over Case 1/2/3.
* Fig. 4: fraction of the vertices touched
  ({i | t[i] != untouched}, Alg. 2's set: D and every ancestor, the root
  excluded -- the scenario log counts it exactly, R19) by every
  Case-2 scenario, sorted ascending.
* Table III: per-insertion update time (fastest / average /
  slowest single-edge call) against one static recompute over the same roots.
Inputs: the bench workload (remove-then-reinsert).  Diagnostics only:
not part of the hot path; the scenario log forces one job per (root, insertion).
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import (FLAG_EDGE_PARALLEL, FLAG_NO_MERGE, FLAG_TIMING,  # noqa: E402
                                                DynamicBC)

name = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 100
wl = W.make_workload(name, insertions=B + 3)
g = wl.graph
k = wl.roots.size
out = {"config": name, "n": g.n, "m": g.m, "k": k, "insertions": B}

with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING) as dbc:
    dbc.static_compute()
    dbc.synchronize()
    dbc.static_compute()
    static_ms = dbc.timings()["static_ms"]
    dbc.scenario_log(B)
    dbc.insert_edges(wl.ins_u[:B], wl.ins_v[:B])
    case, touched, down = dbc.scenarios()
cnt = np.bincount(case.ravel(), minlength=4)[1:]
out["fig2_case_fraction"] = {f"case{i + 1}": float(cnt[i] / cnt.sum()) for i in range(3)}
out["fig2_case2_of_working"] = float(cnt[1] / max(cnt[1] + cnt[2], 1))
out["fig2_paper"] = "Case 2 = 37.3% of all scenarios, 73.5% of the working ones (P:161)"
t2 = np.sort(touched[case == 2].astype(np.float64) / g.n)
if t2.size:
    q = [0.5, 0.9, 0.99, 1.0]
    out["fig4_case2_scenarios"] = int(t2.size)
    out["fig4_touched_fraction_quantiles"] = {str(x): float(np.quantile(t2, x)) for x in q}
    out["fig4_touched_fraction_mean"] = float(t2.mean())
    d2 = down[case == 2].astype(np.float64) / g.n
    out["fig4_down_fraction_mean_max"] = [float(d2.mean()), float(d2.max())]
    out["fig4_sorted_curve"] = [float(x) for x in t2[np.linspace(0, t2.size - 1, min(200, t2.size)).astype(int)]]
out["fig4_paper"] = "max ~35% of the vertices touched over 62,844 Case-2 scenarios, most tiny (P:514)"

# Table III: single-edge calls, one job per (root, insertion), on a fresh
# context (same initial graph); the first 3 insertions are warm-up
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING | FLAG_NO_MERGE) as dbc:
    dbc.static_compute()
    dbc.synchronize()
    per = []
    for i in range(B + 3):
        dbc.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        t = dbc.timings()
        if i >= 3:
            per.append(t["update_ms"])
per = np.array(per)
out["table3"] = {"static_ms": static_ms, "fastest_ms": float(per.min()), "average_ms": float(per.mean()),
                 "slowest_ms": float(per.max()),
                 "speedup_fastest": static_ms / per.min(), "speedup_average": static_ms / per.mean(),
                 "speedup_slowest": static_ms / per.max(),
                 "what": "device time of the update kernel of single-edge dbc_insert_edges calls (graph update neglected as in P:440), "
                         "DBC_FLAG_NO_MERGE, vs one dbc_static_compute over the same roots"}
out["table3_paper"] = "45x mean speedup over static GPU recompute; slowest 2x-43x (P:512-514)"

# Table II: node-based vs edge-based parallelism, same single-edge calls
BE = min(B, int(os.environ.get("EDGE_INSERTIONS", "20")))
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING | FLAG_EDGE_PARALLEL) as dbc:
    dbc.static_compute()
    dbc.synchronize()
    pe = []
    for i in range(BE + 3):
        dbc.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        if i >= 3:
            pe.append(dbc.timings()["update_ms"])
pe = np.array(pe)
out["table2"] = {"insertions": BE, "node_avg_ms": float(per[:BE].mean()), "edge_avg_ms": float(pe.mean()),
                 "node_over_edge": float(pe.mean() / per[:BE].mean()),
                 "what": "same first insertions, single-edge calls: node-based kernel (DBC_FLAG_NO_MERGE) vs "
                         "edge-based kernel (DBC_FLAG_EDGE_PARALLEL, Alg. 4/6)"}
out["table2_paper"] = "node-based 4.0x (small) to 37.2x (coPapersCiteseer) faster than edge-based (P:458-478)"
print(json.dumps(out))
