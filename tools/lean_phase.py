"""Phase clocks of the per-insertion kernel for one traced root (diagnostic):
single-edge calls on a config, SM cycles per phase of root slot `slot`.

    python tools/lean_phase.py config slot calls [tuning k=v,...]
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, slot, N = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
tune = {"trace_slot": slot}
if len(sys.argv) > 4:
    for kv in sys.argv[4].split(","):
        k, v = kv.split("=")
        tune[k] = int(v)
wl = W.make_workload(name, insertions=N)
g = wl.graph
names = ["down_load", "down_scan", "down_pass_final", "up_after_pass", "removal", "up_setup", "up_Drows",
         "up_load", "up_scan", "up_pass"]
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning=tune) as d:
    d.static_compute()
    d.synchronize()
    d.root_profile(True, read=False)
    c0 = d.debug_counters()
    lev = 0
    ns = 0
    jobs = 0
    for i in range(N):
        d.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        p = d.root_profile(True, read=True)
        lev += int(p[slot, 5])
        ns += int(p[slot, 1] - p[slot, 0])
        jobs += int(p[slot, 2])
    c1 = d.debug_counters()
keys = ["ns_down", "ns_removal", "ns_up_setup", "ns_up_epi", "ns_up_l1pairs", "ns_up_end", "ns_up_split",
        "ns_up_scan", "ns_up_pull", "ns_up_push"]
cyc = {names[q]: c1[keys[q]] - c0[keys[q]] for q in range(10)}
tot = sum(cyc.values())
print(json.dumps({"config": name, "slot": slot, "calls": N, "jobs": jobs, "levels": lev, "root_ns": ns,
                  "us_per_level": ns / 1e3 / max(lev, 1),
                  "cycles_per_level": {k: round(v / max(lev, 1), 1) for k, v in cyc.items()},
                  "share": {k: round(v / max(tot, 1), 3) for k, v in cyc.items()}}))
