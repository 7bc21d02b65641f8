"""The slowest root of single-edge calls, traced (diagnostic): for each of the
first `calls` insertions of a config, find the slowest root (root profile),
then replay the same stream with that root traced and report its phase clocks
and the help-board activity of that call.

    python tools/lean_heavy.py config calls
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, N = sys.argv[1], int(sys.argv[2])
wl = W.make_workload(name, insertions=N)
g = wl.graph
names = ["down_load", "down_scan", "down_pass_final", "up_after_pass", "removal", "up_setup", "up_Drows",
         "up_load", "up_scan", "up_pass"]
keys = ["ns_down", "ns_removal", "ns_up_setup", "ns_up_epi", "ns_up_l1pairs", "ns_up_end", "ns_up_split",
        "ns_up_scan", "ns_up_pull", "ns_up_push"]
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING) as d:
    d.static_compute()
    d.root_profile(True, read=False)
    slow = []
    for i in range(N):
        d.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        p = d.root_profile(True, read=True)
        dt = p[:, 1] - p[:, 0]
        slow.append((int(np.argmax(dt)), float(dt.max()) / 1e3, d.timings()["update_ms"] * 1e3))
worst = sorted(range(N), key=lambda i: -slow[i][1])[:3]
for i in worst:
    slot = slow[i][0]
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning={"trace_slot": slot}) as d:
        d.static_compute()
        if i:
            d.insert_edges(wl.ins_u[:i], wl.ins_v[:i])  # the same state (merged batch: same d/sigma/delta)
        d.root_profile(True, read=False)
        c0 = d.debug_counters()
        d.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
        c1 = d.debug_counters()
        p = d.root_profile(True, read=True)
        t = d.timings()
    cyc = {names[q]: c1[keys[q]] - c0[keys[q]] for q in range(10)}
    print(json.dumps({"insertion": i, "slot": slot, "root_us": (p[slot, 1] - p[slot, 0]) / 1e3,
                      "update_us": t["update_ms"] * 1e3, "levels": int(p[slot, 5]), "touched": int(p[slot, 3]),
                      "cycles": cyc, "help_requests": c1["help_requests"] - c0["help_requests"],
                      "help_blocks_all": c1["help_blocks_all"] - c0["help_blocks_all"],
                      "help_blocks_by_helpers": c1["help_blocks_by_helpers"] - c0["help_blocks_by_helpers"],
                      "scanned": {k: c1[k] - c0[k] for k in ("sc_down", "sc_removal", "sc_dpull", "sc_dpush",
                                                             "sc_up2", "sc_up3")}}), flush=True)
