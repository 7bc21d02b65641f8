"""Static Brandes recompute time per mapping (diagnostic).

    python tools/static_probe.py config [variants...]   variants: dbc_tuning fields, e.g.
        static_kernel=1,static_block=1024   static_kernel=2,static_block=512   -> JSON lines
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name = sys.argv[1]
wl = W.make_workload(name, insertions=10)
g = wl.graph
for var in sys.argv[2:] or ["default"]:
    tune = {}
    if var != "default":
        for kv in var.split(","):
            k, v = kv.split("=")
            tune[k] = int(v)
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning=tune or None) as d:
        best = None
        for _ in range(3):
            d.static_compute()
            t = d.timings()
            best = t if best is None or t["static_ms"] < best["static_ms"] else best
        print(json.dumps({"config": name, "variant": var, "static_ms": best["static_ms"],
                          "alg_GBps": best["static_alg_bytes"] / (best["static_ms"] / 1e3) / 1e9}), flush=True)
