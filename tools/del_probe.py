"""Deletion throughput probe (diagnostic): one 1,000-insertion batch, then the
last D inserted edges deleted again newest first (one job per (root, deletion)),
device-timed, for several dbc_tuning variants.

    python tools/del_probe.py config D variants...   -> JSON lines
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC  # noqa: E402

name, D = sys.argv[1], int(sys.argv[2])
wl = W.make_workload(name, insertions=1000)
g = wl.graph
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
for var in sys.argv[3:] or ["default"]:
    tune = {}
    if var != "default":
        for kv in var.split(","):
            k, x = kv.split("=")
            tune[k] = int(x)
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, stream=stream.cuda_stream, tuning=tune or None) as d:
        d.static_compute()
        d.insert_edges(wl.ins_u, wl.ins_v)
        d.synchronize()
        du, dv = wl.ins_u[::-1][:D].copy(), wl.ins_v[::-1][:D].copy()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        d.delete_edges(du, dv)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        print(json.dumps({"config": name, "variant": var, "deletions": D, "ms": ms, "per_s": D / (ms / 1e3)}), flush=True)
