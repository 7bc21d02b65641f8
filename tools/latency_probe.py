"""Per-insertion latency probe (diagnostic): one-job-per-insertion batches,
Mode S launches and single-edge calls on one config, for several launch
configurations (variants: comma-separated dbc_tuning fields, e.g.
lean_block=512,disable=8; "default" = automatic).

    python tools/latency_probe.py [config] [variants...]   -> JSON lines
"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import (FLAG_MODE_S, FLAG_NO_MERGE, FLAG_TIMING,  # noqa: E402
                                                DynamicBC)
import torch  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
variants = sys.argv[2:] or ["default"]
NB, NS, N1 = 1000, 100, 60
wl = W.make_workload(name, insertions=NB + NS + N1 + 200)
g = wl.graph
print(json.dumps({"config": name, "n": g.n, "m": g.m, "k": int(wl.roots.size)}), flush=True)
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)


def ctx(flags, tuning):
    d = DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=flags | FLAG_TIMING, stream=stream.cuda_stream,
                  edge_capacity=NB + NS + N1 + 200, tuning=tuning or None)
    d.static_compute()
    d.synchronize()
    return d


def dev_time(fn):
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    fn()
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


for var in variants:
    env = {}  # dbc_tuning fields, e.g. lean_block=512,disable=8
    if var != "default":
        for kv in var.split(","):
            k, v = kv.split("=")
            env[k] = float(v) if k == "heavy_factor" else int(v)
    res = {"variant": var}
    u, v = wl.ins_u, wl.ins_v
    # one job per (root, insertion): 100 warm-up + a 1000 batch
    d = ctx(FLAG_NO_MERGE, env)
    d.insert_edges(u[NB:NB + 100], v[NB:NB + 100])
    ms = dev_time(lambda: d.insert_edges(u[:NB], v[:NB]))
    res["nomerge_ins_per_s"] = NB / ms * 1e3
    d.close()
    # Mode S
    d = ctx(FLAG_MODE_S, env)
    d.insert_edges(u[NB:NB + 10], v[NB:NB + 10])
    ms = dev_time(lambda: d.insert_edges(u[NB + 10:NB + 10 + NS], v[NB + 10:NB + 10 + NS]))
    res["modeS_ins_per_s"] = NS / ms * 1e3
    d.close()
    # single-edge calls (default merge mode; one insertion = one job per root)
    d = ctx(0, env)
    wall, upd, app = [], [], []
    base = NB + NS + 20
    for i in range(N1 + 5):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        d.insert_edges(u[base + i:base + i + 1], v[base + i:base + i + 1])
        d.synchronize()
        dt = time.perf_counter() - t0
        t = d.timings()
        if i >= 5:
            wall.append(dt * 1e3)
            upd.append(t["update_ms"])
            app.append(t["append_ms"])
    res["single_wall_ms"] = [float(np.mean(wall)), float(np.min(wall)), float(np.max(wall))]
    res["single_update_ms"] = [float(np.mean(upd)), float(np.min(upd)), float(np.max(upd))]
    res["single_append_ms"] = [float(np.mean(app)), float(np.min(app)), float(np.max(app))]
    d.close()
    print(json.dumps(res), flush=True)
