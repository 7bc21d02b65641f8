"""Batch-kernel tuning sweep (diagnostic): device time of window-merged
batches for dbc_tuning variants.   python tools/tune_sweep.py config batch variants..."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, B = sys.argv[1], int(sys.argv[2])
NB = int(os.environ.get("NB", "12"))
wl = W.make_workload(name, insertions=B * NB)
g = wl.graph
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
u = torch.from_numpy(wl.ins_u).cuda()
v = torch.from_numpy(wl.ins_v).cuda()
for var in sys.argv[3:]:
    tune = {}
    if var != "default":
        for kv in var.split(","):
            k, x = kv.split("=")
            tune[k] = float(x) if k == "heavy_factor" else int(x)
    with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, stream=stream.cuda_stream,
                   tuning=tune or None, edge_capacity=B * NB) as d:
        d.static_compute()
        ms = []
        for b in range(NB):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(stream)
            d.insert_edges(u[b * B:(b + 1) * B], v[b * B:(b + 1) * B])
            e1.record(stream)
            torch.cuda.synchronize()
            if b >= 2:
                ms.append(e0.elapsed_time(e1))
        print(json.dumps({"config": name, "variant": var, "ms_mean": float(np.mean(ms)),
                          "ins_per_s": B / float(np.mean(ms)) * 1e3}), flush=True)
