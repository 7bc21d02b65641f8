"""Step clocks inside the up passes of one traced root (diagnostic; needs a
libdbc built with -DDBC_LEAN_PTRACE, loaded through DBC_LIB_PATH)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_TIMING, DynamicBC  # noqa: E402

name, slot, N = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
wl = W.make_workload(name, insertions=N)
g = wl.graph
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING, tuning={"trace_slot": slot}) as d:
    d.static_compute()
    base = 34  # kStTraceN; the trace area follows
    out0 = np.zeros(base + 1 + 8, np.int64)
    d._lib.dbc_debug_counters(d._ctx, out0.ctypes.data_as(__import__("ctypes").c_void_p), out0.size)
    for i in range(N):
        d.insert_edges(wl.ins_u[i:i + 1], wl.ins_v[i:i + 1])
    out = np.zeros(base + 1 + 8, np.int64)
    d._lib.dbc_debug_counters(d._ctx, out.ctypes.data_as(__import__("ctypes").c_void_p), out.size)
t = (out - out0)[base + 1:base + 7]
n = max(int(t[5]), 1)
print(json.dumps({"passes": n, "cycles_per_pass": {"rows+cols": t[0] / n, "gathers issued": t[1] / n,
                  "visit (waits on gathers)": t[2] / n, "claims+appends": t[3] / n, "barrier": t[4] / n}}))
