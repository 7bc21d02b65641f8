"""ncu target (diagnostic): Mode S single-insertion launches of the per-insertion
kernel on one config.   python tools/lean_ncu_target.py [config] [insertions]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_ipps_mclaughlinb14_b200 import FLAG_MODE_S, DynamicBC  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "delaunay18"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 20
wl = W.make_workload(name, insertions=N)
g = wl.graph
with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_MODE_S) as dbc:
    dbc.static_compute()
    dbc.insert_edges(wl.ins_u, wl.ins_v)
    dbc.synchronize()
