"""Debug helper (test infrastructure): find the first insertion/root where the GPU
state diverges from the oracle on a config workload."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle, workloads as W
from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, FLAG_TIMING

name = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
nins = int(sys.argv[2]) if len(sys.argv) > 2 else 1000
bs = int(sys.argv[3]) if len(sys.argv) > 3 else 1
wl = W.make_workload(name, insertions=nins)
g = wl.graph
dbc = DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING)
dbc.static_compute()
bc = dbc.get_bc()
print("static finite:", np.isfinite(bc).all(), flush=True)
ref_bc = oracle.brandes_csr(g, wl.roots, want_state=False)[0]
print("static bc maxerr", np.max(np.abs(bc - ref_bc) / np.maximum(np.abs(ref_bc), 1)), flush=True)
ref = oracle.NaiveDynamicBC(g, wl.roots)
for i in range(0, nins, bs):
    u, v = wl.ins_u[i:i+bs], wl.ins_v[i:i+bs]
    t0 = time.perf_counter()
    st = dbc.insert_edges(u, v, stats=True)
    bc = dbc.get_bc()
    t1 = time.perf_counter()
    for a, b in zip(u, v):
        ref.insert(a, b)
    tm = dbc.timings()
    if i % 50 == 0 or not np.isfinite(bc).all():
        print(i, st, "wall_ms", (t1-t0)*1e3, "upd_ms", tm["update_ms"], flush=True)
    if not np.isfinite(bc).all():
        print("NaN after insertion batch", i, "edges", list(zip(u.tolist(), v.tolist())), flush=True)
        rp, col = ref.csr()
        _, d_ref, s_ref, dl_ref = oracle.brandes(g.n, rp, col, wl.roots)
        for slot in range(wl.roots.size):
            d, s, dl = dbc.get_root_state(slot)
            okd = np.array_equal(d, d_ref[slot]); oks = np.array_equal(s, s_ref[slot])
            okl = np.all(np.abs(dl - dl_ref[slot]) <= 1e-9 * np.maximum(1, np.abs(dl_ref[slot])))
            if not (okd and oks and okl):
                bad = np.nonzero((d != d_ref[slot]) | (s != s_ref[slot]) | ~(np.abs(dl - dl_ref[slot]) <= 1e-9 * np.maximum(1, np.abs(dl_ref[slot]))))[0]
                print("slot", slot, "root", wl.roots[slot], "d ok", okd, "s ok", oks, "dl ok", okl, "nbad", bad.size, flush=True)
                for x in bad[:8]:
                    print("   v", x, "d", d[x], d_ref[slot][x], "s", s[x], s_ref[slot][x], "dl", dl[x], dl_ref[slot][x], flush=True)
        break
print("done")
