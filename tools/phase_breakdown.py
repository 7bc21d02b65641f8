import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, workloads as W
from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, FLAG_TIMING
name = sys.argv[1] if len(sys.argv) > 1 else "rmat16"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 1000
wl = W.make_workload(name, insertions=B, k=int(sys.argv[3]) if len(sys.argv) > 3 and int(sys.argv[3]) > 0 else None)
if len(sys.argv) > 4:  # explicit root list, e.g. 650960,3614
    wl.roots = np.array([int(x) for x in sys.argv[4].split(",")], dtype=np.int32)
g = wl.graph
tr = os.environ.get("DBC_TRACE_SLOT")  # traced root slot (dbc_tuning.trace_slot; -DDBC_PHASE_TIMERS builds)
dbc = DynamicBC(g.n, g.row_ptr, g.col, wl.roots, flags=FLAG_TIMING,
                tuning={"trace_slot": int(tr)} if tr else None)
dbc.static_compute(); dbc.synchronize()
c0 = dbc.debug_counters()
dbc.root_profile(True, read=False)
nb = int(os.environ.get("PB_BATCHES", "1"))
bs = len(wl.ins_u) // nb
for b in range(nb):
    if b == nb - 1:
        c0 = dbc.debug_counters()
    dbc.insert_edges(wl.ins_u[b * bs:(b + 1) * bs], wl.ins_v[b * bs:(b + 1) * bs])
c1 = dbc.debug_counters()
d = {k: c1[k] - c0[k] for k in c1}
print(d)
work = d["case2"] + d["case3"]
print("per working job:", {k: round(v / max(work, 1), 1) for k, v in d.items() if k.startswith("sc_") or k.startswith("ns_") or k.startswith("levels") or k in ("touched", "down", "scanned")})
print("roots deg: median", np.median(g.degree()[wl.roots]), "mean", g.degree()[wl.roots].mean())
print(dbc.timings())
prof = dbc.root_profile(True)
dur = (prof[:, 1] - prof[:, 0]) / 1e6
print("root chain ms: min %.2f median %.2f p90 %.2f max %.2f; kernel span %.2f" % (dur.min(), np.median(dur), np.percentile(dur, 90), dur.max(), (prof[:,1].max()-prof[:,0].min())/1e6))
order = np.argsort(-dur)[:8]
for i in order:
    print("slot", i, "root", wl.roots[i], "deg", g.degree()[wl.roots[i]], "ms %.2f" % dur[i], "jobs", prof[i,2], "touched/job", prof[i,3]//max(prof[i,2],1), "scanned/job", prof[i,4]//max(prof[i,2],1), "levels/job %.1f" % (prof[i,5]/max(prof[i,2],1)), "us/job %.1f" % (dur[i]*1e3/max(prof[i,2],1)), "start %.2f" % ((prof[i,0]-prof[:,0].min())/1e6))
med = np.argsort(dur)[len(dur)//2]
i = med
print("median root: slot", i, "deg", g.degree()[wl.roots[i]], "ms %.2f" % dur[i], "jobs", prof[i,2], "touched/job", prof[i,3]//max(prof[i,2],1), "scanned/job", prof[i,4]//max(prof[i,2],1), "levels/job %.1f" % (prof[i,5]/max(prof[i,2],1)), "us/job %.1f" % (dur[i]*1e3/max(prof[i,2],1)))
print("jobs: median", np.median(prof[:,2]), "max", prof[:,2].max(), "touched/job median", np.median(prof[:,3]/np.maximum(prof[:,2],1)))
st = (prof[:, 0] - prof[:, 0].min()) / 1e6
print("root start ms: min %.2f median %.2f max %.2f; #late(>1ms) %d" % (st.min(), np.median(st), st.max(), (st > 1).sum()))
if os.environ.get("DBC_TRACE_SLOT"):
    ev = dbc.debug_trace()
    t0 = None
    last = None
    for kind, lev, items, t in ev:
        if t0 is None:
            t0 = t
        dt = (t - last) / 1e3 if last is not None else 0.0
        print("trace +%8.1f us (at %8.1f) %s level %d items %d%s" % (dt, (t - t0) / 1e3, {1: "down", 2: "up", 3: "removal", 4: "job-end", 6: "owner-blocks(kind; own|total<<16)", 9: "long-rows(rows; entries)", 10: " chunk-split(long rows)", 11: " C1(entries)", 12: " C2(entries)", 13: " C3(l1 rows)", 14: " epilogue(rows)"}.get(kind, "?"), lev, items, (" own %d of %d" % (items & 0xFFFF, items >> 16)) if kind == 6 else ""))
        last = t
