"""Summarise ncu captures into profiles/ (raw metrics of interest + launch-list shares)."""
import csv, io, json, subprocess, sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__cycles_active.avg.pct_of_peak_sustained_elapsed",
        "launch__shared_mem_per_block_static", "sm__maximum_warps_per_active_cycle_pct"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for k in KEYS:
        if k in h:
            i = h.index(k)
            d[k] = {"value": vals[i], "unit": units[i]}
    d["kernel"] = vals[h.index("Kernel Name")] if "Kernel Name" in h else "?"
    return d


def launches(path):
    rows = list(csv.reader(open(path)))
    for i, r in enumerate(rows):
        if r and r[0] == "ID":
            h = r
            start = i
            break
    ix = {k: j for j, k in enumerate(h)}
    agg = {}
    for r in rows[start + 1:]:
        name = r[ix["Kernel Name"]].split("(")[0]
        ns = float(r[ix["Metric Value"]].replace(",", ""))
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += ns
    tot = sum(v[1] for v in agg.values())
    return {k: {"launches": v[0], "total_ms": v[1] / 1e6, "share": v[1] / tot} for k, v in
            sorted(agg.items(), key=lambda kv: -kv[1][1])}


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "raw":
        print(json.dumps(raw(sys.argv[2]), indent=1))
    else:
        print(json.dumps(launches(sys.argv[2]), indent=1))
