#!/usr/bin/env python
"""bench.py -- edge insertions/s (device-timed) of the B200 dynamic-BC update.

Metric (BASELINE.json): "edge insertions/sec (device-timed), speedup vs static
GPU Brandes recompute".  One step = one batch of B edge insertions through the
whole hot path (validation + append, classification, down phase, up phase, BC
update: SURVEY.md Sec. 8(a) A0-A4) on synthetic inputs of the BASELINE config,
following the paper's protocol: edges are removed from the
generated graph, the static state is built, and the removed edges are
reinserted one at a time, B per batch.

    python bench.py [--gpus N --steps K --warmup W --config rmat16 --batch 1000]
    torchrun --nproc-per-node N bench.py --gpus N ...   (roots sharded slot % N)
    python bench.py --impl reference ...                (the CPU oracle arm)

Prints ONE JSON line on rank 0.
"""

from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

GRAPH_DESC = {
    "karate": "Zachary karate club (34 vertices, 78 edges)",
    "rmat16": "R-MAT/Graph500 Kronecker scale 16 edgefactor 8 (A,B,C=.57,.19,.19), undirected",
    "delaunay18": "Delaunay triangulation of 2^18 uniform points",
    "kron20": "Kronecker scale 20 edgefactor 16",
    "kron22": "Kronecker scale 22 edgefactor 16",
    "smallworld": "Watts-Strogatz n=100000 k=10 p=0.1",
}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="rmat16", choices=sorted(W.CONFIGS))
    p.add_argument("--batch", type=int, default=0, help="insertions per step (default: the config's)")
    p.add_argument("--roots", type=int, default=0, help="override k")
    p.add_argument("--mode", default="A", choices=["A", "S"])
    p.add_argument("--seed", type=int, default=1)
    p.add_argument("--workers", type=int, default=0)
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-merge", action="store_true",
                   help="headline run with DBC_FLAG_NO_MERGE (one job per (root, insertion))")
    p.add_argument("--no-deletions", action="store_true", help="skip the edge-deletion side measurement")
    p.add_argument("--no-per-insertion", action="store_true",
                   help="skip the side measurement with DBC_FLAG_NO_MERGE")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-budget-s", type=float, default=12.0)
    p.add_argument("--shard", default="", help="R/N: run rank R's root shard of an N-GPU job on this "
                   "single GPU (per-GPU view of configs that need N GPUs, e.g. kron22 on 8)")
    return p.parse_args()


# ----------------------------------------------------------------- clocks ----
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) != 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, val in zip(names, parts[2:]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic(config, batch, mode, launches_per_batch):
    """dram bytes per update-kernel launch from the committed ncu capture, if any
    (the capture holds one batch's update in ONE launch; the timed run may split
    it over the heavy and normal lanes, so it is divided like the algorithmic bytes)."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            t = json.load(f)
        e = t.get(f"{config}/b{batch}/{mode}")
        return None if e is None else float(e["dram_bytes_per_batch"]) / max(launches_per_batch, 1.0)
    except Exception:
        return None


# ----------------------------------------------------------- CPU baseline ----
def cpu_baseline(wl, k, budget_s):
    """The oracle as it stands (single thread): the naive rule costs one k-root
    recompute per insertion; time it on a bounded root sample and scale to k."""
    import oracle

    g = wl.graph
    r = 1
    t_root = None
    while True:
        roots = wl.roots[:r]
        t0 = time.perf_counter()
        oracle.brandes(g.n, g.row_ptr, g.col, roots, want_state=False)
        dt = time.perf_counter() - t0
        t_root = dt / r
        if dt > budget_s / 3 or r >= k:
            break
        r = min(k, max(r * 2, int(r * (budget_s / 3) / max(dt, 1e-6))))
    per_ins = t_root * k
    return {"value": 1.0 / per_ins, "unit": "insertions/s", "cores": 1, "kind": "oracle",
            "sample": f"naive rule (recompute all k={k} roots per insertion): {r} of {k} roots "
                      f"recomputed single-threaded, {t_root * 1e3:.2f} ms/root, scaled linearly to k"}


def cpu_dynamic(wl, k, budget_s):
    """The paper's CPU comparison (dynamic sequential Alg. 2 + Case 3, one
    thread, oracle/cpu_dynamic.c; Table II "CPU"): a bounded sample of
    roots and insertions of the same stream, scaled linearly to k roots."""
    import oracle

    g = wl.graph
    t0 = time.perf_counter()
    oracle.brandes(g.n, g.row_ptr, g.col, wl.roots[:1], want_state=False)
    t_root = max(time.perf_counter() - t0, 1e-6)
    r = int(max(1, min(k, (budget_s / 3) / t_root)))  # initial state ~ budget/3
    cd = oracle.CpuDynamicBC(g, wl.roots[:r])
    t_sum, done = 0.0, 0
    while done < wl.ins_u.size and (t_sum < budget_s / 2 or done < 3):
        t0 = time.perf_counter()
        cd.insert(wl.ins_u[done], wl.ins_v[done])
        t_sum += time.perf_counter() - t0
        done += 1
    cd.close()
    per_ins = t_sum / done * k / r
    return {"value": 1.0 / per_ins, "unit": "insertions/s", "cores": 1, "kind": "cpu_dynamic_alg2",
            "sample": f"dynamic CPU algorithm (Alg. 2 + Case 3, O(n) init per update as in P:254-268), "
                      f"first {done} insertions of the stream on {r} of {k} roots, single thread, "
                      f"scaled linearly to k"}


# -------------------------------------------------------------- reference ----
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    cfg = W.CONFIGS[args.config]
    B = args.batch or cfg["insertions"]
    k = args.roots or cfg["k"]
    steps = args.warmup + args.steps
    wl = W.make_workload(args.config, seed=args.seed, insertions=max(steps, 1), k=k)
    g = wl.graph
    # bounded sample: r roots per naive-rule insertion, ~1-2 s per step
    t0 = time.perf_counter()
    oracle.brandes(g.n, g.row_ptr, g.col, wl.roots[:1], want_state=False)
    t_root = max(time.perf_counter() - t0, 1e-6)
    r = int(max(1, min(k, 1.5 / t_root)))
    dyn = oracle.NaiveDynamicBC(g, wl.roots[:r])
    times = []
    for i in range(steps):
        dyn.insert(wl.ins_u[i], wl.ins_v[i])
        t0 = time.perf_counter()
        dyn.compute(want_state=False)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    per_ins = (sum(times) / len(times)) * k / r
    value = 1.0 / per_ins
    line = {
        "impl": "reference", "metric": "edge insertions/sec", "value": value,
        "unit": "insertions/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": per_ins * B * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": args.config, "graph": GRAPH_DESC.get(args.config, args.config),
                   "n": g.n, "m": g.m, "k": k, "batch": B, "seed": args.seed},
        "cpu_baseline": {"value": value, "unit": "insertions/s", "cores": 1, "kind": "oracle",
                         "sample": f"each step: one naive-rule insertion (recompute) over {r} of {k} "
                                   f"roots, single thread, scaled linearly to k"},
        "e2e": {"value": value, "unit": "insertions/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# -------------------------------------------------------------------- ours ----
def run_ours(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    shard_rank, shard_world = rank, world
    if args.shard:
        if world > 1:
            raise SystemExit("--shard emulates one rank on one GPU; do not combine with torchrun")
        shard_rank, shard_world = (int(x) for x in args.shard.split("/"))
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()

    from paper_conf_ipps_mclaughlinb14_b200 import (FLAG_MODE_S, FLAG_NO_MERGE, FLAG_TIMING,
                                                    DynamicBC, allreduce_bc)

    cfg = W.CONFIGS[args.config]
    B = args.batch or cfg["insertions"]
    k = args.roots or cfg["k"]
    Wm, K = args.warmup, args.steps
    e2e_steps = 0 if args.no_e2e else (Wm + K)
    nb = Wm + K + e2e_steps
    wl = W.make_workload(args.config, seed=args.seed, insertions=B * nb, k=k)
    g = wl.graph
    flags = FLAG_TIMING | (FLAG_MODE_S if args.mode == "S" else 0) | (FLAG_NO_MERGE if args.no_merge else 0)
    stream = torch.cuda.Stream(device=dev)  # the library and the timing events share it
    torch.cuda.set_stream(stream)
    dbc = DynamicBC(g.n, g.row_ptr, g.col, wl.roots, device=dev, rank=shard_rank, world=shard_world,
                    workers=args.workers, edge_capacity=B * nb, flags=flags,
                    stream=stream.cuda_stream)

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def barrier():
        if world > 1:
            dist.barrier()

    # initial state + the static recompute baseline (same roots, same GPU count)
    dbc.static_compute()
    dbc.synchronize()
    dbc.static_compute()
    tm = dbc.timings()
    static_ms = max_over_ranks(tm["static_ms"])
    static_bytes = tm["static_alg_bytes"]

    ins_u = torch.from_numpy(wl.ins_u).to(dev)
    ins_v = torch.from_numpy(wl.ins_v).to(dev)

    def batch(i):
        return ins_u[i * B:(i + 1) * B], ins_v[i * B:(i + 1) * B]

    for i in range(Wm):
        dbc.insert_edges(*batch(i))
    dbc.synchronize()
    dbc.reset_timings()

    clocks = ClockSampler(dev)
    clocks.start()
    barrier()
    torch.cuda.synchronize()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    for i in range(Wm, Wm + K):
        dbc.insert_edges(*batch(i))
    ev1.record(stream)
    torch.cuda.synchronize()
    barrier()
    clk = clocks.stop()
    ms = max_over_ranks(ev0.elapsed_time(ev1))
    tm = dbc.timings()

    value = K * B / (ms / 1e3)
    per_ins_s = ms / 1e3 / (K * B)
    upd_ms = tm["update_ms_total"]
    launches = max(tm["update_launches_total"], 1)
    bytes_per_launch = tm["alg_bytes_total"] / launches
    launch_ms = upd_ms / launches
    achieved = bytes_per_launch / (launch_ms / 1e3) / 1e9 if launch_ms > 0 else 0.0
    peak, peak_src = hbm_peak()

    # end to end through the public host API: pinned H2D of each batch + D2H of BC
    e2e = None
    case_mix = None
    if e2e_steps:
        hu = torch.from_numpy(wl.ins_u).pin_memory()
        hv = torch.from_numpy(wl.ins_v).pin_memory()
        out = torch.empty(g.n, dtype=torch.float64).pin_memory()
        outn = out.numpy()
        base = Wm + K
        tot = {"case1": 0, "case2": 0, "case3": 0, "touched": 0, "edges_scanned": 0}
        t_e2e = 0.0
        for j in range(e2e_steps):
            i = base + j
            u = hu[i * B:(i + 1) * B].numpy()
            v = hv[i * B:(i + 1) * B].numpy()
            barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = dbc.insert_edges(u, v, stats=(j < Wm))
            if world > 1:
                outn[:] = allreduce_bc(dbc)
            else:
                dbc.get_bc(out=outn)
            dt = time.perf_counter() - t0
            if j >= Wm:
                t_e2e += dt
            else:
                for kk in tot:
                    tot[kk] += st[kk]
        t_e2e = max_over_ranks(t_e2e)
        e2e = {"value": K * B / t_e2e, "unit": "insertions/s", "h2d_bytes_per_step": 8 * B,
               "d2h_bytes_per_step": 8 * g.n}
        ncase = max(tot["case1"] + tot["case2"] + tot["case3"], 1)
        case_mix = {"case1": tot["case1"] / ncase, "case2": tot["case2"] / ncase,
                    "case3": tot["case3"] / ncase,
                    "touched_per_working_root": tot["touched"] / max(tot["case2"] + tot["case3"], 1),
                    "scanned_per_working_root": tot["edges_scanned"] / max(tot["case2"] + tot["case3"], 1),
                    "sample": f"{Wm} untimed e2e batches, this rank's roots"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu = cpu_baseline(wl, k, args.cpu_budget_s)
        except Exception as ex:  # oracle unavailable on this box
            cpu = {"value": None, "unit": "insertions/s", "cores": 1, "kind": "oracle",
                   "sample": f"unavailable: {ex}"}

    # side measurement: deletions (decremental update, R20) -- the
    # edges of the timed batches deleted again, B per step, one job per deletion
    dels = None
    if not args.no_deletions:
        barrier()
        torch.cuda.synchronize()
        ev0.record(stream)
        for i in range(Wm + K - 1, Wm - 1, -1):
            dbc.delete_edges(wl.ins_u[i * B:(i + 1) * B], wl.ins_v[i * B:(i + 1) * B])
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
        msd = max_over_ranks(ev0.elapsed_time(ev1))
        dels = {"value": K * B / (msd / 1e3), "unit": "deletions/s", "ms_per_step": msd / K,
                "what": "the K timed batches deleted again (B per step, newest first), one job per "
                        "(root, deletion); host-side batch checks inside the timed region"}

    # side measurement: the same batches with one job per (root, insertion)
    # (DBC_FLAG_NO_MERGE: the paper's one-insertion-at-a-time structure)
    per_ins = None
    if not (args.no_per_insertion or args.no_merge or args.mode == "S"):
        dbc.close()
        dbc = DynamicBC(g.n, g.row_ptr, g.col, wl.roots, device=dev, rank=shard_rank,
                        world=shard_world, workers=args.workers, edge_capacity=B * nb,
                        flags=flags | FLAG_NO_MERGE, stream=stream.cuda_stream)
        dbc.static_compute()
        for i in range(Wm):
            dbc.insert_edges(*batch(i))
        barrier()
        torch.cuda.synchronize()
        ev0.record(stream)
        for i in range(Wm, Wm + K):
            dbc.insert_edges(*batch(i))
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ms1 = max_over_ranks(ev0.elapsed_time(ev1))
        per_ins = {"value": K * B / (ms1 / 1e3), "unit": "insertions/s", "ms_per_step": ms1 / K,
                   "speedup_vs_static": (static_ms / 1e3) / (ms1 / 1e3 / (K * B)),
                   "what": "same batches, DBC_FLAG_NO_MERGE: one job per (root, insertion), "
                           "insertions applied one at a time as in P:440"}

    cpu_dyn = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu_dyn = cpu_dynamic(wl, k, args.cpu_budget_s)
            cpu_dyn["gpu_speedup"] = value / cpu_dyn["value"]
            cpu_dyn["paper"] = "110x max GPU-over-CPU dynamic on a GTX-class GPU (P:444-478), context only"
        except Exception as ex:
            cpu_dyn = {"value": None, "kind": "cpu_dynamic_alg2", "sample": f"unavailable: {ex}"}

    state_mb = 24.0 * k * g.n / shard_world / 1e6
    line = {
        "metric": "edge insertions/sec (device-timed)",
        "value": value,
        "unit": "insertions/s",
        "n_gpus": world,
        "steps": K,
        "warmup": Wm,
        "ms_per_step": ms / K,
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": "f64",
        "data": "synthetic",
        "config": {
            "workload": args.config,
            "graph": GRAPH_DESC.get(args.config, args.config),
            "n": g.n, "m": g.m, "k": k, "batch": B, "mode": args.mode, "seed": args.seed,
            "protocol": "remove-then-reinsert (P:440)" if cfg["mode"] == "reinsert" else "uniform non-edges",
            "l2": f"inputs larger than L2: per-GPU d/sigma/delta state {state_mb:.0f} MB vs 126 MB L2",
            "static_recompute_ms": static_ms,
            "shard": (f"rank {shard_rank} of {shard_world} (roots slot % {shard_world} == {shard_rank}) "
                      f"on one GPU" if args.shard else None),
            "speedup_vs_static": (static_ms / 1e3) / per_ins_s,
            "us_per_insertion": per_ins_s * 1e6,
            "case_mix": case_mix,
            "merge": ("one job per (root, insertion)" if args.no_merge or args.mode == "S" else
                      "window-merged: one job per root per window of insertions (DESIGN.md R18)"),
            "per_insertion_jobs": per_ins,
            "deletions": dels,
        },
        "roofline": {
            "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": ncu_traffic(args.config, B, args.mode, launches / K),
            "kernel": "update_kernel", "peak_source": peak_src,
            "alg_bytes_per_launch": bytes_per_launch, "launch_ms": launch_ms,
            "share_of_step": upd_ms / ms if ms > 0 else None,
            "static_kernel_GBps": (static_bytes / (static_ms / 1e3) / 1e9) if static_ms > 0 else None,
        },
        "cpu_baseline": cpu,
        "cpu_dynamic": cpu_dyn,
        "e2e": e2e,
        "gpu_launches": int(tm["kernel_launches_total"]),
        "clocks": clk,
    }
    dbc.close()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
