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
    torchrun --nproc-per-node N bench.py --gpus N ...   (roots sharded slot % N; the
        library's own NCCL communicator all-reduces BC at the end of every batch;
        default config kron20 at N = 2, 4 and kron22 at N = 8)
    python bench.py --impl reference ...                (the CPU oracle arm, same workload)

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
    "delaunay18u": "Delaunay triangulation of 2^18 uniform points, uniform random non-edge insertions (stress)",
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
    p.add_argument("--config", default=None, choices=sorted(W.CONFIGS),
                   help="default: rmat16 (BASELINE configs[1]) on 1 GPU, kron20 (configs[3]) on 2 or 4, "
                        "kron22 (configs[4], 4,096 roots) on 8")
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
                   help="skip the per-insertion side measurements (one job per insertion, Mode S, Table III)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-budget-s", type=float, default=12.0)
    p.add_argument("--side-insertions", type=int, default=1000,
                   help="bound on the insertions of each side measurement")
    p.add_argument("--shard", default="", help="R/N: run rank R's root shard of an N-GPU job on this "
                   "single GPU (per-GPU view of configs that need N GPUs, e.g. kron22 on 8)")
    p.add_argument("--dist-test-one-gpu", action="store_true",
                   help="validation only: every torchrun rank on cuda:0, gloo process group and the "
                        "library's reduce callback instead of NCCL (NCCL refuses two ranks on one GPU)")
    a = p.parse_args()
    if a.config is None:
        world = int(os.environ.get("WORLD_SIZE", str(a.gpus)))
        a.config = "rmat16" if world <= 1 else ("kron22" if world >= 8 else "kron20")
    return a


METRIC = "edge insertions/sec"


def n_batches(args, B):
    """Insertion batches both arms build the workload for (same graph: the
    remove-then-reinsert protocol removes B x n_batches edges)."""
    return args.warmup + args.steps + (0 if args.no_e2e else args.warmup + args.steps)


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


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
        return None if e is None else (float(e["dram_bytes_per_batch"]) / max(launches_per_batch, 1.0),
                                       e.get("sectors_per_request"))
    except Exception:
        return None


# ----------------------------------------------------------- CPU baseline ----
def cpu_baseline(wl, k, budget_s):
    """The oracle as it stands timed on this host (a reported baseline, not the
    target): the naive rule costs one k-root recompute per insertion.  (ii) the
    root-parallel leg on every host core (oracle.brandes_parallel, bit-identical
    to the single-thread oracle) is the value; (i) the single-thread oracle
    ("single-threaded CPU experiments") is reported beside it.  Both on a
    bounded root sample of the same workload, scaled linearly to k."""
    import oracle

    g = wl.graph
    T = oracle.host_threads()
    t0 = time.perf_counter()
    oracle.brandes(g.n, g.row_ptr, g.col, wl.roots[:1], want_state=False)
    t1 = max(time.perf_counter() - t0, 1e-6)
    r = int(max(T, min(k, T * max(1, int((budget_s / 2) / t1)))))  # ~budget/2 of all-core work
    r = min(r, k)
    t0 = time.perf_counter()
    oracle.brandes_parallel(g.n, g.row_ptr, g.col, wl.roots[:r], threads=T)
    tp = time.perf_counter() - t0
    per_ins = tp / r * k
    r1 = int(max(1, min(k, (budget_s / 4) / t1)))
    t0 = time.perf_counter()
    oracle.brandes(g.n, g.row_ptr, g.col, wl.roots[:r1], want_state=False)
    ts = (time.perf_counter() - t0) / r1 * k
    return {"value": 1.0 / per_ins, "unit": "insertions/s", "cores": T, "kind": "oracle",
            "cpu_model": cpu_model(), "nproc": os.cpu_count(),
            "sample": f"naive rule (recompute all k={k} roots per insertion): {r} of {k} roots recomputed "
                      f"root-parallel on {T} threads ({tp / r * 1e3:.2f} ms/root), scaled linearly to k",
            "single_thread": {"value": 1.0 / ts, "cores": 1,
                              "sample": f"{r1} of {k} roots single-threaded ({ts / k * 1e3:.2f} ms/root), "
                                        f"scaled to k"}}


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
    """The reference arm of this tier: the CPU oracle's naive rule (recompute
    every root after each insertion) on the SAME workload our arm builds (same
    config, seed, graph and stream), on every host core.  Each step times one
    insertion's recompute over a bounded root sample and scales linearly to k."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    cfg = W.CONFIGS[args.config]
    B = args.batch or cfg["insertions"]
    k = args.roots or cfg["k"]
    wl = W.make_workload(args.config, seed=args.seed, insertions=B * n_batches(args, B), k=k)
    g = wl.graph
    T = oracle.host_threads()
    t0 = time.perf_counter()
    oracle.brandes(g.n, g.row_ptr, g.col, wl.roots[:1], want_state=False)
    t_root = max(time.perf_counter() - t0, 1e-6)
    r = int(max(1, min(k, T * max(1, int(1.0 / t_root)))))  # ~1 s of all-core work per step
    dyn = oracle.NaiveDynamicBC(g, wl.roots[:r])
    times = []
    for i in range(args.warmup + args.steps):
        dyn.insert(wl.ins_u[i], wl.ins_v[i])
        rp, col = dyn.csr()
        t0 = time.perf_counter()
        oracle.brandes_parallel(g.n, rp, col, wl.roots[:r], threads=T)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    per_ins = (sum(times) / len(times)) * k / r
    value = 1.0 / per_ins
    line = {
        "impl": "reference", "metric": METRIC, "value": value,
        "unit": "insertions/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": per_ins * B * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": args.config, "graph": GRAPH_DESC.get(args.config, args.config),
                   "n": g.n, "m": g.m, "k": k, "batch": B, "seed": args.seed,
                   "protocol": "remove-then-reinsert (P:440)" if cfg["mode"] == "reinsert" else "uniform non-edges",
                   "timing": "host wall clock of the oracle's recompute",
                   "ms_per_step_extrapolated": f"one insertion timed per step on {r} of {k} roots, scaled to k "
                                               f"roots and to the {B}-insertion batch"},
        "cpu_baseline": {"value": value, "unit": "insertions/s", "cores": T, "kind": "oracle",
                         "cpu_model": cpu_model(), "nproc": os.cpu_count(),
                         "sample": f"each step: one naive-rule insertion (recompute) over {r} of {k} roots, "
                                   f"root-parallel on {T} threads, scaled linearly to k"},
        "e2e": {"value": value, "unit": "insertions/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def shared_workload(name, seed, insertions, k, world, rank):
    """The seeded workload; under torchrun rank 0 builds it once and the other
    ranks of the node load its arrays from /tmp (generating Kronecker 22 takes
    ~100 s of host time per process; every rank needs the same replicated graph)."""
    if world == 1:
        return W.make_workload(name, seed=seed, insertions=insertions, k=k)
    import torch.distributed as dist

    tag = os.environ.get("TORCHELASTIC_RUN_ID", "") + os.environ.get("MASTER_PORT", "")
    path = os.path.join("/tmp", f"dbc_wl_{name}_{seed}_{insertions}_{k}_{tag}.npz")
    if rank == 0:
        wl = W.make_workload(name, seed=seed, insertions=insertions, k=k)
        tmp = path + f".{os.getpid()}.npz"
        np.savez(tmp, n=np.int64(wl.graph.n), row_ptr=wl.graph.row_ptr, col=wl.graph.col, roots=wl.roots,
                 ins_u=wl.ins_u, ins_v=wl.ins_v, meta=np.array(json.dumps(wl.meta, default=str)))
        os.replace(tmp, path)
    dist.barrier()
    if rank != 0:
        z = np.load(path)
        g = W.CSR(int(z["n"]), z["row_ptr"], z["col"])
        wl = W.Workload(name, g, z["roots"], z["ins_u"], z["ins_v"], json.loads(str(z["meta"])))
    dist.barrier()
    if rank == 0:
        os.remove(path)
    return wl


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
    nccl_log = None
    one_gpu = args.dist_test_one_gpu
    if world > 1 and one_gpu:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        torch.cuda.set_device(0)
        dist.init_process_group("gloo")
    elif world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        # NCCL's communicator lines (version, transports, NVLS) into a per-rank file
        nccl_log = os.path.join("/tmp", f"dbc_nccl.{os.getpid()}.log")
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", nccl_log)
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    else:
        torch.cuda.set_device(0)
    dev = torch.cuda.current_device()

    from paper_conf_ipps_mclaughlinb14_b200 import (FLAG_MODE_S, FLAG_NO_MERGE, FLAG_TIMING,
                                                    DynamicBC, nccl_unique_id, torch_reducer)

    cfg = W.CONFIGS[args.config]
    B = args.batch or cfg["insertions"]
    k = args.roots or cfg["k"]
    Wm, K = args.warmup, args.steps
    e2e_steps = 0 if args.no_e2e else (Wm + K)
    nb = n_batches(args, B)
    wl = shared_workload(args.config, args.seed, B * nb, k, world, rank)
    g = wl.graph
    flags = FLAG_TIMING | (FLAG_MODE_S if args.mode == "S" else 0) | (FLAG_NO_MERGE if args.no_merge else 0)
    stream = torch.cuda.Stream(device=dev)  # the library and the timing events share it
    torch.cuda.set_stream(stream)
    uid = None
    reducer = torch_reducer() if (world > 1 and one_gpu) else None
    reduction = None
    if world > 1 and not one_gpu:  # the library's own NCCL communicator for the BC all-reduce (opt.nccl_id)
        u0, why = None, None
        if rank == 0:
            try:
                u0 = nccl_unique_id()
            except Exception as ex:  # NCCL not loadable by the library: every rank falls back together
                why = str(ex)
        obj = [(u0, why)]
        dist.broadcast_object_list(obj, src=0)
        uid, why = obj[0]
        if uid is None:
            reducer = torch_reducer()  # torch.distributed's NCCL all-reduce as the reduce callback
            reduction = f"torch.distributed all-reduce callback (library NCCL unavailable: {why})"
        else:
            reduction = "library NCCL communicator (dbc_options.nccl_id)"
    side_ok = world == 1  # side measurements on one GPU only (scaling runs stay short)

    def make(fl):
        return DynamicBC(g.n, g.row_ptr, g.col, wl.roots, device=dev, rank=shard_rank, world=shard_world,
                         workers=args.workers, edge_capacity=B * nb, flags=fl, stream=stream.cuda_stream,
                         nccl_id=uid, reduce=reducer)

    dbc = make(flags)

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if one_gpu else dev)
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

    def step(d, i):
        d.insert_edges(*batch(i))
        if world > 1:  # the end-of-batch BC all-reduce over NVLink, inside T_dev
            d.bc_device_ptr()

    for i in range(Wm):
        step(dbc, i)
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
        step(dbc, i)
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
    gpu_launches = int(tm["kernel_launches_total"])

    # end to end through the public host API: pinned H2D of each batch + D2H of the (global) BC
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
            dbc.get_bc(out=outn)  # global BC (NCCL all-reduce inside at N > 1)
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
                    "sample": f"{Wm} untimed e2e batches (window-merged jobs), this rank's roots"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu = cpu_baseline(wl, k, args.cpu_budget_s)
        except Exception as ex:  # oracle unavailable on this box
            cpu = {"value": None, "unit": "insertions/s", "cores": 1, "kind": "oracle",
                   "sample": f"unavailable: {ex}"}

    S = min(args.side_insertions, B)  # side measurements are bounded

    # side measurement: deletions (decremental update, R20) -- S edges
    # of the last timed batch deleted again (newest first), one job per deletion
    dels = None
    if side_ok and not args.no_deletions:
        D = min(S, 200)
        i = Wm + K - 1
        du, dv = wl.ins_u[i * B:i * B + D][::-1].copy(), wl.ins_v[i * B:i * B + D][::-1].copy()
        torch.cuda.synchronize()
        ev0.record(stream)
        dbc.delete_edges(du, dv)
        ev1.record(stream)
        torch.cuda.synchronize()
        msd = ev0.elapsed_time(ev1)
        dels = {"value": D / (msd / 1e3), "unit": "deletions/s", "deletions": D,
                "what": f"{D} edges of the last timed batch deleted again (newest first), one job per "
                        f"(root, deletion); host-side batch checks inside the timed region"}
    dbc.close()

    # per-insertion side measurements (the paper's structure):
    # one job per (root, insertion) on the same batches, Mode S launches, and
    # Table III's single-edge calls -- all on update_lean.cu
    per_ins = None
    if side_ok and not (args.no_per_insertion or args.no_merge or args.mode == "S"):
        per_ins = {}
        d = make(flags | FLAG_NO_MERGE)
        d.static_compute()
        for i in range(min(Wm, 1)):
            d.insert_edges(*batch(i))
        d.synchronize()
        d.reset_timings()
        i0 = Wm
        torch.cuda.synchronize()
        ev0.record(stream)
        d.insert_edges(ins_u[i0 * B:i0 * B + S], ins_v[i0 * B:i0 * B + S])
        ev1.record(stream)
        torch.cuda.synchronize()
        ms1 = ev0.elapsed_time(ev1)
        t1 = d.timings()
        v1 = S / (ms1 / 1e3)
        l1 = max(t1["update_launches_total"], 1)
        ach1 = (t1["alg_bytes_total"] / l1) / (t1["update_ms_total"] / l1 / 1e3) / 1e9 if t1["update_ms_total"] else 0
        per_ins["jobs"] = {"value": v1, "unit": "insertions/s", "insertions": S,
                           "speedup_vs_static": (static_ms / 1e3) / (ms1 / 1e3 / S),
                           "roofline": {"bound": "hbm", "achieved": ach1, "peak": peak, "unit": "GB/s",
                                        "frac": ach1 / peak, "kernel": "lean_kernel"},
                           "what": "DBC_FLAG_NO_MERGE: one job per (root, insertion), insertions applied one "
                                   "at a time as in P:440, one launch"}
        # Mode S: one launch per insertion over all roots
        NS = min(S, 200)
        i0 = Wm + 1
        dS = make(flags | FLAG_MODE_S)
        dS.static_compute()
        dS.synchronize()
        torch.cuda.synchronize()
        ev0.record(stream)
        dS.insert_edges(ins_u[i0 * B:i0 * B + NS], ins_v[i0 * B:i0 * B + NS])
        ev1.record(stream)
        torch.cuda.synchronize()
        ms2 = ev0.elapsed_time(ev1)
        t2 = dS.timings()
        l2 = max(t2["update_launches_total"], 1)
        ach2 = (t2["alg_bytes_total"] / l2) / (t2["update_ms_total"] / l2 / 1e3) / 1e9 if t2["update_ms_total"] else 0
        per_ins["mode_s"] = {"value": NS / (ms2 / 1e3), "unit": "insertions/s", "insertions": NS,
                             "speedup_vs_static": (static_ms / 1e3) / (ms2 / 1e3 / NS),
                             "launches": int(t2["update_launches_total"]),
                             "roofline": {"bound": "hbm", "achieved": ach2, "peak": peak, "unit": "GB/s",
                                          "frac": ach2 / peak, "kernel": "lean_kernel"},
                             "what": "Mode S: one per-insertion kernel launch over all roots per insertion "
                                     "(P:244-252)"}
        dS.close()
        # Table III: single-edge calls, device time of each call's update
        NT = min(S, 60)
        per = []
        for j in range(NT + 3):
            idx = (Wm + 2) * B + j
            d.insert_edges(ins_u[idx:idx + 1], ins_v[idx:idx + 1])
            if j >= 3:
                per.append(d.timings()["update_ms"])
        per = np.array(per)
        per_ins["table3"] = {"calls": NT, "static_ms": static_ms, "fastest_ms": float(per.min()),
                             "average_ms": float(per.mean()), "slowest_ms": float(per.max()),
                             "speedup_average": static_ms / float(per.mean()),
                             "speedup_slowest": static_ms / float(per.max()),
                             "speedup_fastest": static_ms / float(per.min()),
                             "what": "device time of the update of single-edge dbc_insert_edges calls (graph "
                                     "update neglected as in P:440) vs one static recompute over the same roots "
                                     "(Table III, P:482-514)"}
        d.close()

    cpu_dyn = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu_dyn = cpu_dynamic(wl, k, args.cpu_budget_s)
            ref_v = per_ins["jobs"]["value"] if per_ins else value
            cpu_dyn["gpu_speedup_per_insertion"] = ref_v / cpu_dyn["value"]
            cpu_dyn["gpu_speedup_merged"] = value / cpu_dyn["value"]
            cpu_dyn["paper"] = "110x max GPU-over-CPU dynamic on a GTX-class GPU (P:444-478), context only"
        except Exception as ex:
            cpu_dyn = {"value": None, "kind": "cpu_dynamic_alg2", "sample": f"unavailable: {ex}"}

    nccl = None
    if nccl_log and rank == 0:
        try:
            with open(nccl_log) as f:
                lines = [ln.strip() for ln in f if ("NCCL version" in ln or "NVLS" in ln or "comm " in ln
                                                      or "Init COMPLETE" in ln)]
            nccl = {"log": nccl_log, "lines": lines[:8], "bc_reduction": reduction}
        except OSError:
            nccl = {"log": nccl_log, "lines": [], "bc_reduction": reduction}

    # the committed capture is of one whole-root-set batch: only comparable at one rank
    traffic = ncu_traffic(args.config, B, args.mode, launches / K) if shard_world == 1 else None
    state_mb = 24.0 * k * g.n / shard_world / 1e6
    line = {
        "metric": METRIC,
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
            "dist_test_one_gpu": (f"{world} ranks on cuda:0 over gloo + the reduce callback: validates the "
                                  f"multi-rank path, not a scaling number") if one_gpu else None,
            "graph": GRAPH_DESC.get(args.config, args.config),
            "n": g.n, "m": g.m, "k": k, "batch": B, "mode": args.mode, "seed": args.seed,
            "protocol": "remove-then-reinsert (P:440)" if cfg["mode"] == "reinsert" else "uniform non-edges",
            "timing": "device (CUDA events on the library stream), max over ranks"
                      + ("; the end-of-batch BC all-reduce inside" if world > 1 else ""),
            "l2": f"inputs larger than L2: per-GPU d/sigma/delta state {state_mb:.0f} MB vs 126 MB L2",
            "static_recompute_ms": static_ms,
            "shard": (f"rank {shard_rank} of {shard_world} (roots slot % {shard_world} == {shard_rank}) "
                      f"on one GPU" if args.shard else None),
            "speedup_vs_static": (static_ms / 1e3) / per_ins_s,
            "us_per_insertion": per_ins_s * 1e6,
            "case_mix": case_mix,
            "merge": ("one job per (root, insertion)" if args.no_merge or args.mode == "S" else
                      "window-merged: one job per root per window of insertions (DESIGN.md R18)"),
            "per_insertion": per_ins,
            "deletions": dels,
            "nccl": nccl,
        },
        "roofline": {
            "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": traffic[0] if traffic else None,
            "dram_GBps": (traffic[0] / (launch_ms / 1e3) / 1e9) if traffic and launch_ms > 0 else None,
            "sectors_per_request": traffic[1] if traffic else None,
            "traffic_source": "committed ncu --set full capture of this config's batch (profiles/ncu_traffic.json)"
                              if traffic else None,
            "kernel": "update_kernel", "peak_source": peak_src,
            "alg_bytes_per_launch": bytes_per_launch, "launch_ms": launch_ms,
            "byte_model": "SURVEY.md Sec. 8(d), counted per event in the kernel",
            "share_of_step": upd_ms / ms if ms > 0 else None,
            "static_kernel_GBps": (static_bytes / (static_ms / 1e3) / 1e9) if static_ms > 0 else None,
        },
        "cpu_baseline": cpu,
        "cpu_dynamic": cpu_dyn,
        "e2e": e2e,
        "gpu_launches": gpu_launches,
        "clocks": clk,
    }
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
