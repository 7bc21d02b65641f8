"""Multi-rank host logic on CPU (gloo, world size 2): the root sharding used by
the library (slot % world == rank) plus a sum all-reduce of
per-rank BC partials reproduces the single-rank BC (Eq. (3) is a sum over
roots).  Per-rank partials here come from the oracle (test infrastructure); the
GPU path's per-rank partials are checked against each other in
test_gpu_parity.py::test_fake_multi_gpu_shards_sum_to_single."""

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W
from paper_conf_ipps_mclaughlinb14_b200.dbc import local_slots


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    wl = W.make_workload(name)
    slots = local_slots(wl.roots.size, rank, world)
    dyn = oracle.NaiveDynamicBC(wl.graph, wl.roots[slots])
    for u, v in zip(wl.ins_u, wl.ins_v):
        dyn.insert(u, v)
    part = dyn.compute(want_state=False)[0]
    t = torch.from_numpy(part.copy())
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    if rank == 0:
        q.put((slots, t.numpy().copy()))
    else:
        q.put((slots, None))
    dist.destroy_process_group()


@pytest.mark.parametrize("name", ["karate", "rmat10"])
def test_gloo_world2_shards_and_allreduce(name):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    slots = sorted(sum((o[0] for o in outs), []))
    wl = W.make_workload(name)
    assert slots == list(range(wl.roots.size))  # every slot owned exactly once
    red = [o[1] for o in outs if o[1] is not None][0]
    dyn = oracle.NaiveDynamicBC(wl.graph, wl.roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        dyn.insert(u, v)
    full = dyn.compute(want_state=False)[0]
    np.testing.assert_allclose(red, full, rtol=1e-12, atol=1e-12)


def test_local_slots_partition():
    for k in (0, 1, 5, 34, 256):
        for world in (1, 2, 3, 8):
            got = sorted(s for r in range(world) for s in local_slots(k, r, world))
            assert got == list(range(k))
