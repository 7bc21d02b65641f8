"""The C ABI's multi-rank and allocator boundary on the GPU (SURVEY.md Sec. 8(b),
8(e)): dbc_get_bc returns the GLOBAL BC (Eq. (3) over all roots) through
the context's own NCCL communicator or a reduction callback, and device memory
can be routed through the caller's allocator."""

import os
import socket

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _want(wl, roots=None):
    ref = oracle.NaiveDynamicBC(wl.graph, wl.roots if roots is None else roots)
    for u, v in zip(wl.ins_u, wl.ins_v):
        ref.insert(u, v)
    return ref.compute(want_state=False)[0]


def _err(bc, want):
    return float((np.abs(bc - want) / np.maximum(np.abs(want), 1.0)).max())


def test_library_nccl_communicator_world1():
    """opt.nccl_id: the context joins its own NCCL communicator (dbc_create) and
    dbc_get_bc all-reduces the partial with it (one rank on one GPU here; the
    same calls run one rank per GPU on an 8-GPU box)."""
    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, nccl_unique_id

    uid = nccl_unique_id()
    assert len(uid) == 128
    wl = W.make_workload("rmat10")
    with DynamicBC(wl.graph.n, wl.graph.row_ptr, wl.graph.col, wl.roots, nccl_id=uid) as dbc:
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u, wl.ins_v)
        assert _err(dbc.get_bc(), _want(wl)) <= 1e-9
        p1 = dbc.get_bc()
        assert np.array_equal(p1, dbc.get_bc())  # reducing a copy leaves the partial intact


def test_world2_without_reduction_is_rejected():
    from paper_conf_ipps_mclaughlinb14_b200 import DBCError, DynamicBC

    wl = W.make_workload("karate")
    with DynamicBC(wl.graph.n, wl.graph.row_ptr, wl.graph.col, wl.roots, rank=0, world=2) as dbc:
        dbc.static_compute()
        with pytest.raises(DBCError) as e:
            dbc.get_bc()
        assert e.value.name == "DBC_ESTATE"


def test_reduce_callback_failure_is_enccl():
    from paper_conf_ipps_mclaughlinb14_b200 import DBCError, DynamicBC

    wl = W.make_workload("karate")
    with DynamicBC(wl.graph.n, wl.graph.row_ptr, wl.graph.col, wl.roots, rank=0, world=2,
                   reduce=lambda p, n, s: 7) as dbc:
        dbc.static_compute()
        with pytest.raises(DBCError) as e:
            dbc.get_bc()
        assert e.value.name == "DBC_ENCCL"


def _rank_proc(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, torch_reducer

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        wl = W.make_workload(name)
        g = wl.graph
        with DynamicBC(g.n, g.row_ptr, g.col, wl.roots, rank=rank, world=world,
                       reduce=torch_reducer()) as dbc:
            dbc.static_compute()
            half = wl.ins_u.size // 2
            dbc.insert_edges(wl.ins_u[:half], wl.ins_v[:half])
            dbc.insert_edges(wl.ins_u[half:], wl.ins_v[half:])
            bc = dbc.get_bc()  # collective: the global BC on every rank
            part = np.zeros(g.n)
            ptr = dbc.bc_partial_device_ptr()
            dbc.synchronize()
            from paper_conf_ipps_mclaughlinb14_b200.dbc import _wrap_device_f64

            part[:] = _wrap_device_f64(ptr, g.n, 0).cpu().numpy()
        q.put((rank, bc, part))
    except Exception as ex:  # pragma: no cover - reported to the parent
        q.put((rank, repr(ex), None))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["karate", "rmat10", "delaunay12u"])
def test_two_rank_contexts_global_bc_equals_oracle(name):
    """Two processes, ranks 0 and 1 of world 2 (roots slot % 2 == rank) on one
    GPU, each with its own context; dbc_get_bc returns the global BC through the
    reduction callback (gloo over host copies here; NCCL on an 8-GPU box), equal
    to the oracle over ALL roots, and the partials are the oracle's per-rank
    sums."""
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_rank_proc, args=(r, 2, port, name, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = sorted((q.get(timeout=300) for _ in range(2)), key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
    for r, bc, part in outs:
        assert part is not None, bc
    wl = W.make_workload(name)
    want = _want(wl)
    for r, bc, part in outs:
        assert _err(bc, want) <= 1e-9
        assert _err(part, _want(wl, wl.roots[r::2])) <= 1e-9


def test_torch_caching_allocator_hooks():
    """opt.dev_alloc / dev_free: every device buffer of the context comes from
    torch's caching allocator; results unchanged."""
    import torch

    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, torch_allocator

    wl = W.make_workload("rmat10")
    torch.cuda.synchronize()
    before = torch.cuda.memory_allocated(0)
    with DynamicBC(wl.graph.n, wl.graph.row_ptr, wl.graph.col, wl.roots,
                   allocator=torch_allocator(0)) as dbc:
        held = torch.cuda.memory_allocated(0) - before
        assert held >= dbc.device_bytes()
        dbc.static_compute()
        dbc.insert_edges(wl.ins_u, wl.ins_v)
        assert _err(dbc.get_bc(), _want(wl)) <= 1e-9
    torch.cuda.synchronize()
    assert torch.cuda.memory_allocated(0) == before  # everything returned through dev_free
