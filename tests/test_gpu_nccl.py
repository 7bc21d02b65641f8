"""The multi-GPU exchange path on one GPU: a single-rank NCCL process group runs
the same all-reduce of the device BC partial that N ranks run (A5)."""

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


def test_nccl_allreduce_path_single_rank():
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_mclaughlinb14_b200 import DynamicBC, allreduce_bc

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(_port())
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        wl = W.make_workload("rmat10")
        with DynamicBC(wl.graph.n, wl.graph.row_ptr, wl.graph.col, wl.roots) as dbc:
            dbc.static_compute()
            dbc.insert_edges(wl.ins_u, wl.ins_v)
            bc = allreduce_bc(dbc, force=True)
            ref = oracle.NaiveDynamicBC(wl.graph, wl.roots)
            for u, v in zip(wl.ins_u, wl.ins_v):
                ref.insert(u, v)
            want = ref.compute(want_state=False)[0]
            err = np.abs(bc - want) / np.maximum(np.abs(want), 1.0)
            assert err.max() <= 1e-9
            # the library's partial is untouched by the reduction (a copy is reduced)
            assert np.array_equal(dbc.get_bc(), bc)
    finally:
        dist.destroy_process_group()
