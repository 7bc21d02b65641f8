"""Thin ctypes binding of libdbc.so (include/dbc.h) -- argument marshalling only.

Every step of the method runs in the library's CUDA kernels; this module never
computes BC, d, sigma or delta itself and has no CPU fallback: if the compiled
library is missing it raises.  PyTorch supplies the CUDA stream (and, for
multi-GPU, the process group); numpy arrays are host buffers, torch CUDA
tensors are device buffers.
"""

from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DBC_LIB_PATH") or os.path.join(_HERE, "libdbc.so")

DBC_INF = 2**31 - 1
FLAG_MODE_S = 0x1
FLAG_TIMING = 0x2
FLAG_EXACT_BC = 0x4
FLAG_NO_REORDER = 0x8
FLAG_NO_MERGE = 0x10
FLAG_EDGE_PARALLEL = 0x20
FLAG_PULL_DELTA = 0x40
TUNE_NO_HELP, TUNE_NO_HEAVY, TUNE_NO_LEAN, TUNE_NO_LEAN_HELP, TUNE_NO_LOWDEG = 0x1, 0x2, 0x4, 0x8, 0x10

STATUS = {
    0: "DBC_OK", -1: "DBC_EINVAL", -2: "DBC_ENOMEM", -3: "DBC_ECUDA", -4: "DBC_ENCCL",
    -5: "DBC_ESTATE", -6: "DBC_EEDGE", -7: "DBC_ECAPACITY", -8: "DBC_ENUMERIC",
}


class DBCError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))


REDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p)
ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p)


class Tuning(ctypes.Structure):
    """dbc_tuning (include/dbc.h): launch configuration only, results never depend on it."""
    _fields_ = [
        ("update_block", ctypes.c_int32), ("update_pair", ctypes.c_int32),
        ("static_block", ctypes.c_int32), ("window", ctypes.c_int32), ("heavy_cap", ctypes.c_int32),
        ("heavy_factor", ctypes.c_float), ("help_down_min", ctypes.c_int32),
        ("help_down_block", ctypes.c_int32), ("help_entries", ctypes.c_int32),
        ("help_min_blocks", ctypes.c_int32), ("busy_help", ctypes.c_int32), ("busy_min", ctypes.c_int32),
        ("down_long_min", ctypes.c_int32), ("wide_inlane", ctypes.c_int32), ("lean_block", ctypes.c_int32),
        ("lean_workers", ctypes.c_int32), ("lean_max_batch", ctypes.c_int32), ("lean_short", ctypes.c_int32),
        ("trace_slot", ctypes.c_int32), ("disable", ctypes.c_uint32), ("static_ms", ctypes.c_int32),
        ("static_groups", ctypes.c_int32), ("static_chunk", ctypes.c_int32), ("static_width", ctypes.c_int32),
        ("reserved", ctypes.c_uint32 * 4),
    ]


class Options(ctypes.Structure):
    _fields_ = [
        ("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
        ("workers", ctypes.c_int32), ("edge_capacity", ctypes.c_int64),
        ("stream", ctypes.c_void_p), ("flags", ctypes.c_uint32), ("pad0", ctypes.c_uint32),
        ("tuning", ctypes.POINTER(Tuning)), ("nccl_id", ctypes.c_void_p),
        ("reduce", REDUCE_FN), ("reduce_user", ctypes.c_void_p),
        ("dev_alloc", ALLOC_FN), ("dev_free", FREE_FN), ("alloc_user", ctypes.c_void_p),
        ("reserved", ctypes.c_uint32 * 4),
    ]


class InsertStats(ctypes.Structure):
    _fields_ = [
        ("insertions", ctypes.c_int64), ("case_count", ctypes.c_int64 * 3),
        ("touched", ctypes.c_int64), ("down_vertices", ctypes.c_int64),
        ("edges_scanned", ctypes.c_int64), ("alg_bytes", ctypes.c_int64),
    ]

    def as_dict(self):
        return dict(insertions=self.insertions, case1=self.case_count[0],
                    case2=self.case_count[1], case3=self.case_count[2], touched=self.touched,
                    down_vertices=self.down_vertices, edges_scanned=self.edges_scanned,
                    alg_bytes=self.alg_bytes)


class Timings(ctypes.Structure):
    _fields_ = [
        ("append_ms", ctypes.c_float), ("update_ms", ctypes.c_float),
        ("static_ms", ctypes.c_float), ("update_launches", ctypes.c_int32),
        ("kernel_launches", ctypes.c_int32), ("static_alg_bytes", ctypes.c_int64),
        ("append_ms_total", ctypes.c_double), ("update_ms_total", ctypes.c_double),
        ("update_launches_total", ctypes.c_int64), ("kernel_launches_total", ctypes.c_int64),
        ("insertions_total", ctypes.c_int64), ("alg_bytes_total", ctypes.c_int64),
        ("heavy_roots", ctypes.c_int32), ("reserved2", ctypes.c_int32),
    ]

    def as_dict(self):
        return {name: getattr(self, name) for name, _ in self._fields_}


# every symbol include/dbc.h declares, with its signature
_P = ctypes.c_void_p
SIGNATURES = {
    "dbc_options_default": (None, [_P]),
    "dbc_tuning_default": (None, [_P]),
    "dbc_nccl_unique_id": (ctypes.c_int, [_P]),
    "dbc_create": (ctypes.c_int, [_P, ctypes.c_int32, _P, _P, _P, ctypes.c_int32, _P]),
    "dbc_static_compute": (ctypes.c_int, [_P]),
    "dbc_insert_edges": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "dbc_insert_edges_device": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "dbc_delete_edges": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "dbc_delete_edges_device": (ctypes.c_int, [_P, _P, _P, ctypes.c_int64, _P]),
    "dbc_get_bc": (ctypes.c_int, [_P, _P]),
    "dbc_get_bc_partial_device": (ctypes.c_int, [_P, _P]),
    "dbc_get_bc_device": (ctypes.c_int, [_P, _P]),
    "dbc_get_root_state": (ctypes.c_int, [_P, ctypes.c_int32, _P, _P, _P]),
    "dbc_num_local_roots": (ctypes.c_int, [_P, _P]),
    "dbc_synchronize": (ctypes.c_int, [_P]),
    "dbc_get_timings": (ctypes.c_int, [_P, _P]),
    "dbc_reset_timings": (ctypes.c_int, [_P]),
    "dbc_debug_counters": (ctypes.c_int, [_P, _P, ctypes.c_int32]),
    "dbc_debug_root_profile": (ctypes.c_int, [_P, ctypes.c_int32, _P]),
    "dbc_debug_cta_profile": (ctypes.c_int, [_P, _P, ctypes.c_int64, _P]),
    "dbc_device_bytes": (ctypes.c_int, [_P, _P]),
    "dbc_scenario_log": (ctypes.c_int, [_P, ctypes.c_int64]),
    "dbc_get_scenarios": (ctypes.c_int, [_P, _P, ctypes.c_int64, _P]),
    "dbc_strerror": (ctypes.c_char_p, [ctypes.c_int]),
    "dbc_last_error": (ctypes.c_char_p, [_P]),
    "dbc_abi_version": (ctypes.c_int32, []),
    "dbc_destroy": (None, [_P]),
}

_lib = None


def load_library():
    """Load libdbc.so (raises if it was not built -- there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
        lib = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            if name.startswith("dbc_debug_") and not hasattr(lib, name):
                continue  # diagnostics are optional (older builds)
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _lib = lib
    return _lib


def _check(ctx, rc):
    if rc != 0:
        lib = load_library()
        msg = lib.dbc_last_error(ctx)
        raise DBCError(rc, msg.decode() if msg else "")


def _host(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def _np_ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p)


class DynamicBC:
    """Dynamic betweenness centrality over a root set on one GPU (one rank).

    >>> bc = DynamicBC(n, row_ptr, col, roots)     # dbc_create
    >>> bc.static_compute()                        # Brandes (Alg. 1)
    >>> bc.insert_edges(u, v)                      # sequential insertions, one batch
    >>> bc.get_bc()                                # Eq. (3)
    """

    def __init__(self, n, row_ptr, col, roots, *, device=0, rank=0, world=1, workers=0,
                 edge_capacity=0, stream=None, flags=0, tuning=None, nccl_id=None, reduce=None,
                 allocator=None):
        """tuning: dict of dbc_tuning fields (launch configuration only);
        nccl_id: 128 bytes from nccl_unique_id() on rank 0 (the context then
        owns an NCCL communicator and get_bc() returns the global BC);
        reduce: python callable(ptr, n, stream) -> int summing the partial in
        place across ranks (see torch_reducer); allocator: (alloc, free)
        python callables, e.g. torch_allocator(device)."""
        lib = load_library()
        self._lib = lib
        self._ctx = None
        self._keep = []  # ctypes objects the context points at
        self.n = int(n)
        self.k = int(np.asarray(roots).size)
        self.rank, self.world, self.device = int(rank), int(world), int(device)
        rp = _host(row_ptr, np.int64)
        cl = _host(col, np.int32)
        rt = _host(roots, np.int32)
        opt = Options()
        lib.dbc_options_default(ctypes.byref(opt))
        opt.device, opt.rank, opt.world = self.device, self.rank, self.world
        opt.workers, opt.edge_capacity, opt.flags = int(workers), int(edge_capacity), int(flags)
        if tuning:
            t = Tuning()
            lib.dbc_tuning_default(ctypes.byref(t))
            for k, val in tuning.items():
                if k not in dict(Tuning._fields_):
                    raise KeyError(f"unknown tuning field {k}")
                setattr(t, k, val)
            self._keep.append(t)
            opt.tuning = ctypes.pointer(t)
        if nccl_id is not None:
            buf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            self._keep.append(buf)
            opt.nccl_id = ctypes.cast(buf, ctypes.c_void_p)
        if reduce is not None:
            def _red(ptr, cnt, strm, _user, _f=reduce):
                try:
                    return int(_f(int(ptr), int(cnt), strm))
                except Exception:  # pragma: no cover - reported as DBC_ENCCL
                    return 1
            cb = REDUCE_FN(_red)
            self._keep.append(cb)
            opt.reduce = cb
        if allocator is not None:
            af, ff = allocator
            ca = ALLOC_FN(lambda b, _u, _f=af: _f(int(b)) or None)
            cf = FREE_FN(lambda p, _u, _f=ff: _f(int(p)))
            self._keep += [ca, cf]
            opt.dev_alloc, opt.dev_free = ca, cf
        if stream is None:
            try:
                import torch

                if torch.cuda.is_available():
                    with torch.cuda.device(self.device):
                        stream = torch.cuda.current_stream().cuda_stream
            except Exception:  # pragma: no cover
                stream = None
        if stream == 0:
            stream = 1  # torch's default stream is the legacy stream: cudaStreamLegacy
        opt.stream = stream
        out = ctypes.c_void_p()
        rc = lib.dbc_create(ctypes.byref(out), self.n, _np_ptr(rp), _np_ptr(cl), _np_ptr(rt),
                            self.k, ctypes.byref(opt))
        _check(None, rc)
        self._ctx = out

    # -- lifecycle -----------------------------------------------------------
    def close(self):
        if self._ctx:
            self._lib.dbc_destroy(self._ctx)
            self._ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- calls -----------------------------------------------------------------
    def static_compute(self):
        _check(self._ctx, self._lib.dbc_static_compute(self._ctx))

    def _edges_call(self, host_fn, dev_fn, u, v, stats):
        st = InsertStats() if stats else None
        stp = ctypes.byref(st) if st is not None else None
        if hasattr(u, "is_cuda") and u.is_cuda:
            import torch

            assert u.dtype == torch.int32 and v.dtype == torch.int32 and u.numel() == v.numel()
            assert u.is_contiguous() and v.is_contiguous()
            rc = dev_fn(self._ctx, ctypes.c_void_p(u.data_ptr()), ctypes.c_void_p(v.data_ptr()), u.numel(), stp)
        else:
            uu, vv = _host(u, np.int32).ravel(), _host(v, np.int32).ravel()
            if uu.size != vv.size:
                raise ValueError("u and v differ in length")
            rc = host_fn(self._ctx, _np_ptr(uu), _np_ptr(vv), uu.size, stp)
        _check(self._ctx, rc)
        return st.as_dict() if st is not None else None

    def insert_edges(self, u, v, stats=False):
        """Host arrays -> dbc_insert_edges; CUDA tensors -> dbc_insert_edges_device."""
        return self._edges_call(self._lib.dbc_insert_edges, self._lib.dbc_insert_edges_device, u, v, stats)

    def delete_edges(self, u, v, stats=False):
        """Host arrays -> dbc_delete_edges; CUDA tensors -> dbc_delete_edges_device."""
        return self._edges_call(self._lib.dbc_delete_edges, self._lib.dbc_delete_edges_device, u, v, stats)

    def get_bc(self, out=None):
        out = np.empty(self.n, dtype=np.float64) if out is None else out
        _check(self._ctx, self._lib.dbc_get_bc(self._ctx, _np_ptr(out)))
        return out

    def get_bc_partial(self):
        """This rank's BC partial (Eq. (3) over the local roots) on the host: a copy
        of dbc_get_bc_partial_device's buffer."""
        ptr = self.bc_partial_device_ptr()
        self.synchronize()
        return _wrap_device_f64(ptr, self.n, self.device).cpu().numpy().copy()

    def bc_device_ptr(self) -> int:
        """dbc_get_bc_device: the global BC in device memory (all-reduced across
        ranks on the context stream); a collective call at world > 1."""
        p = ctypes.c_void_p()
        _check(self._ctx, self._lib.dbc_get_bc_device(self._ctx, ctypes.byref(p)))
        return int(p.value)

    def bc_partial_device_ptr(self) -> int:
        p = ctypes.c_void_p()
        _check(self._ctx, self._lib.dbc_get_bc_partial_device(self._ctx, ctypes.byref(p)))
        return int(p.value)

    def get_root_state(self, slot):
        d = np.empty(self.n, dtype=np.int32)
        s = np.empty(self.n, dtype=np.float64)
        dl = np.empty(self.n, dtype=np.float64)
        _check(self._ctx, self._lib.dbc_get_root_state(self._ctx, int(slot), _np_ptr(d), _np_ptr(s),
                                                       _np_ptr(dl)))
        return d, s, dl

    def num_local_roots(self):
        k = ctypes.c_int32()
        _check(self._ctx, self._lib.dbc_num_local_roots(self._ctx, ctypes.byref(k)))
        return k.value

    def local_slots(self):
        return list(range(self.rank, self.k, self.world))

    def synchronize(self):
        _check(self._ctx, self._lib.dbc_synchronize(self._ctx))

    def timings(self):
        t = Timings()
        _check(self._ctx, self._lib.dbc_get_timings(self._ctx, ctypes.byref(t)))
        return t.as_dict()

    def reset_timings(self):
        _check(self._ctx, self._lib.dbc_reset_timings(self._ctx))

    def debug_counters(self):
        names = ["case1", "case2", "case3", "touched", "down", "scanned", "alg_bytes",
                 "static_bytes", "sc_down", "sc_removal", "sc_dpull", "sc_dpush", "sc_up2", "sc_up3",
                 "ns_down", "ns_removal", "ns_up_setup", "ns_up_epi", "ns_up_l1pairs", "ns_up_end",
                 "ns_up_split", "ns_up_scan", "ns_up_pull", "ns_up_push", "levels_down", "levels_up",
                 "help_requests", "help_blocks_by_helpers", "help_blocks_all",
                 "case2_groups", "case2_group_insertions", "help_blocks_busy", "deferred_rows", "up_passes_helped"]
        out = np.zeros(len(names), dtype=np.int64)
        _check(self._ctx, self._lib.dbc_debug_counters(self._ctx, _np_ptr(out), out.size))
        return dict(zip(names, out.tolist()))

    def debug_trace(self):
        """Per-level event trace of the slot named by DBC_TRACE_SLOT (builds with
        -DDBC_PHASE_TIMERS only): list of (kind, level, items, t_ns); kinds 1 down
        level, 2 up level, 3 removal pass, 4 job end."""
        base = 34  # kStTraceN (after the debug_counters names)
        out = np.zeros(base + 1 + 2 * 1024, dtype=np.int64)
        _check(self._ctx, self._lib.dbc_debug_counters(self._ctx, _np_ptr(out), out.size))
        cnt = min(int(out[base]), 1024)
        ev = out[base + 1: base + 1 + 2 * cnt].reshape(-1, 2).astype(np.uint64)
        return [(int(c >> np.uint64(56)), int((c >> np.uint64(32)) & np.uint64(0xFFFFFF)),
                 int(c & np.uint64(0xFFFFFFFF)), int(t)) for c, t in ev]

    def root_profile(self, enable=True, read=True):
        out = np.zeros((self.num_local_roots(), 6), dtype=np.int64) if read else None
        _check(self._ctx, self._lib.dbc_debug_root_profile(
            self._ctx, int(enable), _np_ptr(out) if read else None))
        return out

    def cta_profile(self):
        """Per worker CTA of the last per-insertion launch (root profile on):
        int64 [workers, 3] = {entry, end of work loops, exit} globaltimer ns."""
        cnt = ctypes.c_int64()
        _check(self._ctx, self._lib.dbc_debug_cta_profile(self._ctx, None, 0, ctypes.byref(cnt)))
        out = np.zeros(cnt.value, dtype=np.int64)
        _check(self._ctx, self._lib.dbc_debug_cta_profile(self._ctx, _np_ptr(out), out.size, ctypes.byref(cnt)))
        return out.reshape(-1, 3)

    def scenario_log(self, max_insertions: int):
        """Record case and touched count of every (root, insertion) of later
        insert calls (Fig. 2 / Fig. 4); 0 turns it off."""
        _check(self._ctx, self._lib.dbc_scenario_log(self._ctx, int(max_insertions)))

    def scenarios(self):
        """Scenario log of the last insert call: (case, touched, down) int64
        arrays of shape [insertions, k_local] (case 1/2/3; touched excludes the
        root; down = |D|, the vertices whose sigma was recomputed)."""
        cnt = ctypes.c_int64()
        _check(self._ctx, self._lib.dbc_get_scenarios(self._ctx, None, 0, ctypes.byref(cnt)))
        out = np.zeros(cnt.value, dtype=np.int64)
        _check(self._ctx, self._lib.dbc_get_scenarios(self._ctx, _np_ptr(out), out.size, ctypes.byref(cnt)))
        rec = out.reshape(-1, max(self.num_local_roots(), 1))
        return rec & 3, (rec >> 2) & 0x7FFFFFFF, rec >> 33

    def device_bytes(self):
        b = ctypes.c_int64()
        _check(self._ctx, self._lib.dbc_device_bytes(self._ctx, ctypes.byref(b)))
        return b.value


def nccl_unique_id() -> bytes:
    """dbc_nccl_unique_id: 128 bytes for every rank's DynamicBC(nccl_id=...)."""
    lib = load_library()
    buf = ctypes.create_string_buffer(128)
    _check(None, lib.dbc_nccl_unique_id(buf))
    return buf.raw


def torch_reducer(group=None):
    """A `reduce` callback for DynamicBC: sums the BC partial across the ranks of a
    torch.distributed group, in place -- NCCL groups reduce the device buffer
    directly, gloo groups through a host copy.  The library's stream is
    synchronised first, so the reduction sees the finished partial."""
    import torch
    import torch.distributed as dist

    def red(ptr, n, stream):
        dev = torch.cuda.current_device()
        torch.cuda.synchronize()  # the partial is final on the library's stream
        t = _wrap_device_f64(ptr, n, dev)
        if dist.get_backend(group) == "nccl":
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
            torch.cuda.synchronize()
        else:
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
            t.copy_(h)
            torch.cuda.synchronize()
        return 0

    return red


def torch_allocator(device=0):
    """(alloc, free) hooks routing the library's device memory through torch's
    caching allocator (dbc_options.dev_alloc / dev_free)."""
    import torch

    def alloc(nbytes):
        return int(torch.cuda.caching_allocator_alloc(nbytes, device))

    def free(ptr):
        torch.cuda.caching_allocator_delete(ptr)

    return alloc, free


def local_slots(k: int, rank: int, world: int):
    """Root slots owned by `rank` (slot % world == rank), SURVEY.md Sec. 8(e)."""
    return list(range(rank, k, world))


def allreduce_bc(dbc: DynamicBC, group=None, force=False):
    """Sum the per-rank BC partials over torch.distributed (NCCL on GPUs) and
    return the global BC on the host -- the only cross-GPU exchange of the
    method -- for contexts created without nccl_id /
    reduce (those return the global BC from get_bc() directly).  force=True
    runs the collective even for a single rank (tests)."""
    import torch
    import torch.distributed as dist

    if not dist.is_initialized() or (dbc.world == 1 and not force):
        return dbc.get_bc()
    ptr = dbc.bc_partial_device_ptr()
    dbc.synchronize()
    # reduce a copy: the library keeps accumulating this rank's partial
    t = _wrap_device_f64(ptr, dbc.n, dbc.device).clone()
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t.cpu().numpy()


def _wrap_device_f64(ptr: int, n: int, device: int):
    """Zero-copy torch view of a device fp64 buffer owned by libdbc."""
    import torch

    class _CAI:
        __cuda_array_interface__ = {
            "shape": (n,), "typestr": "<f8", "data": (ptr, False), "version": 3, "strides": None,
        }

    with torch.cuda.device(device):
        return torch.as_tensor(_CAI(), device=f"cuda:{device}")
