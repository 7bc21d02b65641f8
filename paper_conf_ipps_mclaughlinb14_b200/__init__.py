"""B200-native dynamic betweenness centrality (McLaughlin & Bader, dblp conf/ipps 2014).

The compute path is libdbc.so (hand-written sm_100a CUDA behind the C ABI of
include/dbc.h); this package is the thin Python binding.  See DESIGN.md.
"""

from .dbc import (  # noqa: F401
    DBC_INF,
    FLAG_EDGE_PARALLEL,
    FLAG_EXACT_BC,
    FLAG_MODE_S,
    FLAG_NO_MERGE,
    FLAG_NO_REORDER,
    FLAG_PULL_DELTA,
    FLAG_TIMING,
    TUNE_NO_HEAVY,
    TUNE_NO_HELP,
    TUNE_NO_LEAN,
    TUNE_NO_LEAN_HELP,
    TUNE_NO_LOWDEG,
    Tuning,
    DBCError,
    DynamicBC,
    LIB_PATH,
    allreduce_bc,
    load_library,
    local_slots,
    nccl_unique_id,
    torch_allocator,
    torch_reducer,
)

__all__ = [
    "DynamicBC", "DBCError", "DBC_INF", "FLAG_MODE_S", "FLAG_TIMING", "FLAG_EXACT_BC", "FLAG_NO_REORDER", "FLAG_NO_MERGE",
    "FLAG_EDGE_PARALLEL", "FLAG_PULL_DELTA", "Tuning", "TUNE_NO_HELP", "TUNE_NO_HEAVY", "TUNE_NO_LEAN",
    "TUNE_NO_LEAN_HELP", "TUNE_NO_LOWDEG",
    "LIB_PATH", "load_library", "local_slots", "allreduce_bc", "nccl_unique_id", "torch_reducer",
    "torch_allocator",
]
