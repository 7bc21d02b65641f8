#!/bin/bash
O=gpurun_out/r47; mkdir -p $O
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_rmat16.txt 2>&1
PB_BATCHES=4 timeout 300 python -u tools/phase_breakdown.py kron20 20000 > $O/pb_kron20.txt 2>&1
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py delaunay18 4000 > $O/pb_del18.txt 2>&1
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
DBC_TRACE_SLOT=38 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot38.txt 2>&1
