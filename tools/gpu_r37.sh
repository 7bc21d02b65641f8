#!/bin/bash
O=gpurun_out/r37; mkdir -p $O
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
DBC_TRACE_SLOT=38 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot38.txt 2>&1
DBC_TRACE_SLOT=72 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot72.txt 2>&1
