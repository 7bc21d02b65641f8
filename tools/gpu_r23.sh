#!/bin/bash
# phase timers of single roots inside the full rmat16 batch
O=gpurun_out/r23; mkdir -p $O
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
for s in 38 165 41 72; do DBC_TRACE_SLOT=$s PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot$s.txt 2>&1; done
DBC_NO_HELP=1 DBC_TRACE_SLOT=38 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot38_nohelp.txt 2>&1
