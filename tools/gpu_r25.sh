#!/bin/bash
O=gpurun_out/r25; mkdir -p $O
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
for s in 38 165 72; do DBC_TRACE_SLOT=$s PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot$s.txt 2>&1; done
DBC_TRACE_SLOT=38 DBC_HDMIN=256 DBC_HDBLK=128 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot38_hd256.txt 2>&1
