#!/bin/bash
# phase timers: rmat16 all roots, and the slowest root alone
O=gpurun_out/r21; mkdir -p $O
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_all.txt 2>&1
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 0 2223 > $O/pb_2223.txt 2>&1
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 0 2223,17921,62703,59075 > $O/pb_4heavy.txt 2>&1
DBC_NO_HELP=1 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 0 2223 > $O/pb_2223_nohelp.txt 2>&1
unset DBC_LIB_PATH
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 0 2223 > $O/pb_2223_notimer.txt 2>&1
ls -la $O
