#!/bin/bash
O=gpurun_out/r32; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for bh in 1 0 4; do DBC_BUSY_HELP=$bh timeout 300 $B > $O/rmat16_bh$bh.json 2>> $O/err.txt; done
DBC_BUSY_MIN=4 timeout 300 $B > $O/rmat16_bm4.json 2>> $O/err.txt
DBC_BUSY_MIN=64 timeout 300 $B > $O/rmat16_bm64.json 2>> $O/err.txt
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
for bh in 1; do DBC_BUSY_HELP=$bh DBC_TRACE_SLOT=38 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_slot38_bh$bh.txt 2>&1; done
