#!/bin/bash
O=gpurun_out/r51; mkdir -p $O
export DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_timers.so
DBC_TRACE_SLOT=133 PB_BATCHES=2 timeout 300 python -u tools/phase_breakdown.py delaunay18 2000 > $O/pb_del18_slot133.txt 2>&1
