#!/bin/bash
O=gpurun_out/r16; mkdir -p $O
PB_BATCHES=2 timeout 120 python -u tools/phase_breakdown.py rmat16 2000 > $O/pb_normal.txt 2>&1; echo "rc=$?" >> $O/pb_normal.txt
PB_BATCHES=2 DBC_LIB_PATH=$PWD/build_timers/libdbc.so timeout 120 python -u tools/phase_breakdown.py rmat16 2000 > $O/pb_timers.txt 2>&1; echo "rc=$?" >> $O/pb_timers.txt
nvidia-smi > $O/smi.txt 2>&1
