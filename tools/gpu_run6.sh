#!/bin/bash
O=gpurun_out/r6; mkdir -p $O
timeout 400 python bench.py > $O/rmat16_full.json 2> $O/rmat16_full.err
PB_BATCHES=2 DBC_LIB_PATH=$PWD/build_timers/libdbc.so timeout 300 python tools/phase_breakdown.py rmat16 2000 > $O/pb_rmat16.txt 2>&1
DBC_LIB_PATH=$PWD/build_timers/libdbc.so timeout 600 python tools/phase_breakdown.py kron20 10000 > $O/pb_kron20.txt 2>&1
DBC_LIB_PATH=$PWD/build_timers/libdbc.so timeout 600 python tools/phase_breakdown.py delaunay18 1000 > $O/pb_delaunay18.txt 2>&1
