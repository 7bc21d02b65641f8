#!/bin/bash
O=gpurun_out/r10; mkdir -p $O
T=$PWD/build_timers/libdbc.so
# the heaviest root of rmat16 alone (chain = kernel time), 512 vs 1024 threads
for blk in 512 1024 256; do
  DBC_BLOCK=$blk DBC_LIB_PATH=$T timeout 300 python tools/phase_breakdown.py rmat16 2000 0 3621 > $O/pb_root3621_$blk.txt 2>&1
done
DBC_BLOCK=512 DBC_LIB_PATH=$T timeout 300 python tools/phase_breakdown.py rmat16 2000 0 3621,45389,16562,50741 > $O/pb_4roots.txt 2>&1
