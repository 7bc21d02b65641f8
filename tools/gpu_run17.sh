#!/bin/bash
O=gpurun_out/r18; mkdir -p $O
run() { tag=$1; shift; env "$@" PB_BATCHES=2 timeout 60 python -u tools/phase_breakdown.py rmat16 2000 > $O/$tag.txt 2>&1; echo "$tag rc=$?" >> $O/summary.txt; }
run a1
run a2
run nohelp DBC_NO_HELP=1
run noheavy DBC_HEAVY_CAP=0
run nohd DBC_HDMIN=100000000
run a3
run noheavy2 DBC_HEAVY_CAP=0
run nohd2 DBC_HDMIN=100000000
