#!/bin/bash
# rmat16 root-chain breakdown + ncu of one all-roots update launch (heavy lanes off)
O=gpurun_out/r20; mkdir -p $O
PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_rmat16.txt 2>&1
DBC_HEAVY_CAP=0 PB_BATCHES=4 timeout 120 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb_rmat16_noheavy.txt 2>&1
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_HEAVY_CAP=0 timeout 300 $B > $O/bench_noheavy.json 2> $O/err.txt
timeout 300 $B > $O/bench_default.json 2>> $O/err.txt
DBC_HEAVY_CAP=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:update --launch-skip 3 --launch-count 1 -o $O/update_noheavy python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions > $O/ncu_update.log 2>&1
ls -la $O
