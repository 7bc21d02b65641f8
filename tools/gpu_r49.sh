#!/bin/bash
O=gpurun_out/r49; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for w in 4 16 64; do
DBC_WIDE_INLANE=$w timeout 600 $B > $O/rmat16_w$w.json 2>> $O/err.txt
DBC_WIDE_INLANE=$w timeout 600 $B --config kron20 --steps 3 --warmup 3 > $O/kron20_w$w.json 2>> $O/err.txt
done
