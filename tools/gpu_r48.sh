#!/bin/bash
O=gpurun_out/r48; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for w in 1 0; do
DBC_WIDE_INLANE=$w timeout 600 $B > $O/rmat16_w$w.json 2>> $O/err.txt
DBC_WIDE_INLANE=$w timeout 600 $B --config smallworld > $O/sw_w$w.json 2>> $O/err.txt
DBC_WIDE_INLANE=$w timeout 600 $B --config kron20 --steps 3 --warmup 3 > $O/kron20_w$w.json 2>> $O/err.txt
done
timeout 600 $B --config delaunay18 > $O/del18.json 2>> $O/err.txt
