#!/bin/bash
bash tools/gpu_run17.sh
O=gpurun_out/r18
timeout 1500 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for r in 1 2; do timeout 300 $B > $O/rmat16_$r.json 2>> $O/err.txt; done
