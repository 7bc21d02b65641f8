#!/bin/bash
O=gpurun_out/r54; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
timeout 600 $B > $O/rmat16.json 2>> $O/err.txt
