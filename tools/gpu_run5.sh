#!/bin/bash
O=gpurun_out/r5; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "delete" > $O/del_tests.log 2>&1; echo "rc=$?" >> $O/del_tests.log
timeout 1200 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python bench.py --no-cpu-baseline --no-per-insertion --no-e2e > $O/rmat16.json 2> $O/rmat16.err
