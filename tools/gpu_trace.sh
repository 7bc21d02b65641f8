#!/bin/bash
O=gpurun_out/r56; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
timeout 600 $B > $O/rmat16.json 2>> $O/err.txt
timeout 600 $B > $O/rmat16_b.json 2>> $O/err.txt
timeout 600 $B --config smallworld > $O/sw.json 2>> $O/err.txt
timeout 600 $B --config kron20 --steps 3 --warmup 3 > $O/kron20.json 2>> $O/err.txt
timeout 600 $B --config delaunay18 > $O/del18.json 2>> $O/err.txt
