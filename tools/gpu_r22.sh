#!/bin/bash
# busy-worker help: parity + bench sweep
O=gpurun_out/r22; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for bh in 1 0 2 4; do DBC_BUSY_HELP=$bh timeout 300 $B > $O/rmat16_bh$bh.json 2>> $O/err.txt; done
for bh in 1 0; do DBC_BUSY_HELP=$bh timeout 300 $B --config delaunay18 > $O/del18_bh$bh.json 2>> $O/err.txt; done
for bh in 1 0; do DBC_BUSY_HELP=$bh timeout 300 $B --config smallworld > $O/sw_bh$bh.json 2>> $O/err.txt; done
DBC_BUSY_HELP=1 timeout 200 python -u tools/phase_breakdown.py rmat16 4000 > $O/pb.txt 2>&1
