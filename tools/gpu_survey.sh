#!/bin/bash
# Data-gathering pass on the GPU box: bench lines on each config + ncu of the default bench.
set -x
mkdir -p gpurun_out/survey
O=gpurun_out/survey
timeout 300 python bench.py --no-cpu-baseline > $O/rmat16.json 2> $O/rmat16.err
timeout 600 python bench.py --config delaunay18 --no-cpu-baseline > $O/delaunay18.json 2> $O/delaunay18.err
timeout 300 python bench.py --config smallworld --no-cpu-baseline > $O/smallworld.json 2> $O/smallworld.err
timeout 900 python bench.py --config kron20 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > $O/kron20.json 2> $O/kron20.err
PB_BATCHES=2 timeout 300 python tools/phase_breakdown.py rmat16 1000 > $O/pb_rmat16.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-per-insertion > $O/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel -s 4 -c 1 -o $O/update_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-per-insertion --no-e2e > $O/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:static_kernel -s 0 -c 1 -o $O/static_full python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-per-insertion --no-e2e > $O/ncu_static.log 2>&1
ls -la $O
