#!/bin/bash
O=gpurun_out/r4; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
B="python bench.py --no-per-insertion"
for r in 1 2 3; do timeout 300 $B --no-cpu-baseline --no-e2e > $O/rmat16_$r.json 2> $O/rmat16_$r.err; done
timeout 300 python bench.py > $O/rmat16_full.json 2> $O/rmat16_full.err
timeout 600 $B --config delaunay18 --no-cpu-baseline --no-e2e > $O/delaunay18.json 2> $O/delaunay18.err
timeout 900 $B --config kron20 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/kron20.json 2> $O/kron20.err
for c in rmat16 smallworld delaunay18; do timeout 900 python tools/paper_figures.py $c 100 > $O/fig_$c.json 2> $O/fig_$c.err; done
