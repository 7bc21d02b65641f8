mkdir -p gpurun_out/r2
O=gpurun_out/r2
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "scenario" > $O/test_scen.log 2>&1
timeout 300 python tools/paper_figures.py rmat16 100 > $O/fig_rmat16.json 2> $O/fig_rmat16.err
timeout 600 python tools/paper_figures.py delaunay18 100 > $O/fig_delaunay18.json 2> $O/fig_delaunay18.err
timeout 300 python tools/paper_figures.py smallworld 100 > $O/fig_smallworld.json 2> $O/fig_smallworld.err
timeout 300 ncu --set full --clock-control none --import-source on -k regex:update --launch-skip 3 --launch-count 1 -o $O/update_full_a python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-per-insertion --no-e2e > $O/ncu_a.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on --kernel-id ::regex:update:4 -o $O/update_full_b python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-per-insertion --no-e2e > $O/ncu_b.log 2>&1
ls -la $O
