#!/bin/bash
# Round evidence: GPU tests, smoke, bench lines per config, reference arm, launch
# list, ncu captures of the three kernel families, paper figures.
O=gpurun_out/${FINAL_DIR:-final}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q --durations=15 > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_rmat16.json 2> $O/bench_rmat16.err
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > $O/bench_reference.json 2> $O/bench_reference.err
B="python bench.py --no-cpu-baseline"
timeout 900 $B --config delaunay18 > $O/bench_delaunay18.json 2> $O/bench_delaunay18.err
timeout 900 $B --config delaunay18u > $O/bench_delaunay18u.json 2> $O/bench_delaunay18u.err
timeout 600 $B --config smallworld > $O/bench_smallworld.json 2> $O/bench_smallworld.err
timeout 1500 $B --config kron20 --steps 3 --warmup 3 --no-e2e > $O/bench_kron20.json 2> $O/bench_kron20.err
timeout 1500 $B --config kron22 --shard 0/8 --steps 2 --warmup 3 --no-e2e --no-per-insertion --no-deletions > $O/bench_kron22_shard0of8.json 2> $O/bench_kron22.err
N="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv $N --steps 2 --warmup 3 > $O/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel --launch-skip 3 --launch-count 1 -o $O/update_full $N --steps 1 --warmup 3 > $O/ncu_update.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"static_kernel|ms_kernel" --launch-count 1 -o $O/static_full $N --steps 1 --warmup 3 > $O/ncu_static.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ms_kernel --launch-count 1 -o $O/ms_kron20_full python tools/static_probe.py kron20 default > $O/ncu_ms_kron20.log 2>&1
for c in rmat16 kron20 smallworld delaunay18; do timeout 900 python tools/static_probe.py $c static_ms=0 static_ms=1 > $O/static_$c.jsonl 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lean --launch-skip 20 --launch-count 1 -o $O/lean_full python tools/lean_ncu_target.py rmat16 40 > $O/ncu_lean.log 2>&1
for c in rmat16 smallworld delaunay18; do timeout 900 python tools/paper_figures.py $c 100 > $O/fig_$c.json 2> $O/fig_$c.err; done
# the batch kernel on the other configs (DRAM traffic for ncu_traffic.json)
timeout 1200 ncu --set full --clock-control none -k regex:update_kernel --launch-skip 3 --launch-count 1 -o $O/upd_kron20 $N --config kron20 --steps 1 --warmup 3 > $O/ncu_upd_kron20.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:update_kernel --launch-skip 3 --launch-count 1 -o $O/upd_delaunay18 $N --config delaunay18 --steps 1 --warmup 3 > $O/ncu_upd_del18.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:update_kernel --launch-skip 3 --launch-count 1 -o $O/upd_smallworld $N --config smallworld --steps 1 --warmup 3 > $O/ncu_upd_sw.log 2>&1
# per-insertion launch anatomy
timeout 600 python tools/lean_anatomy.py rmat16 40 > $O/anatomy_rmat16.jsonl 2>&1
timeout 600 python tools/batch_anatomy.py rmat16 6 > $O/batch_anatomy_rmat16.jsonl 2>&1
ls -la $O
# summaries on the box (gpurun copies back <= 64 MiB): JSON per capture, then
# only the R-MAT 16 batch-kernel report is kept
for r in $O/*.ncu-rep; do python tools/ncu_summary.py raw $r > ${r%.ncu-rep}_summary.json 2>/dev/null; done
python tools/ncu_summary.py launches $O/launches.csv > $O/launches_summary.json 2>/dev/null
for r in $O/*.ncu-rep; do case $r in *update_full.ncu-rep) ;; *) rm -f $r ;; esac; done
du -sh $O
