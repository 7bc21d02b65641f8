#!/bin/bash
# occupancy experiment: update CTAs per SM / registers per thread
O=gpurun_out/exp; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "scenario" > $O/test_scen.log 2>&1
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e"
run() {  # tag env... -- args
  tag=$1; shift
  env "$@" > $O/$tag.json 2> $O/$tag.err
}
for cfg in rmat16 delaunay18 smallworld; do
  run ${cfg}_base timeout 300 $B --config $cfg
  run ${cfg}_512x2 DBC_LIB_PATH=$PWD/exp/libdbc_512x2.so DBC_UPB=2 timeout 300 $B --config $cfg
  run ${cfg}_256x4 DBC_LIB_PATH=$PWD/exp/libdbc_256x4.so DBC_BLOCK=256 DBC_UPB=4 DBC_NO_HEAVY=1 timeout 300 $B --config $cfg
  run ${cfg}_256x3 DBC_LIB_PATH=$PWD/exp/libdbc_256x3.so DBC_BLOCK=256 DBC_UPB=3 DBC_NO_HEAVY=1 timeout 300 $B --config $cfg
  run ${cfg}_256x2 timeout 300 env DBC_BLOCK=256 $B --config $cfg
done
run kron20_base timeout 600 $B --config kron20 --steps 2 --warmup 3
run kron20_512x2 DBC_LIB_PATH=$PWD/exp/libdbc_512x2.so DBC_UPB=2 timeout 600 $B --config kron20 --steps 2 --warmup 3
run kron20_256x4 DBC_LIB_PATH=$PWD/exp/libdbc_256x4.so DBC_BLOCK=256 DBC_UPB=4 DBC_NO_HEAVY=1 timeout 600 $B --config kron20 --steps 2 --warmup 3
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
