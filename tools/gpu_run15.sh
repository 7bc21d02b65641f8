#!/bin/bash
O=gpurun_out/r15; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for cfg in "4096 3" "2048 3" "1024 4" "2048 2" "8192 2"; do
  set -- $cfg
  DBC_HEENT=$1 DBC_HEMIN=$2 timeout 300 $B > $O/rmat16_$1_$2.json 2>> $O/err.txt
done
for cfg in "4096 3" "2048 3" "1024 4"; do
  set -- $cfg
  DBC_HEENT=$1 DBC_HEMIN=$2 timeout 900 $B --config kron20 --steps 2 --warmup 3 > $O/kron20_$1_$2.json 2>> $O/err.txt
done
T=$PWD/build_timers/libdbc.so
PB_BATCHES=2 DBC_LIB_PATH=$T timeout 300 python tools/phase_breakdown.py rmat16 2000 > $O/pb_rmat16.txt 2>&1
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
