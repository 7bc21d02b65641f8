#!/bin/bash
O=gpurun_out/r13; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for cfg in "3072 1024" "1024 512" "512 256" "2048 256" "1024 1024" "512 512"; do
  set -- $cfg
  DBC_HDMIN=$1 DBC_HDBLK=$2 timeout 300 $B > $O/rmat16_$1_$2.json 2>> $O/err.txt
  DBC_HDMIN=$1 DBC_HDBLK=$2 timeout 300 $B --config smallworld > $O/sw_$1_$2.json 2>> $O/err.txt
done
for cfg in "3072 1024" "1024 512" "512 256"; do
  set -- $cfg
  DBC_HDMIN=$1 DBC_HDBLK=$2 timeout 900 $B --config kron20 --steps 2 --warmup 3 > $O/kron20_$1_$2.json 2>> $O/err.txt
done
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
