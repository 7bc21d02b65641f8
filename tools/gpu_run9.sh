#!/bin/bash
O=gpurun_out/r9; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "heavy or help or rmat16_full or block128" > $O/tests.log 2>&1
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for r in 1 2; do timeout 300 $B > $O/rmat16_$r.json 2>> $O/err.txt; done
DBC_HEAVY_CAP=8 timeout 300 $B > $O/rmat16_cap8.json 2>> $O/err.txt
DBC_HEAVY_CAP=32 DBC_HEAVY_FACTOR=1.5 timeout 300 $B > $O/rmat16_cap32.json 2>> $O/err.txt
DBC_HEAVY_CAP=0 timeout 300 $B > $O/rmat16_noheavy.json 2>> $O/err.txt
timeout 600 $B --config smallworld > $O/smallworld.json 2>> $O/err.txt
DBC_HEAVY_CAP=0 timeout 600 $B --config smallworld > $O/smallworld_noheavy.json 2>> $O/err.txt
timeout 600 $B --config rmat16 --steps 5 --warmup 3 --batch 10000 > $O/rmat16_b10k.json 2>> $O/err.txt
DBC_HEAVY_CAP=0 timeout 600 $B --config rmat16 --steps 5 --warmup 3 --batch 10000 > $O/rmat16_b10k_noheavy.json 2>> $O/err.txt
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
