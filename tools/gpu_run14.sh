#!/bin/bash
O=gpurun_out/r14; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for r in 1 2; do timeout 300 $B > $O/rmat16_$r.json 2>> $O/err.txt; done
DBC_NO_HELP=1 timeout 300 $B > $O/rmat16_nohelp.json 2>> $O/err.txt
timeout 600 $B --config delaunay18 > $O/delaunay18.json 2>> $O/err.txt
timeout 600 $B --config smallworld > $O/smallworld.json 2>> $O/err.txt
timeout 900 $B --config kron20 --steps 2 --warmup 3 > $O/kron20.json 2>> $O/err.txt
timeout 600 $B --config rmat16 --batch 10000 > $O/rmat16_b10k.json 2>> $O/err.txt
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
