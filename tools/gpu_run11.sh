#!/bin/bash
O=gpurun_out/r11; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
timeout 600 $B --config delaunay18 > $O/delaunay18.json 2>> $O/err.txt
DBC_NO_LOWDEG=1 timeout 600 $B --config delaunay18 > $O/delaunay18_nolowdeg.json 2>> $O/err.txt
timeout 300 $B > $O/rmat16.json 2>> $O/err.txt
for f in $O/*.json; do python -c "
import json,sys
try: d=json.load(open('$f'))
except Exception as e: print('$f FAIL'); sys.exit()
print('$f', round(d['value']), 'ms %.2f'%d['ms_per_step'], 'frac %.4f'%d['roofline']['frac'])"; done > $O/summary.txt
