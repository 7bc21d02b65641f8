#!/bin/bash
O=gpurun_out/r53; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --steps 2 --warmup 3"
for sb in 256 512 1024; do
DBC_SBLOCK=$sb timeout 600 $B > $O/rmat16_s$sb.json 2>> $O/err.txt
DBC_SBLOCK=$sb timeout 600 $B --config delaunay18 > $O/del18_s$sb.json 2>> $O/err.txt
DBC_SBLOCK=$sb timeout 600 $B --config smallworld > $O/sw_s$sb.json 2>> $O/err.txt
DBC_SBLOCK=$sb timeout 900 $B --config kron20 > $O/kron20_s$sb.json 2>> $O/err.txt
done
DBC_SBLOCK=128 timeout 600 $B --config delaunay18 > $O/del18_s128.json 2>> $O/err.txt
