#!/bin/bash
O=gpurun_out/r45; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_BLOCK=1024 timeout 600 $B > $O/rmat16_b1024.json 2>> $O/err.txt
timeout 600 $B > $O/rmat16_def.json 2>> $O/err.txt
DBC_BLOCK=1024 timeout 600 $B --config smallworld > $O/sw_b1024.json 2>> $O/err.txt
DBC_BLOCK=1024 timeout 600 $B --config delaunay18 > $O/del18_b1024.json 2>> $O/err.txt
DBC_BLOCK=1024 timeout 600 $B --config kron20 --steps 3 --warmup 3 > $O/kron20_b1024.json 2>> $O/err.txt
