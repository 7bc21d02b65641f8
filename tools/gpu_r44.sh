#!/bin/bash
O=gpurun_out/r44; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_UB2=1 timeout 600 $B > $O/rmat16_ub2.json 2>> $O/err.txt
DBC_UB2=1 timeout 600 $B --config smallworld > $O/sw_ub2.json 2>> $O/err.txt
DBC_UB2=0 timeout 600 $B --config delaunay18 > $O/del18_ub0.json 2>> $O/err.txt
DBC_BLOCK=256 timeout 600 $B --config delaunay18 > $O/del18_b256.json 2>> $O/err.txt
DBC_BLOCK=1024 timeout 600 $B > $O/rmat16_b1024.json 2>> $O/err.txt
timeout 900 $B --config kron22 --shard 0/8 --steps 2 --warmup 3 > $O/kron22s.json 2>> $O/err.txt
