#!/bin/bash
O=gpurun_out/r52; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_BLOCK=256 timeout 600 $B --config delaunay18 > $O/del18_256x4.json 2>> $O/err.txt
timeout 600 $B --config delaunay18 > $O/del18_def.json 2>> $O/err.txt
DBC_BLOCK=256 timeout 600 $B --config kron20 --steps 3 --warmup 3 > $O/kron20_256x4.json 2>> $O/err.txt
DBC_BLOCK=256 timeout 900 $B --config kron22 --shard 0/8 --steps 2 --warmup 3 > $O/kron22s_256x4.json 2>> $O/err.txt
DBC_BLOCK=256 timeout 600 $B > $O/rmat16_256x4.json 2>> $O/err.txt
