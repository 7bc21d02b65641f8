#!/bin/bash
O=gpurun_out/r34; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
timeout 600 $B > $O/kron20.json 2>> $O/err.txt
DBC_BUSY_HELP=0 timeout 600 $B > $O/kron20_bh0.json 2>> $O/err.txt
DBC_DLMIN=2000000000 timeout 600 $B > $O/kron20_nodl.json 2>> $O/err.txt
DBC_DLMIN=2000000000 DBC_BUSY_HELP=0 timeout 600 $B > $O/kron20_nodl_bh0.json 2>> $O/err.txt
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config delaunay18"
timeout 300 $B > $O/del18.json 2>> $O/err.txt
DBC_BUSY_HELP=0 timeout 300 $B > $O/del18_bh0.json 2>> $O/err.txt
