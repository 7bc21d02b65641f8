#!/bin/bash
O=gpurun_out/r35; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
DBC_DLMIN=65536 timeout 600 $B > $O/kron20_dl64k.json 2>> $O/err.txt
DBC_DLMIN=262144 timeout 600 $B > $O/kron20_dl256k.json 2>> $O/err.txt
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
for dl in 12288 65536 262144 2000000000; do DBC_DLMIN=$dl timeout 300 $B > $O/rmat16_dl$dl.json 2>> $O/err.txt; done
DBC_DLMIN=65536 timeout 300 $B --config smallworld > $O/sw_dl64k.json 2>> $O/err.txt
DBC_DLMIN=2000000000 timeout 300 $B --config smallworld > $O/sw_nodl.json 2>> $O/err.txt
