#!/bin/bash
# A/B on one box: round-start library (899b548) vs current, Kronecker 20
O=gpurun_out/r39; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
for r in 1 2; do
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_base.so timeout 600 $B > $O/kron20_base$r.json 2>> $O/err.txt
timeout 600 $B > $O/kron20_cur$r.json 2>> $O/err.txt
done
DBC_BUSY_HELP=0 timeout 600 $B > $O/kron20_cur_bh0.json 2>> $O/err.txt
