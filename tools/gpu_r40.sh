#!/bin/bash
O=gpurun_out/r40; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "forced_help or heavy_lane or help_off or full_size or window" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_base.so timeout 600 $B > $O/kron20_base.json 2>> $O/err.txt
timeout 600 $B > $O/kron20_cur.json 2>> $O/err.txt
DBC_DLMIN=2000000000 timeout 600 $B > $O/kron20_cur_nodl.json 2>> $O/err.txt
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_base.so timeout 600 $B > $O/rmat16_base.json 2>> $O/err.txt
timeout 600 $B > $O/rmat16_cur.json 2>> $O/err.txt
