#!/bin/bash
O=gpurun_out/r42; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
timeout 600 $B > $O/kron20_cur.json 2>> $O/err.txt
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_base.so timeout 600 $B > $O/kron20_base.json 2>> $O/err.txt
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
timeout 600 $B > $O/rmat16_cur.json 2>> $O/err.txt
timeout 600 $B --config delaunay18 > $O/del18_cur.json 2>> $O/err.txt
timeout 600 $B --config smallworld > $O/sw_cur.json 2>> $O/err.txt
