#!/bin/bash
O=gpurun_out/r41; mkdir -p $O
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions --config kron20 --steps 3 --warmup 3"
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_exp.so timeout 600 $B > $O/kron20_exp.json 2>> $O/err.txt
DBC_DLMIN=2000000000 DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_exp.so timeout 600 $B > $O/kron20_exp_nodl.json 2>> $O/err.txt
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_base.so timeout 600 $B > $O/kron20_base.json 2>> $O/err.txt
B="python bench.py --no-cpu-baseline --no-per-insertion --no-e2e --no-deletions"
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_exp.so timeout 600 $B > $O/rmat16_exp.json 2>> $O/err.txt
timeout 600 $B > $O/rmat16_cur.json 2>> $O/err.txt
DBC_LIB_PATH=$PWD/paper_conf_ipps_mclaughlinb14_b200/libdbc_exp.so timeout 600 $B --config delaunay18 > $O/del18_exp.json 2>> $O/err.txt
timeout 600 $B --config delaunay18 > $O/del18_cur.json 2>> $O/err.txt
