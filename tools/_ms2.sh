mkdir -p gpurun_out/ms8
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:ms_kernel -c 1 -o gpurun_out/ms8/ms_kron20 python tools/static_probe.py kron20 static_ms=1,static_chunk=32 > gpurun_out/ms8/ncu.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:ms_kernel -c 1 -o gpurun_out/ms8/ms_rmat16 python tools/static_probe.py rmat16 static_ms=1,static_chunk=8 >> gpurun_out/ms8/ncu.log 2>&1
