mkdir -p gpurun_out/ms9
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "static" 2>&1 | tail -15 > gpurun_out/ms9/tests.log
for c in rmat16 smallworld kron20; do timeout 600 python tools/static_probe.py $c static_ms=0 static_ms=1,static_chunk=8 static_ms=1,static_chunk=16 static_ms=1,static_chunk=32 >> gpurun_out/ms9/probe.jsonl 2>&1; done
for c in rmat16 kron20; do timeout 600 python tools/ms_phases.py $c static_chunk=16 >> gpurun_out/ms9/phases.jsonl 2>&1; done
