for v in variants/libdbc_8dfc0bd.so variants/libdbc_d8fix.so variants/libdbc_nod8.so; do
  for r in 1 2; do
    DBC_LIB_PATH=$PWD/$v timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],1), round(d['config']['static_recompute_ms'],2))"
  done
done
