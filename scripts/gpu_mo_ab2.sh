# quick parity of each variant on small inputs (fails fast), then the A/B timings
mkdir -p gpurun_out
ok=""
for v in $VARIANTS; do
  echo "== $v"; RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 60 python scripts/mo_small_check.py 2>&1 | tail -3
  RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 60 python scripts/mo_small_check.py >/dev/null 2>&1 && ok="$ok $v"
done
for v in $ok; do
  RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 300 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not 2_pow_31" 2>&1 | tail -1
done
for rep in 1 2; do
  timeout -s KILL 120 python scripts/mo_quick.py
  for v in $ok; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 120 python scripts/mo_quick.py; done
done 2>&1 | tee gpurun_out/mo_ab.txt
