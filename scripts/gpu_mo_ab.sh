# A/B of select_multi compile-time variants: parity of each variant's multi-output
# pass, then mo_quick timings (VARIANTS="tpf2 ...": build/libra_<v>.so)
mkdir -p gpurun_out
for v in $VARIANTS; do
  RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 300 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not 2_pow_31" 2>&1 | tail -1
done
for rep in 1 2; do
  timeout -s KILL 120 python scripts/mo_quick.py
  for v in $VARIANTS; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 120 python scripts/mo_quick.py; done
done 2>&1 | tee gpurun_out/mo_ab.txt
