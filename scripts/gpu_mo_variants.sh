mkdir -p gpurun_out
for v in w8wd w8bwd; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 300 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "three_four or many_outputs" 2>&1 | tail -1; done
( timeout -s KILL 120 python scripts/mo_quick.py
  for v in w8 w8b; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 120 python scripts/mo_quick.py; done ) 2>&1 | tee gpurun_out/mo_variants18.txt
