mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_splitwd.so timeout -s KILL 300 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not past_2_pow and not full_size" 2>&1 | tail -2
( timeout -s KILL 120 python scripts/mo_quick.py
  RA_LIB_PATH=$PWD/build/libra_split.so timeout -s KILL 120 python scripts/mo_quick.py ) 2>&1 | tee gpurun_out/mo_variants16.txt
