mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_ng3wd.so timeout -s KILL 300 python -m pytest tests/test_select_gpu.py -x -q -p no:cacheprovider -k "multi_output_pass or both_pass" 2>&1 | tail -1
( timeout -s KILL 120 python scripts/mo_quick.py
  RA_LIB_PATH=$PWD/build/libra_ng3.so timeout -s KILL 120 python scripts/mo_quick.py ) 2>&1 | tee gpurun_out/mo_variants20.txt
