mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_wd.so timeout -s KILL 300 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not past_2_pow and not full_size" 2>&1 | tail -2
( timeout -s KILL 120 python scripts/mo_quick.py
  RA_LIB_PATH=$PWD/build/libra_dh.so timeout -s KILL 120 python scripts/mo_quick.py
  MO_PROF_CASES=dense RA_LIB_PATH=$PWD/build/libra_prof.so timeout -s KILL 120 python scripts/mo_prof.py ) 2>&1 | tee gpurun_out/mo_variants17.txt
