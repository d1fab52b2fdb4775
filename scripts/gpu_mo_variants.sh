mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_wd.so timeout -s KILL 600 python -m pytest tests/test_select_gpu.py tests/test_fission_gpu.py -x -q -p no:cacheprovider -k "not 2_pow_31" 2>&1 | tail -1
timeout -s KILL 600 python scripts/sweeps.py d2 gpurun_out/d2_sweep.txt; echo d2 rc=$?
