# f2 (several SELECTs on one input): parity (watchdog build, then the product
# build), the M-output sweep, the paper's Fig 12 experiment, a cycle profile
mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_wd.so timeout -s KILL 400 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not past_2_pow and not full_size" 2>&1 | tail -2; echo wd-tests done
timeout -s KILL 600 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -2; echo tests done
timeout -s KILL 300 python scripts/multi_sweep.py 2>&1 | tee gpurun_out/multi_sweep.txt; echo sweep done
timeout -s KILL 300 python scripts/fig12.py full 2>&1 | tee gpurun_out/fig12_full.txt
RA_SEL_MAX_CTAS=148 timeout -s KILL 300 python scripts/fig12.py half 2>&1 | tee gpurun_out/fig12_half.txt
RA_LIB_PATH=$PWD/build/libra_prof.so timeout -s KILL 120 python scripts/mo_prof.py 2>&1 | tee gpurun_out/mo_prof.txt
