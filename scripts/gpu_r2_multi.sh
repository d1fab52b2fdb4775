# f2 (several SELECTs on one input): parity of the writer-warp kernel (watchdog
# build first: a stuck wait reports itself), then the M-output sweep
mkdir -p gpurun_out
RA_LIB_PATH=$PWD/build/libra_wd.so timeout -s KILL 400 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider -k "not past_2_pow and not full_size" 2>&1 | tail -12; echo wd-tests done
timeout -s KILL 400 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -5; echo tests done
timeout -s KILL 300 python scripts/multi_sweep.py 2>&1 | tee gpurun_out/multi_sweep.txt; echo sweep done
