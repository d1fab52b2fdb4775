# round 2: full GPU parity suite (select paths first on the watchdog build) + a headline bench line
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
RA_LIB_PATH=$PWD/build/libra_wd.so timeout -s KILL 600 python -m pytest tests/test_select_gpu.py tests/test_fission_gpu.py -x -q -p no:cacheprovider -k "not 2_pow_31" 2>&1 | tail -3; echo wd done
timeout -s KILL 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/gputest.log
timeout -s KILL 600 python bench.py --steps 50 --warmup 5 --no-extras > gpurun_out/head1.json 2> gpurun_out/head1.err; echo head rc=$?
cut -c1-600 gpurun_out/head1.json
