# narrow Q1: per-warp flush sums vs CTA shared 64-bit atomics; parity + timings
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_q1_narrow_gpu.py tests/test_q1_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -2
( timeout -s KILL 300 python scripts/prof_driver.py q1time 20
  RA_LIB_PATH=$PWD/build/libra_q1nold.so timeout -s KILL 300 python scripts/prof_driver.py q1time 20 ) 2>&1 | tee gpurun_out/q1n_ab.txt
