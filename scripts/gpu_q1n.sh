mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 600 python -m pytest tests/test_q1_narrow_gpu.py -x -q > gpurun_out/pytest_q1n.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/pytest_q1n.log
timeout 300 python scripts/prof_driver.py q1time 20 > gpurun_out/q1time.log 2>&1; echo q1time rc=$?
cat gpurun_out/q1time.log
/usr/local/cuda/bin/ncu --set full --import-source on --clock-control none -k regex:q1n_ -s 3 -c 1 -o gpurun_out/prof_q1n -f python scripts/prof_driver.py q1n 5 > gpurun_out/ncu_q1n.log 2>&1; echo ncu rc=$?
