mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 900 python -m pytest tests/test_select_multi_gpu.py tests/test_select_gpu.py tests/test_select_rows_gpu.py -x -q > gpurun_out/pytest_multi.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/pytest_multi.log
