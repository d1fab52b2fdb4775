mkdir -p gpurun_out
make -s all 2>&1 | tail -3
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py tests/test_select_rows_gpu.py -q -x -k "test_single_select_sizes_and_alignment or sizes_offsets" > gpurun_out/san_race_select.log 2>&1; echo select racecheck rc=$?
grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_race_select.log | tail -3
bash scripts/gpu_selvar.sh "8,1,10240,1,1,3"
