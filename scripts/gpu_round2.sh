# one GPU call: tests, smoke, bench, tuple A/B, ncu profiles, sanitizer on the tuple-select kernels
mkdir -p gpurun_out
bash scripts/gpu_bench.sh
bash scripts/gpu_rows_ab.sh > /dev/null 2>&1; echo rows_ab rc=$?
bash scripts/gpu_profiles.sh
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py -q -x -k "phases or never_writes or both_payload or sizes_offsets" > gpurun_out/san_rows2.log 2>&1; echo rows2 memcheck rc=$?
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py -q -x -k "both_payload" > gpurun_out/san_race_rows.log 2>&1; echo rows racecheck rc=$?
for f in gpurun_out/san_rows2.log gpurun_out/san_race_rows.log; do echo "== $f"; grep -E "ERROR SUMMARY|hazard|passed|failed" $f | tail -3; done
