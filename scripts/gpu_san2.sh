# compute-sanitizer over the f2 spill path and the tuple-select kernels (round 1, second pass)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py -q -x -k "dense or sizes_offsets or capacity" > gpurun_out/san_multi2.log 2>&1; echo multi memcheck rc=$?
timeout 900 $CS --tool racecheck python -m pytest tests/test_select_multi_gpu.py -q -x -k "dense" > gpurun_out/san_race_multi2.log 2>&1; echo multi racecheck rc=$?
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py -q -x -k "phases or never_writes or both_payload or sizes_offsets" > gpurun_out/san_rows2.log 2>&1; echo rows memcheck rc=$?
timeout 900 $CS --tool racecheck python -m pytest tests/test_select_rows_gpu.py -q -x -k "both_payload" > gpurun_out/san_race_rows2.log 2>&1; echo rows racecheck rc=$?
for f in gpurun_out/san_multi2.log gpurun_out/san_race_multi2.log gpurun_out/san_rows2.log gpurun_out/san_race_rows2.log; do
  echo "== $f"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" $f | tail -3
  grep -E "Race reported|Error:" -A2 $f | grep -E "at .* in [a-z_]+\.cu:[0-9]+" | sed 's/.*in \([a-z_]*\.cu:[0-9]*\).*/\1/' | sort | uniq -c
done
timeout 900 python bench.py --steps 50 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
