# compute-sanitizer over small-size parity tests of every kernel (memcheck; racecheck/synccheck on a subset)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
CS=/usr/local/cuda/bin/compute-sanitizer
K="test_single_select_sizes_and_alignment or test_extreme_predicates or test_selectivity_zero_one_identity or test_out_cap"
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_gpu.py -q -x -k "$K" > gpurun_out/san_select.log 2>&1; echo select memcheck rc=$?
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_q1_gpu.py -q -x -k "small_sizes or cutoffs or columns_not" > gpurun_out/san_q1.log 2>&1; echo q1 memcheck rc=$?
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_q1_narrow_gpu.py -q -x -k "encode_matches or domain" > gpurun_out/san_q1n.log 2>&1; echo q1n memcheck rc=$?
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py tests/test_select_multi_gpu.py -q -x -k "sizes_offsets or table1 or capacity" > gpurun_out/san_rows.log 2>&1; echo rows/multi memcheck rc=$?
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_gpu.py -q -x -k "test_single_select_sizes_and_alignment" > gpurun_out/san_race_select.log 2>&1; echo select racecheck rc=$?
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_q1_gpu.py tests/test_q1_narrow_gpu.py -q -x -k "small_sizes or encode_matches" > gpurun_out/san_race_q1.log 2>&1; echo q1 racecheck rc=$?
timeout 900 $CS --tool synccheck --error-exitcode 9 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py -q -x -k "test_single_select_sizes_and_alignment or sizes_offsets" > gpurun_out/san_sync.log 2>&1; echo synccheck rc=$?
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py -q -x -k "phases or never_writes or both_payload" > gpurun_out/san_rows2.log 2>&1; echo rows2 memcheck rc=$?
timeout 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_rows_gpu.py -q -x -k "both_payload" > gpurun_out/san_race_rows.log 2>&1; echo rows racecheck rc=$?
for f in gpurun_out/san_*.log; do echo "== $f"; grep -E "ERROR SUMMARY|passed|failed|Error" $f | tail -3; done
