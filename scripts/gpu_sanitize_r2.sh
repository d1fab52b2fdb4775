# round 2: compute-sanitizer over the warp-specialised multi-output pass (now also the fused chain),
# the exchange scan and the narrow Q1 change; memcheck + racecheck + synccheck
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
CS=/usr/local/cuda/bin/compute-sanitizer
K="test_single_select_sizes_and_alignment or test_extreme_predicates or test_selectivity_zero_one_identity or test_out_cap or unfused_workspace or epoch_tag"
timeout -s KILL 1200 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_gpu.py -q -x -p no:cacheprovider -k "$K" > gpurun_out/san2_select.log 2>&1; echo select memcheck rc=$?
timeout -s KILL 1200 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py -q -x -p no:cacheprovider -k "sizes_offsets or capacity or three_four or shared_across" > gpurun_out/san2_multi.log 2>&1; echo multi memcheck rc=$?
timeout -s KILL 1200 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py -q -x -p no:cacheprovider -k "sizes_offsets and (0-5 or 3-8193 or 0-42194)" > gpurun_out/san2_race_multi.log 2>&1; echo multi racecheck rc=$?
timeout -s KILL 1200 $CS --tool synccheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py tests/test_select_gpu.py -q -x -p no:cacheprovider -k "three_four or test_single_select_sizes_and_alignment" > gpurun_out/san2_sync.log 2>&1; echo synccheck rc=$?
timeout -s KILL 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_multi_rank_gpu.py tests/test_q1_narrow_gpu.py -q -x -p no:cacheprovider -k "offsets_kernel or encode_matches or domain or small" > gpurun_out/san2_misc.log 2>&1; echo misc memcheck rc=$?
timeout -s KILL 900 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_q1_narrow_gpu.py -q -x -p no:cacheprovider -k "small or encode_matches" > gpurun_out/san2_race_q1n.log 2>&1; echo q1n racecheck rc=$?
for f in gpurun_out/san2_*.log; do echo "== $f"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed|rror" $f | tail -4; done
