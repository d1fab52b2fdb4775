mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
K="sizes_offsets and (0-5 or 3-8193 or 0-42194)"
timeout -s KILL 600 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py -q -x -p no:cacheprovider -k "$K" > gpurun_out/san2_race_multi.log 2>&1; echo multi racecheck rc=$?
RA_LIB_PATH=$PWD/build/libra_scat256.so timeout -s KILL 600 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_select_multi_gpu.py -q -x -p no:cacheprovider -k "$K" > gpurun_out/san2_race_multi256.log 2>&1; echo multi256 racecheck rc=$?
for f in gpurun_out/san2_race_multi*.log; do echo "== $f"; grep -E "RACECHECK SUMMARY|passed" $f; grep -A1 "Race reported" $f | grep -oE "(Read|Write) access at [^+]*\+0x[0-9a-f]+ in select_multi.cu:[0-9]+|and (Read|Write) access at [^+]*\+0x[0-9a-f]+ in select_multi.cu:[0-9]+" | sed 's/+0x[0-9a-f]*//' | sort | uniq -c | sort -rn | head; done
timeout -s KILL 120 python scripts/mo_quick.py
RA_LIB_PATH=$PWD/build/libra_scat256.so timeout -s KILL 120 python scripts/mo_quick.py
