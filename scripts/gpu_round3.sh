# one GPU call: tests, smoke, bench, ncu launch list + captures, f2 sweep, tuple A/B
mkdir -p gpurun_out
bash scripts/gpu_bench.sh
bash scripts/gpu_profiles.sh
python scripts/multi_sweep.py > gpurun_out/multi_sweep.txt 2>&1; echo multi rc=$?
bash scripts/gpu_rows_ab.sh > /dev/null 2>&1; echo rows_ab rc=$?
