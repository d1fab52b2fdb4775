# round 2 sweeps: d2 (fused vs unfused chain), d4 (fission chunk x streams), f2 multi-output sweep
mkdir -p gpurun_out
timeout -s KILL 600 python scripts/sweeps.py d2 gpurun_out/d2_sweep.txt; echo d2 rc=$?
timeout -s KILL 900 python scripts/sweeps.py d4 gpurun_out/d4_sweep.txt; echo d4 rc=$?
timeout -s KILL 300 python scripts/multi_sweep.py > gpurun_out/multi_sweep.txt 2>&1; echo multi rc=$?
