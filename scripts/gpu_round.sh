# one GPU call: build, new tests, sweeps, bench (outputs under gpurun_out/)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 600 python -m pytest tests/test_q1_fission_gpu.py -x -q > gpurun_out/pytest_q1f.log 2>&1; echo q1f rc=$?; tail -3 gpurun_out/pytest_q1f.log
timeout 300 python scripts/sweeps.py d2 gpurun_out/d2.txt > gpurun_out/d2.log 2>&1; echo d2 rc=$?
timeout 600 python scripts/sweeps.py d4 gpurun_out/d4.txt > gpurun_out/d4.log 2>&1; echo d4 rc=$?
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
