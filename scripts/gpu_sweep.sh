# d2 sweep + full bench with the current kernels
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 300 python scripts/sweeps.py d2 gpurun_out/d2.txt > gpurun_out/d2.log 2>&1; echo d2 rc=$?
cat gpurun_out/d2.txt
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
