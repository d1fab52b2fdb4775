# final round-2 evidence (part A): parity suite, smoke, bench (+ reference arm), launch list, PCIe ranges, sweeps
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout -s KILL 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/gputest.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout -s KILL 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
timeout -s KILL 600 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref rc=$?
NCU=/usr/local/cuda/bin/ncu
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-extras > gpurun_out/launches_bench.log 2>&1; echo launches rc=$?
$NCU --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/pcie.csv python scripts/pcie_ranges.py > gpurun_out/pcie.log 2>&1; echo pcie rc=$?
timeout -s KILL 600 python scripts/sweeps.py d2 gpurun_out/d2_sweep.txt; echo d2 rc=$?
timeout -s KILL 300 python scripts/multi_sweep.py > gpurun_out/multi_sweep.txt 2>&1; echo multi rc=$?
du -sh gpurun_out
