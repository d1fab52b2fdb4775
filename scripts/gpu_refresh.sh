# evidence refresh after a product change: parity suite, smoke, bench (+ reference arm), launch list,
# ncu --set full captures named in $CAPS (scripts/gpu_final_b.sh names)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout -s KILL 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/gputest.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
tail -1 gpurun_out/smoke.log
timeout -s KILL 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
timeout -s KILL 600 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref rc=$?
/usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-extras > gpurun_out/launches_bench.log 2>&1; echo launches rc=$?
[ -n "$CAPS" ] && bash scripts/gpu_final_b.sh "$CAPS"
du -sh gpurun_out
