# re-entry check: parity suite, smoke, headline bench line
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout -s KILL 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/gputest.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
tail -3 gpurun_out/smoke.log
timeout -s KILL 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
tail -3 gpurun_out/bench.err
cut -c1-400 gpurun_out/bench.json
