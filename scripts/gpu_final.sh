# full parity suite, smoke, full bench line, and the ncu captures whose kernels changed
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout -s KILL 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/gputest.log
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout -s KILL 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-extras > gpurun_out/launches_bench.log 2>&1; echo launches rc=$?
cap() { $NCU $F -k regex:$1 -s $2 -c 1 -o gpurun_out/$3 python scripts/prof_driver.py ${@:4} > gpurun_out/ncu_$3.log 2>&1; echo $3 rc=$?; }
cap select_multi 3 prof_select select 5
cap select_multi 3 prof_select_s01 select 5 28 1 0.01
cap select_multi 3 prof_multi multi 5 28 2
cap select_multi 3 prof_multi_dense multi 5 28 2 0.9
cap select_multi 3 prof_multi4 multi 5 28 4
cap q1n_ 2 prof_q1n_sf100 q1nsf100 3
cap q1n_ 3 prof_q1n q1n 5
