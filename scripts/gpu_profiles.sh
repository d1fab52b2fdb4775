# ncu evidence for profiles/: launch list of the bench command, full captures of the top kernels
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
NCU=/usr/local/cuda/bin/ncu
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-extras > gpurun_out/launches_bench.log 2>&1; echo launches rc=$?
$NCU --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select -f python scripts/prof_driver.py select 5 > gpurun_out/ncu_select.log 2>&1; echo select rc=$?
$NCU --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select_s01 -f python scripts/prof_driver.py select 5 28 1 0.01 > gpurun_out/ncu_select01.log 2>&1; echo select01 rc=$?
$NCU --set full --import-source on --clock-control none -k regex:q1_tma -s 3 -c 1 -o gpurun_out/prof_q1 -f python scripts/prof_driver.py q1 5 > gpurun_out/ncu_q1.log 2>&1; echo q1 rc=$?
$NCU --set full --import-source on --clock-control none -k regex:q1n_ -s 3 -c 1 -o gpurun_out/prof_q1n -f python scripts/prof_driver.py q1n 5 > gpurun_out/ncu_q1n.log 2>&1; echo q1n rc=$?
$NCU --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_rows -f python scripts/prof_driver.py rows 5 > gpurun_out/ncu_rows.log 2>&1; echo rows rc=$?
$NCU --set full --import-source on --clock-control none -k regex:compact_kernel -s 3 -c 1 -o gpurun_out/prof_compact -f python scripts/prof_driver.py rows 5 > gpurun_out/ncu_compact.log 2>&1; echo compact rc=$?
