mkdir -p gpurun_out
make -s all 2>&1 | tail -3
NCU=/usr/local/cuda/bin/ncu
$NCU --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select -f python scripts/prof_driver.py select 5 > gpurun_out/ncu_select.log 2>&1; echo ncu select rc=$?
$NCU --set full --import-source on --clock-control none -k regex:q1_fused -s 3 -c 1 -o gpurun_out/prof_q1 -f python scripts/prof_driver.py q1 5 > gpurun_out/ncu_q1.log 2>&1; echo ncu q1 rc=$?
tail -3 gpurun_out/ncu_select.log gpurun_out/ncu_q1.log
