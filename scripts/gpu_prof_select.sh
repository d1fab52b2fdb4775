# ncu --set full of the fused select at 2^28: headline (k=2, s=.5/stage) and s=.01 (k=1)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
NCU="/usr/local/cuda/bin/ncu --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -f"
$NCU -o gpurun_out/prof_select python scripts/prof_driver.py select 5 > gpurun_out/ncu_select.log 2>&1; echo ncu select rc=$?
$NCU -o gpurun_out/prof_select_s01 python scripts/prof_driver.py select 5 28 1 0.01 > gpurun_out/ncu_select_s01.log 2>&1; echo ncu s01 rc=$?
