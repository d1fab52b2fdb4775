mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
$NCU $F -k regex:select_multi -s 3 -c 1 -o gpurun_out/prof_mo1_s001 python scripts/prof_driver.py multi1 5 28 1 0.01 > gpurun_out/ncu_mo1.log 2>&1; echo mo1 rc=$?
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select_s01 python scripts/prof_driver.py select 5 28 1 0.01 > gpurun_out/ncu_sel01.log 2>&1; echo sel01 rc=$?
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select python scripts/prof_driver.py select 5 > gpurun_out/ncu_sel.log 2>&1; echo sel rc=$?
