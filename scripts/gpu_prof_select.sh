mkdir -p gpurun_out
make -s all 2>&1 | tail -3
/usr/local/cuda/bin/ncu --set full --import-source on --clock-control none -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_select -f python scripts/prof_driver.py select 5 > gpurun_out/ncu_select.log 2>&1; echo ncu select rc=$?
