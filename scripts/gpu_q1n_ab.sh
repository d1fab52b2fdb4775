mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
$NCU --set full --import-source on --clock-control none -f -k regex:select_multi -s 2 -c 1 -o gpurun_out/prof_select_n30 python scripts/prof_driver.py select 3 30 > gpurun_out/ncu_n30.log 2>&1; echo n30 rc=$?
( timeout -s KILL 300 python scripts/prof_driver.py q1time 20
  RA_LIB_PATH=$PWD/build/libra_qs5.so timeout -s KILL 300 python scripts/prof_driver.py q1time 20
  RA_LIB_PATH=$PWD/build/libra_qs3.so timeout -s KILL 300 python scripts/prof_driver.py q1time 20 ) 2>&1 | grep narrow | tee gpurun_out/q1n_stages.txt
