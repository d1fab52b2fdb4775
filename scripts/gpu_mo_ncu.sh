# ncu --set full of select_multi_kernel<1> at s=0.01 and <2> at (.5,.5) (2^28 rows)
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
$NCU $F -k regex:select_multi -s 3 -c 1 -o gpurun_out/prof_mo1_s001 python scripts/prof_driver.py multi1 5 28 1 0.01 > gpurun_out/ncu_mo1.log 2>&1; echo mo1 rc=$?
$NCU $F -k regex:select_multi -s 3 -c 1 -o gpurun_out/prof_multi python scripts/prof_driver.py multi 5 28 2 > gpurun_out/ncu_multi.log 2>&1; echo multi rc=$?
$NCU $F -k regex:select_multi -s 3 -c 1 -o gpurun_out/prof_multi_dense python scripts/prof_driver.py multi 5 28 2 0.9 > gpurun_out/ncu_multid.log 2>&1; echo multid rc=$?
