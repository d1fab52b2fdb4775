# ncu --set full captures of the tuple SELECT's sparse path (no caller ids)
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
F="--set full --clock-control none --import-source on -f"
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_sparse_sel python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp1.log 2>&1; echo sp1 rc=$?
$NCU $F -k regex:ids_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_ids python scripts/prof_driver.py sparse 5 28 1 0.05 > gpurun_out/ncu_sp2.log 2>&1; echo sp2 rc=$?
$NCU $F -k regex:gather_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_gather python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp3.log 2>&1; echo sp3 rc=$?
