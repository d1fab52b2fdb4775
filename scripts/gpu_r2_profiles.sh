# round 2 ncu evidence: SF100 Q1 (wide, narrow), f2 M=2 (bench pair + dense pair),
# sparse tuple path, PCIe bytes of the fission paths (app-range replay)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
$NCU $F -k regex:q1_tma -s 2 -c 1 -o gpurun_out/prof_q1_sf100 python scripts/prof_driver.py q1sf100 3 > gpurun_out/ncu_q1_sf100.log 2>&1; echo q1sf100 rc=$?
$NCU $F -k regex:q1n_ -s 2 -c 1 -o gpurun_out/prof_q1n_sf100 python scripts/prof_driver.py q1nsf100 3 > gpurun_out/ncu_q1n_sf100.log 2>&1; echo q1nsf100 rc=$?
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_multi python scripts/prof_driver.py multi 5 28 2 > gpurun_out/ncu_multi.log 2>&1; echo multi rc=$?
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_multi_dense python scripts/prof_driver.py multi 5 28 2 0.9 > gpurun_out/ncu_multi_dense.log 2>&1; echo multid rc=$?
$NCU $F -k regex:select_fused -s 3 -c 1 -o gpurun_out/prof_sparse_sel python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp1.log 2>&1; echo sp1 rc=$?
$NCU $F -k regex:ids_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_ids python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp2.log 2>&1; echo sp2 rc=$?
$NCU $F -k regex:gather_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_gather python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp3.log 2>&1; echo sp3 rc=$?
$NCU --replay-mode app-range --profile-from-start off --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/pcie.csv python scripts/pcie_ranges.py > gpurun_out/pcie.log 2>&1; echo pcie rc=$?
tail -5 gpurun_out/pcie.log
python scripts/pcie_ranges.py > gpurun_out/pcie_timed.log 2>&1; echo pcie_timed rc=$?
cat gpurun_out/pcie_timed.log
ls -la gpurun_out/*.ncu-rep
