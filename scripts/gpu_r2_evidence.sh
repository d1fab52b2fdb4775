# round 2 ncu evidence for profiles/: launch list of the bench headline, --set full
# captures of every hot kernel at bench shapes, PCIe bytes of the fission paths
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-extras > gpurun_out/launches_bench.log 2>&1; echo launches rc=$?
cap() { $NCU $F -k regex:$1 -s $2 -c 1 -o gpurun_out/$3 python scripts/prof_driver.py ${@:4} > gpurun_out/ncu_$3.log 2>&1; echo $3 rc=$?; }
cap select_multi 3 prof_select select 5
cap select_multi 3 prof_select_s01 select 5 28 1 0.01
cap select_multi 3 prof_select_s09 select 5 28 1 0.9
cap select_fused 3 prof_unfused unfused 3
cap select_multi 3 prof_multi multi 5 28 2
cap select_multi 3 prof_multi_dense multi 5 28 2 0.9
cap select_multi 3 prof_multi4 multi 5 28 4
cap q1_tma 3 prof_q1 q1 5
cap q1n_ 3 prof_q1n q1n 5
cap select_fused 3 prof_rows rows 5
cap compact_kernel 3 prof_compact rows 5
$NCU --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/pcie.csv python scripts/pcie_ranges.py > gpurun_out/pcie.log 2>&1; echo pcie rc=$?
tail -3 gpurun_out/pcie.log; head -5 gpurun_out/pcie.csv
