# tuple SELECT sparse path without caller ids: ids_kernel per set bit (libra.so)
# vs per vector (build/libra_ids0.so); then full captures of the sparse kernels.
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
( for v in "" ids0; do
  L=${v:+$PWD/build/libra_$v.so}
  echo "== ids variant ${v:-per-set-bit}"
  RA_LIB_PATH=$L $NCU --metrics gpu__time_duration.sum,smsp__inst_executed.sum,dram__bytes_read.sum -k regex:ids_kernel -s 3 -c 1 python scripts/prof_driver.py sparse 5 28 1 0.01 2>&1 | grep -E "duration|inst_exec|bytes_read" | head -3
  RA_LIB_PATH=$L timeout -s KILL 200 python scripts/rows_ab.py 2>&1 | grep "rowids=0"
done ) > gpurun_out/ids_ab.txt 2>&1
F="--set full --clock-control none --import-source on"
$NCU $F -k regex:ids_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_ids -f python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp2.log 2>&1; echo sp2 rc=$?
$NCU $F -k regex:gather_kernel -s 3 -c 1 -o gpurun_out/prof_sparse_gather -f python scripts/prof_driver.py sparse 5 28 1 0.01 > gpurun_out/ncu_sp3.log 2>&1; echo sp3 rc=$?
