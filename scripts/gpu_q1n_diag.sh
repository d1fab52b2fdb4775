mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
( for v in "" slot0 slotl; do
  L=${v:+$PWD/build/libra_$v.so}
  echo "== ${v:-libra.so}"
  RA_LIB_PATH=$L timeout -s KILL 300 python scripts/prof_driver.py q1time 20 | grep narrow
  RA_LIB_PATH=$L $NCU --metrics gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum,smsp__inst_executed_op_shared_atom.sum -k regex:q1n_ -s 3 -c 1 python scripts/prof_driver.py q1n 5 2>&1 | grep -E "duration|atom|shared" | head -5
done ) > gpurun_out/q1n_diag.txt 2>&1
