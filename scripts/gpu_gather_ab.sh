mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
for v in "" g1 g2; do
  L=${v:+$PWD/build/libra_$v.so}
  RA_LIB_PATH=$L $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum -k regex:gather_kernel -s 3 -c 1 python scripts/prof_driver.py sparse 5 28 1 0.01 2>&1 | grep -E "gather_kernel|duration|bytes_read|sectors" | head -4
  RA_LIB_PATH=$L timeout -s KILL 200 python scripts/rows_ab.py 2>&1 | grep "s=.01"
done
