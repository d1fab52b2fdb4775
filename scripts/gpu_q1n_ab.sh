# narrow Q1 A/B: libra.so vs build/libra_$V.so variants (q1time: SF10 and SF100, CUDA events)
mkdir -p gpurun_out
( for v in "" $VARIANTS; do
  echo "== ${v:-libra.so}"
  L=${v:+$PWD/build/libra_$v.so}
  RA_LIB_PATH=$L timeout -s KILL 300 python scripts/prof_driver.py q1time 20 | grep narrow
done ) 2>&1 | tee gpurun_out/q1n_ab.txt
