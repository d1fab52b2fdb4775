mkdir -p gpurun_out
( RA_SEL_SMALL_ROWS=0 timeout -s KILL 120 python scripts/small_n.py
  RA_SEL_SMALL_ROWS=1000000000000 timeout -s KILL 120 python scripts/small_n.py ) 2>&1 | tee gpurun_out/small_n.txt
