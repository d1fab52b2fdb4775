mkdir -p gpurun_out
( for v in nlb3w4 nlb4w3 nlb3w8 nlb4w7 nlb3w4d2; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 120 python scripts/mo_quick.py; done ) 2>&1 | tee gpurun_out/mo_variants12.txt
