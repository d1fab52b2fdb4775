timeout -s KILL 300 python -m pytest tests/test_q1_narrow_gpu.py tests/test_q1_fission_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -1
RA_LIB_PATH=$PWD/build/libra_mot2.so timeout -s KILL 300 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -1
for v in "" q1t1 q1t2 q1t8 q1old; do if [ -n "$v" ]; then export RA_LIB_PATH=$PWD/build/libra_$v.so; else unset RA_LIB_PATH; fi; timeout -s KILL 200 python scripts/q1_quick.py; done
for v in old mot2 mot4 old mot2 mot4; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 100 python scripts/mo_m1.py 2>&1 | tail -1; done
for v in old mot2 mot4; do RA_LIB_PATH=$PWD/build/libra_$v.so MS_FUSED_ONLY=1 timeout -s KILL 100 python scripts/multi_sweep.py 2>&1 | tail -16 | head -8; done
