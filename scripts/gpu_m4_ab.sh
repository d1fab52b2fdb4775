# select_multi variants for M>=3: parity (multi tests) then m4_quick per variant, twice (VARIANTS="a b")
for v in $VARIANTS; do RA_LIB_PATH=$PWD/build/libra_$v.so timeout -s KILL 300 python -m pytest tests/test_select_multi_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -1; done
for r in 1 2; do for v in "" $VARIANTS; do if [ -n "$v" ]; then export RA_LIB_PATH=$PWD/build/libra_$v.so; else unset RA_LIB_PATH; fi; timeout -s KILL 100 python scripts/m4_quick.py; done; done
