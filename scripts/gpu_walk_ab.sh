# sparse-scatter walk A/B: parity of the default build, then fused-only f2 sweep per variant
mkdir -p gpurun_out
timeout -s KILL 900 python -m pytest tests/test_select_gpu.py tests/test_select_multi_gpu.py -x -q -p no:cacheprovider 2>&1 | tail -2
for v in "" $VARIANTS; do
  if [ -n "$v" ]; then export RA_LIB_PATH=$PWD/build/libra_$v.so; fi
  echo "== ${v:-default}"; MS_FUSED_ONLY=1 timeout -s KILL 200 python scripts/multi_sweep.py 2>&1 | tail -22
done 2>&1 | tee gpurun_out/walk_ab.txt
