mkdir -p gpurun_out
( for b in scripts/micro/selw_1_1_768_3_1 scripts/micro/selw_swar scripts/micro/selw_1_1_768_3_1 scripts/micro/selw_swar; do
  for t in -1073741824 0 -2104533975 1717986918; do timeout 60 $b $t || echo "$b $t FAILED"; done
done ) 2>&1 | tee gpurun_out/variants.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 600 python bench.py --no-extras > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
cat gpurun_out/bench.json
