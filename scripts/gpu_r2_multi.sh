mkdir -p gpurun_out
timeout -s KILL 300 python scripts/fig12.py full 2>&1 | tee gpurun_out/fig12_full.txt
RA_SEL_MAX_CTAS=74 timeout -s KILL 300 python scripts/fig12.py half 2>&1 | tee gpurun_out/fig12_half.txt
timeout -s KILL 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench rc=$?
