# functional check of bench.py's multi-rank path on a 1-GPU box: 2 ranks share
# cuda:0 over gloo (NCCL needs one GPU per rank); numbers are not bench values
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
RA_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 20 --warmup 3 --skip-1g \
  > gpurun_out/ranks2.json 2> gpurun_out/ranks2.err; echo ranks2 rc=$?
tail -5 gpurun_out/ranks2.err
timeout 600 python bench.py --steps 50 --warmup 5 --no-extras > gpurun_out/head1.json 2>&1; echo head1 rc=$?
cat gpurun_out/head1.json | cut -c1-300
