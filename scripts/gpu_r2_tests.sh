# round 2: full GPU parity suite + a headline bench line (no extras)
mkdir -p gpurun_out
make -s all 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest.log 2>&1; echo pytest rc=$?
tail -15 gpurun_out/gputest.log
timeout 600 python bench.py --steps 50 --warmup 5 --no-extras > gpurun_out/head1.json 2> gpurun_out/head1.err; echo head rc=$?
cut -c1-400 gpurun_out/head1.json
