mkdir -p gpurun_out
make -s all >/dev/null 2>&1
python -m pytest tests/test_q1_narrow_gpu.py tests/test_q1_fission_gpu.py -q -x 2>&1 | tail -2
echo "== RED=1"; python scripts/prof_driver.py q1time 20 2>&1 | grep narrow
NVF="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -shared -Xptxas -v --expt-relaxed-constexpr -DRA_Q1N_RED=0"
make -s -B paper_conf_ipps_wudwcyc12_b200/libra.so "NVFLAGS=$NVF" >/dev/null 2>&1
echo "== RED=0"; python scripts/prof_driver.py q1time 20 2>&1 | grep narrow
