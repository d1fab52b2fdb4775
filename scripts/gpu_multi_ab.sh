# f2 variants: rebuild libra.so with extra defines, run scripts/multi_sweep.py for each
mkdir -p gpurun_out
NVF0="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -shared -Xptxas -v --expt-relaxed-constexpr"
for defs in "$@"; do
  make -s -B paper_conf_ipps_wudwcyc12_b200/libra.so "NVFLAGS=$NVF0 $defs" >/dev/null 2>&1 || { echo "build $defs FAILED"; continue; }
  echo "== $defs"; python scripts/multi_sweep.py 2>&1 | tail -7
done
make -s -B all >/dev/null 2>&1
