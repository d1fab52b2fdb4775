# narrow Q1 variants: rebuild libra.so with extra defines, time SF10/SF100 (scripts/prof_driver.py q1time)
mkdir -p gpurun_out
NVF0="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -shared -Xptxas -v --expt-relaxed-constexpr"
for defs in "$@"; do
  make -s -B paper_conf_ipps_wudwcyc12_b200/libra.so "NVFLAGS=$NVF0 $defs" >/dev/null 2>&1 || { echo "build $defs FAILED"; continue; }
  echo "== $defs"; python scripts/prof_driver.py q1time 20 2>&1 | grep narrow
done
make -s -B all >/dev/null 2>&1
