# Build (here) and run (on the box) select kernel variants: VEC,AHEAD,OUTRING,D1,D2,LAG[,EXTRA_DEFINE]
# usage: bash scripts/sel_variants.sh build|run "8,1,10240,2,4,5 ..."
set -e
V=${2:-"8,1,10240,2,4,5"}
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -Iinclude"
for v in $V; do
  IFS=, read vec ah ring d1 d2 lag extra <<< "$v"
  tag=${vec}_${ah}_${ring}_${d1}_${d2}_${lag}${extra:+_$extra}
  ex=${extra:+-D${extra//+/ -D}}
  b=scripts/micro/selv_$tag
  if [ "$1" = build ]; then
    $NV -DRA_SEL_VEC=$vec -DRA_SEL_AHEAD=$ah -DRA_SEL_OUTRING=$ring -DRA_SEL_D1=$d1 -DRA_SEL_D2=$d2 -DRA_SEL_LAG=$lag $ex \
      -DVARIANT="\"$tag\"" -o $b scripts/micro/sel_prof.cu -lpthread &
  else
    for t in -1073741824 0 -2104533975; do timeout 60 $b $t || echo "$b $t FAILED"; done
  fi
done
wait
