# select kernel variant sweep (built here by sel_variants.sh build)
mkdir -p gpurun_out
V="$1"
( for v in $V; do
  IFS=, read vec ah ring d1 d2 lag extra <<< "$v"
  tag=${vec}_${ah}_${ring}_${d1}_${d2}_${lag}${extra:+_$extra}
  b=scripts/micro/selv_$tag
  for t in -2104533975 -1073741824 0 1717986918; do timeout 60 $b $t || echo "$b $t FAILED"; done
done ) 2>&1 | tee gpurun_out/variants.txt
