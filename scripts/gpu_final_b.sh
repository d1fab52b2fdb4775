# final round-2 evidence (part B): ncu --set full captures; $1 = list of capture names to take (keeps gpurun_out < 64 MiB)
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
F="--set full --import-source on --clock-control none -f"
cap() { $NCU $F -k regex:$1 -s $2 -c 1 -o gpurun_out/$3 python scripts/prof_driver.py ${@:4} > gpurun_out/ncu_$3.log 2>&1; echo $3 rc=$?; }
for c in $1; do
  case $c in
    select) cap select_multi 3 prof_select select 5 ;;
    n30) cap select_multi 2 prof_select_n30 select 3 30 ;;
    s01) cap select_multi 3 prof_select_s01 select 5 28 1 0.01 ;;
    s09) cap select_multi 3 prof_select_s09 select 5 28 1 0.9 ;;
    unfused) cap select_fused 3 prof_unfused unfused 3 ;;
    multi) cap select_multi 3 prof_multi multi 5 28 2 ;;
    multid) cap select_multi 3 prof_multi_dense multi 5 28 2 0.9 ;;
    multi4) cap select_multi 3 prof_multi4 multi 5 28 4 ;;
    q1) cap q1_tma 3 prof_q1 q1 5 ;;
    q1sf100) cap q1_tma 2 prof_q1_sf100 q1sf100 3 ;;
    q1n) cap q1n_ 3 prof_q1n q1n 5 ;;
    q1nsf100) cap q1n_ 2 prof_q1n_sf100 q1nsf100 3 ;;
    rows) cap select_fused 3 prof_rows rows 5 ;;
    compact) cap compact_kernel 3 prof_compact rows 5 ;;
  esac
done
du -sh gpurun_out
