# tuple SELECT: payload compaction (device choice) vs the id gather (RA_TUPLE_GATHER=1), 2^28 rows
mkdir -p gpurun_out
( echo "== device choice (gather up to 1/10 [4-B fields] or 1/4 [8-B] selected with caller ids, 1/12 or 1/8 without (first n/32 ids staged by the key pass, the rest by ids_kernel), else streaming compaction)"
  timeout 300 python scripts/rows_ab.py
  echo "== RA_TUPLE_GATHER=1 (id gather always)"
  RA_TUPLE_GATHER=1 timeout 300 python scripts/rows_ab.py ) 2>&1 | tee gpurun_out/rows_ab.txt
