# tuple SELECT without caller ids: how many ids the key pass stages (cap) and
# the gather/compaction crossover (den), 2^28 rows (scripts/rows_ab.py)
mkdir -p gpurun_out
( echo "== default (stage n/32, den 12 | 8)"
  timeout -s KILL 200 python scripts/rows_ab.py 2>&1 | grep "rowids=0"
  for c in 4194304 16777216; do echo "== stage cap $c"; RA_TMP_CAP=$c timeout -s KILL 200 python scripts/rows_ab.py 2>&1 | grep "rowids=0"; done
  for d in 10 16; do echo "== den $d"; RA_TMP_DEN=$d timeout -s KILL 200 python scripts/rows_ab.py 2>&1 | grep "rowids=0" | grep "s=.0\|s=.1 "; done
) > gpurun_out/stage_ab.txt 2>&1
