#!/bin/bash
# A/B of the PDL no-wait launch (ORION_PDL_NOWAIT=1: independent frames backfill the previous
# grid's tail) against the default wait, on workload $1, $2 pairs.
WL=$1; N=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
for i in $(seq 1 $N); do
  for nw in 0 1; do
    ORION_PDL_NOWAIT=$nw python bench.py --workload $WL --only --rounds 3 --no-cpu-baseline --no-carveout-axis "$@" > $OUT/nw_last.log 2>&1
    echo "$WL nowait=$nw $(grep -o '"value": [0-9.]*' $OUT/nw_last.log | head -1) $(grep -o '"ms_per_step": [0-9.]*' $OUT/nw_last.log | head -1)" >> $OUT/nowait_ab.txt
  done
done
cat $OUT/nowait_ab.txt
