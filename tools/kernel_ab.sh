#!/bin/bash
# A/B timing of kernel ids of one family on ONE box (gpurun): bench.py --only on workload $1 with
# each kernel id in turn, $2 rounds; ms_per_step and the sweep's best level appended to
# gpurun_out/kernel_ab.txt.   usage: bash tools/kernel_ab.sh c3 3 hotspot4h_f32 hotspot4t_f32
WL=$1; N=$2; shift 2
OUT=gpurun_out; mkdir -p $OUT
for i in $(seq 1 $N); do
  for k in "$@"; do
    python bench.py --workload $WL --only --kernel $k --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/kab_last.log 2>&1
    echo "$WL $k $(grep -o '"value": [0-9.]*' $OUT/kab_last.log | head -1) $(grep -o '"ms_per_step": [0-9.]*' $OUT/kab_last.log) $(grep -o '"ms_best": [0-9.]*' $OUT/kab_last.log | head -1)" >> $OUT/kernel_ab.txt
  done
done
cat $OUT/kernel_ab.txt
