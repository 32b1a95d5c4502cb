#!/bin/bash
# Run on the GPU box (gpurun): launch list of the bench command + one ncu --set full capture
# per hot kernel.  Outputs land in gpurun_out/ (scratch); summaries are copied to profiles/.
set -x
OUT=gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 20 --warmup 5 --rounds 3 --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1
for spec in "nlm_f4 -1 2048 2048 nlm_box" "knn_f4 -1 2048 2048 knn" "nlm_f4_regheavy orig 4096 4096 nlm_regheavy" \
            "hotspot_f32 -1 8192 8192 hotspot"; do
  set -- $spec
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:orion_$5 -c 1 -f -o $OUT/prof_$1 \
      python tools/ncu_one.py $1 $2 $3 $4 > $OUT/ncu_$1.log 2>&1
done
