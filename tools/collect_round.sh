#!/bin/bash
# Copy a profile_round.sh run from gpurun_out/ into profiles/ (round tag $1, default r01).
R=${1:-r01}
for w in c1 c2 c3 c3_2step c3_1step c4 c5 srad reference; do
  grep '^{' gpurun_out/bench_$w.log > profiles/bench_${R}_$w.json 2>/dev/null || true
done
python tools/launch_summary.py gpurun_out/launches.csv profiles/launches_${R}_bench_c2.txt \
  "ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include timed/ python bench.py --steps 20 --warmup 5 --rounds 3 --no-cpu-baseline --no-carveout-axis (the timed region only)"
for k in nlm_f4 nlm_f4_w knn_f4 knn_f4_p1 knn_f4_t16 nlm_f4_regheavy hotspot_f32 hotspot2h_f32 hotspot4h_f32 srad_f32 srad_f32h; do
  [ -f gpurun_out/prof_$k.ncu-rep ] && python tools/ncu_summary.py $k gpurun_out/prof_$k.ncu-rep $R > /dev/null
done
ls profiles
