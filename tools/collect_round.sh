#!/bin/bash
# Copy a profile_round.sh run from gpurun_out/ into profiles/ (round tag $1, default r02).
R=${1:-r02}
grep '^{' gpurun_out/bench_default.log > profiles/bench_${R}.json 2>/dev/null || true
grep '^{' gpurun_out/bench_reference.log > profiles/bench_${R}_reference.json 2>/dev/null || true
[ -f gpurun_out/pytest_gpu.log ] && tail -3 gpurun_out/pytest_gpu.log > profiles/gpu_tests_${R}.txt && cat gpurun_out/smoke.log >> profiles/gpu_tests_${R}.txt
[ -f gpurun_out/launches.csv ] && python tools/launch_summary.py gpurun_out/launches.csv profiles/launches_${R}_bench_c2.txt \
  "ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include timed/ python bench.py --only --steps 20 --warmup 5 --rounds 3 --no-cpu-baseline --no-carveout-axis (the timed region only)"
for k in nlm_f4_w nlm_f4 knn_f4_t16 nlm_f4_regheavy hotspot4h_f32 hotspot_f32 srad_f32hs srad_f32h srad_f32 hotspot2h_f32 knn_f4; do
  [ -f gpurun_out/prof_$k.ncu-rep ] && python tools/ncu_summary.py $k gpurun_out/prof_$k.ncu-rep $R > /dev/null
done
ls profiles
