#!/bin/bash
# Run on the GPU box (gpurun): the GPU tests + smoke, the default bench line (every config in
# one line), the reference arm, the launch list of the headline's timed region, and one
# ncu --set full capture per default kernel.  Outputs land in gpurun_out/ (scratch);
# tools/collect_round.sh ROUND copies the summaries into profiles/.
OUT=gpurun_out
mkdir -p $OUT
if [ -z "$SKIP_TESTS" ]; then
  python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1
  python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
fi
python bench.py > $OUT/bench_default.log 2>&1
python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference.log 2>&1
[ -n "$SKIP_NCU" ] && exit 0
ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv --log-file $OUT/launches.csv \
    python bench.py --only --steps 20 --warmup 5 --rounds 3 --no-cpu-baseline --no-carveout-axis > $OUT/bench_under_ncu.log 2>&1
for spec in "nlm_f4_w best 2048 2048 nlm_boxw3" "nlm_f4 best 2048 2048 nlm_box3" "knn_f4_t16 best 64 64 knn16" "knn_f4 best 64 64 knn_f4_256 256 1 256" \
            "nlm_f4_regheavy best 4096 4096 nlm_regheavy" "hotspot4h_f32 best 8192 8192 hotspot4h" \
            "hotspot_f32 best 8192 8192 hotspot_f32" "srad_f32hs best 8192 8192 srad4hs" "srad_f32h best 8192 8192 srad4h" $EXTRA_NCU; do
  set -- $spec
  timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "measure/" -k regex:orion_$5 -c 1 -f -o $OUT/prof_$1 \
      python tools/ncu_one.py $1 $2 $3 $4 $6 $7 $8 > $OUT/ncu_$1.log 2>&1
done
