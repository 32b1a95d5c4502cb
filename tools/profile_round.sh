#!/bin/bash
# Run on the GPU box (gpurun): every bench workload, the launch list of the default bench
# command, and one ncu --set full capture per hot kernel.  Outputs land in gpurun_out/
# (scratch); tools/collect_round.sh copies the summaries into profiles/.
OUT=gpurun_out
python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
python bench.py > $OUT/bench_c2.log 2>&1
python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference.log 2>&1
python bench.py --workload c1 --cpu-seconds 5 > $OUT/bench_c1.log 2>&1
python bench.py --workload c3 --steps 25 --warmup 10 --cpu-seconds 5 > $OUT/bench_c3.log 2>&1
python bench.py --workload c3 --kernel hotspot2h_f32 --steps 50 --warmup 10 --no-cpu-baseline > $OUT/bench_c3_2step.log 2>&1
python bench.py --workload c3 --kernel hotspot_f32 --steps 100 --warmup 10 --no-cpu-baseline > $OUT/bench_c3_1step.log 2>&1
python bench.py --workload c4 --steps 20 --warmup 15 --rounds 3 --cpu-seconds 5 > $OUT/bench_c4.log 2>&1
python bench.py --workload c5 --steps 10 --warmup 5 > $OUT/bench_c5.log 2>&1
python bench.py --workload srad --steps 100 --warmup 12 --cpu-seconds 5 > $OUT/bench_srad.log 2>&1
[ -n "$SKIP_NCU" ] && exit 0
ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv --log-file $OUT/launches.csv \
    python bench.py --steps 20 --warmup 5 --rounds 3 --no-cpu-baseline --no-carveout-axis > $OUT/bench_under_ncu.log 2>&1
for spec in "nlm_f4 best 2048 2048 nlm_box3" "nlm_f4_w best 2048 2048 nlm_boxw3" "knn_f4 best 2048 2048 knn_f4" "knn_f4_p1 best 64 64 knn1" "knn_f4_t16 best 64 64 knn16" "nlm_f4_regheavy best 4096 4096 nlm_regheavy" \
            "hotspot_f32 best 8192 8192 hotspot_f32" "hotspot2h_f32 best 8192 8192 hotspot2h" "hotspot4h_f32 best 8192 8192 hotspot4h" "srad_f32 best 8192 8192 srad4" "srad_f32h best 8192 8192 srad4h"; do
  set -- $spec
  timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "measure/" -k regex:orion_$5 -c 1 -f -o $OUT/prof_$1 \
      python tools/ncu_one.py $1 $2 $3 $4 > $OUT/ncu_$1.log 2>&1
done
