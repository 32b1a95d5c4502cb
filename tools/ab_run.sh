OUT=gpurun_out
python -m pytest tests/test_gpu_parity.py tests/test_gpu_fanout.py -q -x -k "nlm" > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
for i in 1 2; do
python bench.py --steps 100 --warmup 10 --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/c2_nlm_f4_$i.log 2>&1
python bench.py --kernel nlm_f4_q --steps 100 --warmup 10 --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/c2_nlm_f4_q_$i.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "measure/" -k regex:orion_nlm_box4 -c 1 -f -o $OUT/prof_nlm_f4_q python tools/ncu_one.py nlm_f4_q best 2048 2048 > $OUT/ncu_q.log 2>&1
