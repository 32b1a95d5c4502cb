OUT=gpurun_out
rm -f $OUT/ab.txt
python -m pytest tests/test_gpu_parity.py tests/test_gpu_fanout.py -q -x -k "knn" > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
for i in 1 2; do
for k in knn_f4_p1 knn_f4_t8; do
python bench.py --workload c1 --kernel $k --steps 300 --warmup 20 --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/c1_$k.log 2>&1
echo "c1 $k $(grep -o '"ms_per_step": [0-9.]*' $OUT/c1_$k.log)" >> $OUT/ab.txt
done; done
timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "measure/" -k regex:orion_knn8 -c 1 -f -o $OUT/prof_knn_f4_t8 python tools/ncu_one.py knn_f4_t8 best 64 64 > $OUT/ncu_t8.log 2>&1
