OUT=gpurun_out
rm -f $OUT/ab.txt
python -m pytest tests/test_gpu_parity.py tests/test_gpu_fanout.py -q -x -k "nlm" > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
for i in 1 2; do
for k in nlm_f4 nlm_f4_w; do
python bench.py --kernel $k --steps 100 --warmup 10 --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/x.log 2>&1
echo "c2 $k $(grep -o '"ms_per_step": [0-9.]*' $OUT/x.log)" >> $OUT/ab.txt
done; done
python tools/wave_probe.py nlm_f4_w -1 2048 2048 2001 1840 1817 > $OUT/wave.log 2>&1
python bench.py --workload c5 --kernel nlm_f4_w --steps 5 --warmup 3 > $OUT/c5w.log 2>&1
echo "c5 nlm_f4_w $(grep -o '"ms_per_step": [0-9.]*' $OUT/c5w.log)" >> $OUT/ab.txt
