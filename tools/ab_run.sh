OUT=gpurun_out
rm -f $OUT/ab.txt
python -m pytest tests/test_gpu_srad.py -q -x > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
for i in 1 2 3; do
for lib in build/liborion_old.so paper_conf_middleware_hayeslcsz16_b200/liborion.so; do
ORION_LIB=$lib python bench.py --workload srad --steps 100 --warmup 12 --rounds 3 --no-cpu-baseline --no-carveout-axis > $OUT/x.log 2>&1
echo "srad $lib $(grep -o '"ms_per_step": [0-9.]*' $OUT/x.log)" >> $OUT/ab.txt
done; done
