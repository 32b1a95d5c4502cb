OUT=gpurun_out
python -m pytest tests/test_gpu_hotspot2.py tests/test_gpu_parity.py tests/test_gpu_run_host.py -q -x -k "hotspot" > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
rm -f $OUT/c3_ab.txt
for k in hotspot4h_f32 hotspot4p_f32 hotspot4h_f32 hotspot4p_f32; do
python bench.py --workload c3 --kernel $k --steps 25 --warmup 6 --rounds 5 --no-cpu-baseline --no-carveout-axis > $OUT/c3_$k.log 2>&1
grep -o '"ms_per_step": [0-9.]*' $OUT/c3_$k.log >> $OUT/c3_ab.txt; echo $k >> $OUT/c3_ab.txt
done
timeout 600 ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "measure/" -k regex:orion_hotspot4p -c 1 -f -o $OUT/prof_hotspot4p_f32 python tools/ncu_one.py hotspot4p_f32 best 8192 8192 > $OUT/ncu_4p.log 2>&1
