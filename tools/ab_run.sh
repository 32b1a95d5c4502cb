OUT=gpurun_out
python -m pytest tests/test_gpu_hotspot2.py tests/test_gpu_parity.py tests/test_gpu_run_host.py -q -x > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
python bench.py --workload c3 --steps 25 --warmup 10 --no-cpu-baseline > $OUT/c3.log 2>&1
