OUT=gpurun_out
python -m pytest tests/test_gpu_parity.py -q -x -k "full_size" > $OUT/t1.log 2>&1
echo "tests rc=$?" >> $OUT/t1.log
python tools/ncu_levels.py run hotspot4h_f32 8192 8192 > $OUT/lv1.log 2>&1
python tools/ncu_levels.py run knn_f4_t8 64 64 > $OUT/lv2.log 2>&1
python tools/ncu_levels.py run nlm_f4 2048 2048 > $OUT/lv3.log 2>&1
