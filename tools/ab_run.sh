python tools/wave_probe.py nlm_f4 -1 2048 2048 2001 1978 1955 1932 1817 1564 1541 1196 > gpurun_out/wave.log 2>&1
