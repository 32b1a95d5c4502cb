#!/bin/bash
# A/B timing of two liborion builds on ONE box (gpurun): the same bench.py workload run
# alternately with ORION_LIB=A and ORION_LIB=B, N pairs, ms_per_step of each run appended to
# gpurun_out/ab.txt.  Build A first (e.g. git stash; build; cp liborion.so build/liborion_old.so;
# git stash pop; build), then:
#   gpurun -- 'bash tools/ab_run.sh c2 build/liborion_old.so paper_conf_middleware_hayeslcsz16_b200/liborion.so 2'
# Extra bench.py flags may follow the pair count.
WL=${1:-c2}
A=${2:-build/liborion_old.so}
B=${3:-paper_conf_middleware_hayeslcsz16_b200/liborion.so}
N=${4:-2}
shift 4 2>/dev/null
OUT=gpurun_out
mkdir -p $OUT
for i in $(seq 1 $N); do
  for lib in $A $B; do
    ORION_LIB=$lib python bench.py --workload $WL --rounds 3 --no-cpu-baseline --no-carveout-axis "$@" > $OUT/ab_last.log 2>&1
    echo "$WL $lib $(grep -o '"ms_per_step": [0-9.]*' $OUT/ab_last.log)" >> $OUT/ab.txt
  done
done
