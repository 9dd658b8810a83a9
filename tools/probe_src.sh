#!/bin/bash
# Baseline bench line + source-level ncu captures of the C3 pass kernels
#   gpurun -- 'bash tools/probe_src.sh TAG'
set -u
TAG=${1:-probe}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 600 python bench.py --steps 20 --no-cpu-baseline --no-other-metric > $OUT/bench.json 2> $OUT/bench.err
tail -c 1500 $OUT/bench.json
export PROCLUS_GRAPH=0
ncu --set full --clock-control none --import-source on -k regex:"k_(locality|assign|cost1)" -s 6 -c 3 \
    -o $OUT/src python tools/profile_run.py C3 1 > $OUT/src.log 2>&1
for k in k_locality k_assign k_cost1; do python tools/ncu_src.py $OUT/src.ncu-rep $k 45 > $OUT/src_$k.txt 2>&1; done
ls -la $OUT
