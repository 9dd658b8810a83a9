#!/bin/bash
# Evidence for profiles/: (1) launch list of bench.py under ncu (per-launch
# device time, cold-cache, serialised), (2) one full ncu capture per pass
# kernel (dram bytes, occupancy, stall reasons).  Runs on the GPU box:
#   gpurun -- 'bash tools/profile_round.sh <tag>'
# Kernels inside CUDA graphs with conditional nodes cannot be profiled per
# kernel, so these passes run the library's stream mode (PROCLUS_GRAPH=0),
# which launches the identical kernels.
set -u
TAG=${1:-r01}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
export PROCLUS_GRAPH=0
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 \
    --no-cpu-baseline --no-e2e > $OUT/launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on \
    -k regex:"k_(locality|assign|cost1|lsum2|labelsum|final|greedy|sdist)" -s 0 -c 16 \
    -o $OUT/full python tools/profile_run.py C3 1 > $OUT/full.log 2>&1
ls -la $OUT
