#!/bin/bash
# Per-launch device durations of one C3 clustering (stream mode), warm caches:
#   gpurun -- 'bash tools/launch_list.sh TAG [CONFIG]'
set -u
TAG=$1; CFG=${2:-C3}
OUT=gpurun_out/ll_$TAG; mkdir -p $OUT
export PROCLUS_GRAPH=0
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv \
    --log-file $OUT/launches.csv python tools/profile_run.py $CFG 2 > $OUT/run.log 2>&1
python tools/launch_summary.py $OUT/launches.csv
