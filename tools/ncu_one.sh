#!/bin/bash
# ncu --set full (source) of one pass kernel in C3 (stream mode) + per-line summary
#   gpurun -- 'bash tools/ncu_one.sh TAG KERNEL_REGEX [CONFIG] [SKIP]'
set -u
TAG=$1; KR=$2; CFG=${3:-C3}; SKIP=${4:-6}
OUT=gpurun_out/$TAG; mkdir -p $OUT
export PROCLUS_GRAPH=0
ncu --set full --clock-control none --import-source on -k regex:"$KR" -s $SKIP -c 1 \
    -o $OUT/one python tools/profile_run.py $CFG 1 > $OUT/one.log 2>&1
python tools/ncu_src.py $OUT/one.ncu-rep "$KR" 50 > $OUT/src.txt 2>&1
ncu -i $OUT/one.ncu-rep --page raw --csv > $OUT/raw.csv 2>&1
cat $OUT/src.txt | head -60
