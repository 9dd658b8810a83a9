#!/bin/bash
# Full ncu capture (with source) of the kernels matching a regex, C3 by default:
#   gpurun -- 'bash tools/prof_kernel.sh TAG REGEX [COUNT] [CONFIG]'
set -u
TAG=$1; RX=$2; CNT=${3:-3}; CFG=${4:-C3}
OUT=gpurun_out/pk_$TAG; mkdir -p $OUT
export PROCLUS_GRAPH=0
ncu --set full --clock-control none --import-source on -k regex:"$RX" -s 0 -c $CNT \
    -o $OUT/full python tools/profile_run.py $CFG 1 > $OUT/full.log 2>&1
tail -3 $OUT/full.log
