#!/bin/bash
# stall reasons of the single-block tails at C3 (split tail kernels, stream mode)
set -u
TAG=${1:-ntail}; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PROCLUS_GRAPH=0 PROCLUS_TAIL_KERNELS=1
ncu --set full --clock-control none --cache-control none --warp-sampling-interval 0 --import-source on -k regex:"k_tail" -s 9 -c 9 \
    -o $OUT/tail python tools/profile_run.py C3 1 > $OUT/tail.log 2>&1
ncu -i $OUT/tail.ncu-rep --page raw --csv > $OUT/raw.csv 2>&1
ncu -i $OUT/tail.ncu-rep --page details --csv > $OUT/details.csv 2>&1
python tools/ncu_src.py $OUT/tail.ncu-rep k_tail 40 0 > $OUT/src0.txt 2>&1
python tools/ncu_src.py $OUT/tail.ncu-rep k_tail 40 2 > $OUT/src2.txt 2>&1
