#!/bin/bash
# Round-2 evidence for profiles/ (keeps gpurun_out under 64 MiB): launch list
# of the C3 bench (stream mode), ncu --set full of the C3 locality / assign /
# cost kernels and of the C4 wide-row kernels and split tails, and the
# compute-sanitizer runs.   gpurun -- 'bash tools/profile_r02.sh TAG'
set -u
TAG=${1:-r02}
OUT=gpurun_out/prof_$TAG
mkdir -p $OUT
export PROCLUS_GRAPH=0
ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 \
    --no-cpu-baseline --no-e2e --no-other-metric > $OUT/launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_locality" -s 1 -c 4 \
    -o $OUT/full python tools/profile_run.py C3 1 > $OUT/full.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_(assign|cost1)" -s 2 -c 4 \
    -o $OUT/full_ac python tools/profile_run.py C3 1 > $OUT/full_ac.log 2>&1
ncu --set full --clock-control none -k regex:"k_(locality|assign|cost1|tail)" -s 4 -c 8 \
    -o $OUT/full_c4 python tools/profile_run.py C4 1 > $OUT/full_c4.log 2>&1
unset PROCLUS_GRAPH
if [ -z "${NO_SAN:-}" ]; then bash tools/sanitize.sh prof_$TAG/san > /dev/null 2>&1; cat $OUT/san/summary.txt; fi
du -sh $OUT; ls -la $OUT
