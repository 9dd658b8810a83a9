# Secondary workloads: C5 sweep, C4 (d=100), C2 bench lines.
set -u
OUT=gpurun_out/${1:-cfg}; mkdir -p $OUT
timeout 400 python bench.py --config C5 --steps 3 --warmup 3 > $OUT/c5.json 2> $OUT/c5.err; tail -c 1500 $OUT/c5.json
timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e > $OUT/c4.json 2> $OUT/c4.err; tail -c 2500 $OUT/c4.json
