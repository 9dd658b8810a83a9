set -u
OUT=gpurun_out/r2a; mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb > $OUT/mb.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -rs > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 400 python bench.py > $OUT/bench.json 2> $OUT/bench.err; tail -c 600 $OUT/bench.json
