set -u
OUT=gpurun_out/s3a; mkdir -p $OUT
nvidia-smi -L > $OUT/smi.txt
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; tail -c 3000 $OUT/bench.json
