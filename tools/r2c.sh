set -u
TAG=${1:-r2c}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -x -rs ${PYTEST_K:-} > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 400 python bench.py > $OUT/bench.json 2> $OUT/bench.err
python - $OUT/bench.json <<'PY'
import json,sys
j=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value",j["value"],"ms",j["ms_per_step"],"e2e",j["e2e"]["value"],"frac",j["roofline"]["frac"])
for k,v in j.get("kernels",{}).items(): print(k, v)
PY
bash tools/prof_kernel.sh $TAG k_locality 4 C3
