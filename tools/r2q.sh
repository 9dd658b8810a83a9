# quick: parity smoke on C1 seeds + C3 full size, then the default bench (kernel table)
set -u
TAG=${1:-q}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "C1_seed or full_size" > $OUT/tests.log 2>&1; tail -1 $OUT/tests.log
timeout 400 python bench.py > $OUT/bench.json 2> $OUT/bench.err
python - $OUT/bench.json <<'PY'
import json,sys
j=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value",j["value"],"ms",j["ms_per_step"],"e2e",j["e2e"]["value"],"frac",j["roofline"]["frac"])
for k,v in j.get("kernels",{}).items():
    if v["launches"]: print(f"  {k:9s} {v['ms_total']/v['launches']*1000:8.2f} us/launch  {v['launches']}")
print("tails", j.get("tails_ms_total"))
PY
