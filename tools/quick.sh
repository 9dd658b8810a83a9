# Quick GPU check: parity tests + a short bench with per-kernel times.
#   gpurun -- 'bash tools/quick.sh TAG [pytest -k expr]'
set -u
TAG=${1:-q}; OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 600 python -m pytest tests -m gpu -q -x ${2:+-k "$2"} > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 200 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench.json 2> $OUT/bench.err
python - "$OUT/bench.json" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), "frac", j["roofline"]["frac"], "parity", j.get("parity"))
for k, v in j["kernels"].items():
    print("  ", k, v["launches"], round(v["ms_total"] / max(v["launches"], 1) * 1000, 1), "us/launch")
print("tails", j.get("tails_ms_total"))
PY
