# full GPU checkpoint: gpu tests, smoke, sanitizers, default bench, reference arm
set -u
TAG=${1:-full}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q -rs ${PYTEST_K:-} > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
if [ -z "${NO_SAN:-}" ]; then bash tools/sanitize.sh $TAG/san; fi
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; tail -c 300 $OUT/bench.err
python - $OUT/bench.json <<'PY'
import json,sys
j=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value",j["value"],"ms",j["ms_per_step"],"e2e",j["e2e"]["value"],"frac",j["roofline"]["frac"])
print("other", {k: j["other_metric"][k] for k in ("metric_name","value")}, j["other_metric"]["roofline"]["frac"])
print("cpu", j["cpu_baseline"]["value"], (j["cpu_baseline"].get("all_cores") or {}).get("value"), j["cpu_baseline"].get("nproc"))
for k,v in j.get("kernels",{}).items(): print(f"  {k:9s} {v['us_per_launch']:8.2f} us/launch  {v['launches']}")
print("tails", j.get("tails_ms_total"))
PY
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/ref.json 2> $OUT/ref.err; tail -c 400 $OUT/ref.json
