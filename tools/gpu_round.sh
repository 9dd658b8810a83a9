# One GPU check: parity tests, a short bench, optional tail-phase profile.
#   gpurun -- 'bash tools/gpu_round.sh TAG [tailprof]'
set -u
TAG=${1:-x}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x > $OUT/tests.log 2>&1; tail -3 $OUT/tests.log
timeout 200 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench.json 2> $OUT/bench.err
python - "$OUT/bench.json" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", j["value"], "ms", j["ms_per_step"], "tails", j.get("tails_ms_total"))
for k, v in j["kernels"].items():
    print(" ", k, v["launches"], round(v["ms_total"] / max(v["launches"], 1) * 1000, 1), "us/launch")
PY
if [ "${2:-}" = "tailprof" ]; then
  PROCLUS_NVCC_EXTRA="-DPROCLUS_TAIL_PROFILE" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
  timeout 300 python tools/tail_prof.py C3 2>&1 | grep tail_cycles | tail -1
fi
