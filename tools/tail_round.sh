# GPU tests of the current build, then the per-phase tail cycles of C3
# (-DPROCLUS_TAIL_PROFILE build, restored afterwards).
set -u
OUT=gpurun_out/tail; mkdir -p $OUT
timeout 400 python -m pytest tests -m gpu -q -x > $OUT/tests.log 2>&1; tail -1 $OUT/tests.log
timeout 200 python bench.py --steps 50 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench.json 2>/dev/null
python - $OUT/bench.json <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), " ".join(
    f"{k}={v['ms_total']/max(v['launches'],1)*1000:.1f}" for k, v in j["kernels"].items()), j["tails_ms_total"])
PY
PROCLUS_NVCC_EXTRA="-DPROCLUS_TAIL_PROFILE" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
timeout 200 python tools/tail_prof.py C3 > $OUT/tail.log 2>&1; grep -v "^$" $OUT/tail.log | tail -4 | cut -c1-400
python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
