set -u
OUT=gpurun_out/${1:-c4}; mkdir -p $OUT
timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/c4.json 2> $OUT/c4.err
python - "$OUT/c4.json" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("C4 value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), "frac", j["roofline"]["frac"])
for k, v in j["kernels"].items():
    print("  ", k, v["launches"], round(v["ms_total"] / max(v["launches"], 1) * 1000, 1), "us/launch")
print("tails", j.get("tails_ms_total"))
PY
