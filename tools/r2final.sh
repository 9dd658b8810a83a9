# round-2 checkpoint: all GPU tests, smoke, sanitizers, bench lines (C3 default
# with every leg, reference arm, C4, C5, L8, L8S)
set -u
TAG=${1:-fin}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q -rs > $OUT/tests.log 2>&1; tail -2 $OUT/tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
if [ -n "${SAN:-}" ]; then bash tools/sanitize.sh $TAG/san > /dev/null 2>&1; cat $OUT/san/summary.txt; fi
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 600 python bench.py --impl reference > $OUT/ref.json 2> $OUT/ref.err
timeout 600 python bench.py --config C4 --steps 20 --no-e2e --no-other-metric > $OUT/c4.json 2> $OUT/c4.err
timeout 900 python bench.py --config C5 --steps 3 --no-cpu-baseline > $OUT/c5.json 2> $OUT/c5.err
timeout 600 python bench.py --config L8 --steps 10 --no-e2e --no-other-metric --no-cpu-baseline > $OUT/l8.json 2> $OUT/l8.err
timeout 600 python bench.py --config L8S --steps 2 --no-cpu-baseline > $OUT/l8s.json 2> $OUT/l8s.err
python - $OUT <<'PY'
import json, sys, os
d = sys.argv[1]
for f in ("bench.json", "ref.json", "c4.json", "c5.json", "l8.json", "l8s.json"):
    try:
        j = json.loads(open(os.path.join(d, f)).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "FAILED", e); continue
    print(f, round(j.get("value", 0), 3), j.get("unit"), "ms", round(j.get("ms_per_step", 0), 3),
          "frac", (j.get("roofline") or {}).get("frac"), "e2e", (j.get("e2e") or {}).get("value"),
          "reuse", j.get("reuse_speedup"))
PY
