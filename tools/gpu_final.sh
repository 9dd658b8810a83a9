# Round checkpoint: all GPU tests, smoke, default bench (+ reference arm),
# secondary configs, ncu launch list + full capture for profiles/.
#   gpurun -- 'bash tools/gpu_final.sh TAG'
set -u
TAG=${1:-fin}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/tests.log 2>&1; tail -1 $OUT/tests.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 400 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e > $OUT/c4.json 2> $OUT/c4.err
timeout 400 python bench.py --config C5 --steps 3 --warmup 3 > $OUT/c5.json 2> $OUT/c5.err
timeout 400 python bench.py --config L8 --steps 5 --warmup 3 --no-e2e > $OUT/l8.json 2> $OUT/l8.err
bash tools/profile_round.sh $TAG > /dev/null 2>&1
python - $OUT <<'PY'
import json, sys, os
d = sys.argv[1]
for f in ("bench.json", "bench_ref.json", "c4.json", "c5.json", "l8.json"):
    try:
        j = json.loads(open(os.path.join(d, f)).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "FAILED", e); continue
    print(f, round(j.get("value", 0), 2), j.get("unit"), "ms", round(j.get("ms_per_step", 0), 3),
          "frac", (j.get("roofline") or {}).get("frac"), "e2e", (j.get("e2e") or {}).get("value"))
PY
