# A/B of a run-time switch: default environment vs "$1" (e.g. PROCLUS_PDL=0),
# each bench run twice interleaved (A B A B) to see the noise.
#   gpurun -- 'bash tools/ab_env.sh PROCLUS_PDL=0 [bench args]'
set -u
OUT=gpurun_out/abe; mkdir -p $OUT
summ() {
python - "$1" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), " ".join(
    f"{k}={v['ms_total']/max(v['launches'],1)*1000:.1f}" for k, v in j["kernels"].items()))
PY
}
for r in 1 2; do
timeout 200 python bench.py --steps 50 --warmup 3 --no-cpu-baseline --no-e2e ${2:-} > $OUT/a$r.json 2>$OUT/a$r.err; echo -n "A$r: "; summ $OUT/a$r.json
env $1 timeout 200 python bench.py --steps 50 --warmup 3 --no-cpu-baseline --no-e2e ${2:-} > $OUT/b$r.json 2>$OUT/b$r.err; echo -n "B$r ($1): "; summ $OUT/b$r.json
done
