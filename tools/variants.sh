set -u
OUT=gpurun_out/var; mkdir -p $OUT
for v in base PROCLUS_ASSIGN3 PROCLUS_ASSIGN2 PROCLUS_OLD_LSUM; do
  if [ $v = base ]; then env_=""; else env_="$v=1"; fi
  env $env_ timeout 200 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/$v.json 2> $OUT/$v.err
  python - "$OUT/$v.json" "$v" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[2], "value", round(j["value"],1), "ms", round(j["ms_per_step"],3), "parity", j.get("parity"))
for k, v in j["kernels"].items():
    print("  ", k, v["launches"], round(v["ms_total"] / max(v["launches"], 1) * 1000, 1), "us/launch")
PY
done
