# GPU-FAST vs GPU-PROCLUS (plain) vs GPU-FAST* at C3 (and C4): the paper's
# ablation on B200, plus the variant parity tests.
set -u
OUT=gpurun_out/${1:-vb}; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k variants > $OUT/tests.log 2>&1; tail -2 $OUT/tests.log
for cfg in C3 C4; do
for v in fast plain star; do
  timeout 300 python bench.py --config $cfg --variant $v --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/${cfg}_$v.json 2> $OUT/${cfg}_$v.err
  python - "$OUT/${cfg}_$v.json" "$cfg $v" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[2], "value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), " ".join(
    f"{k}={v['ms_total']/max(v['launches'],1)*1000:.1f}" for k, v in j["kernels"].items()))
PY
done; done
