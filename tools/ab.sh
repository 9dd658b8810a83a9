# A/B of a compile-time variant: bench with the default build, then with
# PROCLUS_NVCC_EXTRA="$1" (the default build is restored at the end).
set -u
OUT=gpurun_out/ab; mkdir -p $OUT
summ() {
python - "$1" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), " ".join(
    f"{k}={v['ms_total']/max(v['launches'],1)*1000:.1f}" for k, v in j["kernels"].items()))
PY
}
timeout 200 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e ${2:-} > $OUT/a.json 2>/dev/null; echo -n "A: "; summ $OUT/a.json
PROCLUS_NVCC_EXTRA="$1" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
timeout 200 python bench.py --steps 30 --warmup 3 --no-cpu-baseline --no-e2e ${2:-} > $OUT/b.json 2>/dev/null; echo -n "B: "; summ $OUT/b.json
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "C1_seed or C2 or shapes" 2>&1 | tail -1
python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
