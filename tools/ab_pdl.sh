# PDL placement A/B: default build (trigger at entry) with PDL on / off, then
# a -DPROCLUS_PDL_LATE build (trigger after the chunk loop).
set -u
OUT=gpurun_out/abp; mkdir -p $OUT
summ() {
python - "$1" <<'PY'
import json, sys
j = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", round(j["value"], 1), "ms", round(j["ms_per_step"], 3), " ".join(
    f"{k}={v['ms_total']/max(v['launches'],1)*1000:.1f}" for k, v in j["kernels"].items()))
PY
}
B="timeout 200 python bench.py --steps 50 --warmup 3 --no-cpu-baseline --no-e2e"
for r in 1 2; do
$B > $OUT/early$r.json 2>/dev/null; echo -n "early$r: "; summ $OUT/early$r.json
PROCLUS_PDL=0 $B > $OUT/off$r.json 2>/dev/null; echo -n "off$r: "; summ $OUT/off$r.json
done
PROCLUS_NVCC_EXTRA="-DPROCLUS_PDL_LATE" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
for r in 1 2; do
$B > $OUT/late$r.json 2>/dev/null; echo -n "late$r: "; summ $OUT/late$r.json
done
python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
