# A/B the prebuilt variants (libproclus_NAME.so) on one box, arms interleaved:
#   tools/ab_variants.sh TAG ROUNDS NAME...   (C3 bench, 20 steps each)
set -u
TAG=$1; R=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
D=paper_conf_edbt_jorgensensape22_b200
cp $D/libproclus.so $D/libproclus_base.so.keep
for r in $(seq 1 $R); do
  for v in "$@"; do
    lib=${v%%+*}; envs=""
    [ "$lib" != "$v" ] && envs=${v#*+}   # NAME+VAR=VAL: run that variant with an env setting
    cp $D/libproclus_$lib.so $D/libproclus.so
    touch $D/libproclus.so
    env $envs timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e --no-other-metric ${BENCH_ARGS:-} > $OUT/${v}_$r.json 2> $OUT/${v}_$r.err
    python - $OUT/${v}_$r.json $v <<'PY'
import json,sys
j=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
k=j["kernels"]
print(f"{sys.argv[2]:10s} {j['value']:8.1f}/s  loc {k['locality']['us_per_launch']:6.2f}  asg {k['assign']['us_per_launch']:6.2f}  cost {k['cost']['us_per_launch']:6.2f}  fin {k['final']['us_per_launch']:6.2f}  ref {k['refine_x']['us_per_launch']:6.2f}  greedy {k['greedy']['us_per_launch']:6.2f}  tails {j['tails_ms_total']}")
PY
  done
done
cp $D/libproclus_base.so.keep $D/libproclus.so
