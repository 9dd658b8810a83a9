# A/B at C4 of a shape switch: default arm against the arm with the env var
# OLDENV=1 (e.g. PROCLUS_ASG_P1: assign chunks of P; PROCLUS_REF_SMALL:
# refinement X limited to two-blocks-per-SM layouts), arms interleaved,
# after the GPU parity suite.   gpurun -- 'bash tools/ab_c4.sh TAG OLDENV'
set -u
TAG=${1:-abc4}
OLDENV=${2:-PROCLUS_ASG_P1}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/tests.log 2>&1; tail -2 $OUT/tests.log
for r in 1 2; do
  bash tools/c4.sh $TAG/new$r > /dev/null 2>&1
  env $OLDENV=1 bash tools/c4.sh $TAG/old$r > /dev/null 2>&1
done
