# A/B of the C4 assign shape: chunks of 2 P with a shared accumulator copy
# (default) against chunks of P (PROCLUS_ASG_P1=1), arms interleaved, after
# the GPU parity suite.   gpurun -- 'bash tools/ab_c4.sh TAG'
set -u
TAG=${1:-abc4}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/tests.log 2>&1; tail -2 $OUT/tests.log
for r in 1 2; do
  bash tools/c4.sh $TAG/new$r | head -4
  PROCLUS_ASG_P1=1 bash tools/c4.sh $TAG/old$r | head -4
done
