# build libproclus variants: tools/build_variants.sh NAME "NVCC FLAGS" [NAME "FLAGS" ...]
set -eo pipefail
cd "$(dirname "$0")/.."
while [ $# -ge 2 ]; do
  PROCLUS_NVCC_EXTRA="$2" python -c "from paper_conf_edbt_jorgensensape22_b200 import _build; _build.build(force=True)"
  cp paper_conf_edbt_jorgensensape22_b200/libproclus.so paper_conf_edbt_jorgensensape22_b200/libproclus_$1.so
  echo "built $1: $2"
  shift 2
done
python -c "from paper_conf_edbt_jorgensensape22_b200 import _build; _build.build(force=True)"
