set -u
OUT=gpurun_out/ctlexp; mkdir -p $OUT
PROCLUS_NVCC_EXTRA="-DCTL_EXP" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1 || echo BUILD FAILED
timeout 200 python tools/tail_prof.py C3 > $OUT/tail.log 2>&1; grep "tail_cycles\|^iterations" $OUT/tail.log | cut -c1-200
