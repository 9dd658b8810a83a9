set -u
OUT=gpurun_out/icache; mkdir -p $OUT
PROCLUS_NVCC_EXTRA="-DPROCLUS_TAIL_PROFILE -DICACHE_EXP" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
timeout 200 python tools/tail_prof.py C3 > $OUT/tail.log 2>&1; grep "tail_cycles\|loc_phase\|^iterations" $OUT/tail.log | cut -c1-300
