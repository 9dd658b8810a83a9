PROCLUS_NVCC_EXTRA="-DPROCLUS_PHASE_PROFILE" python paper_conf_edbt_jorgensensape22_b200/_build.py > /dev/null 2>&1
PROCLUS_GRAPH=0 python tools/phase_prof.py C3 2>&1 | tail -3
