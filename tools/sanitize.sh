# compute-sanitizer runs of small clusterings (SURVEY 4.2 layer D); logs to gpurun_out/$1
set -u
OUT=gpurun_out/${1:-san}; mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
export PROCLUS_GRAPH=0
for tool in memcheck racecheck synccheck; do
  timeout 900 $CS --tool $tool --error-exitcode 9 python tools/sanitize_run.py > $OUT/$tool.log 2>&1
  echo "$tool rc=$?" | tee -a $OUT/summary.txt
  tail -2 $OUT/$tool.log
done
unset PROCLUS_GRAPH
timeout 900 $CS --tool memcheck --error-exitcode 9 python tools/sanitize_run.py > $OUT/memcheck_graph.log 2>&1
echo "memcheck (graph mode) rc=$?" | tee -a $OUT/summary.txt
timeout 900 $CS --tool initcheck --error-exitcode 9 python -c "
import sys; sys.argv=['x']; sys.path.insert(0,'.')
import numpy as np, synth, paper_conf_edbt_jorgensensape22_b200 as pk
d,c=synth.config_data('C1',1)
with pk.Proclus(d) as h: print(h.run(5,3,seed=1).iterations)" > $OUT/initcheck.log 2>&1
echo "initcheck (C1) rc=$?" | tee -a $OUT/summary.txt
