"""Decode the dbg_cyc phase counters (tail_cycles line) printed by tools/tail_prof.py."""
import sys

line = [l for l in open(sys.argv[1]) if l.startswith("tail_cycles")][-1]
v = [int(x) for x in line.split()[1:]]
M = (1 << 64) - 1
if v[7]:
    b = v[7]
    print("per block ns: prologue %.0f loop %.0f flush %.0f; span %.0f" %
          (v[4] / b, v[5] / b, v[6] / b, v[9] - (M - v[8])))
if v[14]:
    w = v[14]
    print("per warp cycles: wait %.0f A %.0f B %.0f C %.0f (warps %d)" %
          (v[10] / w, v[11] / w, v[12] / w, v[13] / w, w))
