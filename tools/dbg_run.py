"""Debug driver: one clustering of a given shape through the C ABI (used
under compute-sanitizer).  usage: python tools/dbg_run.py [n d k l A B]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402

if len(sys.argv) > 6:
    n, d, k, l, A, B = map(int, sys.argv[1:7])
    data = synth.generate(n, d, max(2, k // 2), max(1, d // 3), seed=n)
else:
    data, cfg = synth.config_data("C1", seed=1)
    k, l, A, B = cfg["k"], cfg["l"], 100, 10
with pk.Proclus(data) as h:
    r = h.run(k, l, A, B, 0.7, 5, 3)
    print("ok", r.iterations, r.cost)
