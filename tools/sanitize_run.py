"""Small clusterings for compute-sanitizer (memcheck / racecheck / synccheck):
C1 with both metrics, a d = 33 shape (k_locality<0>), a d = 100 shape (long
rows: k_assign<1>, k_lsum2 one-block layout) and C2.
  compute-sanitizer --tool racecheck python tools/sanitize_run.py [--big]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402
import synth  # noqa: E402

cases = [("C1", None, 0), ("C1", None, 1), ("shape33", (2049, 33, 8, 6), 0),
         ("shape100", (1500, 100, 10, 10), 1)]
if "--big" in sys.argv:
    cases.append(("C2", None, 0))
for name, shape, metric in cases:
    if shape is None:
        data, cfg = synth.config_data(name, seed=1)
        k, l = cfg["k"], cfg["l"]
    else:
        n, d, k, l = shape
        data = synth.generate(n, d, max(2, k // 2), max(1, d // 3), seed=n)
    with pk.Proclus(data, metric=metric) as h:
        r = h.run(k, l, A=20 if shape else 100, B=5 if shape else 10, seed=1)
    print(f"{name} metric {metric}: iterations {r.iterations} cost {r.cost:.9f} "
          f"labels {np.bincount(r.labels + 1)[:4]}...", flush=True)
