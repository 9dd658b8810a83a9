"""Per-phase cycles of the single-block tails (needs a -DPROCLUS_TAIL_PROFILE
build): runs C3 with stats on and prints the dbg counters per iteration."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["PROCLUS_TAIL_PROFILE"] = "1"
import torch  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402
import synth  # noqa: E402

data, cfg = synth.config_data(sys.argv[1] if len(sys.argv) > 1 else "C3", seed=1)
x = torch.from_numpy(data).cuda()
with pk.Proclus(x, stats=True) as h:
    for s in range(3):
        r = h.run(cfg["k"], cfg["l"], seed=1 + s)
        print("iterations", r.iterations, "stats", h.stats(), flush=True)
