"""Short driver for ncu captures: a few C3 clusterings through the C ABI
(no oracle, no timing).  Usage: python tools/profile_run.py [config] [runs]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
runs = int(sys.argv[2]) if len(sys.argv) > 2 else 2
data, cfg = synth.config_data(name, seed=1)
x = torch.from_numpy(data).cuda()
lab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
with pk.Proclus(x) as h:
    for s in range(runs):
        r = h.run(cfg["k"], cfg["l"], seed=1 + s, labels=lab)
        print(f"run {s}: iterations={r.iterations} cost={r.cost:.12f} launches={h.last_launches}")
torch.cuda.synchronize()
