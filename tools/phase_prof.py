"""Phase timers of k_lsum2 (needs a -DPROCLUS_PHASE_PROFILE build): one C3
run, prints per-launch span numbers of iteration 3 (globaltimer ns)."""
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
    r = h.run(cfg["k"], cfg["l"], seed=1)
    print("iterations", r.iterations, flush=True)
