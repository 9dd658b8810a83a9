"""Does a concurrent copy slow a clustering?  h.run (device labels) timed
alone, with an unrelated 60 MB H2D on a torch side stream, and with a 60 MB
device-to-device copy on that stream (C3)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402
import synth  # noqa: E402

data, cfg = synth.config_data("C3", seed=1)
pinned = torch.from_numpy(data).pin_memory()
dlab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
h = pk.Proclus(pinned.numpy())
dst = torch.empty_like(pinned, device="cuda")
src2 = torch.empty_like(pinned, device="cuda")
side = torch.cuda.Stream()


def timed(pre, reps=10):
    out = []
    for r in range(reps + 1):
        torch.cuda.synchronize()
        pre()
        t0 = time.perf_counter()
        h.run(10, 5, seed=3, labels=dlab)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        if r:
            out.append((t1 - t0) * 1e3)
    return round(sum(out) / len(out), 3)


def h2d():
    with torch.cuda.stream(side):
        dst.copy_(pinned, non_blocking=True)


def d2d():
    with torch.cuda.stream(side):
        dst.copy_(src2, non_blocking=True)


def h2d_half():
    with torch.cuda.stream(side):
        dst[: dst.shape[0] // 2].copy_(pinned[: dst.shape[0] // 2], non_blocking=True)


print("run alone ms", timed(lambda: None))
print("run + torch H2D 60MB ms", timed(h2d))
print("run + torch H2D 30MB ms", timed(h2d_half))
print("run + torch D2D 60MB ms", timed(d2d))
print("run + prefetch ms", timed(lambda: h.prefetch(pinned.numpy())))
