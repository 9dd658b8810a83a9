"""Where the end-to-end time goes: load (H2D + pack + scales), prefetch+load,
run with device labels, run with host labels (C3)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_edbt_jorgensensape22_b200 as pk  # noqa: E402
import synth  # noqa: E402

data, cfg = synth.config_data("C3", seed=1)
pinned = torch.from_numpy(data).pin_memory()
hlab = torch.empty(data.shape[0], dtype=torch.int32).pin_memory()
dlab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
h = pk.Proclus(pinned.numpy())


def t(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps * 1e3


print("load (sync H2D + pack)   ms", round(t(lambda: h.load(pinned.numpy())), 3))
def pl():
    h.prefetch(pinned.numpy())
    torch.cuda.synchronize()
    h.load(pinned.numpy())
print("prefetch, sync, load     ms", round(t(pl), 3))
print("run, device labels       ms", round(t(lambda: h.run(10, 5, seed=3, labels=dlab)), 3))
print("run, host labels         ms", round(t(lambda: h.run(10, 5, seed=3, labels=hlab.numpy())), 3))
def step():
    h.prefetch(pinned.numpy())
    h.run(10, 5, seed=3, labels=hlab.numpy())
    h.load(pinned.numpy())
print("prefetch+run+load step   ms", round(t(step), 3))
def pl2():
    h.prefetch(pinned.numpy())
    time.sleep(0.004)
    t0 = time.perf_counter()
    h.load(pinned.numpy())
    return (time.perf_counter() - t0) * 1e3
pl2()
print("load after a finished prefetch ms", round(sum(pl2() for _ in range(10)) / 10, 3))
x = torch.from_numpy(data).cuda()
hd = pk.Proclus(x)
print("device-resident load (pack+scales) ms", round(t(lambda: hd.load(x)), 3))


def step_parts(reps=10):
    """host time of each call of a pipelined step (prefetch, run, load)"""
    acc = [0.0, 0.0, 0.0]
    for r in range(reps + 1):
        t0 = time.perf_counter()
        h.prefetch(pinned.numpy())
        t1 = time.perf_counter()
        h.run(10, 5, seed=3, labels=hlab.numpy())
        t2 = time.perf_counter()
        h.load(pinned.numpy())
        t3 = time.perf_counter()
        if r:
            for i, v in enumerate((t1 - t0, t2 - t1, t3 - t2)):
                acc[i] += v * 1e3 / reps
    return [round(a, 3) for a in acc]


print("step parts (prefetch, run, load) ms", step_parts())
def run_after_prefetch():
    h.prefetch(pinned.numpy())
    t0 = time.perf_counter()
    h.run(10, 5, seed=3, labels=dlab)
    t1 = time.perf_counter()
    h.load(pinned.numpy())
    return (t1 - t0) * 1e3
run_after_prefetch()
print("run (device labels) with a prefetch in flight ms",
      round(sum(run_after_prefetch() for _ in range(10)) / 10, 3))
