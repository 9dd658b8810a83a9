#!/usr/bin/env python
"""Benchmark of the B200 PROCLUS hot path (BASELINE.json metric).

One step = one full PROCLUS clustering (init + iterative phase + refinement,
Alg 1) of the C3 workload: n = 1,000,000 points x d = 15, k = 10, l = 5,
A = 100, B = 10, minDev = 0.7, itrPat = 5 (PAPER.md P:370 defaults), on
seeded synthetic data from the PROCLUS-style generator (synth/, P:374,
P:386).  Each timed step uses a different run seed (the paper averages over
runs).  value = clusterings / s over the whole job (max over ranks).

  python bench.py [--gpus N --steps K --warmup W] [--impl reference]

N > 1: one process per GPU, launched by torchrun or -- when WORLD_SIZE is not
set -- spawned by bench.py itself (127.0.0.1 rendezvous).  C1-C4 / L8: rows
are sharded across ranks and the k x d partial sums are combined with NCCL
allreduce inside the library (strong scaling: the same clustering).  C5 /
L8S: settings parallelism -- every rank holds the whole dataset and runs its
share of the (k, l) grid (proclus_run_list, no communication).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

BASELINE_METRIC = "PROCLUS clusterings/sec (ms per run) at n=1M,d=15; HBM GB/s vs peak, 1/2/4/8 GPUs"
UNIT = "clusterings/s"
FALLBACK_HBM_GBS = 6650.0
L2_FLUSH_BYTES = 256 << 20
REF_SAMPLE_ROWS = 100_000


def workload_config(args, n_gpus):
    cfg = synth.CONFIGS[args.config]
    return {
        "workload": f"{args.config}: n={cfg['n']:,} d={cfg['d']} k={cfg['k']} l={cfg['l']} "
                    f"A=100 B=10 minDev=0.7 itrPat=5, full-space metric {args.metric.upper()}",
        "n": cfg["n"], "d": cfg["d"], "k": cfg["k"], "l": cfg["l"], "A": 100, "B": 10,
        "minDev": 0.7, "itrPat": 5, "metric": args.metric.upper(),
        "data_seed": args.data_seed, "run_seeds": f"{args.seed0}..{args.seed0 + args.steps - 1}",
        "generator": f"{cfg['n_clusters']} Gaussian clusters in {cfg['subspace_dim']}-d subspaces, "
                     "sd 5 on [0,100], 5% uniform noise, min-max normalised (P:374, P:386)",
        "l2": "256 MiB L2 flush written between timed steps",
        "parallelism": f"rows sharded over {n_gpus} GPU(s)" if n_gpus > 1 else "1 GPU",
        "variant": {"fast": "GPU-FAST-PROCLUS", "plain": "GPU-PROCLUS (no caches, P:239)",
                    "star": "GPU-FAST*-PROCLUS (P:215-219)"}[getattr(args, "variant", "fast")],
    }


def read_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic(kind):
    """dram bytes per launch of `kind` from the committed ncu summary, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            j = json.load(f)
        v = j.get(kind)
        return None if v is None else float(v)
    except Exception:
        return None


class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "50", "-i", str(self.device)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *exc):
        self.out = ""
        if self.proc is not None:
            time.sleep(0.1)
            self.proc.terminate()
            try:
                self.out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                self.out = ""

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in (self.out or "").strip().splitlines():
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for name, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def cpu_info():
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


def cpu_baseline_full(data, cfg, metric):
    """The oracle as it stands: one full clustering of the workload (or of its
    first ORACLE_MAX_ROWS rows, scaled by n / n_sample), 1 core."""
    import oracle

    ns = min(len(data), ORACLE_MAX_ROWS)
    t = time.perf_counter()
    r = oracle.proclus(np.ascontiguousarray(data[:ns]), cfg["k"], cfg["l"], seed=1, metric=metric)
    dt = (time.perf_counter() - t) * len(data) / ns
    return r, dt, ns


def cpu_all_cores(config, data_seed, metric, seed0=1, max_procs=64):
    """All-core throughput of the oracle as it stands: P = min(nproc, 64)
    single-threaded oracle processes, each one full clustering of the whole
    workload with its own run seed, started together; throughput = the sum
    of each process's clusterings per second (data generation untimed)."""
    procs = max(1, min(os.cpu_count() or 1, max_procs))
    cmd = [sys.executable, "-m", "oracle.worker", config, str(data_seed)]
    t0 = time.perf_counter()
    ps = [subprocess.Popen(cmd + [str(seed0 + i), str(metric)], cwd=ROOT,
                           stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
          for i in range(procs)]
    secs = []
    for p in ps:
        out, _ = p.communicate()
        try:
            secs.append(json.loads(out.strip().splitlines()[-1])["seconds"])
        except Exception:
            pass
    wall = time.perf_counter() - t0
    if not secs:
        return None
    return {"value": sum(1.0 / x for x in secs), "unit": UNIT, "cores": procs,
            "processes_ok": len(secs), "per_process_s": {"min": min(secs), "max": max(secs)},
            "wall_s": wall,
            "sample": f"{procs} concurrent single-threaded oracle processes, one full "
                      f"{config} clustering each (run seeds {seed0}..{seed0 + procs - 1})"}


REF_BUDGET_S = 60.0  # the reference arm's timed oracle work (seconds)


def run_reference(args):
    """--impl reference: the CPU oracle (this tier's reference arm) on the
    FULL workload of --config: full clusterings one per step on one host
    core, as many of the requested --steps as fit in REF_BUDGET_S (at least
    one; the line's steps field says how many ran), plus the all-core
    throughput (nproc processes) in cpu_baseline."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle

    oracle.build()
    # the sweeps are timed on their base dataset one setting per step
    base = {"C5": "C3", "L8S": "L8"}.get(args.config, args.config)
    data, cfg = synth.config_data(base, seed=args.data_seed)
    data = np.ascontiguousarray(data)
    metric = 0 if args.metric == "l2" else 1
    times, iters = [], []
    t_start = time.perf_counter()
    for s in range(args.steps):
        t = time.perf_counter()
        r = oracle.proclus(data, cfg["k"], cfg["l"], seed=args.seed0 + s, metric=metric)
        times.append(time.perf_counter() - t)
        iters.append(r.iterations)
        if time.perf_counter() - t_start + times[-1] > REF_BUDGET_S:
            break
    mean = sum(times) / len(times)
    value = 1.0 / mean
    allc = None if args.no_cpu_baseline else cpu_all_cores(base, args.data_seed, metric)
    desc = (f"oracle (single-threaded fp64 C, -O2) on the full {base} dataset "
            f"({cfg['n']:,} x {cfg['d']}), {len(times)} full clusterings (run seeds "
            f"{args.seed0}..{args.seed0 + len(times) - 1}, {min(iters)}..{max(iters)} "
            f"iterations), 1 core; {args.steps} steps requested, at most "
            f"{REF_BUDGET_S:.0f} s of oracle time")
    line = {
        "impl": "reference", "metric": BASELINE_METRIC, "value": value, "unit": UNIT,
        "n_gpus": args.gpus, "steps": len(times), "steps_requested": args.steps, "warmup": 0,
        "ms_per_step": mean * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(args, args.gpus),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": desc, "all_cores": allc, **cpu_info()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def spawn_ranks(args):
    """--gpus N without torchrun: start N copies of this script as ranks
    0..N-1 (RANK / LOCAL_RANK / WORLD_SIZE, 127.0.0.1 rendezvous) and pass
    rank 0's JSON line through."""
    import socket

    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    procs = []
    for r in range(args.gpus):
        env = dict(os.environ, RANK=str(r), LOCAL_RANK=str(r), WORLD_SIZE=str(args.gpus),
                   LOCAL_WORLD_SIZE=str(args.gpus), MASTER_ADDR="127.0.0.1",
                   MASTER_PORT=str(port))
        procs.append(subprocess.Popen([sys.executable, os.path.abspath(__file__)] + sys.argv[1:],
                                      env=env, stdout=subprocess.PIPE if r == 0 else
                                      subprocess.DEVNULL, text=True))
    out, _ = procs[0].communicate()
    rc = procs[0].returncode
    for p in procs[1:]:
        rc = max(rc, p.wait())
    sys.stdout.write(out)
    sys.stdout.flush()
    return rc


DTYPE = "f32+f64+i64"
DTYPE_NOTE = ("per-point decisions on certified fp32 distances with an exact fp64 fallback "
              "(the oracle's fp64 expression), sums over points in int64 fixed point, "
              "delta / Delta / greedy / Z-scores in fp64: results identical to the fp64 oracle")


def roofline_of(agg, kind):
    a = agg[kind]
    peak, peak_src = read_peak()
    achieved = (a["alg_bytes"] / (a["ms"] / 1e3)) / 1e9 if a["ms"] > 0 and a["alg_bytes"] > 0 else None
    return {"bound": "hbm", "kernel": kind,
            "achieved": round(achieved, 1) if achieved else None, "peak": peak,
            "unit": "GB/s", "frac": round(achieved / peak, 4) if achieved else None,
            "traffic": ncu_traffic(kind), "peak_source": peak_src,
            "bytes_per_launch": a["alg_bytes"] / max(a["launches"], 1),
            "us_per_launch": round(1e3 * a["ms"] / max(a["launches"], 1), 2),
            "model": "data 4nd + Dist rows 4n per active slot (locality); data 4nd + u8 "
                     "labels n (assign, cost)",
            "timing": "CUDA events around every launch on the launching stream, in an "
                      "instrumented pass of the same steps/seeds right after the timed "
                      "region (graph mode cannot bracket single kernels)"}


def run_gpu(args):
    import torch
    import torch.distributed as dist

    import paper_conf_edbt_jorgensensape22_b200 as pk

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    pk.lib()

    data, cfg = synth.config_data(args.config, seed=args.data_seed)
    n, d, k, l = cfg["n"], cfg["d"], cfg["k"], cfg["l"]
    from paper_conf_edbt_jorgensensape22_b200.sharding import shard_rows

    lo, hi = shard_rows(n, world, rank)  # boundaries on sub-chunk multiples
    shard = np.ascontiguousarray(data[lo:hi])

    def new_uid():
        if world == 1:
            return None
        obj = [torch.cuda.nccl.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        return obj[0]

    stream = torch.cuda.Stream()
    xdev = torch.from_numpy(shard).cuda()
    labels = torch.empty(hi - lo, dtype=torch.int32, device="cuda")
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device="cuda")
    variant = {"fast": 0, "plain": 1, "star": 2}[args.variant]

    def handle(metric, stats):
        return pk.Proclus(xdev, metric=metric, device=local, stream=stream.cuda_stream,
                          world_size=world, variant=variant, rank=rank,
                          n_global=n if world > 1 else 0, row_offset=lo if world > 1 else 0,
                          nccl_unique_id=new_uid(), stats=stats)

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local])
        torch.cuda.synchronize()

    def max_over_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def measure(metric, steps, clocks=True):
        """W warm-up runs, then `steps` timed clusterings (production handle:
        one CUDA graph per clustering on one GPU), then the same steps on an
        event-instrumented handle for the per-kernel table."""
        h = handle(metric, stats=False)
        for s in range(args.warmup):
            h.run(k, l, seed=args.seed0 + 1000 + s, labels=labels)
        barrier()
        step_ms, iters, launches = [], [], 0
        clk = ClockSampler(local) if clocks else None
        if clk:
            clk.__enter__()
        barrier()
        for s in range(steps):
            with torch.cuda.stream(stream):
                flush.zero_()
            ev0 = torch.cuda.Event(enable_timing=True)
            ev1 = torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            r = h.run(k, l, seed=args.seed0 + s, labels=labels)
            ev1.record(stream)
            ev1.synchronize()
            step_ms.append(ev0.elapsed_time(ev1))
            iters.append(r.iterations)
            launches += h.last_launches
        barrier()
        if clk:
            clk.__exit__(None, None, None)
        h.close()
        total_ms = max_over_ranks(sum(step_ms))
        agg, tails, fallbacks = {}, {}, {}
        hs = handle(metric, stats=True)
        for s in range(steps):
            with torch.cuda.stream(stream):
                flush.zero_()
            hs.run(k, l, seed=args.seed0 + s, labels=labels)
            st = hs.stats()
            for kk, v in st["tail_ms"].items():
                tails[kk] = tails.get(kk, 0.0) + v
            for kk, v in st["fallbacks"].items():
                fallbacks[kk] = fallbacks.get(kk, 0) + v
            for kind in pk.STAT_KINDS:
                a = agg.setdefault(kind, dict(launches=0, ms=0.0, alg_bytes=0.0))
                for f in ("launches", "ms", "alg_bytes"):
                    a[f] += st[kind][f]
        torch.cuda.synchronize()
        hs.close()
        return dict(total_ms=total_ms, iters=iters, launches=launches, agg=agg, tails=tails,
                    fallbacks=fallbacks, clocks=clk.summary() if clk else None)

    metric = pk.METRIC_L2 if args.metric == "l2" else pk.METRIC_L1
    m = measure(metric, args.steps)
    total_ms, agg = m["total_ms"], m["agg"]
    value = args.steps / (total_ms / 1e3)

    passes = ["locality", "assign", "cost", "refine_x", "final", "greedy"]
    dom = max(passes, key=lambda kk: agg[kk]["ms"])
    roofline = roofline_of(agg, dom)
    tot_ms = max(sum(v["ms"] for v in agg.values()), 1e-9)
    kernels = {kk: {"launches": agg[kk]["launches"], "ms_total": round(agg[kk]["ms"], 4),
                    "us_per_launch": round(1e3 * agg[kk]["ms"] / agg[kk]["launches"], 2),
                    "share": round(agg[kk]["ms"] / tot_ms, 4),
                    "GBps": round(agg[kk]["alg_bytes"] / (agg[kk]["ms"] / 1e3) / 1e9, 1)
                    if agg[kk]["ms"] > 0 and agg[kk]["alg_bytes"] > 0 else None}
               for kk in pk.STAT_KINDS if agg[kk]["launches"] > 0}

    # the other full-space metric on the same workload (north_star names L1,
    # the paper L2: reading R1) -- value and roofline of its dominant kernel
    other = None
    if not args.no_other_metric:
        om = pk.METRIC_L1 if metric == pk.METRIC_L2 else pk.METRIC_L2
        o_steps = max(3, min(args.steps, 20))
        mo = measure(om, o_steps, clocks=False)
        odom = max(passes, key=lambda kk: mo["agg"][kk]["ms"])
        other = {"metric_name": "L1" if om == pk.METRIC_L1 else "L2",
                 "value": o_steps / (mo["total_ms"] / 1e3), "unit": UNIT, "steps": o_steps,
                 "ms_per_step": mo["total_ms"] / o_steps,
                 "iterations_per_run": sum(mo["iters"]) / len(mo["iters"]),
                 "roofline": roofline_of(mo["agg"], odom)}

    # end to end through the public API with host buffers: H2D of the step's
    # data (pinned) + the whole run + D2H of labels / medoids / dims
    e2e = None
    if world == 1 and not args.no_e2e:
        pinned = torch.from_numpy(shard).pin_memory()
        hh = pk.Proclus(pinned.numpy(), metric=metric, device=local, variant=variant)
        hlab = torch.empty(hi - lo, dtype=torch.int32).pin_memory()
        e_steps = max(3, min(args.steps, 20))
        for s in range(2):
            hh.load(pinned.numpy())
            hh.run(k, l, seed=args.seed0 + s, labels=hlab.numpy())
        torch.cuda.synchronize()
        # every step's input crosses PCIe inside the timed region; the copy of
        # step s+1 (proclus_prefetch) overlaps the clustering of step s
        t0 = time.perf_counter()
        hh.load(pinned.numpy())
        for s in range(e_steps):
            if s + 1 < e_steps:
                hh.prefetch(pinned.numpy())
            hh.run(k, l, seed=args.seed0 + s, labels=hlab.numpy())
            if s + 1 < e_steps:
                hh.load(pinned.numpy())
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        hh.close()
        e2e = {"value": e_steps / dt, "unit": UNIT, "steps": e_steps,
               "h2d_bytes_per_step": int(shard.nbytes),
               "pipelining": "step s+1's H2D (proclus_prefetch) overlaps step s's clustering",
               "d2h_bytes_per_step": int(4 * (hi - lo) + 8 * k + k * d)}

    cpu = None
    parity = None
    if world == 1 and rank == 0 and not args.no_cpu_baseline:
        import oracle

        oracle.build()
        o, dt, ns = cpu_baseline_full(data, cfg, metric)
        what = (f"one full clustering of the {args.config} workload" if ns == n else
                f"one clustering of the first {ns:,} rows of the {args.config} workload, "
                f"scaled by n / n_sample")
        cpu = {"value": 1.0 / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"{what} (seed 1) by the single-threaded fp64 C oracle: "
                         f"{dt:.2f} s, {o.iterations} iterations", **cpu_info()}
        if ns == n and not args.no_all_cores:
            cpu["all_cores"] = cpu_all_cores(args.config, args.data_seed, metric)
        if ns == n:
            hp = handle(metric, stats=False)
            g = hp.run(k, l, seed=1, labels=labels)
            hp.close()
            glab = labels.cpu().numpy()
            parity = {"seed": 1, "labels_equal": bool(np.array_equal(glab, o.labels)),
                      "medoids_equal": bool(np.array_equal(g.medoids, o.medoids)),
                      "dims_equal": bool(np.array_equal(g.dims, o.dims)),
                      "iterations": [g.iterations, o.iterations],
                      "cost_rel_err": abs(g.cost - o.cost) / abs(o.cost)}
        else:
            parity = {"note": "full-size parity: tests/test_gpu_parity.py::test_L8_oracle_parity"}

    if rank == 0:
        iters = m["iters"]
        line = {
            "metric": BASELINE_METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": total_ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": DTYPE, "dtype_note": DTYPE_NOTE, "data": "synthetic",
            "config": workload_config(args, world),
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": m["launches"], "clocks": m["clocks"],
            "iterations_per_run": {"mean": sum(iters) / len(iters), "min": min(iters),
                                   "max": max(iters)},
            "kernels": kernels, "other_metric": other, "parity": parity,
            "tails_ms_total": {kk: round(v, 4) for kk, v in m["tails"].items()},
            "exact_fallbacks": m["fallbacks"],
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier(device_ids=[local])
        dist.destroy_process_group()
    return 0


SWEEP_KS = list(range(5, 21))   # C5: k in {5..20}
SWEEP_LS = list(range(3, 11))   # C5: l in {3..10}
# L8S: 9 combinations of k and l (Fig 3e; the paper does not list
# them -- reading R22: the 3 x 3 grid around the defaults k = 10, l = 5)
GRID9_KS, GRID9_LS = [5, 10, 15], [3, 5, 7]
ORACLE_MAX_ROWS = 2_000_000     # larger workloads: the oracle runs on a prefix


def run_sweep(args):
    """--config C5: the multi-parameter sweep of
    BASELINE.json configs[4] -- k in {5..20} x l in {3..10} (128 settings) at
    n=1M, d=15 through proclus_run_multi with reuse level 2 (S and M drawn
    once for k_max; Dist rows, H, delta', |L| shared by every setting).  One
    step = one whole sweep; value = settings (clusterings) per second.  The
    same 128 settings as independent proclus_run calls are timed beside it
    (the paper's level-0 baseline of Fig 3e)."""
    import torch
    import torch.distributed as dist

    import paper_conf_edbt_jorgensensape22_b200 as pk

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    pk.lib()
    base, ks_grid, ls_grid = (("C3", SWEEP_KS, SWEEP_LS) if args.config == "C5"
                              else ("L8", GRID9_KS, GRID9_LS))
    data, cfg = synth.config_data(base, seed=args.data_seed)
    n, d = cfg["n"], cfg["d"]
    metric = pk.METRIC_L2 if args.metric == "l2" else pk.METRIC_L1
    # settings parallelism: every rank holds the whole dataset and runs the
    # settings r, r + N, ... of the grid (no communication; level 2 draws S
    # and M for the grid's k_max on every rank, so each setting's result is
    # the one the 1-GPU sweep computes)
    stream = torch.cuda.Stream()
    xdev = torch.from_numpy(np.ascontiguousarray(data)).cuda()
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device="cuda")
    h = pk.Proclus(xdev, metric=metric, device=local, stream=stream.cuda_stream)
    settings = [(k, l) for k in ks_grid for l in ls_grid]
    mine = settings[rank::world]
    kmax = max(ks_grid)
    nset = len(settings)

    def barrier():
        if world > 1:
            dist.barrier(device_ids=[local])
        torch.cuda.synchronize()

    lc = [0]

    def timed(fn, steps):
        out = []
        for s in range(steps):
            with torch.cuda.stream(stream):
                flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn(s)
            e1.record(stream)
            e1.synchronize()
            out.append(e0.elapsed_time(e1))
            lc[0] += h.last_launches
        return out

    if world == 1:
        sweep = lambda s: h.run_multi(ks_grid, ls_grid, seed=args.seed0 + s, reuse_level=2)
    else:
        sweep = lambda s: h.run_list(mine, k_sample=kmax, seed=args.seed0 + s, reuse_level=2)
    for s in range(args.warmup):
        sweep(1000 + s)
    barrier()
    with ClockSampler(local) as clk:
        barrier()
        ms = timed(sweep, args.steps)
        barrier()
    total_ms = sum(ms)
    launches = lc[0]
    # level 0: this rank's settings as independent runs (one step); every
    # variant is run once untimed first, as the level-2 sweep was (warm-up),
    # so that each is timed with its CUDA graphs already instantiated
    indep = lambda s: [h.run(k, l, seed=args.seed0 + s) for k, l in mine]
    lev1 = lambda s: h.run_list(mine, k_sample=kmax, seed=args.seed0 + s, reuse_level=1)
    lev3 = lambda s: h.run_multi(ks_grid, ls_grid, seed=args.seed0 + s, reuse_level=3)
    if args.warmup > 0:
        indep(2000)
        lev1(2000)
        if world == 1:
            lev3(2000)
    ms0 = timed(indep, 1)
    ms1 = timed(lev1, 1)
    # level 3: warm start from the previous MBest -- changes results,
    # sequential over the whole grid (one GPU only)
    ms3 = timed(lev3, 1) if world == 1 else [float("nan")]
    if world > 1:
        t = torch.tensor([total_ms, ms0[0], ms1[0]], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms, ms0[0], ms1[0] = (float(v) for v in t.tolist())
    value = args.steps * nset / (total_ms / 1e3)
    cpu = None
    if world == 1 and rank == 0 and not args.no_cpu_baseline:
        import oracle

        oracle.build()
        ns = REF_SAMPLE_ROWS
        ks, ls = [ks_grid[0], ks_grid[-1]], [ls_grid[0], ls_grid[-1]]
        t0 = time.perf_counter()
        oracle.proclus_multi(np.ascontiguousarray(data[:ns]), ks, ls, seed=1, reuse_level=2,
                             metric=0 if args.metric == "l2" else 1)
        dt = (time.perf_counter() - t0) * n / ns
        cpu = {"value": len(ks) * len(ls) / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"oracle multi-parameter run (level 2) of the corner settings "
                         f"k in {ks} x l in {ls} on the first {ns:,} rows, scaled by n/n_sample"}
    h.close()
    if rank == 0:
        line = {
            "metric": BASELINE_METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": total_ms / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": DTYPE,
            "dtype_note": DTYPE_NOTE, "data": "synthetic",
            "config": {"workload": f"{args.config}: multi-parameter grid k in {ks_grid} x l in "
                                   f"{ls_grid} ({nset} settings) at n={n:,} d={d}, reuse level 2 "
                                   f"(P:207-213), A=100 B=10 minDev=0.7 itrPat=5",
                       "settings_per_step": nset, "l2": "256 MiB L2 flush between steps",
                       "parallelism": (f"settings parallel over {world} GPUs (each rank: whole "
                                       f"dataset, settings r::{world} via proclus_run_list)")
                       if world > 1 else "1 GPU"},
            "sweep_ms": {"level2": total_ms / args.steps, "level1": ms1[0],
                         "level3_warm_start": ms3[0], "independent_runs": ms0[0]},
            "reuse_speedup": {"level1": ms0[0] / ms1[0], "level2": ms0[0] / (total_ms / args.steps),
                              "level3": ms0[0] / ms3[0] if world == 1 else None},
            "gpu_launches": launches,
            "cpu_baseline": cpu, "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier(device_ids=[local])
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=["C1", "C2", "C3", "C4", "C5", "L8", "L8S"], default="C3",
                    help="C1-C4: one clustering per step; C5: the k 5..20 x l 3..10 sweep "
                         "at n=1M; L8: one clustering of 8M points; L8S: the 9-setting grid "
                         "at 8M points (Fig 3e)")
    ap.add_argument("--metric", choices=["l2", "l1"], default="l2")
    ap.add_argument("--data-seed", type=int, default=1)
    ap.add_argument("--seed0", type=int, default=1)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-other-metric", action="store_true",
                    help="skip the second full-space metric (L1 beside L2) on the same workload")
    ap.add_argument("--no-all-cores", action="store_true",
                    help="skip the all-core oracle throughput in cpu_baseline")
    ap.add_argument("--variant", choices=["fast", "plain", "star"], default="fast",
                    help="GPU-FAST-PROCLUS (default), GPU-PROCLUS without caches (P:239) "
                         "or GPU-FAST*-PROCLUS (P:215-219)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3  # timing rule: at least 3 warm-up steps
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args)
    if args.config in ("C5", "L8S"):
        return run_sweep(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
