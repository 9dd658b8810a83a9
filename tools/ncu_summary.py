"""Summarise the ncu evidence of one profiling round into profiles/.

usage: python tools/ncu_summary.py gpurun_out/prof_r01 r01

Reads <dir>/launches.csv (ncu --metrics gpu__time_duration.sum over
bench.py) and <dir>/full.ncu-rep (ncu --set full of the pass kernels) and
writes profiles/<tag>_launches.csv (copy), profiles/<tag>_ncu_summary.md and
profiles/ncu_traffic.json (dram bytes per launch of each kernel, read by
bench.py for roofline.traffic)."""
import csv
import io
import json
import os
import re
import shutil
import subprocess
import sys
from collections import defaultdict

src, tag = sys.argv[1], sys.argv[2]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
prof = os.path.join(ROOT, "profiles")
os.makedirs(prof, exist_ok=True)


def short(name):
    m = re.search(r"(k_[a-z_]+)(<[^>]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else name[:40]


# ---- launch list: share of device time per kernel
rows = []
with open(os.path.join(src, "launches.csv")) as f:
    lines = [l for l in f if l.startswith('"')]
rd = csv.DictReader(io.StringIO("".join(lines)))
for r in rd:
    if r.get("Metric Name") == "gpu__time_duration.sum":
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        us = v * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0,
                  "ms": 1e3, "msecond": 1e3}.get(unit, 1.0)
        rows.append((short(r["Kernel Name"]), us))
shutil.copy(os.path.join(src, "launches.csv"), os.path.join(prof, f"{tag}_launches.csv"))
tot = sum(u for _, u in rows) or 1.0
by = defaultdict(lambda: [0, 0.0])
for n, u in rows:
    by[n][0] += 1
    by[n][1] += u

# ---- full captures (every <dir>/full*.ncu-rep): per-launch metrics
want = {
    "dur_us": "gpu__time_duration.sum",
    "dram_rd_MB": "dram__bytes_read.sum",
    "dram_wr_MB": "dram__bytes_write.sum",
    "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "warps_active": "sm__warps_active.avg.per_cycle_active",
    "issue_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "inst_M": "smsp__inst_executed.sum",
    "regs": "launch__registers_per_thread",
    "grid": "launch__grid_size",
    "block": "launch__block_size",
    "smem_KB": "launch__shared_mem_per_block_dynamic",
}
full = []
reps = sorted(f for f in os.listdir(src) if f.startswith("full") and f.endswith(".ncu-rep"))
for rep in reps:
  raw = subprocess.run(["ncu", "-i", os.path.join(src, rep), "--page", "raw", "--csv"],
                       capture_output=True, text=True).stdout
  rr = list(csv.reader(io.StringIO(raw)))
  hdr, data = rr[0], rr[2:]
  idx = {k: hdr.index(v) for k, v in want.items() if v in hdr}
  units = rr[1]
  for r in data:
      rec = {"kernel": short(r[hdr.index("Kernel Name")]), "capture": rep}
      for k, i in idx.items():
          try:
              val = float(r[i].replace(",", ""))
          except ValueError:
              continue
          u = units[i]
          if k.startswith("dram_") and k.endswith("MB"):
              val = val * {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}.get(u, 1.0)
          if k == "dur_us":
              val = val * {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(u, 1.0)
          if k == "inst_M":
              val = val / 1e6
          if k == "smem_KB":
              val = val * {"byte": 1 / 1024, "Kbyte": 1.0, "Mbyte": 1024.0}.get(u, 1.0)
          rec[k] = round(val, 3)
      full.append(rec)

traffic, tcount = {}, {}
for rec in full:
    if rec["capture"] != "full.ncu-rep" and rec["capture"] != "full_ac.ncu-rep":
        continue  # roofline traffic: the C3 workload only
    kname = rec["kernel"]
    base = re.sub(r"<.*", "", kname).replace("k_", "")
    if base in ("lsum2", "labelsum"):
        base = "refine_x" if "<1>" in kname else "cost"
    name = {"cost1": "cost", "greedy_cluster": "greedy", "sdist": "greedy"}.get(base, base)
    if "dram_rd_MB" in rec:
        traffic[name] = traffic.get(name, 0.0) + (rec["dram_rd_MB"] + rec.get("dram_wr_MB", 0.0)) * 1e6
        tcount[name] = tcount.get(name, 0) + 1
traffic = {kk: v / tcount[kk] for kk, v in traffic.items()}
with open(os.path.join(prof, "ncu_traffic.json"), "w") as f:
    json.dump({"source": f"profiles/{tag}_ncu_summary.md (ncu --set full, cold L2, mean "
                         f"dram read+write bytes per launch over the captured launches)",
               **traffic}, f, indent=1)

with open(os.path.join(prof, f"{tag}_ncu_summary.md"), "w") as f:
    f.write(f"# ncu summary, {tag}\n\n")
    f.write("Source: `bash tools/profile_round.sh` on one B200 (PROCLUS_GRAPH=0: the same\n"
            "kernels launched from the stream, since ncu cannot profile kernels inside a\n"
            "graph with conditional nodes).  Launch list: `ncu --metrics\n"
            "gpu__time_duration.sum --clock-control none` over `bench.py --steps 2\n"
            "--warmup 3` (cold-cache and serialised: compare shares, not absolutes).\n"
            "Full captures: `ncu --set full --clock-control none` (tools/profile_r02.sh):\n"
            "full.ncu-rep = C3 k_locality launches 2-5, full_ac.ncu-rep = C3 assign / cost,\n"
            "full_c4.ncu-rep = C4 (256k x 100) pass kernels and split tails\n"
            "(tools/profile_run.py C3|C4 1).\n\n")
    f.write("## Share of device time by kernel (launch list)\n\n")
    f.write("| kernel | launches | total us | mean us | share |\n|---|---|---|---|---|\n")
    for n, (c, u) in sorted(by.items(), key=lambda kv: -kv[1][1]):
        f.write(f"| {n} | {c} | {u:.1f} | {u / c:.2f} | {u / tot:.3f} |\n")
    f.write("\n## Full capture, per launch\n\n")
    cols = ["kernel", "capture"] + [k for k in want if any(k in r for r in full)]
    f.write("| " + " | ".join(cols) + " |\n|" + "---|" * len(cols) + "\n")
    for rec in full:
        f.write("| " + " | ".join(str(rec.get(c, "")) for c in cols) + " |\n")
print(open(os.path.join(prof, f"{tag}_ncu_summary.md")).read())
