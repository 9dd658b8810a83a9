"""Per-CUDA-line instruction counts and stall samples of one kernel from an
ncu report with imported source (--print-source cuda,sass):
  python tools/ncu_src.py REPORT KERNEL_REGEX [TOP] [LAUNCH_SKIP]"""
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
skip = sys.argv[4] if len(sys.argv) > 4 else "0"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "-k", f"regex:{kern}", "--launch-skip", skip, "--launch-count", "1"],
                     capture_output=True, text=True).stdout
rows = []
fname = "?"
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if r[0] and r[0].isdigit() and len(r) > 8:
        num = lambda v: int(v) if v.strip().isdigit() else 0
        rows.append((fname, int(r[0]), r[1], num(r[4]), num(r[7])))
ti = sum(x[4] for x in rows) or 1
ts = sum(x[3] for x in rows) or 1
print(f"total inst {ti:,}  samples {ts:,}")
for f, ln, src, smp, ins in sorted(rows, key=lambda x: -x[4])[:top]:
    print(f"{100*ins/ti:5.1f}% inst {100*smp/ts:5.1f}% smp  {f}:{ln:<5d} {src.strip()[:80]}")
