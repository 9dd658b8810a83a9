"""Summarise an ncu report's source page: top SASS instructions by warp-stall
samples for one kernel, with the dominant stall reasons.
usage: python tools/ncu_hot.py REPORT KERNEL_REGEX [TOP]"""
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", f"regex:{kern}", "--launch-count", "1"],
                     capture_output=True, text=True).stdout
lines = out.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
hdr = rows[0]
si = hdr.index("Warp Stall Sampling (All Samples)")
rows = [hdr] + [r for r in rows[1:] if len(r) > si and r[si].strip().isdigit()]
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
total = sum(int(r[si] or 0) for r in rows[1:])
print(f"total samples {total}")
agg = {}
for r in rows[1:]:
    for i in stall_cols:
        agg[hdr[i]] = agg.get(hdr[i], 0) + int(r[i] or 0)
print("stalls:", sorted(((v, k) for k, v in agg.items() if v), reverse=True)[:8])
for r in sorted(rows[1:], key=lambda r: -int(r[si] or 0))[:top]:
    st = sorted(((int(r[i] or 0), hdr[i]) for i in stall_cols), reverse=True)[:2]
    print(f"{int(r[si]):6d} {r[0][-5:]} {r[1].strip()[:60]:60s} {st}")
