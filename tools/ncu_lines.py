"""Attribute ncu warp-stall samples of one kernel to CUDA source lines.

usage: python tools/ncu_lines.py REPORT KERNEL_REGEX MANGLED_NAME [TOP]
Aligns the report's SASS rows (address order) with `nvdisasm -g` of the
in-tree libproclus.so (which carries -lineinfo)."""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, kern, mangled = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 25
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
so = os.path.join(ROOT, "paper_conf_edbt_jorgensensape22_b200", "libproclus.so")
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", so], cwd=tmp, capture_output=True)
cub = [f for f in os.listdir(tmp) if f.startswith("proclus_kernels") and "api" not in f][0]
dis = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(tmp, cub)], capture_output=True,
                     text=True).stdout.splitlines()
seq, cur, inside = [], None, False
for ln in dis:
    if ln.startswith(".text.") and ln.rstrip(":").endswith(mangled):
        inside = True
        continue
    if inside and ln.startswith("//---------------------"):
        break
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    if re.match(r"\s+/\*[0-9a-f]{4,}\*/", ln):
        seq.append(cur)
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", f"regex:{kern}", "--launch-count", "1"], capture_output=True,
                     text=True).stdout.splitlines()
start = next(i for i, l in enumerate(out) if l.startswith('"Address"'))
rows = list(csv.reader(io.StringIO("\n".join(out[start:]))))
hdr = rows[0]
si = hdr.index(os.environ.get("NCU_COL", "Warp Stall Sampling (All Samples)"))
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
data, seen = [], set()
for r in rows[1:]:
    if len(r) > si and re.fullmatch(r"[0-9.]+", r[si].strip() or "x") and r[0] not in seen:
        seen.add(r[0])
        data.append(r)
if len(data) != len(seq):
    print(f"warning: {len(data)} ncu rows vs {len(seq)} disassembled instructions")
src = {}
agg = {}
for r, loc in zip(data, seq):
    a = agg.setdefault(loc, [0, {}])
    a[0] += int(float(r[si]))
    for i in stall_cols:
        v = int(r[i] or 0)
        if v:
            a[1][hdr[i]] = a[1].get(hdr[i], 0) + v
tot = sum(v[0] for v in agg.values())
print(f"total samples {tot}")
files = {}
for (loc, (n, st)) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    if loc is None:
        print(f"{n:6d} {100*n/tot:5.1f}%  ?")
        continue
    f, line = loc
    if f not in files:
        for d in (os.path.join(ROOT, "paper_conf_edbt_jorgensensape22_b200", "csrc"),):
            p = os.path.join(d, f)
            files[f] = open(p).read().splitlines() if os.path.exists(p) else []
    text = files[f][line - 1].strip() if 0 < line <= len(files[f]) else ""
    s = sorted(st.items(), key=lambda kv: -kv[1])[:2]
    print(f"{n:6d} {100*n/tot:5.1f}%  {f}:{line:<5d} {text[:70]:70s} {s}")
