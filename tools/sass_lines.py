"""Static SASS instruction counts per source line of one kernel (nvdisasm -g):
  python tools/sass_lines.py CUBIN KERNEL_SUBSTR [LINE_LO LINE_HI]"""
import collections
import re
import subprocess
import sys

cubin, kern = sys.argv[1], sys.argv[2]
lo, hi = (int(sys.argv[3]), int(sys.argv[4])) if len(sys.argv) > 4 else (0, 10 ** 9)
out = subprocess.run(["nvdisasm", "-g", cubin], capture_output=True, text=True).stdout
infn, cur = False, None
cnt, ops = collections.Counter(), collections.defaultdict(collections.Counter)
for l in out.split("\n"):
    if l.startswith(".text."):
        infn = kern in l
        continue
    if not infn:
        continue
    m = re.search(r"line (\d+)", l)
    if "## File" in l and m:
        cur = (l.split('"')[1].split("/")[-1] if '"' in l else "?", int(m.group(1)))
        continue
    m2 = re.match(r"\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", l)
    if m2 and cur:
        cnt[cur] += 1
        ops[cur][m2.group(2).split(".")[0]] += 1
tot = 0
for k in sorted(cnt):
    if k[0] == "proclus_kernels.cu" and lo <= k[1] <= hi:
        print(k[1], cnt[k], dict(ops[k]))
        tot += cnt[k]
print("total", tot)
