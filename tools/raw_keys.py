"""Key metrics of every launch in an ncu --page raw --csv dump:
  python tools/raw_keys.py RAW.csv"""
import csv
import sys

KEYS = [("gpu__time_duration.sum", "dur_us", 1e-3),
        ("dram__bytes_read.sum", "rd_MB", 1e-6), ("dram__bytes_write.sum", "wr_MB", 1e-6),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps%", 1),
        ("sm__inst_issued.avg.pct_of_peak_sustained_active", "issue%", 1),
        ("smsp__inst_executed.sum", "inst_M", 1e-6),
        ("launch__registers_per_thread", "regs", 1),
        ("launch__grid_size", "grid", 1)]
rows = list(csv.reader(open(sys.argv[1])))
hdr, units = rows[0], rows[1]
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    out = [d.get("Kernel Name", "?")[:30]]
    for k, name, sc in KEYS:
        v = d.get(k, "")
        try:
            x = float(v.replace(",", ""))
            u = units[hdr.index(k)]
            if k == "gpu__time_duration.sum" and u == "usecond":
                x *= 1e3
            if k.startswith("dram__bytes") and u in ("Mbyte", "MB"):
                x *= 1e6
            if k.startswith("dram__bytes") and u in ("Kbyte", "KB"):
                x *= 1e3
            if k.startswith("dram__bytes") and u in ("Gbyte", "GB"):
                x *= 1e9
            out.append(f"{name}={x * sc:.2f}")
        except Exception:
            out.append(f"{name}={v}")
    print(" ".join(out))
