"""Per-launch table from an ncu --csv launch list (second half = the timed step)."""
import csv, sys
from collections import OrderedDict
rows = OrderedDict()
lines = open(sys.argv[1]).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
for r in csv.DictReader(lines[start:]):
    k = int(r["ID"])
    d = rows.setdefault(k, {"name": r["Kernel Name"][:28]})
    d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
ids = list(rows)
half = ids[len(ids) // 2:]
tot = sum(rows[i]["gpu__time_duration.sum"] for i in half)
print(f"{'id':>3} {'kernel':28} {'ms':>8} {'share':>6} {'rd GB':>7} {'wr GB':>7} {'GB/s':>7} {'fp64%':>6} {'iss%':>6}")
for i in half:
    d = rows[i]
    ms = d["gpu__time_duration.sum"] / 1e6
    rd, wr = d.get("dram__bytes_read.sum", 0) / 1e9, d.get("dram__bytes_write.sum", 0) / 1e9
    print(f"{i:>3} {d['name']:28} {ms:8.3f} {ms*1e6/tot:6.3f} {rd:7.2f} {wr:7.2f} {(rd+wr)/ms*1e3 if ms else 0:7.0f} "
          f"{d.get('sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active', 0):6.1f} "
          f"{d.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):6.1f}")
print(f"total {tot/1e6:.2f} ms")
