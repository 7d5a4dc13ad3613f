"""Hot SASS basic blocks (by executed instructions) of the biggest kernel launch in an ncu report.

    python scripts/ncu_sass_blocks.py report.ncu-rep [--top 25] [--section K]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
his = [i for i, x in enumerate(r) if x and x[0] == "Address"] + [len(r)]
secs = []
for si in range(len(his) - 1):
    h = r[his[si]]
    ie, src, st = h.index("Instructions Executed"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
    rows = [(x[0], x[src], int(x[ie]), int(x[st])) for x in r[his[si] + 1:his[si + 1]]
            if len(x) == len(h) and x[ie].isdigit()]
    secs.append(rows)
if "--section" in sys.argv:
    rows = secs[int(sys.argv[sys.argv.index("--section") + 1])]
else:
    rows = max(secs, key=lambda rr: sum(x[2] for x in rr))
tot = sum(x[2] for x in rows)
print("sections", len(secs), "totals", [sum(x[2] for x in rr) for rr in secs])
blocks, cur = [], None
for a, s_, i, stl in rows:
    op = s_.split()[1] if s_.strip().startswith("@") else s_.split()[0]
    if cur and cur[1] == i:
        cur[2] += 1; cur[3] += stl; cur[4].append(op)
    else:
        if cur:
            blocks.append(cur)
        cur = [a, i, 1, stl, [op]]
blocks.append(cur)
tot_st = sum(b[3] for b in blocks) or 1
blocks.sort(key=lambda b: -b[1] * b[2])
for b in blocks[:top]:
    print(b[0][-5:], "exec", b[1], "len", b[2], f"{100*b[1]*b[2]/tot:5.1f}% instr",
          f"{100*b[3]/tot_st:5.1f}% stall", " ".join(b[4][:18]))
