"""Summarise an ncu report's source page: stall samples and executed instructions per CUDA
source line (needs -lineinfo), top N lines.

    python scripts/ncu_source_summary.py gpurun_out/prof.ncu-rep [--top 25] [--kernel tile_kernel]
"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 25
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    res = []
    hdr = None
    for r in rows:
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr) or r[2] != "-":
            continue
        try:
            res.append((int(r[4]), int(r[7]), r[0], r[1][:110]))
        except ValueError:
            pass
    tot_s = sum(x[0] for x in res) or 1
    tot_i = sum(x[1] for x in res) or 1
    print(f"total stall samples {tot_s}, warp instructions {tot_i}")
    for s, i, ln, src in sorted(res, reverse=True)[:top]:
        print(f"{100*s/tot_s:5.1f}% samples {100*i/tot_i:5.1f}% instr  L{ln:>4}  {src}")


if __name__ == "__main__":
    main()
