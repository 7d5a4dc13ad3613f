"""Append an A/B table (gpurun_out/<tag>/ab/<variant>_<rep>.json from scripts/gpu_ab.sh) to a
markdown file: ms per step / per-pass binding fraction / e2e ms per repetition.

    python scripts/ab_table.py <tag> <variants file> "<title>" [--out profiles/r02b/ab_runs.md]
"""
import argparse
import json
import os

ap = argparse.ArgumentParser()
ap.add_argument("tag")
ap.add_argument("variants")
ap.add_argument("title")
ap.add_argument("--out", default="profiles/r02b/ab_runs.md")
args = ap.parse_args()
names = [ln.split()[0] for ln in open(args.variants) if ln.strip()]
rows = [f"## {args.tag} ({args.variants}): {args.title}", "", "| variant | run 1 (ms / binding / e2e ms) | run 2 |",
        "|---|---|---|"]
for nm in names:
    cells = []
    for rep in (1, 2):
        f = f"gpurun_out/{args.tag}/ab/{nm}_{rep}.json"
        try:
            d = json.load(open(f))
            cells.append(f"{d['ms_per_step']:.2f} / {d['roofline']['binding']['frac']:.3f} / {d['e2e']['value'] * 1e3:.2f}")
        except Exception:
            cells.append("(failed)")
    rows.append(f"| {nm} | {cells[0]} | {cells[1]} |")
with open(args.out, "a") as fh:
    fh.write("\n" + "\n".join(rows) + "\n")
print("\n".join(rows))
