"""Turn the ncu outputs brought back by gpurun into committed summaries under profiles/.

    python scripts/make_profiles.py --launches gpurun_out/launches.csv [--full gpurun_out/prof.ncu-rep]
                                    --tag r01 --workload qft28 --n 28

* launches.csv: `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
  --clock-control none --csv` of scripts/profile_step.py (1 warm-up + 1 step). The second step's
  launches are summarised (kernel, duration, DRAM bytes, share of the step) and the mean DRAM
  traffic per fused-tile launch is written to profiles/ncu_traffic.json (bench.py's
  roofline.traffic).
* prof.ncu-rep: `ncu --set full` capture; key raw metrics per launch are written as CSV.
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import OrderedDict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__shared_mem_per_block_dynamic",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio"]


def parse_launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    launches = OrderedDict()
    for r in rows[hi + 1:]:
        d = launches.setdefault(int(r[0]), {"kernel": r[ki]})
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        if unit == "ns":
            v *= 1e-6
        elif unit == "us":
            v *= 1e-3
        elif unit in ("Kbyte", "KB"):
            v *= 1e3
        elif unit in ("Mbyte", "MB"):
            v *= 1e6
        elif unit in ("Gbyte", "GB"):
            v *= 1e9
        d[r[mi]] = v
    return launches


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--full")
    ap.add_argument("--tag", default="r01")
    ap.add_argument("--workload", default="qft28")
    ap.add_argument("--n", type=int, default=28)
    ap.add_argument("--stats", help="profile_step.py --stats-out of the profiled run (plan fingerprint)")
    args = ap.parse_args()
    out = os.path.join(ROOT, "profiles", args.tag)
    os.makedirs(out, exist_ok=True)
    if args.launches:
        L = parse_launches(args.launches)
        ids = list(L)
        # steps start at set_amp_kernel (qgpu_state_reset); keep the last step
        starts = [i for i in ids if "set_amp" in L[i]["kernel"]]
        last = [i for i in ids if i >= starts[-1]] if starts else ids
        tot = sum(L[i].get("gpu__time_duration.sum", 0) for i in last)
        lines = ["launch,kernel,ms,dram_read_GB,dram_write_GB,share_of_step"]
        tile = []
        for i in last:
            d = L[i]
            ms = d.get("gpu__time_duration.sum", 0.0)
            rd, wr = d.get("dram__bytes_read.sum", 0.0), d.get("dram__bytes_write.sum", 0.0)
            name = d["kernel"].split("(")[0]
            lines.append(f"{i},{name},{ms:.4f},{rd/1e9:.4f},{wr/1e9:.4f},{ms/tot if tot else 0:.3f}")
            if "tile" in name:
                tile.append((ms, rd + wr))
        open(os.path.join(out, f"{args.workload}_launches.csv"), "w").write("\n".join(lines) + "\n")
        if tile:
            # keyed "<workload>_<n>" entries read by bench.py (roofline.traffic), with the plan's
            # fingerprint (tile launches and algorithmic bytes per launch of the profiled circuit)
            tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
            allt = json.load(open(tp)) if os.path.exists(tp) else {}
            tr = {"workload": args.workload, "n": args.n,
                  "dram_bytes_per_launch": sum(t[1] for t in tile) / len(tile),
                  "launches_per_circuit": len(tile), "dram_bytes_per_circuit": sum(t[1] for t in tile),
                  "tile_share_of_step": sum(t[0] for t in tile) / tot if tot else None,
                  "source": f"profiles/{args.tag}/{args.workload}_launches.csv (ncu --metrics gpu__time_duration.sum,"
                            "dram__bytes_read.sum,dram__bytes_write.sum --clock-control none, "
                            "scripts/profile_step.py: second circuit)"}
            if args.stats:
                st = json.load(open(args.stats))["stats"]
                if st["tile_kernel_launches"]:  # (filled when the profiled run had timing on)
                    nl, ab = st["tile_kernel_launches"], st["tile_algo_bytes"]
                else:  # every launched kernel a tile pass (QAOA / QFT): the totals are the tile ones
                    assert st["kernels_launched"] == len(tile), st
                    nl, ab = st["kernels_launched"], st["algo_bytes"]
                tr["algo_bytes_per_launch"] = ab / nl
                tr["launches_per_circuit_stats"] = nl
            allt[f"{args.workload}_{args.n}"] = tr
            json.dump(allt, open(tp, "w"), indent=1)
        print("\n".join(lines))
    if args.full:
        txt = subprocess.run(["ncu", "-i", args.full, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        r = list(csv.reader(io.StringIO(txt)))
        h = r[0]
        rows = ["metric," + ",".join(f"launch{i}" for i in range(len(r) - 2))]
        for k in KEYS:
            if k in h:
                rows.append(k + "," + ",".join(x[h.index(k)] for x in r[2:]))
        name = os.path.splitext(os.path.basename(args.full))[0]
        open(os.path.join(out, f"{args.workload}_{name}_raw.csv"), "w").write("\n".join(rows) + "\n")
        print("\n".join(rows))


if __name__ == "__main__":
    main()
