"""Text summary of an ncu report (--set full): per kernel launch the time, DRAM bytes, pipe and
issue utilisation, registers / occupancy, the stall mix per issued instruction, shared-memory
wavefronts and shuffles, and the SASS opcode mix with stall samples (source page, SASS view).

    python scripts/ncu_summary.py <report.ncu-rep> [--top 18]
"""
import collections
import csv
import io
import subprocess
import sys

METRICS = [
    ("time_ms", "gpu__time_duration.sum"), ("dram_read_GB", "dram__bytes_read.sum"),
    ("dram_write_GB", "dram__bytes_write.sum"),
    ("fp64_pipe_pct", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"),
    ("issue_active_pct", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
    ("warps_active_pct", "sm__warps_active.avg.pct_of_peak_sustained_active"),
    ("registers", "launch__registers_per_thread"), ("grid", "launch__grid_size"),
    ("block", "launch__block_size"), ("warp_instr", "smsp__inst_executed.sum"),
    ("shared_wavefronts", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
    ("local_loads", "sass__inst_executed_local_loads"), ("local_stores", "sass__inst_executed_local_stores"),
]


def ncu(rep, *args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


def main():
    rep = sys.argv[1]
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 18
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    hdr, units, data = rows[0], rows[1], rows[2:]
    idx = {h: i for i, h in enumerate(hdr)}
    for k, r in enumerate(data):
        print(f"== launch {k}: {r[idx['Kernel Name']]}")
        for name, m in METRICS:
            if m in idx:
                print(f"  {name:18s} {r[idx[m]]} {units[idx[m]]}")
        stalls = []
        for h, i in idx.items():
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(r[i]), h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        print("  stalls per issue: " + ", ".join(f"{n} {v:.2f}" for v, n in sorted(stalls, reverse=True)[:10]))
    src = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source", "sass"))))
    blocks, cur = [], None
    for r in src:
        if r and r[0] == "Kernel Name":
            cur = []
            blocks.append(cur)
        elif cur is not None:
            cur.append(r)
    for k, b in enumerate(blocks):
        if not b:
            continue
        h = b[0]
        ix = {x: i for i, x in enumerate(h)}
        inst, samp = collections.Counter(), collections.Counter()
        for r in b[1:]:
            if len(r) != len(h):
                continue
            op = r[1].strip().split()
            if not op:
                continue
            o = op[1] if op[0].startswith("@") and len(op) > 1 else op[0]
            o = o.split(".")[0]
            inst[o] += int(r[ix["Instructions Executed"]] or 0)
            samp[o] += int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        ti, ts = sum(inst.values()) or 1, sum(samp.values()) or 1
        print(f"== launch {k} SASS mix (share of warp instructions / of stall samples)")
        for o, v in inst.most_common(top):
            print(f"  {o:10s} {100 * v / ti:5.1f}% {100 * samp[o] / ts:5.1f}%")


if __name__ == "__main__":
    main()
