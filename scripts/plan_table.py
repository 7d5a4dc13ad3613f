"""Pass plans of the workload families with the pass-aware execution order on (default) and off
(QGPU_PASS_SCHED=0): passes, passes at the full live size, HBM bytes per circuit (16 B x live
input + output amplitudes of every pass), planning time. CPU only.

    python scripts/plan_table.py [--n 30]
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=30)
args = ap.parse_args()
q.load()
print("| workload | plan | passes | at full size | GB per circuit | plan ms |")
print("|---|---|---|---|---|---|")
for name, n in (("qaoa32", 32), ("qaoa32", args.n), ("qft28", 28), ("rqc", args.n), ("hlf", args.n), ("gs", args.n),
                ("iqp", args.n), ("bv", args.n)):
    circ, desc = bench.workload(name, n)
    for sched in ("1", "0"):
        os.environ["QGPU_PASS_SCHED"] = sched
        c = q.Circuit(circ.qasm())
        t0 = time.perf_counter()
        plan = c.plan(circ.n, 1, 2, 12)
        ms = (time.perf_counter() - t0) * 1e3
        gb = sum(16.0 * (2.0 ** r[3] + 2.0 ** r[4]) for r in plan if r[2] == 0) / 1e9
        full = sum(1 for r in plan if r[2] == 0 and r[3] == circ.n)
        print(f"| {desc.split(' ')[0]} | {'auto' if sched == '1' else 'consecutive'} | {len(plan)} | {full} | "
              f"{gb:.1f} | {ms:.1f} |")
