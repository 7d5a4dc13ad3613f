"""One warm-up + one timed step of a workload through the C ABI (for ncu / compute-sanitizer).

    python scripts/profile_step.py [--workload qft28] [--n N] [--fuse-bits 12] [--steps 1]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="qft28")
ap.add_argument("--n", type=int, default=None)
ap.add_argument("--fuse-bits", type=int, default=12)
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--single", type=int, default=None, help="instead: one 1-qubit gate at this target on a full state")
ap.add_argument("--stats-out", default=None, help="write the last circuit's qgpu_stats as JSON here")
args = ap.parse_args()

import numpy as np  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

if args.single is not None:
    n = args.n or 30
    s = q.State(n, fuse_bits=0)
    H = np.array([[1, 1], [1, -1]]) / np.sqrt(2)
    for t in range(n):
        s.apply_gate(H, [t])
    for _ in range(args.steps):
        s.apply_gate(H, [args.single])
    s.synchronize()
    sys.exit(0)

circ, desc = bench.workload(args.workload, args.n)
c = q.Circuit(circ.qasm())
s = q.State(circ.n, fuse_bits=args.fuse_bits)
for i in range(1 + args.steps):
    s.reset()
    if i == args.steps:
        s.reset_stats()
    s.apply_circuit(c)
s.synchronize()
st = s.stats()
print(desc, st)
if args.stats_out:
    import json
    json.dump({"workload": args.workload, "n": circ.n, "desc": desc, "stats": st}, open(args.stats_out, "w"), indent=1)
