"""Small circuits through every kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck). Exits non-zero on a parity failure.

    compute-sanitizer --tool racecheck python scripts/sanitize_run.py [--jit 0|2]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import statevector as osv  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402
from workloads import circuits as wc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--jit", type=int, default=0)
ap.add_argument("--big", action="store_true", help="multi-tile-per-CTA cases (buffer reuse)")
ap.add_argument("--new", action="store_true",
                help="zero halves (QFT|0>), host tier with swaps, refined involvement rule")
ap.add_argument("--meas", action="store_true",
                help="round-2 paths: scheduled plans, two-CTA passes, op clustering, scalar folding, "
                     "fused measurement with unrequested lane bits (reduce-scatter epilogue, global reductions)")
args = ap.parse_args()
if args.meas:
    worst = 0.0
    for c in (wc.qaoa(18, 2, seed=3), wc.rqc(18, 6, seed=3), wc.hlf(3, 6, seed=2)):
        plan = q.Circuit(c.qasm()).plan_text(c.n)
        fmap = [int(x) for x in plan.strip().splitlines()[-1].split()[1:]]
        at = {pp: lq for lq, pp in enumerate(fmap) if pp >= 0}
        qubits = [at[0]] + [at[pp] for pp in sorted(at)[-3:]]
        for hglob in ("1", "2"):
            os.environ["QGPU_HGLOB"] = hglob
            with q.State(c.n, fuse_bits=12, jit=args.jit) as s:
                p = s.apply_circuit_probabilities(q.Circuit(c.qasm()), qubits)
                got = s.amplitudes()
            psi = osv.simulate(c.qasm())
            worst = max(worst, float(np.abs(got - psi).max()),
                        float(np.abs(p - osv.probabilities(psi, c.n, qubits)).max()))
    print("max |delta| =", worst)
    sys.exit(0 if worst <= 1e-10 else 1)
cases = [(wc.random_circuit(13, 120, seed=1), 12, 1), (wc.qft(14, x=99), 12, 1), (wc.qaoa(12, 1, seed=2), 9, 1),
         (wc.rqc(13, 4, seed=3), 12, 2), (wc.random_circuit(12, 80, seed=4), 0, 1)]
if args.big:  # > 3 tiles per CTA: exercises the prefetch / triple-buffer reuse and remaps
    cases = [(wc.random_circuit(21, 60, seed=7), 12, 1), (wc.qaoa(20, 1, seed=3), 12, 1),
             (wc.qft(21, x=12345), 12, 1)]
extra = [{}] * len(cases)
if args.new:
    cases = [(wc.qft(17), 12, 1), (wc.qft(15), 9, 1), (wc.random_circuit(13, 120, seed=5), 9, 1),
             (wc.qaoa(14, 1, seed=2), 9, 1), (wc.qft(14), 12, 1)]
    extra = [{}, {}, dict(host_slice_bits=2), dict(host_slice_bits=3), dict(involve_rule=1)]
worst = 0.0
for (c, fuse, world), kw in zip(cases, extra):
    with q.State(c.n, fuse_bits=fuse, jit=args.jit, world_size=world, **kw) as s:
        if args.new:  # stale non-zero data under the skipped halves
            s.apply_circuit(q.Circuit(wc.random_circuit(c.n, 40, seed=9).qasm()))
            s.reset()
        s.apply_circuit(q.Circuit(c.qasm()))
        got = s.amplitudes()
        s.probabilities([0, 3, 5])
    worst = max(worst, float(np.abs(got - osv.simulate(c.qasm())).max()))
print("max |delta| =", worst)
sys.exit(0 if worst <= 1e-10 else 1)
