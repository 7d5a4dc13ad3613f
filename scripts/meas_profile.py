"""Per-pass times (timing=2) of a circuit with and without the fused end-of-circuit measurement
(qgpu_apply_circuit_probabilities of qubits 0..9): what the measurement epilogue costs the pass."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

circ, _ = bench.workload(sys.argv[1] if len(sys.argv) > 1 else "qaoa32", None)
c = q.Circuit(circ.qasm())
s = q.State(circ.n, timing=2)
qs = list(range(10))
for fused in (False, True, False, True):
    s.reset()
    s.pass_profile()
    if fused:
        s.apply_circuit_probabilities(c, qs)
    else:
        s.apply_circuit(c)
    prof = s.pass_profile()
    print("fused" if fused else "plain", " ".join(f"{p['k_in']}->{p['k_out']}:{p['ms']:.2f}" for p in prof),
          f"total {sum(p['ms'] for p in prof):.2f} ms")
