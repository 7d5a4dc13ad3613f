"""Host wall-clock breakdown of the bench e2e step (parse, reset+apply, probabilities)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

circ, _ = bench.workload(sys.argv[1] if len(sys.argv) > 1 else "qft28", None)
text = circ.qasm()
s = q.State(circ.n)
for it in range(6):
    t0 = time.perf_counter()
    c = q.Circuit(text)
    t1 = time.perf_counter()
    s.reset()
    s.apply_circuit(c)
    s.synchronize()
    t2 = time.perf_counter()
    p = s.probabilities(list(range(10)))
    t3 = time.perf_counter()
    p2 = s.probabilities([])
    t4 = time.perf_counter()
    print(f"parse {1e3*(t1-t0):.3f} ms  apply+sync {1e3*(t2-t1):.3f} ms  probs(10) {1e3*(t3-t2):.3f} ms  norm {1e3*(t4-t3):.3f} ms")
