"""Host wall-clock breakdown of the bench e2e step (parse, reset, apply + fused probabilities),
next to the separate path (apply, then the readout kernel) and a host-only re-apply of the cached
plan (no device work pending: what the host adds per call)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

circ, _ = bench.workload(sys.argv[1] if len(sys.argv) > 1 else "qft28", None)
text = circ.qasm()
s = q.State(circ.n)
qs = list(range(10))
for it in range(8):
    s.synchronize()
    t0 = time.perf_counter()
    c = q.Circuit(text)
    t1 = time.perf_counter()
    s.reset()
    t2 = time.perf_counter()
    p = s.apply_circuit_probabilities(c, qs)
    t3 = time.perf_counter()
    s.reset()
    s.apply_circuit(c)
    t4 = time.perf_counter()
    s.synchronize()
    t5 = time.perf_counter()
    p2 = s.probabilities(qs)
    t6 = time.perf_counter()
    st = s.stats()
    print(f"parse {1e3*(t1-t0):.3f}  reset {1e3*(t2-t1):.3f}  apply+fused probs {1e3*(t3-t2):.3f}  | "
          f"apply enqueue {1e3*(t4-t3):.3f}  sync {1e3*(t5-t4):.3f}  readout {1e3*(t6-t5):.3f} ms  "
          f"kernel_ms {st.get('kernel_ms', 0):.3f}")
    c.close()
