"""Time the GFC kernels (qgpu_gfc_compress / _decompress) on the state left by a workload."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import torch  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402

w = sys.argv[1] if len(sys.argv) > 1 else "qft28"
nq = int(sys.argv[2]) if len(sys.argv) > 2 else None
seg = int(sys.argv[3]) if len(sys.argv) > 3 else 4096
circ, desc = bench.workload(w, nq)
s = q.State(circ.n)
s.apply_circuit(q.Circuit(circ.qasm()))
s.synchronize()
n_q, n_loc, dev = s.info()
n = 2 << n_loc
cap = q.gfc_max_bytes(n, seg)
out = torch.empty(cap, dtype=torch.uint8, device="cuda")
off = torch.empty((n + seg - 1) // seg + 1, dtype=torch.int64, device="cuda")
back = torch.empty(n, dtype=torch.float64, device="cuda")
for it in range(4):
    torch.cuda.synchronize()
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record()
    nb = q.gfc_compress(dev, n, seg, out.data_ptr(), cap, off.data_ptr())
    e1.record()
    q.gfc_decompress(out.data_ptr(), off.data_ptr(), n, seg, back.data_ptr())
    e2.record()
    torch.cuda.synchronize()
    tc, td = e0.elapsed_time(e1), e1.elapsed_time(e2)
print(f"{desc[:30]} n={n} doubles seg={seg}: ratio {8*n/nb:.3f}  compress {tc:.3f} ms ({8*n/tc/1e6:.0f} GB/s in)  "
      f"decompress {td:.3f} ms ({8*n/td/1e6:.0f} GB/s out)")
# lossless check: compress the decompressed copy again, the streams must be identical
out2 = torch.empty(cap, dtype=torch.uint8, device="cuda")
off2 = torch.empty_like(off)
nb2 = q.gfc_compress(back.data_ptr(), n, seg, out2.data_ptr(), cap, off2.data_ptr())
assert nb2 == nb and torch.equal(out[:nb], out2[:nb]) and torch.equal(off, off2), "round trip mismatch"
print("round trip: re-compressed stream identical")
