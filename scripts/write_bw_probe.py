"""Write-only and read-only HBM bandwidth on this GPU (torch fill_ / sum over a 4 GiB buffer,
CUDA events, best of 10): the ceiling of write-dominated expansion passes (e.g. QFT_28's last,
0.54 GB read + 4.23 GB written)."""
import json

import torch

x = torch.empty(1 << 29, dtype=torch.float64, device="cuda")  # 4 GiB
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {}
for name, fn, nbytes in (("write_fill", lambda: x.fill_(1.5), x.numel() * 8),
                         ("read_sum", lambda: x.sum(), x.numel() * 8),
                         ("copy", lambda: y.copy_(x), 2 * x.numel() * 8)):
    if name == "copy":
        y = torch.empty_like(x)
    best = 1e9
    for _ in range(12):
        torch.cuda.synchronize()
        ev0.record()
        fn()
        ev1.record()
        torch.cuda.synchronize()
        best = min(best, ev0.elapsed_time(ev1))
    res[name] = {"ms": best, "GBps": nbytes / best / 1e6}
print(json.dumps(res))
