#!/usr/bin/env python
"""Benchmark of the B200 Q-GPU hot path (one JSON line on rank 0).

Default workload (BASELINE.json configs[2], the largest single-GPU configuration): QAOA MaxCut
p=2 on a random 3-regular graph, 32 qubits (2^32 complex128 amplitudes = 64 GiB resident in
HBM) on 1x B200 with delayed qubit involvement and pruning (reorder=2, prune=1, fused passes
b=12). A step = qgpu_state_reset + qgpu_apply_circuit of the whole circuit (every gate); the
metric is circuit seconds (lower is better). configs[1] (QFT_28 on |0...0> and on a random
basis state |x>) and the SURVEY §8d single-gate microbenchmark at n=32 are reported as extra
keys. See DESIGN.md §7 for the byte / FP64 models and the peaks.

    python bench.py [--gpus N --steps K --warmup W] [--workload qaoa32|qft28|qft28x|rqc|gs|hlf|grqc|iqp|bv]
    python bench.py --impl reference ...     # the oracle (plain CPU simulator) as the baseline arm

N > 1 (torchrun): each rank runs its own replica of the workload (weak scaling, no data-path
collective), timed on the device, max over ranks. With --sharded one state is sharded over the N
ranks (top log2 N qubits on rank bits, global-local swaps over NCCL; configs[3]: --workload rqc
--n 34 --sharded), strong scaling.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "circuit sec & gate-apply HBM GB/s vs peak, 28–36 qubits, 1/2/4/8 B200"


def qft_x(nbits: int) -> int:
    """The basis state of QFT_n|x> ("x = rng 28-bit", seed 2)."""
    import numpy as np
    return int(np.random.default_rng(2).integers(0, 1 << nbits))


def run_config(args, circ, desc, world: int = 1, sharded: bool = False) -> dict:
    """The `config` object of the JSON line, shared by both arms (same workload, same keys)."""
    return {"workload": desc, "n_qubits": circ.n, "gates": len(circ.ops), "reorder": args.reorder,
            "prune": int(not args.no_prune), "fuse_bits": args.fuse_bits,
            "replicas_per_gpu": 0 if sharded else 1,
            "parallelism": (f"sharded x{world} (NCCL global-local swaps)" if sharded else
                            f"replicas x{world}" if world > 1 else "1 GPU"),
            "l2": "flushed between timed steps (256 MiB write) and state 16*2^n B > L2"}


def grid_shape(n: int):
    """rows x cols = n with rows <= cols as close as possible (grid workloads)."""
    r = int(math.isqrt(n))
    while n % r:
        r -= 1
    return r, n // r


def workload(name: str, n: int | None, world: int = 1):
    from workloads import circuits as wc
    if name == "qft28":
        nn = n or 28
        return wc.qft(nn), f"qft_{nn} (configs[1]: {nn}-qubit QFT on 1xB200, |0...0>, delayed involvement)"
    if name == "qft28x":
        nn = n or 28
        x = qft_x(nn)
        return wc.qft(nn, x=x), f"qft_{nn}|x> x={x} (configs[1]: {nn}-qubit QFT on a basis state, X gates first)"
    if name == "qaoa32":
        nn = n or 32
        return wc.qaoa(nn, 2, seed=1), f"qaoa_{nn} MaxCut p=2, 3-regular seed 1 (configs[2])"
    if name == "rqc":
        nn = n or 30
        return wc.rqc(nn, 20, seed=3), f"rqc_{nn} depth 20 seed 3 (configs[3] shape)"
    if name == "grqc":
        # Table III's deep Google circuit: 4x8 grid, 7238 operations at 32 qubits
        nn = n or 32
        r, cc = grid_shape(nn)
        return wc.grqc(r, cc, 473, seed=5), f"grqc_{nn} {r}x{cc} grid depth 473 seed 5 (Table III deep circuit)"
    if name == "iqp":
        nn = n or 30
        return wc.iqp(nn), f"iqp_{nn} seed 4"
    if name == "bv":
        nn = n or 30
        return wc.bv(nn, (0b1011 * 0x11111111) & ((1 << (nn - 1)) - 1)), f"bv_{nn}"
    # grid workloads (configs[4]: 36 qubits on 8 GPUs = 128 GB per GPU): 2^33 amplitudes per GPU
    if name == "gs":
        r, cc = grid_shape(n or min(36, 33 + int(math.log2(world))))
        return wc.gs(r, cc), f"gs_{r * cc} {r}x{cc} grid (configs[4] shape, 128 GB per GPU at 36 qubits / 8 GPUs)"
    if name == "hlf":
        r, cc = grid_shape(n or min(36, 33 + int(math.log2(world))))
        return wc.hlf(r, cc, seed=2), f"hlf_{r * cc} {r}x{cc} grid seed 2 (configs[4] shape)"
    raise SystemExit(f"unknown workload {name}")


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """SM clocks and throttle reasons sampled DURING the timed region. NVML (pynvml) is polled
    from a thread every ~1 ms, so even a few-millisecond timed region gets samples; without
    NVML, `nvidia-smi -lms 200` (the profiling recipe's clocks line) is the fallback."""
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4))
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.rows = []
        self.nv = None
        self.proc = None
        self.f = None
        self.source = None

    def _nvml_handle(self):
        import pynvml
        import torch
        pynvml.nvmlInit()
        try:
            p = torch.cuda.get_device_properties(self.device)
            bus = f"{p.pci_domain_id:08x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.device)

    def _poll(self):
        nv, h = self.nv
        while not self.stop.is_set():
            try:
                self.rows.append((nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM),
                                  nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM),
                                  nv.nvmlDeviceGetCurrentClocksEventReasons(h)))
            except Exception:
                break
            time.sleep(0.001)

    def __enter__(self):
        import threading
        try:
            self.nv = self._nvml_handle()
            self.stop = threading.Event()
            self.th = threading.Thread(target=self._poll, daemon=True)
            # the timed region can be a few ms: let the poller take the GIL every 0.2 ms instead
            # of the default 5 ms switch interval, and start timing once it is sampling
            self._switch = sys.getswitchinterval()
            sys.setswitchinterval(0.0002)
            self.th.start()
            t0 = time.time()
            while not self.rows and time.time() - t0 < 1.0:
                time.sleep(0.0005)
            self.rows.clear()
            self.source = "nvml poll ~1 ms"
            return self
        except Exception:
            self.nv = None
        try:
            self.f = tempfile.NamedTemporaryFile("w+", delete=False, suffix=".csv")
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"], stdout=self.f,
                stderr=subprocess.DEVNULL)
            self.source = "nvidia-smi -lms 200"
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.nv is not None:
            self.stop.set()
            self.th.join(timeout=5)
            sys.setswitchinterval(self._switch)
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if self.nv is not None:
            rows = [(c, m, r) for c, m, r in self.rows]
        elif self.proc is not None:
            self.f.flush()
            rows = []
            for line in open(self.f.name):
                parts = [x.strip() for x in line.split(",")]
                if len(parts) == 6 and parts[0].isdigit():
                    bits = sum(b for (_, b), v in zip(self.REASONS, parts[2:]) if v == "Active")
                    rows.append((int(parts[0]), int(parts[1]), bits))
            os.unlink(self.f.name)
        else:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no NVML / nvidia-smi"], "samples": 0}
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0, "source": self.source}
        reasons = sorted({name for _, _, r in rows for name, bit in self.REASONS if r & bit})
        return {"sm_mhz": statistics.median(c for c, _, _ in rows), "sm_max_mhz": max(m for _, m, _ in rows),
                "reasons": reasons, "samples": len(rows), "source": self.source}


def dist_setup(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def allreduce_max(x: float, world: int, device) -> float:
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def allreduce_sum(x: float, world: int, device) -> float:
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


# ----------------------------------------------------------------------------- oracle arm

def oracle_sample(text: str, budget_s: float, start_gate: int = 0, max_gates: int | None = None,
                  threads: int | None = None, psi=None):
    """Time the oracle (as it stands: program order, no pruning) on consecutive gates of the
    workload at full size, starting at gate `start_gate`, until `budget_s` elapses; returns
    (sec_per_circuit extrapolated linearly from the per-gate time, sample dict)."""
    from oracle import qasm as oq
    from oracle import statevector as osv
    n, gates = oq.parse(text)
    threads = threads or osv.default_threads()
    if psi is None:
        psi = osv.zero_state(n)
        psi.real[1:] = 0.0  # touch every page before the clock starts (np.zeros maps them lazily)
    t0 = time.perf_counter()
    done = 0
    while done < len(gates) and (time.perf_counter() - t0) < budget_s:
        g = gates[(start_gate + done) % len(gates)]
        osv.apply_gate(psi, n, g.U, g.targets, g.controls, threads)
        done += 1
        if max_gates and done >= max_gates:
            break
    dt = time.perf_counter() - t0
    per_gate = dt / max(done, 1)
    return per_gate * len(gates), {"gates_timed": done, "gates_total": len(gates), "first_gate": start_gate,
                                   "seconds": dt, "threads": threads, "n": n}


def host_info() -> dict:
    """CPU model, logical cores and MemAvailable of this host (SURVEY §8d oracle timing)."""
    info = {"cpu_model": None, "logical_cpus": os.cpu_count(), "mem_available_gib": None}
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                info["cpu_model"] = line.split(":", 1)[1].strip()
                break
        for line in open("/proc/meminfo"):
            if line.startswith("MemAvailable"):
                info["mem_available_gib"] = round(int(line.split()[1]) / 2**20, 1)
    except OSError:
        pass
    return info


def oracle_single_thread() -> dict:
    """the oracle on one thread at C1 (GHZ_5 + QFT_5, whole circuit) and at n = 20
    (QFT_20 on |0...0>, whole circuit), wall clock."""
    from oracle import qasm as oq
    from oracle import statevector as osv
    from workloads import circuits as wc
    out = {}
    for key, c in (("c1_ghz_qft5", wc.ghz_qft(5)), ("qft_20", wc.qft(20))):
        n, gates = oq.parse(c.qasm())
        psi = osv.zero_state(n)
        t0 = time.perf_counter()
        osv.simulate_gates(n, gates, psi=psi, threads=1)
        out[key] = {"seconds": time.perf_counter() - t0, "gates": len(gates), "threads": 1}
    return out


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    circ, desc = workload(args.workload, args.n)
    text = circ.qasm()
    from oracle import statevector as osv
    osv.build()
    psi = osv.zero_state(circ.n)
    psi.real[1:] = 0.0  # first touch of the full state, before any timing
    for _ in range(args.warmup):
        oracle_sample(text, 0.0, max_gates=1, psi=psi)
    vals, samples = [], []
    start = 0
    for k in range(args.steps):
        # each step times the next consecutive gates (wrapping), so the steps together sample
        # the whole circuit rather than its first layer only
        v, smp = oracle_sample(text, args.ref_step_seconds, start_gate=start, max_gates=args.ref_gates, psi=psi)
        start = (start + smp["gates_timed"]) % smp["gates_total"]
        vals.append(v)
        samples.append(smp)
    value = statistics.mean(vals)
    step_s = statistics.mean(x["seconds"] for x in samples)
    cores = samples[0]["threads"]
    timed = sum(x["gates_timed"] for x in samples)
    sample = (f"per step: the next ~{timed // len(samples)} consecutive gates (of {samples[0]['gates_total']}, "
              f"program order, wrapping; {timed} gates over the {len(samples)} steps) on the full "
              f"2^{samples[0]['n']} state, {step_s:.1f} s of CPU work per step; value = per-gate time x "
              f"gates in the circuit (extrapolated); ms_per_step = the measured sample time")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_s * 1e3,
        "value_is_extrapolated": True,
        "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "c128",
        "data": "synthetic (seeded generator, QASM text)",
        "config": run_config(args, circ, desc, world),
        "cpu_baseline": {"value": value, "unit": "s", "cores": cores, "kind": "oracle", "sample": sample,
                         "host": host_info()},
        "e2e": {"value": value, "unit": "s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- GPU arm

def single_qubit_sweep(q, torch, n: int, reps: int = 3):
    """a6 microbenchmark: one generic 1-qubit gate at every target position on a fully involved
    2^n state (SURVEY §8d 'formal >= 70%' number). Bytes = 32 * 2^n per gate."""
    import numpy as np
    stream = torch.cuda.Stream()
    s = q.State(n, stream=stream.cuda_stream, fuse_bits=0)
    H = np.array([[1, 1], [1, -1]], dtype=complex) / math.sqrt(2)
    for t in range(n):
        s.apply_gate(H, [t])
    s.synchronize()
    rng = np.random.default_rng(1)
    U = np.linalg.qr(rng.normal(size=(2, 2)) + 1j * rng.normal(size=(2, 2)))[0]
    res = []
    for t in range(n):
        s.apply_gate(U, [t])
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            s.apply_gate(U, [t])
        e1.record(stream)
        e1.synchronize()
        ms = e0.elapsed_time(e1) / reps
        res.append(32.0 * (1 << n) / (ms * 1e-3) / 1e9)
    s.close()
    return res


def gate_sweep(q, torch, n: int, reps: int = 3):
    """SURVEY §8d microbenchmark, the other gate kinds: for every position t on a fully involved
    2^n state, a generic 2-qubit gate on (t, t+1), CX (control t, target t+1) and CP (t, t+1).
    Algorithmic bytes per gate: 2q generic 32 * 2^n (every quad read and written), CX 16 * 2^n
    (the half with the control set), CP 8 * 2^n (the quarter whose phase is not 1).
    Returns {kind: [GB/s per t]}."""
    import numpy as np
    stream = torch.cuda.Stream()
    s = q.State(n, stream=stream.cuda_stream, fuse_bits=0)
    H = np.array([[1, 1], [1, -1]], dtype=complex) / math.sqrt(2)
    for t in range(n):
        s.apply_gate(H, [t])
    s.synchronize()
    rng = np.random.default_rng(2)
    U4 = np.linalg.qr(rng.normal(size=(4, 4)) + 1j * rng.normal(size=(4, 4)))[0]
    X = np.array([[0, 1], [1, 0]], dtype=complex)
    P = np.diag([1, np.exp(0.7j)])
    kinds = {"u2q": (lambda t: s.apply_gate(U4, [t, (t + 1) % n]), 32.0),
             "cx": (lambda t: s.apply_gate(X, [(t + 1) % n], [t]), 16.0),
             "cp": (lambda t: s.apply_gate(P, [(t + 1) % n], [t]), 8.0)}
    out = {}
    for kind, (fn, bpa) in kinds.items():
        res = []
        for t in range(n):
            fn(t)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(reps):
                fn(t)
            e1.record(stream)
            e1.synchronize()
            ms = e0.elapsed_time(e1) / reps
            res.append(bpa * (1 << n) / (ms * 1e-3) / 1e9)
        out[kind] = res
    s.close()
    return out


def gfc_measure(q, torch, st, seg: int = 4096):
    """NEXT-3: GFC compression of the state left by the workload (the physical
    buffer, as a host-link or swap transfer would send it): ratio and device throughput of
    qgpu_gfc_compress / qgpu_gfc_decompress (CUDA events, best of 3), lossless check."""
    _, n_loc, dev = st.info()
    n = 2 << n_loc
    cap = q.gfc_max_bytes(n, seg)
    if 16 * (1 << n_loc) + cap + 8 * n > 0.8 * torch.cuda.mem_get_info()[0] + 16 * (1 << n_loc):
        return {"skipped": "state too large for a compressed copy + decompressed copy"}
    out = torch.empty(cap, dtype=torch.uint8, device="cuda")
    off = torch.empty((n + seg - 1) // seg + 1, dtype=torch.int64, device="cuda")
    back = torch.empty(n, dtype=torch.int64, device="cuda")
    best_c = best_d = float("inf")
    nb = 0
    for _ in range(3):
        torch.cuda.synchronize()
        e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        e0.record()
        nb = q.gfc_compress(dev, n, seg, out.data_ptr(), cap, off.data_ptr())
        e1.record()
        q.gfc_decompress(out.data_ptr(), off.data_ptr(), n, seg, back.data_ptr())
        e2.record()
        torch.cuda.synchronize()
        best_c, best_d = min(best_c, e0.elapsed_time(e1)), min(best_d, e1.elapsed_time(e2))
    out2 = torch.empty_like(out)
    off2 = torch.empty_like(off)
    nb2 = q.gfc_compress(back.data_ptr(), n, seg, out2.data_ptr(), cap, off2.data_ptr())
    lossless = bool(nb2 == nb and torch.equal(out[:nb], out2[:nb]))
    res = {"seg_len": seg, "doubles": n, "compressed_bytes": nb, "ratio": 8.0 * n / nb,
           "compress_ms": best_c, "decompress_ms": best_d,
           "compress_GBps_in": 8.0 * n / best_c / 1e6, "decompress_GBps_out": 8.0 * n / best_d / 1e6,
           "lossless": lossless}
    del out, off, back, out2, off2
    torch.cuda.empty_cache()
    return res


def host_link_peak(torch, device, nbytes: int = 1 << 30, reps: int = 3):
    """Measured host-link copy bandwidth (GB/s): pinned H2D, D2H, and both at once on two
    streams (what a streaming sweep overlaps)."""
    h_a = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    h_b = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d_a = torch.empty(nbytes, dtype=torch.uint8, device=device)
    d_b = torch.empty(nbytes, dtype=torch.uint8, device=device)
    s1, s2 = torch.cuda.Stream(device=device), torch.cuda.Stream(device=device)

    def timed(fn):
        best = None
        for _ in range(reps):
            torch.cuda.synchronize(device)
            t0 = time.perf_counter()
            fn()
            torch.cuda.synchronize(device)
            dt = time.perf_counter() - t0
            best = dt if best is None else min(best, dt)
        return best

    def h2d():
        with torch.cuda.stream(s1):
            d_a.copy_(h_a, non_blocking=True)

    def d2h():
        with torch.cuda.stream(s2):
            h_b.copy_(d_b, non_blocking=True)

    def both():
        h2d()
        d2h()

    out = {"h2d": nbytes / timed(h2d) / 1e9, "d2h": nbytes / timed(d2h) / 1e9,
           "bidir": 2 * nbytes / timed(both) / 1e9}
    del h_a, h_b, d_a, d_b
    return out


def measure_workload(q, torch, device, stream, args, text, n, steps, warmup, world=1, cfg_extra=None,
                     flush=None, clocks=False):
    """Timed steps of one workload: W untimed warm-up steps, then `steps` steps each bracketed by
    CUDA events on the state's stream (L2 flushed before each, untimed). Returns the state (open),
    the circuit, per-step ms, per-step stats and the clock summary."""
    cfg = dict(device=device.index or 0, stream=stream.cuda_stream, fuse_bits=args.fuse_bits,
               reorder=args.reorder, prune=int(not args.no_prune), timing=1,
               host_slice_bits=args.host_slice_bits, host_compress=args.host_compress)
    cfg.update(cfg_extra or {})
    st = q.State(n, **cfg)
    c = q.Circuit(text)
    for _ in range(warmup):
        st.reset()
        st.apply_circuit(c)
    st.synchronize()
    times, stats = [], []
    barrier(world)
    torch.cuda.synchronize(device)
    clk = ClockSampler(device.index or 0) if clocks else None
    if clk:
        clk.__enter__()
    try:
        for _ in range(steps):
            with torch.cuda.stream(stream):
                flush.zero_()          # L2 flush between timed steps (untimed)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            st.reset()
            st.apply_circuit(c)
            e1.record(stream)
            e1.synchronize()
            times.append(e0.elapsed_time(e1))
            stats.append(st.stats())
        torch.cuda.synchronize(device)
    finally:
        if clk:
            clk.__exit__(None, None, None)
    barrier(world)
    return st, c, times, stats, (clk.summary() if clk else None)


def ncu_traffic(key: str, roof: dict):
    """DRAM bytes per tile launch from the committed ncu launch list of this workload (or None).
    The entry is used only if it was taken on the same pass plan: its launch count and its
    algorithmic bytes per launch (recorded from the profiled run's stats) must match this run's
    (a plan change leaves a stale entry, reported as such instead of a wrong traffic figure)."""
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        t = json.load(open(tp)).get(key)
    except Exception:
        return None, None
    if not t:
        return None, None
    algo = t.get("algo_bytes_per_launch")
    if (algo is None or t.get("launches_per_circuit") != roof["launches_per_step"]
            or abs(algo - roof["algo_bytes_per_launch"]) > 0.01 * roof["algo_bytes_per_launch"]):
        return None, f"stale: {t.get('source')} was taken on another pass plan"
    return t.get("dram_bytes_per_launch"), t.get("source")


def tile_roofline(stats, ms, peak, peak_src):
    """Roofline of the dominant kernel (fused tile pass): algorithmic bytes / CUDA-event time."""
    tile_ms = statistics.mean(x["tile_kernel_ms"] for x in stats)
    tile_bytes = statistics.mean(x["tile_algo_bytes"] for x in stats)
    tile_launches = statistics.mean(x["tile_kernel_launches"] for x in stats)
    achieved = tile_bytes / (tile_ms * 1e-3) / 1e9 if tile_ms > 0 else 0.0
    return {"kernel": "fused tile pass (qgpu_tile_pass, NVRTC-specialised per pass)", "bound": "hbm",
            "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak, "traffic": None,
            "peak_source": peak_src, "algo_bytes_per_launch": tile_bytes / max(tile_launches, 1),
            "launches_per_step": tile_launches, "tile_ms_per_step": tile_ms,
            "share_of_step": tile_ms / ms if ms else None, "frac_of_8TBs_spec": achieved / 8000.0}


def per_pass_binding(prof, hbm_gbs, fp64_fma_per_s):
    """SURVEY §8d / P:401 roofline per pass: bound = max(bytes / HBM peak, FP64 instructions /
    FP64 peak); frac = bound / measured time. Also the step total. Supplementary `sm_bound`: the
    SM side of the same pass with the shared-memory / shuffle (MIO) pipe the kernel design adds
    (4 shuffles per amplitude per lane-bit op, 32 B per amplitude per remap, at one MIO op per
    clock per SM) on top of the FP64 instructions: max(HBM, FP64 + MIO)."""
    rows = []
    tb = tm = tsm = 0.0
    by = {"hbm": [0.0, 0.0], "fp64": [0.0, 0.0]}  # binding -> [bound ms, measured ms]
    clk = fp64_fma_per_s / (148 * 64.0) if fp64_fma_per_s else 1.9e9  # SM clock implied by the FP64 probe
    kinds = {0: "tile", 1: "pair", 2: "quad", 3: "diag", 5: "swap", 7: "zero"}
    for r in prof:
        t_hbm = r["bytes"] / (hbm_gbs * 1e9) * 1e3
        t_fp = r["fp64_ops"] / fp64_fma_per_s * 1e3 if fp64_fma_per_s else 0.0
        bound = max(t_hbm, t_fp)
        mio_clk = r.get("lane_ops", 0) * 4.0 / 32.0 + r.get("remaps", 0) * 32.0 / 128.0
        t_mio = r["amps_computed"] * mio_clk / (148 * clk) * 1e3
        tsm += max(t_hbm, t_fp + t_mio)
        rows.append({"kind": kinds.get(r["kind"], r["kind"]), "k": f"{r['k_in']}->{r['k_out']}",
                     "gates": r["n_gates"], "ms": round(r["ms"], 4), "bytes": r["bytes"],
                     "fp64_per_amp": round(r["fp64_ops"] / r["amps_computed"], 2) if r["amps_computed"] else 0.0,
                     "hbm_ms": round(t_hbm, 4), "fp64_ms": round(t_fp, 4),
                     "binding": "fp64" if t_fp > t_hbm else "hbm", "lane_ops": r.get("lane_ops"),
                     "remaps": r.get("remaps"), "mio_ms": round(t_mio, 4),
                     "frac_of_binding": round(bound / r["ms"], 3) if r["ms"] > 0 else None})
        tb += bound
        tm += r["ms"]
        by[rows[-1]["binding"]][0] += bound
        by[rows[-1]["binding"]][1] += r["ms"]
    return {"passes": rows, "bound_ms": tb, "measured_ms": tm, "frac": tb / tm if tm else None,
            "by_binding": {k: {"bound_ms": v[0], "measured_ms": v[1], "frac": v[0] / v[1] if v[1] else None}
                           for k, v in by.items()},
            "sm_bound": {"bound_ms": tsm, "frac": tsm / tm if tm else None,
                         "model": "per pass max(HBM, FP64 + MIO); MIO = shuffles of lane-bit ops and "
                                  "shared-memory remaps at one op per clock per SM"}}


def run_ours(args):
    import numpy as np
    import torch

    world, rank, local = dist_setup(args)
    device = torch.device("cuda", local)
    torch.cuda.set_device(device)
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build as qbuild
    if rank == 0 or world == 1:
        qbuild.build()
    barrier(world)
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q
    q.load()

    sharded = args.sharded and world > 1
    vr = args.virtual_ranks if not sharded else 0
    circ, desc = workload(args.workload, args.n, world if sharded else (vr or 1))
    text = circ.qasm()
    n = circ.n
    stream = torch.cuda.Stream(device=device)
    cfg_extra = {}
    if sharded:
        # one state sharded over the ranks: top log2(N) qubits on rank bits, global-local swaps
        # over NCCL (a10); the ncclUniqueId goes from rank 0 to all ranks through torch
        import torch.distributed as dist
        obj = [q.nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        cfg_extra = dict(world_size=world, rank=rank, nccl_unique_id=obj[0])
    elif vr > 1:
        # the sharded plan on ONE GPU: 2^g shards in this process, rank-bit conditions, copy
        # activations and batched swaps through the same pack / unpack slab loop, with device
        # copies between the shards' staging as the transport instead of NVLink
        cfg_extra = dict(world_size=vr)
    flush = torch.empty(64 << 20, dtype=torch.float32, device=device)  # 256 MiB > 126 MB L2
    peak, peak_src = peaks()

    st, c, times, stats, clocks = measure_workload(q, torch, device, stream, args, text, n, args.steps,
                                                   args.warmup, world, cfg_extra, flush, clocks=True)
    ngates = c.info()[1]
    ms_local = statistics.mean(times)
    ms = allreduce_max(ms_local, world, device)
    roof = tile_roofline(stats, ms, peak, peak_src)
    kernel_ms = statistics.mean(x["kernel_ms"] for x in stats)
    algo_bytes = statistics.mean(x["algo_bytes"] for x in stats)
    unfused = statistics.mean(x["unfused_bytes"] for x in stats)
    roof["traffic"], roof["traffic_source"] = ncu_traffic(f"{args.workload}_{n}", roof)
    s0 = stats[-1]
    launches = s0["kernels_launched"]

    # e2e through the public API with host buffers: QASM text -> parse -> reset -> apply ->
    # probabilities of 10 qubits back to the host (measurement fused into the last pass).
    # warm: the plan cache hits (the same circuit text planned by an earlier call);
    # cold: QGPU_PLAN_CACHE=0, every call re-runs the Alg.3 reorder and the pass planning
    # (the NVRTC kernel cache stays warm: kernels are compiled once per pass structure)
    e2e_qubits = list(range(min(10, n)))

    def e2e_run(cold: bool, reps: int, warm: int):
        if cold:
            os.environ["QGPU_PLAN_CACHE"] = "0"
        try:
            for _ in range(warm):  # untimed: the measurement pass's NVRTC variant compiles here
                cc = q.Circuit(text)
                st.reset()
                st.apply_circuit_probabilities(cc, e2e_qubits)
                cc.close()
            barrier(world)
            ts, h2d, d2h, p = [], 0, 0, None
            for _ in range(max(1, reps)):
                torch.cuda.synchronize(device)
                t0 = time.perf_counter()
                cc = q.Circuit(text)
                st.reset()
                p = st.apply_circuit_probabilities(cc, e2e_qubits)
                ts.append(time.perf_counter() - t0)
                ss = st.stats()
                h2d, d2h = ss["h2d_bytes"], ss["d2h_bytes"]
                cc.close()
            assert abs(p.sum() - 1) < 1e-9, "e2e readout not normalised"
            return allreduce_max(statistics.mean(ts), world, device), h2d, d2h
        finally:
            os.environ.pop("QGPU_PLAN_CACHE", None)

    e2e_val, h2d, d2h = e2e_run(False, args.steps, args.warmup)
    e2e_cold, h2d_c, d2h_c = e2e_run(True, max(3, args.steps // 4), 1)

    # per-pass binding bound (timing = 2: every pass its own CUDA-event interval)
    fp64 = q.measure_fp64_peak(local)
    st.set_timing(2)
    st.pass_profile()
    for _ in range(2):
        st.reset()
        st.apply_circuit(c)
        prof = st.pass_profile()
    st.set_timing(1)
    binding = per_pass_binding(prof, peak, fp64)
    binding["fp64_peak"] = {"fma_per_s": fp64, "tflops": 2 * fp64 / 1e12,
                            "source": "measured here: qgpu_measure_fp64_peak (DFMA chains on every SM, best of 3)"}
    binding["hbm_peak_gbs"] = peak
    binding["model"] = ("per pass: bound = max(algorithmic bytes / HBM peak, modelled FP64 instructions / "
                        "FP64 peak), frac = sum of bounds / sum of measured pass times (P:401)")
    roof["binding"] = binding

    line = {
        "metric": METRIC, "value": ms / 1e3, "unit": "s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": False,
        "ms_per_step_median": statistics.median(times), "ms_per_step_best": min(times),
        "scaling": "strong" if sharded else "weak",
        "vs_baseline": None, "dtype": "c128", "data": "synthetic (seeded generator, QASM text)",
        "config": run_config(args, circ, desc, world, sharded),
        "roofline": roof,
        "gates_per_s": ngates / (ms / 1e3),
        "gate_apply_GBps": {"algorithmic": algo_bytes / (ms / 1e3) / 1e9,
                            "unfused_equivalent": unfused / (ms / 1e3) / 1e9,
                            "kernel_ms_per_step": kernel_ms},
        "pruning": {"chunks_processed": s0["chunks_processed"], "chunks_skipped": s0["chunks_skipped"],
                    "amps_processed": s0["amps_processed"], "amps_full": s0["amps_full"],
                    "ops_before_full_involvement": s0["ops_before_full_involvement"],
                    "passes": s0["passes"], "relabels": s0["relabels"]},
        "e2e": {"value": e2e_val, "unit": "s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "path": "qgpu_circuit_from_qasm + qgpu_state_reset + qgpu_apply_circuit_probabilities(10 qubits), "
                        "plan-cache hit (the same circuit planned by an earlier call)"},
        "e2e_cold": {"value": e2e_cold, "unit": "s", "h2d_bytes_per_step": h2d_c, "d2h_bytes_per_step": d2h_c,
                     "path": "as e2e with the plan cache off (QGPU_PLAN_CACHE=0): Alg.3 reorder + pass "
                             "planning + program packing inside every call; NVRTC kernels already compiled"},
        "gpu_launches": launches * args.steps,
        "gpu_launches_per_step": launches,
        "clocks": clocks,
    }
    if vr > 1:
        sb = statistics.mean(x["swap_bytes"] for x in stats)
        sms = statistics.mean(x["swap_ms"] for x in stats)
        line["config"]["parallelism"] = f"1 GPU, {vr} virtual ranks (sharded plan, device-copy transport)"
        line["swap"] = {"transport": "device copies between the shards' staging (virtual ranks, one GPU)",
                        "swaps_per_step": s0["swaps"], "swap_bits_per_step": s0["swap_bits"],
                        "bytes_moved_per_step": sb, "swap_ms_per_step": sms}
    if sharded:
        # global-local swap throughput per GPU (bytes this rank sent / CUDA-event time
        # of its swap passes on the state's stream), against NVLink 5's 900 GB/s per direction
        sb = statistics.mean(x["swap_bytes"] for x in stats)
        sms = statistics.mean(x["swap_ms"] for x in stats)
        sms_max = allreduce_max(sms, world, device)
        line["swap"] = {"swaps_per_step": s0["swaps"], "bytes_sent_per_gpu_per_step": sb,
                        "swap_ms_per_step_max_over_ranks": sms_max,
                        "GBps_per_gpu": sb / (sms_max * 1e-3) / 1e9 if sms_max > 0 else None,
                        "peak": 770.0, "peak_source": "measured NVLink peer copy per direction "
                                                      "(B200_PROFILING.md; 900 nominal)",
                        "frac": (sb / (sms_max * 1e-3) / 1e9) / 770.0 if sms_max > 0 else None}
    if args.host_slice_bits:
        # host-memory tier (NEXT-2): the state lives in pinned host memory; the bound is the
        # host link, so report link bytes / sweep time against the measured pinned-copy peak
        link = host_link_peak(torch, device)
        hb = statistics.mean(x["host_h2d_bytes"] + x["host_d2h_bytes"] for x in stats)
        hms = statistics.mean(x["host_ms"] for x in stats)
        ach = hb / (hms * 1e-3) / 1e9 if hms > 0 else 0.0
        hh = statistics.mean(x["host_h2d_bytes"] for x in stats)
        hd = statistics.mean(x["host_d2h_bytes"] for x in stats)
        bound_ms = max(hh / (link["h2d"] * 1e9), hd / (link["d2h"] * 1e9)) * 1e3
        line["config"]["parallelism"] = f"1 GPU, host tier: 2^{args.host_slice_bits} slices in pinned host memory"
        line["config"]["state_location"] = "host (pinned), streamed through device slots"
        line["host_tier"] = {
            "slice_bits": args.host_slice_bits, "slice_bytes": 16 << (n - args.host_slice_bits),
            "compressed": bool(args.host_compress),
            "h2d_bytes_per_step": hh, "d2h_bytes_per_step": hd, "full_state_bytes": 16 << n,
            "sweeps_per_step": s0["host_runs"], "slice_loads": s0["host_slice_loads"],
            "slice_skips": s0["host_slice_skips"], "sweep_ms_per_step": hms,
            "link": {"bound": "host link", "achieved": ach, "peak": link["bidir"], "unit": "GB/s",
                     "frac": bound_ms / hms if hms > 0 else None,
                     "frac_definition": "max(h2d bytes / h2d peak, d2h bytes / d2h peak) / sweep time",
                     "bound_ms_per_step": bound_ms,
                     "peak_source": "measured here: pinned torch copies, 1 GiB each way, concurrent "
                                    "H2D + D2H on two streams",
                     "h2d_peak": link["h2d"], "d2h_peak": link["d2h"]},
        }
    st.close()
    del st
    torch.cuda.empty_cache()

    # configs[1] beside the headline: QFT_28 on |0...0> and on |x>
    if args.extras and not sharded and not args.host_slice_bits:
        extras = {}
        for key in ("qft28", "qft28x"):
            ec, edesc = workload(key, None)
            # short circuits (~1 ms): at least 20 timed steps, so one slow step does not move it
            est, _, et, estats, _ = measure_workload(q, torch, device, stream, args, ec.qasm(), ec.n,
                                                     max(args.steps, 20), args.warmup, world, None, flush)
            ems = allreduce_max(statistics.mean(et), world, device)
            extras[key] = {"workload": edesc, "value": ems / 1e3, "unit": "s", "ms_per_step": ems,
                           "ms_per_step_best": min(et), "gates": len(ec.ops),
                           "roofline": tile_roofline(estats, ems, peak, peak_src),
                           "passes": estats[-1]["passes"],
                           "ops_before_full_involvement": estats[-1]["ops_before_full_involvement"]}
            er = extras[key]["roofline"]
            er["traffic"], er["traffic_source"] = ncu_traffic(f"{key}_{ec.n}", er)
            # per-pass binding bound of this circuit too (its middle passes are FP64-bound)
            est.set_timing(2)
            est.pass_profile()
            eprof = None
            for _ in range(3):
                est.reset()
                est.apply_circuit(q.Circuit(ec.qasm()))
                eprof = est.pass_profile()
            est.set_timing(1)
            eb = per_pass_binding(eprof, peak, fp64)
            er["binding"] = {"passes": eb["passes"], "bound_ms": eb["bound_ms"], "measured_ms": eb["measured_ms"],
                             "frac": eb["frac"], "by_binding": eb["by_binding"]}
            if key == "qft28" and args.gfc:
                extras[key]["gfc_compression"] = gfc_measure(q, torch, est)
            est.close()
            del est
        line["configs_1"] = extras

    if args.micro and rank == 0:
        nm = args.micro_n
        gbs = single_qubit_sweep(q, torch, nm)
        line["single_qubit_gate"] = {"n": nm, "GBps_min": min(gbs), "GBps_median": statistics.median(gbs),
                                     "GBps_per_target": [round(x, 1) for x in gbs],
                                     "frac_min": min(gbs) / peak, "frac_median": statistics.median(gbs) / peak,
                                     "frac_min_of_8TBs": min(gbs) / 8000.0}
        for kind, g in gate_sweep(q, torch, nm).items():
            line["single_qubit_gate"]["other_gates"] = line["single_qubit_gate"].get("other_gates", {})
            line["single_qubit_gate"]["other_gates"][kind] = {
                "GBps_min": min(g), "GBps_median": statistics.median(g), "frac_min": min(g) / peak,
                "GBps_per_target": [round(x, 1) for x in g]}

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, smp = oracle_sample(text, args.cpu_seconds)
        line["cpu_baseline"] = {"value": v, "unit": "s", "cores": smp["threads"], "kind": "oracle",
                                "sample": f"first {smp['gates_timed']} of {smp['gates_total']} gates of "
                                          f"{args.workload} (program order, unpruned, full 2^{n} state, "
                                          f"{smp['seconds']:.1f} s), extrapolated linearly to the circuit",
                                "host": host_info(), "single_thread": oracle_single_thread()}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="qaoa32")
    ap.add_argument("--n", "--qubits", dest="n", type=int, default=None)
    ap.add_argument("--fuse-bits", type=int, default=12)
    ap.add_argument("--reorder", type=int, default=2)
    ap.add_argument("--no-prune", action="store_true")
    ap.add_argument("--micro", type=int, default=1)
    ap.add_argument("--micro-n", type=int, default=32)
    ap.add_argument("--extras", type=int, default=1, help="1: also time configs[1] (QFT_28 |0> and |x>)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=20.0)
    ap.add_argument("--ref-step-seconds", type=float, default=8.0)
    ap.add_argument("--ref-gates", type=int, default=None)
    ap.add_argument("--gfc", type=int, default=1, help="1: also measure GFC compression of the final state")
    ap.add_argument("--host-slice-bits", type=int, default=0,
                    help="h > 0: host-memory tier, state in pinned host memory as 2^h slices (NEXT-2)")
    ap.add_argument("--host-compress", type=int, default=0,
                    help="1: host tier slices cross the link GFC-compressed (NEXT-3 on the NEXT-2 link)")
    ap.add_argument("--virtual-ranks", type=int, default=0,
                    help="G > 1 (N = 1): plan and run the sharded path with G shards on this one GPU")
    ap.add_argument("--sharded", action="store_true",
                    help="N>1: shard one state over the ranks (NCCL swaps) instead of N replicas")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
