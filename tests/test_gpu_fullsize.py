"""Parity at BASELINE.json's full sizes, in the configuration bench.py times (reorder=2,
prune=1, fused b=12, NVRTC-specialised kernels): closed forms checked on the whole state or on
sampled ranges, full oracle comparison where the oracle finishes in seconds (28 qubits), and
properties that hold at any size (norm, mirror U U^dagger = I)."""
import math

import numpy as np
import pytest

from oracle import statevector as osv
from workloads import circuits as wc

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

TOL = 1e-10


@pytest.fixture(autouse=True)
def library_default_jit_threshold():
    """Run these tests in exactly the configuration bench.py times: the library's default JIT
    threshold (every fused pass of >= 2^12 amplitudes NVRTC-specialised), not the suite-wide
    2^20 of conftest.py (the library reads QGPU_JIT_MIN_BITS per call)."""
    import os
    old = os.environ.get("QGPU_JIT_MIN_BITS")
    os.environ.pop("QGPU_JIT_MIN_BITS", None)
    yield
    if old is not None:
        os.environ["QGPU_JIT_MIN_BITS"] = old


@pytest.fixture(scope="module")
def q():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


def test_c2_qft28_basis_state_full_state(q):
    """configs[1]: QFT_28 on |x> (x from rng seed 2); every amplitude vs e^{2 pi i x y / 2^n} / 2^{n/2}."""
    c = wc.config_circuit("C2x")
    n, x = c.n, c.meta["x"]
    with q.State(n) as s:
        s.apply_circuit(q.Circuit(c.qasm()))
        worst = 0.0
        step = 1 << 24
        for start in range(0, 1 << n, step):
            got = s.amplitudes(start, step)
            y = np.arange(start, start + step, dtype=np.int64)
            ph = ((x * y) % (1 << n)).astype(np.float64) / (1 << n)
            exp = np.exp(2j * np.pi * ph) / math.sqrt(1 << n)
            worst = max(worst, float(np.abs(got - exp).max()))
        p = s.probabilities([])
    assert worst <= TOL
    assert abs(p[0] - 1) <= 1e-12


def test_c2_qft28_zero_state_full_state_and_stats(q):
    """configs[1], the bench's QFT_28 on |0...0>: all 2^28 amplitudes vs the closed form
    QFT|0> = 2^-14 everywhere (P3), read in 2^24-amplitude pieces; the fused passes of
    >= 2^12 amplitudes ran NVRTC-specialised kernels (as in bench.py)."""
    c = wc.qft(28)
    with q.State(28, chunk_bits=21) as s:
        s.apply_circuit(q.Circuit(c.qasm()))
        u = 1 / math.sqrt(1 << 28)
        worst = 0.0
        for start in range(0, 1 << 28, 1 << 24):
            worst = max(worst, float(np.abs(s.amplitudes(start, 1 << 24) - u).max()))
        st = s.stats()
    assert worst <= TOL
    assert st["chunks_skipped"] > 0 and st["ops_before_full_involvement"] > 300
    plan = q.Circuit(c.qasm()).plan(28)
    want = int(sum(1 for r in plan if r[2] == 0 and r[4] >= 12))
    assert want >= 3 and st["jit_launches"] == want


def test_c3_qaoa32_vs_oracle_full_state(q):
    """configs[2] at full size: QAOA MaxCut p=2, 32 qubits, the bench's exact
    configuration (reorder=2, prune=1, b=12, default JIT threshold) against the oracle's plain
    program-order simulation of the same QASM (64 GiB on the host, all cores), every one of the
    2^32 amplitudes compared in 2^24-amplitude pieces."""
    import os
    c = wc.config_circuit("C3")
    text = c.qasm()
    avail = 0
    for line in open("/proc/meminfo"):
        if line.startswith("MemAvailable"):
            avail = int(line.split()[1]) * 1024
    if avail < (16 << c.n) + (8 << 30):
        pytest.skip(f"needs {16 << c.n} B of host memory for the oracle state, {avail} available")
    ref = osv.simulate(text, threads=os.cpu_count())
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(text))
        worst = 0.0
        for start in range(0, 1 << c.n, 1 << 24):
            got = s.amplitudes(start, 1 << 24)
            worst = max(worst, float(np.abs(got - ref[start:start + (1 << 24)]).max()))
        p = s.probabilities([])
    del ref
    assert worst <= TOL
    assert abs(p[0] - 1) <= 1e-12


@pytest.mark.parametrize("n", [31, 32])
def test_unfused_kernels_full_size_high_indices(q, n):
    """a6/a7/a8 unfused kernels (fuse_bits=0, as the bench's microbenchmark) at n = 31, 32, i.e.
    amplitude indices above 2^31: a random product state built gate by gate from |0> (first-touch
    expansion of every qubit), then generic 1-qubit gates at low / middle / top positions with and
    without controls on the top qubits, 2-qubit gates spanning bit 0 and the top bits, CX with
    control 0, CP on (top, 0) and a 2-qubit diagonal; sampled amplitudes (contiguous ranges at the
    bottom, middle and top of the index space) vs the oracle's light-cone evaluation."""
    from oracle import qasm as oq
    from lightcone import product_light_cone
    rng = np.random.default_rng(100 + n)
    top = n - 1
    factors = []
    prep = []
    for t in range(n):
        U = oq.u3(*rng.uniform(-3, 3, 3))
        prep.append(U)
        factors.append(U[:, 0].copy())            # U|0>
    U4 = np.linalg.qr(rng.normal(size=(4, 4)) + 1j * rng.normal(size=(4, 4)))[0]
    X = np.array([[0, 1], [1, 0]], dtype=complex)
    gates = [(oq.u3(*rng.uniform(-3, 3, 3)), [0], []),
             (oq.u3(*rng.uniform(-3, 3, 3)), [top], []),
             (oq.u3(*rng.uniform(-3, 3, 3)), [17], [top]),
             (oq.u3(*rng.uniform(-3, 3, 3)), [2], [top - 1, top]),
             (U4, [top, 3], []),
             (U4.conj().T @ np.diag(np.exp(1j * rng.uniform(-3, 3, 4))), [0, top - 1], []),
             (X, [top], [0]),
             (oq.phase(0.7), [0], [top]),
             (np.diag(np.exp(1j * rng.uniform(-3, 3, 4))), [top, 1], [])]
    with q.State(n, fuse_bits=0) as s:
        for t in range(n):
            s.apply_gate(prep[t], [t])
        for U, t, cs in gates:
            s.apply_gate(U, t, cs)
        worst = 0.0
        starts = [0, (1 << (n - 1)) - 2048, 1 << (n - 1), 3 << (n - 2), (1 << n) - 4096,
                  int(rng.integers(1 << (n - 1), (1 << n) - 4096))]
        for st_ in starts:
            got = s.amplitudes(st_, 4096)
            idx = np.arange(st_, st_ + 4096, dtype=np.int64)
            exp = product_light_cone(n, factors, gates, idx)
            worst = max(worst, float(np.abs(got - exp).max()))
        p = s.probabilities([])
    assert worst <= TOL
    assert abs(p[0] - 1) <= 1e-12


def test_qaoa28_vs_oracle_full(q):
    c = wc.qaoa(28, 2, seed=1)
    text = c.qasm()
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL


def test_c3_qaoa32_norm_mirror_and_marginals(q):
    """configs[2]: QAOA MaxCut p=2 at 32 qubits (64 GiB): norm, marginal symmetry of MaxCut
    (global bit flip: p(y) = p(~y) on any qubit subset), and the mirror returns |0>."""
    c = wc.config_circuit("C3")
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(c.qasm()))
        p = s.probabilities(list(range(8)))
        assert abs(p.sum() - 1) <= 1e-12
        assert np.abs(p - p[::-1]).max() <= 1e-12
        s.reset()
        s.apply_circuit(q.Circuit(wc.mirror(c).qasm()))
        a = s.amplitudes(0, 4096)
    assert abs(a[0] - 1) <= TOL and np.abs(a[1:]).max() <= TOL


def test_rqc30_mirror(q):
    c = wc.rqc(30, 20, seed=3)
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(wc.mirror(c).qasm()))
        a = s.amplitudes(0, 4096)
        p = s.probabilities([])
    assert abs(a[0] - 1) <= TOL and np.abs(a[1:]).max() <= TOL
    assert abs(p[0] - 1) <= 1e-12


def test_grqc30_deep_mirror(q):
    """The paper's deep-circuit case (Table III): a 5x6 grid Google-style circuit of
    ~2200 operations and its mirror (~4400 operations) returns |0...0> at 30 qubits."""
    c = wc.grqc(5, 6, 120, seed=5)
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(wc.mirror(c).qasm()))
        a = s.amplitudes(0, 4096)
        p = s.probabilities([])
    assert abs(a[0] - 1) <= TOL and np.abs(a[1:]).max() <= TOL
    assert abs(p[0] - 1) <= 1e-12


def test_graph_state_30_sampled_ranges(q):
    c = wc.gs(5, 6)
    n, edges = c.n, c.meta["edges"]
    with q.State(n) as s:
        s.apply_circuit(q.Circuit(c.qasm()))
        for start in (0, 123456789, (1 << n) - (1 << 16)):
            got = s.amplitudes(start, 1 << 16)
            xs = np.arange(start, start + (1 << 16), dtype=np.int64)
            par = np.zeros_like(xs)
            for u, v in edges:
                par ^= ((xs >> u) & 1) & ((xs >> v) & 1)
            assert np.abs(got - (1 - 2 * par) / math.sqrt(1 << n)).max() <= TOL


@pytest.mark.parametrize("comp", [0, 1])
def test_host_tier_qft30_basis_state_sampled(q, comp):
    """NEXT-2 (+ NEXT-3 on the link) at 30 qubits (16 GiB in pinned host memory, 2^2 slices):
    QFT|x> sampled ranges in every slice vs e^{2 pi i x y / 2^n} / 2^{n/2}, and the norm."""
    n = 30
    x = 0x2A5F3C1B & ((1 << n) - 1)
    c = wc.qft(n, x=x)
    with q.State(n, host_slice_bits=2, host_compress=comp) as s:
        s.apply_circuit(q.Circuit(c.qasm()))
        worst = 0.0
        for start in [0, (1 << 28) - 4096, 1 << 28, 3 << 28, (1 << n) - (1 << 16)]:
            got = s.amplitudes(start, 1 << 16)
            y = np.arange(start, start + (1 << 16), dtype=np.int64)
            ph = ((x * y) % (1 << n)).astype(np.float64) / (1 << n)
            worst = max(worst, float(np.abs(got - np.exp(2j * np.pi * ph) / math.sqrt(1 << n)).max()))
        p = s.probabilities([])
        st = s.stats()
    assert worst <= TOL
    assert abs(p[0] - 1) <= 1e-12
    assert st["host_runs"] >= 1


def test_bench_e2e_fused_measurement_full_size(q):
    """The bench's e2e call at full size: QFT_28 on |0> and on |x>, qubits 0..9 measured inside
    the last pass (mode 2 epilogue). QFT of a basis state has |amplitude|^2 = 2^-n everywhere, so
    every marginal over 10 qubits is 2^-10 (closed form); QAOA_28 marginals vs the oracle's."""
    qs = list(range(10))
    for name in ("C2", "C2x"):
        c = wc.config_circuit(name)
        with q.State(c.n) as s:
            p = s.apply_circuit_probabilities(q.Circuit(c.qasm()), qs)
            p2 = s.probabilities(qs)
            mixed = s.probabilities([27, 0, 13, 5])
        assert np.abs(p - 2.0 ** -10).max() <= 1e-12, name
        assert np.abs(p - p2).max() <= 1e-12, name
        assert np.abs(mixed - 2.0 ** -4).max() <= 1e-12, name
    c = wc.qaoa(28, 2, seed=1)
    text = c.qasm()
    for sel in (qs, [27, 26, 0, 1, 14], [3, 17, 9]):
        with q.State(c.n) as s:
            p = s.apply_circuit_probabilities(q.Circuit(text), sel)
        if sel is qs:
            ref_psi = osv.simulate(text)
        ref = osv.probabilities(ref_psi, c.n, sel)
        assert np.abs(p - ref).max() <= 1e-12, sel
