"""Measurement at the end of the circuit fused into its last pass (qgpu_apply_circuit_probabilities;
P:81, Eq.1): the last fused pass histograms the amplitudes it stores. Checked against the
oracle's marginals and against the unfused readout (qgpu_apply_circuit + qgpu_probabilities)."""
import numpy as np
import pytest

from oracle import statevector as osv
from workloads import circuits as wc

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True, params=["default", "force_mode2", "global_hist", "round2_rule"])
def hacc_mode(request, monkeypatch):
    """Every test runs with the library's choice (mode 2 with unrequested lane bits is fused when
    the last pass is an NVRTC kernel -- compile-time reduce-scatter epilogue -- else the separate
    readout), with QGPU_HACC=2 (mode 2 forced, the interpreted kernel's run-time butterfly too),
    with QGPU_HGLOB=2 (mode 2 adds straight to the global histogram instead of per-warp shared-
    memory histograms) and with QGPU_HACC=3 (never fused with unrequested lane bits), so the fused
    kernels and the fallback stay covered."""
    for k in ("QGPU_HACC", "QGPU_HGLOB"):
        monkeypatch.delenv(k, raising=False)
    if request.param == "force_mode2":
        monkeypatch.setenv("QGPU_HACC", "2")
    elif request.param == "global_hist":
        monkeypatch.setenv("QGPU_HACC", "2")
        monkeypatch.setenv("QGPU_HGLOB", "2")
    elif request.param == "round2_rule":
        monkeypatch.setenv("QGPU_HACC", "3")
    return request.param


@pytest.fixture(scope="module")
def q():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


CIRCS = {
    "qft0": lambda: wc.qft(16),
    "qftx": lambda: wc.qft(15, x=12345),
    "qaoa": lambda: wc.qaoa(14, 2, seed=3),
    "rqc": lambda: wc.rqc(14, 8, seed=3),
    "hlf": lambda: wc.hlf(3, 5, seed=2),
    "random": lambda: wc.random_circuit(13, 200, seed=61),
    "partial": lambda: wc.random_circuit(10, 60, seed=62),  # qubits above 9 never involved
}


@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [9, 12])
@pytest.mark.parametrize("qsel", ["low", "high", "mixed", "none", "many"])
def test_fused_measurement_vs_oracle(q, name, fuse, qsel):
    c = CIRCS[name]()
    n = c.n if name != "partial" else 14
    text = c.qasm()
    qubits = {"low": [0, 1, 2, 3], "high": list(range(n - 1, n - 6, -1)), "mixed": [5, 0, n - 1, 3, 7],
              "none": [], "many": list(range(12))[::-1]}[qsel]
    with q.State(n, fuse_bits=fuse) as s:
        s.apply_circuit(q.Circuit(wc.random_circuit(n, 30, seed=1).qasm()))  # stale buffer
        s.reset()
        p = s.apply_circuit_probabilities(q.Circuit(text), qubits)
        p2 = s.probabilities(qubits)
        amps = s.amplitudes()
    psi = osv.simulate(text) if n == c.n else np.kron(np.eye(1 << (n - c.n))[:, 0], osv.simulate(text))
    ref = osv.probabilities(psi, n, qubits)
    assert np.abs(p - ref).max() <= 1e-12
    assert np.abs(p - p2).max() <= 1e-12          # same as reading the final state
    assert np.abs(amps - psi).max() <= 1e-10      # the state is left as apply_circuit leaves it


def test_fused_measurement_host_tier_and_unfused_fall_back(q):
    c = wc.qft(14, x=77)
    text = c.qasm()
    ref = osv.probabilities(osv.simulate(text), 14, [0, 5, 13])
    for kw in (dict(host_slice_bits=2), dict(fuse_bits=0), dict(world_size=2)):
        with q.State(14, **kw) as s:
            p = s.apply_circuit_probabilities(q.Circuit(text), [0, 5, 13])
        assert np.abs(p - ref).max() <= 1e-12, kw


def test_fused_measurement_reads_no_state(q):
    """The fused call launches no readout kernel when the requested qubits sit on warp-uniform
    bits of the last pass (here the tile-index bits of QFT_18's last pass): fewer launches."""
    text = wc.qft(18).qasm()
    with q.State(18) as s:
        s.apply_circuit_probabilities(q.Circuit(text), [6, 7, 8])
        k_fused = s.stats()["kernels_launched"]
        s.reset()
        s.apply_circuit(q.Circuit(text))
        s.probabilities([6, 7, 8])
        k_plain = s.stats()["kernels_launched"]
    assert k_fused < k_plain


@pytest.mark.parametrize("name", ["qft0", "qftx", "qaoa", "rqc", "partial"])
@pytest.mark.parametrize("qsel", ["low", "many", "mixed", "high"])
def test_fused_measurement_jit_vs_oracle(q, name, qsel):
    """jit=2: the NVRTC-specialised measurement variant (compile-time slot offsets), including
    the per-slot register sums used when every requested qubit is a tile bit of the last pass."""
    c = CIRCS[name]()
    n = c.n if name != "partial" else 14
    text = c.qasm()
    qubits = {"low": [0, 1, 2, 3], "high": list(range(n - 1, n - 6, -1)), "mixed": [5, 0, n - 1, 3, 7],
              "many": list(range(12))[::-1]}[qsel]
    with q.State(n, fuse_bits=12, jit=2) as s:
        p = s.apply_circuit_probabilities(q.Circuit(text), qubits)
        p2 = s.probabilities(qubits)
    psi = osv.simulate(text) if n == c.n else np.kron(np.eye(1 << (n - c.n))[:, 0], osv.simulate(text))
    ref = osv.probabilities(psi, n, qubits)
    assert np.abs(p - ref).max() <= 1e-12
    assert np.abs(p - p2).max() <= 1e-12


@pytest.mark.parametrize("jit", [0, 2])
def test_fused_measurement_lane_register_bits_read_no_state(q, jit):
    """Qubits 0..9 of QFT_18 sit on lane, register and tile-index bits of the last pass: per-warp
    private histograms (or per-slot register sums) in the pass, so no readout kernel is launched."""
    text = wc.qft(18).qasm()
    qubits = list(range(10))
    with q.State(18, jit=jit) as s:
        p = s.apply_circuit_probabilities(q.Circuit(text), qubits)
        k_fused = s.stats()["kernels_launched"]
        s.reset()
        s.apply_circuit(q.Circuit(text))
        p2 = s.probabilities(qubits)
        k_plain = s.stats()["kernels_launched"]
    assert k_fused < k_plain
    assert np.abs(p - p2).max() <= 1e-12
    assert np.abs(p - 2.0 ** -10).max() <= 1e-12  # QFT|0> is uniform: every marginal is 2^-10


@pytest.mark.parametrize("name", ["qaoa", "rqc", "hlf"])
def test_fused_measurement_unrequested_lane_bits_jit(q, name, hacc_mode):
    """A requested set that leaves lane bits of the last pass unrequested (the qubit on position 0
    plus qubits on high positions): with NVRTC kernels (jit=2) the library fuses it (compile-time
    reduce-scatter epilogue; per-warp or global histogram) and launches no readout kernel (with
    QGPU_HACC=3 it may take the separate readout). Both match the oracle."""
    c = CIRCS[name]()
    text = c.qasm()
    plan = q.Circuit(text).plan_text(c.n)
    fmap = [int(x) for x in plan.strip().splitlines()[-1].split()[1:]]
    at = {p: lq for lq, p in enumerate(fmap) if p >= 0}
    qubits = [at[0]] + [at[p] for p in sorted(at)[-3:]]
    with q.State(c.n, fuse_bits=12, jit=2) as s:
        p = s.apply_circuit_probabilities(q.Circuit(text), qubits)
        k_fused = s.stats()["kernels_launched"]
        s.reset()
        s.apply_circuit(q.Circuit(text))
        p2 = s.probabilities(qubits)
        k_plain = s.stats()["kernels_launched"]
    ref = osv.probabilities(osv.simulate(text), c.n, qubits)
    assert np.abs(p - ref).max() <= 1e-12
    assert np.abs(p - p2).max() <= 1e-12
    if hacc_mode != "round2_rule":
        assert k_fused < k_plain
