"""Host-memory tier (the paper's setting): the state lives
in pinned host memory as 2^h slices and every run of passes between global-local swaps streams
the active slices through device slots. Checked against the oracle on the same seeded circuits,
bit-identical to the HBM-resident virtual-rank path (same plan, same kernels), with pruning
visible as skipped slices and live-prefix-only transfers."""
import numpy as np
import pytest

from oracle import qasm as oq
from oracle import statevector as osv
from workloads import circuits as wc

pytestmark = pytest.mark.gpu

TOL = 1e-10


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
    "random": lambda: wc.random_circuit(11, 250, seed=78),
    "qft": lambda: wc.qft(12, x=1234),
    "qft0": lambda: wc.qft(12),
    "rqc": lambda: wc.rqc(12, 8, seed=3),
    "qaoa": lambda: wc.qaoa(12, 2, seed=5),
    "gs": lambda: wc.gs(3, 4),
    "hlf": lambda: wc.hlf(3, 4, seed=2),
    "grqc": lambda: wc.grqc(3, 4, 48, seed=5),
}


@pytest.mark.parametrize("comp", [0, 1])
@pytest.mark.parametrize("h", [1, 2, 3])
@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [0, 9])
def test_host_tier_vs_oracle(q, h, name, fuse, comp):
    c = CIRCS[name]()
    text = c.qasm()
    qs = list(range(c.n))[::-1][:6]
    with q.State(c.n, host_slice_bits=h, fuse_bits=fuse, timing=1, host_compress=comp) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        st = s.stats()
        p = s.probabilities(qs)
        norm = s.probabilities([])[0]
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert np.abs(p - osv.probabilities(ref, c.n, qs)).max() <= 1e-12
    assert abs(norm - 1.0) <= 1e-12
    assert st["host_runs"] >= 1 and st["host_slice_loads"] >= 1
    # the live prefix only crosses the link: never more than a full state per sweep each way
    assert st["host_d2h_bytes"] <= st["host_runs"] * 16 * (1 << c.n)


@pytest.mark.parametrize("name", ["random", "qaoa", "grqc"])
def test_host_tier_bit_identical_to_resident_virtual_ranks(q, name, monkeypatch):
    """Same plan and kernels as 2^h HBM-resident virtual ranks: the streamed result is the same
    bits (the host tier only changes where the slices live between runs). The host tier keeps
    local-first placement, so the virtual ranks are planned without the cross-rank expand."""
    monkeypatch.setenv("QGPU_GLOBAL_FIRST", "0")
    c = CIRCS[name]()
    text = c.qasm()
    with q.State(c.n, host_slice_bits=2, fuse_bits=9) as s:
        s.apply_circuit(q.Circuit(text))
        a = s.amplitudes()
    with q.State(c.n, world_size=4, fuse_bits=9) as s:
        s.apply_circuit(q.Circuit(text))
        b = s.amplitudes()
    assert np.array_equal(a, b)


def test_host_tier_pruning_skips_zero_slices(q):
    """Alg.1 pruning on the host link: while the involved qubits fit one slice, the other slices
    are never loaded and only the live prefix is copied."""
    n, h = 14, 3
    c = wc.Circuit(n)
    c.add("h", [0])
    for k in range(1, 6):
        c.add("cx", [k - 1, k])
    text = c.qasm()
    with q.State(n, host_slice_bits=h) as s:
        s.apply_circuit(q.Circuit(text))
        st = s.stats()
        got = s.amplitudes()
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert st["host_slice_loads"] == st["host_runs"]  # slice 0 only
    assert st["host_slice_skips"] == st["host_runs"] * ((1 << h) - 1)
    assert st["host_d2h_bytes"] == 16 * (1 << 6) * st["host_runs"]  # 2^6 live amplitudes


@pytest.mark.parametrize("h", [0, 2])
@pytest.mark.parametrize("prune", [1, 0])
def test_host_tier_gate_stream_reset_and_set_amplitudes(q, prune, h):
    """Also the HBM-resident path (h = 0): after reset() the buffer holds the previous run's
    amplitudes, so a controlled gate that expands its target must write the control-0 part of
    the new half as zeros (regression: it used to rely on a fresh cudaMalloc being zero)."""
    n = 11
    c = wc.random_circuit(n, 90, seed=9)
    _, gates = oq.parse(c.qasm())
    ref = osv.zero_state(n)
    with q.State(n, host_slice_bits=h, prune=prune) as s:
        for rep in range(2):  # the second round starts from reset(): the host slices are reused
            s.reset()
            ref = osv.zero_state(n)
            for g in gates:
                s.apply_gate(g.U, list(g.targets), list(g.controls))
                osv.apply_gate(ref, n, g.U, g.targets, g.controls)
            assert np.abs(s.amplitudes() - ref).max() <= TOL
        # set_amplitudes writes the host slices directly; then a circuit runs on top
        rng = np.random.default_rng(4)
        psi = rng.normal(size=1 << n) + 1j * rng.normal(size=1 << n)
        psi /= np.linalg.norm(psi)
        s.set_amplitudes(psi)
        text = wc.random_circuit(n, 60, seed=10).qasm()
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
    _, g2 = oq.parse(text)
    ref2 = psi.copy()
    for g in g2:
        osv.apply_gate(ref2, n, g.U, g.targets, g.controls)
    assert np.abs(got - ref2).max() <= TOL


def test_host_tier_prune_neutrality(q):
    text = wc.random_circuit(12, 200, seed=11).qasm()
    outs = []
    for prune in (1, 0):
        with q.State(12, host_slice_bits=2, prune=prune, fuse_bits=9) as s:
            s.apply_circuit(q.Circuit(text))
            outs.append(s.amplitudes())
    assert np.array_equal(outs[0], outs[1])


def test_host_tier_argument_errors(q):
    with pytest.raises(q.QgpuError) as e:
        q.State(8, host_slice_bits=4)  # n - h < 5
    assert e.value.kind == "INVALID_ARG"
    with pytest.raises(q.QgpuError) as e:
        q.State(12, host_slice_bits=2, world_size=2)
    assert e.value.kind == "UNSUPPORTED"


@pytest.mark.parametrize("name", ["qft0", "gs", "qaoa", "grqc", "random"])
def test_host_compress_bit_identical_and_smaller_link(q, name):
    """GFC on the host link (P:344-362 on the NEXT-2 link) is lossless: the compressed host tier
    gives the same bits as the raw one; structured states (QFT of |0>, graph states) cross the
    link in fewer bytes."""
    c = CIRCS[name]()
    text = c.qasm()
    out = {}
    for comp in (0, 1):
        with q.State(c.n, host_slice_bits=2, fuse_bits=9, host_compress=comp) as s:
            s.apply_circuit(q.Circuit(text))
            s.apply_circuit(q.Circuit(text))  # loads compressed slices written by the first apply
            out[comp] = (s.amplitudes(), s.stats(), s.probabilities([0, 1, 2]))
    assert np.array_equal(out[0][0], out[1][0])
    assert np.abs(out[0][2] - out[1][2]).max() <= 1e-15  # (reduction order of the readout)
    if name in ("qft0", "gs"):
        assert out[1][1]["host_d2h_bytes"] < 0.6 * out[0][1]["host_d2h_bytes"]


def test_host_compress_gate_stream_and_set_amplitudes(q):
    n = 11
    c = wc.random_circuit(n, 60, seed=19)
    _, gates = oq.parse(c.qasm())
    ref = osv.zero_state(n)
    with q.State(n, host_slice_bits=2, host_compress=1) as s:
        for g in gates:
            s.apply_gate(g.U, list(g.targets), list(g.controls))
            osv.apply_gate(ref, n, g.U, g.targets, g.controls)
        assert np.abs(s.amplitudes() - ref).max() <= TOL
        rng = np.random.default_rng(5)
        psi = rng.normal(size=1 << n) + 1j * rng.normal(size=1 << n)
        psi /= np.linalg.norm(psi)
        s.set_amplitudes(psi)  # raw slices again
        assert np.array_equal(s.amplitudes(), psi)
        text = wc.random_circuit(n, 40, seed=20).qasm()
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
    _, g2 = oq.parse(text)
    for g in g2:
        osv.apply_gate(psi, n, g.U, g.targets, g.controls)
    assert np.abs(got - psi).max() <= TOL

