"""Zero-position skipping ("zero halves"): a qubit first touched by a diagonal gate or
as a control leaves its new half of the state exactly zero; the fused passes neither
store nor load that half until a non-diagonal op targets the position, and a PK_ZERO pass writes
the zeros if the plan ends before that. The device memory of the skipped half holds stale data,
so every test here first fills the buffer with a dense state, resets, and then checks the skipped
circuit against the oracle -- a half that was read or left unwritten would show up."""
import numpy as np
import pytest

from oracle import statevector as osv
from workloads import circuits as wc

pytestmark = pytest.mark.gpu

TOL = 1e-10
DIAG_HEAVY = ["cp", "cz", "rz", "cx", "crx", "ccx", "t", "h", "rzz", "cswap", "x", "u1", "crz", "s"]


@pytest.fixture(scope="module")
def q():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


def _ends_diag_only(n):
    """H on qubit 0, then CP / CZ / controlled gates that place the other qubits without ever
    targeting them non-diagonally: every half stays zero to the end (PK_ZERO materialises)."""
    c = wc.Circuit(n)
    c.add("h", [0])
    for k in range(1, n):
        c.add("cp", [k - 1, k], [0.3 * k])
        c.add("crx", [k, 0], [0.2])  # control on a zero qubit
    c.add("h", [1])
    return c


CIRCS = {
    "qft0_16": lambda: wc.qft(16),
    "qft0_21": lambda: wc.qft(21),
    "diag_only": lambda: _ends_diag_only(14),
    "randdiag": lambda: wc.random_circuit(14, 300, seed=51, names=DIAG_HEAVY),
    "ghz_qft5": lambda: wc.ghz_qft(5),
}


@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [9, 12])
def test_zero_skip_vs_oracle_after_dense_state(q, name, fuse):
    c = CIRCS[name]()
    text = c.qasm()
    dense = wc.random_circuit(c.n, 80, seed=7).qasm()
    with q.State(c.n, fuse_bits=fuse) as s:
        s.apply_circuit(q.Circuit(dense))   # fill the buffer with non-zero amplitudes
        s.reset()
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        p = s.probabilities(list(range(min(6, c.n))))
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert np.abs(p - osv.probabilities(ref, c.n, list(range(min(6, c.n))))).max() <= 1e-12


@pytest.mark.parametrize("name", sorted(CIRCS))
def test_zero_skip_bit_identical_and_fewer_bytes(q, name, monkeypatch):
    text = CIRCS[name]().qasm()
    n = CIRCS[name]().n
    out = {}
    for z in ("1", "0"):
        monkeypatch.setenv("QGPU_ZSKIP", z)
        with q.State(n) as s:
            s.apply_circuit(q.Circuit(text))
            out[z] = (s.amplitudes(), s.stats())
    assert np.array_equal(out["1"][0], out["0"][0])
    assert out["1"][1]["algo_bytes"] <= out["0"][1]["algo_bytes"]
    if name.startswith("qft0"):  # (diag_only: the final PK_ZERO writes the same zeros back)
        assert out["1"][1]["algo_bytes"] < out["0"][1]["algo_bytes"]
