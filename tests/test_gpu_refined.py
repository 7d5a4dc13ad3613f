"""Refined involvement rule (involve_rule=1; exact by P:221): gates with a
control on a never-involved qubit are skipped, diagonal gates on never-involved targets are
restricted to that bit = 0 (global phases become a scalar), neither involves anything. Checked
on the GPU: amplitudes vs the oracle (which applies every gate by definition), the executed
schedule and involvement trace bit-exact vs the oracle's refined Alg.2/3 replay, the pruning
bitmap after every gate of a stream, and the resident / virtual-rank / host-tier paths."""
import numpy as np
import pytest

from oracle import qasm as oq
from oracle import schedule as osch
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


CIRCS = {
    "qft0": lambda: wc.qft(14),
    "qftx": lambda: wc.qft(13, x=4321),
    "ghz_qft5": lambda: wc.ghz_qft(5),
    "random": lambda: wc.random_circuit(12, 250, seed=31),
    "randdiag": lambda: wc.random_circuit(12, 250, seed=32, names=DIAG_HEAVY),
    "qaoa": lambda: wc.qaoa(12, 2, seed=5),
    "hlf": lambda: wc.hlf(3, 4, seed=2),
}


@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [0, 9, 12])
@pytest.mark.parametrize("mode", [0, 2])
def test_refined_rule_vs_oracle(q, name, fuse, mode):
    c = CIRCS[name]()
    text = c.qasm()
    n, gates = oq.parse(text)
    with q.State(n, involve_rule=1, fuse_bits=fuse, reorder=mode) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        order, invs = s.schedule()
        st = s.stats()
        inv_now = s.involvement()
        bm = s.chunk_bitmap(3)
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    ref_order = osch.reorder(gates, mode, rule=1)
    assert list(order) == ref_order
    ref_trace = osch.involvement_trace(gates, ref_order, rule=1)
    assert [int(x) for x in invs] == ref_trace
    assert inv_now == ref_trace[-1]
    assert list(bm) == osch.chunk_bitmap(ref_trace[-1], n, 3)
    assert st["ops_before_full_involvement"] == (osch.ops_before_full_involvement(gates, n, ref_order, rule=1)
                                                if ref_trace[-1] == (1 << n) - 1 else -1)


@pytest.mark.parametrize("zskip", ["1", "0"])
def test_refined_rule_shrinks_qft_on_zero(q, zskip, monkeypatch):
    """QFT|0...0> under rule 1: the CP ladders meet uninvolved qubits and are skipped, so the
    state is H^n (plus relabels). Without zero-position skipping it moves fewer bytes than the
    paper's rule; with it (the default) the paper's rule already skips the same zero halves at the
    data level, so the bytes are at most equal while the involvement traces still differ."""
    monkeypatch.setenv("QGPU_ZSKIP", zskip)
    # both rules under the consecutive-run planner (the pass-aware order applies to rule 0 only)
    monkeypatch.setenv("QGPU_PASS_SCHED", "0")
    c = wc.qft(20)
    text = c.qasm()
    out = {}
    for rule in (0, 1):
        with q.State(20, involve_rule=rule) as s:
            s.apply_circuit(q.Circuit(text))
            out[rule] = (s.amplitudes(), s.stats(), s.schedule()[1])
    assert np.abs(out[0][0] - out[1][0]).max() <= TOL
    if zskip == "0":
        assert out[1][1]["algo_bytes"] < out[0][1]["algo_bytes"]
    else:
        assert out[1][1]["algo_bytes"] <= out[0][1]["algo_bytes"]
    assert list(out[0][2]) != list(out[1][2])
    assert np.abs(out[1][0] - 2.0 ** -10).max() <= TOL  # QFT|0> = uniform superposition


@pytest.mark.parametrize("seed", range(3))
def test_refined_rule_gate_stream_bitmap(q, seed):
    """Gate-by-gate: involvement and the chunk bitmap after every gate equal the oracle's
    refined trace; amplitudes vs the oracle; global phases of diagonal gates applied while
    nothing is involved (scalar on psi[0]) are kept."""
    n = 11
    c = wc.Circuit(n)
    c.add("rz", [3], [0.9])            # global phase e^{-0.45i} on |0...0>
    c.add("crz", [1, 2], [0.4])        # control uninvolved: skipped
    c.add("u1", [0], [1.1])            # diag(1, e^{1.1i}) on |0>: identity
    for op in wc.random_circuit(n, 70, seed=200 + seed, names=DIAG_HEAVY).ops:
        c.ops.append(op)
    text = c.qasm()
    _, gates = oq.parse(text)
    ref = osv.zero_state(n)
    inv = 0
    with q.State(n, involve_rule=1) as s:
        for k, g in enumerate(gates):
            s.apply_gate(g.U, list(g.targets), list(g.controls))
            osv.apply_gate(ref, n, g.U, g.targets, g.controls)
            inv = osch.update_involvement(inv, osch.involved_by(g, inv, 1))
            assert s.involvement() == inv
            assert list(s.chunk_bitmap(4)) == osch.chunk_bitmap(inv, n, 4)
            if k < 3 or k % 10 == 9:
                assert np.abs(s.amplitudes() - ref).max() <= TOL
        order, invs = s.schedule()
    assert [int(x) for x in invs] == osch.involvement_trace(gates, rule=1)


@pytest.mark.parametrize("kw", [dict(world_size=4), dict(host_slice_bits=2)])
@pytest.mark.parametrize("name", ["qft0", "randdiag", "qaoa"])
def test_refined_rule_sharded_and_host_tier(q, kw, name):
    c = CIRCS[name]()
    text = c.qasm()
    with q.State(c.n, involve_rule=1, fuse_bits=9, **kw) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
    assert np.abs(got - osv.simulate(text)).max() <= TOL


def test_refined_rule_prune_neutrality(q):
    text = wc.random_circuit(13, 200, seed=41, names=DIAG_HEAVY).qasm()
    outs = [None, None]
    for prune in (1, 0):
        with q.State(13, involve_rule=1, prune=prune, fuse_bits=9) as s:
            s.apply_circuit(q.Circuit(text))
            outs[prune] = s.amplitudes()
    assert np.array_equal(outs[0], outs[1])
