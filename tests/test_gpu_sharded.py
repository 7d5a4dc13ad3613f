"""Sharded path on one GPU: "virtual ranks" (world_size > 1 without an NCCL id) keep all 2^g
shards in one process, so the rank-bit conditions of the kernels, rank activation and the
global-local swaps (a10) run on the device and are checked against the oracle. The NCCL
exchange itself is covered by the same protocol on CPU (tests/test_sharded_cpu.py)."""
import numpy as np
import pytest

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
    "random": lambda: wc.random_circuit(11, 250, seed=77),
    "qft": lambda: wc.qft(12, x=2345),
    "rqc": lambda: wc.rqc(12, 8, seed=3),
    "qaoa": lambda: wc.qaoa(12, 2, seed=5),
    "hlf": lambda: wc.hlf(3, 4, seed=2),
    "grqc": lambda: wc.grqc(3, 4, 48, seed=5),  # deep 2-D circuit: many global-local swaps
}


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [0, 9])
def test_virtual_ranks_vs_oracle(q, world, name, fuse):
    c = CIRCS[name]()
    text = c.qasm()
    with q.State(c.n, world_size=world, fuse_bits=fuse) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        st = s.stats()
        p = s.probabilities(list(range(c.n))[::-1][:6])
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert np.abs(p - osv.probabilities(ref, c.n, list(range(c.n))[::-1][:6])).max() <= 1e-12
    if name in ("random", "rqc", "qaoa"):
        assert st["swaps"] > 0


@pytest.mark.parametrize("world", [2, 4])
def test_virtual_ranks_gate_stream_and_prune_neutrality(q, world):
    n = 10
    c = wc.random_circuit(n, 120, seed=5)
    from oracle import qasm as oq
    _, gates = oq.parse(c.qasm())
    ref = osv.zero_state(n)
    with q.State(n, world_size=world) as s:
        for g in gates:
            s.apply_gate(g.U, list(g.targets), list(g.controls))
            osv.apply_gate(ref, n, g.U, g.targets, g.controls)
        got = s.amplitudes()
    assert np.abs(got - ref).max() <= TOL
    text = wc.random_circuit(12, 200, seed=6).qasm()
    outs = []
    for prune in (1, 0):
        with q.State(12, world_size=world, prune=prune, fuse_bits=9) as s:
            s.apply_circuit(q.Circuit(text))
            outs.append(s.amplitudes())
    assert np.array_equal(outs[0], outs[1])
