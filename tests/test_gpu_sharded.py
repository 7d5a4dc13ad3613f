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


EARLY = {
    "rqc": lambda: wc.rqc(16, 8, seed=3),
    "qaoa": lambda: wc.qaoa(16, 2, seed=5),
    "gs": lambda: wc.gs(3, 5),
    "random": lambda: wc.random_circuit(15, 300, seed=78),
    "grqc": lambda: wc.grqc(3, 5, 40, seed=5),
}


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("name", sorted(EARLY))
@pytest.mark.parametrize("fuse", [0, 9])
def test_virtual_ranks_batched_swaps_cross_rank_expand(q, world, name, fuse, monkeypatch):
    """a10 as built for NCCL, on one GPU: copy activations (cross-rank first-touch expand of the
    first log2 G qubits, here once 3 local positions are assigned), batched s-bit swaps with
    farthest-next-use victims, the pack / unpack kernels and the slab loop (small slabs: many
    slabs per swap) with device copies between the shards' staging as the transport."""
    monkeypatch.setenv("QGPU_GLOBAL_MIN_LOCAL", "3")
    c = EARLY[name]()
    text = c.qasm()
    with q.State(c.n, world_size=world, fuse_bits=fuse, swap_slab_bytes=4096) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        st = s.stats()
        p = s.probabilities([c.n - 1, 0, 5])
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert np.abs(p - osv.probabilities(ref, c.n, [c.n - 1, 0, 5])).max() <= 1e-12
    plan = q.Circuit(text).plan_text(c.n, world, 2, fuse)
    if name != "random":  # H-first families: the first log2 G qubits go to rank bits by copy
        assert any(l.startswith("P 6 ") and int(l.split()[5]) < 0 for l in plan.splitlines())
    if name in ("rqc", "random", "grqc"):
        assert st["swaps"] > 0 and st["swap_bits"] >= st["swaps"]


@pytest.mark.parametrize("world", [4, 8])
def test_virtual_ranks_prune_neutrality_with_global_first(q, world, monkeypatch):
    """P:221 with the sharded plan: prune=1 and prune=0 give bit-identical amplitudes (the copy
    activation and the live-prefix-only swaps move exactly the non-zero part)."""
    monkeypatch.setenv("QGPU_GLOBAL_MIN_LOCAL", "3")
    text = wc.rqc(14, 6, seed=9).qasm()
    outs = []
    for prune in (1, 0):
        with q.State(14, world_size=world, prune=prune, fuse_bits=9, swap_slab_bytes=8192) as s:
            s.apply_circuit(q.Circuit(text))
            outs.append(s.amplitudes())
    assert np.array_equal(outs[0], outs[1])
    assert np.abs(outs[0] - osv.simulate(text)).max() <= TOL
