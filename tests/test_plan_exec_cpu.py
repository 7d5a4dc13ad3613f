"""The host planner's physical plan, executed independently on the CPU (single device).

qgpu_circuit_plan_text lists every pass the library would launch with every gate in PHYSICAL
positions at execution time -- after Alg.2/3 reorder, first-touch placement, the fusion
lookahead, the CX.D.CX peephole, SWAP relabels, the refined involvement rule's skips and
restrictions (reorder mode + 4), zero-half materialisation passes. A plain numpy executor applies
those gates in order and maps the result back through the final qubit map; it must equal the
oracle (program-order definition). This pins the whole host side of the fused path (a2-a4 and
NEXT-1) without a GPU, over many seeded circuits and every planner option.
"""
import numpy as np
import pytest

from oracle import statevector as osv
from workloads import circuits as wc

from test_sharded_cpu import _apply, _parse_plan

DIAG_HEAVY = ["cp", "cz", "rz", "cx", "crx", "ccx", "t", "h", "rzz", "cswap", "x", "u1", "crz", "s", "swap"]


@pytest.fixture(scope="module")
def q():
    from paper_conf_hpca_zhaogydmuzjyt22_b200 import build, qgpu
    build.build()
    qgpu.load()
    return qgpu


def _run_plan(text, n):
    passes, fmap = _parse_plan(text)
    psi = np.zeros(1 << n, dtype=np.complex128)
    psi[0] = 1.0
    for p in passes:
        assert p["kind"] != 5  # single device: no global-local swaps
        for (nt, targets, pc, diag, U) in p["gates"]:
            _apply(psi, 0, n, nt, targets, pc, U)
    xs = np.arange(1 << n)
    phys = np.zeros(1 << n, dtype=np.int64)
    never = np.zeros(1 << n, dtype=bool)
    for lq, pos in enumerate(fmap):
        bit = (xs >> lq) & 1
        if pos < 0:
            never |= bit.astype(bool)
        else:
            phys |= bit << pos
    return np.where(never, 0, psi[phys])


CIRCS = {
    "random": lambda s: wc.random_circuit(9, 150, seed=s),
    "randdiag": lambda s: wc.random_circuit(9, 150, seed=100 + s, names=DIAG_HEAVY),
    "qft0": lambda s: wc.qft(9),
    "qftx": lambda s: wc.qft(9, x=37 * s + 5),
    "qaoa": lambda s: wc.qaoa(10, 2, seed=s),
    "grqc": lambda s: wc.grqc(2, 5, 30, seed=s),
}


@pytest.mark.parametrize("name", sorted(CIRCS))
@pytest.mark.parametrize("fuse", [0, 7, 9])
@pytest.mark.parametrize("mode", [0, 1, 2])
@pytest.mark.parametrize("rule", [0, 1])
@pytest.mark.parametrize("sched", ["1", "0", "2"])
def test_physical_plan_executes_to_the_oracle(q, name, fuse, mode, rule, sched, monkeypatch):
    """sched: QGPU_PASS_SCHED -- 1 the default (plan_circuit_auto picks), 0 consecutive runs of
    the execution order only, 2 the pass-aware execution order always. 0 and 2 only where they
    differ from the default: fused passes under the paper's involvement rule."""
    if sched != "1" and (rule == 1 or fuse == 0 or (sched == "0" and fuse != 9)):
        pytest.skip("same plan as the default")
    monkeypatch.setenv("QGPU_PASS_SCHED", sched)
    for seed in (1, 2):
        c = CIRCS[name](seed)
        text = c.qasm()
        plan = q.Circuit(text).plan_text(c.n, 1, mode + 4 * rule, fuse)
        got = _run_plan(plan, c.n)
        ref = osv.simulate(text)
        assert np.abs(got - ref).max() <= 1e-12, (name, fuse, mode, rule, seed)
