"""Parity of every synthetic family at the library's DEFAULT NVRTC threshold (passes of >= 2^12
amplitudes specialised; the suite-wide conftest raises it to 2^20 to bound compile time), so the
kernels bench.py runs -- NVRTC bodies with unit-diagonal gate forms, kernel-parameter matrices,
two CTAs per SM for FP64-heavy passes, the lane-bit policy chosen by the planner -- are checked
against the oracle at sizes where the oracle takes a second, and bit-identical with the generic
(interpreted) kernel's prune on/off behaviour."""
import os

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


@pytest.fixture(autouse=True)
def default_threshold():
    old = os.environ.pop("QGPU_JIT_MIN_BITS", None)
    yield
    if old is not None:
        os.environ["QGPU_JIT_MIN_BITS"] = old


FAMILIES = {
    "qft16": lambda: wc.qft(16),
    "qft16x": lambda: wc.qft(16, x=40503),
    "qaoa16": lambda: wc.qaoa(16, 2, seed=1),
    "rqc16": lambda: wc.rqc(16, 12, seed=3),
    "grqc16": lambda: wc.grqc(4, 4, 40, seed=5),
    "gs16": lambda: wc.gs(4, 4),
    "hlf16": lambda: wc.hlf(4, 4, seed=2),
    "iqp15": lambda: wc.iqp(15),
    "fuzz15": lambda: wc.random_circuit(15, 400, seed=21),
}


@pytest.mark.parametrize("name", sorted(FAMILIES))
@pytest.mark.parametrize("two_cta", ["2", "1", "0"])
def test_default_jit_threshold_vs_oracle(q, name, two_cta, monkeypatch):
    monkeypatch.setenv("QGPU_2CTA", two_cta)
    c = FAMILIES[name]()
    text = c.qasm()
    with q.State(c.n) as s:
        s.apply_circuit(q.Circuit(text))
        got = s.amplitudes()
        st = s.stats()
    ref = osv.simulate(text)
    assert np.abs(got - ref).max() <= TOL
    assert abs(np.vdot(got, got).real - 1) <= 1e-12
    assert st["jit_launches"] >= 1


@pytest.mark.parametrize("name", ["qaoa16", "rqc16", "fuzz15"])
def test_default_jit_prune_neutrality_and_unit_forms(q, name, monkeypatch):
    """prune on / off exactly equal with the default kernels; the unit-diagonal forms
    change only rounding (QGPU_UNIT_FORMS=0 restores the plain classes)."""
    text = FAMILIES[name]().qasm()
    n = FAMILIES[name]().n
    outs = {}
    for prune in (1, 0):
        with q.State(n, prune=prune) as s:
            s.apply_circuit(q.Circuit(text))
            outs[prune] = s.amplitudes()
    assert np.array_equal(outs[0], outs[1])
    monkeypatch.setenv("QGPU_UNIT_FORMS", "0")
    with q.State(n) as s:
        s.apply_circuit(q.Circuit(text))
        plain = s.amplitudes()
    assert np.abs(plain - outs[1]).max() <= 1e-12
