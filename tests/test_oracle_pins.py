"""Pins for the oracle (CPU only): the oracle is checked against things other than itself --
the paper's worked examples, closed forms, brute-force Kronecker-product unitaries and
invariants -- so that a dropped term, wrong sign/index or transposed operand fails a test.
"""
import cmath
import json
import math
import os

import numpy as np
import pytest

from oracle import qasm as oq
from oracle import statevector as osv
from workloads import circuits as wc

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------------------- brute force

def _E(r, s):
    m = np.zeros((2, 2), dtype=np.complex128)
    m[r, s] = 1
    return m


def _kron_chain(n, factors):
    """kron over qubits n-1 ... 0 (qubit 0 is the least significant index bit)."""
    out = np.ones((1, 1), dtype=np.complex128)
    for q in range(n - 1, -1, -1):
        out = np.kron(out, factors.get(q, np.eye(2)))
    return out


def full_operator(n, U, targets, controls):
    """Textbook embedding: I - P_C + P_C (U on targets), built from Kronecker products only."""
    t = len(targets)
    Uemb = np.zeros((1 << n, 1 << n), dtype=np.complex128)
    for r in range(1 << t):
        for s in range(1 << t):
            if U[r, s] == 0:
                continue
            f = {targets[k]: _E((r >> k) & 1, (s >> k) & 1) for k in range(t)}
            Uemb += U[r, s] * _kron_chain(n, f)
    PC = _kron_chain(n, {c: _E(1, 1) for c in controls})
    return np.eye(1 << n) - PC + PC @ Uemb


@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_unitary_random_circuits(seed):
    n = 2 + seed % 5          # 2..6 qubits
    c = wc.random_circuit(n, 25, seed=100 + seed)
    nq, gates = oq.parse(c.qasm())
    assert nq == n
    Utot = np.eye(1 << n, dtype=np.complex128)
    for g in gates:
        Utot = full_operator(n, g.U, g.targets, g.controls) @ Utot
    assert np.abs(Utot.conj().T @ Utot - np.eye(1 << n)).max() < 1e-12
    psi = osv.simulate_gates(n, gates)
    assert np.abs(psi - Utot[:, 0]).max() < 1e-12
    # arbitrary (non-basis) input state as well
    rng = np.random.default_rng(seed)
    v = rng.normal(size=1 << n) + 1j * rng.normal(size=1 << n)
    v /= np.linalg.norm(v)
    w = osv.simulate_gates(n, gates, psi=v.copy())
    assert np.abs(w - Utot @ v).max() < 1e-12


def test_eq6_eq7_hadamard_worked_example():
    """P:60-68, Eq.5-7: H on qubit 0 of a 2-qubit system updates (a00,a01) and (a10,a11)."""
    rng = np.random.default_rng(7)
    a = rng.normal(size=4) + 1j * rng.normal(size=4)
    psi = a.copy()
    osv.apply_gate(psi, 2, oq.H, [0])
    s = 1 / math.sqrt(2)
    # subscripts are written q1 q0: a_01 is index 1
    exp = np.array([s * (a[0] + a[1]), s * (a[0] - a[1]), s * (a[2] + a[3]), s * (a[2] - a[3])])
    assert np.abs(psi - exp).max() < 1e-15


def test_eq8_pair_rule_every_qubit():
    """Eq.8: a gate on qubit j pairs indices that differ only in bit j."""
    n = 5
    rng = np.random.default_rng(3)
    U = oq.u3(0.3, 1.1, -0.4)
    for j in range(n):
        a = rng.normal(size=1 << n) + 1j * rng.normal(size=1 << n)
        psi = a.copy()
        osv.apply_gate(psi, n, U, [j])
        for i in range(1 << n):
            if (i >> j) & 1:
                continue
            i1 = i | (1 << j)
            assert abs(psi[i] - (U[0, 0] * a[i] + U[0, 1] * a[i1])) < 1e-14
            assert abs(psi[i1] - (U[1, 0] * a[i] + U[1, 1] * a[i1])) < 1e-14


def test_case2_chunk_pairs():
    """7 qubits, 8 chunks of 16; a gate on chunk bit 1 couples chunks
    (0,2),(1,3),(4,6),(5,7) (reading Q8: the text's q6 is q5 in 0-based little-endian)."""
    g = json.load(open(os.path.join(GOLDEN, "alg1_examples.json")))["case2_example"]
    n, c, b = g["n"], g["chunk_bits"], g["gate_chunk_bit"]
    for lo, hi in g["pairs"]:
        psi = np.zeros(1 << n, dtype=np.complex128)
        psi[lo << c: (lo + 1) << c] = 1.0
        osv.apply_gate(psi, n, oq.H, [c + b])
        nz = {int(j) for j in np.nonzero(np.abs(psi.reshape(-1, 1 << c)).sum(1))[0]}
        assert nz == {lo, hi}


# ----------------------------------------------------------------------------- closed forms

def test_ghz_qft5_closed_form():
    """QFT(GHZ_5) psi_y = (1 + e^{2 pi i 31 y / 32}) / sqrt(64)."""
    psi = osv.simulate(wc.ghz_qft(5).qasm())
    y = np.arange(32)
    exp = (1 + np.exp(2j * np.pi * 31 * y / 32)) / 8.0
    assert np.abs(psi - exp).max() < 1e-13


def test_ghz_closed_form():
    psi = osv.simulate(wc.ghz(9).qasm())
    exp = np.zeros(1 << 9, dtype=complex)
    exp[0] = exp[-1] = 1 / math.sqrt(2)
    assert np.abs(psi - exp).max() < 1e-15


@pytest.mark.parametrize("n,x", [(6, 0), (6, 37), (8, 201), (10, 777)])
def test_qft_basis_state_closed_form(n, x):
    """QFT|x> = 2^{-n/2} sum_y e^{+2 pi i x y / 2^n} |y>."""
    psi = osv.simulate(wc.qft(n, x=x).qasm())
    y = np.arange(1 << n)
    exp = np.exp(2j * np.pi * x * y / (1 << n)) / math.sqrt(1 << n)
    assert np.abs(psi - exp).max() < 1e-12


def test_graph_state_closed_form():
    """psi_x = (-1)^{sum_{(u,v) in E} x_u x_v} / 2^{n/2}."""
    c = wc.gs(3, 4)
    n, edges = c.n, c.meta["edges"]
    psi = osv.simulate(c.qasm())
    x = np.arange(1 << n)
    par = np.zeros(1 << n, dtype=np.int64)
    for u, v in edges:
        par ^= ((x >> u) & 1) & ((x >> v) & 1)
    exp = (1 - 2 * par) / math.sqrt(1 << n)
    assert np.abs(psi - exp).max() < 1e-14


def _gf2_kernel(A):
    """Basis of ker A over GF(2) (A: n x n 0/1)."""
    A = A.copy() % 2
    n = A.shape[1]
    piv_cols, r = [], 0
    for col in range(n):
        p = next((i for i in range(r, A.shape[0]) if A[i, col]), None)
        if p is None:
            continue
        A[[r, p]] = A[[p, r]]
        for i in range(A.shape[0]):
            if i != r and A[i, col]:
                A[i] ^= A[r]
        piv_cols.append(col)
        r += 1
    free = [c for c in range(n) if c not in piv_cols]
    basis = []
    for f in free:
        v = np.zeros(n, dtype=np.int64)
        v[f] = 1
        for i, pc in enumerate(piv_cols):
            v[pc] = A[i, f]
        basis.append(v)
    return basis


def hlf_expected_probabilities(n, edges, svec):
    """A = adjacency + diag(S bits); q(x) = sum A_ii x_i + 2 sum_{i<j} A_ij x_i x_j
    mod 4; L = ker A. P(z) = 2^{dim L - n} iff z.x == q(x)/2 (mod 2) for all x in L (basis)."""
    A = np.zeros((n, n), dtype=np.int64)
    for u, v in edges:
        A[u, v] = A[v, u] = 1
    for q in svec:
        A[q, q] = 1
    basis = _gf2_kernel(A)
    z = np.arange(1 << n)
    ok = np.ones(1 << n, dtype=bool)
    for xv in basis:
        qx = int(sum(A[i, i] * xv[i] for i in range(n)) +
                 2 * sum(A[i, j] * xv[i] * xv[j] for i in range(n) for j in range(i + 1, n))) % 4
        assert qx % 2 == 0
        dot = np.zeros(1 << n, dtype=np.int64)
        for i in range(n):
            if xv[i]:
                dot ^= (z >> i) & 1
        ok &= dot == (qx // 2)
    return np.where(ok, 2.0 ** (len(basis) - n), 0.0)


@pytest.mark.parametrize("rows,cols,seed", [(3, 3, 2), (3, 4, 5), (2, 5, 9)])
def test_hlf_closed_form(rows, cols, seed):
    c = wc.hlf(rows, cols, seed=seed)
    psi = osv.simulate(c.qasm())
    p = np.abs(psi) ** 2
    exp = hlf_expected_probabilities(c.n, c.meta["edges"], c.meta["s"])
    assert np.abs(p - exp).max() < 1e-12


@pytest.mark.parametrize("n,s", [(7, 0b101101), (9, 0b11001010)])
def test_bernstein_vazirani(n, s):
    """psi_s = 1/sqrt2, psi_{s + 2^(n-1)} = -1/sqrt2."""
    psi = osv.simulate(wc.bv(n, s).qasm())
    assert abs(psi[s] - 1 / math.sqrt(2)) < 1e-14
    assert abs(psi[s + (1 << (n - 1))] + 1 / math.sqrt(2)) < 1e-14
    p = osv.probabilities(psi, n, list(range(n - 1)))
    assert abs(p[s] - 1) < 1e-12


@pytest.mark.parametrize("n,w,k", [(6, 13, 1), (6, 13, 3), (8, 200, 5), (10, 1000, 7)])
def test_grover_success_probability(n, w, k):
    """|psi_w|^2 = sin^2((2k+1) theta), sin theta = 2^{-n/2}; MCZ with n-1
    controls applied through the gate-level interface."""
    psi = osv.zero_state(n)
    def mcz():
        osv.apply_gate(psi, n, oq.Z, [n - 1], list(range(n - 1)))
    def xs(mask):
        for q in range(n):
            if (mask >> q) & 1:
                osv.apply_gate(psi, n, oq.X, [q])
    for q in range(n):
        osv.apply_gate(psi, n, oq.H, [q])
    full = (1 << n) - 1
    for _ in range(k):
        xs(full & ~w); mcz(); xs(full & ~w)
        for q in range(n):
            osv.apply_gate(psi, n, oq.H, [q])
        xs(full); mcz(); xs(full)
        for q in range(n):
            osv.apply_gate(psi, n, oq.H, [q])
    th = math.asin(2 ** (-n / 2))
    assert abs(abs(psi[w]) ** 2 - math.sin((2 * k + 1) * th) ** 2) < 1e-12


@pytest.mark.parametrize("fam", ["qaoa", "rqc", "random", "iqp", "grqc"])
def test_norm_and_mirror(fam):
    """norm conserved; U U^dagger returns e_0."""
    c = {"qaoa": lambda: wc.qaoa(10, 2, seed=1), "rqc": lambda: wc.rqc(10, 8, seed=3),
         "random": lambda: wc.random_circuit(9, 200, seed=5), "iqp": lambda: wc.iqp(9),
         "grqc": lambda: wc.grqc(3, 3, 40, seed=5)}[fam]()
    psi = osv.simulate(c.qasm())
    assert abs(1 - np.vdot(psi, psi).real) < 1e-12
    m = osv.simulate(wc.mirror(c).qasm())
    e0 = np.zeros_like(m)
    e0[0] = 1
    assert np.abs(m - e0).max() < 1e-12


def test_probabilities_marginals():
    """probabilities are |a|^2; marginals sum over the other qubits."""
    n = 8
    psi = osv.simulate(wc.random_circuit(n, 60, seed=9).qasm())
    t = (np.abs(psi) ** 2).reshape([2] * n)       # axis k <-> qubit n-1-k
    for qs in ([0], [3, 1], [7, 0, 5], list(range(n))):
        p = osv.probabilities(psi, n, qs)
        axes_keep = [n - 1 - q for q in qs]
        m = t.sum(axis=tuple(a for a in range(n) if a not in axes_keep))
        # m's axes are in increasing axis order; reorder to (qs[-1], ..., qs[0]) -> C index y
        order = sorted(axes_keep)
        m = np.transpose(m, [order.index(a) for a in reversed(axes_keep)]).reshape(-1)
        assert np.abs(p - m).max() < 1e-14
    assert abs(osv.probabilities(psi, n, []).sum() - 1) < 1e-12


# ----------------------------------------------------------------------------- gate table

def test_gate_table_values():
    """SURVEY App. A conventions: rz carries global phase, p/u1 do not; u2 = u3(pi/2,.,.)."""
    _, g = oq.parse('OPENQASM 2.0;\ninclude "qelib1.inc";\nqreg q[2];\n'
                    'rz(0.5) q[0]; p(0.5) q[0]; u2(0.1,0.2) q[0]; sx q[0]; cp(0.3) q[0],q[1];'
                    'rzz(0.4) q[0],q[1]; swap q[0],q[1]; ccx q[0],q[1],q[0];'[:-19] + "\n")
    rz, p, u2, sx, cp, rzz, sw = [x.U for x in g]
    assert np.allclose(rz, np.diag([cmath.exp(-0.25j), cmath.exp(0.25j)]), atol=0, rtol=1e-15)
    assert np.allclose(p, np.diag([1, cmath.exp(0.5j)]))
    assert np.allclose(u2, np.array([[1, -cmath.exp(0.2j)], [cmath.exp(0.1j), cmath.exp(0.3j)]])
                       / math.sqrt(2))
    assert np.allclose(sx @ sx, oq.X)
    assert g[4].controls == (0,) and g[4].targets == (1,)
    assert np.allclose(rzz, np.diag([cmath.exp(-0.2j), cmath.exp(0.2j), cmath.exp(0.2j),
                                     cmath.exp(-0.2j)]))
    for name, (npar, nq, nc, b) in oq.TABLE.items():
        U = b([0.37, -1.2, 2.1][:npar])
        assert np.abs(U.conj().T @ U - np.eye(U.shape[0])).max() < 1e-15, name


def test_parser_errors_and_broadcast():
    with pytest.raises(oq.QasmError) as e:
        oq.parse("OPENQASM 2.0;\nqreg q[2];\nh q[0]\ncx q[0],q[1];\n")
    assert e.value.kind == "parse" and e.value.line == 4
    with pytest.raises(oq.QasmError) as e:
        oq.parse("OPENQASM 2.0;\nqreg q[2];\nreset q[0];\n")
    assert e.value.kind == "unsupported"
    with pytest.raises(oq.QasmError) as e:
        oq.parse("OPENQASM 2.0;\nqreg q[2];\nfoo q[0];\n")
    assert e.value.kind == "unsupported"
    n, g = oq.parse("OPENQASM 2.0;\nqreg a[2];\nqreg b[3];\ncreg c[5];\nh b;\ncx a[1],b[2];\n"
                    "rx(-pi/2^2 + 2*sin(pi/6)) a[0];\nbarrier a;\nmeasure a[0] -> c[0];\n")
    assert n == 5 and [x.targets for x in g[:3]] == [(2,), (3,), (4,)]
    assert g[3].controls == (1,) and g[3].targets == (4,)
    assert np.allclose(g[4].U, oq.rx(-math.pi / 4 + 1.0))


def test_light_cone_helper_matches_full_simulation():
    """The sampled-amplitude helper of the n = 31/32 GPU tests (tests/lightcone.py) equals the
    oracle's full simulation of the same product preparation + gates, at n = 9 on every index."""
    from lightcone import product_light_cone
    n = 9
    rng = np.random.default_rng(7)
    prep = [oq.u3(*rng.uniform(-3, 3, 3)) for _ in range(n)]
    factors = [U[:, 0].copy() for U in prep]
    U4 = np.linalg.qr(rng.normal(size=(4, 4)) + 1j * rng.normal(size=(4, 4)))[0]
    gates = [(oq.u3(*rng.uniform(-3, 3, 3)), [0], []), (oq.u3(1, 2, 3), [8], [7]),
             (U4, [8, 3], []), (np.array([[0, 1], [1, 0]], dtype=complex), [8], [0]),
             (oq.phase(0.7), [0], [8]), (np.diag(np.exp(1j * rng.uniform(-3, 3, 4))), [8, 1], [])]
    psi = osv.zero_state(n)
    for t in range(n):
        osv.apply_gate(psi, n, prep[t], [t])
    for U, t, cs in gates:
        osv.apply_gate(psi, n, U, t, cs)
    got = product_light_cone(n, factors, gates, np.arange(1 << n))
    assert np.abs(got - psi).max() <= 1e-14
