"""Seeded synthetic circuit generators, emitted as OpenQASM-2 text.

This module is the ONLY code shared by the oracle (``oracle/``) and the CUDA path
(``paper_conf_hpca_zhaogydmuzjyt22_b200``). It holds none of the method's
arithmetic: it only decides *which* gates, on *which* qubits, with *which*
angles, and writes them as text. Gate matrices, parsing, scheduling and state
updates are implemented independently on each side.

Workload shapes follow the paper's benchmark table (Table I)
and the concrete recipes of SURVEY.md §8(d):

* ``ghz_qft``  -- config C1: GHZ_5 followed by QFT_5.
* ``qft``      -- Quantum Fourier Transform, Qiskit construction
                  (SURVEY §8c-Q11), optionally on a basis state |x> prepared by X.
* ``qaoa``     -- MaxCut QAOA on a seeded random 3-regular graph.
* ``rqc``      -- Google-style random circuit.
* ``gs``       -- graph state on a grid.
* ``hlf``      -- hidden linear function.
* ``bv``       -- Bernstein-Vazirani.
* ``iqp``      -- IQP: H, diagonal layer, H.
* ``random_circuit`` -- fuzz circuits over the whole supported gate set.
* ``mirror``   -- U followed by U^dagger (adjoint written at the text level).

A circuit is a list of ``Op(name, params, qubits)``; ``params`` are QASM
expression strings (``"pi/8"``) or floats (written with ``repr`` so the text
round-trips bit-exactly).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import List, Sequence, Tuple, Union

import numpy as np

Param = Union[str, float]


@dataclass
class Op:
    name: str
    params: Tuple[Param, ...] = ()
    qubits: Tuple[int, ...] = ()


@dataclass
class Circuit:
    n: int
    ops: List[Op] = field(default_factory=list)
    meta: dict = field(default_factory=dict)

    def add(self, name: str, qubits: Sequence[int], params: Sequence[Param] = ()) -> "Circuit":
        self.ops.append(Op(name, tuple(params), tuple(int(q) for q in qubits)))
        return self

    def __len__(self) -> int:
        return len(self.ops)

    def qasm(self) -> str:
        lines = ["OPENQASM 2.0;", 'include "qelib1.inc";', f"qreg q[{self.n}];"]
        for op in self.ops:
            ps = ""
            if op.params:
                ps = "(" + ",".join(_fmt(p) for p in op.params) + ")"
            qs = ",".join(f"q[{q}]" for q in op.qubits)
            lines.append(f"{op.name}{ps} {qs};")
        return "\n".join(lines) + "\n"


def _fmt(p: Param) -> str:
    if isinstance(p, str):
        return p
    return repr(float(p))


# --------------------------------------------------------------------------- families

def qft_ops(c: Circuit, qubits: Sequence[int], swaps: bool = True) -> Circuit:
    """Qiskit ``QFT(n)`` construction: for j = n-1..0: H(j), then
    CP(pi/2^(j-k)) on (j, k) for k = j-1..0; finally SWAP(i, n-1-i)."""
    n = len(qubits)
    for j in range(n - 1, -1, -1):
        c.add("h", [qubits[j]])
        for k in range(j - 1, -1, -1):
            c.add("cp", [qubits[j], qubits[k]], [f"pi/{2 ** (j - k)}"])
    if swaps:
        for i in range(n // 2):
            c.add("swap", [qubits[i], qubits[n - 1 - i]])
    return c


def qft(n: int, x: int | None = None, swaps: bool = True) -> Circuit:
    """QFT_n on |0...0> (x=None) or on the basis state |x> prepared with X gates."""
    c = Circuit(n, meta={"family": "qft", "x": x})
    if x is not None:
        for q in range(n):
            if (x >> q) & 1:
                c.add("x", [q])
    return qft_ops(c, list(range(n)), swaps)


def ghz_qft(n: int = 5) -> Circuit:
    """Config C1: GHZ_n (H q0, CX(0,k) for k=1..n-1) followed by QFT_n."""
    c = Circuit(n, meta={"family": "ghz_qft"})
    c.add("h", [0])
    for k in range(1, n):
        c.add("cx", [0, k])
    return qft_ops(c, list(range(n)))


def ghz(n: int) -> Circuit:
    c = Circuit(n, meta={"family": "ghz"})
    c.add("h", [0])
    for k in range(1, n):
        c.add("cx", [k - 1, k])
    return c


def random_regular_graph(n: int, d: int, rng: np.random.Generator) -> List[Tuple[int, int]]:
    """Pairing (configuration) model with rejection: simple d-regular graph."""
    assert (n * d) % 2 == 0
    while True:
        stubs = np.repeat(np.arange(n), d)
        rng.shuffle(stubs)
        pairs = stubs.reshape(-1, 2)
        ok = True
        seen = set()
        for u, v in pairs:
            u, v = int(min(u, v)), int(max(u, v))
            if u == v or (u, v) in seen:
                ok = False
                break
            seen.add((u, v))
        if ok:
            return [(int(a), int(b)) for a, b in pairs]


def qaoa(n: int, p: int = 2, seed: int = 1,
         gammas: Sequence[float] = (0.4, 0.8), betas: Sequence[float] = (0.7, 0.35)) -> Circuit:
    """MaxCut QAOA on a random 3-regular graph: H on all; per layer, for
    each edge (u,v) in order: CX(u,v), RZ(2*gamma) on v, CX(u,v); then RX(2*beta) on all."""
    rng = np.random.default_rng(seed)
    edges = random_regular_graph(n, 3, rng)
    c = Circuit(n, meta={"family": "qaoa", "edges": edges, "p": p, "seed": seed})
    for q in range(n):
        c.add("h", [q])
    for layer in range(p):
        g, b = gammas[layer % len(gammas)], betas[layer % len(betas)]
        for u, v in edges:
            c.add("cx", [u, v])
            c.add("rz", [v], [2.0 * g])
            c.add("cx", [u, v])
        for q in range(n):
            c.add("rx", [q], [2.0 * b])
    return c


def rqc(n: int, depth: int = 20, seed: int = 3) -> Circuit:
    """Google-style random circuit on a 1-D chain: H on all; each cycle t
    applies one random gate per qubit from {sqrt X, sqrt Y, sqrt W} (never the same twice in
    a row on a qubit), then CZ on (i, i+1) for i = t mod 2, t mod 2 + 2, ..."""
    rng = np.random.default_rng(seed)
    choices = [("rx", ("pi/2",)), ("ry", ("pi/2",)), ("u3", ("pi/2", "-pi/4", "pi/4"))]
    c = Circuit(n, meta={"family": "rqc", "depth": depth, "seed": seed})
    for q in range(n):
        c.add("h", [q])
    last = [-1] * n
    for t in range(depth):
        for q in range(n):
            k = int(rng.integers(0, 3))
            while k == last[q]:
                k = int(rng.integers(0, 3))
            last[q] = k
            name, ps = choices[k]
            c.add(name, [q], ps)
        for i in range(t % 2, n - 1, 2):
            c.add("cz", [i, i + 1])
    return c


def grqc(rows: int, cols: int, depth: int, seed: int = 5) -> Circuit:
    """Google-style deep random circuit on a 2-D grid (the paper's "grqc", Table III,
    generated "under rules defined in [9]"; the exact rules are not given, reading in DESIGN.md):
    H on all; cycle t = 1..depth applies CZ on the couplers of class (t - 1) mod 8 (horizontal
    couplers split by (row mod 2, col mod 2), then vertical ones likewise), then on every qubit
    that was in a CZ in the previous cycle and is not in one now a single-qubit gate: T if it
    has had none yet, else one of {sqrt X, sqrt Y, T} different from its previous one. A 4x8
    grid with depth 473 gives 7238 operations, the size of Table III's grqc_32 (7241)."""
    rng = np.random.default_rng(seed)
    n = rows * cols
    c = Circuit(n, meta={"family": "grqc", "rows": rows, "cols": cols, "depth": depth, "seed": seed})
    for q in range(n):
        c.add("h", [q])
    classes: List[List[Tuple[int, int]]] = [[] for _ in range(8)]
    for r in range(rows):
        for cc in range(cols):
            q = r * cols + cc
            if cc + 1 < cols:
                classes[2 * (r % 2) + (cc % 2)].append((q, q + 1))
            if r + 1 < rows:
                classes[4 + 2 * (r % 2) + (cc % 2)].append((q, q + cols))
    gates = [("rx", ("pi/2",)), ("ry", ("pi/2",)), ("t", ())]
    last = [-1] * n
    prev_cz: set = set()
    for t in range(1, depth + 1):
        cur = classes[(t - 1) % 8]
        busy = set()
        for u, v in cur:
            c.add("cz", [u, v])
            busy.update((u, v))
        for q in range(n):
            if q in prev_cz and q not in busy:
                if last[q] < 0:
                    k = 2
                else:
                    k = int(rng.integers(0, 3))
                    while k == last[q]:
                        k = int(rng.integers(0, 3))
                last[q] = k
                name, ps = gates[k]
                c.add(name, [q], ps)
        prev_cz = busy
    return c


def grid_edges(rows: int, cols: int) -> List[Tuple[int, int]]:
    e = []
    for r in range(rows):
        for cc in range(cols):
            q = r * cols + cc
            if cc + 1 < cols:
                e.append((q, q + 1))
            if r + 1 < rows:
                e.append((q, q + cols))
    return e


def gs(rows: int, cols: int) -> Circuit:
    """Graph state on a rows x cols grid: H on all, CZ on every grid edge."""
    n = rows * cols
    edges = grid_edges(rows, cols)
    c = Circuit(n, meta={"family": "gs", "edges": edges})
    for q in range(n):
        c.add("h", [q])
    for u, v in edges:
        c.add("cz", [u, v])
    return c


def graph_state(n: int, edges: Sequence[Tuple[int, int]]) -> Circuit:
    c = Circuit(n, meta={"family": "gs", "edges": list(edges)})
    for q in range(n):
        c.add("h", [q])
    for u, v in edges:
        c.add("cz", [u, v])
    return c


def hlf(rows: int, cols: int, seed: int = 2) -> Circuit:
    """Hidden linear function (BGK) on a grid: H^n; CZ on each grid edge kept with p=1/2;
    S on each qubit with p=1/2; H^n."""
    rng = np.random.default_rng(seed)
    n = rows * cols
    edges = [e for e in grid_edges(rows, cols) if rng.random() < 0.5]
    svec = [q for q in range(n) if rng.random() < 0.5]
    c = Circuit(n, meta={"family": "hlf", "edges": edges, "s": svec, "seed": seed})
    for q in range(n):
        c.add("h", [q])
    for u, v in edges:
        c.add("cz", [u, v])
    for q in svec:
        c.add("s", [q])
    for q in range(n):
        c.add("h", [q])
    return c


def bv(n: int, s: int) -> Circuit:
    """Bernstein-Vazirani: data q0..q(n-2), ancilla q(n-1). X anc; H all; CX(q_i, anc)
    for s_i=1; H on data."""
    c = Circuit(n, meta={"family": "bv", "s": s})
    a = n - 1
    c.add("x", [a])
    for q in range(n):
        c.add("h", [q])
    for q in range(n - 1):
        if (s >> q) & 1:
            c.add("cx", [q, a])
    for q in range(n - 1):
        c.add("h", [q])
    return c


def iqp(n: int, seed: int = 4) -> Circuit:
    """IQP: H^n, a random diagonal layer (CP on random pairs, T on random qubits), H^n."""
    rng = np.random.default_rng(seed)
    c = Circuit(n, meta={"family": "iqp", "seed": seed})
    for q in range(n):
        c.add("h", [q])
    for i in range(n):
        for j in range(i + 1, n):
            if rng.random() < 0.3:
                c.add("cp", [i, j], [float(rng.uniform(0, 2 * math.pi))])
    for q in range(n):
        if rng.random() < 0.5:
            c.add("t", [q])
    for q in range(n):
        c.add("h", [q])
    return c


# gate name -> (n_params, n_qubits)
GATE_ARITY = {
    "id": (0, 1), "x": (0, 1), "y": (0, 1), "z": (0, 1), "h": (0, 1), "s": (0, 1),
    "sdg": (0, 1), "t": (0, 1), "tdg": (0, 1), "sx": (0, 1), "sxdg": (0, 1),
    "rx": (1, 1), "ry": (1, 1), "rz": (1, 1), "p": (1, 1), "u1": (1, 1),
    "u2": (2, 1), "u3": (3, 1), "u": (3, 1),
    "cx": (0, 2), "cy": (0, 2), "cz": (0, 2), "ch": (0, 2), "cp": (1, 2), "cu1": (1, 2),
    "crx": (1, 2), "cry": (1, 2), "crz": (1, 2), "cu3": (3, 2),
    "swap": (0, 2), "rzz": (1, 2), "ccx": (0, 3), "cswap": (0, 3),
}


def random_circuit(n: int, n_gates: int, seed: int, names: Sequence[str] | None = None) -> Circuit:
    """Fuzz circuit: uniformly random gates from ``names`` (default: the whole supported
    set), random distinct operand qubits, random angles."""
    rng = np.random.default_rng(seed)
    names = list(names) if names is not None else sorted(GATE_ARITY)
    names = [g for g in names if GATE_ARITY[g][1] <= n]
    c = Circuit(n, meta={"family": "random", "seed": seed})
    for _ in range(n_gates):
        g = names[int(rng.integers(0, len(names)))]
        npar, nq = GATE_ARITY[g]
        qs = rng.choice(n, size=nq, replace=False)
        ps = [float(rng.uniform(-math.pi, math.pi)) for _ in range(npar)]
        c.add(g, qs, ps)
    return c


_SELF_ADJOINT = {"id", "x", "y", "z", "h", "cx", "cy", "cz", "ch", "swap", "ccx", "cswap"}
_SWAP_ADJ = {"s": "sdg", "sdg": "s", "t": "tdg", "tdg": "t", "sx": "sxdg", "sxdg": "sx"}
_NEG1 = {"rx", "ry", "rz", "p", "u1", "cp", "cu1", "crx", "cry", "crz", "rzz"}


def _neg(p: Param) -> Param:
    if isinstance(p, str):
        return f"-({p})"
    return -float(p)


def adjoint_op(op: Op) -> Op:
    """Text-level adjoint of one op (used only to build mirror circuits)."""
    if op.name in _SELF_ADJOINT:
        return op
    if op.name in _SWAP_ADJ:
        return Op(_SWAP_ADJ[op.name], op.params, op.qubits)
    if op.name in _NEG1:
        return Op(op.name, (_neg(op.params[0]),), op.qubits)
    if op.name in ("u3", "u", "cu3"):
        th, ph, la = op.params
        return Op(op.name, (_neg(th), _neg(la), _neg(ph)), op.qubits)
    if op.name == "u2":
        ph, la = op.params
        return Op("u3", ("-pi/2", _neg(la), _neg(ph)), op.qubits)
    raise ValueError(f"no adjoint rule for {op.name}")


def mirror(c: Circuit) -> Circuit:
    """U followed by U^dagger: returns |0...0> exactly in exact arithmetic."""
    m = Circuit(c.n, list(c.ops), dict(c.meta, mirror=True))
    for op in reversed(c.ops):
        m.ops.append(adjoint_op(op))
    return m


# --------------------------------------------------------------------------- configs

def config_circuit(name: str, n: int | None = None) -> Circuit:
    """BASELINE.json configs as named workloads."""
    if name == "C1":
        return ghz_qft(5)
    if name == "C2":
        return qft(n or 28)
    if name == "C2x":
        nn = n or 28
        x = int(np.random.default_rng(2).integers(0, 2 ** nn))
        return qft(nn, x=x)
    if name == "C3":
        return qaoa(n or 32, p=2, seed=1)
    if name == "C4":
        return rqc(n or 34, depth=20, seed=3)
    if name == "C5a":
        return gs(6, 6)
    if name == "C5b":
        return hlf(6, 6, seed=2)
    raise KeyError(name)
