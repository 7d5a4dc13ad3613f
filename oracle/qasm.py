"""ORACLE (test infrastructure only) -- OpenQASM-2 subset parser and gate table.

Independent of the product's C++ parser (no shared code). Accepted subset: SURVEY App. B
(the paper converts its benchmarks to OpenQASM; format ref [14]).

Gate table: SURVEY App. A, i.e. Qiskit's matrices including global phase, because the paper
extends Qiskit-Aer 0.7.0 (reading §8c-Q10 in DESIGN.md). H is Eq.5,
CNOT P:239, "cp" P:409. Little-endian: qubit q is bit q of the amplitude index (Eq.8,
reading Q8).

Each gate is lowered to ``Gate(U, targets, controls)``: U is a 2^t x 2^t complex128 matrix,
row/column bit j refers to ``targets[j]``, and the gate acts only where every control is |1>.
"""
from __future__ import annotations

import cmath
import math
import re
from dataclasses import dataclass
from typing import List, Tuple

import numpy as np


class QasmError(Exception):
    def __init__(self, kind: str, msg: str, line: int = 0, col: int = 0):
        super().__init__(f"{kind} at {line}:{col}: {msg}")
        self.kind, self.line, self.col = kind, line, col


@dataclass
class Gate:
    name: str
    U: np.ndarray            # (2^t, 2^t) complex128
    targets: Tuple[int, ...]
    controls: Tuple[int, ...]

    @property
    def qubits(self) -> Tuple[int, ...]:
        return tuple(self.targets) + tuple(self.controls)


# ----------------------------------------------------------------------------- gate table
SQ2 = 1.0 / math.sqrt(2.0)
I2 = np.eye(2, dtype=np.complex128)
X = np.array([[0, 1], [1, 0]], dtype=np.complex128)
Y = np.array([[0, -1j], [1j, 0]], dtype=np.complex128)
Z = np.array([[1, 0], [0, -1]], dtype=np.complex128)
H = np.array([[1, 1], [1, -1]], dtype=np.complex128) * SQ2          # Eq.5
S = np.array([[1, 0], [0, 1j]], dtype=np.complex128)
T = np.array([[1, 0], [0, cmath.exp(1j * math.pi / 4)]], dtype=np.complex128)
SX = 0.5 * np.array([[1 + 1j, 1 - 1j], [1 - 1j, 1 + 1j]], dtype=np.complex128)
SWAP = np.array([[1, 0, 0, 0], [0, 0, 1, 0], [0, 1, 0, 0], [0, 0, 0, 1]], dtype=np.complex128)


def rx(t):
    c, s = math.cos(t / 2), math.sin(t / 2)
    return np.array([[c, -1j * s], [-1j * s, c]], dtype=np.complex128)


def ry(t):
    c, s = math.cos(t / 2), math.sin(t / 2)
    return np.array([[c, -s], [s, c]], dtype=np.complex128)


def rz(l):
    return np.array([[cmath.exp(-0.5j * l), 0], [0, cmath.exp(0.5j * l)]], dtype=np.complex128)


def phase(l):
    return np.array([[1, 0], [0, cmath.exp(1j * l)]], dtype=np.complex128)


def u3(t, p, l):
    c, s = math.cos(t / 2), math.sin(t / 2)
    return np.array([[c, -cmath.exp(1j * l) * s],
                     [cmath.exp(1j * p) * s, cmath.exp(1j * (p + l)) * c]], dtype=np.complex128)


def rzz(t):
    a, b = cmath.exp(-0.5j * t), cmath.exp(0.5j * t)
    return np.diag([a, b, b, a]).astype(np.complex128)


# name -> (n_params, n_qubits, n_controls, builder(params) -> target matrix)
TABLE = {
    "id": (0, 1, 0, lambda p: I2), "x": (0, 1, 0, lambda p: X), "y": (0, 1, 0, lambda p: Y),
    "z": (0, 1, 0, lambda p: Z), "h": (0, 1, 0, lambda p: H), "s": (0, 1, 0, lambda p: S),
    "sdg": (0, 1, 0, lambda p: S.conj().T), "t": (0, 1, 0, lambda p: T),
    "tdg": (0, 1, 0, lambda p: T.conj().T), "sx": (0, 1, 0, lambda p: SX),
    "sxdg": (0, 1, 0, lambda p: SX.conj().T),
    "rx": (1, 1, 0, lambda p: rx(p[0])), "ry": (1, 1, 0, lambda p: ry(p[0])),
    "rz": (1, 1, 0, lambda p: rz(p[0])), "p": (1, 1, 0, lambda p: phase(p[0])),
    "u1": (1, 1, 0, lambda p: phase(p[0])), "u2": (2, 1, 0, lambda p: u3(math.pi / 2, p[0], p[1])),
    "u3": (3, 1, 0, lambda p: u3(*p)), "u": (3, 1, 0, lambda p: u3(*p)),
    "U": (3, 1, 0, lambda p: u3(*p)),
    # controlled: first operand(s) are controls, the rest targets
    "cx": (0, 2, 1, lambda p: X), "CX": (0, 2, 1, lambda p: X), "cy": (0, 2, 1, lambda p: Y),
    "cz": (0, 2, 1, lambda p: Z), "ch": (0, 2, 1, lambda p: H),
    "cp": (1, 2, 1, lambda p: phase(p[0])), "cu1": (1, 2, 1, lambda p: phase(p[0])),
    "crx": (1, 2, 1, lambda p: rx(p[0])), "cry": (1, 2, 1, lambda p: ry(p[0])),
    "crz": (1, 2, 1, lambda p: rz(p[0])), "cu3": (3, 2, 1, lambda p: u3(*p)),
    "ccx": (0, 3, 2, lambda p: X), "cswap": (0, 3, 1, lambda p: SWAP),
    # uncontrolled two-qubit: local index j = b_first + 2*b_second
    "swap": (0, 2, 0, lambda p: SWAP), "rzz": (1, 2, 0, lambda p: rzz(p[0])),
}

# ----------------------------------------------------------------------------- tokenizer
_TOK = re.compile(r"""
    (?P<ws>[ \t\r]+) | (?P<nl>\n) | (?P<comment>//[^\n]*) |
    (?P<num>(\d+\.\d*|\.\d+|\d+)([eE][+-]?\d+)?) |
    (?P<id>[A-Za-z_][A-Za-z0-9_]*) | (?P<str>"[^"\n]*") |
    (?P<arrow>->) | (?P<eqeq>==) | (?P<sym>[;,\[\]\(\)\{\}+\-*/^])
""", re.X)


def _tokenize(text: str):
    pos, line, lstart = 0, 1, 0
    toks = []
    while pos < len(text):
        m = _TOK.match(text, pos)
        if not m:
            raise QasmError("parse", f"unexpected character {text[pos]!r}", line, pos - lstart + 1)
        kind = m.lastgroup
        if kind == "nl":
            line += 1
            lstart = m.end()
        elif kind not in ("ws", "comment"):
            toks.append((kind, m.group(), line, pos - lstart + 1))
        pos = m.end()
    toks.append(("eof", "", line, pos - lstart + 1))
    return toks


_FUNCS = {"sin": math.sin, "cos": math.cos, "tan": math.tan, "exp": math.exp,
          "ln": math.log, "sqrt": math.sqrt}


class _Parser:
    def __init__(self, text: str):
        self.toks = _tokenize(text)
        self.i = 0
        self.regs = {}          # name -> (offset, size)
        self.n = 0
        self.gates: List[Gate] = []

    # -- helpers
    def peek(self):
        return self.toks[self.i]

    def next(self):
        t = self.toks[self.i]
        self.i += 1
        return t

    def expect(self, val):
        t = self.next()
        if t[1] != val:
            raise QasmError("parse", f"expected {val!r}, got {t[1]!r}", t[2], t[3])
        return t

    def err(self, msg, t=None, kind="parse"):
        t = t or self.peek()
        raise QasmError(kind, msg, t[2], t[3])

    # -- expressions (precedence: + - < * / < unary - < ^ (right assoc))
    def expr(self):
        v = self.term()
        while self.peek()[1] in ("+", "-"):
            op = self.next()[1]
            r = self.term()
            v = v + r if op == "+" else v - r
        return v

    def term(self):
        v = self.unary()
        while self.peek()[1] in ("*", "/"):
            op = self.next()[1]
            r = self.unary()
            v = v * r if op == "*" else v / r
        return v

    def unary(self):
        if self.peek()[1] == "-":
            self.next()
            return -self.unary()
        if self.peek()[1] == "+":
            self.next()
            return self.unary()
        return self.power()

    def power(self):
        b = self.primary()
        if self.peek()[1] == "^":
            self.next()
            return b ** self.unary()
        return b

    def primary(self):
        t = self.next()
        if t[0] == "num":
            return float(t[1])
        if t[0] == "id":
            if t[1] == "pi":
                return math.pi
            if t[1] in _FUNCS:
                self.expect("(")
                v = self.expr()
                self.expect(")")
                return _FUNCS[t[1]](v)
            self.err(f"unknown identifier {t[1]!r} in expression", t)
        if t[1] == "(":
            v = self.expr()
            self.expect(")")
            return v
        self.err(f"unexpected token {t[1]!r} in expression", t)

    # -- operands
    def operand(self):
        t = self.next()
        if t[0] != "id" or t[1] not in self.regs:
            self.err(f"unknown register {t[1]!r}", t)
        off, size = self.regs[t[1]]
        if self.peek()[1] == "[":
            self.next()
            it = self.next()
            if it[0] != "num":
                self.err("expected index", it)
            idx = int(it[1])
            self.expect("]")
            if idx >= size:
                self.err(f"index {idx} out of range for {t[1]}[{size}]", it, "invalid")
            return [off + idx]
        return [off + k for k in range(size)]

    def skip_statement(self):
        while self.peek()[1] != ";":
            if self.peek()[0] == "eof":
                self.err("unexpected end of input")
            self.next()
        self.next()

    def parse(self):
        t = self.peek()
        if t[1] == "OPENQASM":
            self.next()
            self.next()
            self.expect(";")
        while self.peek()[0] != "eof":
            t = self.next()
            w = t[1]
            if w == "include":
                s = self.next()
                if s[0] != "str":
                    self.err("expected file name", s)
                self.expect(";")
            elif w in ("qreg", "creg"):
                name = self.next()
                self.expect("[")
                sz = self.next()
                self.expect("]")
                self.expect(";")
                if w == "qreg":
                    self.regs[name[1]] = (self.n, int(sz[1]))
                    self.n += int(sz[1])
            elif w in ("measure", "barrier"):
                self.skip_statement()
            elif w in ("gate", "opaque", "reset", "if"):
                self.err(f"'{w}' is not supported", t, "unsupported")
            elif t[0] == "id" and w in TABLE:
                self.gate(t)
            elif t[0] == "id":
                self.err(f"unknown gate {w!r}", t, "unsupported")
            else:
                self.err(f"unexpected token {w!r}", t)
        return self.n, self.gates

    def gate(self, t):
        npar, nq, nctl, build = TABLE[t[1]]
        params = []
        if self.peek()[1] == "(":
            self.next()
            if self.peek()[1] != ")":
                params.append(self.expr())
                while self.peek()[1] == ",":
                    self.next()
                    params.append(self.expr())
            self.expect(")")
        if len(params) != npar:
            self.err(f"{t[1]} takes {npar} parameters, got {len(params)}", t, "invalid")
        ops = [self.operand()]
        while self.peek()[1] == ",":
            self.next()
            ops.append(self.operand())
        self.expect(";")
        if len(ops) != nq:
            self.err(f"{t[1]} takes {nq} qubits, got {len(ops)}", t, "invalid")
        width = max(len(o) for o in ops)
        for o in ops:
            if len(o) not in (1, width):
                self.err("register size mismatch", t, "invalid")
        U = build(params)
        for k in range(width):
            qs = [o[k] if len(o) > 1 else o[0] for o in ops]
            if len(set(qs)) != len(qs):
                self.err("repeated qubit operand", t, "invalid")
            self.gates.append(Gate(t[1], U, tuple(qs[nctl:]), tuple(qs[:nctl])))


def parse(text: str) -> Tuple[int, List[Gate]]:
    """QASM text -> (n_qubits, gates in file order)."""
    return _Parser(text).parse()


def is_diagonal(g: Gate) -> bool:
    """True when the target matrix is diagonal (used by the reference schedule statistics)."""
    U = g.U
    return bool(np.all(U[~np.eye(U.shape[0], dtype=bool)] == 0))
