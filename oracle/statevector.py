"""ORACLE (test infrastructure only) -- program-order state-vector simulation.

SURVEY §8c-c1: psi <- e_0 (all qubits start in |0>), then every gate in file order
(or in an explicitly given order, for schedule-soundness checks) through the plain loops of
``sv.c`` (Eq.8). No pruning, no reorder: pruning and reorder are exact (P:221,
P:340-342), so the plain definition is the reference for the pruned, reordered GPU path.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import List, Optional, Sequence

import numpy as np

from .qasm import Gate, parse

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sv.c")
_LIB = os.path.join(_HERE, "liboracle_sv.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile sv.c with plain -O2 (no -ffast-math) and OpenMP."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-shared", "-fPIC",
                               _SRC, "-o", _LIB + ".tmp"])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        lib.sv_apply.argtypes = [P, ctypes.c_int, P, ctypes.c_int, P, ctypes.c_int, P, ctypes.c_int]
        lib.sv_apply.restype = ctypes.c_int
        lib.sv_probabilities.argtypes = [P, ctypes.c_int, ctypes.c_int, P, P]
        lib.sv_zero_map.argtypes = [P, ctypes.c_int, ctypes.c_int, P]
        _lib = lib
    return _lib


def default_threads() -> int:
    return os.cpu_count() or 1


def zero_state(n: int) -> np.ndarray:
    psi = np.zeros(1 << n, dtype=np.complex128)
    psi[0] = 1.0
    return psi


def apply_gate(psi: np.ndarray, n: int, U: np.ndarray, targets: Sequence[int],
               controls: Sequence[int] = (), threads: Optional[int] = None) -> None:
    lib = _load()
    assert psi.dtype == np.complex128 and psi.flags.c_contiguous and psi.size == (1 << n)
    U = np.ascontiguousarray(U, dtype=np.complex128)
    t = np.asarray(targets, dtype=np.int32)
    c = np.asarray(controls, dtype=np.int32) if len(controls) else np.zeros(1, np.int32)
    rc = lib.sv_apply(psi.ctypes.data, n, U.ctypes.data, len(targets), t.ctypes.data,
                      len(controls), c.ctypes.data, threads or default_threads())
    if rc:
        raise ValueError("sv_apply: unsupported gate arity")


def simulate_gates(n: int, gates: Sequence[Gate], order: Optional[Sequence[int]] = None,
                   psi: Optional[np.ndarray] = None, threads: Optional[int] = None) -> np.ndarray:
    psi = zero_state(n) if psi is None else psi
    idx = range(len(gates)) if order is None else order
    for i in idx:
        g = gates[i]
        apply_gate(psi, n, g.U, g.targets, g.controls, threads)
    return psi


def simulate(qasm_text: str, threads: Optional[int] = None) -> np.ndarray:
    """QASM text -> final state (program order, unpruned)."""
    n, gates = parse(qasm_text)
    return simulate_gates(n, gates, threads=threads)


def probabilities(psi: np.ndarray, n: int, qubits: Sequence[int]) -> np.ndarray:
    lib = _load()
    q = np.asarray(qubits, dtype=np.int32) if len(qubits) else np.zeros(1, np.int32)
    out = np.zeros(1 << len(qubits), dtype=np.float64)
    lib.sv_probabilities(psi.ctypes.data, n, len(qubits), q.ctypes.data, out.ctypes.data)
    return out


def zero_map(psi: np.ndarray, n: int, c: int) -> np.ndarray:
    lib = _load()
    z = np.zeros(1 << (n - c), dtype=np.uint8)
    lib.sv_zero_map(psi.ctypes.data, n, c, z.ctypes.data)
    return z.astype(bool)
