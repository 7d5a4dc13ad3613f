"""Test helper (uses only oracle/): sampled amplitudes of "product state + a few gates" at any n.

The state prod_q v_q (v_q = factors[q], the 2-vector U_q|0>) followed by `gates` (matrix,
targets, controls) that act on a small qubit set A equals (prod_{q not in A} v_q) (x) phi_A with
phi_A = the gates applied to the |A|-qubit product state. So amplitude i is
    prod_{q not in A} v_q[bit_q(i)] * phi_A[bits_A(i)],
phi_A from the oracle's plain simulation (Eq.8). Pinned against the oracle's full
simulation by tests/test_oracle_pins.py::test_light_cone_helper_matches_full_simulation.
"""
import numpy as np

from oracle import statevector as osv


def product_light_cone(n, factors, gates, idx):
    A = sorted({q for U, t, cs in gates for q in list(t) + list(cs)})
    loc = {q: j for j, q in enumerate(A)}
    phi = np.zeros(1 << len(A), dtype=np.complex128)
    for y in range(1 << len(A)):
        v = 1.0 + 0j
        for j, q in enumerate(A):
            v *= factors[q][(y >> j) & 1]
        phi[y] = v
    for U, t, cs in gates:
        osv.apply_gate(phi, len(A), U, [loc[x] for x in t], [loc[x] for x in cs], threads=1)
    idx = np.asarray(idx, dtype=np.int64)
    out = np.ones(len(idx), dtype=np.complex128)
    for q in range(n):
        if q in loc:
            continue
        out *= np.where((idx >> q) & 1, factors[q][1], factors[q][0])
    y = np.zeros(len(idx), dtype=np.int64)
    for j, q in enumerate(A):
        y |= ((idx >> q) & 1) << j
    return out * phi[y]
