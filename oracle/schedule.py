"""ORACLE (test infrastructure only) -- replay of the paper's scheduling algorithms.

Written step by step in the paper's order and notation (§IV-B, §IV-C):

* ``involvement`` flags and Algorithm 1 (pruning zero state amplitudes).
* ``getChunkSize`` -- reading Q1: number of trailing 1-bits of involvement
  ("least non-zero bit"; the worked example 00000011 -> 2).
* the fixed-chunk-size bitmap, bit j = ((j << c) & ~involvement) == 0.
* the dependency DAG (reading Q5: one edge per distinct most-recent predecessor on
  each operand qubit), Algorithm 2 greedy reorder and Algorithm 3
  forward-looking reorder, with the deterministic tie-break of reading Q4
  (the paper breaks ties at random) and the +inf initialisation of Q3.
* Table II statistic: number of operations strictly before all qubits are involved (Q17).

"Involve" uses the paper's rule (reading Q7) by default: every operand qubit, targets and
controls, of every gate, diagonal or not (P:223, P:229 l.11). ``rule=1`` is the refined rule of
SURVEY §8f NEXT-1, read off P:221 ("if a qubit is not involved ... the amplitudes with that bit
set are zero"): on such a state a gate with a control on an uninvolved qubit is the identity,
and a diagonal gate maps every zero amplitude to zero, so neither involves anything; every other
gate involves all its operands. Alg.2/3 then count the new qubits a gate would involve under
the same rule.
"""
from __future__ import annotations

import math
from typing import List, Optional, Sequence, Set, Tuple

import numpy as np


def gate_qubits(g) -> Tuple[int, ...]:
    """Qubits an operation acts on (targets and controls), accepts oracle Gate or tuple."""
    if hasattr(g, "qubits"):
        return tuple(g.qubits)
    return tuple(g)


def qubit_mask(qs: Sequence[int]) -> int:
    m = 0
    for q in qs:
        m |= 1 << q
    return m


# ----------------------------------------------------------------------------- Algorithm 1

def get_chunk_size(involvement: int) -> int:
    """Reading Q1: index of the lowest 0 bit = count of trailing ones (00000011 -> 2)."""
    cs = 0
    while (involvement >> cs) & 1:
        cs += 1
    return cs


def alg1_chunks(involvement: int, n: int) -> Tuple[int, List[int]]:
    """Algorithm 1 lines 1-8: the chunks whose amplitudes are updated.

    Returns (chunkSize, processed chunk indices). N = 2^(n - chunkSize) chunks.
    """
    chunk_size = get_chunk_size(involvement)
    N = 1 << (n - chunk_size) if chunk_size <= n else 1
    processed = []
    for iChunk in range(N):
        iChunk_p = iChunk << chunk_size           # line 4
        if iChunk_p > involvement:                # line 5
            break                                 # line 6
        if iChunk_p & involvement != iChunk_p:    # line 7
            continue                              # line 8
        processed.append(iChunk)                  # line 10: amplitudes update
    return chunk_size, processed


def is_diagonal(U) -> bool:
    """Every off-diagonal entry exactly zero."""
    U = np.asarray(U)
    return bool(np.all(U[~np.eye(U.shape[0], dtype=bool)] == 0))


def involved_by(g, involvement: int, rule: int = 0) -> Tuple[int, ...]:
    """The qubits gate g involves when executed after ``involvement`` (bit mask).
    rule 0: all operands (Q7). rule 1 (NEXT-1): none if a control is uninvolved or g is
    diagonal, else all operands."""
    qs = gate_qubits(g)
    if rule == 0:
        return qs
    if any(not (involvement >> c) & 1 for c in g.controls):
        return ()
    if is_diagonal(g.U):
        return ()
    return qs


def update_involvement(involvement: int, qubits: Sequence[int]) -> int:
    """Algorithm 1 line 11: set the bits of the qubits this operation involves."""
    for q in qubits:
        involvement |= 1 << q
    return involvement


def chunk_bitmap(involvement: int, n: int, c: int) -> List[int]:
    """Fixed chunk size c: bit j is 1 iff chunk j (indices [j 2^c, (j+1) 2^c)) may be non-zero,
    i.e. every set bit of (j << c) is an involved qubit."""
    full = (1 << n) - 1
    return [1 if ((j << c) & ~involvement & full) == 0 else 0 for j in range(1 << (n - c))]


def bitmap_words(bits: Sequence[int]) -> List[int]:
    """Pack a bitmap into uint64 words, bit j -> word j//64, bit j%64."""
    words = [0] * max(1, (len(bits) + 63) // 64)
    for j, b in enumerate(bits):
        if b:
            words[j >> 6] |= 1 << (j & 63)
    return words


def involvement_trace(gates: Sequence, order: Optional[Sequence[int]] = None,
                      rule: int = 0) -> List[int]:
    """involvement after each executed operation (P:229 l.11)."""
    order = range(len(gates)) if order is None else order
    inv, out = 0, []
    for i in order:
        inv = update_involvement(inv, involved_by(gates[i], inv, rule))
        out.append(inv)
    return out


def ops_before_full_involvement(gates: Sequence, n: int,
                                order: Optional[Sequence[int]] = None, rule: int = 0) -> int:
    """Table II, reading Q17: number of operations strictly before the first op
    after which all n qubits are involved (len(order) if never)."""
    full = (1 << n) - 1
    for k, inv in enumerate(involvement_trace(gates, order, rule)):
        if inv == full:
            return k
    return len(gates) if order is None else len(order)


# ----------------------------------------------------------------------------- DAG

class DAG:
    """Nodes are gate indices. One edge per distinct predecessor: the most recent earlier
    gate on each of the gate's qubits (reading Q5)."""

    def __init__(self, gates: Sequence):
        self.n = len(gates)
        self.qubits = [gate_qubits(g) for g in gates]
        self.preds: List[Set[int]] = [set() for _ in range(self.n)]
        self.desc: List[List[int]] = [[] for _ in range(self.n)]
        last = {}
        for i, qs in enumerate(self.qubits):
            for q in qs:
                if q in last:
                    self.preds[i].add(last[q])
            for q in qs:
                last[q] = i
        for i in range(self.n):
            for p in self.preds[i]:
                self.desc[p].append(i)
        for p in range(self.n):
            self.desc[p].sort()              # ascending program index (reading Q4)

    def num_predecessors(self) -> List[int]:
        return [len(p) for p in self.preds]


def _new_qubits(qs: Sequence[int], involved: Set[int]) -> int:
    return sum(1 for q in set(qs) if q not in involved)


def _involves(gates: Sequence, g: int, involved: Set[int], rule: int) -> Tuple[int, ...]:
    """Operands gate g would involve given the involved set (rule 0: all of them)."""
    if rule == 0:
        return tuple(gate_qubits(gates[g]))
    return involved_by(gates[g], qubit_mask(involved), rule)


def reorder_greedy(gates: Sequence, forced: Sequence[int] = (), rule: int = 0) -> List[int]:
    """Algorithm 2. Cost = number of new qubits the gate involves. Ties: first in
    exeList (reading Q4). ``forced`` pins the first picks (to reproduce the paper's random
    picks g1,g3,g5,g2 in the gs_5 walk-through)."""
    dag = DAG(gates)
    npred = dag.num_predecessors()
    gates_list: List[int] = []                               # line 1
    exe_list = [i for i in range(dag.n) if npred[i] == 0]    # lines 2-6
    involved: Set[int] = set()
    forced = list(forced)
    while exe_list:                                          # line 8
        next_gate, min_cost = None, math.inf                 # lines 9-10 (Q3: +inf)
        if forced:
            next_gate = forced.pop(0)
            assert next_gate in exe_list, "forced pick must be ready"
        else:
            for g in exe_list:                               # line 11
                cost = _new_qubits(_involves(gates, g, involved, rule), involved)  # line 12
                if cost < min_cost:                          # line 13
                    min_cost, next_gate = cost, g            # lines 14-15
        exe_list.remove(next_gate)                           # line 16
        gates_list.append(next_gate)                         # line 17
        involved.update(_involves(gates, next_gate, involved, rule))
        for g in dag.desc[next_gate]:                        # line 18
            npred[g] -= 1                                    # line 19
            if npred[g] == 0:                                # line 20
                exe_list.append(g)                           # line 21
    return gates_list


def forward_cost(g: int, dag: DAG, npred: List[int], exe_list: List[int],
                 involved: Set[int], gates: Sequence = (), rule: int = 0) -> Tuple[int, int]:
    """Algorithm 3 on copies of exeList / involvedQubits. Returns
    (cost, costCurrent). Under rule 1 a gate's qubits are those it would involve."""
    qubits = (lambda h, inv: dag.qubits[h]) if rule == 0 else \
        (lambda h, inv: _involves(gates, h, inv, rule))
    involved = set(involved)                      # copies
    exe_list = list(exe_list)
    cost_current, cost_look_ahead = 0, math.inf   # line 1 (Q3: look-ahead starts at +inf)
    for q in set(qubits(g, involved)):            # lines 3-6
        if q not in involved:
            cost_current += 1
            involved.add(q)
    exe_list.remove(g)                            # line 7
    for d in dag.desc[g]:                         # lines 8-10
        if npred[d] == 1:
            exe_list.append(d)
    for g2 in exe_list:                           # lines 12-18
        cur = 0
        for q in set(qubits(g2, involved)):
            if q not in involved:
                cur += 1
        if cur < cost_look_ahead:
            cost_look_ahead = cur
    if cost_look_ahead == math.inf:               # empty look-ahead set (Q3)
        cost_look_ahead = 0
    return cost_current + cost_look_ahead, cost_current   # line 19


def reorder_forward(gates: Sequence, rule: int = 0) -> List[int]:
    """Forward-looking reorder: Algorithm 2's traversal with Algorithm 3's cost; the
    minimum of the key (cost, costCurrent, position in exeList) wins (reading Q4)."""
    dag = DAG(gates)
    npred = dag.num_predecessors()
    gates_list: List[int] = []
    exe_list = [i for i in range(dag.n) if npred[i] == 0]
    involved: Set[int] = set()
    while exe_list:
        best, best_key = None, None
        for pos, g in enumerate(exe_list):
            cost, cur = forward_cost(g, dag, npred, exe_list, involved, gates, rule)
            key = (cost, cur, pos)
            if best_key is None or key < best_key:
                best, best_key = g, key
        exe_list.remove(best)
        gates_list.append(best)
        involved.update(_involves(gates, best, involved, rule))
        for d in dag.desc[best]:
            npred[d] -= 1
            if npred[d] == 0:
                exe_list.append(d)
    return gates_list


def reorder(gates: Sequence, mode: int, rule: int = 0) -> List[int]:
    """mode 0: program order, 1: greedy (Alg.2), 2: forward-looking (Alg.3)."""
    if mode == 0:
        return list(range(len(gates)))
    if mode == 1:
        return reorder_greedy(gates, rule=rule)
    if mode == 2:
        return reorder_forward(gates, rule)
    raise ValueError(mode)


def is_topological(gates: Sequence, order: Sequence[int]) -> bool:
    dag = DAG(gates)
    pos = {g: k for k, g in enumerate(order)}
    if sorted(order) != list(range(len(gates))):
        return False
    return all(pos[p] < pos[i] for i in range(dag.n) for p in dag.preds[i])
