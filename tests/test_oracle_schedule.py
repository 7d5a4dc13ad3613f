"""Pins for the oracle's replay of Algorithms 1-3 (§IV-B/§IV-C)."""
import json
import os

import numpy as np
import pytest

from oracle import qasm as oq
from oracle import schedule as os_
from oracle import statevector as osv
from workloads import circuits as wc

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _gs5():
    g = json.load(open(os.path.join(GOLDEN, "gs5_walkthrough.json")))
    gates = [tuple(t) + tuple(c) for t, c in g["gates"]]
    return g, gates


def test_get_chunk_size_paper_example():
    g = json.load(open(os.path.join(GOLDEN, "alg1_examples.json")))
    for ex in g["getChunkSize"]:
        assert os_.get_chunk_size(int(ex["involvement"], 2)) == ex["chunkSize"]


def test_chunk_count_paper_example():
    """34 qubits, 2^21-amplitude chunks -> 8192 chunks; 16 B per amplitude."""
    g = json.load(open(os.path.join(GOLDEN, "alg1_examples.json")))["chunk_count"]
    assert 1 << (g["n"] - g["chunk_amplitudes_log2"]) == g["n_chunks"]
    assert len(os_.chunk_bitmap((1 << 34) - 1, 34, 21)) == 8192
    # 496 chunks of 2^21 * 16 B = 32 MiB = 15.5 GiB fit in a 16 GiB P100
    assert 496 * (1 << 21) * g["bytes_per_amplitude"] <= 16 * 2**30


@pytest.mark.parametrize("inv,cs,chunks", [
    (0b00000011, 2, [0]),
    (0b00100111, 3, [0, 4]),
    (0b10110111, 3, [0, 2, 4, 6, 16, 18, 20, 22]),
    (0b00000000, 0, [0]),
    (0b11111111, 8, [0]),
])
def test_alg1_hand_values(inv, cs, chunks):
    got_cs, got = os_.alg1_chunks(inv, 8)
    assert (got_cs, got) == (cs, chunks)


def test_alg1_processes_exactly_the_nonzero_support():
    """with m uninvolved qubits exactly 2^(n-m) amplitudes may be non-zero; Alg.1's
    processed chunks cover exactly {i : i & ~involvement == 0} (brute force, all 8-bit I)."""
    n = 8
    for inv in range(1 << n):
        cs, ch = os_.alg1_chunks(inv, n)
        covered = {(j << cs) + k for j in ch for k in range(1 << cs)}
        support = {i for i in range(1 << n) if i & ~inv == 0}
        assert covered == support
        assert len(covered) == 1 << bin(inv).count("1")


def test_bitmap_definition_vs_bruteforce():
    n, c = 9, 3
    for inv in [0, 1, 0b101, 0b110010111, (1 << n) - 1, 0b100000000]:
        bm = os_.chunk_bitmap(inv, n, c)
        for j in range(1 << (n - c)):
            may = any(((i & ~inv) == 0) for i in range(j << c, (j + 1) << c))
            assert bm[j] == int(may)


def test_gs5_original_greedy_forward():
    """P:239 baseline 1,2,3,4,5,5,5,5,5; P:286 greedy 1,2,3,4,4,4,5,5,5 (paper's random picks
    g1,g3,g5,g2); P:336 forward-looking 1,2,2,3,3,4,4,4,5."""
    g, gates = _gs5()
    cnt = lambda order: [bin(i).count("1") for i in os_.involvement_trace(gates, order)]
    assert cnt(None) == g["original_involved_counts"]
    gr = os_.reorder_greedy(gates, forced=g["greedy_forced_picks"])
    assert cnt(gr) == g["greedy_involved_counts"]
    fw = os_.reorder_forward(gates)
    assert cnt(fw) == g["forward_involved_counts"]
    for o in (gr, fw):
        assert os_.is_topological(gates, o)


@pytest.mark.parametrize("seed", range(6))
def test_reorder_is_topological_and_exact(seed):
    """reorder obeys dependencies and does not change results."""
    c = wc.random_circuit(7, 60, seed=seed)
    n, gates = oq.parse(c.qasm())
    ref = osv.simulate_gates(n, gates)
    for mode in (1, 2):
        order = os_.reorder(gates, mode)
        assert os_.is_topological(gates, order)
        psi = osv.simulate_gates(n, gates, order=order)
        assert np.abs(psi - ref).max() < 1e-12


@pytest.mark.parametrize("fam", ["qft", "gs", "hlf", "random"])
def test_pruning_soundness(fam):
    """after every step of a schedule, every bitmap-0 chunk is exactly zero in the
    unpruned state evolved along the same schedule."""
    c = {"qft": lambda: wc.qft(9), "gs": lambda: wc.gs(3, 3), "hlf": lambda: wc.hlf(3, 3, 2),
         "random": lambda: wc.random_circuit(9, 40, seed=2)}[fam]()
    n, gates = oq.parse(c.qasm())
    for mode in (0, 2):
        order = os_.reorder(gates, mode)
        psi = osv.zero_state(n)
        inv = 0
        for i in order:
            g = gates[i]
            osv.apply_gate(psi, n, g.U, g.targets, g.controls)
            inv = os_.update_involvement(inv, g.qubits)
            for cb in (0, 2, 4):
                bm = np.array(os_.chunk_bitmap(inv, n, cb), dtype=bool)
                z = osv.zero_map(psi, n, cb)
                assert np.all(z[~bm])


def test_forward_reorder_delays_involvement_on_qft():
    """Fig.9: forward-looking reordering delays involvement on qft."""
    n, gates = oq.parse(wc.qft(12).qasm())
    base = os_.ops_before_full_involvement(gates, n)
    fw = os_.ops_before_full_involvement(gates, n, os_.reorder_forward(gates))
    assert fw > base


# ------------------------------------------------------------- refined involvement (NEXT-1)

def _g(name, qubits, params=()):
    text = 'OPENQASM 2.0;\ninclude "qelib1.inc";\nqreg q[4];\n'
    p = f"({','.join(str(x) for x in params)})" if params else ""
    text += f"{name}{p} " + ",".join(f"q[{q}]" for q in qubits) + ";\n"
    return oq.parse(text)[1][0]


def test_refined_rule_hand_cases():
    """NEXT-1 / P:221: on a state where qubit q is |0> everywhere, a gate controlled by q is the
    identity and a diagonal gate leaves the zeros zero: neither involves anything."""
    assert os_.involved_by(_g("cp", [0, 1], [0.3]), 0, 1) == ()        # both uninvolved
    assert os_.involved_by(_g("cx", [0, 1]), 0, 1) == ()               # control uninvolved
    assert set(os_.involved_by(_g("cx", [0, 1]), 0b01, 1)) == {0, 1}   # control involved: X moves
    assert os_.involved_by(_g("rz", [2], [0.7]), 0, 1) == ()           # diagonal: a phase
    assert os_.involved_by(_g("cz", [0, 1]), 0b11, 1) == ()            # diagonal on involved
    assert set(os_.involved_by(_g("h", [3]), 0, 1)) == {3}
    assert set(os_.involved_by(_g("swap", [0, 1]), 0, 1)) == {0, 1}    # non-diagonal: all
    for g in (_g("cp", [0, 1], [0.3]), _g("cx", [0, 1]), _g("rz", [2], [0.7])):
        assert set(os_.involved_by(g, 0, 0)) == set(g.qubits)          # the paper's rule Q7


def test_refined_rule_qft_on_zero_is_hadamards_only():
    """QFT|0...0> = H^n up to the final SWAP layer: every CP meets an uninvolved control or
    target-side |0>, so under rule 1 only the H gates (and SWAPs of involved qubits) involve."""
    n, gates = oq.parse(wc.qft(8).qasm())
    trace = os_.involvement_trace(gates, rule=1)
    inv = 0
    for g, t in zip(gates, trace):
        if g.name == "h":
            inv |= 1 << g.targets[0]
        assert t == inv
    assert os_.ops_before_full_involvement(gates, n, rule=1) < len(gates)


@pytest.mark.parametrize("fam", ["qft0", "random", "randdiag", "qaoa"])
def test_refined_rule_pruning_soundness(fam):
    """P:221 under the refined rule: after every step of a schedule (program order and the
    refined Alg.2/3 orders), every bitmap-0 chunk is exactly zero in the unpruned state evolved
    along that schedule. A rule that skipped involving a qubit a gate can make non-zero fails."""
    c = {"qft0": lambda: wc.qft(8), "random": lambda: wc.random_circuit(8, 60, seed=3),
         "randdiag": lambda: wc.random_circuit(8, 60, seed=4,
                                               names=["cp", "cz", "rz", "cx", "crx", "ccx", "t", "h", "rzz", "cswap"]),
         "qaoa": lambda: wc.qaoa(8, 1, seed=2)}[fam]()
    n, gates = oq.parse(c.qasm())
    ref = osv.simulate_gates(n, gates)
    for mode in (0, 1, 2):
        order = os_.reorder(gates, mode, rule=1)
        assert os_.is_topological(gates, order)
        psi = osv.zero_state(n)
        inv = 0
        for i in order:
            g = gates[i]
            osv.apply_gate(psi, n, g.U, g.targets, g.controls)
            inv = os_.update_involvement(inv, os_.involved_by(g, inv, 1))
            for cb in (0, 2, 4):
                bm = np.array(os_.chunk_bitmap(inv, n, cb), dtype=bool)
                z = osv.zero_map(psi, n, cb)
                assert np.all(z[~bm])
        assert np.abs(psi - ref).max() < 1e-12


def test_refined_rule_delays_involvement_at_least_as_much():
    """The refined involved set is a subset of the paper's after every step of the same order."""
    for seed in range(4):
        n, gates = oq.parse(wc.random_circuit(9, 80, seed=seed).qasm())
        a = os_.involvement_trace(gates, rule=0)
        b = os_.involvement_trace(gates, rule=1)
        assert all((y & ~x) == 0 for x, y in zip(a, b))


# ------------------------------------------------------ pins of the soundness-check helpers

def test_zero_map_hand_states():
    """sv_zero_map (the data zero map of the pruning-soundness checks) on hand-built
    states whose map is obvious: z[j] = 1 iff every amplitude of chunk j is exactly 0.0.
    A map that wrongly reports "all zero" would make every soundness check vacuous."""
    n, c = 4, 2                                        # 4 chunks of 4 amplitudes
    psi = np.zeros(1 << n, dtype=np.complex128)
    psi[7] = 1e-300                                    # the LAST slot of chunk 1
    psi[8] = complex(-0.0, -0.0)                       # -0.0 is zero (chunk 2 stays zero)
    psi[12] = complex(0.0, 5e-324)                     # a denormal imaginary part is non-zero
    assert osv.zero_map(psi, n, c).tolist() == [True, False, True, False]
    psi[0] = complex(0.0, -2.0)                        # the FIRST slot, imaginary only
    assert osv.zero_map(psi, n, c).tolist() == [False, False, True, False]
    # c = 0: every amplitude is its own chunk
    z0 = osv.zero_map(psi, n, 0)
    assert z0.tolist() == [not (x.real != 0.0 or x.imag != 0.0) for x in psi]
    assert z0.sum() == 16 - 3
    # c = n: one chunk covering the whole state
    assert osv.zero_map(psi, n, n).tolist() == [False]
    assert osv.zero_map(np.zeros(1 << n, np.complex128), n, n).tolist() == [True]
    neg = np.full(1 << n, complex(-0.0, -0.0))
    assert osv.zero_map(neg, n, 1).tolist() == [True] * 8


def test_zero_map_sees_the_nonzero_support():
    """After H on qubits {0, 2} of |0000>, exactly the indices with bits 1 and 3 clear are
    non-zero: with c = 1 the chunks j with (j << 1) & 0b1010 == 0 are the non-zero ones."""
    n, c = 4, 1
    psi = osv.zero_state(n)
    H = np.array([[1, 1], [1, -1]]) / np.sqrt(2)
    for q in (0, 2):
        osv.apply_gate(psi, n, H, [q])
    z = osv.zero_map(psi, n, c)
    assert z.tolist() == [((j << c) & 0b1010) != 0 for j in range(1 << (n - c))]


def test_ops_before_full_involvement_gs5():
    """Table II statistic (reading Q17) fixed by the three published gs_5 profiles:
    4 operations before full involvement in program order, 6 with the paper's greedy
    picks, 8 with forward-looking reordering."""
    g, gates = _gs5()
    want = g["ops_before_full_involvement"]
    assert os_.ops_before_full_involvement(gates, 5) == want["original"] == 4
    gr = os_.reorder_greedy(gates, forced=g["greedy_forced_picks"])
    assert os_.ops_before_full_involvement(gates, 5, gr) == want["greedy"] == 6
    fw = os_.reorder_forward(gates)
    assert os_.ops_before_full_involvement(gates, 5, fw) == want["forward"] == 8


def test_ops_before_full_involvement_edge_cases():
    """The first op involves everything -> 0; full involvement never reached -> the number of
    operations; reached by the last op -> len - 1 (off-by-one checks of reading Q17)."""
    one = [(0, 1, 2)]                                         # ccx-like: all 3 qubits at once
    assert os_.ops_before_full_involvement(one, 3) == 0
    never = [(0,), (1,), (0, 1)]
    assert os_.ops_before_full_involvement(never, 3) == 3          # qubit 2 never touched
    last = [(0,), (1,), (2,)]
    assert os_.ops_before_full_involvement(last, 3) == 2
    assert os_.ops_before_full_involvement(last, 3, order=[2, 1, 0]) == 2
    assert os_.ops_before_full_involvement(last, 2) == 1           # n = 2: q2 is outside
