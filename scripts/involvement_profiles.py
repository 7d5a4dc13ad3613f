"""NEXT-1 diagnostics at the BASELINE configs' sizes (no GPU needed): Table II's "operations
before all qubits are involved" (reading Q17), the Fig.9-style involvement profile
(involved qubits after each operation) and the live work sum_k 2^(k_g) / (G 2^n) --
the fraction of the unpruned gate-by-gate work that pruning leaves -- for program order, Alg.2
greedy and Alg.3 forward-looking orders, under the paper's involvement rule
and the refined rule (mode + 4). The orders come from the library (qgpu_circuit_reorder) and the
traces from oracle/schedule.py; both are cross-checked on the fly.

    python scripts/involvement_profiles.py [--out profiles/r01/involvement_profiles.json]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from oracle import qasm as oq  # noqa: E402
from oracle import schedule as osch  # noqa: E402
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q  # noqa: E402
from workloads import circuits as wc  # noqa: E402

CONFIGS = [("C2 qft_28", lambda: wc.qft(28)), ("C3 qaoa_32", lambda: wc.qaoa(32, 2, seed=1)),
           ("C4 rqc_34", lambda: wc.rqc(34, 20, seed=3)), ("C5 gs_36", lambda: wc.gs(6, 6)),
           ("C5 hlf_36", lambda: wc.hlf(6, 6, seed=2)), ("grqc_32", lambda: wc.grqc(4, 8, 473, seed=5))]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--points", type=int, default=20)
    args = ap.parse_args()
    q.load()
    res = []
    for name, mk in CONFIGS:
        c = mk()
        text = c.qasm()
        n, gates = oq.parse(text)
        qc = q.Circuit(text)
        row = {"config": name, "n": n, "gates": len(gates)}
        for rule in (0, 1):
            for mode, mname in ((0, "program"), (1, "greedy"), (2, "forward")):
                order = [int(x) for x in qc.reorder(mode + 4 * rule)]
                if len(gates) <= 1500:  # the oracle replay is O(G n^2) per pick in Python
                    assert order == osch.reorder(gates, mode, rule=rule), (name, mode, rule)
                trace = osch.involvement_trace(gates, order, rule=rule)
                ks = [bin(v).count("1") for v in trace]
                live = sum(2.0 ** (k - n) for k in ks) / len(ks)
                step = max(1, len(ks) // args.points)
                key = f"{mname}{'_refined' if rule else ''}"
                row[key] = {"ops_before_full_involvement": osch.ops_before_full_involvement(gates, n, order, rule=rule),
                            "live_work": live, "profile": ks[::step] + [ks[-1]]}
        res.append(row)
        print(f"{name:12} G={len(gates):5d}  Table II program {row['program']['ops_before_full_involvement']:5d} "
              f"-> greedy {row['greedy']['ops_before_full_involvement']:5d} -> forward "
              f"{row['forward']['ops_before_full_involvement']:5d}   live work "
              f"{100 * row['program']['live_work']:5.1f}% -> {100 * row['greedy']['live_work']:5.1f}% -> "
              f"{100 * row['forward']['live_work']:5.1f}%  (refined forward {100 * row['forward_refined']['live_work']:5.1f}%)",
              flush=True)
        qc.close()
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
