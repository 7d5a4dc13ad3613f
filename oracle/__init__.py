"""ORACLE -- test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what the Q-GPU hot path computes
(Zhao et al., HPCA'22, /root/reference/PAPER.md, cited as P:<line>). It exists to check the
CUDA path; it is NOT a fallback. Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import or execute anything
under ``oracle/``. It shares no code with ``paper_conf_hpca_zhaogydmuzjyt22_b200`` (own QASM
parser, own gate table, own index arithmetic, own scheduler replay); the only common input is
the QASM text produced by ``workloads/``.

Modules
  qasm.py        OpenQASM-2 subset parser + gate table
  sv.c           state-vector update loops in plain C (Eq.8) and readout
  statevector.py ctypes wrapper around sv.c, program-order simulation
  schedule.py    Alg.1 pruning replay, Alg.2 greedy and Alg.3 forward-looking reorder,
                 chunk bitmap, Table II statistic
  gfc.py         GFC-style lossless compression of amplitude doubles, segment/micro-chunk
                 residual coding with 4-bit sign + leading-zero-byte prefixes

Parity status: every function is pinned by tests in tests/test_oracle_*.py (closed forms,
brute-force unitaries, the paper's worked examples); see DESIGN.md "Oracle pins".
"""
