import os, sys
sys.path.insert(0, "/root/repo")
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu as q
from workloads import circuits as wc
c = q.Circuit(wc.qft(28).qasm())
s = q.State(28)
s.apply_circuit(c)
print("map", list(s.qubit_map()))
for _ in range(2):
    s.probabilities(list(range(10)))
    s.probabilities([])
    s.probabilities([20, 21, 22])
