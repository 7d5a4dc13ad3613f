import sys, numpy as np, torch
sys.path.insert(0,'.')
sys.path.insert(0,"tests")
from test_gpu_gfc import gpu_compress
from paper_conf_hpca_zhaogydmuzjyt22_b200 import qgpu
from oracle import gfc
from workloads import circuits as wc
env=(torch,qgpu,gfc)
with qgpu.State(22) as s:
    s.apply_circuit(qgpu.Circuit(wc.qaoa(22,2,seed=1).qasm()))
    psi=s.amplitudes()
seg=4096
stream,off=gpu_compress(env,psi,seg)
words=psi.view(np.float64)
nseg=len(off)-1
bad=0
for sidx in range(0,nseg,97):
    ref=gfc.encode_segment(gfc.as_words(words[sidx*seg:(sidx+1)*seg]))
    got=stream[int(off[sidx]):int(off[sidx+1])]
    if ref!=got:
        bad+=1
        i=next((k for k in range(min(len(ref),len(got))) if ref[k]!=got[k]), None)
        print("seg",sidx,"len ref",len(ref),"got",len(got),"first diff",i, ref[i-4:i+8].hex() if i else None, got[i-4:i+8].hex() if i else None)
        if bad>4: break
print("bad",bad)
