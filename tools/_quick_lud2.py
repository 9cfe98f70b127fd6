import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
n = 8192
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda(); A = A0.clone()
def t(panel, g):
    A.copy_(A0); rg.rodinia_lud(A, panel, g=g); torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True); ts = []
    for _ in range(2):
        A.copy_(A0); e0.record(); rg.rodinia_lud(A, panel, g=g); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return min(ts)
for panel, V in [(16, 4), (16, 8), (32, 2), (32, 4)]:
    for by in (4, 8, 16, 32):
        g = (V, 1, 1, by, 1, 1, 2)
        print(panel, g, round(t(panel, g), 2), "ms", flush=True)
print("ref16", round(t(16, (4, 2, 2, 2, 1, 1, 0)), 2), "ref32", round(t(32, (2, 4, 4, 2, 1, 1, 0)), 2))
