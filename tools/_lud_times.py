import sys, os
sys.path.insert(0, "/root/repo")
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
n = 8192
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
for panel, g in ((128, (1,1,1,1,1,0,0)), (32, (4,4,2,2,1,1,0)), (16, (4,2,2,2,1,1,0)), (16, (1,1,1,1,1,0,0))):
    a = A0.clone(); rg.rodinia_lud(a, panel, g=g); torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        a.copy_(A0)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_lud(a, panel, g=g); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(panel, g, round(sorted(ts)[2], 3), "ms", flush=True)
