"""srad_v1 / srad_v2 C4-size timing (development aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
N, it = 8192, 100
J0 = torch.from_numpy(synth.srad_input(N, N)).cuda()
img0 = torch.from_numpy(synth.srad_v1_image(N, N)).cuda()
def t(f):
    f(); torch.cuda.synchronize(); ts = []
    for _ in range(3):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); f(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return sorted(ts)[1]
g = (4, 1, 1, 3, 1, 1, 2)
J = J0.clone(); img = img0.clone()
print("srad_v2", round(t(lambda: (J.copy_(J0), rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g))), 3), "ms")
print("srad_v1", round(t(lambda: (img.copy_(img0), rg.rodinia_srad_v1(img, 0.5, it, g=g))), 3), "ms")
print("srad_v1 unc", round(t(lambda: (img.copy_(img0), rg.rodinia_srad_v1(img, 0.5, it, g=(1, 1, 1, 1, 1, 0, 0)))), 3), "ms")
