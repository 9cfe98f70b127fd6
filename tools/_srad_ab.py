"""srad C4 timing of a few stream granularities (A/B development aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
N, it = 8192, 100
J0 = torch.from_numpy(synth.srad_input(N, N)).cuda()
J = J0.clone()
tag = os.path.basename(os.environ.get("RODINIA_GRAN_LIB", "default"))
for g in [(4, 1, 1, 2, 1, 1, 2), (4, 1, 1, 2, 1, 1, 4098), (4, 1, 1, 3, 1, 1, 2), (4, 1, 1, 3, 1, 1, 4098)]:
    J.copy_(J0); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); torch.cuda.synchronize()
    ts = []
    for _ in range(3):
        J.copy_(J0)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{tag:24s} {str(g):24s} {sorted(ts)[1]:8.3f} ms", flush=True)
