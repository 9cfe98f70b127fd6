"""A/B timing of srad_v1 at 8192^2 x 100 (development aid; not the bench).
  RODINIA_GRAN_LIB=<lib.so> python tools/ab_srad_v1.py [g;g;...]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

grans = [tuple(int(x) for x in g.split(",")) for g in sys.argv[1].split(";")] if len(sys.argv) > 1 else \
    [(4, 1, 1, 3, 1, 1, 2), (1, 1, 1, 1, 1, 0, 0)]
N, it = 8192, 100
I0 = torch.from_numpy(synth.srad_v1_image(N, N)).cuda()
I = I0.clone()
tag = os.path.basename(os.environ.get("RODINIA_GRAN_LIB", "default"))
for g in grans:
    I.copy_(I0); rg.rodinia_srad_v1(I, 0.5, it, g=g); torch.cuda.synchronize()
    ts = []
    for _ in range(3):
        I.copy_(I0)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_srad_v1(I, 0.5, it, g=g); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{tag:14s} {str(g):26s} {statistics.median(ts):8.3f} ms", flush=True)
