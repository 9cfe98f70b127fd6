"""Panel-16/32 lud timing of selected granularities (development aid).
  python tools/ab_lud16.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
S = rg.RODINIA_STREAM
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
A = A0.clone()
cases = [(16, (4, 2, 2, 2, 1, 1, 0))] + [(16, (v, 1, 1, by, 1, 1, S)) for v in (4, 8) for by in (2, 4, 8, 16)] + \
        [(32, (4, 8, 2, 1, 1, 1, 0))] + [(32, (v, 1, 1, by, 1, 1, S)) for v in (2, 4) for by in (2, 4, 8)]
ref = {}
for panel, g in cases:
    A.copy_(A0)
    rg.rodinia_lud(A, panel, g=g)
    torch.cuda.synchronize()
    if panel not in ref:
        ref[panel] = A.clone()
    same = bool(torch.equal(A, ref[panel]))
    ts = []
    for _ in range(3):
        A.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        rg.rodinia_lud(A, panel, g=g)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"panel {panel} {str(g):32s} {min(ts):8.2f} ms  bitwise-equal-to-first {same}", flush=True)
