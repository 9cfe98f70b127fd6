"""A/B timing of hotspot3D (development aid).  RODINIA_GRAN_LIB=<lib.so> python tools/ab_h3.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_cgo_ivanovzdem24_b200 as rg

S = rg.RODINIA_STREAM
tag = os.path.basename(os.environ.get("RODINIA_GRAN_LIB", "default"))
for (nx, ny, nz, it) in [(1024, 1024, 64, 20), (512, 512, 8, 100)]:
    T = torch.rand(nz, ny, nx, device="cuda") * 20 + 323.15
    P = torch.rand(nz, ny, nx, device="cuda") * 1e-3
    c = rg.rodinia_hotspot3d_coeffs_rodinia(nx, ny, nz)
    for g in [(2, 2, 1, 1, 1, 1, S), (4, 2, 1, 1, 1, 1, S), (2, 1, 1, 1, 1, 1, S), (4, 1, 1, 1, 1, 1, S)]:
        rg.rodinia_hotspot3d(T, P, it, coeffs=c, g=g)
        torch.cuda.synchronize()
        best = 1e30
        for _ in range(3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            rg.rodinia_hotspot3d(T, P, it, coeffs=c, g=g)
            e1.record()
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1))
        ms = best / it
        print(f"{tag:10s} {nx}x{ny}x{nz} {str(g):26s} {ms*1e3:8.1f} us/step  {12*nx*ny*nz/(ms*1e-3)/1e9:7.0f} GB/s eff", flush=True)
