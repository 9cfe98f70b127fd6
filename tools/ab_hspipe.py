"""hs_pipe (one-sided halo pipeline) vs hs_stream: bitwise equality on ragged shapes, then timing
(development aid).  python tools/ab_hspipe.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_cgo_ivanovzdem24_b200 as rg

S, P = rg.RODINIA_STREAM, 8
OCC10 = 10 << 8
for (R, C, it) in [(300, 700, 24), (1000, 1537, 40), (64, 64, 9), (4096, 4096, 16), (997, 4099, 17)]:
    T = torch.rand(R, C, device="cuda") * 20 + 323.15
    Pw = torch.rand(R, C, device="cuda") * 1e-3
    c = rg.rodinia_hotspot_coeffs_rodinia(R, C, R * 31.25e-6, C * 31.25e-6)
    ref = rg.rodinia_hotspot(T, Pw, it, coeffs=c, g=(4, 1, 1, 4, 8, 1, S | OCC10))
    for W in (2, 5):
        got = rg.rodinia_hotspot(T, Pw, it, coeffs=c, g=(4, 1, W, 4, 8, 1, S | P | OCC10))
        torch.cuda.synchronize()
        print(f"{R}x{C}x{it} W={W} bitwise {bool(torch.equal(got, ref))} maxdiff {float((got - ref).abs().max()):.3e}",
              flush=True)
N = 16384
t = torch.rand(N, N, device="cuda") * 20 + 323.15
p = torch.rand(N, N, device="cuda") * 1e-3
c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
out = torch.empty_like(t)
scr = torch.empty_like(t)
grans = [(4, 1, 1, 12, 8, 1, S | OCC10), (4, 1, 5, 12, 8, 1, S | P | OCC10), (4, 1, 5, 8, 8, 1, S | P | OCC10),
         (4, 1, 5, 16, 8, 1, S | P | OCC10), (4, 1, 2, 12, 8, 1, S | P | OCC10)]
for rep in range(2):
    for g in grans:
        rg.rodinia_hotspot(t, p, 200, coeffs=c, g=g, out=out, scratch=scr)
        torch.cuda.synchronize()
        best = 1e30
        for _ in range(3):
            rg.rodinia_kernel_timing(True)
            rg.rodinia_hotspot(t, p, 200, coeffs=c, g=g, out=out, scratch=scr)
            torch.cuda.synchronize()
            ms, n = rg.rodinia_kernel_time()
            rg.rodinia_kernel_timing(False)
            best = min(best, ms / max(n, 1))
        print(f"{str(g):34s} {best:.4f} ms/launch  {N * N * 8 / (best * 1e-3) / 1e12:.3f} T upd/s", flush=True)
