"""hotspot3d 1024x1024x64 timing of the plane family (development aid)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
nz, ny, nx, it = 64, 1024, 1024, 20
T = torch.rand(nz, ny, nx, device="cuda") * 20 + 323.15
P = torch.rand(nz, ny, nx, device="cuda") * 1e-3
c = rg.rodinia_hotspot3d_coeffs_rodinia(nx, ny, nz)
out = torch.empty_like(T); scr = torch.empty_like(T)
for g in [(1, 1, 1, 1, 1, 0, 0), (2, 2, 1, 1, 1, 1, 2), (2, 1, 1, 1, 1, 1, 2), (4, 1, 1, 1, 1, 1, 2),
          (4, 2, 1, 1, 1, 1, 2), (1, 4, 1, 1, 1, 1, 2)]:
    rg.rodinia_hotspot3d(T, P, it, coeffs=c, g=g, out=out, scratch=scr); torch.cuda.synchronize()
    ts = []
    for _ in range(3):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_hotspot3d(T, P, it, coeffs=c, g=g, out=out, scratch=scr); e1.record()
        torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    ms = sorted(ts)[1]
    print(f"{str(g):26s} {ms:8.3f} ms  {12 * nx * ny * nz * it / (ms * 1e-3) / 1e9:7.0f} GB/s eff", flush=True)
