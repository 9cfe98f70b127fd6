"""A/B timing of hotspot stepping launches (development aid; not the bench).

  RODINIA_GRAN_LIB=<lib.so> python tools/ab_hotspot.py [N] [iters] [g,g,...]
Prints the event-timed average duration of the stepping launches (rodinia_kernel_time) for
each granularity, so the state-conversion passes are excluded.
"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg

N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 200
grans = [tuple(int(x) for x in g.split(",")) for g in sys.argv[3].split(";")] if len(sys.argv) > 3 else \
    [(4, 1, 1, by, 8, 1, occ) for by in (6, 12) for occ in (2562, 3074)]
t = torch.rand(N, N, device="cuda") * 20 + 323.15
p = torch.rand(N, N, device="cuda") * 1e-3
c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
out = torch.empty_like(t); scr = torch.empty_like(t)
tag = os.path.basename(os.environ.get("RODINIA_GRAN_LIB", "default"))
for g in grans:
    rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g, out=out, scratch=scr)
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(3):
        rg.rodinia_kernel_timing(True)
        rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g, out=out, scratch=scr)
        torch.cuda.synchronize()
        ms, n = rg.rodinia_kernel_time()
        rg.rodinia_kernel_timing(False)
        best = min(best, ms / max(n, 1))
    h = g[4]
    rate = N * N * h / (best * 1e-3)
    print(f"{tag:24s} {str(g):30s} {best:8.4f} ms/launch  {rate/1e12:6.3f} T upd/s", flush=True)
