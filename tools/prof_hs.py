"""Run one hotspot solve (16384^2 by default) with a given granularity: target for ncu captures."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
g = tuple(int(x) for x in sys.argv[1].split(","))
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 48
N = int(sys.argv[3]) if len(sys.argv) > 3 else 16384
t = torch.rand(N, N, device="cuda") * 20 + 323.15
p = torch.rand(N, N, device="cuda") * 1e-3
c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
out = torch.empty_like(t); scr = torch.empty_like(t)
rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g, out=out, scratch=scr)
torch.cuda.synchronize()
