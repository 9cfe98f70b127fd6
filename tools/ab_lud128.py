"""Panel-128 lud A/B (development aid): backward error on a few sizes, then the median time of
5 factorisations at n (default 8192).  The chain is chosen at graph capture from the
environment (RODINIA_LUD128_V2=1: the round-2 panel-32 inner steps), so run it once per arm:
    python tools/ab_lud128.py; RODINIA_LUD128_V2=1 python tools/ab_lud128.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

UNC = (1, 1, 1, 1, 1, 0, 0)
arm = "v2" if os.environ.get("RODINIA_LUD128_V2") == "1" else "v3"


def backward(A, p):
    p = p.double()
    n = p.shape[0]
    L = torch.tril(p, -1) + torch.eye(n, dtype=p.dtype, device=p.device)
    U = torch.triu(p)
    Ad = torch.from_numpy(np.asarray(A, np.float64)).to(p.device)
    return float((Ad - L @ U).abs().max() / Ad.abs().max())


for n in (1, 100, 128, 129, 257, 300, 1000, 1100, 2048):
    A = synth.lud_rodinia_matrix(n)
    t = torch.from_numpy(A).cuda()
    rg.rodinia_lud(t, 128, g=UNC)
    torch.cuda.synchronize()
    print(f"[{arm}] n={n} backward {backward(A, t):.2e}", flush=True)
for n in (7, 300, 777):
    A, L0, U0 = synth.lud_integer_factors(n)
    t = torch.from_numpy(A).cuda()
    rg.rodinia_lud(t, 128, g=UNC)
    p = t.cpu().numpy().astype(np.float64)
    L = np.tril(p, -1) + np.eye(n)
    U = np.triu(p)
    print(f"[{arm}] integer n={n} exact {np.array_equal(L, L0) and np.array_equal(U, U0)}", flush=True)

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
a = A0.clone()
rg.rodinia_lud(a, 128, g=UNC)
torch.cuda.synchronize()
ts = []
for _ in range(7):
    a.copy_(A0)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    rg.rodinia_lud(a, 128, g=UNC)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
print(f"[{arm}] n={n} panel 128: median {sorted(ts)[3]:.3f} ms (all {', '.join(f'{x:.2f}' for x in ts)}) "
      f"backward(row sample) ...", flush=True)
p = a.double()
L = torch.tril(p, -1) + torch.eye(n, dtype=p.dtype, device=p.device)
U = torch.triu(p)
rows = torch.arange(0, n, 61, device=p.device)
Ad = A0.double()[rows]
print(f"[{arm}] n={n} backward(row sample) {float((Ad - L[rows] @ U).abs().max() / A0.abs().max()):.2e}", flush=True)
