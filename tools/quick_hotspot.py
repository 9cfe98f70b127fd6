"""Quick hotspot timing sweep on one GPU (development aid; not the bench)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg

N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 48
which = sys.argv[3] if len(sys.argv) > 3 else "all"
bys = [int(x) for x in sys.argv[4].split(",")] if len(sys.argv) > 4 else [2, 4, 8]
t = torch.rand(N, N, device="cuda") * 20 + 323.15
p = torch.rand(N, N, device="cuda") * 1e-3
c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
out = torch.empty_like(t); scr = torch.empty_like(t)
grans = []
if which in ("all", "direct"):
    grans += [(1,1,1,1,1,0,0), (4,1,1,1,1,1,0), (4,1,2,1,1,1,0), (4,1,4,1,1,1,0), (4,2,2,1,1,1,0), (4,1,2,2,1,1,0)]
if which in ("all", "stream"):
    for r in rg.rodinia_variants("hotspot"):
        g = r["g"]
        if not (g[6] & 2) or r["status"] != 0:
            continue
        for by in bys:
            grans.append((g[0], 1, 1, by, g[4], 1, g[6]))
res = []
for g in grans:
    try:
        rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g, out=out, scratch=scr)
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        ts = []
        for _ in range(3):
            e0.record(); rg.rodinia_hotspot(t, p, iters, coeffs=c, g=g, out=out, scratch=scr); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = sorted(ts)[1]
        rate = N * N * iters / (ms * 1e-3)
        res.append((rate, g, ms))
        print(f"{str(g):32s} {ms:9.3f} ms  {rate/1e9:8.1f} Gupd/s  eff {12*rate/1e9:7.0f} GB/s", flush=True)
    except Exception as e:
        print(g, "ERR", e, flush=True)
res.sort(reverse=True)
for r in res[:6]:
    print("BEST", r)
