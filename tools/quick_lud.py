import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda(); A = A0.clone()
res = []
for panel in (16, 32):
    for r in rg.rodinia_variants("lud"):
        g = r["g"]
        for bx, by in [(1, 1), (2, 1), (2, 2), (4, 1), (4, 2), (4, 4)]:
            gg = (g[0], g[1], bx, by, 1, g[5], 0)
            try:
                A.copy_(A0); rg.rodinia_lud(A, panel, g=gg); torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True); ts = []
                for _ in range(2):
                    A.copy_(A0); e0.record(); rg.rodinia_lud(A, panel, g=gg); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
                res.append((min(ts), panel, gg))
            except Exception as e:
                pass
res.sort()
for r in res[:12]: print(r)
print("uncoarsened", [r for r in res if r[2] == (1, 1, 1, 1, 1, 0, 0) and r[1] == 16])
