"""Quick srad timing sweep on one GPU (development aid; not the bench)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

N = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
it = int(sys.argv[2]) if len(sys.argv) > 2 else 20
J0 = torch.from_numpy(synth.srad_input(N, N)).cuda()
J = J0.clone()
grans = [(1,1,1,1,1,0,0), (2,1,4,2,1,0,0), (2,1,4,2,1,1,0)]
for v in (1, 2, 4, 8):
    for bx in (1, 2):
        for by in (1, 2, 3, 4, 8):
            grans.append((v, 1, bx, by, 1, 1, 2))
res = []
for g in grans:
    try:
        J.copy_(J0); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); torch.cuda.synchronize()
        ts = []
        for _ in range(3):
            J.copy_(J0)
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = sorted(ts)[1]
        rate = N * N * it / (ms * 1e-3)
        res.append((rate, g, ms))
        print(f"{str(g):28s} {ms:9.3f} ms {rate/1e9:8.1f} Gupd/s  eff {8*rate/1e9:7.0f} GB/s", flush=True)
    except Exception as e:
        print(g, "ERR", e, flush=True)
res.sort(reverse=True)
for r in res[:5]:
    print("BEST", r)
