"""Quick lud timing: panel 128 (tensor cores) vs panel 32 tuned (development aid)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
for panel, g in ((128, (1, 1, 1, 1, 1, 0, 0)), (32, (4, 4, 2, 2, 1, 1, 0))):
    a = A0.clone(); rg.rodinia_lud(a, panel, g=g); torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        a.copy_(A0)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_lud(a, panel, g=g); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = sorted(ts)[2]
    print(f"panel {panel}: {ms:.3f} ms  {2*n**3/3/ms/1e9:.1f} GFLOP/s", flush=True)
