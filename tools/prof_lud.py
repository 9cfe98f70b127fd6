"""ncu target: one lud factorisation (n, granularity, panel from argv)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
g = tuple(int(x) for x in sys.argv[2].split(",")) if len(sys.argv) > 2 else (2, 2, 2, 2, 1, 1, 0)
panel = int(sys.argv[3]) if len(sys.argv) > 3 else 16
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
A = A0.clone()
rg.rodinia_lud(A, panel, g=g)
torch.cuda.synchronize()
