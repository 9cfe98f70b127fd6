"""ncu target: 4 srad_v2 iterations on the 8192^2 image at a given granularity."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
g = tuple(int(x) for x in sys.argv[1].split(",")) if len(sys.argv) > 1 else (4, 1, 1, 2, 1, 1, 2)
J = torch.from_numpy(synth.srad_input(8192, 8192)).cuda()
rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, 4, g=g)
torch.cuda.synchronize()
