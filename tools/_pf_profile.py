import sys, os
sys.path.insert(0, "/root/repo")
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
w = torch.from_numpy(synth.pathfinder_wall(100, 100000)).cuda()
r = torch.empty(100000, dtype=torch.int32, device="cuda")
gs = [tuple(int(x) for x in a.split(",")) for a in sys.argv[1:]] or [(4, 1, 1, 1, 24, 1, 2)]
for g in gs:
    for _ in range(3):
        rg.rodinia_pathfinder(w, g=g, out=r)
torch.cuda.synchronize()
