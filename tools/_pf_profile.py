import sys, os
sys.path.insert(0, "/root/repo")
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
w = torch.from_numpy(synth.pathfinder_wall(100, 100000)).cuda()
r = torch.empty(100000, dtype=torch.int32, device="cuda")
for g in [(2,1,1,1,33,1,0), (1,1,1,1,20,0,0), (4,1,1,1,99,1,0), (8,1,1,1,16,1,0)]:
    for _ in range(3):
        rg.rodinia_pathfinder(w, g=g, out=r)
torch.cuda.synchronize()
