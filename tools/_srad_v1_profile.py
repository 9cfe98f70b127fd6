import sys; sys.path.insert(0, "/root/repo")
import torch, paper_conf_cgo_ivanovzdem24_b200 as rg, synth
img = torch.from_numpy(synth.srad_v1_image(8192, 8192)).cuda()
rg.rodinia_srad_v1(img, 0.5, 10, g=(4, 1, 1, 3, 1, 1, 2)); torch.cuda.synchronize()
