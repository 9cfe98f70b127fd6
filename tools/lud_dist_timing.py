"""Timing of the 2-D block-cyclic LU (rodinia_lud_dist) through the LOCAL communicator on one
GPU (all ranks serialised on one device; development aid), beside the single-GPU
panel-128 rodinia_lud.  Usage: python tools/lud_dist_timing.py [n]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
from paper_conf_cgo_ivanovzdem24_b200 import dist

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()


def timed(fn, reps=5):
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]


a = A.clone()
def single():
    a.copy_(A)
    rg.rodinia_lud(a, 128, g=(1, 1, 1, 1, 1, 0, 0))
single()
print(f"rodinia_lud panel 128: {timed(single):.2f} ms (incl. a {4*n*n/1e6:.0f} MB copy)", flush=True)
for prow, pcol in [(1, 1), (1, 2), (2, 2), (2, 4)]:
    comm = dist.HaloComm.local_slabs(prow * pcol)
    src = dist.block_cyclic_scatter(A, prow, pcol)
    parts = [x.clone() for x in src]
    def run():
        for x, y in zip(parts, src):
            x.copy_(y)
        comm.lud(parts, n, prow, pcol)
    run()
    print(f"rodinia_lud_dist LOCAL {prow}x{pcol}: {timed(run):.2f} ms (serialised on one GPU)", flush=True)
    comm.close()
