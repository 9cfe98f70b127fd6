"""A/B timing of srad_v2 at 8192^2 (development aid; not the bench).

  RODINIA_GRAN_LIB=<lib.so> python tools/ab_srad.py [iters] [g;g;...]
Median of 5 CUDA-event-timed solves per granularity (ms per solve and per iteration)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

it = int(sys.argv[1]) if len(sys.argv) > 1 else 100
grans = [tuple(int(x) for x in g.split(",")) for g in sys.argv[2].split(";")] if len(sys.argv) > 2 else \
    [(4, 1, 1, 3, 1, 1, 2), (4, 1, 1, 4, 1, 1, 2)]
N = 8192
J0 = torch.from_numpy(synth.srad_input(N, N)).cuda()
J = J0.clone()
tag = os.path.basename(os.environ.get("RODINIA_GRAN_LIB", "default"))
for g in grans:
    J.copy_(J0); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        J.copy_(J0)
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, it, g=g); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = statistics.median(ts)
    print(f"{tag:14s} {str(g):26s} {ms:8.3f} ms  {1000*ms/it:7.2f} us/iter  {8*N*N*it/(ms*1e-3)/1e9:6.0f} GB/s", flush=True)
