"""Row-slab overhead on one GPU: the LOCAL communicator runs all P slabs of the multi-GPU path
(same schedule, halos, overlap split, side stream) one after another on one device, so
t_single / t_local(P) is the compute efficiency of the decomposition without NCCL latency
(halo recompute, strip launches, copies, per-slab launch gaps).  Development aid for
DESIGN.md §6; prints one JSON line.
  python tools/dist_local_timing.py [hotspot_iters] [srad_iters]"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth

hi = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
si = int(sys.argv[2]) if len(sys.argv) > 2 else 100


def split(a, P):
    R = a.shape[0]
    return [a[r0:r0 + n].contiguous() for r0, n in (rg.rodinia_slab(R, P, r) for r in range(P))]


def timed(fn, reps=3):
    fn(); torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


out = {}
N = 16384
T, Pw = synth.hotspot_inputs(N, N)
c = rg.rodinia_hotspot_coeffs_rodinia(N, N, N * 31.25e-6, N * 31.25e-6)
t, p = torch.from_numpy(T).cuda(), torch.from_numpy(Pw).cuda()
del T, Pw
g = (4, 1, 1, 12, 8, 1, 2 | (10 << 8))
o = torch.empty_like(t); s = torch.empty_like(t)
single = timed(lambda: rg.rodinia_hotspot(t, p, hi, coeffs=c, g=g, out=o, scratch=s))
out["hotspot"] = {"granularity": list(g), "iterations": hi, "single_ms": single}
for P in (2, 4, 8):
    comm = rg.dist.HaloComm.local_slabs(P)
    ts_, ps_ = split(t, P), split(p, P)
    os_ = [torch.empty_like(x) for x in ts_]
    gP, _ = rg.rodinia_tune("hotspot", N // P, N, hi, reps=2)  # re-tuned at the slab shape (bench --gpus P)
    ms = timed(lambda: comm.hotspot(ts_, ps_, os_, N, hi, coeffs=c, g=gP))
    out["hotspot"][f"local_P{P}_ms"] = ms
    out["hotspot"][f"granularity_P{P}"] = list(gP.astuple())
    out["hotspot"][f"efficiency_P{P}"] = single / ms
    comm.close()
del t, p, o, s
M = 8192
J0 = torch.from_numpy(synth.srad_input(M, M)).cuda()
J = J0.clone()
gs = (4, 1, 1, 3, 1, 1, 2)
single = timed(lambda: (J.copy_(J0), rg.rodinia_srad(J, 0, 127, 0, 127, 0.5, si, g=gs)))
out["srad"] = {"granularity": list(gs), "iterations": si, "single_ms": single}
for P in (2, 4, 8):
    comm = rg.dist.HaloComm.local_slabs(P)
    js = split(J0, P)
    j0s = [x.clone() for x in js]
    gP, _ = rg.rodinia_tune("srad", M // P, M, si, reps=3)  # re-tuned at the slab shape
    gP = gP.astuple()
    ms = timed(lambda: ([a.copy_(b) for a, b in zip(js, j0s)],
                        comm.srad(js, M, 0, 127, 0, 127, 0.5, si, g=gP[:4] + (8,) + gP[5:])))
    out["srad"][f"local_P{P}_ms"] = ms
    out["srad"][f"granularity_P{P}"] = list(gP)
    out["srad"][f"efficiency_P{P}"] = single / ms
    comm.close()
print(json.dumps(out), flush=True)
