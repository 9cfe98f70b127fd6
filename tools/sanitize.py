"""Small-shape run of every kernel family, the target of the compute-sanitizer pass
(tools/sanitize.sh: memcheck, racecheck, synccheck).

Shapes are ragged (not multiples of the tiles) so edge CTAs, remainder launches and masked
lanes run; every family of every workload is launched at least once.  Results are not checked
here (the parity tests do that); the sanitizer's report is the output.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cgo_ivanovzdem24_b200 as rg  # noqa: E402
import synth  # noqa: E402

STREAM = rg.RODINIA_STREAM
only = sys.argv[1] if len(sys.argv) > 1 else ""


def want(name):
    return not only or name in only.split(",")


torch.cuda.set_device(0)
if want("hotspot"):
    T, P = synth.hotspot_inputs(150, 270)
    t, p = torch.from_numpy(T).cuda(), torch.from_numpy(P).cuda()
    c = rg.rodinia_hotspot_coeffs_rodinia(150, 270, 150 * 31.25e-6, 270 * 31.25e-6)
    for g in [(1, 1, 1, 1, 1, 0, 0), (4, 1, 2, 1, 1, 1, 0), (2, 2, 3, 2, 1, 0, 0), (16, 1, 1, 1, 1, 1, 0),
              (4, 1, 1, 2, 8, 1, STREAM), (4, 1, 2, 3, 4, 1, STREAM), (2, 1, 1, 2, 8, 1, STREAM),
              (1, 1, 1, 1, 4, 1, STREAM)]:
        rg.rodinia_hotspot(t, p, 11, coeffs=c, g=g)
    rg.rodinia_hotspot(t[1:], p[1:], 9, coeffs=c, g=(4, 1, 1, 2, 8, 1, STREAM))  # unaligned rows
    torch.cuda.synchronize()
    print("hotspot ok", flush=True)
if want("srad"):
    J0 = torch.from_numpy(synth.srad_input(130, 210)).cuda()
    for g in [(1, 1, 1, 1, 1, 0, 0), (2, 2, 2, 1, 1, 1, 0), (1, 1, 2, 1, 1, 0, 0), (4, 1, 1, 2, 1, 1, STREAM),
              (2, 1, 1, 1, 1, 1, STREAM), (8, 1, 1, 3, 1, 1, STREAM), (1, 1, 1, 1, 1, 1, STREAM)]:
        J = J0.clone()
        rg.rodinia_srad(J, 3, 70, 5, 101, 0.5, 4, g=g)
    I = torch.from_numpy(synth.srad_v1_image(97, 133)).cuda()
    rg.rodinia_srad_v1(I, 0.5, 3, g=(4, 1, 1, 2, 1, 1, STREAM))
    torch.cuda.synchronize()
    print("srad ok", flush=True)
if want("pathfinder"):
    w = torch.from_numpy(synth.pathfinder_wall(40, 3001)).cuda()
    for g in [(1, 1, 1, 1, 20, 0, 0), (2, 1, 1, 1, 8, 1, 0), (3, 1, 2, 1, 5, 0, 0), (4, 1, 1, 1, 20, 1, STREAM),
              (2, 1, 1, 1, 12, 1, STREAM), (8, 1, 1, 1, 16, 1, STREAM)]:
        rg.rodinia_pathfinder(w, g=g)
    torch.cuda.synchronize()
    print("pathfinder ok", flush=True)
if want("lud"):
    A = torch.from_numpy(synth.lud_rodinia_matrix(300)).cuda()
    for panel, g in [(16, (1, 1, 1, 1, 1, 0, 0)), (16, (2, 2, 2, 2, 1, 1, 0)), (32, (4, 2, 2, 2, 1, 1, 0)),
                     (16, (4, 1, 1, 2, 1, 1, STREAM)), (32, (2, 1, 1, 1, 1, 1, STREAM)), (128, None)]:
        a = A.clone()
        rg.rodinia_lud(a, panel, g=g)
    B = torch.from_numpy(synth.lud_rodinia_matrix(301)).cuda()  # n % 4 != 0: scalar paths of panel 128
    rg.rodinia_lud(B.clone(), 128)
    # 2-D block-cyclic LU (LOCAL communicator): 2 x 2 on n = 300, 1 x 3 on n = 301
    from paper_conf_cgo_ivanovzdem24_b200 import dist
    for M, prow, pcol in [(A, 2, 2), (B, 1, 3)]:
        parts = dist.block_cyclic_scatter(M, prow, pcol)
        comm = dist.HaloComm.local_slabs(prow * pcol)
        comm.lud(parts, M.shape[0], prow, pcol)
        torch.cuda.synchronize()
        comm.close()
    torch.cuda.synchronize()
    print("lud ok", flush=True)
if want("hotspot3d"):
    T3 = torch.rand(5, 37, 70, device="cuda") * 20 + 323.15
    P3 = torch.rand(5, 37, 70, device="cuda") * 1e-3
    c3 = rg.rodinia_hotspot3d_coeffs_rodinia(70, 37, 5)
    for g in [(1, 1, 1, 1, 1, 0, 0), (2, 2, 1, 1, 1, 1, STREAM), (1, 1, 1, 1, 1, 1, STREAM), (2, 1, 2, 1, 1, 1, 0)]:
        rg.rodinia_hotspot3d(T3, P3, 3, coeffs=c3, g=g)
    torch.cuda.synchronize()
    print("hotspot3d ok", flush=True)
if want("dist"):
    from paper_conf_cgo_ivanovzdem24_b200 import dist
    comm = dist.HaloComm.local_slabs(3)
    R, C = 61, 140
    T, P = synth.hotspot_inputs(R, C)
    sl = [rg.rodinia_slab(R, 3, r) for r in range(3)]
    ts = [torch.from_numpy(T[a:a + n]).cuda() for a, n in sl]
    ps = [torch.from_numpy(P[a:a + n]).cuda() for a, n in sl]
    os_ = [torch.empty_like(x) for x in ts]
    c = rg.rodinia_hotspot_coeffs_rodinia(R, C, R * 31.25e-6, C * 31.25e-6)
    comm.hotspot(ts, ps, os_, R, 9, coeffs=c, g=(4, 1, 1, 1, 4, 1, STREAM))
    J = synth.srad_input(R, C)
    js = [torch.from_numpy(J[a:a + n]).cuda() for a, n in sl]
    comm.srad(js, R, 2, 20, 3, 40, 0.5, 5, g=(4, 1, 1, 1, 1, 1, STREAM))
    torch.cuda.synchronize()
    print("dist ok", flush=True)
print("sanitize targets done", flush=True)
