"""Reproduce the paper's lud coarsening study on B200 (Fig. 14/15, Table II).

Fig. 14 analogue: total block factor b x total thread factor t, each split over (x, y) with
rodinia_split_total (footnote 4), runtime of the whole 8192^2 panel-16 factorisation relative to
the uncoarsened (1, 1).  Fig. 15 analogue: x-only block coarsening bx = 1..16 (t = 1) and with
thread factor 2/4 along x.  Writes JSON to stdout (tools/lud_sweep.py > out.json).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_cgo_ivanovzdem24_b200 as rg  # noqa: E402
import synth  # noqa: E402

n = int(os.environ.get("LUD_N", "8192"))
A0 = torch.from_numpy(synth.lud_rodinia_matrix(n)).cuda()
A = A0.clone()


def timed(g, panel=16):
    A.copy_(A0)
    rg.rodinia_lud(A, panel, g=g)
    torch.cuda.synchronize()
    ts = []
    for _ in range(2):
        A.copy_(A0)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        rg.rodinia_lud(A, panel, g=g)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return min(ts)


base = timed((1, 1, 1, 1, 1, 0, 0))
out = {"n": n, "panel": 16, "uncoarsened_ms": base, "fig14": [], "fig15": []}
for bt in (1, 2, 4, 7, 8, 14, 16):
    bx, by = rg.rodinia_split_total(bt, 2)
    for tt in (1, 2, 4, 8, 16):
        tx, ty = rg.rodinia_split_total(tt, 2)
        for mode in (0, 1):
            g = (tx, ty, bx, by, 1, mode, 0)
            try:
                ms = timed(g)
            except rg.RodiniaError as e:
                out["fig14"].append({"block": bt, "thread": tt, "g": g, "status": e.status})
                continue
            out["fig14"].append({"block": bt, "thread": tt, "g": g, "ms": ms, "speedup": base / ms})
for tx in (1, 2, 4):
    for bx in range(1, 17):
        g = (tx, 1, bx, 1, 1, 1, 0)
        try:
            ms = timed(g)
            out["fig15"].append({"bx": bx, "tx": tx, "ms": ms, "speedup": base / ms})
        except rg.RodiniaError as e:
            out["fig15"].append({"bx": bx, "tx": tx, "status": e.status})
print(json.dumps(out))
