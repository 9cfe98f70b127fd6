"""A/B per-call pathfinder timing of warp-band granularities across library builds.

Usage: python tools/ab_pf.py lib1.so [lib2.so ...]   (each lib timed in its own process,
interleaved twice; RODINIA_GRAN_LIB selects the build).  Prints us/call per (lib, granularity).
"""
import json
import os
import subprocess
import sys

GRANS = [(4, 1, 1, 1, 20, 1, 2)] + [(2, 1, 1, 1, h, 1, 2) for h in (4, 8, 12, 16, 20)] + \
        [(c, 1, 1, 1, h, 1, 2) for c in (4, 8) for h in (12, 16, 24, 28)] + \
        [(16, 1, 1, 1, h, 1, 2) for h in (33, 50, 99)]

CHILD = r"""
import json, sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
w = torch.from_numpy(synth.pathfinder_wall(100, 100000)).cuda()
r = torch.empty(100000, dtype=torch.int32, device="cuda")
ref = None
out = {}
for g in json.loads(sys.argv[1]):
    g = tuple(g)
    try:
        rg.rodinia_pathfinder(w, g=g, out=r)
    except Exception as e:
        out[str(g)] = str(e)[:60]
        continue
    torch.cuda.synchronize()
    if ref is None:
        ref = r.clone()
    assert torch.equal(ref, r), g
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(graph, stream=s):
            for _ in range(200):
                rg.rodinia_pathfinder(w, g=g, out=r)
    torch.cuda.synchronize()
    graph.replay(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(5):
        e0.record(); graph.replay(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 200 * 1e3)
    out[str(g)] = sorted(ts)[2]
print(json.dumps(out))
"""

if __name__ == "__main__":
    libs = sys.argv[1:]
    res = {}
    for rep in range(2):
        for lib in libs:
            env = dict(os.environ, RODINIA_GRAN_LIB=os.path.abspath(lib))
            p = subprocess.run([sys.executable, "-c", CHILD, json.dumps(GRANS)], env=env,
                               capture_output=True, text=True)
            if p.returncode:
                print(lib, p.stderr[-800:])
                continue
            d = json.loads(p.stdout.strip().splitlines()[-1])
            for k, v in d.items():
                res.setdefault(k, {}).setdefault(lib, []).append(v)
    for k, d in res.items():
        print(k, "  ".join(f"{os.path.basename(l)}={v}" for l, v in d.items()))
