"""Quick pathfinder per-call timing (CUDA graph of 200 calls)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_cgo_ivanovzdem24_b200 as rg
import synth
w = torch.from_numpy(synth.pathfinder_wall(100, 100000)).cuda()
r = torch.empty(100000, dtype=torch.int32, device="cuda")
res = []
def timeit(g, batch=200):
    rg.rodinia_pathfinder(w, g=g, out=r)
    s = torch.cuda.Stream(); s.wait_stream(torch.cuda.current_stream())
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(graph, stream=s):
            for _ in range(batch):
                rg.rodinia_pathfinder(w, g=g, out=r)
    torch.cuda.synchronize()
    graph.replay(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(3):
        e0.record(); graph.replay(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) / batch)
    return sorted(ts)[1]
for cells in (4, 8, 16, 32):
    for h in (16, 24, 33, 50, 99):
        g = (cells, 1, 1, 1, h, 1, 2)
        try:
            res.append((timeit(g), g))
        except Exception as e:
            print(g, e)
for t in range(1, 9):
    for b in (1, 2, 4):
        for h in (8, 16, 33, 50, 99):
            for mode in (0, 1):
                g = (t, 1, b, 1, h, mode, 0)
                try:
                    ms = timeit(g)
                except Exception as e:
                    continue
                res.append((ms, g))
res.sort()
for ms, g in res[:12]:
    print(f"{g} {ms*1e3:.2f} us")
print("uncoarsened", timeit((1, 1, 1, 1, 20, 0, 0)) * 1e3, "us")
