"""Evaluate heuristic pre-pruning on the benchmark shapes: full TDO vs
rodinia_tune_pruned at several `keep` values.  Reports per workload the number of candidates
timed, tuning wall time, the winner, the regret (full-TDO median of the pruned winner over the
full-TDO best) and the Spearman rank correlation between model estimate and measured median.

  python tools/prune_eval.py [out.json]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_cgo_ivanovzdem24_b200 as rg  # noqa: E402

CASES = [("hotspot", dict(rows=16384, cols=16384, iterations=1000)),
         ("srad", dict(rows=8192, cols=8192, iterations=100)),
         ("hotspot3d", dict(rows=1024, cols=1024, iterations=10, depth=64))]


def spearman(a, b):
    ra = np.argsort(np.argsort(a)).astype(float)
    rb = np.argsort(np.argsort(b)).astype(float)
    return float(np.corrcoef(ra, rb)[0, 1])


def timed(rows):
    return {tuple(r["g"]): r["median_ms"] for r in rows if r["status"] == 0 and r["median_ms"] > 0}


def main():
    out = {"device": torch.cuda.get_device_name(0), "cases": []}
    for kernel, shape in CASES:
        t0 = time.perf_counter()
        best, rows = rg.rodinia_tune(kernel, reps=3, **shape)
        t_full = time.perf_counter() - t0
        full = timed(rows)
        ref = min(full.values())
        both = [(r["model_ms"], r["median_ms"]) for r in rows
                if r["status"] == 0 and r["median_ms"] > 0 and r["model_ms"] > 0]
        rho = spearman([m for m, _ in both], [t for _, t in both]) if len(both) > 2 else None
        case = {"kernel": kernel, "shape": shape,
                "full": {"timed": len(full), "seconds": round(t_full, 2), "best": list(best.astuple()),
                         "best_ms": ref},
                "spearman_model_vs_measured": rho, "pruned": [],
                "rows": [[list(r["g"]), r["model_ms"], r["median_ms"], r["regs"], r["ctas_per_sm"]]
                         for r in rows if r["status"] == 0 and r["median_ms"] > 0]}
        for keep in (2, 4, 8):
            t0 = time.perf_counter()
            bp, rp = rg.rodinia_tune_pruned(kernel, keep=keep, reps=3, **shape)
            t_p = time.perf_counter() - t0
            tp = timed(rp)
            got = full.get(bp.astuple(), tp.get(bp.astuple()))
            case["pruned"].append({"keep": keep, "timed": len(tp), "seconds": round(t_p, 2),
                                   "best": list(bp.astuple()), "best_ms_in_full_run": got,
                                   "regret": got / ref if got else None})
        out["cases"].append(case)
        print(json.dumps({k: v for k, v in case.items() if k != "rows"}), flush=True)
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/prune_eval.json"
    with open(path, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
