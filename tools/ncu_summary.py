"""Summarise ncu output for profiles/: a launch list CSV (gpu__time_duration.sum per launch)
and/or a --set full report (.ncu-rep) of the top kernel.

  python tools/ncu_summary.py --launches gpurun_out/launches.csv --rep gpurun_out/prof.ncu-rep \
      --out profiles/r01_hotspot --algo-bytes 3221225472
"""
import argparse
import collections
import csv
import io
import json
import subprocess

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "sm__cycles_elapsed.avg.per_second",
        "launch__occupancy_limit_registers", "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = []
    for r in rows:
        if "Kernel Name" in r and "Metric Value" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") == "gpu__time_duration.sum":
                v = float(d["Metric Value"].replace(",", ""))
                unit = d.get("Metric Unit", "")
                us = v / 1000 if unit in ("nsecond", "ns") else (v if unit in ("usecond", "us") else v * 1000)
                out.append((d["Kernel Name"], us))
    agg = collections.OrderedDict()
    for k, us in out:
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += us
    tot = sum(a[1] for a in agg.values()) or 1.0
    return [{"kernel": k, "launches": a[0], "total_us": a[1], "avg_us": a[1] / a[0], "share": a[1] / tot}
            for k, a in sorted(agg.items(), key=lambda kv: -kv[1][1])]


def rep(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    out = []
    for vals in rows[2:]:
        d = {"kernel": vals[hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                d[k] = (vals[i], units[i])
        out.append(d)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--out", required=True)
    ap.add_argument("--algo-bytes", type=float, default=None)
    ap.add_argument("--gran", default="", help="granularity the capture was taken with")
    a = ap.parse_args()
    res = {"granularity": [int(x) for x in a.gran.split(",")] if a.gran else None}
    md = [f"granularity: {a.gran}\n"] if a.gran else []
    if a.launches:
        L = launches(a.launches)
        res["launch_list"] = L
        md.append("| kernel | launches | avg us | share |\n|---|---|---|---|")
        for r in L[:15]:
            md.append(f"| `{r['kernel'][:90]}` | {r['launches']} | {r['avg_us']:.1f} | {100*r['share']:.1f}% |")
    if a.rep:
        R = rep(a.rep)
        res["full"] = R
        for r in R:
            md.append(f"\n**{r['kernel'][:120]}**\n")
            for k in KEYS:
                if k in r:
                    md.append(f"- {k}: {r[k][0]} {r[k][1]}")
            def num(k):
                v, u = r[k]
                v = float(v.replace(",", ""))
                return v * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "Tbyte": 1e12}.get(u, 1)
            if "dram__bytes_read.sum" in r:
                traffic = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
                res["traffic_bytes_per_launch"] = traffic
                md.append(f"- traffic (read+write): {traffic/1e9:.3f} GB per launch")
                if a.algo_bytes:
                    md.append(f"- traffic / algorithmic bytes: {traffic / a.algo_bytes:.3f}")
    json.dump(res, open(a.out + ".json", "w"), indent=1)
    open(a.out + ".md", "w").write("\n".join(md) + "\n")


if __name__ == "__main__":
    main()
