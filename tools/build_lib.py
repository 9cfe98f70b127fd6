"""Build librodinia_gran.so (sm_100a) in-tree with nvcc, plus the compile-time variant filter.

Steps:
 1. nvcc -c every csrc/*.cu with -Xptxas -v (logs kept in build/ptxas_<tu>.log);
 2. tools/ptxas_filter.py parses the logs -> build/variant_stats.cpp (the ptxas table the
    runtime filter and rodinia_variants() use);
 3. link everything into paper_conf_cgo_ivanovzdem24_b200/librodinia_gran.so
    (static cudart; NCCL is dlopen'ed at run time, never linked).

Usage: python tools/build_lib.py [--force] [-j N]
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_cgo_ivanovzdem24_b200")
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build")
LIB = os.path.join(PKG, "librodinia_gran.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

sys.path.insert(0, os.path.join(ROOT, "tools"))
import ptxas_filter  # noqa: E402

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2",
                 "-I" + os.path.join(ROOT, "include"), "-I" + CSRC,
                 "--expt-relaxed-constexpr", "-Xptxas", "-v"]


def _newest(paths):
    return max((os.path.getmtime(p) for p in paths), default=0.0)


def _compile(src: str, force: bool, extra=()) -> tuple[str, str]:
    name = os.path.splitext(os.path.basename(src))[0]
    obj = os.path.join(BUILD, name + ".o")
    log = os.path.join(BUILD, f"ptxas_{name}.log")
    deps = [src] + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "rodinia_gran.h")]
    if not force and os.path.exists(obj) and os.path.exists(log) and os.path.getmtime(obj) >= _newest(deps):
        return obj, log
    cmd = [NVCC, *CFLAGS, *extra, "-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    with open(log, "w") as f:
        f.write(r.stderr)
    return obj, log


def build(force: bool = False, jobs: int = 8, verbose: bool = True, defines=(), out: str = "",
          builddir: str = "") -> str:
    """defines/out/builddir: development A/B builds (e.g. -D RG_SR_D=8 into a second .so that
    the binding loads when RODINIA_GRAN_LIB names it); the default build uses none of them."""
    global BUILD, LIB
    if builddir:
        BUILD = os.path.abspath(builddir)
    if out:
        LIB = os.path.abspath(out)
    os.makedirs(BUILD, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    extra = [f"-D{d}" for d in defines]
    with cf.ThreadPoolExecutor(max_workers=jobs) as ex:
        results = list(ex.map(lambda s: _compile(s, force, extra), srcs))
    objs = [o for o, _ in results]
    text = "".join(open(l).read() for _, l in results)
    stats = ptxas_filter.parse_ptxas_log(text)
    stats_cpp = os.path.join(BUILD, "variant_stats.cpp")
    ptxas_filter.write_stats_cpp(stats, stats_cpp + ".new")
    if not os.path.exists(stats_cpp) or open(stats_cpp).read() != open(stats_cpp + ".new").read():
        os.replace(stats_cpp + ".new", stats_cpp)
    else:
        os.remove(stats_cpp + ".new")
    stats_obj = os.path.join(BUILD, "variant_stats.o")
    if force or not os.path.exists(stats_obj) or os.path.getmtime(stats_obj) < os.path.getmtime(stats_cpp):
        subprocess.check_call([NVCC, *ARCH, "-std=c++17", "-Xcompiler", "-fPIC",
                               "-I" + os.path.join(ROOT, "include"), "-I" + CSRC, "-x", "cu",
                               "-c", stats_cpp, "-o", stats_obj])
    objs.append(stats_obj)
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < _newest(objs):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-cudart", "static", "-ldl",
                               "-lpthread"])
        os.replace(tmp, LIB)
    if verbose:
        print(f"[build] {LIB} ({len(stats)} kernel instantiations in the ptxas table)")
    return LIB


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=8)
    ap.add_argument("--define", action="append", default=[])
    ap.add_argument("--out", default="")
    ap.add_argument("--builddir", default="")
    a = ap.parse_args()
    build(force=a.force, jobs=a.j, defines=a.define, out=a.out, builddir=a.builddir)
