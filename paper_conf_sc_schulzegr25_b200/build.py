"""Build libmdh.so in-tree with nvcc for sm_100a (B200).

    python -m paper_conf_sc_schulzegr25_b200.build [--force] [-j N]

Every .cu/.cpp under csrc/ is compiled with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17`` (ptxas -v
output goes to build/ptxas/<file>.log), then linked into a shared library with the
CUDA runtime linked statically (so the .so loads on machines without a GPU or
driver — planning and validation need none) and NCCL loaded lazily with dlopen.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(ROOT, "build", "libmdh")
LIB = os.path.join(PKG, "libmdh.so")
TILES = os.path.join(ROOT, "tiles", "b200.json")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-Wall", "-I" + os.path.join(ROOT, "include"),
         "--expt-relaxed-constexpr", "-Xptxas", "-v", "-diag-suppress", "177,550"]


def _sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cu", ".cpp")))


def _headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh", ".inc"))]
    return hs + [os.path.join(ROOT, "include", "mdh.h")]


def _write_tiles_inc():
    inc = os.path.join(CSRC, "tiles_builtin.inc")
    with open(TILES) as f:
        text = f.read()
    body = 'R"MDHJSON(' + text + ')MDHJSON"\n'
    old = open(inc).read() if os.path.exists(inc) else None
    if old != body:
        with open(inc, "w") as f:
            f.write(body)


def _compile(src, force):
    os.makedirs(os.path.join(BUILD, "ptxas"), exist_ok=True)
    obj = os.path.join(BUILD, os.path.basename(src) + ".o")
    newest = max(os.path.getmtime(h) for h in _headers() + [src])
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= newest:
        return obj, None
    cmd = [NVCC, *ARCH, *FLAGS, "-c", src, "-o", obj]
    if src.endswith(".cpp"):
        cmd = [NVCC, *FLAGS, "-x", "cu", "-c", src, "-o", obj] if False else [NVCC, *ARCH, *FLAGS, "-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    log = os.path.join(BUILD, "ptxas", os.path.basename(src) + ".log")
    with open(log, "w") as f:
        f.write(r.stdout + r.stderr)
    if r.returncode != 0:
        return obj, f"{' '.join(cmd)}\n{r.stdout}\n{r.stderr}"
    return obj, None


def build(force: bool = False, jobs: int = 0) -> str:
    _write_tiles_inc()
    srcs = _sources()
    jobs = jobs or min(len(srcs), os.cpu_count() or 4)
    with cf.ThreadPoolExecutor(jobs) as ex:
        res = list(ex.map(lambda s: _compile(s, force), srcs))
    errs = [e for _, e in res if e]
    if errs:
        raise RuntimeError("libmdh build failed:\n" + "\n\n".join(errs))
    objs = [o for o, _ in res]
    newest = max(os.path.getmtime(o) for o in objs)
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < newest:
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-ldl", "-lpthread", "-lrt"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"libmdh link failed:\n{' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, LIB)
    return LIB


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=0)
    a = ap.parse_args(argv)
    print(build(a.force, a.j))


if __name__ == "__main__":
    sys.exit(main())
