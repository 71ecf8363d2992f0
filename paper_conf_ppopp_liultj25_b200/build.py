"""Build libmario.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with gpurun).

    python -m paper_conf_ppopp_liultj25_b200.build [-v] [-j N]
"""
from __future__ import annotations

import glob
import hashlib
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT = os.path.join(PKG, "libmario.so")
BUILD = os.path.join(ROOT, "build", "obj")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    base = None
    if spec and spec.submodule_search_locations:
        base = os.path.join(list(spec.submodule_search_locations)[0], "nccl")
    if base and os.path.exists(os.path.join(base, "include", "nccl.h")):
        return os.path.join(base, "include"), os.path.join(base, "lib")
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
          "-Xptxas", "-v", "-DNDEBUG"]
EXTRA = os.environ.get("NVCC_EXTRA", "").split()   # A/B switches, e.g. -DMARIO_EPI_EF=1


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "**", "*.cu"), recursive=True) +
                  glob.glob(os.path.join(CSRC, "**", "*.cpp"), recursive=True))


def _headers_digest():
    h = hashlib.sha1()
    for f in sorted(glob.glob(os.path.join(CSRC, "**", "*.h*"), recursive=True) +
                    glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True) +
                    glob.glob(os.path.join(ROOT, "include", "*.h"))):
        h.update(open(f, "rb").read())
    return h.hexdigest()[:12]


def build(verbose: bool = False, jobs: int = 8) -> str:
    inc, lib = _nccl_dirs()
    os.makedirs(BUILD, exist_ok=True)
    hd = _headers_digest()
    srcs = sources()
    objs = []

    def compile_one(src):
        rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
        flags = [NVCC, *ARCH, *COMMON, *EXTRA, "-I", os.path.join(ROOT, "include"), "-I", CSRC, "-I", inc]
        # the object name hashes the source, every header, the full nvcc command line and this
        # script, so a flag or -D change (e.g. NVCC_EXTRA="-DMARIO_EPI_EF=1") never links stale objects
        digest = hashlib.sha1(open(src, "rb").read() + hd.encode() + " ".join(flags).encode() +
                              open(os.path.abspath(__file__), "rb").read()).hexdigest()[:12]
        obj = os.path.join(BUILD, f"{rel}.{digest}.o")
        log = obj + ".log"
        if not os.path.exists(obj):
            cmd = [*flags, "-c", src, "-o", obj]
            r = subprocess.run(cmd, capture_output=True, text=True)
            open(log, "w").write(r.stdout + r.stderr)
            if r.returncode != 0:
                raise RuntimeError(f"nvcc failed on {src}:\n{r.stderr[-6000:]}")
        if verbose:
            sys.stdout.write(open(log).read() if os.path.exists(log) else "")
        return obj

    with ThreadPoolExecutor(jobs) as ex:
        objs = list(ex.map(compile_one, srcs))
    cmd = [NVCC, *ARCH, "-shared", "-o", OUT + ".tmp", *objs, "-L", lib, "-l:libnccl.so.2",
           "-Xlinker", f"-rpath={lib}", "-lcudart_static", "-ldl", "-lpthread", "-lrt"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr[-6000:]}")
    os.replace(OUT + ".tmp", OUT)
    return OUT


if __name__ == "__main__":
    v = "-v" in sys.argv
    print(build(verbose=v))
