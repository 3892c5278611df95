"""Build libhccmf.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo).

Each csrc/*.cu compiles to its own object under build/ (in parallel, and only when it or
a header changed); the objects link into libhccmf.so against torch's bundled NCCL.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OBJ = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "libhccmf.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dir() -> str:
    import nvidia.nccl  # torch's bundled NCCL (site-packages/nvidia/nccl)
    return os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def headers():
    return sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [os.path.join(ROOT, "include", "hccmf.h")]


def deps():
    return sources() + headers()


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps())


def _flags(defines, verbose):
    nd = nccl_dir()
    f = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC,-fvisibility=hidden",
         "-I", os.path.join(ROOT, "include"), "-I", os.path.join(nd, "include"), *[f"-D{d}" for d in defines]]
    if verbose:
        f.insert(0, "-Xptxas=-v")
    return f


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    if out is None and not force and not stale():
        return LIB
    nd = nccl_dir()
    target = out or LIB
    tag = "_".join(d.replace("=", "-") for d in defines) or "default"
    odir = os.path.join(OBJ, tag)
    os.makedirs(odir, exist_ok=True)
    flags = _flags(defines, verbose)
    hdr_t = max(os.path.getmtime(h) for h in headers())

    def obj(src):
        o = os.path.join(odir, os.path.basename(src)[:-3] + ".o")
        if force or not os.path.exists(o) or os.path.getmtime(o) < max(hdr_t, os.path.getmtime(src)):
            cmd = [NVCC, *flags, "-c", "-o", o + ".tmp", src]
            if verbose:
                print(" ".join(cmd), file=sys.stderr)
            subprocess.check_call(cmd)
            os.replace(o + ".tmp", o)
        return o

    with ThreadPoolExecutor(max_workers=len(sources())) as ex:
        objs = list(ex.map(obj, sources()))
    tmp = target + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-L", os.path.join(nd, "lib"), "-l:libnccl.so.2",
                           "-Xlinker", "-rpath," + os.path.join(nd, "lib")])
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a.split("=", 1)[1] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, out=outs[0] if outs else None, defines=defs))
