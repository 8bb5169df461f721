"""Builds libjitc.so in-tree for sm_100a (nvcc cross-compiles; no GPU needed).

    python -m paper_conf_eurosys_guptakkvgkrs24_b200.build [--force]

C++17 host code + CUDA kernels compiled with
`-gencode arch=compute_100a,code=sm_100a -lineinfo -O3`, linked against the
NCCL that torch ships (same version the harness's process group loads) with
an rpath, and cudart statically.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
OUT = os.path.join(PKG, "libjitc.so")
BUILD = os.path.join(PKG, "_build")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _cuda_home() -> str:
    for c in (os.environ.get("CUDA_HOME"), "/usr/local/cuda"):
        if c and os.path.exists(os.path.join(c, "bin", "nvcc")):
            return c
    nvcc = shutil.which("nvcc")
    if nvcc:
        return os.path.dirname(os.path.dirname(nvcc))
    raise RuntimeError("nvcc not found")


def _nccl_home() -> str:
    try:
        import nvidia.nccl as m
        base = list(m.__path__)[0]
        if os.path.exists(os.path.join(base, "include", "nccl.h")):
            return base
    except Exception:
        pass
    for base in ("/usr",):
        if os.path.exists(os.path.join(base, "include", "nccl.h")):
            return base
    raise RuntimeError("nccl.h not found")


def _run(cmd):
    print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)


def build(force: bool = False, verbose_ptxas: bool = False, sanitize: bool = False, tsan: bool = False) -> str:
    """sanitize=True builds libjitc_asan.so: host code with AddressSanitizer +
    UndefinedBehaviorSanitizer (tests/test_asan.py drives it); tsan=True builds
    libjitc_tsan.so: host code with ThreadSanitizer (tests/test_tsan.py).
    Neither is the product."""
    cuda, nccl = _cuda_home(), _nccl_home()
    nvcc = os.path.join(cuda, "bin", "nvcc")
    nccl_lib = os.path.join(nccl, "lib") if os.path.isdir(os.path.join(nccl, "lib")) else "/usr/lib/x86_64-linux-gnu"
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cc")))
    hdrs = sorted(glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(INCLUDE, "*.h")))
    out = OUT.replace("libjitc.so", "libjitc_asan.so") if sanitize else \
        OUT.replace("libjitc.so", "libjitc_tsan.so") if tsan else OUT
    bdir = BUILD + ("_asan" if sanitize else "_tsan" if tsan else "")
    newest = max(os.path.getmtime(p) for p in srcs + hdrs + [__file__])
    if not force and os.path.exists(out) and os.path.getmtime(out) >= newest:
        return out
    os.makedirs(bdir, exist_ok=True)
    san = ["-Xcompiler", "-fsanitize=address", "-Xcompiler", "-fsanitize=undefined", "-Xcompiler",
           "-fno-omit-frame-pointer", "-Xcompiler", "-g"] if sanitize else \
        ["-Xcompiler", "-fsanitize=thread", "-Xcompiler", "-fno-omit-frame-pointer", "-Xcompiler", "-g"] if tsan else []
    incs = ["-I", INCLUDE, "-I", CSRC, "-I", os.path.join(nccl, "include")]
    objs = []
    for s in srcs:
        o = os.path.join(bdir, os.path.basename(s) + ".o")
        if s.endswith(".cu"):
            cmd = [nvcc, *ARCH, "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC", *incs, "-c", s, "-o", o]
            if verbose_ptxas:
                cmd.insert(1, "-Xptxas=-v")
        else:
            cmd = [nvcc, "-x", "cu", *ARCH, "-O3", "-std=c++17", "-Xcompiler", "-fPIC,-Wall", *san, *incs, "-c", s,
                   "-o", o]
        _run(cmd)
        objs.append(o)
    tmp = out + ".tmp"
    _run([nvcc, *ARCH, "-shared", "-o", tmp, *objs, "-L", nccl_lib, "-l:libnccl.so.2",
          f"-Xlinker=-rpath={nccl_lib}", "-cudart", "static", *san])
    os.replace(tmp, out)
    return out


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose_ptxas="-v" in sys.argv, sanitize="--asan" in sys.argv,
          tsan="--tsan" in sys.argv)
