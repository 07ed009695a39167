"""Build libdeepum_b200.so in-tree for sm_100a (nvcc, no torch extension).

    python -m paper_conf_asplos_jungkl23_b200.build [--force] [--verbose]
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys
import time

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.path.join(HERE, "libdeepum_b200.so")
BUILD = os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O3",
         "-I" + os.path.join(HERE, "..", "include")]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return _sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [
        os.path.join(HERE, "..", "include", "deepum_b200.h")]


def up_to_date() -> bool:
    if not os.path.exists(OUT):
        return False
    t = os.path.getmtime(OUT)
    return all(os.path.getmtime(p) <= t for p in _deps())


def build(force: bool = False, verbose: bool = False, ptxas_v: bool = False, checks: bool = False) -> str:
    out = OUT if not checks else OUT.replace(".so", "_checks.so")
    if not force and not checks and up_to_date():
        return OUT
    bdir = BUILD if not checks else BUILD + "_checks"
    os.makedirs(bdir, exist_ok=True)
    objs = []

    hdr_t = max(os.path.getmtime(p) for p in _deps() if not p.endswith(".cu"))
    start = time.time()

    def one(src):
        obj = os.path.join(bdir, os.path.basename(src) + ".o")
        if (not force and os.path.exists(obj) and os.path.getmtime(obj) >= os.path.getmtime(src)
                and os.path.getmtime(obj) >= hdr_t):
            return obj  # incremental: object newer than its source and every header
        cmd = [NVCC, *ARCH, *FLAGS, "-c", src, "-o", obj] + (["-DDUM_CHECKS", "-DDUM_POISON"] if checks else [])
        if ptxas_v:
            cmd[1:1] = ["-Xptxas", "-v"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, r.stdout, r.stderr))
        if verbose and (r.stderr or r.stdout):
            sys.stderr.write(r.stdout + r.stderr)
        # stamp the object with the build's start time: a source or header edited
        # while it compiled is newer than the object, so the next build redoes it
        os.utime(obj, (start, start))
        return obj

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        objs = list(ex.map(one, _sources()))
    tmp = out + ".tmp%d" % os.getpid()
    cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("link failed:\n%s\n%s" % (r.stdout, r.stderr))
    os.replace(tmp, out)
    return out


HOOK_SRC = os.path.join(CSRC, "alloc_hook.cpp")
HOOK_OUT = os.path.join(HERE, "libdeepum_hook.so")


def build_hook(force: bool = False) -> str:
    """libdeepum_hook.so: host C++ against PyTorch's c10 /
    c10_cuda (its CUDA caching allocator's trace tracker) and libdeepum_b200.so."""
    import torch
    import torch.utils.cpp_extension as ce
    deps = [HOOK_SRC, os.path.join(HERE, "..", "include", "deepum_hook.h"),
            os.path.join(HERE, "..", "include", "deepum_b200.h")]
    if not force and os.path.exists(HOOK_OUT) and all(os.path.getmtime(p) <= os.path.getmtime(HOOK_OUT)
                                                      for p in deps):
        return HOOK_OUT
    tlib = os.path.join(os.path.dirname(torch.__file__), "lib")
    abi = int(torch._C._GLIBCXX_USE_CXX11_ABI)
    tmp = HOOK_OUT + ".tmp%d" % os.getpid()
    cmd = ["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-D_GLIBCXX_USE_CXX11_ABI=%d" % abi,
           "-I" + os.path.join(HERE, "..", "include"), "-I/usr/local/cuda/include",
           *["-I" + p for p in ce.include_paths()], HOOK_SRC, "-o", tmp,
           "-L" + tlib, "-lc10", "-lc10_cuda", "-L/usr/local/cuda/lib64", "-lcudart",
           "-L" + HERE, "-ldeepum_b200", "-Wl,-rpath,$ORIGIN", "-Wl,-rpath," + tlib]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("g++ failed for alloc_hook.cpp:\n%s\n%s" % (r.stdout, r.stderr))
    os.replace(tmp, HOOK_OUT)
    return HOOK_OUT


UM_SRC = os.path.join(CSRC, "um", "um_runtime.cu")
UM_OUT = os.path.join(HERE, "libdeepum_um.so")


def build_um(force: bool = False) -> str:
    """libdeepum_um.so: the real-UM runtime -- managed
    arena, CUPTI launch interposition / fault records, cudaMemPrefetchAsync --
    with the shared CUDA runtime (the process's other launches go through it)."""
    deps = [UM_SRC, os.path.join(HERE, "..", "include", "deepum_um.h"),
            os.path.join(HERE, "..", "include", "deepum_b200.h")]
    if not force and os.path.exists(UM_OUT) and all(os.path.getmtime(p) <= os.path.getmtime(UM_OUT) for p in deps):
        return UM_OUT
    tmp = UM_OUT + ".tmp%d" % os.getpid()
    cmd = [NVCC, *ARCH, *FLAGS, "-shared", "-cudart", "shared", UM_SRC, "-o", tmp,
           "-L/usr/local/cuda/lib64", "-lcupti", "-lcuda", "-Xlinker", "-rpath=/usr/local/cuda/lib64"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for um_runtime.cu:\n%s\n%s" % (r.stdout, r.stderr))
    os.replace(tmp, UM_OUT)
    return UM_OUT


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv, ptxas_v="-v" in sys.argv,
                checks="--checks" in sys.argv))
    if "--checks" not in sys.argv:
        print(build_hook(force="--force" in sys.argv))
        print(build_um(force="--force" in sys.argv))
