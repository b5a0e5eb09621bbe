"""Build libbf.so (the C-ABI library of include/bf.h) for sm_100a with nvcc.

In-tree build: the .so lands in paper_conf_ipps_madougouvln16_b200/_lib/ so
that it travels with the repository snapshot to the GPU box.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "_lib")
LIB = os.path.join(LIBDIR, "libbf.so")
TORCH_ALLOC = os.path.join(LIBDIR, "libbf_torch_alloc.so")
SOURCES = ["capi.cu", "fit.cu", "predict.cu", "importance.cu", "pca.cu", "models.cu", "prims.cu"]
HEADERS = ["bf_internal.cuh"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", "nvcc"):
        if c and (os.path.isabs(c) and os.path.exists(c) or not os.path.isabs(c)):
            return c
    return "nvcc"


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "bf.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    objs = []
    jobs = []
    for src in SOURCES:
        obj = os.path.join(LIBDIR, src.replace(".cu", ".o"))
        cmd = [nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include"),
               "-c", os.path.join(CSRC, src), "-o", obj]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
        jobs.append(subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT))
        objs.append(obj)
    errs = []
    for src, j in zip(SOURCES, jobs):
        out, _ = j.communicate()
        if j.returncode != 0:
            errs.append(f"--- {src}\n{out.decode()}")
        elif verbose:
            sys.stderr.write(out.decode())
    if errs:
        raise RuntimeError("nvcc failed:\n" + "\n".join(errs))
    tmp = LIB + ".tmp"
    subprocess.check_call([nvcc(), *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-lrt", "-lpthread", "-ldl"])
    os.replace(tmp, LIB)
    for o in objs:
        os.remove(o)
    return LIB


def build_torch_alloc(force: bool = False) -> str:
    """libbf_torch_alloc.so: the bf_set_allocator hooks over torch's CUDA caching allocator (csrc/torch_alloc.cpp),
    compiled with g++ against the installed torch's c10 headers and libraries (rpath to torch/lib)."""
    src = os.path.join(CSRC, "torch_alloc.cpp")
    if not force and os.path.exists(TORCH_ALLOC) and os.path.getmtime(TORCH_ALLOC) >= os.path.getmtime(src):
        return TORCH_ALLOC
    import torch
    tdir = os.path.dirname(torch.__file__)
    inc = [os.path.join(tdir, "include"), "/usr/local/cuda/include"]
    lib = os.path.join(tdir, "lib")
    os.makedirs(LIBDIR, exist_ok=True)
    tmp = TORCH_ALLOC + ".tmp"
    cmd = ["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-D_GLIBCXX_USE_CXX11_ABI=%d" % int(torch._C._GLIBCXX_USE_CXX11_ABI),
           *[f"-I{d}" for d in inc], src, "-o", tmp, f"-L{lib}", "-lc10_cuda", "-lc10", f"-Wl,-rpath,{lib}"]
    subprocess.check_call(cmd)
    os.replace(tmp, TORCH_ALLOC)
    return TORCH_ALLOC


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
    print(build_torch_alloc(force="--force" in sys.argv))
