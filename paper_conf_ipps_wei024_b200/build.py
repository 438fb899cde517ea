"""Build libgcsm.so in-tree: hand-written CUDA for sm_100a + host C++ (nvcc, static cudart, NCCL)."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB_PATH = os.path.join(HERE, "libgcsm.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    cands = []
    if spec and spec.submodule_search_locations:
        for loc in spec.submodule_search_locations:
            cands.append(os.path.join(loc, "nccl"))
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return os.path.join(c, "include"), os.path.join(c, "lib")
    raise RuntimeError("nccl.h not found (expected the torch-bundled nvidia/nccl package)")


def sources():
    return sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu")) + glob.glob(os.path.join(HERE, "csrc", "*.cpp")))


def build(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    """Compile libgcsm.so (or a variant to `out` with extra -D defines, for tuning experiments)."""
    srcs = sources()
    target = out or LIB_PATH
    deps = srcs + glob.glob(os.path.join(HERE, "csrc", "*.h")) + glob.glob(os.path.join(HERE, "csrc", "*.cuh")) + \
        [os.path.join(ROOT, "include", "gcsm.h")]
    if not force and os.path.exists(target) and os.path.getmtime(target) >= max(os.path.getmtime(d) for d in deps):
        return target
    inc, lib = _nccl_dirs()
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    cmd = [nvcc, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xptxas", "-v", "-Xcompiler", "-fPIC,-O3",
           "-shared", "-cudart", "static", f"-I{os.path.join(ROOT, 'include')}", f"-I{inc}", *srcs,
           *[f"-D{d}" for d in defines], "-o", target + ".tmp", f"-L{lib}", "-l:libnccl.so.2", "-Xlinker", f"-rpath,{lib}", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc build of libgcsm.so failed")
    if out is None:
        with open(os.path.join(HERE, "build_ptxas.log"), "w") as f:
            f.write(r.stderr)
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
