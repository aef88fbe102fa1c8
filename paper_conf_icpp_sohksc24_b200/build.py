"""Build libcstf.so in-tree (nvcc, sm_100a).  No torch JIT: the .so travels
with the repo snapshot to the GPU box.  Usage: python -m paper_conf_icpp_sohksc24_b200.build"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
LIB = os.path.join(LIBDIR, "libcstf.so")
ABL_SRC = os.path.join(HERE, "ablation", "ablation.cu")      # bench-only Fig. 4 arms (not part of libcstf)
ABL_LIB = os.path.join(LIBDIR, "libcstf_ablation.so")
ROOT = os.path.dirname(HERE)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_include() -> str:
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations or []) if spec else []:
        inc = os.path.join(base, "nccl", "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    raise RuntimeError("nccl.h not found (nvidia-nccl wheel)")


def flags():
    return ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2,-Wall",
                   "-I", os.path.join(ROOT, "include"), "-I", nccl_include(),
                   "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "cstf.h"), __file__]
    return any(os.path.getmtime(d) > t for d in deps)


def build_ablation(force: bool = False) -> str:
    """libcstf_ablation.so: the paper's Fig. 4 ADMM arms (cuBLAS DGEAM/DTRSM/DGEMM + plain
    kernels), used only by bench.py --ablation and tests/test_gpu_ablation.py."""
    deps = [ABL_SRC, os.path.join(ROOT, "include", "cstf_ablation.h"), __file__]
    if not force and os.path.exists(ABL_LIB) and all(os.path.getmtime(d) <= os.path.getmtime(ABL_LIB) for d in deps):
        return ABL_LIB
    os.makedirs(LIBDIR, exist_ok=True)
    tmp = ABL_LIB + f".tmp{os.getpid()}"
    cmd = [NVCC] + ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2,-Wall", "-shared",
                           "-o", tmp, ABL_SRC, "-lcublas"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {ABL_SRC}:\n{r.stderr}")
    os.replace(tmp, ABL_LIB)
    return ABL_LIB


def build(force: bool = False, verbose: bool = False) -> str:
    build_ablation(force)
    if not force and not _stale():
        return LIB
    os.makedirs(os.path.join(LIBDIR, "obj"), exist_ok=True)
    fl = flags()

    def compile_one(src):
        obj = os.path.join(LIBDIR, "obj", os.path.basename(src) + ".o")
        cmd = [NVCC] + fl + ["-c", src, "-o", obj]
        if verbose:
            cmd += ["-Xptxas", "-v"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
        return obj, r.stderr

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        results = list(ex.map(compile_one, sources()))
    if verbose:
        for _, err in results:
            sys.stderr.write(err)
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + [o for o, _ in results] + ["-ldl", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr}")
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
