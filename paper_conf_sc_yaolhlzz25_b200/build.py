"""Build liblowdiff.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

    python -m paper_conf_sc_yaolhlzz25_b200.build [--force]

Each csrc/*.cu is compiled to an object with
  -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false
(no FMA contraction: the path's fp32 results are defined op by op) and linked
against the NCCL that torch loads (the pip nvidia-nccl 2.28.9), so the process holds a single
libnccl.so.2. The CUDA runtime is linked statically (it shares the driver's primary context with
torch, so torch-allocated device pointers and streams are valid here).
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
SO = os.environ.get("LOWDIFF_SO") or os.path.join(HERE, "liblowdiff.so")
BUILD = os.environ.get("LOWDIFF_BUILD_DIR") or os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ["-O3", "-lineinfo", "-std=c++17", "-fmad=false", "-Xcompiler", "-fPIC",
          "-Xptxas", "-warn-spills", "--expt-relaxed-constexpr"]


def nccl_dir() -> str:
    import nvidia.nccl  # the NCCL torch loads
    return os.path.dirname(os.path.abspath(nvidia.nccl.__file__)) if nvidia.nccl.__file__ else \
        list(nvidia.nccl.__path__)[0]


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu"))) + sorted(glob.glob(os.path.join(CSRC, "*.cpp")))


# plain C++ (the LowDiff+ host replica update): IEEE fp32 with no FMA contraction, vectorised
CXX = os.environ.get("CXX", "g++")
CXXFLAGS = ["-O3", "-std=c++17", "-fPIC", "-pthread", "-ffp-contract=off", "-fno-math-errno", "-g"]


def _deps() -> list[str]:
    return sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + \
        [os.path.join(INCLUDE, "lowdiff.h"), __file__]


def up_to_date() -> bool:
    if not os.path.exists(SO):
        return False
    t = os.path.getmtime(SO)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and up_to_date():
        return SO
    os.makedirs(BUILD, exist_ok=True)
    nd = nccl_dir()
    inc = ["-I", INCLUDE, "-I", CSRC, "-I", os.path.join(nd, "include")]

    def compile_one(src: str) -> str:
        obj = os.path.join(BUILD, os.path.basename(src) + ".o")
        extra = os.environ.get("LOWDIFF_NVCC_EXTRA", "").split()   # experiments, e.g. -DLOWDIFF_REPLAY_MINB=4
        if src.endswith(".cpp"):
            cmd = [CXX, *CXXFLAGS, "-I", INCLUDE, "-I", CSRC, "-c", src, "-o", obj]
        else:
            cmd = [NVCC, *ARCH, *CFLAGS, *extra, *inc, "-c", src, "-o", obj]
        if verbose:
            print(" ".join(cmd), flush=True)
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"compile failed for {src}:\n{r.stdout}\n{r.stderr}")
        if verbose and r.stderr.strip():
            print(r.stderr, file=sys.stderr)
        return obj

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(compile_one, sources()))
    lib = os.path.join(nd, "lib")
    tmp = SO + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-L", lib, "-l:libnccl.so.2",
           "-Xlinker", f"-rpath,{lib}", "-cudart", "static", "-lpthread"]
    if verbose:
        print(" ".join(cmd), flush=True)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, SO)
    return SO


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
