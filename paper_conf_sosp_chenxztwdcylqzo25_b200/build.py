"""Build libmoe_b200.so (all CUDA sources of csrc/) for sm_100a, in-tree.

nvcc -gencode arch=compute_100a,code=sm_100a (NOT -arch=sm_100a, which also
emits compute_100 PTX and rejects tcgen05; SURVEY.md §7 toolchain note).
Each .cu compiles to its own object (in parallel, rebuilt when it or any
header is newer), then one nvcc link produces the shared library.

MOE_EXPERIMENTS=1 in the environment compiles the timing-experiment modes
(-DMOE_EXPERIMENTS: stale-smem / loads-only GEMM modes, the two-launch decode
chain selector, ...) into the library; the default build has none of them.
"""
import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libmoe_b200.so")
OBJ = os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_dir():
    """NCCL 2.28 headers + libnccl.so.2 (the torch-bundled nvidia-nccl wheel)."""
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations if spec else []):
        d = os.path.join(base, "nccl")
        if os.path.exists(os.path.join(d, "include", "nccl.h")):
            return d
    raise RuntimeError("NCCL headers not found (nvidia.nccl)")


FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]


def experiments() -> bool:
    return os.environ.get("MOE_EXPERIMENTS", "0") == "1"


def sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".cu"))


def headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".cuh", ".h"))]
    hs.append(os.path.join(HERE, "..", "include", "moe.h"))
    return hs


def _flags():
    f = list(FLAGS)
    if experiments():
        f.append("-DMOE_EXPERIMENTS=1")
    return f


def _stamp():
    return os.path.join(OBJ, "flags.txt")


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    if not os.path.exists(_stamp()) or open(_stamp()).read() != " ".join(_flags()):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in sources() + headers())


def _compile(src, obj, inc, verbose):
    cmd = [NVCC, *_flags(), *inc, "-c", src, "-o", obj + ".tmp"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed on {os.path.basename(src)} ({r.returncode}):\n{r.stderr[-8000:]}")
    if verbose and r.stderr.strip():
        print(r.stderr[-4000:], file=sys.stderr)
    os.replace(obj + ".tmp", obj)
    return obj


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    nccl = _nccl_dir()
    inc = ["-I", os.path.join(HERE, "..", "include"), "-I", os.path.join(nccl, "include")]
    flags_changed = not os.path.exists(_stamp()) or open(_stamp()).read() != " ".join(_flags())
    hmax = max(os.path.getmtime(h) for h in headers())
    jobs = []
    for src in sources():
        obj = os.path.join(OBJ, os.path.basename(src)[:-3] + ".o")
        if force or flags_changed or not os.path.exists(obj) or \
                os.path.getmtime(obj) < max(os.path.getmtime(src), hmax):
            jobs.append((src, obj))
    with cf.ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 4))) as ex:
        for f in [ex.submit(_compile, s, o, inc, verbose) for s, o in jobs]:
            f.result()
    objs = [os.path.join(OBJ, os.path.basename(s)[:-3] + ".o") for s in sources()]
    tmp = LIB + ".tmp"
    cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", *objs, "-o", tmp, "-lcuda",
           "-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2", "-Xlinker", "-rpath=" + os.path.join(nccl, "lib")]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc link failed ({r.returncode}):\n{r.stderr[-8000:]}")
    os.replace(tmp, LIB)
    with open(_stamp(), "w") as f:
        f.write(" ".join(_flags()))
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
    print(LIB)
