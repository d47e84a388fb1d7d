"""Build libhydro_b200.so in-tree: nvcc for sm_100a (cross-compiles without a GPU).

Every kernel is compiled with ``-gencode arch=compute_100a,code=sm_100a -lineinfo``; the NCCL
headers and library are the pip copy torch loads (one libnccl.so.2 per process).
"""
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libhydro_b200.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_dir():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations or []) if spec else []:
        d = os.path.join(base, "nccl")
        if os.path.exists(os.path.join(d, "include", "nccl.h")):
            return d
    raise RuntimeError("pip NCCL (nvidia/nccl) not found")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def strict_sources():
    """STRICT path (HYDRO_FLAG_STRICT): compiled on its own without FMA contraction (reading
    R12), so its operation order is exactly the written one."""
    return sorted(glob.glob(os.path.join(CSRC, "strict", "*.cu")))


def _stale():
    if not os.path.exists(LIB):
        return True
    deps = (sources() + strict_sources() + glob.glob(os.path.join(CSRC, "*.h")) +
            glob.glob(os.path.join(CSRC, "*.cuh")))
    deps.append(os.path.join(ROOT, "include", "hydro.h"))
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    nccl = _nccl_dir()
    nvcc = os.environ.get("NVCC", "nvcc")
    extra = os.environ.get("HYDRO_NVCC_FLAGS", "").split()
    objs = []
    for src in strict_sources():
        obj = os.path.join(CSRC, "strict", os.path.basename(src)[:-3] + ".o")
        c = [nvcc, "-c", *extra, "-Xcompiler", "-fPIC", "-O3", "-std=c++17", "-lineinfo", *ARCH,
             "-fmad=false", "-prec-div=true", "-prec-sqrt=true",
             "-I", os.path.join(ROOT, "include"), "-o", obj, src]
        r = subprocess.run(c, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed (strict)")
        objs.append(obj)
    cmd = [nvcc, "-shared", *extra, "-Xcompiler", "-fPIC", "-O3", "-std=c++17", "-lineinfo", *ARCH,
           "-Xptxas", "-v" if verbose else "-O3",
           "-I", os.path.join(ROOT, "include"), "-I", os.path.join(nccl, "include"),
           "-o", LIB + ".tmp", *sources(), *objs,
           "-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2",
           "-Xlinker", "-rpath=" + os.path.join(nccl, "lib")]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed")
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(LIB + ".tmp", LIB)
    return LIB


def build_c_example() -> str:
    """examples/sedov.c against include/hydro.h only (plain C99, no Python): build/sedov_c."""
    out_dir = os.path.join(ROOT, "build")
    os.makedirs(out_dir, exist_ok=True)
    exe = os.path.join(out_dir, "sedov_c")
    cmd = ["gcc", "-O2", "-std=c99", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
           os.path.join(ROOT, "examples", "sedov.c"), "-L", HERE, "-l:libhydro_b200.so",
           "-Wl,-rpath," + HERE, "-lm", "-o", exe]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("C example build failed")
    return exe


if __name__ == "__main__":
    print(build(force=True, verbose="-v" in sys.argv))
