"""Build libavgpipe_ea.so in-tree for sm_100a (nvcc cross-compiles; no GPU needed).

    python -m paper_conf_ppopp_chen0qz23_b200.build [--force]

The library links NCCL from the torch-bundled ``nvidia.nccl`` wheel (the one
torch itself loads, so only one libnccl.so.2 is ever mapped) and the CUDA
runtime statically.
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
LIB_NAME = "libavgpipe_ea.so"
LIB_PATH = os.path.join(PKG, LIB_NAME)

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
              "--expt-relaxed-constexpr", "-Xptxas", "-v"]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia.nccl")
    if spec is not None and spec.submodule_search_locations:
        base = list(spec.submodule_search_locations)[0]
        inc, lib = os.path.join(base, "include"), os.path.join(base, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")) and glob.glob(os.path.join(lib, "libnccl.so*")):
            return inc, lib
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def _stale() -> bool:
    if not os.path.exists(LIB_PATH):
        return True
    t = os.path.getmtime(LIB_PATH)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(INCLUDE, "*.h")) + [__file__]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB_PATH
    nccl_inc, nccl_lib = nccl_dirs()
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    for src in sources():
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        cmd = [nvcc(), *ARCH, *NVCC_FLAGS, "-I", INCLUDE, "-I", CSRC, "-I", nccl_inc, "-c", src, "-o", obj]
        if src.endswith(".cpp"):
            cmd[1:1] = ["-x", "cu"]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            raise RuntimeError(f"nvcc failed on {src}:\n{res.stdout}\n{res.stderr}")
        if verbose:
            print(res.stderr, file=sys.stderr)
        with open(obj + ".ptxas.txt", "w") as f:
            f.write(res.stderr)
        objs.append(obj)
    tmp = LIB_PATH + ".tmp"
    link = [nvcc(), *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-L", nccl_lib, "-l:libnccl.so.2",
            "-Xlinker", "-rpath", "-Xlinker", nccl_lib]
    res = subprocess.run(link, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError(f"link failed:\n{res.stdout}\n{res.stderr}")
    os.replace(tmp, LIB_PATH)
    return LIB_PATH


NCCL_EMU_SRC = os.path.join(ROOT, "tests", "nccl_emu", "nccl_emu.cu")
NCCL_EMU_LIB = os.path.join(ROOT, "tests", "nccl_emu", "libnccl_emu.so")


def build_nccl_emu(force: bool = False) -> str:
    """Test infrastructure: the in-process NCCL emulation (tests/nccl_emu, LD_PRELOAD) that runs the
    library's NCCL spread path with N > 1 ranks on one GPU.  Not linked into the product library."""
    if not force and os.path.exists(NCCL_EMU_LIB) and os.path.getmtime(NCCL_EMU_LIB) >= os.path.getmtime(NCCL_EMU_SRC):
        return NCCL_EMU_LIB
    nccl_inc, _ = nccl_dirs()
    tmp = NCCL_EMU_LIB + ".tmp"
    cmd = [nvcc(), *ARCH, "-O2", "-std=c++17", "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", "-I", nccl_inc,
           NCCL_EMU_SRC, "-o", tmp]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError(f"nvcc failed on {NCCL_EMU_SRC}:\n{res.stdout}\n{res.stderr}")
    os.replace(tmp, NCCL_EMU_LIB)
    return NCCL_EMU_LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
