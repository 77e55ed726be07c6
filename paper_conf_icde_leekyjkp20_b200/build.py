"""Build libspgemm.so in-tree with nvcc for sm_100a (B200).  No JIT cache, no torch extension:
the shared library travels with the repository snapshot to the GPU box."""
import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SO = os.path.join(HERE, "libspgemm.so")
MAIN = os.path.join(HERE, "csrc", "spgemm.cu")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared"] + os.environ.get("SPGEMM_NVCC_EXTRA", "").split()


def sources():
    return glob.glob(os.path.join(HERE, "csrc", "*.cu*")) + [os.path.join(ROOT, "include", "spgemm.h")]


def build_library(force: bool = False, verbose: bool = False) -> str:
    newest = max(os.path.getmtime(s) for s in sources())
    if force or not os.path.exists(SO) or os.path.getmtime(SO) < newest:
        cmd = [NVCC, *FLAGS, "-o", SO, MAIN]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
        subprocess.check_call(cmd)
    return SO


if __name__ == "__main__":
    print(build_library(force=True, verbose=True))
