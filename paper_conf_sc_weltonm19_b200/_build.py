"""Build libffm.so in-tree for sm_100a (nvcc; cross-compiles without a GPU)."""
import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libffm.so")
SOURCES = [os.path.join(HERE, "csrc", f) for f in ("kernels.cu", "shard.cu", "online.cu", "comm.cu", "ffm_api.cu", "shard_plan.cpp")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-shared", "-Xcompiler", "-fPIC,-fopenmp", "-O3", "-lineinfo", "-std=c++17",
         "-gencode", "arch=compute_100a,code=sm_100a", "-ldl", "-lgomp"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = SOURCES + glob.glob(os.path.join(HERE, "csrc", "*.h")) + glob.glob(os.path.join(HERE, "csrc", "*.cuh")) + \
        glob.glob(os.path.join(HERE, "..", "include", "*.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if force or _stale():
        cmd = [NVCC] + FLAGS + SOURCES + ["-o", LIB]
        if verbose:
            print(" ".join(cmd))
        subprocess.run(cmd, check=True)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
